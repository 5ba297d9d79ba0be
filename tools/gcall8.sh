mkdir -p gpurun_out
timeout 500 python -m pytest tests/test_gpu_parity.py -x -q -m gpu -k "c1_single or c2_small or class_by_key or xl_wide or c3_sampled or assembler_k_rounds or pins_on_gpu" > gpurun_out/q8_tests.log 2>&1; echo "tests rc=$?" >> gpurun_out/q8_tests.log
CFG=C4S REPS=2 STEPS=3 RUN_TIMEOUT=200 BENCH_ARGS="--no-replay --no-select --coexec-share 0" timeout 1000 bash tools/ab.sh base wp wpf wpfs f > gpurun_out/ab4.txt 2>&1
for v in base wpf wpfs; do for t in _1 _2; do cp gpurun_out/ab_${v}${t}.json gpurun_out/ab4s_${v}${t}.json 2>/dev/null; done; done
CFG=C4 REPS=1 STEPS=3 RUN_TIMEOUT=300 BENCH_ARGS="--no-replay --no-select --coexec-share 0" timeout 900 bash tools/ab.sh base wpf wpfs > gpurun_out/ab4_c4.txt 2>&1
