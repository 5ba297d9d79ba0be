mkdir -p gpurun_out
timeout 600 python -m pytest tests/test_gpu_parity.py tests/test_select.py -x -q -m gpu -k "c1_single or c2_small or class_by_key or xl_wide or c3_sampled or assembler_k_rounds or pins_on_gpu or streamed_matches or empty or select_then" > gpurun_out/q11_tests.log 2>&1; echo "tests rc=$?" >> gpurun_out/q11_tests.log
if grep -q "tests rc=0" gpurun_out/q11_tests.log; then
CFG=C4S REPS=2 STEPS=3 RUN_TIMEOUT=200 BENCH_ARGS="--no-replay --no-select --coexec-share 0" timeout 900 bash tools/ab.sh nouni uni > gpurun_out/ab6.txt 2>&1
CFG=C4 REPS=1 STEPS=3 RUN_TIMEOUT=300 BENCH_ARGS="--no-replay --no-select --coexec-share 0" timeout 900 bash tools/ab.sh nouni uni > gpurun_out/ab6_c4.txt 2>&1
fi
