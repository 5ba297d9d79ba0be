mkdir -p gpurun_out
timeout 600 python -m pytest tests/test_gpu_parity.py -x -q -m gpu -k "c1_single or c2_small or class_by_key or xl_wide or c3_sampled or assembler_k_rounds or pins_on_gpu or coexec" > gpurun_out/q9_tests.log 2>&1; echo "tests rc=$?" >> gpurun_out/q9_tests.log
if grep -q "tests rc=0" gpurun_out/q9_tests.log; then
CFG=C4 REPS=1 STEPS=3 RUN_TIMEOUT=300 BENCH_ARGS="--no-replay --no-select --coexec-share 0" timeout 900 bash tools/ab.sh wpf str > gpurun_out/ab5_c4.txt 2>&1
timeout 600 python bench.py --steps 3 --warmup 2 --no-e2e --no-replay --no-select --coexec-share 0 --parity-min-ends 100000 --ref-budget 5 > gpurun_out/q9_parity_c4.json 2> gpurun_out/q9_parity_c4.err; echo "parity rc=$?" >> gpurun_out/q9_tests.log
fi
