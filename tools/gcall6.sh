mkdir -p gpurun_out
timeout 400 python -m pytest tests/test_gpu_parity.py -x -q -m gpu -k "c1_single or c2_small_full or class_by_key or xl_wide or c3_sampled or assembler_k_rounds" > gpurun_out/q6_tests.log 2>&1; echo "tests rc=$?" >> gpurun_out/q6_tests.log
if grep -q "tests rc=0" gpurun_out/q6_tests.log; then
  CFG=C4S REPS=1 STEPS=3 RUN_TIMEOUT=200 BENCH_ARGS="--no-replay --no-select --coexec-share 0" timeout 1500 bash tools/ab.sh base seg nl wp all allx0 > gpurun_out/ab2.txt 2>&1
fi
