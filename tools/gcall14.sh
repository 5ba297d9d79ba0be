mkdir -p gpurun_out
timeout 400 python -m pytest tests/test_gpu_parity.py -x -q -m gpu -k "c_abi_client or c1_single" > gpurun_out/q14_tests.log 2>&1; echo "tests rc=$?" >> gpurun_out/q14_tests.log
CFG=C4 REPS=1 STEPS=3 RUN_TIMEOUT=300 BENCH_ARGS="--no-replay --no-select --coexec-share 0" timeout 1500 bash tools/ab.sh base u4 u1 l75 l80 > gpurun_out/ab8_c4.txt 2>&1
