mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_select.py -x -q -m gpu > gpurun_out/q15_tests.log 2>&1; echo "tests rc=$?" >> gpurun_out/q15_tests.log
CFG=C4S REPS=2 STEPS=3 RUN_TIMEOUT=200 BENCH_ARGS="--no-replay --no-select --coexec-share 0" timeout 900 bash tools/ab.sh l70 l80 l85 > gpurun_out/ab9.txt 2>&1
CFG=C4 REPS=1 STEPS=3 RUN_TIMEOUT=300 BENCH_ARGS="--no-replay --no-select --coexec-share 0" timeout 900 bash tools/ab.sh l70 l80 l85 > gpurun_out/ab9_c4.txt 2>&1
