mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_parity.py -x -q -m gpu > gpurun_out/q17_tests.log 2>&1; echo "tests rc=$?" >> gpurun_out/q17_tests.log
if grep -q "tests rc=0" gpurun_out/q17_tests.log; then
CFG=C4 REPS=1 STEPS=3 RUN_TIMEOUT=300 BENCH_ARGS="--no-replay --no-select --coexec-share 0" timeout 900 bash tools/ab.sh base e32 m23 > gpurun_out/ab10_c4.txt 2>&1
CFG=C4F REPS=2 STEPS=5 RUN_TIMEOUT=300 BENCH_ARGS="--no-replay --no-select --coexec-share 0" timeout 900 bash tools/ab.sh base e32 m23 > gpurun_out/ab10_c4f.txt 2>&1
fi
