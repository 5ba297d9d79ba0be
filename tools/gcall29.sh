mkdir -p gpurun_out
timeout 1500 python -m pytest tests -x -q -m gpu > gpurun_out/q29_tests.log 2>&1; echo "tests rc=$?" >> gpurun_out/q29_tests.log
PARITY_ARGS="--ref-budget 4 --parity-min-ends 30000" CFG=C4 REPS=1 STEPS=3 RUN_TIMEOUT=400 BENCH_ARGS="--no-replay --no-select --coexec-share 0" timeout 900 bash tools/ab.sh base c2 > gpurun_out/ab19_c4.txt 2>&1
PARITY_ARGS="--ref-budget 4 --parity-min-ends 30000" CFG=C4F REPS=1 STEPS=5 RUN_TIMEOUT=400 BENCH_ARGS="--no-replay --no-select --coexec-share 0" timeout 600 bash tools/ab.sh base c2 > gpurun_out/ab19_c4f.txt 2>&1
