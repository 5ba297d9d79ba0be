mkdir -p gpurun_out
timeout 1500 python -m pytest tests -x -q -m gpu > gpurun_out/q26_tests.log 2>&1; echo "tests rc=$?" >> gpurun_out/q26_tests.log
PARITY_ARGS="--ref-budget 4 --parity-min-ends 30000" CFG=C4 REPS=1 STEPS=3 RUN_TIMEOUT=400 BENCH_ARGS="--no-replay --no-select --coexec-share 0" timeout 900 bash tools/ab.sh base lds2 > gpurun_out/ab17_c4.txt 2>&1
PARITY_ARGS="--ref-budget 4 --parity-min-ends 30000" CFG=C3 REPS=1 STEPS=5 RUN_TIMEOUT=400 BENCH_ARGS="--no-replay --no-select --coexec-share 0" timeout 900 bash tools/ab.sh base lds2 > gpurun_out/ab17_c3.txt 2>&1
