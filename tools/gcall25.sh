mkdir -p gpurun_out
timeout 1500 python -m pytest tests -x -q -m gpu > gpurun_out/q25_tests.log 2>&1; echo "tests rc=$?" >> gpurun_out/q25_tests.log
PARITY_ARGS="--ref-budget 4 --parity-min-ends 30000" CFG=C4 REPS=1 STEPS=3 RUN_TIMEOUT=400 BENCH_ARGS="--no-replay --no-select --coexec-share 0" timeout 900 bash tools/ab.sh base lds > gpurun_out/ab16_c4.txt 2>&1
PARITY_ARGS="--ref-budget 4 --parity-min-ends 30000" CFG=C4F REPS=1 STEPS=5 RUN_TIMEOUT=400 BENCH_ARGS="--no-replay --no-select --coexec-share 0" timeout 900 bash tools/ab.sh base lds > gpurun_out/ab16_c4f.txt 2>&1
PARITY_ARGS="--ref-budget 4 --parity-min-ends 30000" CFG=C4S REPS=1 STEPS=3 RUN_TIMEOUT=400 BENCH_ARGS="--no-replay --no-select --coexec-share 0" timeout 900 bash tools/ab.sh base lds > gpurun_out/ab16_c4s.txt 2>&1
