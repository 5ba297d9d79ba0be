mkdir -p gpurun_out
PARITY_ARGS="--ref-budget 4 --parity-min-ends 30000" CFG=C4 REPS=1 STEPS=3 RUN_TIMEOUT=400 BENCH_ARGS="--no-replay --no-select --coexec-share 0" timeout 900 bash tools/ab.sh l80 l75 l85 > gpurun_out/ab20_c4.txt 2>&1
PARITY_ARGS="--ref-budget 4 --parity-min-ends 30000" CFG=C4S REPS=1 STEPS=3 RUN_TIMEOUT=400 BENCH_ARGS="--no-replay --no-select --coexec-share 0" timeout 900 bash tools/ab.sh l80 l75 l85 > gpurun_out/ab20_c4s.txt 2>&1
