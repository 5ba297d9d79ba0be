mkdir -p gpurun_out
CFG=C4S REPS=2 STEPS=3 RUN_TIMEOUT=200 BENCH_ARGS="--no-replay --no-select --coexec-share 0" timeout 1300 bash tools/ab.sh base seg nl wp all allx0 allf > gpurun_out/ab3.txt 2>&1
CFG=C4 REPS=1 STEPS=3 RUN_TIMEOUT=300 BENCH_ARGS="--no-replay --no-select --coexec-share 0" timeout 900 bash tools/ab.sh base all allf > gpurun_out/ab3_c4.txt 2>&1
