mkdir -p gpurun_out
CFG=C4 REPS=1 STEPS=3 RUN_TIMEOUT=300 BENCH_ARGS="--no-replay --no-select --coexec-share 0" timeout 1200 bash tools/ab.sh m23 m4 m23u1 m23w0 > gpurun_out/ab11_c4.txt 2>&1
CFG=C4F REPS=1 STEPS=5 RUN_TIMEOUT=300 BENCH_ARGS="--no-replay --no-select --coexec-share 0" timeout 900 bash tools/ab.sh m23 m4 m23u1 > gpurun_out/ab11_c4f.txt 2>&1
