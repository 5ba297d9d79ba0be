mkdir -p gpurun_out
timeout 1200 python -m pytest tests -x -q -m gpu > gpurun_out/q19_tests.log 2>&1; echo "tests rc=$?" >> gpurun_out/q19_tests.log
CFG=C4 REPS=1 STEPS=3 RUN_TIMEOUT=300 BENCH_ARGS="--no-replay --no-select --coexec-share 0" timeout 900 bash tools/ab.sh hyb m23 m4 > gpurun_out/ab12_c4.txt 2>&1
CFG=C4F REPS=1 STEPS=5 RUN_TIMEOUT=300 BENCH_ARGS="--no-replay --no-select --coexec-share 0" timeout 900 bash tools/ab.sh hyb m23 m4 > gpurun_out/ab12_c4f.txt 2>&1
CFG=C4S REPS=1 STEPS=3 RUN_TIMEOUT=300 BENCH_ARGS="--no-replay --no-select --coexec-share 0" timeout 900 bash tools/ab.sh hyb m23 > gpurun_out/ab12_c4s.txt 2>&1
