mkdir -p gpurun_out
timeout 1500 python -m pytest tests -x -q -m gpu > gpurun_out/q20_tests.log 2>&1; echo "tests rc=$?" >> gpurun_out/q20_tests.log
CFG=C4 REPS=1 STEPS=3 RUN_TIMEOUT=300 BENCH_ARGS="--no-replay --no-select --coexec-share 0" timeout 900 bash tools/ab.sh hyb m23 > gpurun_out/ab13_c4.txt 2>&1
CFG=C4F REPS=1 STEPS=5 RUN_TIMEOUT=300 BENCH_ARGS="--no-replay --no-select --coexec-share 0" timeout 900 bash tools/ab.sh hyb m23 > gpurun_out/ab13_c4f.txt 2>&1
timeout 600 python bench.py --steps 3 --warmup 2 --no-e2e --no-replay --no-select --coexec-share 0 --parity-min-ends 200000 --ref-budget 8 > gpurun_out/q20_parity_c4.json 2> gpurun_out/q20_parity_c4.err; echo "parity rc=$?" >> gpurun_out/q20_tests.log
