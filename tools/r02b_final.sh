#!/bin/bash
# Round-2 (second session) evidence run on one box: GPU parity suite, smoke, the default C4 bench line
# (the driver's command), C4S / C3 lines, the ncu launch list of one C4 step, the serial-class traffic
# + instruction summary of a C4S step, one ncu --set full capture of the top class kernel, and the
# sanitizers over every table class.  Outputs under gpurun_out/r02b_*.
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/r02b_build.log 2>&1
timeout 1500 python -m pytest tests -m gpu -x -q > gpurun_out/r02b_pytest_gpu.log 2>&1; echo "pytest rc=$?" >> gpurun_out/r02b_pytest_gpu.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/r02b_smoke.log 2>&1; echo "smoke rc=$?" >> gpurun_out/r02b_smoke.log
timeout 1500 python bench.py --steps 10 --warmup 3 > gpurun_out/r02b_bench_c4.json 2> gpurun_out/r02b_bench_c4.err; echo "c4 rc=$?"
timeout 900 python bench.py --config C4S --steps 10 --warmup 3 --no-select > gpurun_out/r02b_bench_c4s.json 2> gpurun_out/r02b_bench_c4s.err; echo "c4s rc=$?"
timeout 900 python bench.py --config C3 --steps 10 --warmup 3 --no-select > gpurun_out/r02b_bench_c3.json 2> gpurun_out/r02b_bench_c3.err; echo "c3 rc=$?"
timeout 900 python bench.py --config C4F --steps 10 --warmup 3 --no-select > gpurun_out/r02b_bench_c4f.json 2> gpurun_out/r02b_bench_c4f.err; echo "c4f rc=$?"
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv --log-file gpurun_out/r02b_launches_c4.csv \
  python bench.py --steps 2 --warmup 1 --no-e2e --no-cpu-baseline --no-replay --no-select --coexec-share 0 > /dev/null 2>&1; echo "launches rc=$?"
timeout 900 bash tools/ncu_traffic.sh r02b_c4s > gpurun_out/r02b_c4s_traffic.txt 2>&1; echo "traffic rc=$?"
timeout 1200 bash tools/diag.sh r02b_k512 'k_smem<\(int\)512' C4 > gpurun_out/r02b_diag.log 2>&1; echo "diag rc=$?"
timeout 900 compute-sanitizer --tool memcheck --print-limit 20 python tools/sanitize_run.py --ends 2000 > gpurun_out/r02b_sanitize_memcheck.log 2>&1; echo "memcheck rc=$?"
timeout 900 compute-sanitizer --tool synccheck --print-limit 20 python tools/sanitize_run.py --ends 1000 > gpurun_out/r02b_sanitize_synccheck.log 2>&1; echo "synccheck rc=$?"
timeout 1500 compute-sanitizer --tool racecheck --racecheck-report hazard --print-limit 20 python tools/sanitize_run.py --ends 300 > gpurun_out/r02b_sanitize_racecheck.log 2>&1; echo "racecheck rc=$?"
echo done
