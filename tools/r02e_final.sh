#!/bin/bash
# Final r02b state: full GPU suite, smoke, the default C4 bench line and C4S / C3 / C4F lines, the ncu
# launch list of one C4 step.  Outputs under gpurun_out/r02e_*.
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/r02e_build.log 2>&1
timeout 1500 python -m pytest tests -m gpu -x -q > gpurun_out/r02e_pytest_gpu.log 2>&1; echo "pytest rc=$?" >> gpurun_out/r02e_pytest_gpu.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/r02e_smoke.log 2>&1; echo "smoke rc=$?" >> gpurun_out/r02e_smoke.log
timeout 1500 python bench.py --steps 10 --warmup 3 > gpurun_out/r02e_bench_c4.json 2> gpurun_out/r02e_bench_c4.err; echo "c4 rc=$?"
timeout 900 python bench.py --config C4S --steps 10 --warmup 3 --no-select > gpurun_out/r02e_bench_c4s.json 2> gpurun_out/r02e_bench_c4s.err; echo "c4s rc=$?"
timeout 900 python bench.py --config C3 --steps 10 --warmup 3 --no-select > gpurun_out/r02e_bench_c3.json 2> gpurun_out/r02e_bench_c3.err; echo "c3 rc=$?"
timeout 900 python bench.py --config C4F --steps 10 --warmup 3 --no-select > gpurun_out/r02e_bench_c4f.json 2> gpurun_out/r02e_bench_c4f.err; echo "c4f rc=$?"
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv --log-file gpurun_out/r02e_launches_c4.csv \
  python bench.py --steps 2 --warmup 1 --no-e2e --no-cpu-baseline --no-replay --no-select --coexec-share 0 > /dev/null 2>&1; echo "launches rc=$?"
echo done
