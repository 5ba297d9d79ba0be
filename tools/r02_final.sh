#!/bin/bash
# Round-2 evidence run: default C4 bench (the driver's command), C4S and C3 lines, the serial-class
# ncu traffic / instruction summary of a C4S step.  Outputs under gpurun_out/r02final_*.
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
timeout 1500 python bench.py --steps 10 --warmup 3 > gpurun_out/r02final_c4.json 2> gpurun_out/r02final_c4.err; echo "c4 rc=$?"
timeout 900 python bench.py --config C4S --steps 10 --warmup 3 > gpurun_out/r02final_c4s.json 2> gpurun_out/r02final_c4s.err; echo "c4s rc=$?"
timeout 900 python bench.py --config C3 --steps 10 --warmup 3 > gpurun_out/r02final_c3.json 2> gpurun_out/r02final_c3.err; echo "c3 rc=$?"
bash tools/ncu_traffic.sh r02final_c4s > gpurun_out/r02final_c4s_traffic.txt 2>&1
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv --log-file gpurun_out/r02final_launches_c4.csv \
  python bench.py --steps 2 --warmup 1 --no-e2e --no-cpu-baseline --no-replay --coexec-share 0 > /dev/null 2>&1; echo "launches rc=$?"
