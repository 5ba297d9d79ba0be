#!/bin/bash
# Evidence run: compute-sanitizer (memcheck / synccheck / racecheck) over every table class, a C3
# bench line, the default C4 bench line, and the ncu launch list of one C4 step.
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
timeout 900 compute-sanitizer --tool memcheck --print-limit 20 python tools/sanitize_run.py --ends 2000 > gpurun_out/r02_sanitize_memcheck.log 2>&1; echo "memcheck rc=$?"; tail -3 gpurun_out/r02_sanitize_memcheck.log
timeout 900 compute-sanitizer --tool synccheck --print-limit 20 python tools/sanitize_run.py --ends 1000 > gpurun_out/r02_sanitize_synccheck.log 2>&1; echo "synccheck rc=$?"; tail -3 gpurun_out/r02_sanitize_synccheck.log
timeout 1500 compute-sanitizer --tool racecheck --racecheck-report hazard --print-limit 20 python tools/sanitize_run.py --ends 300 > gpurun_out/r02_sanitize_racecheck.log 2>&1; echo "racecheck rc=$?"; tail -3 gpurun_out/r02_sanitize_racecheck.log
timeout 900 python bench.py --config C3 --steps 5 --warmup 3 > gpurun_out/r02_bench_c3.json 2> gpurun_out/r02_bench_c3.err; echo "c3 rc=$?"
