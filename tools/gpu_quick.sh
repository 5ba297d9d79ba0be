#!/bin/bash
# Quick GPU iteration: build, GPU parity tests, a short bench line (no CPU baseline / e2e), phase profile.
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || { cat gpurun_out/build.log; exit 1; }
timeout 900 python -m pytest tests -m gpu -x -q > gpurun_out/pytest_gpu.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_gpu.log
tail -3 gpurun_out/pytest_gpu.log
timeout 600 python bench.py --steps 3 --warmup 3 --no-cpu-baseline --no-e2e > gpurun_out/bench_quick.json 2> gpurun_out/bench_quick.err
python -c "
import json; d=json.load(open('gpurun_out/bench_quick.json'))
print('ms/step', d['ms_per_step'], 'value', d['value'], 'frac', d['roofline']['frac'])
for k,v in d['work']['classes'].items(): print(k, v)
"
if [ -n "$PHASE" ]; then LA_SERIAL_CLASSES=1 timeout 600 python tools/phase_profile.py > gpurun_out/phase.json 2> gpurun_out/phase.err; fi
