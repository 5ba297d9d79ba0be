#!/bin/bash
# Compare build / runtime variants on the C4 bench: each argument is "NAME|ENV ASSIGNMENTS".
# A variant whose env sets LA_NVCC_EXTRA forces a rebuild of liblocassm.so.
mkdir -p gpurun_out
: > gpurun_out/variants.txt
for spec in "$@"; do
  name="${spec%%|*}"; envs="${spec#*|}"
  env $envs python -c "from paper_conf_sc_awanhedbdoy21_b200.build import build; build(force=True)" > gpurun_out/build_$name.log 2>&1 || { echo "$name build failed" >> gpurun_out/variants.txt; continue; }
  if [ -n "$TESTS" ]; then env $envs timeout 900 python -m pytest tests -m gpu -x -q > gpurun_out/pytest_$name.log 2>&1; echo "$name pytest rc=$? $(tail -1 gpurun_out/pytest_$name.log)" >> gpurun_out/variants.txt; fi
  env $envs timeout 600 python bench.py --steps 3 --warmup 2 --no-cpu-baseline --no-e2e > gpurun_out/bench_$name.json 2> gpurun_out/bench_$name.err
  python - "$name" >> gpurun_out/variants.txt <<'PY'
import json, sys
n = sys.argv[1]
try:
    d = json.load(open(f"gpurun_out/bench_{n}.json"))
    cl = " ".join(f"{k}:{v['ms']}" for k, v in d["work"]["classes"].items())
    print(f"{n}: ms/step {d['ms_per_step']:.2f} value {d['value']:.4g} | {cl} | global {d['phase_ms']['global_rounds']:.2f}")
except Exception as e:
    print(n, "failed", e, open(f"gpurun_out/bench_{n}.err").read()[-400:])
PY
done
cat gpurun_out/variants.txt
