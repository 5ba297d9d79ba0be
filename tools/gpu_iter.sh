#!/bin/bash
# One GPU iteration: build, GPU parity tests, a short C4S bench (kernel path only).
#   gpurun -- bash tools/gpu_iter.sh [tag] [pytest-args]
tag=${1:-iter}
shift
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/${tag}_build.log 2>&1 || { tail -20 gpurun_out/${tag}_build.log; exit 1; }
if [ "${SKIP_TESTS:-0}" != "1" ]; then
  timeout 1200 python -m pytest tests -x -q -m gpu "$@" > gpurun_out/${tag}_pytest.log 2>&1
  tail -5 gpurun_out/${tag}_pytest.log
fi
timeout 900 python bench.py --config ${CFG:-C4S} --steps ${STEPS:-10} --warmup 3 --no-e2e ${BENCH_ARGS:-} > gpurun_out/${tag}_bench.json 2> gpurun_out/${tag}_bench.err
echo "bench rc=$?"
python - <<PY
import json
d=json.loads(open("gpurun_out/${tag}_bench.json").read().strip().splitlines()[-1])
print("ms/step", round(d["ms_per_step"],2), "value %.3e"%d["value"], "parity", d.get("parity"))
rb=d.get("roofline_build") or {}
print("build ms", rb.get("ms"), "frac", rb.get("frac"), {k:(v["ms"],round(v["frac"] or 0,4)) for k,v in (rb.get("classes") or {}).items()})
print({k:v["ms"] for k,v in d["work"]["classes"].items()}, d["phase_ms"])
PY
