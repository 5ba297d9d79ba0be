#!/bin/bash
# A/B of library variants (built HERE by tools/ab_build.sh into build_ab/<name>.so): serial-class C4S
# bench per variant on the same GPU box, kernel path only.
#   gpurun -- bash tools/ab.sh name1 name2 ...
mkdir -p gpurun_out
python bench.py --config ${CFG:-C4S} --steps 1 --warmup 0 --no-e2e --no-cpu-baseline --no-replay > /dev/null 2>&1
for rep in $(seq 1 ${REPS:-2}); do
for v in "$@"; do
  LA_SO=$PWD/build_ab/$v.so LA_SERIAL_CLASSES=${SERIAL:-1} timeout 600 python bench.py --config ${CFG:-C4S} --steps ${STEPS:-5} --warmup 2 \
      --no-e2e --no-cpu-baseline ${BENCH_ARGS:-} > gpurun_out/ab_${v}_${rep}.json 2> gpurun_out/ab_${v}_${rep}.err
  python - "$v" "$rep" <<'PY'
import json, sys
v, rep = sys.argv[1], sys.argv[2]
try:
    d = json.loads(open(f"gpurun_out/ab_{v}_{rep}.json").read().strip().splitlines()[-1])
except Exception as e:
    print(v, rep, "FAILED", e); sys.exit(0)
w = d["work"]["classes"]
rb = d.get("roofline_build") or {}
print(f"{v:14s} rep{rep} ms/step {d['ms_per_step']:7.2f} build {rb.get('ms') or 0:7.2f} parity {d['parity']['mismatches'] if d.get('parity') else None} xl_ends {d['work']['ends_xl']} "
      + " ".join(f"{k}:{c['ms']:.1f}/{c['inserts']/max(c['ms'],1e-9)/1e6:.0f}G" for k, c in w.items()))
PY
done; done
