#!/bin/bash
# A/B of library variants (built HERE by tools/ab_build.sh into build_ab/<name>.so): serial-class C4S
# bench per variant on the same GPU box, kernel path only.
#   gpurun -- bash tools/ab.sh name1 "name2:ENV=1;ENV2=x" ...   (env assignments separated by ';')
mkdir -p gpurun_out
timeout 400 python bench.py --config ${CFG:-C4S} --steps 1 --warmup 0 --no-e2e --no-cpu-baseline --no-replay --no-select --coexec-share 0 > /dev/null 2>&1
i=0
for rep in $(seq 1 ${REPS:-2}); do
for spec in "$@"; do
  i=$((i+1))
  v=${spec%%:*}; envs=""; [[ "$spec" == *:* ]] && envs=${spec#*:}
  tag=$(echo "$spec" | tr -c 'A-Za-z0-9_\n' '_')
  ( IFS=';'; for kv in $envs; do export "$kv"; done; unset IFS
    LA_SO=$PWD/build_ab/$v.so LA_SERIAL_CLASSES=${SERIAL:-1} timeout ${RUN_TIMEOUT:-300} python bench.py --config ${CFG:-C4S} --steps ${STEPS:-5} --warmup 2 \
      --no-e2e ${PARITY_ARGS:---no-cpu-baseline} ${BENCH_ARGS:-} > gpurun_out/ab_${tag}_${rep}.json 2> gpurun_out/ab_${tag}_${rep}.err )
  python - "$tag" "$rep" <<'PY'
import json, sys
v, rep = sys.argv[1], sys.argv[2]
try:
    d = json.loads(open(f"gpurun_out/ab_{v}_{rep}.json").read().strip().splitlines()[-1])
except Exception as e:
    print(v, rep, "FAILED", e); sys.exit(0)
w = d["work"]["classes"]
rb = d.get("roofline_build") or {}
par = d.get("parity") or {}
print(f"{v:28s} r{rep} parity {par.get('mismatches', '-')}/{par.get('ends_checked', '-')} ms/step {d['ms_per_step']:7.2f} build {rb.get('ms') or 0:7.2f} xl {d['work']['ends_xl']} ovf {d['work']['ends_by_class'][4]} "
      + " ".join(f"{c['ends']//1000}k:{c['ms']:.1f}/{c['inserts']/max(c['ms'],1e-9)/1e6:.0f}G" for k, c in w.items()))
PY
done; done
