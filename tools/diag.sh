#!/bin/bash
# Diagnostics of the table kernels on one box: per-class phase split (clock64), probe-round statistics,
# and one ncu --set full capture of a class kernel (source level).
#   gpurun -- bash tools/diag.sh [tag] [kernel-regex] [config]
tag=${1:-diag}; kre=${2:-k_smem<512}; cfg=${3:-C4}
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/${tag}_build.log 2>&1
timeout 900 python tools/phase_profile.py --config $cfg > gpurun_out/${tag}_phase.json 2> gpurun_out/${tag}_phase.err; echo "phase rc=$?"
timeout 900 python tools/probe_stats.py --config $cfg --scale 1.0 > gpurun_out/${tag}_probe.json 2> gpurun_out/${tag}_probe.err; echo "probe rc=$?"
if [ -n "$kre" ] && [ "$kre" != "none" ]; then
  timeout 1500 ncu --set full --import-source on --clock-control none --kernel-name-base demangled -k "regex:$kre" -c 1 \
    -o gpurun_out/${tag} python bench.py --config $cfg --steps 1 --warmup 0 --no-e2e --no-cpu-baseline --no-replay > gpurun_out/${tag}_ncu.log 2>&1
  echo "ncu rc=$?"
  ncu -i gpurun_out/${tag}.ncu-rep --page source --csv --print-source sass > gpurun_out/${tag}_source.csv 2>/dev/null
  ncu -i gpurun_out/${tag}.ncu-rep --page details --csv > gpurun_out/${tag}_details.csv 2>/dev/null
  (cd /tmp && cuobjdump -xelf all $GRAFT_REPO_ROOT/paper_conf_sc_awanhedbdoy21_b200/liblocassm.so > /dev/null 2>&1 && nvdisasm -g -c locassm.sm_100a.cubin > /tmp/all.sass 2>/dev/null)
  python tools/ncu_lines.py gpurun_out/${tag}_source.csv /tmp/all.sass > gpurun_out/${tag}_lines.txt 2>&1
  rm -f gpurun_out/${tag}.ncu-rep
fi
echo done
