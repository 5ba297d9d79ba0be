#!/bin/bash
# ncu --set full of one table-class kernel launch (source-level), plus the serial-classes bench.
#   gpurun -- bash tools/ncu_class.sh <tag> <kernel-regex> [config]
tag=$1; kre=$2; cfg=${3:-C4S}
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
python bench.py --config $cfg --steps 1 --warmup 0 --no-e2e --no-cpu-baseline --no-replay > /dev/null 2>&1   # cache the workload
timeout 1200 ncu --set full --import-source on --clock-control none --kernel-name-base demangled -k "regex:$kre" -c 1 \
  -o gpurun_out/${tag} python bench.py --config $cfg --steps 1 --warmup 0 --no-e2e --no-cpu-baseline --no-replay > gpurun_out/${tag}_ncu.log 2>&1
echo "ncu rc=$?"
ncu -i gpurun_out/${tag}.ncu-rep --page source --csv --print-source sass > gpurun_out/${tag}_source.csv 2>/dev/null
ncu -i gpurun_out/${tag}.ncu-rep --page details --csv > gpurun_out/${tag}_details.csv 2>/dev/null
cuobjdump -xelf all paper_conf_sc_awanhedbdoy21_b200/liblocassm.so > /dev/null 2>&1 && nvdisasm -g -c locassm.sm_100a.cubin > gpurun_out/${tag}_all.sass 2>/dev/null; rm -f *.cubin
ls -la gpurun_out/${tag}*
