#!/bin/bash
# Phase profile + one `ncu --set full` capture per hot kernel (k_small<128>, k_smem<256,0>, XL k_smem<512,1>).
set -x
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
LA_SERIAL_CLASSES=1 timeout 600 python tools/phase_profile.py > gpurun_out/phase.json 2> gpurun_out/phase.err
for K in ${KERNELS:-"k_small:1" "k_smem:4"}; do
  name=${K%%:*}; cnt=${K##*:}
  timeout 1200 ncu --set full --import-source on --clock-control none -k regex:"$name" --launch-count $cnt \
    -o gpurun_out/${name}_full python bench.py --steps 1 --warmup 0 --no-cpu-baseline --no-e2e > gpurun_out/ncu_${name}.log 2>&1
done
echo done
