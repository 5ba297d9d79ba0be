set -x
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
timeout 600 python tools/phase_profile.py > gpurun_out/phase.json 2> gpurun_out/phase.err
timeout 1200 ncu --set full --import-source on --clock-control none -k regex:k_smem --launch-count 6 -o gpurun_out/ksmem_full python bench.py --steps 1 --warmup 0 --no-cpu-baseline --no-e2e > gpurun_out/ncu_full.log 2>&1
echo done
