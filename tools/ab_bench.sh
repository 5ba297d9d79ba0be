set -e
# Usage: populate _headcsrc/ (git-ignored) with the HEAD sources first, e.g.
#   mkdir -p _headcsrc/csrc _headcsrc/include; for f in la_device.cuh la_global.cuh la_kernels.cuh la_smem.cuh locassm.cu; do
#     git show HEAD:paper_conf_sc_awanhedbdoy21_b200/csrc/$f > _headcsrc/csrc/$f; done; git show HEAD:include/locassm.h > _headcsrc/include/locassm.h
# then: gpurun -- bash tools/ab_bench.sh
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
nvcc -gencode arch=compute_100a,code=sm_100a -O3 -lineinfo -std=c++17 -shared -Xcompiler -fPIC -I_headcsrc/include -o /tmp/head.so _headcsrc/csrc/locassm.cu
for rep in 1 2; do
for v in head new; do
  so=""; [ $v = head ] && so=/tmp/head.so
  LA_SO=$so timeout 600 python bench.py --steps 3 --warmup 2 --no-cpu-baseline --no-e2e 2>/dev/null | python -c "import json,sys; d=json.load(sys.stdin); print('$v', d['ms_per_step'])"
done; done
