#!/bin/bash
# DRAM bytes + duration per launch of the table-class kernels of one C4S step (ncu, serial classes).
#   gpurun -- bash tools/ncu_traffic.sh <tag> [so]
tag=$1; so=${2:-}
mkdir -p gpurun_out
python bench.py --config ${CFG:-C4S} --steps 1 --warmup 0 --no-e2e --no-cpu-baseline --no-replay > /dev/null 2>&1
LA_SO=$so LA_SERIAL_CLASSES=1 timeout 1200 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum,smsp__inst_executed.sum,sm__warps_active.avg.pct_of_peak_sustained_active \
  --clock-control none -k regex:"k_small|k_smem" --csv --log-file gpurun_out/${tag}_traffic.csv \
  python bench.py --config ${CFG:-C4S} --steps 1 --warmup 0 --no-e2e --no-cpu-baseline --no-replay > /dev/null 2>&1
echo "ncu rc=$?"
python - "$tag" <<'PY'
import csv, sys, collections
tag = sys.argv[1]
rows = [r for r in csv.reader(open(f"gpurun_out/{tag}_traffic.csv")) if len(r) > 10]
h = rows[0]
agg = collections.defaultdict(dict)
for r in rows[1:]:
    d = dict(zip(h, r))
    agg[(d["ID"], d["Kernel Name"][:40])][d["Metric Name"]] = float(d["Metric Value"].replace(",", ""))
for (i, n), m in sorted(agg.items(), key=lambda x: int(x[0][0])):
    print(i, n, "ms %.2f" % (m.get("gpu__time_duration.sum", 0) / 1e6), "dram GB %.3f" % ((m.get("dram__bytes_read.sum", 0) + m.get("dram__bytes_write.sum", 0)) / 1e9),
          "winst %.3g" % m.get("smsp__inst_executed.sum", 0), "occ %.0f%%" % m.get("sm__warps_active.avg.pct_of_peak_sustained_active", 0))
PY
