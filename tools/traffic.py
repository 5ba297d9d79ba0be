"""Per-kernel DRAM traffic and duration from an ncu launch list with dram metrics.

  ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none \
      --csv --log-file launches.csv python bench.py --steps 1 --warmup 0 --no-cpu-baseline --no-e2e
  python tools/traffic.py launches.csv > profiles/r01_traffic.json

The table kernels (k_small*, k_smem*) are summed per step: bench.py reports that sum as
roofline.traffic (bytes per step of the dominant phase).
"""
import collections
import csv
import json
import sys

UNIT = {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9, "ns": 1, "us": 1e3, "ms": 1e6, "usecond": 1e3,
        "nsecond": 1, "msecond": 1e6}


def main():
    rows = list(csv.reader(open(sys.argv[1])))
    hdr = None
    per = collections.defaultdict(lambda: collections.defaultdict(float))
    launches = collections.defaultdict(set)
    for r in rows:
        if "Kernel Name" in r:
            hdr = r
            continue
        if not hdr or len(r) != len(hdr):
            continue
        d = dict(zip(hdr, r))
        name = d["Kernel Name"].split("(")[0].replace("void ", "")
        v = float(d["Metric Value"].replace(",", "")) * UNIT.get(d["Metric Unit"], 1)
        per[name][d["Metric Name"]] += v
        launches[name].add(d["ID"])
    out = {"kernels": {}}
    tab = {"dram_bytes": 0.0, "time_ns": 0.0}
    for n, m in per.items():
        b = m.get("dram__bytes_read.sum", 0) + m.get("dram__bytes_write.sum", 0)
        out["kernels"][n] = {"launches": len(launches[n]), "dram_bytes": b, "time_ns": m.get("gpu__time_duration.sum", 0)}
        if "k_small" in n or "k_smem" in n:
            tab["dram_bytes"] += b
            tab["time_ns"] += m.get("gpu__time_duration.sum", 0)
    out["table_kernels_per_step"] = tab
    print(json.dumps(out, indent=1))


if __name__ == "__main__":
    main()
