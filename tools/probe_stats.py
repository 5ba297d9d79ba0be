"""Probe-length statistics of the shared-memory table passes (debug build with -DLA_PROBE_STATS).

  python tools/probe_stats.py [--config C4] [--scale 0.2]
"""
import argparse
import ctypes
import json
import os
import subprocess
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--config", default="C4")
    ap.add_argument("--scale", type=float, default=0.2)
    a = ap.parse_args()
    so = "/tmp/liblocassm_dbg.so"
    os.environ["LA_SO"] = so   # before the package (and its ctypes binding) is imported
    import importlib.util
    spec = importlib.util.spec_from_file_location("la_build", os.path.join(ROOT, "paper_conf_sc_awanhedbdoy21_b200", "build.py"))
    b = importlib.util.module_from_spec(spec)
    spec.loader.exec_module(b)
    subprocess.check_call([b.NVCC, *b.FLAGS, "-DLA_PROBE_STATS", "-o", so, *b.SRC])
    import bench
    from paper_conf_sc_awanhedbdoy21_b200 import LocalAssembler
    lib = ctypes.CDLL(so)
    batch, params = bench.load_workload(a.config, 0, a.scale)
    out = (ctypes.c_ulonglong * 12)()
    res = {}
    for cls in ["64x12,128x6,256x3,256x2,512x1"]:
        with LocalAssembler(0) as la:
            la.load(batch, params)
            lib.la_debug_probe_stats(out, 1)
            la.extend_device()
            lib.la_debug_probe_stats(out, 1)
            v = list(out)
            st = la.stats()
        res[cls] = {"insert_calls": v[0], "insert_rounds_per_call": v[1] / max(v[0], 1),
                    "inserting_lanes_per_call": v[2] / max(v[0], 1), "claims": v[3],
                    "lookup_calls": v[4], "lookup_rounds_per_call": v[5] / max(v[4], 1),
                    "lookup_lanes_per_call": v[6] / max(v[4], 1),
                    "filter_warp_iters": v[8], "filter_lanes_per_iter": v[9] / max(v[8], 1),
                    "cas_issued": v[10], "rereads": v[11], "inserts": st["inserts"],
                    "ms_total": st["ms_total"]}
    print(json.dumps(res, indent=1))


if __name__ == "__main__":
    main()
