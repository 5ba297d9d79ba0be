"""Per-class phase breakdown of the shared-memory kernels (clock64 counters: builds a copy of the
library with -DLA_PROFILE_CLOCKS=1 and runs it with LA_PROFILE=1).

  python tools/phase_profile.py [--config C4] [--scale 1.0]
Prints, per table class, the builders' leader cycles split into wait / prefix / clear / filter /
build / link, and the walker's wait / walk cycles, as fractions, plus per-attempt averages.
"""
import argparse
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--config", default="C4")
    ap.add_argument("--scale", type=float, default=1.0)
    a = ap.parse_args()
    os.environ["LA_PROFILE"] = "1"
    # the phase clocks are compiled out of the production library: build a profiling copy
    import importlib.util
    import subprocess
    so = "/tmp/liblocassm_prof.so"
    os.environ["LA_SO"] = so   # before the package (and its ctypes binding) is imported
    spec = importlib.util.spec_from_file_location("la_build", os.path.join(ROOT, "paper_conf_sc_awanhedbdoy21_b200", "build.py"))
    b = importlib.util.module_from_spec(spec)
    spec.loader.exec_module(b)
    subprocess.check_call([b.NVCC, *b.FLAGS, "-DLA_PROFILE_CLOCKS=1", "-o", so, *b.SRC])
    import bench
    from paper_conf_sc_awanhedbdoy21_b200 import LocalAssembler
    batch, params = bench.load_workload(a.config, 0, a.scale)
    with LocalAssembler(0) as la:
        la.load(batch, params)
        la.extend_device()
        la.extend_device()
        st = la.stats()
    names = ["smem64x12", "smem128x6", "smem256x3", "smem512x2", "smem1024x1", "xl1024x1"]
    out = {}
    for c, n in enumerate(names):
        p = st["prof_cycles"][c]
        att = max(st["cls_attempts"][c], 1)
        b = p[:6]
        tb = max(sum(b), 1)
        out[n] = {"ms": round(st["cls_ms"][c], 2), "ends": st["cls_ends"][c], "attempts": att,
                  "inserts_per_attempt": round(st["cls_inserts"][c] / att),
                  "builder_cycles_per_attempt": round(tb / att),
                  "builder_split": dict(zip(["wait_walker", "prefix", "clear", "filter", "build", "link"],
                                            [round(x / tb, 3) for x in b])),
                  "walker_cycles_per_attempt": {"wait": round(p[6] / att), "walk": round(p[7] / att)}}
    print(json.dumps(out, indent=1))


if __name__ == "__main__":
    main()
