"""Wall-clock sweep of la_extend_streamed chunk counts on a pinned host copy of the C4 batch.

  python tools/e2e_sweep.py [--chunks 1,4,8,16] [--scale 1.0]
"""
import argparse
import json
import os
import sys
import time

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--chunks", default="1,4,8,16")
    ap.add_argument("--scale", type=float, default=1.0)
    a = ap.parse_args()
    import torch
    import bench
    from paper_conf_sc_awanhedbdoy21_b200 import LocalAssembler
    batch, params = bench.load_workload("C4", 0, a.scale)
    pinned = type("HostBatch", (), {})()
    for f in ("contig_seq", "contig_off", "read_seq", "read_qual", "read_off", "end_read_off"):
        setattr(pinned, f, torch.from_numpy(getattr(batch, f)).pin_memory())
    out = {}
    with LocalAssembler(0) as la:
        ref = None
        for n in [int(x) for x in a.chunks.split(",")]:
            la.extend_streamed(pinned, params, n)
            ts = []
            for _ in range(3):
                torch.cuda.synchronize()
                t0 = time.perf_counter()
                r = la.extend_streamed(pinned, params, n)
                ts.append(time.perf_counter() - t0)
            st = la.stats()
            same = None
            if ref is None:
                ref = (r.ext_off.copy(), r.ext_seq.copy(), r.term.copy())
            else:
                same = bool((ref[0] == r.ext_off).all() and (ref[1] == r.ext_seq).all() and (ref[2] == r.term).all())
            out[n] = {"ms": round(min(ts) * 1e3, 2), "device_ms": round(st["ms_total"], 2), "same_as_first": same}
            print(n, out[n], file=sys.stderr)
        la.load(batch, params)
        t0 = time.perf_counter()
        la.load(pinned, params).extend()
        out["load+extend"] = {"ms": round((time.perf_counter() - t0) * 1e3, 2)}
    print(json.dumps(out))


if __name__ == "__main__":
    main()
