"""Time la_append_extensions (NEXT N1, Fig 4 "Append extensions to contigs") on the C4 workload:
load -> extend_device -> append, the append timed with CUDA events on the context stream, against the
measured HBM copy peak.  Algorithmic bytes per launch = read (contig bytes + extension bytes +
contig_off + ext_off) + write (extended-contig bytes + out_off).  Prints one JSON line.

  python tools/append_bw.py [--config C4] [--iters 20]
"""
import argparse
import json
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))

import torch  # noqa: E402

import bench  # noqa: E402
from paper_conf_sc_awanhedbdoy21_b200 import LocalAssembler  # noqa: E402


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--config", default="C4")
    ap.add_argument("--scale", type=float, default=1.0)
    ap.add_argument("--iters", type=int, default=20)
    a = ap.parse_args()
    batch, params = bench.load_workload(a.config, 0, a.scale)
    st = torch.cuda.Stream()
    la = LocalAssembler(0, stream=st)
    d = la.load(batch, params).extend_device()
    n = batch.n_contigs
    cseq = torch.from_numpy(batch.contig_seq).cuda()
    coff = torch.from_numpy(batch.contig_off).cuda()
    torch.cuda.synchronize()
    for _ in range(3):
        seq, off = la.append_extensions(cseq, coff, d["ext_off"], d["ext_seq"])
    ev0, ev1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    ms = []
    for _ in range(a.iters):
        ev0.record(st)
        seq, off = la.append_extensions(cseq, coff, d["ext_off"], d["ext_seq"])
        ev1.record(st)
        ev1.synchronize()
        ms.append(ev0.elapsed_time(ev1))
    ms.sort()
    med = ms[len(ms) // 2]
    contig_b = int(batch.contig_off[-1] - batch.contig_off[0])
    ext_b = int(la.stats()["ext_bases"])
    byts = 2 * (contig_b + ext_b) + 8 * ((n + 1) + (2 * n + 1) + (n + 1))
    peak = json.load(open(os.path.join(bench.ROOT, "MEASURED_PEAKS.json")))["hbm_gbs"]
    gbs = byts / (med * 1e-3) / 1e9
    print(json.dumps({"kernel": "k_append_ext", "config": a.config, "n_contigs": n, "contig_bytes": contig_b,
                      "ext_bytes": ext_b, "alg_bytes": byts, "ms_median": med, "ms_min": ms[0],
                      "achieved_gbs": gbs, "peak_gbs": peak, "frac": gbs / peak,
                      "note": "event pair includes the call's host-side launch; stream synchronised by the call"}))


if __name__ == "__main__":
    main()
