"""Small runs of every table class for compute-sanitizer (memcheck / racecheck / synccheck):

  compute-sanitizer --tool racecheck python tools/sanitize_run.py [--ends 2000]

C1 (all 400 ends) and a slice of C3 (the sparse ends plus two hot ends), each run with the planner's
own routing and with every end forced into each table class (LA_FORCE_CLASS 0..5; 5 = XL), at the
default schedule and at k >= 64 (pointer keys).  Every run is compared with the oracle end by end, so
a sanitizer run is also a parity run.
"""
import argparse
import os
import sys

import numpy as np

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--ends", type=int, default=2000)
    ap.add_argument("--classes", default="none,0,1,2,3,4,5,6")
    a = ap.parse_args()
    import oracle
    from gen import Params, make
    from paper_conf_sc_awanhedbdoy21_b200 import LocalAssembler
    c1 = make("C1")
    c3 = make("C3")
    r = c3.reads_per_end()
    rng = np.random.default_rng(0)
    sparse = rng.choice(np.nonzero(r < 2000)[0] // 2, a.ends // 2, replace=False)
    hot = np.nonzero(r >= 10000)[0][:2] // 2
    c3s = c3.select_contigs(np.unique(np.concatenate([sparse, hot])))
    runs = [("C1", c1, Params(k_start=21, k_min=21, k_max=21)), ("C3slice", c3s, Params()),
            ("C3slice_k65", c3s, Params(k_start=65, k_min=57, k_max=97))]
    bad = 0
    with LocalAssembler(0) as la:
        for name, b, p in runs:
            ref = oracle.extend(b, p)
            for cls in a.classes.split(","):
                if cls == "none":
                    os.environ.pop("LA_FORCE_CLASS", None)
                else:
                    os.environ["LA_FORCE_CLASS"] = cls
                res = la.load(b, p).extend()
                st = la.stats()
                ok = (res.ext_list() == ref["ext"] and np.array_equal(res.term, ref["term"])
                      and np.array_equal(res.k_used, ref["k_used"]) and np.array_equal(res.n_attempts, ref["n_attempts"]))
                bad += not ok
                print(f"{name} force_class={cls}: {b.n_ends} ends, parity {'ok' if ok else 'MISMATCH'}, "
                      f"inl/ref attempts per class {st['cls_inl_attempts']} {st['cls_ref_attempts']}, "
                      f"overflow->global {st['ends_by_class'][4]}", flush=True)
    os.environ.pop("LA_FORCE_CLASS", None)
    return 1 if bad else 0


if __name__ == "__main__":
    sys.exit(main())
