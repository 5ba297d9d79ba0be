import sys, os, time
sys.path.insert(0, os.getcwd()); sys.path.insert(0, os.path.join(os.getcwd(), "tests"))
import numpy as np
from gen import Params, make
from paper_conf_sc_awanhedbdoy21_b200 import LocalAssembler
b = make("C2", scale=0.03)
P = Params()
la = LocalAssembler(0)
for n in [int(x) for x in (sys.argv[1:] or ["1", "3", "8"])]:
    t = time.time()
    print("chunks", n, flush=True)
    r = la.extend_streamed(b, P, n)
    print("  ok", time.time() - t, la.stats()["inserts"], flush=True)
