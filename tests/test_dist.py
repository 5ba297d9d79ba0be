"""Multi-process (world_size 2, gloo, CPU) checks of the multi-GPU driver's host logic: the contig
partition and the final result gather.  The per-rank "device" is the CPU oracle here, so the test
checks partition + gather, not the kernels (those are covered by the GPU parity tests)."""
import os
import socket

import numpy as np
import pytest

from conftest import cached_batch


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def test_partition_balanced_and_deterministic():
    from paper_conf_sc_awanhedbdoy21_b200.dist import contig_work, partition
    b = cached_batch("C2", scale=0.03)
    w = contig_work(b)
    for world in (2, 4, 8):
        o1, o2 = partition(w, world), partition(w, world)
        assert np.array_equal(o1, o2)
        assert o1.min() >= 0 and o1.max() < world
        loads = np.bincount(o1, weights=w, minlength=world)
        assert loads.max() <= 1.15 * w.sum() / world + w.max()
    assert (partition(w, 1) == 0).all()


def _rank(rank, world, port, out_q):
    import torch.distributed as dist
    import oracle
    from gen import Params
    from paper_conf_sc_awanhedbdoy21_b200.api import Result
    from paper_conf_sc_awanhedbdoy21_b200.dist import contig_work, gather_results, partition, select_contigs
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    b = cached_batch("C2", scale=0.03).select_contigs(np.arange(120))
    owner = partition(contig_work(b), world)
    mine = np.nonzero(owner == rank)[0]
    sub = select_contigs(b, mine)

    class B:  # adapt to the oracle's interface
        pass
    x = B()
    for f in ("contig_seq", "contig_off", "read_seq", "read_qual", "read_off", "end_read_off"):
        setattr(x, f, getattr(sub, f))
    x.n_contigs = len(mine)
    x.n_ends = 2 * len(mine)
    x.n_reads = int(sub.read_off.shape[0] - 1)
    r = oracle.extend(x, Params())
    lens = np.array([len(s) for s in r["ext"]], np.int64)
    res = Result(np.concatenate([[0], np.cumsum(lens)]).astype(np.int64),
                 np.frombuffer("".join(r["ext"]).encode(), np.uint8).copy(), r["term"], r["k_used"],
                 r["n_attempts"])
    g = gather_results(res, mine, b.n_contigs)
    if rank == 0:
        out_q.put((g.ext_list(), g.term.tolist(), g.k_used.tolist(), g.n_attempts.tolist()))
    dist.destroy_process_group()


def test_gather_world2_gloo(orc):
    import torch.multiprocessing as mp
    from gen import Params
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_rank, args=(r, 2, port, q)) for r in range(2)]
    for p in procs:
        p.start()
    got = q.get(timeout=300)
    for p in procs:
        p.join(timeout=120)
        assert p.exitcode == 0
    b = cached_batch("C2", scale=0.03).select_contigs(np.arange(120))
    ref = orc.extend(b, Params())
    assert got[0] == ref["ext"]
    assert got[1] == ref["term"].tolist() and got[2] == ref["k_used"].tolist()
    assert got[3] == ref["n_attempts"].tolist()
