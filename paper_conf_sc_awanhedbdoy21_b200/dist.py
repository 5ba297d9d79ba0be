"""Multi-GPU driver: contig-batch partitioning across ranks and the final result gather.

Local assembly is embarrassingly parallel over contig ends and node-local with no
communication, so the only collective is one gather of the results to rank 0 after
all extension is done.  One process per GPU; torch.distributed is plumbing only.
"""
from __future__ import annotations

import numpy as np

from .api import Result


def contig_work(batch, k_start: int = 33) -> np.ndarray:
    """Per-contig work estimate: sum over both ends of sum_reads max(0, len - k_start)."""
    roff = np.asarray(batch.read_off)
    eoff = np.asarray(batch.end_read_off)
    nbases = roff[eoff[1:]] - roff[eoff[:-1]]
    nreads = np.diff(eoff)
    w = np.maximum(0, nbases - nreads * k_start)
    return w[0::2] + w[1::2]


def partition(work: np.ndarray, world: int, heavy_q: float = 0.99) -> np.ndarray:
    """Rank of every contig.  Contigs above the `heavy_q` work quantile are placed by LPT (largest
    first onto the least-loaded rank); the rest are cut into contiguous chunks that fill each rank
    up to the balanced share.  Deterministic: every rank computes the same assignment."""
    n = work.shape[0]
    owner = np.full(n, -1, np.int64)
    if world <= 1 or n == 0:
        return np.zeros(n, np.int64)
    thr = np.quantile(work, heavy_q) if n > 100 else np.inf
    heavy = np.nonzero(work > thr)[0]
    load = np.zeros(world, np.float64)
    for c in heavy[np.argsort(-work[heavy], kind="stable")]:
        r = int(np.argmin(load))
        owner[c] = r
        load[r] += work[c]
    light = np.nonzero(owner < 0)[0]
    total = float(work.sum())
    target = total / world
    # contiguous fill of the remaining capacity of each rank, in rank order
    cum = np.cumsum(work[light].astype(np.float64))
    room = np.maximum(0.0, target - load)
    bounds = np.cumsum(room)
    r = np.searchsorted(bounds, cum, side="left")
    owner[light] = np.minimum(r, world - 1)
    return owner


def select_contigs(batch, contig_ids):
    """Sub-batch (numpy arrays, same layout) holding the given contigs in the given order."""
    from types import SimpleNamespace
    contig_ids = np.asarray(contig_ids, np.int64)
    coff = np.asarray(batch.contig_off)
    eoff = np.asarray(batch.end_read_off)
    roff = np.asarray(batch.read_off)

    def ranges(starts, lens):
        tot = int(lens.sum())
        if tot == 0:
            return np.zeros(0, np.int64)
        base = np.repeat(starts - np.concatenate([[0], np.cumsum(lens)[:-1]]), lens)
        return base + np.arange(tot, dtype=np.int64)

    clen = coff[contig_ids + 1] - coff[contig_ids]
    ends = np.stack([2 * contig_ids, 2 * contig_ids + 1], 1).reshape(-1)
    nre = eoff[ends + 1] - eoff[ends]
    rids = ranges(eoff[ends], nre)
    rlen = roff[rids + 1] - roff[rids]
    out = SimpleNamespace()
    out.contig_seq = np.asarray(batch.contig_seq)[ranges(coff[contig_ids], clen)]
    out.contig_off = np.concatenate([[0], np.cumsum(clen)]).astype(np.int64)
    bidx = ranges(roff[rids], rlen)
    out.read_seq = np.asarray(batch.read_seq)[bidx]
    out.read_qual = np.asarray(batch.read_qual)[bidx]
    out.read_off = np.concatenate([[0], np.cumsum(rlen)]).astype(np.int64)
    out.end_read_off = np.concatenate([[0], np.cumsum(nre)]).astype(np.int64)
    return out


def _ranges(starts, lens):
    """Concatenation of arange(starts[i], starts[i] + lens[i]) (vectorised)."""
    lens = np.asarray(lens, np.int64)
    tot = int(lens.sum())
    if tot == 0:
        return np.zeros(0, np.int64)
    base = np.repeat(np.asarray(starts, np.int64) - np.concatenate([[0], np.cumsum(lens)[:-1]]), lens)
    return base + np.arange(tot, dtype=np.int64)


def merge_results(parts, n_contigs_total: int) -> Result:
    """Scatter per-rank packed results into global end order (vectorised, no per-end loop).
    parts: list of (end_ids int64[ne], lens int64[ne], codes uint8[ne, 3], seq uint8[nb])."""
    N = 2 * n_contigs_total
    glen = np.zeros(N, np.int64)
    term = np.zeros(N, np.uint8)
    k = np.zeros(N, np.uint8)
    att = np.zeros(N, np.uint8)
    for ids, lens, codes, _ in parts:
        glen[ids] = lens
        term[ids], k[ids], att[ids] = codes[:, 0], codes[:, 1], codes[:, 2]
    ext_off = np.concatenate([[0], np.cumsum(glen)]).astype(np.int64)
    ext_seq = np.zeros(int(ext_off[-1]), np.uint8)
    for ids, lens, _, seq in parts:
        if seq.shape[0]:
            ext_seq[_ranges(ext_off[ids], lens)] = seq
    return Result(ext_off, ext_seq, term, k, att)


def gather_results(res: Result, contig_ids: np.ndarray, n_contigs_total: int, group=None, device=None):
    """Gather every rank's Result to rank 0 and scatter it back into global end order.

    One all_gather of the per-rank sizes, then exact-size point-to-point transfers of the packed
    arrays to rank 0 (the only inter-GPU traffic, after extension; no padding to the largest rank),
    merged without a per-end loop.  Returns the merged Result on rank 0, None elsewhere."""
    import torch
    import torch.distributed as dist
    rank, world = dist.get_rank(group), dist.get_world_size(group)
    dev = device if device is not None else (torch.device("cuda", torch.cuda.current_device())
                                             if dist.get_backend(group) == "nccl" else torch.device("cpu"))
    contig_ids = np.asarray(contig_ids, np.int64)
    ids = np.stack([2 * contig_ids, 2 * contig_ids + 1], 1).reshape(-1)
    lens = np.diff(res.ext_off).astype(np.int64)
    codes = np.stack([res.term, res.k_used, res.n_attempts], 1).astype(np.uint8).reshape(-1, 3)
    meta = torch.tensor([ids.shape[0], int(res.ext_off[-1])], dtype=torch.int64, device=dev)
    sizes = [torch.zeros(2, dtype=torch.int64, device=dev) for _ in range(world)]
    dist.all_gather(sizes, meta, group=group)
    sizes = [s.cpu().numpy() for s in sizes]
    if rank != 0:
        for a in (ids, lens, codes.reshape(-1), np.asarray(res.ext_seq, np.uint8)):
            if a.shape[0]:
                dist.send(torch.from_numpy(np.ascontiguousarray(a)).to(dev), dst=0, group=group)
        return None
    parts = [(ids, lens, codes, np.asarray(res.ext_seq, np.uint8))]
    for r in range(1, world):
        ne, nb = int(sizes[r][0]), int(sizes[r][1])
        got = []
        for n, dt in ((ne, torch.int64), (ne, torch.int64), (3 * ne, torch.uint8), (nb, torch.uint8)):
            t = torch.empty(n, dtype=dt, device=dev)
            if n:
                dist.recv(t, src=r, group=group)
            got.append(t.cpu().numpy())
        parts.append((got[0], got[1], got[2].reshape(-1, 3), got[3]))
    return merge_results(parts, n_contigs_total)
