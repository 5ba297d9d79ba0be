"""NEXT N4, candidate-read selection (readings S1-S6; paper P:L308-311, L399-402).

CPU: the oracle (oracle/select.cpp) pinned against what the construction fixes — the truth coordinates
of an error-free pool on a genome with unique seeds (closed form), hand-built reads at the mismatch,
overlap, N and strand boundaries, and the reverse-complement symmetry of the definition.
GPU (-m gpu): la_select_reads against the oracle, record by record and byte by byte, and the selected
batch extended by la_extend against the oracle's extension of the oracle's selection.
"""
import numpy as np
import pytest

from gen.pool import make_pool

SP = dict(w=150, s=16, t=4, o=20, mm_pct=4)
GPU_SP = dict(window=150, seed_len=16, seed_stride=4, min_overlap=20, max_mism_pct=4)
_COMP = bytes.maketrans(b"ACGTN", b"TGCAN")
ASC = np.frombuffer(b"ACGT", np.uint8)


def _rc(b: bytes) -> bytes:
    return b[::-1].translate(_COMP)


def _truth_selection(pool, o=20, L=150):
    """Closed form of S1-S4 on an error-free pool whose genome has unique seeds on both strands: a read
    aligns exactly at its true placement, so pair i is a candidate of the RIGHT end of contig [cs, ce)
    iff its forward read [f, f+L) overlaps the window [ce-150, ce) by >= o (strand +, outward), or its
    reverse read [g, g+L), g = f+ins-L, does and reaches past ce; LEFT end [cs, cs+150): the reverse read
    overlaps by >= o (strand -), or the forward read does and starts before cs.  o >= s+t-1 makes a stride
    seed inside the overlap certain.  The pair's flip is its strand z; both reads come out genome-forward."""
    T = pool.truth
    f, ins, z = T["frag_start"], T["ins"], T["strand"]
    g = f + ins - L
    rec = []
    for c, (cs, ce) in enumerate(zip(T["contig_start"], T["contig_end"])):
        for side in (0, 1):
            wl, wh = (max(cs, ce - 150), ce) if side else (cs, min(cs + 150, ce))
            ovf = np.minimum(f + L, wh) - np.maximum(f, wl)
            ovr = np.minimum(g + L, wh) - np.maximum(g, wl)
            if side:
                sel = (ovf >= o) | ((ovr >= o) & (g + L > ce))
            else:
                sel = (ovr >= o) | ((ovf >= o) & (f < cs))
            for i in np.nonzero(sel)[0]:
                rec.append((2 * c + side, int(i), int(z[i])))
    rec.sort()
    return rec


def _select(orc, pool, **kw):
    return orc.select_reads(pool.contig_seq, pool.contig_off, pool.read_seq, pool.read_qual, pool.read_off,
                            **dict(SP, **kw))


def test_select_closed_form_error_free(orc):
    pool = make_pool(seed=7, genome_len=30000, n_contigs=14, coverage=12, err=0.0, n_rate=0.0, unique_k=16)
    r = _select(orc, pool)
    got = list(zip(r["sel_end"].tolist(), r["sel_pair"].tolist(), r["sel_flip"].tolist()))
    assert got == _truth_selection(pool)
    assert len(got) > 100
    # S5: every selected read is the genome forward substring of its true placement
    G = ASC[pool.truth["genome"]].tobytes()
    f, ins = pool.truth["frag_start"], pool.truth["ins"]
    seq, off = r["read_seq"].tobytes(), r["read_off"]
    for n, (e, i, z) in enumerate(got):
        fwd = G[f[i]:f[i] + 150]
        rev = G[f[i] + ins[i] - 150:f[i] + ins[i]]
        m0, m1 = (fwd, rev) if z == 0 else (rev, fwd)
        assert seq[off[2 * n]:off[2 * n + 1]] == m0
        assert seq[off[2 * n + 1]:off[2 * n + 2]] == m1


def _one_pair_pool(contig: bytes, mate0: bytes, mate1: bytes):
    class P:
        pass
    p = P()
    p.contig_seq = np.frombuffer(contig, np.uint8).copy()
    p.contig_off = np.array([0, len(contig)], np.int64)
    p.read_seq = np.frombuffer(mate0 + mate1, np.uint8).copy()
    p.read_qual = np.full(len(mate0) + len(mate1), ord("I"), np.uint8)
    p.read_off = np.array([0, len(mate0), len(mate0) + len(mate1)], np.int64)
    return p


def _rand(rng, n):
    return ASC[rng.integers(0, 4, n)].tobytes()


def _mutate(b: bytes, pos):
    x = bytearray(b)
    for p in pos:
        x[p] = {65: 67, 67: 71, 71: 84, 84: 65}[x[p]]
    return bytes(x)


@pytest.mark.parametrize("M,ok", [(0, True), (4, True), (5, False)])
def test_select_mismatch_rate_boundary(orc, M, ok):
    """S2(c): a read overlapping the contig's last 100 bases (L = 100) with M mismatches is kept iff
    100*M <= 4*100, i.e. M <= 4; mismatches placed away from the read's first 40 bases keep the seeds."""
    rng = np.random.default_rng(11)
    C = _rand(rng, 600)
    m0 = _mutate(C[500:] + _rand(rng, 50), [50 + 10 * i for i in range(M)])
    p = _one_pair_pool(C, m0, _rand(rng, 150))
    r = _select(orc, p)
    assert (r["sel_end"].tolist() == [1]) == ok
    if ok:
        assert r["sel_pair"].tolist() == [0] and r["sel_flip"].tolist() == [0]


def test_select_n_counts_as_mismatch_and_breaks_seeds(orc):
    rng = np.random.default_rng(12)
    C = _rand(rng, 600)
    base = C[500:] + _rand(rng, 50)
    # 5 N in the overlap (far from the first seeds): 5 mismatches > 4 -> rejected
    x = bytearray(base)
    for i in range(5):
        x[60 + 8 * i] = ord("N")
    assert _select(orc, _one_pair_pool(C, bytes(x), _rand(rng, 150)))["sel_end"].size == 0
    # 4 N: kept
    x = bytearray(base)
    for i in range(4):
        x[60 + 8 * i] = ord("N")
    assert _select(orc, _one_pair_pool(C, bytes(x), _rand(rng, 150)))["sel_end"].tolist() == [1]
    # a read overlapping the window by 24 bases (d = 576): seeds at j = 0, 4, 8 lie in the overlap;
    # an N at positions 8 and 15 of the read hits every one of them.  With mm_pct = 10 its 2 mismatches
    # of 24 pass S2(c) (200 <= 240), so only the seed rule rejects it; without N it is kept
    y = C[576:] + _rand(rng, 126)
    assert _select(orc, _one_pair_pool(C, y, _rand(rng, 150)), mm_pct=10)["sel_end"].tolist() == [1]
    yn = bytearray(y)
    yn[8] = ord("N")
    yn[15] = ord("N")
    assert _select(orc, _one_pair_pool(C, bytes(yn), _rand(rng, 150)), mm_pct=10)["sel_end"].size == 0
    # the N moved to 16 and 17: the seed at j = 0 is N-free again -> kept
    yn[8], yn[15] = y[8], y[15]
    yn[16] = yn[17] = ord("N")
    assert _select(orc, _one_pair_pool(C, bytes(yn), _rand(rng, 150)), mm_pct=10)["sel_end"].tolist() == [1]


def test_select_overlap_and_strand_rules(orc):
    rng = np.random.default_rng(13)
    C = _rand(rng, 600)
    tail = _rand(rng, 150)
    # S2(b): window overlap 20 kept, 19 rejected (d = 580 / 581; the seed at j = 0 or 4 still fits)
    assert _select(orc, _one_pair_pool(C, C[580:] + tail[:130], _rand(rng, 150)))["sel_end"].tolist() == [1]
    assert _select(orc, _one_pair_pool(C, C[581:] + tail[:131], _rand(rng, 150)))["sel_end"].size == 0
    # S3: a read lying inside the RIGHT window: kept on strand + (its mate is past the end) ...
    inside = C[460:590]
    r = _select(orc, _one_pair_pool(C, inside, _rand(rng, 150)))
    assert r["sel_end"].tolist() == [1] and r["sel_flip"].tolist() == [0]
    # ... rejected on strand - (its mate lies inside the contig)
    assert 1 not in _select(orc, _one_pair_pool(C, _rc(inside), _rand(rng, 150)))["sel_end"].tolist()
    # ... but a - strand read reaching past the end is kept, and orients the pair (mate 0 on -: flip 1)
    past = _rc(C[500:] + tail[:50])
    r = _select(orc, _one_pair_pool(C, past, _rand(rng, 150)))
    assert r["sel_end"].tolist() == [1] and r["sel_flip"].tolist() == [1]
    # LEFT end (mirror): - strand inside the left window kept; + strand inside rejected
    inl = C[10:140]
    assert 0 in _select(orc, _one_pair_pool(C, _rc(inl), _rand(rng, 150)))["sel_end"].tolist()
    assert 0 not in _select(orc, _one_pair_pool(C, inl, _rand(rng, 150)))["sel_end"].tolist()


def test_select_first_alignment_decides(orc):
    """S4: mate 0 (strand +) and mate 1 (strand -, reaching past the end) both align to the RIGHT end;
    mate 0's alignment comes first, so the pair is written with mate 0 as is and mate 1 rc'd."""
    rng = np.random.default_rng(14)
    C = _rand(rng, 600)
    m0 = C[470:] + _rand(rng, 20)
    m1 = _rc(C[520:] + _rand(rng, 70))
    r = _select(orc, _one_pair_pool(C, m0, m1))
    assert r["sel_end"].tolist() == [1] and r["sel_flip"].tolist() == [0]
    seq = r["read_seq"].tobytes()
    assert seq[:150] == m0 and seq[150:] == _rc(m1)


def test_select_reverse_complement_symmetry(orc):
    """Reverse-complementing every contig swaps its LEFT and RIGHT ends (S1), turns strand + into -
    (S2) and keeps the outward rule (S3): the same pairs are selected for the swapped ends, with their
    reads reverse-complemented and in the same order (orientation decided by the same alignment).
    Exact only when the stride seed positions map onto each other under reversal, (|read| - s) ≡ 0
    (mod t): t = 1 here (with t = 4 and 150 bp reads the seed sets of the two strands differ)."""
    pool = make_pool(seed=21, genome_len=25000, n_contigs=10, coverage=15, err=0.01, n_rate=1e-3, repeats=3)
    a = _select(orc, pool, t=1)

    class P:
        pass
    q = P()
    cs = pool.contig_seq.tobytes()
    q.contig_seq = np.frombuffer(b"".join(_rc(cs[pool.contig_off[c]:pool.contig_off[c + 1]])
                                          for c in range(pool.n_contigs)), np.uint8).copy()
    q.contig_off = pool.contig_off
    q.read_seq, q.read_qual, q.read_off = pool.read_seq, pool.read_qual, pool.read_off
    b = _select(orc, q, t=1)
    swap = lambda e: e ^ 1   # noqa: E731
    ra = sorted((swap(e), p) for e, p in zip(a["sel_end"].tolist(), a["sel_pair"].tolist()))
    rb = sorted(zip(b["sel_end"].tolist(), b["sel_pair"].tolist()))
    assert ra == rb and len(ra) > 50
    # the reads of each selected pair are the reverse complements, mates in the same order
    sa, oa = a["read_seq"].tobytes(), a["read_off"]
    sb, ob = b["read_seq"].tobytes(), b["read_off"]
    ia = {(e, p): n for n, (e, p) in enumerate(zip(a["sel_end"].tolist(), a["sel_pair"].tolist()))}
    for n, (e, p) in enumerate(zip(b["sel_end"].tolist(), b["sel_pair"].tolist())):
        m = ia[(e ^ 1, p)]
        for mate in (0, 1):
            assert sb[ob[2 * n + mate]:ob[2 * n + mate + 1]] == _rc(sa[oa[2 * m + mate]:oa[2 * m + mate + 1]])


# ---------------------------------------------------------------------------------------------- GPU

def _gpu_select(pool, **kw):
    from paper_conf_sc_awanhedbdoy21_b200 import LocalAssembler
    la = LocalAssembler(0)
    rec, db = la.select_reads(pool, **dict(GPU_SP, **kw))
    return la, rec, db


def _check_same(orc_r, rec, host):
    for f in ("sel_end", "sel_pair", "sel_flip"):
        assert np.array_equal(rec[f], orc_r[f]), f
    for f in ("end_read_off", "read_off", "read_seq", "read_qual"):
        assert np.array_equal(host[f], orc_r[f]), f


@pytest.mark.gpu
@pytest.mark.parametrize("kind", ["error_free", "errors_repeats_N", "short_contigs"])
def test_gpu_select_matches_oracle(orc, kind):
    if kind == "error_free":
        pool = make_pool(seed=7, genome_len=30000, n_contigs=14, coverage=12, err=0.0, n_rate=0.0, unique_k=16)
    elif kind == "errors_repeats_N":
        pool = make_pool(seed=31, genome_len=80000, n_contigs=50, coverage=25, err=0.015, n_rate=2e-3, repeats=6)
    else:
        pool = make_pool(seed=32, genome_len=20000, n_contigs=25, contig_len=(10, 300), coverage=20)
    r = _select(orc, pool)
    la, rec, db = _gpu_select(pool)
    try:
        _check_same(r, rec, db.host())
    finally:
        la.close()
    assert kind == "short_contigs" or rec["sel_end"].size > 100


@pytest.mark.gpu
def test_gpu_select_parameters_and_device_input(orc):
    import torch
    pool = make_pool(seed=33, genome_len=40000, n_contigs=20, coverage=20, err=0.02, n_rate=1e-3, repeats=4)
    for kw in (dict(w=100, s=12, t=1, o=12, mm_pct=0), dict(w=300, s=31, t=7, o=40, mm_pct=10)):
        r = _select(orc, pool, **kw)
        gkw = dict(window=kw["w"], seed_len=kw["s"], seed_stride=kw["t"], min_overlap=kw["o"], max_mism_pct=kw["mm_pct"])
        la, rec, db = _gpu_select(pool, **gkw)
        _check_same(r, rec, db.host())
        la.close()
    # device-memory pool (torch CUDA tensors)

    class D:
        pass
    d = D()
    for f in ("contig_seq", "contig_off", "read_seq", "read_qual", "read_off"):
        setattr(d, f, torch.from_numpy(getattr(pool, f)).cuda())
    r = _select(orc, pool)
    la, rec, db = _gpu_select(d)
    _check_same(r, rec, db.host())
    la.close()


@pytest.mark.gpu
def test_gpu_select_degenerate_and_invalid():
    from paper_conf_sc_awanhedbdoy21_b200 import LocalAssembler
    from paper_conf_sc_awanhedbdoy21_b200._lib import LocAssmError

    class P:
        pass
    p = P()
    p.contig_seq = np.frombuffer(b"ACGT" * 50, np.uint8).copy()
    p.contig_off = np.array([0, 200], np.int64)
    p.read_seq = np.zeros(0, np.uint8)
    p.read_qual = np.zeros(0, np.uint8)
    p.read_off = np.zeros(1, np.int64)
    with LocalAssembler(0) as la:
        rec, db = la.select_reads(p)
        assert rec["sel_end"].size == 0
        assert np.array_equal(db.host()["end_read_off"], np.zeros(3, np.int64))
        p.contig_off = np.array([0, 250], np.int64)[::-1].copy()
        with pytest.raises(LocAssmError):
            la.select_reads(p)
        p.contig_off = np.array([0, 200], np.int64)
        with pytest.raises(LocAssmError):
            la.select_reads(p, seed_len=40)


@pytest.mark.gpu
def test_gpu_select_then_extend_matches_oracle(orc):
    """N4 -> local assembly on the device: la_select_reads' batch goes straight into la_load_batch
    (LA_MEM_DEVICE) and la_extend; the oracle extends the oracle's selection of the same pool."""
    from gen import Batch, Params
    from paper_conf_sc_awanhedbdoy21_b200 import LocalAssembler
    pool = make_pool(seed=34, genome_len=120000, n_contigs=60, coverage=30, err=0.01, n_rate=1e-4, repeats=4)
    r = _select(orc, pool)
    qual = r["read_qual"].copy()
    b = Batch(pool.contig_seq, pool.contig_off, r["read_seq"], qual, r["read_off"], r["end_read_off"])
    ref = orc.extend(b, Params())
    with LocalAssembler(0) as la:
        rec, db = la.select_reads(pool, **GPU_SP)
        la.load_device_batch(db, Params())
        res = la.extend()
    assert res.ext_list() == ref["ext"]
    for f in ("term", "k_used", "n_attempts"):
        assert np.array_equal(getattr(res, f), ref[f]), f
    assert sum(len(x) for x in ref["ext"]) > 1000
