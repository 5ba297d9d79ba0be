"""Pins of the CPU oracle against what the paper and the mathematics fix.

Each construction has a closed-form answer derived from its parameters;
a dropped vote, an off-by-one in the walk bound, a wrong shift direction, a missing reverse
complement or a loop check after (instead of before) the lookup fails at least one of them.
"""
import numpy as np
import pytest

from gen import Params
from gen import cases as C

DEADEND, FORK, LOOP, MAXLEN, NOREADS, SHORT = range(6)
P0 = Params()   # k 33/21/99/8, W=300, V=2, F=20


def run1(orc, batch, P, end=1):
    r = orc.extend(batch, P, ends=[end])
    return r["ext"][0], int(r["term"][0]), int(r["k_used"][0]), int(r["n_attempts"][0])


def downshift_attempts(P):
    return (P.k_start - P.k_min) // P.k_shift + 1


def upshift_attempts(P, kmax_eff):
    return (kmax_eff - P.k_start) // P.k_shift + 1


# ---- P2: tiled error-free genome, closed form --------------------------------------------------
def p2_len(a_hi, l, V, e):
    """Votes for the (k+1)-window at p: #{a: p+k+1-l <= a <= min(p, a_hi)} -> the last extended
    base is a_hi + l - V, so the walk from e has a_hi + l - V + 1 - e bases (any k)."""
    return a_hi + l - V + 1 - e


@pytest.mark.parametrize("seed,a_hi,e", [(1, 600, 500), (2, 560, 470), (3, 620, 520)])
def test_p2_tiled_genome(orc, seed, a_hi, e):
    rng = np.random.default_rng(seed)
    G = C.unique_genome(rng, 800)
    l = 150
    reads = C.tile(G, 200, a_hi, l)
    batch = C.single_end(G[e - 200:e], reads)
    n = p2_len(a_hi, l, P0.min_votes, e)
    assert n < P0.max_walk_len
    w, t, k, a = run1(orc, batch, P0)
    assert (w, t, k, a) == (G[e:e + n], DEADEND, P0.k_start, downshift_attempts(P0))


def test_p2_worked_example(orc):
    """SURVEY §8(c) P2 worked check: l=10, V=2, a_hi=20, e=15 -> 14 bases G[15..28]."""
    rng = np.random.default_rng(7)
    while True:
        G = C.random_seq(rng, 30)
        if C.kmers_unique(G, 5):
            break
    P = Params(k_start=5, k_min=5, k_max=5, k_shift=1)
    batch = C.single_end(G[:15], C.tile(G, 0, 20, 10))
    w, t, k, a = run1(orc, batch, P)
    assert (w, t, k, a) == (G[15:29], DEADEND, 5, 1)


@pytest.mark.parametrize("V", [2, 3, 5])
def test_p2_vote_threshold(orc, V):
    rng = np.random.default_rng(11)
    G = C.unique_genome(rng, 800)
    P = P0.replace(min_votes=V)
    batch = C.single_end(G[300:500], C.tile(G, 200, 600, 150))
    w, t, k, a = run1(orc, batch, P)
    assert w == G[500:500 + p2_len(600, 150, V, 500)] and t == DEADEND


def test_p2_low_quality_fallback(orc):
    """Reads with Q15 (q_lo <= q < q_hi): no high-quality votes, the low-quality tier decides —
    same walk.  Reads with Q5 (< q_lo): no votes at all -> empty DEADEND walk."""
    rng = np.random.default_rng(12)
    G = C.unique_genome(rng, 800)
    for qc, n in ((chr(33 + 15), p2_len(600, 150, 2, 500)), (chr(33 + 5), 0)):
        batch = C.single_end(G[300:500], C.tile(G, 200, 600, 150, qchar=qc))
        w, t, k, a = run1(orc, batch, P0)
        assert (w, t) == (G[500:500 + n], DEADEND)


# ---- P3: constructed fork, P4: short repeat resolved by upshift ---------------------------------
def two_loci(rng, r_len, y_len=300, x_len=400):
    while True:
        X1, X2 = C.random_seq(rng, x_len), C.random_seq(rng, x_len)
        R = C.random_seq(rng, r_len)
        Y1, Y2 = C.random_seq(rng, y_len), C.random_seq(rng, y_len)
        if Y1[0] == Y2[0] or X1[-1] == X2[-1]:   # the shared segment is exactly R
            continue
        L1, L2 = X1 + R + Y1, X2 + R + Y2
        if C.kmers_unique(L1, 21) and C.kmers_unique(X2 + "N" + Y2 + "N" + X1 + "N" + Y1, 21) and \
                C.kmers_unique(L2, 21):
            return L1, L2, x_len, x_len + r_len


def test_p3_fork(orc):
    rng = np.random.default_rng(3)
    L1, L2, r0, r1 = two_loci(rng, 120)
    reads = C.tile(L1, 0, len(L1) - 150, 150) + C.tile(L2, 0, len(L2) - 150, 150)
    e = 350
    batch = C.single_end(L1[100:e], reads)
    w, t, k, a = run1(orc, batch, P0)
    assert (w, t, k, a) == (L1[e:r1], FORK, P0.k_start, upshift_attempts(P0, P0.k_max))


def test_p4_repeat_resolved_by_upshift(orc):
    rng = np.random.default_rng(4)
    L1, L2, r0, r1 = two_loci(rng, 40, y_len=100)      # k_start <= |R| < k_start + shift
    reads = C.tile(L1, 0, len(L1) - 150, 150) + C.tile(L2, 0, len(L2) - 150, 150)
    e = 350
    batch = C.single_end(L1[100:e], reads)
    n = p2_len(len(L1) - 150, 150, 2, e)
    w, t, k, a = run1(orc, batch, P0)
    assert (w, t, k, a) == (L1[e:e + n], DEADEND, P0.k_start + P0.k_shift, 2)
    # the first attempt alone (no upshift allowed) stops with a fork at the end of R
    w1, t1, k1, a1 = run1(orc, batch, P0.replace(k_max=P0.k_start))
    assert (w1, t1, a1) == (L1[e:r1], FORK, 1)


# ---- P5: tandem loop ---------------------------------------------------------------------------
def test_p5_tandem_loop(orc):
    rng = np.random.default_rng(5)
    u = 110
    while True:
        U, FL, FR = C.random_seq(rng, u), C.random_seq(rng, 200), C.random_seq(rng, 200)
        reg = FL + U * 7 + FR
        if C.kmers_unique(FL + U + FR, 21):
            break
    e = 200 + 3 * u + 50
    batch = C.single_end(reg[300:e], C.tile(reg, 0, len(reg) - 150, 150))
    w, t, k, a = run1(orc, batch, P0)
    assert (w, t, k, a) == (reg[e:e + u], LOOP, P0.k_start, upshift_attempts(P0, P0.k_max))
    # reading #8 alternative (LOOP accepted): same walk, one attempt
    r = orc.extend(batch, P0, ends=[1], loop_accepts=True)
    assert (r["ext"][0], int(r["term"][0]), int(r["n_attempts"][0])) == (reg[e:e + u], LOOP, 1)


# ---- P6: MAXLEN ----------------------------------------------------------------------------------
def test_p6_maxlen(orc):
    rng = np.random.default_rng(6)
    G = C.unique_genome(rng, 1200)
    batch = C.single_end(G[300:500], C.tile(G, 200, 1000, 150))
    assert p2_len(1000, 150, 2, 500) > P0.max_walk_len
    assert run1(orc, batch, P0) == (G[500:800], MAXLEN, P0.k_start, 1)
    assert run1(orc, batch, P0.replace(max_walk_len=0)) == ("", MAXLEN, P0.k_start, 1)
    assert run1(orc, batch, P0.replace(max_walk_len=17)) == (G[500:517], MAXLEN, P0.k_start, 1)


# ---- P7: N handling --------------------------------------------------------------------------
@pytest.mark.parametrize("d,k_used,walks", [(27, 25, True), (10, 33, False), (40, 33, True)])
def test_p7_n_in_contig(orc, d, k_used, walks):
    rng = np.random.default_rng(8)
    G = C.unique_genome(rng, 800)
    contig = list(G[300:500])
    contig[len(contig) - 1 - d] = "N"
    batch = C.single_end("".join(contig), C.tile(G, 200, 600, 150))
    n = p2_len(600, 150, 2, 500) if walks else 0
    assert run1(orc, batch, P0) == (G[500:500 + n], DEADEND, k_used, downshift_attempts(P0))


def test_p7_n_in_reads(orc):
    """An N at read position j removes the k-mers covering j and the vote of the k-mer ending at
    j-1; with single coverage at the frontier the walk stops exactly there."""
    rng = np.random.default_rng(9)
    G = C.unique_genome(rng, 800)
    reads = C.tile(G, 200, 600, 150)
    # kill every occurrence of base 560 in the reads: votes for G[560] vanish
    reads = [(s[:560 - a] + "N" + s[561 - a:], q) if 0 <= 560 - a < 150 else (s, q)
             for (s, q), a in zip(reads, range(200, 601))]
    batch = C.single_end(G[300:500], reads)
    assert run1(orc, batch, P0) == (G[500:560], DEADEND, P0.k_start, downshift_attempts(P0))


# ---- P8: special ends ----------------------------------------------------------------------
def test_p8_special_ends(orc):
    rng = np.random.default_rng(10)
    G = C.unique_genome(rng, 800)
    reads = C.tile(G, 200, 600, 150)
    assert run1(orc, C.single_end(G[300:500], []), P0) == ("", NOREADS, 0, 0)
    assert run1(orc, C.single_end(G[468:500], reads), P0) == ("", SHORT, 0, 0)      # |C|=32 < 33
    short = [(s[:21], q[:21]) for s, q in reads]
    assert run1(orc, C.single_end(G[300:500], short), P0) == ("", DEADEND, 33, downshift_attempts(P0))
    # k_max capped by the contig length: |C| = 50 -> kmax_eff = 50, fork chain 33, 41, 49
    L1, L2, r0, r1 = two_loci(np.random.default_rng(3), 120)
    rr = C.tile(L1, 0, len(L1) - 150, 150) + C.tile(L2, 0, len(L2) - 150, 150)
    w, t, k, a = run1(orc, C.single_end(L1[300:350], rr), P0)
    assert (w, t, k, a) == (L1[350:r1], FORK, 33, upshift_attempts(P0, 50))


# ---- P12: vote rule truth table -----------------------------------------------------------
@pytest.mark.parametrize("lo,hi,expect", [
    ((5, 0, 0, 0), (5, 0, 0, 0), 0),
    ((5, 5, 0, 0), (5, 5, 0, 0), -1),
    ((1, 0, 0, 0), (0, 0, 0, 0), -2),
    ((9, 1, 0, 0), (9, 1, 0, 0), 0),
    ((10, 3, 0, 0), (0, 0, 0, 0), -1),     # 100*3 = 300 >= 20*13 = 260 -> both qualify
    ((10, 2, 0, 0), (0, 0, 0, 0), 0),      # 200 < 240
    ((0, 0, 7, 0), (0, 0, 1, 0), 2),       # hi has no qualifying base -> lo decides
    ((3, 0, 0, 9), (3, 0, 0, 1), 0),       # hi decides: A (3 >= V, 300 >= 80); T has 1 < V
    ((2, 2, 2, 2), (2, 2, 2, 2), -1),      # four-way tie
    ((0, 0, 0, 0), (0, 0, 0, 0), -2),      # present k-mer without votes = dead end
])
def test_p12_vote_rule(orc, lo, hi, expect):
    assert orc.ext_rule(lo, hi, P0) == expect


# ---- P9 / P10: invariances -----------------------------------------------------------------
def test_p9_rc_invariance_cases(orc):
    rng = np.random.default_rng(3)
    L1, L2, r0, r1 = two_loci(rng, 40, y_len=100)
    reads = C.tile(L1, 0, len(L1) - 150, 150) + C.tile(L2, 0, len(L2) - 150, 150)
    left = C.tile(L1, 0, 200, 150, qchar="5")
    batch = C.single_end(L1[100:350], reads, left)
    tw = C.twin(batch)
    r, rt = orc.extend(batch, P0), orc.extend(tw, P0)
    assert rt["ext"][0] == C.rc(r["ext"][1]) and rt["ext"][1] == C.rc(r["ext"][0])
    for f in ("term", "k_used", "n_attempts"):
        assert rt[f][0] == r[f][1] and rt[f][1] == r[f][0]


def _assert_twin(r, rt, n_contigs):
    for c in range(n_contigs):
        assert rt["ext"][2 * c] == C.rc(r["ext"][2 * c + 1])
        assert rt["ext"][2 * c + 1] == C.rc(r["ext"][2 * c])
    sw = np.arange(2 * n_contigs) ^ 1
    for f in ("term", "k_used", "n_attempts"):
        assert np.array_equal(rt[f], r[f][sw])


def test_p9_rc_invariance_metagenome(orc):
    from conftest import cached_batch
    b = cached_batch("C2", scale=0.03).select_contigs(np.arange(120))
    _assert_twin(orc.extend(b, P0), orc.extend(C.twin(b), P0), b.n_contigs)


def test_p10_permutation_invariance(orc):
    from conftest import cached_batch
    b = cached_batch("C2", scale=0.03).select_contigs(np.arange(120))
    r = orc.extend(b, P0)
    bp, perm = C.permuted(b, 99)
    rp = orc.extend(bp, P0)
    idx = np.stack([2 * perm, 2 * perm + 1], 1).reshape(-1)
    assert [r["ext"][i] for i in idx] == rp["ext"]
    for f in ("term", "k_used", "n_attempts", "inserts", "walk_steps"):
        assert np.array_equal(r[f][idx], rp[f])


# ---- P11: brute force ------------------------------------------------------------------------
def _compare_brute(orc, batch, P, ends=None):
    import brute
    r = orc.extend(batch, P, ends=ends)
    b = brute.extend(batch, P, ends=r["ends"])
    assert r["ext"] == b["ext"]
    for f in ("term", "k_used", "n_attempts"):
        assert r[f].tolist() == b[f]
    return r


def test_p11_brute_c1(orc):
    from conftest import cached_batch
    b = cached_batch("C1")
    r = _compare_brute(orc, b, Params(k_start=21, k_min=21, k_max=21))
    assert (r["term"] == DEADEND).all()
    # C1 truth: error-free reads from one genome -> every extension is the true genome sequence
    G, cs, ce = b.meta["genome"], b.meta["contig_start"], b.meta["contig_end"]
    for c in range(b.n_contigs):
        L, R = r["ext"][2 * c], r["ext"][2 * c + 1]
        assert G[cs[c] - len(L):cs[c]] == L and G[ce[c]:ce[c] + len(R)] == R


def test_p11_brute_c2_slice(orc):
    from conftest import cached_batch
    b = cached_batch("C2", scale=0.03)
    ends = np.random.default_rng(0).choice(b.n_ends, min(500, b.n_ends), replace=False)
    r = _compare_brute(orc, b, Params(), ends=ends)
    # the slice must exercise the schedule: forks, dead-ends and multi-attempt ends
    t = r["term"]
    assert (t == DEADEND).any() and (r["n_attempts"] > 1).any()


def test_p11_brute_small_params(orc):
    """Same comparison under a different schedule / thresholds (guards hard-coded defaults)."""
    from conftest import cached_batch
    b = cached_batch("C2", scale=0.03)
    ends = np.random.default_rng(1).choice(b.n_ends, 150, replace=False)
    P = Params(k_start=25, k_min=17, k_max=45, k_shift=4, max_walk_len=120, q_lo=5, q_hi=30,
               min_votes=3, min_frac_pct=30)
    _compare_brute(orc, b, P, ends=ends)


def test_p1_load_factor_bound():
    """P1: table size l*r against (l-k+1)*r k-mers -> load factor (l-k+1)/l,
    worst case (300-21+1)/300 = 0.9333 ('about 0.93')."""
    lf = lambda l, k: (l - k + 1) / l
    assert abs(lf(300, 21) - 0.9333) < 1e-4
    assert round(lf(300, 21), 2) == 0.93


def test_oracle_counters(orc):
    """inserts = sum over attempts and reads of max(0, len-k) (the work unit)."""
    rng = np.random.default_rng(1)
    G = C.unique_genome(rng, 800)
    reads = C.tile(G, 200, 600, 150)
    batch = C.single_end(G[300:500], reads)
    r = orc.extend(batch, P0, ends=[1])
    assert int(r["inserts"][0]) == len(reads) * ((150 - 33) + (150 - 25))
    n = p2_len(600, 150, 2, 500)
    assert int(r["walk_steps"][0]) == 2 * (n + 1)


# ---- N1: append extensions to contigs (Fig 4) ---------------------------------
def test_append_extensions_reassembles_genome(orc):
    """An error-free contig G[500:700] with reads tiling both flanks: once both extensions are
    appended, the extended contig is the contiguous genome window G[500-nl : 700+nr] — a left
    extension prepended in the wrong orientation, or the ends swapped, breaks the window. The right
    length is the P2 closed form."""
    rng = np.random.default_rng(11)
    G = C.unique_genome(rng, 1200)
    l = 150
    batch = C.single_end(G[500:700], C.tile(G, 560, 800, l), left_reads=C.tile(G, 300, 560, l))
    r = orc.extend(batch, P0)
    nl, nr = len(r["ext"][0]), len(r["ext"][1])
    assert nr == p2_len(800, l, P0.min_votes, 700)
    assert nl > 100
    (out,) = orc.append_extensions([G[500:700]], r["ext"])
    assert len(out) == nl + 200 + nr
    assert out == G[500 - nl:700 + nr]


def test_append_extensions_small():
    import oracle
    assert oracle.append_extensions(["ACGT", "", "GG"], ["TT", "CA", "", "", "A", ""]) == [
        "TTACGTCA", "", "AGG"]
    assert oracle.append_extensions([], []) == []
