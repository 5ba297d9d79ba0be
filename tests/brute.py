"""Brute-force local assembly (pin P11) — no hash tables.

For every k-mer the walk looks up, scan all reads of the end (str.find over the reads joined by a
separator) and recount the votes from scratch.  It restates the paper's Alg 1 + Alg 2 + shift rule
 and the readings of DESIGN.md §3 with different data structures from
oracle/oracle.cpp; it shares no code with it.
"""
from __future__ import annotations

DEADEND, FORK, LOOP, MAXLEN, NOREADS, SHORT = range(6)
_IDX = {"A": 0, "C": 1, "G": 2, "T": 3}
_COMP = str.maketrans("ACGTN", "TGCAN")


def rc(s):
    return s.translate(_COMP)[::-1]


def _decide(lo, hi, P):
    for tier in (hi, lo):
        tot = sum(tier)
        ok = [b for b in range(4) if tier[b] >= P.min_votes and 100 * tier[b] >= P.min_frac_pct * tot]
        if len(ok) == 1:
            return "ACGT"[ok[0]]
        if len(ok) > 1:
            return FORK
    return DEADEND


class _Reads:
    def __init__(self, reads, qual_offset):
        self.S = "#".join(s for s, _ in reads)
        self.Q = "#".join(q for _, q in reads)
        self.off = qual_offset

    def lookup(self, K, P):
        """Extension for K, or DEADEND when K never occurs (or contains N)."""
        if "N" in K:
            return DEADEND
        lo, hi = [0] * 4, [0] * 4
        S, Q = self.S, self.Q
        i = S.find(K)
        if i < 0:
            return DEADEND
        while i >= 0:
            j = i + len(K)
            if j < len(S) and S[j] in _IDX:
                b = _IDX[S[j]]
                q = ord(Q[j]) - self.off
                if q >= P.q_lo:
                    lo[b] += 1
                if q >= P.q_hi:
                    hi[b] += 1
            i = S.find(K, i + 1)
        return _decide(lo, hi, P)


def _walk(C, reads, k, P):
    K = C[len(C) - k:]
    w = []
    seen = set()
    for _ in range(P.max_walk_len):
        if K in seen:
            return "".join(w), LOOP
        seen.add(K)
        x = reads.lookup(K, P)
        if x == DEADEND or x == FORK:
            return "".join(w), x
        w.append(x)
        K = K[1:] + x
    return "".join(w), MAXLEN


def extend_end(C, reads, P):
    if not reads:
        return "", NOREADS, 0, 0
    kmax = min(P.k_max, len(C))
    if P.k_start > kmax:
        return "", SHORT, 0, 0
    R = _Reads(reads, P.qual_offset)
    k, direction, attempts, best = P.k_start, 0, 0, None
    while True:
        w, t = _walk(C, R, k, P)
        attempts += 1
        if best is None or len(w) > len(best[0]):
            best = (w, t, k)
        if t == MAXLEN:
            break
        if t == DEADEND:
            if direction > 0:
                break
            direction = -1
        else:
            if direction < 0:
                break
            direction = 1
        k += direction * P.k_shift
        if k < P.k_min or k > kmax:
            break
    return best[0], best[1], best[2], attempts


def extend(batch, P, ends=None):
    """Same result fields as oracle.extend (ext, term, k_used, n_attempts), as Python lists."""
    if ends is None:
        ends = range(batch.n_ends)
    out = dict(ext=[], term=[], k_used=[], n_attempts=[])
    for e in ends:
        e = int(e)
        C = batch.contig(e // 2)
        reads = batch.end_reads(e)
        if e % 2 == 1:
            w, t, k, a = extend_end(C, reads, P)
        else:
            w, t, k, a = extend_end(rc(C), [(rc(s), q[::-1]) for s, q in reads], P)
            w = rc(w)
        out["ext"].append(w)
        out["term"].append(t)
        out["k_used"].append(k)
        out["n_attempts"].append(a)
    return out
