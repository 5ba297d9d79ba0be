"""Constructed inputs with known answers (the pins of DESIGN.md §5 / SURVEY.md §8(c) P2-P9).

Inputs only: genomes, tilings of reads, contigs.  The expected results are derived in the tests
from the construction parameters (closed forms), never computed here.
"""
from __future__ import annotations

import numpy as np

from .batch import Batch

_A = "ACGT"
_COMP = str.maketrans("ACGTN", "TGCAN")


def rc(s: str) -> str:
    return s.translate(_COMP)[::-1]


def random_seq(rng, n: int) -> str:
    return "".join(_A[i] for i in rng.integers(0, 4, n))


def kmers_unique(s: str, k: int) -> bool:
    seen = set()
    for i in range(len(s) - k + 1):
        x = s[i:i + k]
        if x in seen:
            return False
        seen.add(x)
    return True


def unique_genome(rng, n: int, k: int = 21, also=()) -> str:
    """Random genome whose k-mers are all distinct (and distinct from those of `also`)."""
    while True:
        g = random_seq(rng, n)
        if kmers_unique(g + "".join("N" + x for x in also), k):
            return g


def tile(g: str, a_lo: int, a_hi: int, l: int, qchar: str = "I", step: int = 1):
    """Error-free forward reads of length l starting at every a in [a_lo, a_hi] (step)."""
    return [(g[a:a + l], qchar * l) for a in range(a_lo, a_hi + 1, step) if a + l <= len(g) and a >= 0]


def single_end(contig: str, right_reads, left_reads=()) -> Batch:
    """One contig; end 0 = LEFT (left_reads), end 1 = RIGHT (right_reads)."""
    return Batch.from_lists([contig], [list(left_reads), list(right_reads)])


def twin(batch: Batch) -> Batch:
    """Reverse-strand twin (pin P9): contig' = rc(C), left' = rc(right reads), right' = rc(left
    reads), qualities reversed."""
    contigs, ends = [], []
    for c in range(batch.n_contigs):
        contigs.append(rc(batch.contig(c)))
        left = batch.end_reads(2 * c)
        right = batch.end_reads(2 * c + 1)
        ends.append([(rc(s), q[::-1]) for s, q in right])
        ends.append([(rc(s), q[::-1]) for s, q in left])
    return Batch.from_lists(contigs, ends)


def permuted(batch: Batch, seed: int):
    """Pin P10: shuffle reads within each end and the contig order.  Returns (batch', perm) with
    contig i of batch' = contig perm[i] of batch."""
    rng = np.random.default_rng(seed)
    perm = rng.permutation(batch.n_contigs)
    contigs, ends = [], []
    for c in perm:
        contigs.append(batch.contig(int(c)))
        for e in (2 * int(c), 2 * int(c) + 1):
            rs = batch.end_reads(e)
            o = rng.permutation(len(rs))
            ends.append([rs[i] for i in o])
    return Batch.from_lists(contigs, ends), perm
