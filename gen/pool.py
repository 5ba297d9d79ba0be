"""Seeded read pools for NEXT N4 (candidate-read selection): contigs plus a pool of
FR read pairs as sequenced, with the truth coordinates of every pair.  Holds no arithmetic of the
method (no alignment, no selection): it only synthesises genomes, contigs and reads.

Pair i = reads 2i (mate 0) and 2i+1 (mate 1) from a fragment [f, f+ins) of a genome; strand z = 0:
mate 0 = G[f, f+L) forward, mate 1 = rc(G[f+ins-L, f+ins)); z = 1: the two swapped (mate 0 is the
reverse read).  Substitutions, N calls and Phred qualities as the C2 recipe (gen/_synth.c); the
qualities of a reverse read are reversed with it (they follow the read as sequenced).
"""
from __future__ import annotations

from dataclasses import dataclass, field

import numpy as np

from .synth import ASCII, RL, _c, _kmers_unique

_COMP = bytes.maketrans(b"ACGTN", b"TGCAN")


@dataclass
class Pool:
    contig_seq: np.ndarray          # uint8 ASCII, contigs back to back
    contig_off: np.ndarray          # int64[n_contigs+1]
    read_seq: np.ndarray            # uint8 ASCII, 2*n_pairs reads as sequenced
    read_qual: np.ndarray
    read_off: np.ndarray            # int64[2*n_pairs+1]
    truth: dict = field(default_factory=dict)   # genome, contig_start/end, frag_start, ins, strand

    @property
    def n_contigs(self) -> int:
        return int(self.contig_off.shape[0] - 1)

    @property
    def n_pairs(self) -> int:
        return int((self.read_off.shape[0] - 1) // 2)


def _rc_rows(seq: np.ndarray) -> np.ndarray:
    """Reverse complement of each row of an (n, L) ASCII array."""
    return np.frombuffer(seq[:, ::-1].tobytes().translate(_COMP), np.uint8).reshape(seq.shape)


def make_pool(seed: int = 20211119, genome_len: int = 60_000, n_contigs: int = 40, contig_len=(400, 1200),
              coverage: float = 20.0, err: float = 0.01, n_rate: float = 1e-4, ins_mu: float = 350.0,
              ins_sd: float = 35.0, repeats: int = 0, unique_k: int = 0) -> Pool:
    """One genome (i.i.d. ACGT), `n_contigs` disjoint contigs cut from it (gaps >= 300 bp between
    them), read pairs at `coverage` over the whole genome.  repeats > 0 copies a 400 bp segment of
    the genome that many times to other places (multi-mapping reads, alignment to several ends).
    unique_k > 0: regenerate the genome until all its unique_k-mers (both strands) are distinct."""
    rng = np.random.default_rng(seed)
    while True:
        g = rng.integers(0, 4, genome_len, dtype=np.uint8)
        if repeats:
            src = int(rng.integers(0, genome_len - 400))
            for _ in range(repeats):
                dst = int(rng.integers(0, genome_len - 400))
                g[dst:dst + 400] = g[src:src + 400]
        if not unique_k:
            break
        both = np.concatenate([g, np.array([4], np.uint8), (3 - g)[::-1]])
        if _kmers_unique(both, unique_k):
            break
    # contigs: disjoint intervals, separated by >= 300 bp
    starts, ends = [], []
    pos = 300
    for _ in range(n_contigs):
        L = int(rng.integers(contig_len[0], contig_len[1] + 1))
        gap = int(rng.integers(300, 900))
        if pos + L + 300 > genome_len:
            break
        starts.append(pos)
        ends.append(pos + L)
        pos += L + gap
    cs = np.asarray(starts, np.int64)
    ce = np.asarray(ends, np.int64)
    cseq = np.concatenate([ASCII[g[a:b]] for a, b in zip(cs, ce)]) if cs.size else np.zeros(0, np.uint8)
    coff = np.zeros(cs.shape[0] + 1, np.int64)
    coff[1:] = np.cumsum(ce - cs)
    # FR pairs
    nf = int(round(coverage * genome_len / (2 * RL)))
    ins = np.clip(np.rint(rng.normal(ins_mu, ins_sd, nf)), 2 * RL - 50, 2 * ins_mu).astype(np.int64)
    f = (rng.random(nf) * (genome_len - ins + 1)).astype(np.int64)
    z = rng.integers(0, 2, nf).astype(np.int64)
    fwd_start = f
    rev_start = f + ins - RL
    starts2 = np.ascontiguousarray(np.stack([fwd_start, rev_start], 1).reshape(-1), np.int64)
    uid = np.arange(2 * nf, dtype=np.int64)
    seq = np.empty((2 * nf, RL), np.uint8)
    qual = np.empty((2 * nf, RL), np.uint8)
    gg = np.ascontiguousarray(g)
    _c().synth_reads(gg.ctypes.data, starts2.ctypes.data, uid.ctypes.data, 2 * nf, RL,
                     int(rng.integers(0, 2 ** 63)), float(err), float(n_rate), seq.ctypes.data, qual.ctypes.data)
    fwd, fq = seq[0::2], qual[0::2]
    rev, rq = _rc_rows(seq[1::2]), qual[1::2][:, ::-1]
    m0 = np.where(z[:, None] == 0, fwd, rev)
    m1 = np.where(z[:, None] == 0, rev, fwd)
    q0 = np.where(z[:, None] == 0, fq, rq)
    q1 = np.where(z[:, None] == 0, rq, fq)
    read_seq = np.ascontiguousarray(np.stack([m0, m1], 1).reshape(-1))
    read_qual = np.ascontiguousarray(np.stack([q0, q1], 1).reshape(-1))
    read_off = np.arange(2 * nf + 1, dtype=np.int64) * RL
    return Pool(cseq, coff, read_seq, read_qual, read_off,
                truth=dict(genome=g, contig_start=cs, contig_end=ce, frag_start=f, ins=ins, strand=z))
