"""Batch container and parameter set shared (as plain data) by the oracle and the CUDA path.

This module holds NO arithmetic of the method: it only stores arrays in the layout of the
C ABI (include/locassm.h, `la_batch`) and converts to/from Python strings for tests.

Layout (paper P:L396-402 — per contig, left and right candidate reads):
  contig_seq  uint8[sum |C|]      ASCII uppercase ACGTN, contigs back to back
  contig_off  int64[n_contigs+1]
  read_seq    uint8[sum |r|]      ASCII ACGTN, every read in its end's contig-forward orientation
  read_qual   uint8[sum |r|]      Phred+qual_offset characters
  read_off    int64[n_reads+1]
  end_read_off int64[2*n_contigs+1]  end 2c = LEFT of contig c, 2c+1 = RIGHT; end e owns reads
                                     end_read_off[e] .. end_read_off[e+1]-1
"""
from __future__ import annotations

import dataclasses
from dataclasses import dataclass, field

import numpy as np


@dataclass
class Params:
    """The `la_params` knobs; defaults per DESIGN.md §3 readings #2, #3, #7, #9."""
    k_start: int = 33
    k_min: int = 21
    k_max: int = 99
    k_shift: int = 8
    max_walk_len: int = 300      # Alg 2 line 5, "up to 300 steps"
    qual_offset: int = 33
    q_lo: int = 10
    q_hi: int = 20
    min_votes: int = 2
    min_frac_pct: int = 20

    def replace(self, **kw) -> "Params":
        return dataclasses.replace(self, **kw)

    def as_tuple(self):
        return (self.k_start, self.k_min, self.k_max, self.k_shift, self.max_walk_len,
                self.qual_offset, self.q_lo, self.q_hi, self.min_votes, self.min_frac_pct)


@dataclass
class Batch:
    contig_seq: np.ndarray
    contig_off: np.ndarray
    read_seq: np.ndarray
    read_qual: np.ndarray
    read_off: np.ndarray
    end_read_off: np.ndarray
    meta: dict = field(default_factory=dict)

    @property
    def n_contigs(self) -> int:
        return int(self.contig_off.shape[0] - 1)

    @property
    def n_ends(self) -> int:
        return 2 * self.n_contigs

    @property
    def n_reads(self) -> int:
        return int(self.read_off.shape[0] - 1)

    def reads_per_end(self) -> np.ndarray:
        return np.diff(self.end_read_off)

    def nbytes(self) -> int:
        return sum(int(a.nbytes) for a in (self.contig_seq, self.contig_off, self.read_seq,
                                           self.read_qual, self.read_off, self.end_read_off))

    # ---- string helpers (tests) -------------------------------------------------------------
    def contig(self, c: int) -> str:
        return self.contig_seq[self.contig_off[c]:self.contig_off[c + 1]].tobytes().decode()

    def end_reads(self, e: int):
        out = []
        for r in range(int(self.end_read_off[e]), int(self.end_read_off[e + 1])):
            a, b = int(self.read_off[r]), int(self.read_off[r + 1])
            out.append((self.read_seq[a:b].tobytes().decode(), self.read_qual[a:b].tobytes().decode()))
        return out

    @staticmethod
    def from_lists(contigs, end_reads, meta=None) -> "Batch":
        """contigs: list[str]; end_reads: list (len 2*len(contigs)) of list[(seq, qual)]."""
        assert len(end_reads) == 2 * len(contigs)
        cs = "".join(contigs).encode()
        coff = np.zeros(len(contigs) + 1, np.int64)
        coff[1:] = np.cumsum([len(c) for c in contigs])
        seqs, quals, lens, eoff = [], [], [], [0]
        for rs in end_reads:
            for s, q in rs:
                assert len(s) == len(q)
                seqs.append(s)
                quals.append(q)
                lens.append(len(s))
            eoff.append(len(lens))
        roff = np.zeros(len(lens) + 1, np.int64)
        roff[1:] = np.cumsum(lens) if lens else []
        return Batch(np.frombuffer(cs, np.uint8).copy() if cs else np.zeros(0, np.uint8), coff,
                     np.frombuffer("".join(seqs).encode(), np.uint8).copy() if seqs else np.zeros(0, np.uint8),
                     np.frombuffer("".join(quals).encode(), np.uint8).copy() if quals else np.zeros(0, np.uint8),
                     roff, np.asarray(eoff, np.int64), meta or {})

    def select_contigs(self, contig_ids) -> "Batch":
        """Sub-batch with the given contigs (both ends each), in the given order."""
        contig_ids = np.asarray(contig_ids, np.int64)
        clen = np.diff(self.contig_off)[contig_ids]
        coff = np.zeros(len(contig_ids) + 1, np.int64)
        coff[1:] = np.cumsum(clen)
        cseq = _gather_ranges(self.contig_seq, self.contig_off[contig_ids], clen)
        ends = np.stack([2 * contig_ids, 2 * contig_ids + 1], 1).reshape(-1)
        nre = np.diff(self.end_read_off)[ends]
        eoff = np.zeros(len(ends) + 1, np.int64)
        eoff[1:] = np.cumsum(nre)
        read_ids = _ranges_to_ids(self.end_read_off[ends], nre)
        rlen = np.diff(self.read_off)[read_ids]
        roff = np.zeros(len(read_ids) + 1, np.int64)
        roff[1:] = np.cumsum(rlen)
        rseq = _gather_ranges(self.read_seq, self.read_off[read_ids], rlen)
        rqual = _gather_ranges(self.read_qual, self.read_off[read_ids], rlen)
        return Batch(cseq, coff, rseq, rqual, roff, eoff, dict(self.meta))

    def save(self, path):
        np.savez(path, contig_seq=self.contig_seq, contig_off=self.contig_off, read_seq=self.read_seq,
                 read_qual=self.read_qual, read_off=self.read_off, end_read_off=self.end_read_off)

    @staticmethod
    def load(path) -> "Batch":
        z = np.load(path)
        return Batch(z["contig_seq"], z["contig_off"], z["read_seq"], z["read_qual"], z["read_off"],
                     z["end_read_off"])


def _ranges_to_ids(starts: np.ndarray, lens: np.ndarray) -> np.ndarray:
    """Concatenation of arange(s, s+l) for each (s, l)."""
    starts = np.asarray(starts, np.int64)
    lens = np.asarray(lens, np.int64)
    tot = int(lens.sum())
    if tot == 0:
        return np.zeros(0, np.int64)
    base = np.repeat(starts - np.concatenate([[0], np.cumsum(lens)[:-1]]), lens)
    return base + np.arange(tot, dtype=np.int64)


def _gather_ranges(arr: np.ndarray, starts, lens) -> np.ndarray:
    return arr[_ranges_to_ids(starts, lens)]
