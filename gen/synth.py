"""Seeded synthetic workloads C1-C4 (recipe restated in DESIGN.md §4).

Only input synthesis lives here: genomes, abundances, reads with errors and Phred qualities,
contigs and per-end candidate read sets.  Nothing here computes k-mers, votes or walks — the
method's arithmetic lives only in oracle/ (test infrastructure) and in the CUDA library.

Every generator is a pure function of (config, seed); numpy default_rng(seed), seed default
20211114 + config index.
"""
from __future__ import annotations

import ctypes
import math
import os
import subprocess
from dataclasses import dataclass, field

import numpy as np

from .batch import Batch, _gather_ranges, _ranges_to_ids

ASCII = np.frombuffer(b"ACGTN", np.uint8)
RL = 150                      # read length (150 bp reads)
GEN_VERSION = 2               # bumped when a config's recipe changes (bench.py cache key)

_HERE = os.path.dirname(os.path.abspath(__file__))
_SO = os.path.join(_HERE, "libsynth.so")
_clib = None


def _c():
    """Seeded C helpers (_synth.c): genome and read synthesis, OpenMP, counter-based RNG."""
    global _clib
    if _clib is None:
        src = os.path.join(_HERE, "_synth.c")
        if not os.path.exists(_SO) or os.path.getmtime(_SO) < os.path.getmtime(src):
            subprocess.check_call(["gcc", "-O3", "-fopenmp", "-shared", "-fPIC", "-o", _SO, src])
        lib = ctypes.CDLL(_SO)
        V = ctypes.c_void_p
        lib.synth_genome.argtypes = [V, ctypes.c_int64, ctypes.c_double, ctypes.c_uint64]
        lib.synth_reads.argtypes = [V, V, V, ctypes.c_int64, ctypes.c_int, ctypes.c_uint64, ctypes.c_double,
                                    ctypes.c_double, V, V]
        _clib = lib
    return _clib


def seed_for(cfg_index: int) -> int:
    return 20211114 + cfg_index


# ---------------------------------------------------------------------------------------------
# C1: tiny single-genome check
# ---------------------------------------------------------------------------------------------
def _kmers_unique(g: np.ndarray, k: int) -> bool:
    """True iff all k-mers of the code array g (values 0..3) are distinct (k <= 31)."""
    n = g.shape[0] - k + 1
    codes = np.zeros(n, np.int64)
    for j in range(k):
        codes = (codes << 2) | g[j:j + n].astype(np.int64)
    return np.unique(codes).shape[0] == n


def make_c1(seed: int = seed_for(0), genome_len: int = 50_000, n_reads: int = 20_000,
            n_contigs: int = 200, contig_len: int = 150, gap: int = 100, uniq_k: int = 21) -> Batch:
    """1 genome of i.i.d. uniform ACGT with all 21-mers unique; error-free forward reads, all Q40;
    200 contigs of 150 bp separated by 100 bp gaps.  Right-end reads: reads overlapping
    [e-50, e+100); left-end reads: reads overlapping [s-100, s+50)."""
    rng = np.random.default_rng(seed)
    while True:
        g = rng.integers(0, 4, genome_len, dtype=np.uint8)
        if _kmers_unique(g, uniq_k):
            break
    starts = np.sort(rng.integers(0, genome_len - RL + 1, n_reads))
    period = contig_len + gap
    first = (genome_len - n_contigs * period + gap) // 2
    cs = first + period * np.arange(n_contigs)
    ce = cs + contig_len
    gseq = ASCII[g]
    contigs = [gseq[s:e].tobytes().decode() for s, e in zip(cs, ce)]
    qual = "I" * RL
    end_reads = []
    for s, e in zip(cs, ce):
        for lo, hi in ((s - 100, s + 50), (e - 50, e + 100)):
            sel = starts[(starts < hi) & (starts + RL > lo)]
            end_reads.append([(gseq[a:a + RL].tobytes().decode(), qual) for a in sel])
    b = Batch.from_lists(contigs, end_reads)
    b.meta = dict(config="C1", seed=seed, genome=gseq.tobytes().decode(), contig_start=cs,
                  contig_end=ce, read_starts=starts)
    return b


# ---------------------------------------------------------------------------------------------
# Metagenome simulator (C2, C3, C4)
# ---------------------------------------------------------------------------------------------
@dataclass
class Species:
    length: int
    gc: float
    coverage: float            # read coverage (both mates), x
    cut_rate: float = 0.0      # extra contig breakpoints per bp (strain variants, repeats)
    forced_contigs: int = 0    # if >0: cut covered region into exactly this many contigs


@dataclass
class MetaCfg:
    name: str
    species: list
    n_me_fam: int = 20                 # mobile-element families
    me_len: tuple = (300, 1500)
    me_copies: tuple = (2, 10)
    me_div: tuple = (0.0, 0.02)
    err: float = 0.01                  # uniform substitution rate
    n_rate: float = 1e-4               # N calls (Q2)
    min_depth: int = 3
    min_contig: int = 200
    ins_mu: float = 350.0
    ins_sd: float = 35.0
    overlap_min: int = 20
    meta: dict = field(default_factory=dict)


def _species_genome(rng, sp: Species) -> np.ndarray:
    g = np.empty(sp.length, np.uint8)
    _c().synth_genome(g.ctypes.data, sp.length, float(sp.gc), int(rng.integers(0, 2 ** 63)))
    return g


def _intervals(mask: np.ndarray):
    """Maximal runs of True -> (starts, ends)."""
    d = np.diff(np.concatenate([[0], mask.view(np.int8), [0]]))
    return np.nonzero(d == 1)[0], np.nonzero(d == -1)[0]


def _select_end_fragments(f, ins, ends, sides, cstart, cend, ovl):
    """For each end (position, side, contig extent), return (end_idx, frag_idx) of fragments with a
    mate overlapping the 150 bp at the end (inside the contig) by >= ovl and with the fragment
    reaching past the end.  f sorted ascending."""
    max_ins = int(ins.max()) if ins.size else RL
    out_e, out_f = [], []
    CH = 200_000
    for c0 in range(0, ends.shape[0], CH):
        e = ends[c0:c0 + CH]
        sd = sides[c0:c0 + CH]
        cs = cstart[c0:c0 + CH]
        ce = cend[c0:c0 + CH]
        # window W = [wlo, whi) = the end's last 150 bp, clipped to the contig
        wlo = np.where(sd == 1, np.maximum(e - RL, cs), cs)
        whi = np.where(sd == 1, ce, np.minimum(cs + RL, ce))
        lo = np.searchsorted(f, wlo - max_ins + ovl, "left")
        hi = np.searchsorted(f, whi - ovl, "right")
        n = hi - lo
        fid = _ranges_to_ids(lo, n)
        eid = np.repeat(np.arange(c0, c0 + e.shape[0]), n)
        if fid.size == 0:
            continue
        ff = f[fid]
        ii = ins[fid]
        m1s, m1e = ff, ff + RL
        m2s, m2e = ff + ii - RL, ff + ii
        wl, wh = wlo[eid - c0], whi[eid - c0]
        ov1 = np.minimum(m1e, wh) - np.maximum(m1s, wl)
        ov2 = np.minimum(m2e, wh) - np.maximum(m2s, wl)
        hit = (ov1 >= ovl) | (ov2 >= ovl)
        right = sd[eid - c0] == 1
        past = np.where(right, m2e > e[eid - c0], m1s < e[eid - c0])
        keep = hit & past
        out_e.append(eid[keep])
        out_f.append(fid[keep])
    if not out_e:
        return np.zeros(0, np.int64), np.zeros(0, np.int64)
    return np.concatenate(out_e), np.concatenate(out_f)


def make_metagenome(cfg: MetaCfg, seed: int, max_contigs: int | None = None) -> Batch:
    rng = np.random.default_rng(seed)
    S = len(cfg.species)
    genomes = [_species_genome(rng, sp) for sp in cfg.species]

    # mobile elements: families of random sequence, copies diverged and written (forward) into
    # random species positions; their boundaries cut contigs, and reads of other copies of the
    # family align to ends that reach into a copy (synthetic multi-mapping alignment).
    me_copies = []            # (species, pos, fam, length)
    lens = np.array([sp.length for sp in cfg.species], np.float64)
    for fam in range(cfg.n_me_fam):
        L = int(rng.integers(cfg.me_len[0], cfg.me_len[1] + 1))
        seq = rng.integers(0, 4, L, dtype=np.uint8)
        for _ in range(int(rng.integers(cfg.me_copies[0], cfg.me_copies[1] + 1))):
            s = int(rng.choice(S, p=lens / lens.sum()))
            if cfg.species[s].length < L + 2000:
                continue
            pos = int(rng.integers(500, cfg.species[s].length - L - 500))
            div = rng.uniform(*cfg.me_div)
            cp = seq.copy()
            mut = rng.random(L) < div
            cp[mut] = (cp[mut] + rng.integers(1, 4, int(mut.sum()))) % 4
            genomes[s][pos:pos + L] = cp
            me_copies.append((s, pos, fam, L))

    # fragments (read pairs) per species
    frags = []
    for s, sp in enumerate(cfg.species):
        nf = int(round(sp.coverage * sp.length / (2 * RL)))
        ins = np.clip(np.rint(rng.normal(cfg.ins_mu, cfg.ins_sd, nf)), 2 * RL - 50, 2 * cfg.ins_mu).astype(np.int64)
        f = (rng.random(nf) * (sp.length - ins + 1)).astype(np.int64)
        o = np.argsort(f, kind="stable")
        frags.append((f[o], ins[o]))

    # contigs: maximal runs of depth >= min_depth, cut at ME boundaries and random breakpoints
    contig_sp, contig_s, contig_e = [], [], []
    for s, sp in enumerate(cfg.species):
        f, ins = frags[s]
        d = np.zeros(sp.length + 1, np.int64)
        for a, b in ((f, f + RL), (f + ins - RL, f + ins)):
            d += np.bincount(a, minlength=sp.length + 1)
            d -= np.bincount(b, minlength=sp.length + 1)
        depth = np.cumsum(d[:-1])
        cov = depth >= cfg.min_depth
        cuts = [p for (sx, p, _, L) in me_copies if sx == s for p in (p, p + L)]
        if sp.forced_contigs:
            st, en = _intervals(cov)
            if st.size:
                a, b = int(st[0]), int(en[-1])
                cuts += list(np.linspace(a, b, sp.forced_contigs + 1)[1:-1].astype(np.int64))
        elif sp.cut_rate > 0:
            nc = rng.poisson(sp.cut_rate * sp.length)
            cuts += list(rng.integers(0, sp.length, nc))
        cuts = np.asarray(sorted(set(int(c) for c in cuts)), np.int64)
        if cuts.size:
            cov = cov.copy()
            cov[cuts] = False     # a one-base gap at each breakpoint
        st, en = _intervals(cov)
        keep = (en - st) >= cfg.min_contig
        contig_sp.append(np.full(int(keep.sum()), s, np.int64))
        contig_s.append(st[keep].astype(np.int64))
        contig_e.append(en[keep].astype(np.int64))
    contig_sp = np.concatenate(contig_sp)
    contig_s = np.concatenate(contig_s)
    contig_e = np.concatenate(contig_e)
    if max_contigs is not None and contig_sp.shape[0] > max_contigs:
        pick = np.sort(rng.choice(contig_sp.shape[0], max_contigs, replace=False))
        contig_sp, contig_s, contig_e = contig_sp[pick], contig_s[pick], contig_e[pick]
    n_contigs = contig_sp.shape[0]

    # candidate reads per end: synthetic alignment to the end's locus, plus the equivalent locus
    # in every other copy of an ME family the end's window reaches into
    ends_sp = np.repeat(contig_sp, 2)
    side = np.tile(np.array([0, 1], np.int64), n_contigs)
    epos = np.where(side == 1, np.repeat(contig_e, 2), np.repeat(contig_s, 2))
    ecs = np.repeat(contig_s, 2)
    ece = np.repeat(contig_e, 2)
    q_end, q_sp, q_pos, q_cs, q_ce = [np.arange(2 * n_contigs)], [ends_sp], [epos], [ecs], [ece]
    fam_copies = {}
    for (s, p, fam, L) in me_copies:
        fam_copies.setdefault(fam, []).append((s, p))
    ends_of_sp = {}
    o_sp = np.argsort(ends_sp, kind="stable")
    b_sp = np.searchsorted(ends_sp[o_sp], np.arange(S + 1))
    for s in range(S):
        ends_of_sp[s] = o_sp[b_sp[s]:b_sp[s + 1]]
    ewl = np.where(side == 1, epos - RL, epos)
    extra = []
    for (s, p, fam, L) in me_copies:
        es = ends_of_sp[s]
        hit = es[(ewl[es] < p + L) & (ewl[es] + RL > p)]
        for e in hit.tolist():
            for (s2, p2) in fam_copies[fam]:
                if s2 == s and p2 == p:
                    continue
                off = p2 - p
                extra.append((e, s2, int(epos[e]) + off, int(ecs[e]) + off, int(ece[e]) + off))
    if extra:
        ex = np.asarray(extra, np.int64)
        q_end.append(ex[:, 0]); q_sp.append(ex[:, 1]); q_pos.append(ex[:, 2])
        q_cs.append(ex[:, 3]); q_ce.append(ex[:, 4])
    q_end = np.concatenate(q_end); q_sp = np.concatenate(q_sp); q_pos = np.concatenate(q_pos)
    q_cs = np.concatenate(q_cs); q_ce = np.concatenate(q_ce)
    q_side = q_end % 2

    sel_end, sel_sp, sel_frag = [], [], []
    for s in range(S):
        m = np.nonzero(q_sp == s)[0]
        if m.size == 0:
            continue
        f, ins = frags[s]
        ei, fi = _select_end_fragments(f, ins, q_pos[m], q_side[m], q_cs[m], q_ce[m], cfg.overlap_min)
        sel_end.append(q_end[m][ei]); sel_sp.append(np.full(fi.shape[0], s, np.int64)); sel_frag.append(fi)
    sel_end = np.concatenate(sel_end) if sel_end else np.zeros(0, np.int64)
    sel_sp = np.concatenate(sel_sp) if sel_sp else np.zeros(0, np.int64)
    sel_frag = np.concatenate(sel_frag) if sel_frag else np.zeros(0, np.int64)

    # both mates of every selected pair; a read is identified by (species, fragment, mate)
    frag_base = np.zeros(S + 1, np.int64)
    frag_base[1:] = np.cumsum([fr[0].shape[0] for fr in frags])
    gfrag = frag_base[sel_sp] + sel_frag
    r_end = np.repeat(sel_end, 2)
    r_id = np.repeat(gfrag * 2, 2) + np.tile(np.array([0, 1], np.int64), gfrag.shape[0])
    # drop duplicates of the same read in the same end (an end and its ME twin can pick the same)
    key = r_end * (2 * frag_base[-1] + 2) + r_id
    key, first = np.unique(key, return_index=True)
    r_end, r_id = r_end[first], r_id[first]
    o = np.lexsort((r_id, r_end))
    r_end, r_id = r_end[o], r_id[o]
    uniq, inv = np.unique(r_id, return_inverse=True)

    # realise each unique read once: genome substring + substitutions + N + Phred qualities
    all_f = np.concatenate([fr[0] for fr in frags])
    all_i = np.concatenate([fr[1] for fr in frags])
    sp_of = np.repeat(np.arange(S), np.diff(frag_base))
    gbase = np.zeros(S + 1, np.int64)
    gbase[1:] = np.cumsum([g.shape[0] for g in genomes])
    gall = np.concatenate(genomes)
    uf = uniq // 2
    mate = uniq % 2
    ustart = gbase[sp_of[uf]] + all_f[uf] + mate * (all_i[uf] - RL)
    U = uniq.shape[0]
    useq = np.empty((U, RL), np.uint8)
    uqual = np.empty((U, RL), np.uint8)
    ustart = np.ascontiguousarray(ustart, np.int64)
    uniq = np.ascontiguousarray(uniq, np.int64)
    _c().synth_reads(gall.ctypes.data, ustart.ctypes.data, uniq.ctypes.data, U, RL,
                     int(rng.integers(0, 2 ** 63)), float(cfg.err), float(cfg.n_rate),
                     useq.ctypes.data, uqual.ctypes.data)

    # assemble the batch
    read_seq = useq[inv].reshape(-1)
    read_qual = uqual[inv].reshape(-1)
    n_reads = r_end.shape[0]
    read_off = np.arange(n_reads + 1, dtype=np.int64) * RL
    end_read_off = np.zeros(2 * n_contigs + 1, np.int64)
    end_read_off[1:] = np.cumsum(np.bincount(r_end, minlength=2 * n_contigs))
    clen = contig_e - contig_s
    contig_off = np.zeros(n_contigs + 1, np.int64)
    contig_off[1:] = np.cumsum(clen)
    cidx = _ranges_to_ids(gbase[contig_sp] + contig_s, clen)
    contig_seq = ASCII[gall[cidx]]
    meta = dict(config=cfg.name, seed=seed, n_species=S, me_copies=len(me_copies),
                unique_reads=int(U), **cfg.meta)
    return Batch(contig_seq, contig_off, read_seq, read_qual, read_off, end_read_off, meta)


def _loguniform(rng, lo, hi, n):
    return np.exp(rng.uniform(math.log(lo), math.log(hi), n))


def c2_cfg(seed: int = seed_for(1), scale: float = 1.0) -> MetaCfg:
    """20 species, 1-3 Mbp, GC 35-65%, lognormal(0,1) abundance, ~8M reads (~30x mean)."""
    rng = np.random.default_rng(seed ^ 0x5EED)
    n = 20
    L = (_loguniform(rng, 1e6, 3e6, n) * scale).astype(np.int64)
    gc = rng.uniform(0.35, 0.65, n)
    a = rng.lognormal(0.0, 1.0, n)
    total_reads = 8e6 * scale
    cov = a * total_reads * RL / float((a * L).sum())
    # breakpoint rate tuned so the batch has ~50k contigs (strain-variant/repeat fragmentation)
    sp = [Species(int(L[i]), float(gc[i]), float(cov[i]), cut_rate=1 / 820) for i in range(n)]
    return MetaCfg("C2", sp)


def c3_cfg(seed: int = seed_for(2)) -> MetaCfg:
    """High skew: one hyper-abundant species (~20,000x, 10 contigs -> 20 hot ends with 10^4+ reads)
    plus many low-abundance species (2-8x) giving ~50k sparse ends with 0-20 reads."""
    rng = np.random.default_rng(seed ^ 0x5EED)
    sp = [Species(24_000, 0.5, 20_000.0, forced_contigs=10)]
    n = 60
    L = _loguniform(rng, 0.3e6, 1.2e6, n).astype(np.int64)
    gc = rng.uniform(0.35, 0.65, n)
    cov = rng.uniform(2.0, 8.0, n)
    sp += [Species(int(L[i]), float(gc[i]), float(cov[i]), cut_rate=1 / 4000) for i in range(n)]
    return MetaCfg("C3", sp, n_me_fam=10)


def c4_cfg(seed: int = seed_for(3), scale: float = 1.0, cut_rate: float = 1 / 400) -> MetaCfg:
    """Paper-shaped: 500 species 0.5-6 Mbp (~1.1 Gbp), lognormal(0,1.5) abundance, ~100M reads."""
    rng = np.random.default_rng(seed ^ 0x5EED)
    n = max(2, int(round(500 * scale)))
    L = _loguniform(rng, 0.5e6, 6e6, n).astype(np.int64)
    gc = rng.uniform(0.35, 0.65, n)
    a = rng.lognormal(0.0, 1.5, n)
    total_reads = 100e6 * scale
    cov = a * total_reads * RL / float((a * L).sum())
    # breakpoint rate tuned so the batch has ~1M contigs (2M ends), the size SURVEY §8(d) states for
    # C4 (r01 used 1/2000: 510k contigs); ~97M candidate-read copies
    sp = [Species(int(L[i]), float(gc[i]), float(cov[i]), cut_rate=cut_rate) for i in range(n)]
    return MetaCfg("C4", sp)


def fig3_subsample(b: Batch, seed: int, zero: float = 0.70, light: float = 0.29) -> Batch:
    """The paper's bin mix (Fig 3, arcticsynth): "the majority of contigs have zero reads",
    10-30% have fewer than 10, "less than 1%" the rest.  Applied per contig end to a C4 batch: with
    probability `zero` the end keeps no reads, with `light` the first U{1..9} of its reads (all if it
    has fewer), otherwise (1%) all of them (C4's heavy ends: up to ~700 reads; the paper's up to 3000)."""
    rng = np.random.default_rng(seed ^ 0xF163)
    r = np.diff(b.end_read_off)
    u = rng.random(r.shape[0])
    keep = np.where(u < zero, 0, np.where(u < zero + light, np.minimum(r, rng.integers(1, 10, r.shape[0])), r))
    read_ids = _ranges_to_ids(b.end_read_off[:-1], keep)
    rlen = np.diff(b.read_off)[read_ids]
    roff = np.zeros(read_ids.shape[0] + 1, np.int64)
    roff[1:] = np.cumsum(rlen)
    eoff = np.zeros(r.shape[0] + 1, np.int64)
    eoff[1:] = np.cumsum(keep)
    rseq = _gather_ranges(b.read_seq, b.read_off[read_ids], rlen)
    rqual = _gather_ranges(b.read_qual, b.read_off[read_ids], rlen)
    return Batch(b.contig_seq, b.contig_off, rseq, rqual, roff, eoff, dict(b.meta, fig3_subsample=True))


def make(config: str, seed: int | None = None, **kw) -> Batch:
    """Build a named workload: C1, C2, C3, C4 (C5 = C4 sharded, see the multi-GPU driver)."""
    config = config.upper()
    if config == "C1":
        return make_c1(seed if seed is not None else seed_for(0), **kw)
    if config == "C2":
        s = seed if seed is not None else seed_for(1)
        return make_metagenome(c2_cfg(s, kw.pop("scale", 1.0)), s, **kw)
    if config == "C3":
        s = seed if seed is not None else seed_for(2)
        return make_metagenome(c3_cfg(s), s, **kw)
    if config in ("C4", "C5"):
        s = seed if seed is not None else seed_for(3)
        return make_metagenome(c4_cfg(s, kw.pop("scale", 1.0)), s, **kw)
    if config == "C4F":   # C4 with the paper's Fig 3 mix of reads per end (fig3_subsample)
        s = seed if seed is not None else seed_for(3)
        return fig3_subsample(make_metagenome(c4_cfg(s, kw.pop("scale", 1.0)), s, **kw), s)
    if config == "C4S":   # r01's C4 (510k contigs, 31.7M read copies): quicker A/B comparisons
        s = seed if seed is not None else seed_for(3)
        return make_metagenome(c4_cfg(s, kw.pop("scale", 1.0), cut_rate=1 / 2000), s, **kw)
    raise ValueError(f"unknown config {config}")
