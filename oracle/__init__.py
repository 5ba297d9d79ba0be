"""CPU oracle of MetaHipMer local assembly — TEST INFRASTRUCTURE ONLY.

Only tests/, __graft_entry__.smoke() and bench.py (cpu_baseline / --impl reference) may import
this package.  The product package paper_conf_sc_awanhedbdoy21_b200 never imports it.

`extend(batch, params, ends=None)` runs oracle.cpp (plain single-threaded C++ written from the
paper; see oracle.h for the citations and the parity status) on host arrays.
"""
from __future__ import annotations

import ctypes
import os
import subprocess

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SO = os.path.join(_HERE, "liblaoracle.so")
_lib = None

TERM_NAMES = ["DEADEND", "FORK", "LOOP", "MAXLEN", "NOREADS", "SHORT"]


class OrcParams(ctypes.Structure):
    _fields_ = [(n, ctypes.c_int32) for n in (
        "k_start", "k_min", "k_max", "k_shift", "max_walk_len", "qual_offset", "q_lo", "q_hi",
        "min_votes", "min_frac_pct", "loop_accepts")]


def build(force: bool = False) -> str:
    """Compile oracle.cpp into liblaoracle.so (g++ -O2, single thread)."""
    srcs = [os.path.join(_HERE, "oracle.cpp"), os.path.join(_HERE, "select.cpp")]
    if force or not os.path.exists(_SO) or os.path.getmtime(_SO) < max(
            [os.path.getmtime(p) for p in srcs] + [os.path.getmtime(os.path.join(_HERE, "oracle.h"))]):
        subprocess.check_call(["g++", "-O2", "-std=c++17", "-shared", "-fPIC", "-o", _SO, *srcs])
    return _SO


def _load():
    global _lib
    if _lib is None:
        build()
        lib = ctypes.CDLL(_SO)
        P = ctypes.c_void_p
        lib.orc_extend.argtypes = [ctypes.c_int32, P, P, ctypes.c_int64, P, P, P, P, P, P,
                                   ctypes.c_int64, P, P, P, P, P, P, P]
        lib.orc_extend.restype = ctypes.c_int
        lib.orc_ext_rule.argtypes = [P, P, P]
        lib.orc_ext_rule.restype = ctypes.c_int
        lib.orc_select.argtypes = [ctypes.c_int32, P, P, ctypes.c_int64, P, P] + [ctypes.c_int32] * 5 + [
            ctypes.c_int64, P, P, P]
        lib.orc_select.restype = ctypes.c_int64
        _lib = lib
    return _lib


def _params(params, loop_accepts=False) -> OrcParams:
    return OrcParams(*params.as_tuple(), int(bool(loop_accepts)))


def _ptr(a):
    return ctypes.c_void_p(a.ctypes.data) if a is not None and a.size else ctypes.c_void_p(
        a.ctypes.data if a is not None else None)


def ext_rule(lo, hi, params) -> int:
    """Vote rule of reading #1: 0..3 = ACGT, -1 = FORK, -2 = DEADEND."""
    lib = _load()
    lo = np.ascontiguousarray(lo, np.uint32)
    hi = np.ascontiguousarray(hi, np.uint32)
    p = _params(params)
    return lib.orc_ext_rule(_ptr(lo), _ptr(hi), ctypes.byref(p))


def extend(batch, params, ends=None, loop_accepts=False):
    """Run the oracle on the selected ends (default: all, in order).

    Returns dict: ext (list[str]), term/k_used/n_attempts (uint8 arrays), inserts, walk_steps
    (int64 arrays), ends (int64 array of end ids)."""
    lib = _load()
    if ends is None:
        ends = np.arange(batch.n_ends, dtype=np.int64)
    ends = np.ascontiguousarray(ends, np.int64)
    n = ends.shape[0]
    W = max(int(params.max_walk_len), 1)
    ext_len = np.zeros(n, np.int64)
    ext_buf = np.zeros(n * W, np.uint8)
    term = np.zeros(n, np.uint8)
    k_used = np.zeros(n, np.uint8)
    n_att = np.zeros(n, np.uint8)
    ins = np.zeros(n, np.int64)
    steps = np.zeros(n, np.int64)
    arrs = [np.ascontiguousarray(x) for x in (batch.contig_seq, batch.contig_off, batch.read_seq,
                                              batch.read_qual, batch.read_off, batch.end_read_off)]
    p = _params(params, loop_accepts)
    rc = lib.orc_extend(batch.n_contigs, _ptr(arrs[0]), _ptr(arrs[1]), batch.n_reads, _ptr(arrs[2]),
                        _ptr(arrs[3]), _ptr(arrs[4]), _ptr(arrs[5]), ctypes.byref(p), _ptr(ends), n,
                        _ptr(ext_len), _ptr(ext_buf), _ptr(term), _ptr(k_used), _ptr(n_att),
                        _ptr(ins), _ptr(steps))
    if rc != 0:
        raise ValueError("oracle: invalid arguments")
    buf = ext_buf.tobytes()
    ext = [buf[i * W:i * W + int(ext_len[i])].decode() for i in range(n)]
    return dict(ends=ends, ext=ext, term=term, k_used=k_used, n_attempts=n_att, inserts=ins,
                walk_steps=steps)


def append_extensions(contigs, ext):
    """Fig 4 "Append extensions to contigs" (L558-563) and P:L464 ("appended to the end of contig"),
    both sides by the symmetry of P:L399-402: extended contig c = ext[2c] + contigs[c] + ext[2c+1],
    ext[2c] (LEFT end) being in contig-forward orientation already (the oracle returns it so).
    Plain definition, written out per contig."""
    out = []
    for c, seq in enumerate(contigs):
        out.append(ext[2 * c] + seq + ext[2 * c + 1])
    return out


_COMP = bytes.maketrans(b"ACGTN", b"TGCAN")


def select_reads(contig_seq, contig_off, read_seq, read_qual, read_off, w=150, s=16, t=4, o=20, mm_pct=4):
    """NEXT N4, candidate-read selection (select.cpp, readings S1-S6 of DESIGN.md §10d): from a pool of
    FR read pairs (reads 2i, 2i+1), the candidate reads of every contig end, written as la_load_batch
    takes them.  Returns dict(end_read_off, read_seq, read_qual, read_off, sel_end, sel_pair, sel_flip).
    S5-S6 (the batch layout) are written out here: per selected (end, pair) record in (end, pair)
    order, mate 0 then mate 1, each reverse-complemented (qualities reversed) when its strand is -."""
    lib = _load()
    contig_seq = np.ascontiguousarray(contig_seq, np.uint8)
    contig_off = np.ascontiguousarray(contig_off, np.int64)
    read_seq = np.ascontiguousarray(read_seq, np.uint8)
    read_qual = np.ascontiguousarray(read_qual, np.uint8)
    read_off = np.ascontiguousarray(read_off, np.int64)
    n_contigs = contig_off.shape[0] - 1
    n_pairs = (read_off.shape[0] - 1) // 2
    cap = max(16, 4 * n_pairs + 16)
    while True:
        se = np.zeros(cap, np.int64)
        sp = np.zeros(cap, np.int64)
        sf = np.zeros(cap, np.uint8)
        n = lib.orc_select(n_contigs, _ptr(contig_seq), _ptr(contig_off), n_pairs, _ptr(read_seq), _ptr(read_off),
                           int(w), int(s), int(t), int(o), int(mm_pct), cap, _ptr(se), _ptr(sp), _ptr(sf))
        if n == -2:
            cap *= 4
            continue
        if n < 0:
            raise ValueError("oracle.select_reads: invalid arguments")
        break
    se, sp, sf = se[:n], sp[:n], sf[:n]
    seq_out, qual_out, lens = [], [], []
    rs, rq = read_seq.tobytes(), read_qual.tobytes()
    for e, p, f in zip(se.tolist(), sp.tolist(), sf.tolist()):
        for mate in (0, 1):
            rid = 2 * p + mate
            x, q = rs[read_off[rid]:read_off[rid + 1]], rq[read_off[rid]:read_off[rid + 1]]
            flip = (mate == 0) == bool(f)     # f = 0: mate 0 as is, mate 1 rc'd; f = 1: the opposite
            if flip:
                x, q = x[::-1].translate(_COMP), q[::-1]
            seq_out.append(x)
            qual_out.append(q)
            lens.append(len(x))
    end_read_off = np.zeros(2 * n_contigs + 1, np.int64)
    if n:
        end_read_off[1:] = np.cumsum(2 * np.bincount(se, minlength=2 * n_contigs))
    off = np.zeros(len(lens) + 1, np.int64)
    off[1:] = np.cumsum(lens)
    return dict(end_read_off=end_read_off, read_seq=np.frombuffer(b"".join(seq_out), np.uint8).copy(),
                read_qual=np.frombuffer(b"".join(qual_out), np.uint8).copy(), read_off=off,
                sel_end=se, sel_pair=sp, sel_flip=sf)
