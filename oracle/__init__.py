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
    src = os.path.join(_HERE, "oracle.cpp")
    if force or not os.path.exists(_SO) or os.path.getmtime(_SO) < max(
            os.path.getmtime(src), os.path.getmtime(os.path.join(_HERE, "oracle.h"))):
        subprocess.check_call(["g++", "-O2", "-std=c++17", "-shared", "-fPIC", "-o", _SO, src])
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
