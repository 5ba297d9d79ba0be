"""Python face of the C ABI: `LocalAssembler` (one context per device/stream).

Argument marshalling only — every step of the path (validation, encoding, planning, table build,
walk, retry, compaction) runs in the CUDA library.  Inputs may be numpy arrays (host) or torch
tensors (host, pinned or CUDA); a batch is any object with the attributes contig_seq, contig_off,
read_seq, read_qual, read_off, end_read_off (uint8 / int64 arrays in the layout of locassm.h).
"""
from __future__ import annotations

import ctypes
from dataclasses import dataclass

import numpy as np

from . import _lib as L

PARAM_FIELDS = ("k_start", "k_min", "k_max", "k_shift", "max_walk_len", "qual_offset", "q_lo",
                "q_hi", "min_votes", "min_frac_pct")
DEFAULTS = dict(k_start=33, k_min=21, k_max=99, k_shift=8, max_walk_len=300, qual_offset=33,
                q_lo=10, q_hi=20, min_votes=2, min_frac_pct=20)


def _params(p) -> L.la_params:
    if p is None:
        p = DEFAULTS
    get = (lambda n: p[n]) if isinstance(p, dict) else (lambda n: getattr(p, n))
    return L.la_params(*[int(get(n)) for n in PARAM_FIELDS])


_BYTE_KINDS = ("uint8", "int8")


def _ptr_and_mem(a, name, want, device=None):
    """(pointer, is_device, keepalive) of a numpy array or torch tensor.  The library reads offsets as
    int64 and sequences as bytes: any other dtype (e.g. int32 offsets from a cumsum), a tensor on
    another GPU than the context's, or a non-contiguous layout is rejected here (ValueError)
    instead of being read out of bounds in C."""
    try:
        import torch
        if isinstance(a, torch.Tensor):
            dt = str(a.dtype).replace("torch.", "")
            if (want == "int64" and dt != "int64") or (want == "bytes" and dt not in _BYTE_KINDS):
                raise ValueError(f"{name}: dtype {dt}, need {'int64' if want == 'int64' else 'uint8/int8'}")
            if a.is_cuda and device is not None and a.device.index != device:
                raise ValueError(f"{name}: tensor on cuda:{a.device.index}, the context is on cuda:{device}")
            a = a.contiguous()
            return a.data_ptr(), a.is_cuda, a
    except ImportError:  # pragma: no cover
        pass
    a = np.asarray(a)
    if want == "int64" and a.dtype != np.int64:
        raise ValueError(f"{name}: dtype {a.dtype}, need int64")
    if want == "bytes" and a.dtype not in (np.uint8, np.int8):
        raise ValueError(f"{name}: dtype {a.dtype}, need uint8/int8")
    a = np.ascontiguousarray(a)
    return a.ctypes.data, False, a


@dataclass
class Result:
    ext_off: np.ndarray
    ext_seq: np.ndarray      # uint8 ASCII
    term: np.ndarray
    k_used: np.ndarray
    n_attempts: np.ndarray

    @property
    def n_ends(self):
        return self.term.shape[0]

    def ext(self, e: int) -> str:
        return self.ext_seq[self.ext_off[e]:self.ext_off[e + 1]].tobytes().decode()

    def ext_list(self):
        b = self.ext_seq.tobytes()
        o = self.ext_off
        return [b[o[i]:o[i + 1]].decode() for i in range(self.n_ends)]


class LocalAssembler:
    """la_create / la_load_batch / la_extend / la_destroy."""

    def __init__(self, device: int = 0, stream=None):
        self._lib = L.load()
        self._ctx = ctypes.c_void_p()
        sp = None
        if stream is not None:
            sp = stream if isinstance(stream, int) else getattr(stream, "cuda_stream", None)
        st = self._lib.la_create(ctypes.byref(self._ctx), int(device), ctypes.c_void_p(sp) if sp else None)
        if st != L.LA_OK:
            raise L.LocAssmError(st, "la_create failed (no CUDA device?)")
        self._keep = None
        self._device = int(device)

    def _check(self, st):
        if st != L.LA_OK:
            raise L.LocAssmError(st, self._lib.la_last_error(self._ctx).decode())

    _FIELDS = (("contig_seq", "bytes"), ("contig_off", "int64"), ("read_seq", "bytes"), ("read_qual", "bytes"),
               ("read_off", "int64"), ("end_read_off", "int64"))

    def _batch(self, batch):
        arrs = [getattr(batch, f) for f, _ in self._FIELDS]
        ptrs, devs, keep = zip(*[_ptr_and_mem(a, f, w, self._device) for a, (f, w) in zip(arrs, self._FIELDS)])
        if len(set(devs)) != 1:
            raise ValueError("batch arrays must all be host or all be device memory")
        n_contigs = int(arrs[1].shape[0]) - 1
        n_reads = int(arrs[4].shape[0]) - 1
        if 2 * n_contigs + 1 != int(arrs[5].shape[0]):
            raise ValueError("end_read_off must have 2*n_contigs+1 entries")
        b = L.la_batch(L.LA_MEM_DEVICE if devs[0] else L.LA_MEM_HOST, n_contigs, ptrs[0], ptrs[1], n_reads,
                       ptrs[2], ptrs[3], ptrs[4], ptrs[5])
        return b, keep

    def load(self, batch, params=None):
        b, keep = self._batch(batch)
        p = _params(params)
        self._check(self._lib.la_load_batch(self._ctx, ctypes.byref(b), ctypes.byref(p)))
        self._keep = keep
        return self

    def extend(self) -> Result:
        r = L.la_result()
        self._check(self._lib.la_extend(self._ctx, ctypes.byref(r)))
        return self._result(r)

    def extend_streamed(self, batch, params=None, n_chunks: int = 8) -> Result:
        """la_extend_streamed: load + extend a HOST batch in n_chunks contig ranges, the host-to-device
        copy of each chunk overlapping the extension of the previous one."""
        b, keep = self._batch(batch)
        p = _params(params)
        r = L.la_result()
        self._check(self._lib.la_extend_streamed(self._ctx, ctypes.byref(b), ctypes.byref(p), int(n_chunks),
                                                 ctypes.byref(r)))
        del keep
        return self._result(r)

    @staticmethod
    def _result(r) -> Result:
        n = int(r.n_ends)

        def arr(ptr, count, dtype):
            if count == 0:
                return np.zeros(0, dtype)
            buf = (ctypes.c_char * (count * np.dtype(dtype).itemsize)).from_address(ptr)
            return np.frombuffer(buf, dtype=dtype, count=count).copy()

        off = arr(r.ext_off, n + 1, np.int64)
        return Result(off, arr(r.ext_seq, int(off[-1]) if n else 0, np.uint8), arr(r.term, n, np.uint8),
                      arr(r.k_used, n, np.uint8), arr(r.n_attempts, n, np.uint8))

    def extend_device(self) -> dict:
        """Run without copying results to the host; returns device pointers (valid until the next call)."""
        r = L.la_result()
        self._check(self._lib.la_extend_device(self._ctx, ctypes.byref(r)))
        return dict(n_ends=int(r.n_ends), ext_off=r.ext_off, ext_seq=r.ext_seq, term=r.term,
                    k_used=r.k_used, n_attempts=r.n_attempts)

    def append_extensions(self, contig_seq, contig_off, ext_off, ext_seq):
        """la_append_extensions on CUDA tensors: extended contig c = ext(2c) + contig c + ext(2c+1)
        (Fig 4 "Append extensions to contigs").  ext_off / ext_seq may be the
        device pointers (ints) of extend_device() or CUDA tensors.  Returns (out_seq uint8, out_off
        int64) CUDA tensors."""
        import torch
        n = int(contig_off.shape[0]) - 1
        if not contig_off.is_cuda or not contig_seq.is_cuda:
            raise ValueError("append_extensions: contig arrays must be CUDA tensors")
        for name, t, ok in (("contig_off", contig_off, (torch.int64,)), ("contig_seq", contig_seq, (torch.uint8, torch.int8))) + (
                () if isinstance(ext_off, int) else
                (("ext_off", ext_off, (torch.int64,)), ("ext_seq", ext_seq, (torch.uint8, torch.int8)))):
            if t.dtype not in ok:
                raise ValueError(f"append_extensions: {name} has dtype {t.dtype}")
            if not t.is_cuda or t.device.index != self._device:
                raise ValueError(f"append_extensions: {name} must be a CUDA tensor on cuda:{self._device}")
            if not t.is_contiguous():
                raise ValueError(f"append_extensions: {name} must be contiguous")
        dev = contig_off.device
        if isinstance(ext_off, int):   # extend_device() pointers: total length from la_get_stats
            eoff_ptr, eseq_ptr = ext_off, ext_seq
            ext_tot = int(self.stats()["ext_bases"])
        else:
            eoff_ptr, eseq_ptr = ext_off.data_ptr(), ext_seq.data_ptr()
            ext_tot = int(ext_off[-1].item() - ext_off[0].item())
        tot = int(contig_off[-1].item() - contig_off[0].item()) + ext_tot
        out_seq = torch.empty(max(tot, 1), dtype=torch.uint8, device=dev)
        out_off = torch.empty(n + 1, dtype=torch.int64, device=dev)
        self._check(self._lib.la_append_extensions(self._ctx, n, contig_seq.data_ptr(), contig_off.data_ptr(),
                                                   eoff_ptr, eseq_ptr, out_seq.data_ptr(), out_off.data_ptr()))
        return out_seq[:tot], out_off

    SEL_DEFAULTS = dict(window=150, seed_len=16, seed_stride=4, min_overlap=20, max_mism_pct=4)

    def select_reads(self, pool, **sel):
        """la_select_reads (NEXT N4): candidate reads of every contig end from a pool of FR read pairs
        (attributes contig_seq, contig_off, read_seq, read_qual, read_off; reads 2i, 2i+1 are mates),
        readings S1-S6 of DESIGN.md §10d.  Returns (records, batch): records = dict of host arrays
        sel_end / sel_pair / sel_flip; batch = a DeviceBatch whose arrays stay on the device (context-owned,
        valid until the next select_reads) and can be passed to load()."""
        fields = (("contig_seq", "bytes"), ("contig_off", "int64"), ("read_seq", "bytes"), ("read_qual", "bytes"),
                  ("read_off", "int64"))
        arrs = [getattr(pool, f) for f, _ in fields]
        ptrs, devs, keep = zip(*[_ptr_and_mem(a, f, w, self._device) for a, (f, w) in zip(arrs, fields)])
        if len(set(devs)) != 1:
            raise ValueError("pool arrays must all be host or all be device memory")
        n_reads = int(arrs[4].shape[0]) - 1
        if n_reads % 2:
            raise ValueError("read_off must describe an even number of reads (pairs)")
        pl = L.la_pool(L.LA_MEM_DEVICE if devs[0] else L.LA_MEM_HOST, int(arrs[1].shape[0]) - 1, ptrs[0], ptrs[1],
                       n_reads // 2, ptrs[2], ptrs[3], ptrs[4])
        sp = dict(self.SEL_DEFAULTS, **sel)
        spc = L.la_sel_params(*[int(sp[n]) for n, _ in L.la_sel_params._fields_])
        out = L.la_selection()
        self._check(self._lib.la_select_reads(self._ctx, ctypes.byref(pl), ctypes.byref(spc), ctypes.byref(out)))
        del keep
        return _selection(out)

    def load_device_batch(self, b, params=None):
        """la_load_batch on an la_batch struct of device pointers (e.g. select_reads()'s batch)."""
        p = _params(params)
        self._check(self._lib.la_load_batch(self._ctx, ctypes.byref(b.raw), ctypes.byref(p)))
        return self

    def set_coexec(self, n_threads: int, cpu_share: float):
        """la_set_coexec: NEXT N3 CPU+GPU co-execution (the lightest ends of the smallest class on host
        threads while the GPU runs); n_threads = 0 turns it off."""
        self._check(self._lib.la_set_coexec(self._ctx, int(n_threads), float(cpu_share)))
        return self

    def replay_build(self) -> dict:
        """la_replay_build: rerun the last extension's table builds only (the hash-build phase) and
        return the stats with ms_build / cls_build_ms / cls_build_inserts filled in."""
        self._check(self._lib.la_replay_build(self._ctx))
        return self.stats()

    def stats(self) -> dict:
        s = L.la_stats()
        self._check(self._lib.la_get_stats(self._ctx, ctypes.byref(s)))
        d = {f: getattr(s, f) for f, _ in L.la_stats._fields_}
        for f, t in L.la_stats._fields_:
            if hasattr(t, "_length_"):
                v = getattr(s, f)
                d[f] = [list(x) if hasattr(x, "_length_") else x for x in v]
        return d

    def close(self):
        if getattr(self, "_ctx", None) and self._ctx.value:
            self._lib.la_destroy(self._ctx)
            self._ctx = ctypes.c_void_p()

    def __enter__(self):
        return self

    def __exit__(self, *a):
        self.close()

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass


@dataclass
class DeviceBatch:
    """An la_batch of context-owned device pointers (select_reads); `host()` copies it to numpy."""
    raw: object
    n_contigs: int
    n_reads: int

    def host(self) -> dict:
        b = self.raw
        coff = _d2h(b.contig_off, self.n_contigs + 1, np.int64)
        roff = _d2h(b.read_off, self.n_reads + 1, np.int64)
        return dict(contig_off=coff, contig_seq=_d2h(b.contig_seq, int(coff[-1]), np.uint8), read_off=roff,
                    read_seq=_d2h(b.read_seq, int(roff[-1]), np.uint8),
                    read_qual=_d2h(b.read_qual, int(roff[-1]), np.uint8),
                    end_read_off=_d2h(b.end_read_off, 2 * self.n_contigs + 1, np.int64))


_CUDART = None


def _d2h(ptr, count: int, dtype) -> np.ndarray:
    """Copy `count` elements at a library-owned device pointer into a new numpy array (cudaMemcpy of the
    CUDA runtime torch loads; the library's own runtime is linked statically and not exported)."""
    global _CUDART
    out = np.zeros(count, dtype)
    if count == 0:
        return out
    if _CUDART is None:
        import torch   # noqa: F401  (loads libcudart)
        _CUDART = ctypes.CDLL("libcudart.so.12")
        _CUDART.cudaMemcpy.argtypes = [ctypes.c_void_p, ctypes.c_void_p, ctypes.c_size_t, ctypes.c_int]
        _CUDART.cudaMemcpy.restype = ctypes.c_int
    if _CUDART.cudaMemcpy(out.ctypes.data, ctypes.c_void_p(ptr), out.nbytes, 2) != 0:   # cudaMemcpyDeviceToHost
        raise RuntimeError("cudaMemcpy (device to host) failed")
    return out


def _selection(out):
    n = int(out.n_sel)
    rec = dict(sel_end=_d2h(out.sel_end, n, np.int64), sel_pair=_d2h(out.sel_pair, n, np.int64),
               sel_flip=_d2h(out.sel_flip, n, np.uint8))
    b = out.batch
    return rec, DeviceBatch(b, int(b.n_contigs), int(b.n_reads))


def extend(batch, params=None, device: int = 0) -> Result:
    """One-shot convenience: create, load, extend, destroy."""
    with LocalAssembler(device) as la:
        return la.load(batch, params).extend()
