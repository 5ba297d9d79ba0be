"""ctypes binding of include/locassm.h (argument marshalling only).

The shared library liblocassm.so is built in-tree by build.py; if it is missing this module raises
— there is no CPU fallback anywhere in the product package.
"""
from __future__ import annotations

import ctypes
import os

HERE = os.path.dirname(os.path.abspath(__file__))
SO = os.environ.get("LA_SO") or os.path.join(HERE, "liblocassm.so")   # LA_SO: debug builds (tools/)

LA_OK, LA_ERR_INVALID_ARG, LA_ERR_OOM, LA_ERR_CUDA, LA_ERR_STATE, LA_ERR_CAPACITY = 0, -1, -2, -3, -4, -5
LA_MEM_HOST, LA_MEM_DEVICE = 0, 1
LA_HIST = 16
LA_N_CLASSES = 7   # 0-4 shared memory, 5 XL, 6 XLC
STATUS = {0: "LA_OK", -1: "LA_ERR_INVALID_ARG", -2: "LA_ERR_OOM", -3: "LA_ERR_CUDA",
          -4: "LA_ERR_STATE", -5: "LA_ERR_CAPACITY"}
TERM_NAMES = ["DEADEND", "FORK", "LOOP", "MAXLEN", "NOREADS", "SHORT"]


class la_params(ctypes.Structure):
    _fields_ = [(n, ctypes.c_int32) for n in (
        "k_start", "k_min", "k_max", "k_shift", "max_walk_len", "qual_offset", "q_lo", "q_hi",
        "min_votes", "min_frac_pct")]


class la_batch(ctypes.Structure):
    _fields_ = [("mem", ctypes.c_int32), ("n_contigs", ctypes.c_int32),
                ("contig_seq", ctypes.c_void_p), ("contig_off", ctypes.c_void_p),
                ("n_reads", ctypes.c_int64),
                ("read_seq", ctypes.c_void_p), ("read_qual", ctypes.c_void_p),
                ("read_off", ctypes.c_void_p), ("end_read_off", ctypes.c_void_p)]


class la_result(ctypes.Structure):
    _fields_ = [("n_ends", ctypes.c_int64), ("ext_off", ctypes.c_void_p),
                ("ext_seq", ctypes.c_void_p), ("term", ctypes.c_void_p),
                ("k_used", ctypes.c_void_p), ("n_attempts", ctypes.c_void_p)]


class la_stats(ctypes.Structure):
    _fields_ = [("ms_total", ctypes.c_double), ("ms_smem", ctypes.c_double),
                ("ms_global", ctypes.c_double), ("ms_emit", ctypes.c_double),
                ("inserts", ctypes.c_int64), ("inserts_smem", ctypes.c_int64), ("walk_steps", ctypes.c_int64),
                ("attempts", ctypes.c_int64), ("ext_bases", ctypes.c_int64),
                ("ends_by_class", ctypes.c_int64 * 5), ("kernel_launches", ctypes.c_int64),
                ("smem_bytes_per_cta", ctypes.c_int64), ("smem_ctas_per_sm", ctypes.c_int32),
                ("global_rounds", ctypes.c_int32), ("ends_medium", ctypes.c_int64),
                ("ms_smem_medium", ctypes.c_double), ("ends_xl", ctypes.c_int64),
                ("xl_scratch_bytes", ctypes.c_int64), ("cls_ends", ctypes.c_int64 * LA_N_CLASSES),
                ("cls_inserts", ctypes.c_int64 * LA_N_CLASSES), ("cls_attempts", ctypes.c_int64 * LA_N_CLASSES),
                ("cls_filtered", ctypes.c_int64 * LA_N_CLASSES), ("cls_ms", ctypes.c_double * LA_N_CLASSES),
                ("prof_cycles", (ctypes.c_uint64 * 8) * LA_N_CLASSES),
                ("ms_build", ctypes.c_double), ("ms_walk", ctypes.c_double),
                ("cls_build_ms", ctypes.c_double * LA_N_CLASSES), ("cls_build_inserts", ctypes.c_int64 * LA_N_CLASSES),
                ("cls_inl_attempts", ctypes.c_int64 * LA_N_CLASSES), ("cls_ref_attempts", ctypes.c_int64 * LA_N_CLASSES),
                ("attempts_hist", ctypes.c_int64 * LA_HIST), ("cls_dead0", ctypes.c_int64 * LA_N_CLASSES),
                ("cpu_ends", ctypes.c_int64), ("cpu_inserts", ctypes.c_int64), ("cpu_walk_steps", ctypes.c_int64),
                ("cpu_attempts", ctypes.c_int64)]


class la_pool(ctypes.Structure):
    _fields_ = [("mem", ctypes.c_int32), ("n_contigs", ctypes.c_int32),
                ("contig_seq", ctypes.c_void_p), ("contig_off", ctypes.c_void_p),
                ("n_pairs", ctypes.c_int64),
                ("read_seq", ctypes.c_void_p), ("read_qual", ctypes.c_void_p), ("read_off", ctypes.c_void_p)]


class la_sel_params(ctypes.Structure):
    _fields_ = [(n, ctypes.c_int32) for n in ("window", "seed_len", "seed_stride", "min_overlap", "max_mism_pct")]


class la_selection(ctypes.Structure):
    _fields_ = [("n_sel", ctypes.c_int64), ("sel_end", ctypes.c_void_p), ("sel_pair", ctypes.c_void_p),
                ("sel_flip", ctypes.c_void_p), ("batch", la_batch)]


EXPORTS = ["la_create", "la_load_batch", "la_extend", "la_extend_device", "la_extend_streamed", "la_append_extensions",
           "la_replay_build", "la_set_coexec", "la_select_reads",
           "la_get_stats", "la_destroy", "la_last_error", "la_plan_global_capacity", "la_paper_load_factor"]

_lib = None


class LocAssmError(RuntimeError):
    def __init__(self, status, msg):
        super().__init__(f"{STATUS.get(status, status)}: {msg}")
        self.status = status


def load():
    """Load liblocassm.so; raises if it has not been built (no fallback)."""
    global _lib
    if _lib is not None:
        return _lib
    if not os.path.exists(SO):
        raise RuntimeError(f"CUDA extension {SO} is missing: run paper_conf_sc_awanhedbdoy21_b200/build.py "
                           "(or __graft_entry__.build()) first")
    lib = ctypes.CDLL(SO)
    V = ctypes.c_void_p
    lib.la_create.argtypes = [ctypes.POINTER(V), ctypes.c_int, V]
    lib.la_load_batch.argtypes = [V, ctypes.POINTER(la_batch), ctypes.POINTER(la_params)]
    lib.la_extend.argtypes = [V, ctypes.POINTER(la_result)]
    lib.la_extend_device.argtypes = [V, ctypes.POINTER(la_result)]
    lib.la_extend_streamed.argtypes = [V, ctypes.POINTER(la_batch), ctypes.POINTER(la_params), ctypes.c_int32,
                                       ctypes.POINTER(la_result)]
    lib.la_append_extensions.argtypes = [V, ctypes.c_int32, V, V, V, V, V, V]
    lib.la_get_stats.argtypes = [V, ctypes.POINTER(la_stats)]
    lib.la_replay_build.argtypes = [V]
    lib.la_set_coexec.argtypes = [V, ctypes.c_int32, ctypes.c_double]
    lib.la_select_reads.argtypes = [V, ctypes.POINTER(la_pool), ctypes.POINTER(la_sel_params),
                                    ctypes.POINTER(la_selection)]
    lib.la_destroy.argtypes = [V]
    lib.la_last_error.argtypes = [V]
    lib.la_last_error.restype = ctypes.c_char_p
    lib.la_plan_global_capacity.argtypes = [ctypes.c_int64]
    lib.la_plan_global_capacity.restype = ctypes.c_int64
    lib.la_paper_load_factor.argtypes = [ctypes.c_int32, ctypes.c_int32]
    lib.la_paper_load_factor.restype = ctypes.c_double
    for f in ("la_create", "la_load_batch", "la_extend", "la_extend_device", "la_extend_streamed", "la_append_extensions",
              "la_replay_build", "la_set_coexec", "la_select_reads", "la_get_stats", "la_destroy"):
        getattr(lib, f).restype = ctypes.c_int
    _lib = lib
    return lib
