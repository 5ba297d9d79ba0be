"""B200 (sm_100a) local assembly of MetaHipMer (Awan et al., SC'21), rebuilt from the paper.

The hot path lives in the CUDA library csrc/ (C ABI: include/locassm.h); this package only
marshals arguments (api.py) and shards batches across GPUs (dist.py).
"""
from .api import LocalAssembler, Result, extend, DEFAULTS  # noqa: F401
