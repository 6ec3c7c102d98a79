"""B200-native DNN-occu batched ANEE GNN hot path (C-ABI library + thin binding).

The compute lives in ``lib/libocc_b200.so`` (built from ``csrc/`` by
``build.py``); ``occu`` is the ctypes binding.  There is no CPU fallback.
"""
from . import occu  # noqa: F401
from .occu import Csr, Model, OccuError, config, pack  # noqa: F401
