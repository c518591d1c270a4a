"""B200-native (sm_100a) Seastar hot path: fused vertex-centric GCN / APPNP / GAT / R-GCN kernels.

Everything computes in ``libseastar.so`` (hand-written CUDA, see ``csrc/`` and ``include/seastar.h``).
``_lib`` is the ctypes binding (same names as the C ABI), ``graph.Graph`` owns a preprocessed graph,
``models`` runs whole training epochs through the C ABI.
"""
from . import _lib  # noqa: F401
from ._lib import SeastarError  # noqa: F401

__all__ = ["_lib", "SeastarError"]
