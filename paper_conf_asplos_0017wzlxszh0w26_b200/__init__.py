"""B200-native Bipartite Attention (BAT) prefill: a C-ABI library (libbat.so, sm_100a kernels)
and its thin ctypes binding (``bat``) plus device-memory helpers (``runtime``).

The binding loads ``libbat.so`` lazily; nothing here computes any step of the method."""
from . import bat  # noqa: F401

__all__ = ["bat"]
