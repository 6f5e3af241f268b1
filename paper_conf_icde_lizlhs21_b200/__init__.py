"""dycuckoo-b200: B200-native hot path of DyCuckoo (Li et al., ICDE'21).

Batched insert / find / delete on a two-layer cuckoo hash table with
one-subtable-at-a-time resizing, implemented as sm_100a CUDA kernels behind the
C ABI of include/dycuckoo.h (libdyc.so).  Importing this package does not load
the library; ``Table`` does, and fails loudly if it is missing.
"""
from .table import Table  # noqa: F401
from .wide import WideTable  # noqa: F401

__all__ = ["Table", "WideTable"]
