"""B200-native CloverLeaf 2D timestep (the hot path of Reguly, Mudalige,
Giles, CLUSTER 2015; sec. V).

The product is the C-ABI library libclover.so (include/clover.h) built from
csrc/ for sm_100a; `clover` is its thin ctypes binding.  There is no CPU
fallback: the binding raises if the library is missing.
"""
from .clover import Clover, CloverError, load, nccl_unique_id  # noqa: F401

__all__ = ["Clover", "CloverError", "load", "nccl_unique_id"]
