"""cpu_baseline — the optional all-core CPU BFS of BASELINE.md's CPU-baseline
plan (OpenMP level-synchronous top-down BFS over an uncompressed CSR).  A
reported baseline only; checked against the oracle by tests.  Shares no code
with the oracle or the product."""
from __future__ import annotations

import ctypes as C
import os

import numpy as np

_LIB = os.path.join(os.path.dirname(os.path.abspath(__file__)), "libompbfs.so")
_lib = None


def lib():
    global _lib
    if _lib is None:
        L = C.CDLL(_LIB)
        L.cb_bfs_omp.restype = C.c_uint64
        L.cb_bfs_omp.argtypes = [C.c_uint64, C.c_void_p, C.c_void_p, C.c_uint32, C.c_void_p, C.c_int]
        _lib = L
    return _lib


def bfs(vlist: np.ndarray, elist: np.ndarray, source: int, threads: int = 0) -> np.ndarray:
    n = vlist.size - 1
    depth = np.empty(n, np.int32)
    el = elist if elist.size else np.zeros(1, np.uint32)
    lib().cb_bfs_omp(n, vlist.ctypes.data, el.ctypes.data, source, depth.ctypes.data, threads)
    return depth
