"""oracle — TEST INFRASTRUCTURE ONLY.

Thin ctypes wrapper over ``oracle/liboracle.so`` (built from ``oracle/oracle.c``
by ``__graft_entry__.build()``).  The C file holds the plain, slow,
single-threaded CPU definition of everything the EFG hot path computes; see its
header for the per-function PAPER.md citations and DESIGN.md §Readings for the
interpretations of silent or garbled passages.

Only ``tests/``, ``__graft_entry__.smoke()`` and ``bench.py``'s ``cpu_baseline``
/ ``--impl reference`` legs may import this package.  It shares no code with
``paper_conf_ipps_gerak23_b200`` and never imports it.

Parity status: every function here is pinned by ``tests/test_oracle_*.py``
(paper worked examples Figs. 2-6, closed forms, brute force).  Sizes against the
paper's real datasets are "parity unpinned" (datasets absent).
"""
from __future__ import annotations

import ctypes as C
import os

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_LIB_PATH = os.path.join(_HERE, "liboracle.so")
_lib = None

u64p = C.POINTER(C.c_uint64)
u32p = C.POINTER(C.c_uint32)
u8p = C.POINTER(C.c_uint8)
i32p = C.POINTER(C.c_int32)
f32p = C.POINTER(C.c_float)
f64p = C.POINTER(C.c_double)


def _ptr(a: np.ndarray, t):
    return a.ctypes.data_as(t)


def lib():
    global _lib
    if _lib is None:
        if not os.path.exists(_LIB_PATH):
            raise RuntimeError(f"{_LIB_PATH} missing: run __graft_entry__.build()")
        L = C.CDLL(_LIB_PATH)
        L.or_csr_build.restype = C.c_void_p
        L.or_csr_build.argtypes = [C.c_uint64, C.c_uint64, u32p, u32p, C.c_int, C.c_int, C.c_int]
        L.or_csr_n.restype = C.c_uint64
        L.or_csr_n.argtypes = [C.c_void_p]
        L.or_csr_m.restype = C.c_uint64
        L.or_csr_m.argtypes = [C.c_void_p]
        L.or_csr_vlist.restype = u64p
        L.or_csr_vlist.argtypes = [C.c_void_p]
        L.or_csr_elist.restype = u32p
        L.or_csr_elist.argtypes = [C.c_void_p]
        L.or_csr_free.restype = None
        L.or_csr_free.argtypes = [C.c_void_p]
        L.or_bfs.restype = C.c_uint64
        L.or_bfs.argtypes = [C.c_uint64, u64p, u32p, C.c_uint32, i32p]
        L.or_bfs_bounded.restype = C.c_uint64
        L.or_bfs_bounded.argtypes = [C.c_uint64, u64p, u32p, C.c_uint32, i32p, C.c_uint64, u64p]
        L.or_ef_lower_bits.restype = C.c_uint32
        L.or_ef_lower_bits.argtypes = [C.c_uint64, C.c_uint64]
        L.or_ef_sections.restype = None
        L.or_ef_sections.argtypes = [C.c_uint64, C.c_uint64, C.c_uint32, u64p, u64p, u64p]
        L.or_ef_encode_list.restype = C.c_uint64
        L.or_ef_encode_list.argtypes = [u32p, C.c_uint64, C.c_uint32, u8p, u32p]
        L.or_ef_select1.restype = C.c_uint64
        L.or_ef_select1.argtypes = [u8p, C.c_uint64, C.c_uint32, C.c_uint32, C.c_uint64]
        L.or_ef_decode_list.restype = None
        L.or_ef_decode_list.argtypes = [u8p, C.c_uint64, C.c_uint32, C.c_uint32, u32p]
        L.or_ef_fwd.restype = C.c_uint32
        L.or_ef_fwd.argtypes = [u8p, C.c_uint64]
        L.or_efg_offsets.restype = C.c_uint64
        L.or_efg_offsets.argtypes = [C.c_uint64, u64p, u32p, C.c_uint32, u64p]
        L.or_efg_encode.restype = None
        L.or_efg_encode.argtypes = [C.c_uint64, u64p, u32p, C.c_uint32, u64p, u8p, u8p]
        L.or_efg_decode_range.restype = None
        L.or_efg_decode_range.argtypes = [u64p, u8p, u64p, u8p, C.c_uint32, C.c_uint64,
                                          C.c_uint64, u32p]
        L.or_maxle.restype = C.c_int64
        L.or_maxle.argtypes = [u64p, C.c_uint64, C.c_uint64]
        L.or_exclusive_scan.restype = None
        L.or_exclusive_scan.argtypes = [u64p, C.c_uint64, u64p]
        L.or_sssp.restype = C.c_int
        L.or_sssp.argtypes = [C.c_uint64, u64p, u32p, f32p, C.c_uint32, f32p]
        L.or_pagerank.restype = None
        L.or_pagerank.argtypes = [C.c_uint64, u64p, u32p, C.c_double, C.c_uint32, f64p]
        _lib = L
    return _lib


# --------------------------------------------------------------------------
# CSR
# --------------------------------------------------------------------------
def csr_build(n: int, src, dst, symmetrize=True, dedup=True, drop_self=True):
    """Return (vlist uint64[n+1], elist uint32[m]) per P:75-77 + readings C11/C12."""
    src = np.ascontiguousarray(src, dtype=np.uint32)
    dst = np.ascontiguousarray(dst, dtype=np.uint32)
    assert src.shape == dst.shape
    L = lib()
    h = L.or_csr_build(n, src.size, _ptr(src, u32p), _ptr(dst, u32p), int(symmetrize),
                       int(dedup), int(drop_self))
    if not h:
        raise ValueError("oracle csr_build: id out of range or out of memory")
    try:
        m = L.or_csr_m(h)
        vlist = np.ctypeslib.as_array(L.or_csr_vlist(h), shape=(n + 1,)).copy()
        elist = (np.ctypeslib.as_array(L.or_csr_elist(h), shape=(m,)).copy()
                 if m else np.zeros(0, np.uint32))
    finally:
        L.or_csr_free(h)
    return vlist, elist


# --------------------------------------------------------------------------
# BFS (Alg. 1)
# --------------------------------------------------------------------------
def bfs(vlist: np.ndarray, elist: np.ndarray, source: int) -> np.ndarray:
    n = vlist.size - 1
    depth = np.empty(n, np.int32)
    el = elist if elist.size else np.zeros(1, np.uint32)
    lib().or_bfs(n, _ptr(vlist, u64p), _ptr(el, u32p), source, _ptr(depth, i32p))
    return depth


def bfs_bounded(vlist: np.ndarray, elist: np.ndarray, source: int, max_edges: int):
    """FIFO BFS stopped once `max_edges` adjacency entries were scanned:
    (depth, dequeued vertices, edges scanned).  Assigned depths are final."""
    n = vlist.size - 1
    depth = np.empty(n, np.int32)
    el = elist if elist.size else np.zeros(1, np.uint32)
    scanned = np.zeros(1, np.uint64)
    nv = lib().or_bfs_bounded(n, _ptr(vlist, u64p), _ptr(el, u32p), source, _ptr(depth, i32p),
                              max_edges, _ptr(scanned, u64p))
    return depth, int(nv), int(scanned[0])


# --------------------------------------------------------------------------
# Elias-Fano
# --------------------------------------------------------------------------
def ef_lower_bits(n: int, u: int) -> int:
    return int(lib().or_ef_lower_bits(n, u))


def ef_sections(n: int, u: int, k: int):
    a, b, c = C.c_uint64(), C.c_uint64(), C.c_uint64()
    lib().or_ef_sections(n, u, k, C.byref(a), C.byref(b), C.byref(c))
    return a.value, b.value, c.value


def ef_encode_list(x, k: int = 512):
    """Return (bytes, l) for a sorted list x."""
    x = np.ascontiguousarray(x, dtype=np.uint32)
    n = x.size
    if n == 0:
        return b"", 0
    fb, lb, ub = ef_sections(n, int(x[-1]), k)
    out = np.zeros(max(1, fb + lb + ub), np.uint8)
    l = C.c_uint32()
    s = lib().or_ef_encode_list(_ptr(x, u32p), n, k, _ptr(out, u8p), C.byref(l))
    return out[:s].tobytes(), l.value


def ef_select1(enc: bytes, n: int, l: int, k: int, i: int) -> int:
    buf = np.frombuffer(enc + b"\0" * 8, np.uint8).copy()
    return int(lib().or_ef_select1(_ptr(buf, u8p), n, l, k, i))


def ef_decode_list(enc: bytes, n: int, l: int, k: int = 512) -> np.ndarray:
    buf = np.frombuffer(enc + b"\0" * 8, np.uint8).copy()
    out = np.zeros(max(n, 1), np.uint32)
    lib().or_ef_decode_list(_ptr(buf, u8p), n, l, k, _ptr(out, u32p))
    return out[:n]


def ef_fwd(enc: bytes, j: int) -> int:
    buf = np.frombuffer(enc + b"\0" * 8, np.uint8).copy()
    return int(lib().or_ef_fwd(_ptr(buf, u8p), j))


def efg_encode(vlist: np.ndarray, elist: np.ndarray, k: int = 512):
    """Whole-graph EFG arrays: returns (offsets u64[n+1], nlb u8[n], data u8[])."""
    n = vlist.size - 1
    el = elist if elist.size else np.zeros(1, np.uint32)
    offsets = np.zeros(n + 1, np.uint64)
    total = lib().or_efg_offsets(n, _ptr(vlist, u64p), _ptr(el, u32p), k, _ptr(offsets, u64p))
    nlb = np.zeros(max(n, 1), np.uint8)
    data = np.zeros(max(int(total), 1), np.uint8)
    lib().or_efg_encode(n, _ptr(vlist, u64p), _ptr(el, u32p), k, _ptr(offsets, u64p),
                        _ptr(nlb, u8p), _ptr(data, u8p))
    return offsets, nlb[:n], data[:int(total)]


def efg_decode_range(vlist, nlb, offsets, data, k, v0, v1) -> np.ndarray:
    cnt = int(vlist[v1] - vlist[v0])
    out = np.zeros(max(cnt, 1), np.uint32)
    d = np.concatenate([data, np.zeros(8, np.uint8)])
    nl = nlb if nlb.size else np.zeros(1, np.uint8)
    lib().or_efg_decode_range(_ptr(vlist, u64p), _ptr(nl, u8p), _ptr(offsets, u64p),
                              _ptr(d, u8p), k, v0, v1, _ptr(out, u32p))
    return out[:cnt]


# --------------------------------------------------------------------------
# scans / searches (Fig. 4)
# --------------------------------------------------------------------------
def exclusive_scan(a) -> np.ndarray:
    a = np.ascontiguousarray(a, dtype=np.uint64)
    out = np.zeros(a.size + 1, np.uint64)
    aa = a if a.size else np.zeros(1, np.uint64)
    lib().or_exclusive_scan(_ptr(aa, u64p), a.size, _ptr(out, u64p))
    return out


def maxle(a, key: int) -> int:
    a = np.ascontiguousarray(a, dtype=np.uint64)
    aa = a if a.size else np.zeros(1, np.uint64)
    return int(lib().or_maxle(_ptr(aa, u64p), a.size, key))


# --------------------------------------------------------------------------
# SSSP / PageRank
# --------------------------------------------------------------------------
def sssp(vlist, elist, w, source: int) -> np.ndarray:
    n = vlist.size - 1
    dist = np.empty(n, np.float32)
    el = elist if elist.size else np.zeros(1, np.uint32)
    ww = np.ascontiguousarray(w, np.float32) if elist.size else np.zeros(1, np.float32)
    rc = lib().or_sssp(n, _ptr(vlist, u64p), _ptr(el, u32p), _ptr(ww, f32p), source,
                       _ptr(dist, f32p))
    if rc != 0:
        raise ValueError("oracle sssp failed")
    return dist


def pagerank(vlist, elist, damping=0.85, iters=50) -> np.ndarray:
    n = vlist.size - 1
    rank = np.empty(n, np.float64)
    el = elist if elist.size else np.zeros(1, np.uint32)
    lib().or_pagerank(n, _ptr(vlist, u64p), _ptr(el, u32p), damping, iters, _ptr(rank, f64p))
    return rank
