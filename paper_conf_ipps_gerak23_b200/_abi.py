"""ctypes declarations of include/efg.h (argument marshalling only).

Every computation behind these calls runs in libefg.so (host builder in C++,
traversal in the sm_100a kernels).  If the library is missing this module raises
at import: there is no Python or CPU fallback.
"""
from __future__ import annotations

import ctypes as C
import os

_HERE = os.path.dirname(os.path.abspath(__file__))
# EFG_LIB: an alternative build of the same library (tuning experiments only)
LIB_PATH = os.environ.get("EFG_LIB") or os.path.join(_HERE, "libefg.so")

EFG_OK, EFG_EINVAL, EFG_ERANGE, EFG_ENOMEM, EFG_ECUDA, EFG_ENCCL, EFG_ENOTSUP, EFG_ESTATE, EFG_EIO = range(9)
STATUS_NAMES = {0: "EFG_OK", 1: "EFG_EINVAL", 2: "EFG_ERANGE", 3: "EFG_ENOMEM", 4: "EFG_ECUDA",
                5: "EFG_ENCCL", 6: "EFG_ENOTSUP", 7: "EFG_ESTATE", 8: "EFG_EIO"}
EFG_SYMMETRIZE, EFG_DEDUP, EFG_DROP_SELF_LOOPS = 0x1, 0x2, 0x4
EFG_DEFAULT_FLAGS = 0x7
EFG_REORDER_DEGREE = 0x8
EFG_HOST_RESIDENT = 0x10
EFG_OPT_LEVEL_LOOP = 1
EFG_OPT_PREFIX_SKIP = 2
EFG_OPT_PAGERANK_PULL = 3
EFG_OPT_EXPAND_VARIANT = 4


class BuildOpts(C.Structure):
    _fields_ = [("fwd_quantum", C.c_uint32), ("flags", C.c_uint32), ("device", C.c_int32),
                ("n_threads", C.c_uint32), ("stream", C.c_void_p), ("weights", C.c_void_p),
                ("row_lo", C.c_uint64), ("row_hi", C.c_uint64)]


class Info(C.Structure):
    _fields_ = [("n", C.c_uint64), ("m", C.c_uint64), ("m_input", C.c_uint64),
                ("fwd_quantum", C.c_uint32), ("device", C.c_uint32), ("data_bytes", C.c_uint64),
                ("fwd_bytes", C.c_uint64), ("lower_bytes", C.c_uint64), ("upper_bytes", C.c_uint64),
                ("apriori_bits", C.c_uint64), ("vertex_bytes", C.c_uint64),
                ("device_bytes", C.c_uint64), ("row_lo", C.c_uint64), ("row_hi", C.c_uint64),
                ("build_seconds", C.c_double), ("device_quantum", C.c_uint32),
                ("data_location", C.c_uint32)]


class Stats(C.Structure):
    _fields_ = [("levels", C.c_uint32), ("level_cap", C.c_uint32),
                ("edges_traversed", C.c_uint64), ("vertices_reached", C.c_uint64),
                ("device_ms", C.c_float), ("expand_ms", C.c_float),
                ("expand_launches", C.c_uint32), ("kernel_launches", C.c_uint32),
                ("expand_bytes", C.c_uint64), ("level_frontier", C.c_void_p),
                ("level_edges", C.c_void_p), ("level_expand_ms", C.c_void_p),
                ("level_end_ms", C.c_void_p), ("d2h_bytes", C.c_uint64),
                ("xchg_sparse_levels", C.c_uint32)]


# (name, restype, argtypes) for every symbol include/efg.h declares
SIGNATURES = [
    ("efg_default_opts", None, [C.POINTER(BuildOpts)]),
    ("efg_build", C.c_int, [C.c_uint64, C.c_uint64, C.c_void_p, C.c_void_p, C.POINTER(BuildOpts),
                            C.POINTER(C.c_void_p)]),
    ("efg_build_stream", C.c_int, [C.c_uint64, C.c_uint64, C.c_void_p, C.c_void_p, C.c_int,
                                   C.POINTER(BuildOpts), C.POINTER(C.c_void_p)]),
    ("efg_free", None, [C.c_void_p]),
    ("efg_save", C.c_int, [C.c_void_p, C.c_char_p]),
    ("efg_load", C.c_int, [C.c_char_p, C.POINTER(BuildOpts), C.POINTER(C.c_void_p)]),
    ("efg_info", C.c_int, [C.c_void_p, C.POINTER(Info)]),
    ("efg_export", C.c_int, [C.c_void_p, C.c_void_p, C.c_void_p, C.c_void_p, C.c_void_p]),
    ("efg_export_perm", C.c_int, [C.c_void_p, C.c_void_p]),
    ("efg_decode", C.c_int, [C.c_void_p, C.c_uint32, C.c_uint32, C.c_void_p]),
    ("efg_bfs", C.c_int, [C.c_void_p, C.c_uint32, C.c_void_p, C.c_void_p, C.POINTER(Stats)]),
    ("efg_sssp", C.c_int, [C.c_void_p, C.c_uint32, C.c_void_p, C.POINTER(Stats)]),
    ("efg_pagerank", C.c_int, [C.c_void_p, C.c_double, C.c_uint32, C.c_void_p, C.POINTER(Stats)]),
    ("efg_set_option", C.c_int, [C.c_void_p, C.c_int, C.c_int64]),
    ("efg_xchg_geometry", C.c_int, [C.c_void_p, C.c_int, C.c_void_p, C.POINTER(C.c_uint64)]),
    ("efg_bfs_begin", C.c_int, [C.c_void_p, C.c_uint32, C.c_void_p]),
    ("efg_bfs_expand", C.c_int, [C.c_void_p]),
    ("efg_xchg_pack", C.c_int, [C.c_void_p, C.c_int, C.c_void_p, C.c_uint64, C.c_void_p]),
    ("efg_xchg_reduce", C.c_int, [C.c_void_p, C.c_int, C.c_uint64, C.c_void_p, C.c_void_p]),
    ("efg_xchg_unpack", C.c_int, [C.c_void_p, C.c_int, C.c_void_p, C.c_uint64, C.c_void_p]),
    ("efg_peer_alloc", C.c_int, [C.c_void_p, C.c_int, C.POINTER(C.c_void_p), C.c_void_p]),
    ("efg_peer_open", C.c_int, [C.c_void_p, C.c_int, C.c_int, C.c_void_p, C.c_void_p, C.c_void_p]),
    ("efg_xchg_peer", C.c_int, [C.c_void_p]),
    ("efg_xchg_peer_phase", C.c_int, [C.c_void_p, C.c_int]),
    ("efg_bfs_finish_level", C.c_int, [C.c_void_p, C.POINTER(C.c_uint64)]),
    ("efg_bfs_end", C.c_int, [C.c_void_p, C.POINTER(Stats)]),
    ("efg_partition", C.c_int, [C.c_uint64, C.c_void_p, C.c_void_p, C.c_int, C.c_void_p]),
    ("efg_last_error", C.c_char_p, []),
    ("efg_version", C.c_char_p, []),
]


def load() -> C.CDLL:
    if not os.path.exists(LIB_PATH):
        raise ImportError(f"{LIB_PATH} is missing: build it with `python __graft_entry__.py` "
                          "(there is no CPU fallback)")
    lib = C.CDLL(LIB_PATH)
    for name, res, args in SIGNATURES:
        fn = getattr(lib, name)
        fn.restype = res
        fn.argtypes = args
    return lib


lib = load()


class EFGError(RuntimeError):
    def __init__(self, status: int, where: str):
        msg = lib.efg_last_error().decode(errors="replace")
        super().__init__(f"{where}: {STATUS_NAMES.get(status, status)}: {msg}")
        self.status = status


def check(status: int, where: str) -> None:
    if status != EFG_OK:
        raise EFGError(status, where)
