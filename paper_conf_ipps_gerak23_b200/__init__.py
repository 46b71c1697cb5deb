"""paper_conf_ipps_gerak23_b200 — B200-native BFS over Elias-Fano-compressed graphs.

Python binding of the C ABI in ``include/efg.h`` (libefg.so).  This layer only
marshals arguments: buffers are passed as raw pointers (numpy arrays as host
pointers, torch CUDA tensors as device pointers) and every step of the path —
the host EFG builder and the sm_100a traversal kernels — runs in the library.

Paper: P. Gera, H. Kim, "Traversing Large Compressed Graphs on GPUs", IPDPS'23
(PAPER.md).  The method: EF-compress each sorted neighbour list and
decode lists inside the BFS frontier-expansion kernel.
"""
from __future__ import annotations

import ctypes as C
import os

import numpy as np

from . import _abi
from ._abi import (EFG_DEDUP, EFG_DEFAULT_FLAGS, EFG_DROP_SELF_LOOPS, EFG_HOST_RESIDENT,  # noqa: F401
                   EFG_REORDER_DEGREE, EFG_SYMMETRIZE, EFGError, check, lib)

__all__ = ["Graph", "EFGError", "EFG_DEFAULT_FLAGS", "EFG_SYMMETRIZE", "EFG_DEDUP",
           "EFG_DROP_SELF_LOOPS", "EFG_REORDER_DEGREE", "EFG_HOST_RESIDENT", "version", "partition"]


def version() -> str:
    return lib.efg_version().decode()


def _ptr(x):
    """Raw pointer of a numpy array (host) or a torch tensor (device or host)."""
    if x is None:
        return None
    if isinstance(x, np.ndarray):
        assert x.flags["C_CONTIGUOUS"]
        return x.ctypes.data
    return x.data_ptr()  # torch.Tensor


def _is_torch(x) -> bool:
    return type(x).__module__.startswith("torch")


class Graph:
    """Handle over an ``efg_graph`` (host EFG arrays + device copy)."""

    def __init__(self, handle: int, stream: int | None):
        self._h = C.c_void_p(handle)
        self.stream = stream
        self.info = self._info()

    # -- construction -----------------------------------------------------
    @classmethod
    def build(cls, n: int, src, dst, *, k: int = 512, flags: int = EFG_DEFAULT_FLAGS,
              device: int = 0, stream: int | None = None, weights=None, n_threads: int = 0,
              rows: tuple[int, int] | None = None):
        """efg_build: host edge arrays (uint32) -> EFG handle (uploaded to `device`).

        `stream` is a cudaStream_t as an int (e.g. ``torch.cuda.current_stream().cuda_stream``);
        None = the legacy default stream."""
        src = np.ascontiguousarray(src, dtype=np.uint32)
        dst = np.ascontiguousarray(dst, dtype=np.uint32)
        if src.shape != dst.shape:
            raise ValueError("src and dst differ in length")
        o = _abi.BuildOpts()
        lib.efg_default_opts(C.byref(o))
        o.fwd_quantum = k
        o.flags = flags
        o.device = device
        o.n_threads = n_threads
        o.stream = stream
        if rows is not None:
            o.row_lo, o.row_hi = int(rows[0]), int(rows[1])
        w = None
        if weights is not None:
            w = np.ascontiguousarray(weights, dtype=np.float32)
            if w.shape != src.shape:
                raise ValueError("weights must have one entry per input edge")
            o.weights = w.ctypes.data
        h = C.c_void_p()
        check(lib.efg_build(n, src.size, _ptr(src), _ptr(dst), C.byref(o), C.byref(h)), "efg_build")
        return cls(h.value, stream)

    @classmethod
    def build_stream(cls, n: int, m: int, gen_fn: int, gen_user: int, *, weighted: bool = False,
                     k: int = 512, flags: int = EFG_DEFAULT_FLAGS, device: int = 0,
                     stream: int | None = None, n_threads: int = 0, rows: tuple[int, int] | None = None):
        """efg_build_stream: edges produced on demand by a C callback (efg_edge_gen_fn
        address `gen_fn`, its context address `gen_user`), read twice in chunks; the
        edge list is never materialised."""
        o = _abi.BuildOpts()
        lib.efg_default_opts(C.byref(o))
        o.fwd_quantum = k
        o.flags = flags
        o.device = device
        o.n_threads = n_threads
        o.stream = stream
        if rows is not None:
            o.row_lo, o.row_hi = int(rows[0]), int(rows[1])
        h = C.c_void_p()
        check(lib.efg_build_stream(n, m, gen_fn, gen_user, 1 if weighted else 0, C.byref(o), C.byref(h)),
              "efg_build_stream")
        return cls(h.value, stream)

    def save(self, path: str) -> None:
        """efg_save: write the built graph to `path` (the on-disk EFG)."""
        check(lib.efg_save(self._h, os.fsencode(path)), "efg_save")

    @classmethod
    def load(cls, path: str, *, flags: int = 0, device: int = 0, stream: int | None = None):
        """efg_load: a graph saved with save(); `flags` may add EFG_HOST_RESIDENT,
        `device` = -1 keeps it host-only."""
        o = _abi.BuildOpts()
        lib.efg_default_opts(C.byref(o))
        o.flags = flags
        o.device = device
        o.stream = stream
        h = C.c_void_p()
        check(lib.efg_load(os.fsencode(path), C.byref(o), C.byref(h)), "efg_load")
        return cls(h.value, stream)

    def set_level_loop(self, host: bool) -> None:
        """EFG_OPT_LEVEL_LOOP: False = device-side CUDA-graph loop (default),
        True = host loop with per-level CUDA-event timing of the expand kernel."""
        check(lib.efg_set_option(self._h, _abi.EFG_OPT_LEVEL_LOOP, 1 if host else 0), "efg_set_option")

    def set_prefix_skip(self, on: bool) -> None:
        """EFG_OPT_PREFIX_SKIP: True (default) = BFS skips upper-bit words whose ids are
        all below the visited prefix; False = decode and probe every element."""
        check(lib.efg_set_option(self._h, _abi.EFG_OPT_PREFIX_SKIP, 1 if on else 0), "efg_set_option")

    def set_pagerank_pull(self, on: bool) -> None:
        """EFG_OPT_PAGERANK_PULL: True (default) = gather on symmetric graphs, False = push."""
        check(lib.efg_set_option(self._h, _abi.EFG_OPT_PAGERANK_PULL, 1 if on else 0), "efg_set_option")

    def set_expand_variant(self, mask: int) -> None:
        """EFG_OPT_EXPAND_VARIANT (A/B switch): bit 0 lane-per-chunk decode, bit 1 span staging."""
        check(lib.efg_set_option(self._h, _abi.EFG_OPT_EXPAND_VARIANT, int(mask)), "efg_set_option")

    def free(self) -> None:
        if self._h:
            lib.efg_free(self._h)
            self._h = C.c_void_p()

    def __del__(self):
        try:
            self.free()
        except Exception:
            pass

    # -- introspection ----------------------------------------------------
    def _info(self) -> dict:
        i = _abi.Info()
        check(lib.efg_info(self._h, C.byref(i)), "efg_info")
        return {f: getattr(i, f) for f, _ in _abi.Info._fields_}

    @property
    def n(self) -> int:
        return self.info["n"]

    @property
    def m(self) -> int:
        return self.info["m"]

    def perm(self) -> np.ndarray:
        """old_of_new relabelling (identity unless built with EFG_REORDER_DEGREE)."""
        p = np.empty(max(self.info["n"], 1), np.uint32)
        check(lib.efg_export_perm(self._h, _ptr(p)), "efg_export_perm")
        return p[:self.info["n"]]

    def export(self):
        """(vlist u64[n+1], num_lower_bits u8[n], offsets u64[n+1], data u8[]) — P:113."""
        n, nb = self.info["n"], self.info["data_bytes"]
        vlist = np.empty(n + 1, np.uint64)
        nlb = np.empty(n, np.uint8)
        offsets = np.empty(n + 1, np.uint64)
        data = np.empty(max(nb, 1), np.uint8)
        check(lib.efg_export(self._h, _ptr(vlist), _ptr(nlb), _ptr(offsets), _ptr(data)), "efg_export")
        return vlist, nlb, offsets, data[:nb]

    # -- hot path ---------------------------------------------------------
    def decode(self, v0: int, v1: int, out=None):
        """efg_decode: neighbour lists of [v0, v1) in CSR order (GPU decode)."""
        if out is None:
            vl = self.export()[0] if not hasattr(self, "_vlist") else self._vlist
            self._vlist = vl
            out = np.empty(max(int(vl[v1] - vl[v0]), 1), np.uint32)
            check(lib.efg_decode(self._h, v0, v1, _ptr(out)), "efg_decode")
            return out[:int(vl[v1] - vl[v0])]
        check(lib.efg_decode(self._h, v0, v1, _ptr(out)), "efg_decode")
        return out

    def bfs(self, source: int, depth=None, parent=None, stats: bool = False, level_cap: int = 256):
        """efg_bfs: depth (int32, host numpy or device torch) from `source`.

        parent: None, True (allocate a host array) or a buffer.  Returns depth,
        or (depth, parent, stats-dict) when parent/stats are requested."""
        n = self.info["n"]
        if depth is None:
            depth = np.empty(n, np.int32)
        par = None
        if parent is True:
            par = np.empty(n, np.uint32)
        elif parent is not None and parent is not False:
            par = parent
        st = None
        arrs = None
        if stats:
            st = _abi.Stats()
            st.level_cap = level_cap
            arrs = (np.zeros(level_cap, np.uint64), np.zeros(level_cap, np.uint64),
                    np.zeros(level_cap, np.float32), np.zeros(level_cap, np.float32))
            st.level_frontier = arrs[0].ctypes.data
            st.level_edges = arrs[1].ctypes.data
            st.level_expand_ms = arrs[2].ctypes.data
            st.level_end_ms = arrs[3].ctypes.data
        check(lib.efg_bfs(self._h, source, _ptr(depth), _ptr(par),
                          C.byref(st) if st is not None else None), "efg_bfs")
        if not stats and par is None:
            return depth
        sd = None
        if stats:
            L = st.levels
            sd = {"levels": L, "edges_traversed": st.edges_traversed,
                  "vertices_reached": st.vertices_reached, "device_ms": st.device_ms,
                  "expand_ms": st.expand_ms, "expand_launches": st.expand_launches,
                  "kernel_launches": st.kernel_launches, "d2h_bytes": st.d2h_bytes,
                  "xchg_sparse_levels": st.xchg_sparse_levels,
                  "level_frontier": arrs[0][:min(L, level_cap)].copy(),
                  "level_edges": arrs[1][:min(L, level_cap)].copy(),
                  "level_expand_ms": arrs[2][:min(L, level_cap)].copy(),
                  "level_end_ms": arrs[3][:min(L, level_cap)].copy()}
        return depth, par, sd

    # -- stepwise partitioned BFS (efg.h "multi-GPU"); device buffers only --
    def xchg_geometry(self, bounds: np.ndarray) -> int:
        b = np.ascontiguousarray(bounds, np.uint64)
        S = C.c_uint64()
        check(lib.efg_xchg_geometry(self._h, b.size - 1, _ptr(b), C.byref(S)), "efg_xchg_geometry")
        return S.value

    def bfs_begin(self, source: int, depth) -> None:
        check(lib.efg_bfs_begin(self._h, source, _ptr(depth)), "efg_bfs_begin")

    def bfs_expand(self) -> None:
        check(lib.efg_bfs_expand(self._h), "efg_bfs_expand")

    def xchg_pack(self, bounds: np.ndarray, S: int, send) -> None:
        b = np.ascontiguousarray(bounds, np.uint64)
        check(lib.efg_xchg_pack(self._h, b.size - 1, _ptr(b), S, _ptr(send)), "efg_xchg_pack")

    def xchg_reduce(self, world: int, S: int, recv, mine) -> None:
        check(lib.efg_xchg_reduce(self._h, world, S, _ptr(recv), _ptr(mine)), "efg_xchg_reduce")

    def xchg_unpack(self, bounds: np.ndarray, S: int, gathered) -> None:
        b = np.ascontiguousarray(bounds, np.uint64)
        check(lib.efg_xchg_unpack(self._h, b.size - 1, _ptr(b), S, _ptr(gathered)), "efg_xchg_unpack")

    # -- the same exchange over peer memory (efg_peer_alloc / _open / efg_xchg_peer) --
    def peer_alloc(self, world: int) -> tuple[int, bytes]:
        """Allocate this rank's exchange region; returns (device address, 64-byte IPC handle)."""
        reg = C.c_void_p()
        h = (C.c_uint8 * 64)()
        check(lib.efg_peer_alloc(self._h, world, C.byref(reg), h), "efg_peer_alloc")
        return int(reg.value or 0), bytes(h)

    def peer_open(self, rank: int, bounds: np.ndarray, *, handles: list[bytes] | None = None,
                  regions: list[int] | None = None) -> None:
        """Map every rank's region: IPC handles (one process per GPU) or, for
        handles sharing one process, their device addresses."""
        b = np.ascontiguousarray(bounds, np.uint64)
        world = b.size - 1
        if (handles is None) == (regions is None):
            raise ValueError("peer_open: pass exactly one of handles / regions")
        if handles is not None:
            hb = np.frombuffer(b"".join(handles), np.uint8).copy()
            check(lib.efg_peer_open(self._h, world, rank, _ptr(b), _ptr(hb), None), "efg_peer_open")
        else:
            rg = (C.c_void_p * world)(*regions)
            check(lib.efg_peer_open(self._h, world, rank, _ptr(b), None, rg), "efg_peer_open")

    def xchg_peer(self) -> None:
        check(lib.efg_xchg_peer(self._h), "efg_xchg_peer")

    def xchg_peer_phase(self, phase: int) -> None:
        """One phase of the peer exchange without device barriers (0 publish,
        1 owner OR + broadcast, 2 unpack); returns after the stream is idle —
        the caller orders the phases across ranks with a host barrier."""
        check(lib.efg_xchg_peer_phase(self._h, phase), "efg_xchg_peer_phase")

    def bfs_finish_level(self) -> int:
        n = C.c_uint64()
        check(lib.efg_bfs_finish_level(self._h, C.byref(n)), "efg_bfs_finish_level")
        return n.value

    def bfs_end(self, level_cap: int = 256) -> dict:
        st = _abi.Stats()
        st.level_cap = level_cap
        lf, le = np.zeros(level_cap, np.uint64), np.zeros(level_cap, np.uint64)
        st.level_frontier, st.level_edges = lf.ctypes.data, le.ctypes.data
        check(lib.efg_bfs_end(self._h, C.byref(st)), "efg_bfs_end")
        L = min(st.levels + 1, level_cap)
        return {"levels": st.levels, "edges_traversed": st.edges_traversed,
                "vertices_reached": st.vertices_reached, "kernel_launches": st.kernel_launches,
                "xchg_sparse_levels": st.xchg_sparse_levels,
                "level_frontier": lf[:L].copy(), "level_edges": le[:L].copy()}

    def sssp(self, source: int, dist=None, stats: bool = False):
        n = self.info["n"]
        if dist is None:
            dist = np.empty(n, np.float32)
        st = _abi.Stats() if stats else None
        check(lib.efg_sssp(self._h, source, _ptr(dist), C.byref(st) if st else None), "efg_sssp")
        if not stats:
            return dist
        return dist, {"iterations": st.levels, "edges_relaxed": st.edges_traversed,
                      "device_ms": st.device_ms}

    def pagerank(self, damping: float = 0.85, iters: int = 50, rank=None):
        n = self.info["n"]
        if rank is None:
            rank = np.empty(n, np.float64)
        check(lib.efg_pagerank(self._h, damping, iters, _ptr(rank), None), "efg_pagerank")
        return rank


def partition(vlist: np.ndarray, offsets: np.ndarray, world: int) -> np.ndarray:
    """efg_partition: 1-D row ranges balanced by compressed bytes."""
    n = vlist.size - 1
    b = np.empty(world + 1, np.uint64)
    vl = np.ascontiguousarray(vlist, np.uint64)
    of = np.ascontiguousarray(offsets, np.uint64)
    check(lib.efg_partition(n, _ptr(vl), _ptr(of), world, _ptr(b)), "efg_partition")
    return b
