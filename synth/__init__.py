"""synth — seeded synthetic input generators (inputs only).

ctypes wrapper over ``synth/libsynth.so`` (``synth/gen.c``).  Serves both the
oracle tests and the CUDA path; holds none of the method's arithmetic (no
Elias-Fano coding, CSR construction or traversal).  Every array is a pure
function of its parameters and seed (counter-based splitmix64 streams).

The workload recipes are named by BASELINE.json
config index: ``config_edges(1)`` = RMAT scale 16 / ef 16, ``config_edges(2)``
= RMAT scale 24 / ef 16, ... Seeds per SURVEY §8(d): generator c, permutation
100+c, sources 1000+c, weights 2000+c.
"""
from __future__ import annotations

import ctypes as C
import os

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_LIB_PATH = os.path.join(_HERE, "libsynth.so")
_lib = None

u64p = C.POINTER(C.c_uint64)
u32p = C.POINTER(C.c_uint32)
f32p = C.POINTER(C.c_float)

RMAT_ABC = (0.57, 0.19, 0.19)


def _ptr(a, t):
    return a.ctypes.data_as(t)


def lib():
    global _lib
    if _lib is None:
        if not os.path.exists(_LIB_PATH):
            raise RuntimeError(f"{_LIB_PATH} missing: run __graft_entry__.build()")
        L = C.CDLL(_LIB_PATH)
        L.synth_splitmix64.restype = C.c_uint64
        L.synth_splitmix64.argtypes = [C.c_uint64]
        L.synth_draw.restype = C.c_uint64
        L.synth_draw.argtypes = [C.c_uint64, C.c_uint64, C.c_uint64]
        L.synth_rmat.restype = None
        L.synth_rmat.argtypes = [C.c_int, C.c_uint64, C.c_double, C.c_double, C.c_double,
                                 C.c_uint64, u32p, u32p]
        L.synth_uniform.restype = None
        L.synth_uniform.argtypes = [C.c_uint64, C.c_uint64, C.c_uint64, u32p, u32p]
        L.synth_permutation.restype = None
        L.synth_permutation.argtypes = [C.c_uint64, C.c_uint64, u32p]
        L.synth_apply_permutation.restype = None
        L.synth_apply_permutation.argtypes = [C.c_uint64, u32p, u32p, u32p]
        L.synth_chunglu.restype = None
        L.synth_chunglu.argtypes = [C.c_uint64, C.c_uint64, C.c_double, C.c_double, C.c_double,
                                    C.c_uint64, u32p, u32p]
        L.synth_web_hosts.restype = C.c_uint64
        L.synth_web_hosts.argtypes = [C.c_uint64, C.c_double, C.c_double, C.c_uint64, C.c_uint64, u64p,
                                      C.c_uint64]
        L.synth_gen_range.restype = None
        L.synth_gen_range.argtypes = [C.c_void_p, C.c_uint64, C.c_uint64, u32p, u32p, f32p]
        L.synth_web_host_of.restype = None
        L.synth_web_host_of.argtypes = [C.c_uint64, u64p, u32p]
        L.synth_web.restype = None
        L.synth_web.argtypes = [C.c_uint64, C.c_uint64, u64p, C.c_uint64, u32p, C.c_double,
                                C.c_double, C.c_double, C.c_uint64, u32p, u32p]
        L.synth_weights.restype = None
        L.synth_weights.argtypes = [C.c_uint64, u32p, u32p, C.c_uint64, f32p]
        L.synth_weight_pair.restype = C.c_float
        L.synth_weight_pair.argtypes = [C.c_uint64, C.c_uint32, C.c_uint32]
        _lib = L
    return _lib


def rmat(scale: int, edgefactor: int, seed: int, abc=RMAT_ABC):
    """Graph500 R-MAT: n = 2**scale, m = edgefactor * n undirected samples."""
    n = 1 << scale
    m = edgefactor * n
    src = np.empty(m, np.uint32)
    dst = np.empty(m, np.uint32)
    lib().synth_rmat(scale, m, abc[0], abc[1], abc[2], seed, _ptr(src, u32p), _ptr(dst, u32p))
    return n, src, dst


def uniform(n: int, m: int, seed: int):
    src = np.empty(m, np.uint32)
    dst = np.empty(m, np.uint32)
    lib().synth_uniform(n, m, seed, _ptr(src, u32p), _ptr(dst, u32p))
    return n, src, dst


def permutation(n: int, seed: int) -> np.ndarray:
    p = np.empty(n, np.uint32)
    lib().synth_permutation(n, seed, _ptr(p, u32p))
    return p


def apply_permutation(perm, src, dst):
    lib().synth_apply_permutation(src.size, _ptr(perm, u32p), _ptr(src, u32p), _ptr(dst, u32p))


def chunglu(n: int, m: int, alpha_src: float, alpha_dst: float, rho: float, seed: int):
    src = np.empty(m, np.uint32)
    dst = np.empty(m, np.uint32)
    lib().synth_chunglu(n, m, alpha_src, alpha_dst, rho, seed, _ptr(src, u32p), _ptr(dst, u32p))
    return n, src, dst


WEB_HOST_XM = 100.0 / 3.0  # Pareto(1.5) host sizes with mean ~100 pages


def web(n: int, m: int, seed: int, pareto_alpha=1.5, host_cap=20000, p_intra=0.85,
        p_near=0.10, zipf_alpha=1.4, host_xm=WEB_HOST_XM):
    max_hosts = n
    hs = np.zeros(max_hosts + 1, np.uint64)
    nh = lib().synth_web_hosts(n, pareto_alpha, host_xm, host_cap, seed, _ptr(hs, u64p), max_hosts)
    hs = np.ascontiguousarray(hs[:nh + 1])
    host_of = np.empty(n, np.uint32)
    lib().synth_web_host_of(nh, _ptr(hs, u64p), _ptr(host_of, u32p))
    src = np.empty(m, np.uint32)
    dst = np.empty(m, np.uint32)
    lib().synth_web(n, m, _ptr(hs, u64p), nh, _ptr(host_of, u32p), p_intra, p_near, zipf_alpha,
                    seed, _ptr(src, u32p), _ptr(dst, u32p))
    return n, src, dst


def weights(src, dst, seed: int) -> np.ndarray:
    w = np.empty(src.size, np.float32)
    lib().synth_weights(src.size, _ptr(src, u32p), _ptr(dst, u32p), seed, _ptr(w, f32p))
    return w


def weight_pair(seed: int, u: int, v: int) -> float:
    return float(lib().synth_weight_pair(seed, u, v))


def sources(n: int, count: int, seed: int, nonisolated_mask=None) -> np.ndarray:
    """`count` source vertices drawn with the counter stream (reading C19: among
    vertices with degree > 0 when a mask is given)."""
    L = lib()
    out = []
    j = 0
    while len(out) < count:
        r = L.synth_draw(seed, j, 99)
        v = int((r * n) >> 64)
        j += 1
        if nonisolated_mask is not None and not nonisolated_mask[v]:
            if j > 1000 * (count + 1):
                break
            continue
        out.append(v)
    return np.array(out, np.uint32)


# ---------------------------------------------------------------------------
# BASELINE.json configs
# ---------------------------------------------------------------------------
CONFIGS = {
    1: dict(name="rmat16_ef16", kind="rmat", scale=16, ef=16, permute=False),
    2: dict(name="rmat24_ef16", kind="rmat", scale=24, ef=16, permute=False),
    3: dict(name="twitter_like", kind="chunglu", n=41_652_230, m=1_468_365_182,
            alpha_src=0.85, alpha_dst=0.8, rho=0.18, permute=False),
    4: dict(name="web_like", kind="web", n=100_000_000, m=5_200_000_000, permute=False),
    5: dict(name="rmat29_ef32", kind="rmat", scale=29, ef=32, permute=True),
}


def config_edges(c: int, scale_override: int | None = None, permute: bool | None = None):
    """Return (n, src, dst) for BASELINE.json config index c (1-based)."""
    cfg = CONFIGS[c]
    perm_flag = cfg["permute"] if permute is None else permute
    if cfg["kind"] == "rmat":
        scale = scale_override if scale_override is not None else cfg["scale"]
        n, src, dst = rmat(scale, cfg["ef"], seed=c)
    elif cfg["kind"] == "chunglu":
        n, src, dst = chunglu(cfg["n"], cfg["m"], cfg["alpha_src"], cfg["alpha_dst"],
                              cfg["rho"], seed=c)
    elif cfg["kind"] == "web":
        n, src, dst = web(cfg["n"], cfg["m"], seed=c)
    else:
        raise ValueError(cfg)
    if perm_flag:
        apply_permutation(permutation(n, 100 + c), src, dst)
    return n, src, dst


# ---------------------------------------------------------------------------
# Streamed generation (efg_build_stream): samples produced on demand by range
# ---------------------------------------------------------------------------
class _GenCtx(C.Structure):
    _fields_ = [("kind", C.c_int), ("scale", C.c_int), ("n", C.c_uint64), ("seed", C.c_uint64),
                ("a", C.c_double), ("b", C.c_double), ("c", C.c_double),
                ("alpha_src", C.c_double), ("alpha_dst", C.c_double), ("rho", C.c_double),
                ("host_start", C.c_void_p), ("n_hosts", C.c_uint64), ("host_of", C.c_void_p),
                ("p_intra", C.c_double), ("p_near", C.c_double), ("zipf_alpha", C.c_double),
                ("perm", C.c_void_p), ("wseed", C.c_uint64)]


class StreamGen:
    """A config's edge generator as a C callback (synth_gen_range, the
    efg_edge_gen_fn signature): `fn` and `user` are raw addresses to hand to
    efg_build_stream; samples [first, first+count) equal the same indices of
    config_edges(c).  Keeps its arrays alive."""

    def __init__(self, n: int, m: int, ctx: _GenCtx, keep: list):
        self.n, self.m, self._ctx, self._keep = n, m, ctx, keep
        self.fn = C.cast(lib().synth_gen_range, C.c_void_p).value
        self.user = C.addressof(ctx)

    def range(self, first: int, count: int, weighted: bool = False):
        src = np.empty(count, np.uint32)
        dst = np.empty(count, np.uint32)
        w = np.empty(count, np.float32) if weighted else None
        lib().synth_gen_range(C.byref(self._ctx), first, count, _ptr(src, u32p), _ptr(dst, u32p),
                              _ptr(w, f32p) if weighted else None)
        return (src, dst, w) if weighted else (src, dst)


def config_stream(c: int, scale_override: int | None = None, permute: bool | None = None,
                  weight_seed: int | None = None) -> StreamGen:
    """StreamGen of BASELINE.json config c (same samples as config_edges)."""
    cfg = CONFIGS[c]
    perm_flag = cfg["permute"] if permute is None else permute
    ctx = _GenCtx()
    keep = []
    ctx.seed = c
    ctx.wseed = 2000 + c if weight_seed is None else weight_seed
    if cfg["kind"] == "rmat":
        scale = scale_override if scale_override is not None else cfg["scale"]
        n, m = 1 << scale, cfg["ef"] << scale
        ctx.kind, ctx.scale, ctx.n = 0, scale, n
        ctx.a, ctx.b, ctx.c = RMAT_ABC
    elif cfg["kind"] == "chunglu":
        n, m = cfg["n"], cfg["m"]
        ctx.kind, ctx.n = 1, n
        ctx.alpha_src, ctx.alpha_dst, ctx.rho = cfg["alpha_src"], cfg["alpha_dst"], cfg["rho"]
    elif cfg["kind"] == "web":
        n, m = cfg["n"], cfg["m"]
        hs = np.zeros(n + 1, np.uint64)
        nh = lib().synth_web_hosts(n, 1.5, WEB_HOST_XM, 20000, c, _ptr(hs, u64p), n)
        hs = np.ascontiguousarray(hs[:nh + 1])
        host_of = np.empty(n, np.uint32)
        lib().synth_web_host_of(nh, _ptr(hs, u64p), _ptr(host_of, u32p))
        keep += [hs, host_of]
        ctx.kind, ctx.n = 2, n
        ctx.host_start, ctx.n_hosts, ctx.host_of = hs.ctypes.data, nh, host_of.ctypes.data
        ctx.p_intra, ctx.p_near, ctx.zipf_alpha = 0.85, 0.10, 1.4
    else:
        raise ValueError(cfg)
    if perm_flag:
        p = permutation(n, 100 + c)
        keep.append(p)
        ctx.perm = p.ctypes.data
    return StreamGen(n, m, ctx, keep)
