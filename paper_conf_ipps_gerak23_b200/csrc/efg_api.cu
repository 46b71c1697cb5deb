// efg_api.cu — the C ABI (include/efg.h): handle lifetime, device upload, the
// BFS level loop (L5 driver) and the decode hook.
#include <cuda_runtime.h>

#include <algorithm>
#include <chrono>
#include <cstring>
#include <new>
#include <string>
#include <vector>

#include "efg_internal.h"
#include "efg_kernels.cuh"

#include <nvtx3/nvToolsExt.h>  // header-only NVTX v3: no-ops unless a profiler injects itself

namespace {
// NVTX range over one C-ABI call (tracing): ncu --nvtx / Nsight
// Systems show every efg_* call of the host timeline by name
struct NvtxRange {
    explicit NvtxRange(const char *name) { nvtxRangePushA(name); }
    ~NvtxRange() { nvtxRangePop(); }
    NvtxRange(const NvtxRange &) = delete;
    NvtxRange &operator=(const NvtxRange &) = delete;
};
}  // namespace

using namespace efg;

#define CUDA_TRY(expr)                                                                         \
    do {                                                                                       \
        cudaError_t _e = (expr);                                                               \
        if (_e != cudaSuccess)                                                                 \
            return set_error(EFG_ECUDA, std::string(#expr) + ": " + cudaGetErrorString(_e)); \
    } while (0)

#define EFG_TRY(expr)                \
    do {                             \
        efg_status _s = (expr);      \
        if (_s != EFG_OK) return _s; \
    } while (0)

namespace {

// a handle of a 1-D row partition (efg_build_opts.row_lo / row_hi)
bool partitioned(const efg_graph *g) { return !(g->host.row_lo == 0 && g->host.row_hi == g->host.n); }

efg_status check_handle(efg_graph *g)
{
    if (!g) return set_error(EFG_EINVAL, "null handle");
    if (!g->on_device) return set_error(EFG_ESTATE, "host-only handle (built with device = -1)");
    return EFG_OK;
}

}  // namespace

extern "C" void efg_default_opts(efg_build_opts *o)
{
    if (!o) return;
    std::memset(o, 0, sizeof(*o));
    o->fwd_quantum = 512;
    o->flags = EFG_DEFAULT_FLAGS;
    o->device = 0;
}

namespace {

// common part of efg_build / efg_build_stream: options, host build, upload
template <class HostBuild>
efg_status build_common(uint64_t n, const efg_build_opts *opts, efg_graph **out, HostBuild &&host_build)
{
    if (!out) return set_error(EFG_EINVAL, "efg_build: out is NULL");
    *out = nullptr;
    efg_build_opts o;
    if (opts)
        o = *opts;
    else
        efg_default_opts(&o);
    if (n == 0 || n > 0xFFFFFFFFull) return set_error(EFG_EINVAL, "efg_build: need 1 <= n <= 2^32-1");
    if (o.row_hi > o.row_lo && (o.row_lo % 64 || (o.row_hi % 64 && o.row_hi < n)))
        return set_error(EFG_EINVAL, "efg_build: row range bounds must be multiples of 64 (or n)");
    efg_graph *g = new (std::nothrow) efg_graph();
    if (!g) return set_error(EFG_ENOMEM, "efg_build: handle allocation failed");
    efg_status st = host_build(o, g->host);
    if (st != EFG_OK) {
        delete g;
        return st;
    }
    if (o.device >= 0) {
        st = device_upload(g, o);
        if (st != EFG_OK) {
            device_free(g->dev);
            delete g;
            return st;
        }
        g->on_device = true;
    }
    *out = g;
    return EFG_OK;
}

}  // namespace

extern "C" efg_status efg_build(uint64_t n, uint64_t m, const uint32_t *src, const uint32_t *dst,
                                const efg_build_opts *opts, efg_graph **out)
{
    NvtxRange nvtx_range("efg_build");
    clear_error();
    if (m && (!src || !dst)) {
        if (out) *out = nullptr;
        return set_error(EFG_EINVAL, "efg_build: src/dst is NULL");
    }
    return build_common(n, opts, out, [&](const efg_build_opts &o, HostEFG &h) {
        return build_host(n, m, src, dst, o, h);
    });
}

extern "C" efg_status efg_build_stream(uint64_t n, uint64_t m, efg_edge_gen_fn gen, void *user, int weighted,
                                       const efg_build_opts *opts, efg_graph **out)
{
    NvtxRange nvtx_range("efg_build_stream");
    clear_error();
    if (m && !gen) {
        if (out) *out = nullptr;
        return set_error(EFG_EINVAL, "efg_build_stream: gen is NULL");
    }
    return build_common(n, opts, out, [&](const efg_build_opts &o, HostEFG &h) {
        efg_build_opts o2 = o;
        o2.weights = nullptr;
        return build_host_stream(n, m, gen, user, weighted, o2, h);
    });
}

extern "C" efg_status efg_save(const efg_graph *g, const char *path)
{
    NvtxRange nvtx_range("efg_save");
    clear_error();
    if (!g || !path) return set_error(EFG_EINVAL, "efg_save: null handle or path");
    return save_host(g->host, path);
}

extern "C" efg_status efg_load(const char *path, const efg_build_opts *opts, efg_graph **out)
{
    NvtxRange nvtx_range("efg_load");
    clear_error();
    if (!path) {
        if (out) *out = nullptr;
        return set_error(EFG_EINVAL, "efg_load: path is NULL");
    }
    efg_build_opts o;
    if (opts)
        o = *opts;
    else
        efg_default_opts(&o);
    o.row_lo = o.row_hi = 0;  // the file's row range applies
    o.weights = nullptr;
    return build_common(1, &o, out, [&](const efg_build_opts &, HostEFG &h) { return load_host(path, h); });
}

extern "C" void efg_free(efg_graph *g)
{
    if (!g) return;
    if (g->on_device) device_free(g->dev);
    delete g;
}

extern "C" efg_status efg_info(const efg_graph *g, efg_info_t *info)
{
    clear_error();
    if (!g || !info) return set_error(EFG_EINVAL, "efg_info: null argument");
    const HostEFG &h = g->host;
    std::memset(info, 0, sizeof(*info));
    info->n = h.n;
    info->m = h.m;
    info->m_input = h.m_input;
    info->fwd_quantum = h.k;
    info->device = g->on_device ? (uint32_t)g->dev.device : 0xFFFFFFFFu;
    info->data_bytes = h.offsets.empty() ? 0 : h.offsets[h.n];
    info->fwd_bytes = h.fwd_bytes;
    info->lower_bytes = h.lower_bytes;
    info->upper_bytes = h.upper_bytes;
    info->apriori_bits = h.apriori_bits;
    info->vertex_bytes = 17 * h.n + 16;
    info->device_bytes = g->on_device ? g->dev.device_bytes : 0;
    info->row_lo = h.row_lo;
    info->row_hi = h.row_hi;
    info->build_seconds = h.build_seconds;
    info->device_quantum = g->on_device ? g->dev.k : 0;
    info->data_location = (g->on_device && g->dev.data_host) ? 1u : 0u;
    return EFG_OK;
}

extern "C" efg_status efg_export(const efg_graph *g, uint64_t *vlist, uint8_t *nlb, uint64_t *offsets,
                                 uint8_t *data)
{
    clear_error();
    if (!g) return set_error(EFG_EINVAL, "efg_export: null handle");
    const HostEFG &h = g->host;
    if (vlist) std::memcpy(vlist, h.vlist.data(), (h.n + 1) * 8);
    if (nlb) std::memcpy(nlb, h.nlb.data(), h.n);
    if (offsets) std::memcpy(offsets, h.offsets.data(), (h.n + 1) * 8);
    if (data && !h.data.empty()) std::memcpy(data, h.data.data(), h.data.size());
    return EFG_OK;
}

extern "C" efg_status efg_export_perm(const efg_graph *g, uint32_t *old_of_new)
{
    clear_error();
    if (!g || !old_of_new) return set_error(EFG_EINVAL, "efg_export_perm: null argument");
    const HostEFG &h = g->host;
    if (h.old_of_new.empty()) {
        for (uint64_t i = 0; i < h.n; ++i) old_of_new[i] = (uint32_t)i;
    } else {
        std::memcpy(old_of_new, h.old_of_new.data(), h.n * 4);
    }
    return EFG_OK;
}

extern "C" efg_status efg_decode(efg_graph *g, uint32_t v0, uint32_t v1, uint32_t *out)
{
    NvtxRange nvtx_range("efg_decode");
    clear_error();
    EFG_TRY(check_handle(g));
    const HostEFG &h = g->host;
    if (v0 > v1 || v1 > h.n) return set_error(EFG_ERANGE, "efg_decode: bad vertex range");
    if (h.vlist[v1] == h.vlist[v0]) return EFG_OK;
    if (!out) return set_error(EFG_EINVAL, "efg_decode: out is NULL");
    return device_decode(g, v0, v1, out);
}

extern "C" efg_status efg_bfs(efg_graph *g, uint32_t source, int32_t *depth, uint32_t *parent, efg_stats *st)
{
    NvtxRange nvtx_range("efg_bfs");
    clear_error();
    EFG_TRY(check_handle(g));
    if (source >= g->dev.n) return set_error(EFG_ERANGE, "efg_bfs: source >= n");
    if (!depth) return set_error(EFG_EINVAL, "efg_bfs: depth is NULL");
    const uint32_t s = g->host.new_of_old.empty() ? source : g->host.new_of_old[source];
    return device_bfs(g, s, depth, parent, st);
}

extern "C" efg_status efg_set_option(efg_graph *g, int option, int64_t value)
{
    clear_error();
    EFG_TRY(check_handle(g));
    switch (option) {
    case EFG_OPT_LEVEL_LOOP:
        if (value != 0 && value != 1) return set_error(EFG_EINVAL, "EFG_OPT_LEVEL_LOOP: 0 or 1");
        g->dev.level_loop = (int)value;
        return EFG_OK;
    case EFG_OPT_PAGERANK_PULL:
        if (value != 0 && value != 1) return set_error(EFG_EINVAL, "EFG_OPT_PAGERANK_PULL: 0 or 1");
        g->dev.pr_pull = (int)value;
        return EFG_OK;
    case EFG_OPT_PREFIX_SKIP:
        if (value != 0 && value != 1) return set_error(EFG_EINVAL, "EFG_OPT_PREFIX_SKIP: 0 or 1");
        if (g->dev.prefix_skip != (int)value) {
            g->dev.prefix_skip = (int)value;
            efg::device_drop_graphs(g->dev);  // the captured level loops carry the old value
        }
        return EFG_OK;
    case EFG_OPT_EXPAND_VARIANT:
        if (value < 0 || value > 127) return set_error(EFG_EINVAL, "EFG_OPT_EXPAND_VARIANT: 0..127");
        if (g->dev.expand_variant != (int)value) {
            g->dev.expand_variant = (int)value;
            efg::device_drop_graphs(g->dev);
        }
        return EFG_OK;
    default:
        return set_error(EFG_EINVAL, "efg_set_option: unknown option");
    }
}

extern "C" efg_status efg_sssp(efg_graph *g, uint32_t source, float *dist, efg_stats *st)
{
    NvtxRange nvtx_range("efg_sssp");
    clear_error();
    EFG_TRY(check_handle(g));
    if (source >= g->dev.n) return set_error(EFG_ERANGE, "efg_sssp: source >= n");
    if (!dist) return set_error(EFG_EINVAL, "efg_sssp: dist is NULL");
    if (!g->dev.weights && g->host.m) return set_error(EFG_EINVAL, "efg_sssp: graph built without weights");
    if (partitioned(g)) return set_error(EFG_ENOTSUP, "efg_sssp: not available on a partitioned (row-range) handle");
    const uint32_t s = g->host.new_of_old.empty() ? source : g->host.new_of_old[source];
    return device_sssp(g, s, dist, st);
}

extern "C" efg_status efg_pagerank(efg_graph *g, double damping, uint32_t iters, double *rank, efg_stats *st)
{
    NvtxRange nvtx_range("efg_pagerank");
    clear_error();
    EFG_TRY(check_handle(g));
    if (!rank) return set_error(EFG_EINVAL, "efg_pagerank: rank is NULL");
    if (!(damping >= 0.0 && damping <= 1.0)) return set_error(EFG_EINVAL, "efg_pagerank: damping outside [0,1]");
    if (partitioned(g)) return set_error(EFG_ENOTSUP, "efg_pagerank: not available on a partitioned (row-range) handle");
    return device_pagerank(g, damping, iters, rank, st);
}

extern "C" efg_status efg_xchg_geometry(const efg_graph *g, int world, const uint64_t *bounds, uint64_t *slice_words)
{
    clear_error();
    if (!g || !bounds || !slice_words || world < 1) return set_error(EFG_EINVAL, "efg_xchg_geometry: bad args");
    uint64_t s = 0;
    for (int r = 0; r < world; ++r) {
        if (bounds[r + 1] < bounds[r] || bounds[r] % 64) return set_error(EFG_EINVAL, "efg_xchg_geometry: bounds");
        const uint64_t w0 = bounds[r] / 32, w1 = (bounds[r + 1] + 31) / 32;
        s = std::max<uint64_t>(s, w1 - w0);
    }
    *slice_words = s;
    return EFG_OK;
}

extern "C" efg_status efg_bfs_begin(efg_graph *g, uint32_t source, int32_t *depth_device)
{
    NvtxRange nvtx_range("efg_bfs_begin");
    clear_error();
    EFG_TRY(check_handle(g));
    if (source >= g->dev.n) return set_error(EFG_ERANGE, "efg_bfs_begin: source >= n");
    if (!depth_device) return set_error(EFG_EINVAL, "efg_bfs_begin: depth is NULL");
    const uint32_t s = g->host.new_of_old.empty() ? source : g->host.new_of_old[source];
    return device_step_begin(g, s, depth_device);
}

extern "C" efg_status efg_bfs_expand(efg_graph *g)
{
    NvtxRange nvtx_range("efg_bfs_expand");
    clear_error();
    EFG_TRY(check_handle(g));
    return device_step_expand(g);
}

extern "C" efg_status efg_xchg_pack(efg_graph *g, int world, const uint64_t *bounds, uint64_t slice_words,
                                    uint32_t *send)
{
    NvtxRange nvtx_range("efg_xchg_pack");
    clear_error();
    EFG_TRY(check_handle(g));
    if (world < 1 || !bounds || !send) return set_error(EFG_EINVAL, "efg_xchg_pack: bad args");
    return device_xchg(g, 0, world, bounds, slice_words, send, nullptr);
}

extern "C" efg_status efg_xchg_reduce(efg_graph *g, int world, uint64_t slice_words, const uint32_t *recv,
                                      uint32_t *mine)
{
    NvtxRange nvtx_range("efg_xchg_reduce");
    clear_error();
    EFG_TRY(check_handle(g));
    if (world < 1 || !recv || !mine) return set_error(EFG_EINVAL, "efg_xchg_reduce: bad args");
    return device_xchg(g, 1, world, nullptr, slice_words, mine, recv);
}

extern "C" efg_status efg_xchg_unpack(efg_graph *g, int world, const uint64_t *bounds, uint64_t slice_words,
                                      const uint32_t *gathered)
{
    NvtxRange nvtx_range("efg_xchg_unpack");
    clear_error();
    EFG_TRY(check_handle(g));
    if (world < 1 || !bounds || !gathered) return set_error(EFG_EINVAL, "efg_xchg_unpack: bad args");
    return device_xchg(g, 2, world, bounds, slice_words, nullptr, gathered);
}

extern "C" efg_status efg_peer_alloc(efg_graph *g, int world, void **region, uint8_t *ipc_handle)
{
    NvtxRange nvtx_range("efg_peer_alloc");
    clear_error();
    EFG_TRY(check_handle(g));
    if (world < 1 || world > kPeerMaxWorld) return set_error(EFG_EINVAL, "efg_peer_alloc: world outside [1, 64]");
    return device_peer_alloc(g, world, region, ipc_handle);
}

extern "C" efg_status efg_peer_open(efg_graph *g, int world, int rank, const uint64_t *bounds,
                                    const uint8_t *ipc_handles, void *const *regions)
{
    NvtxRange nvtx_range("efg_peer_open");
    clear_error();
    EFG_TRY(check_handle(g));
    if (world < 1 || world > kPeerMaxWorld || rank < 0 || rank >= world || !bounds ||
        (ipc_handles == nullptr) == (regions == nullptr))
        return set_error(EFG_EINVAL, "efg_peer_open: bad args");
    return device_peer_open(g, world, rank, bounds, ipc_handles, regions);
}

extern "C" efg_status efg_xchg_peer(efg_graph *g)
{
    NvtxRange nvtx_range("efg_xchg_peer");
    clear_error();
    EFG_TRY(check_handle(g));
    return device_xchg_peer(g);
}

extern "C" efg_status efg_xchg_peer_phase(efg_graph *g, int phase)
{
    NvtxRange nvtx_range("efg_xchg_peer_phase");
    clear_error();
    EFG_TRY(check_handle(g));
    if (phase < 0 || phase > 2) return set_error(EFG_EINVAL, "efg_xchg_peer_phase: phase 0..2");
    return device_xchg_peer_phase(g, phase);
}

extern "C" efg_status efg_bfs_finish_level(efg_graph *g, uint64_t *global_new)
{
    NvtxRange nvtx_range("efg_bfs_finish_level");
    clear_error();
    EFG_TRY(check_handle(g));
    return device_step_finish(g, global_new);
}

extern "C" efg_status efg_bfs_end(efg_graph *g, efg_stats *st)
{
    NvtxRange nvtx_range("efg_bfs_end");
    clear_error();
    EFG_TRY(check_handle(g));
    return device_step_end(g, st);
}

extern "C" efg_status efg_partition(uint64_t n, const uint64_t *vlist, const uint64_t *offsets, int world,
                                    uint64_t *bounds)
{
    NvtxRange nvtx_range("efg_partition");
    clear_error();
    if (!vlist || !offsets || !bounds || world < 1 || n == 0) return set_error(EFG_EINVAL, "efg_partition: bad args");
    // weight of a vertex: compressed bytes + 29 bytes of per-vertex state
    const double total = (double)offsets[n] + 29.0 * (double)n;
    bounds[0] = 0;
    uint64_t v = 0;
    double acc = 0.0;
    for (int r = 1; r < world; ++r) {
        const double target = total * r / world;
        while (v < n && acc + (double)(offsets[v + 1] - offsets[v]) + 29.0 <= target) {
            acc += (double)(offsets[v + 1] - offsets[v]) + 29.0;
            ++v;
        }
        uint64_t b = (v + 32) / 64 * 64;  // round to a multiple of 64
        b = std::min<uint64_t>(std::max<uint64_t>(b, bounds[r - 1]), n);
        bounds[r] = b;
    }
    bounds[world] = n;
    (void)vlist;
    return EFG_OK;
}
