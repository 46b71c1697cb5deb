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

using namespace efg;

#define CUDA_TRY(expr)                                                                         \
    do {                                                                                       \
        cudaError_t _e = (expr);                                                               \
        if (_e != cudaSuccess)                                                                 \
            return set_error(EFG_ECUDA, std::string(#expr) + ": " + cudaGetErrorString(_e)); \
    } while (0)

namespace {

bool is_device_ptr(const void *p)
{
    cudaPointerAttributes at;
    if (cudaPointerGetAttributes(&at, p) != cudaSuccess) {
        cudaGetLastError();
        return false;
    }
    return at.type == cudaMemoryTypeDevice || at.type == cudaMemoryTypeManaged;
}

template <typename T>
efg_status dev_alloc(DeviceGraph &d, T **p, uint64_t count)
{
    const size_t bytes = std::max<uint64_t>(count, 1) * sizeof(T);
    cudaError_t e = cudaMalloc(reinterpret_cast<void **>(p), bytes);
    if (e != cudaSuccess) {
        cudaGetLastError();
        *p = nullptr;
        return set_error(e == cudaErrorMemoryAllocation ? EFG_ENOMEM : EFG_ECUDA,
                         std::string("cudaMalloc(") + std::to_string(bytes) + "): " + cudaGetErrorString(e));
    }
    d.device_bytes += bytes;
    return EFG_OK;
}

#define EFG_TRY(expr)                        \
    do {                                     \
        efg_status _s = (expr);              \
        if (_s != EFG_OK) return _s;         \
    } while (0)

void free_device(DeviceGraph &d)
{
    if (d.device >= 0) cudaSetDevice(d.device);
    cudaFree(d.data);
    cudaFree(d.rec);
    cudaFree(d.deg32);
    cudaFree(d.vlist);
    cudaFree(d.weights);
    cudaFree(d.vis);
    cudaFree(d.prev);
    cudaFree(d.queue);
    cudaFree(d.tiles);
    cudaFree(d.depth);
    cudaFree(d.parent);
    cudaFree(d.status);
    cudaFree(d.ctrl);
    cudaFree(d.fbuf);
    cudaFree(d.dbuf);
    if (d.ctrl_host) cudaFreeHost(d.ctrl_host);
    d = DeviceGraph{};
}

efg_status upload(efg_graph *g, const efg_build_opts &o)
{
    DeviceGraph &d = g->dev;
    const HostEFG &h = g->host;
    CUDA_TRY(cudaSetDevice(o.device));
    d.device = o.device;
    d.stream = o.stream;
    d.n = h.n;
    d.k = h.k;
    cudaStream_t s = static_cast<cudaStream_t>(o.stream);
    cudaDeviceProp prop;
    CUDA_TRY(cudaGetDeviceProperties(&prop, o.device));
    d.num_sms = prop.multiProcessorCount;

    // EF data, padded so 32-bit word reads past the last list stay in bounds
    d.data_bytes = h.data.size();
    const uint64_t padded = ((d.data_bytes + 64) + 15) & ~15ull;
    EFG_TRY(dev_alloc(d, &d.data, padded));
    CUDA_TRY(cudaMemsetAsync(d.data, 0, padded, s));
    if (d.data_bytes) CUDA_TRY(cudaMemcpyAsync(d.data, h.data.data(), d.data_bytes, cudaMemcpyHostToDevice, s));

    // packed vertex records (one 16-byte load per frontier vertex)
    std::vector<VRec> rec(h.n);
#pragma omp parallel for schedule(static)
    for (int64_t v = 0; v < (int64_t)h.n; ++v) {
        const uint64_t deg = h.vlist[v + 1] - h.vlist[v];
        const uint32_t l = h.nlb[v];
        const uint64_t size = h.offsets[v + 1] - h.offsets[v];
        const uint64_t fwd = h.k ? 4 * (deg / h.k) : 0;
        const uint64_t lower = (deg * l + 7) / 8;
        VRec r;
        r.off_l = (h.offsets[v] & kOffMask) | ((uint64_t)l << kOffBits);
        r.deg = (uint32_t)deg;
        r.ubytes = (uint32_t)(deg ? size - fwd - lower : 0);
        rec[v] = r;
    }
    EFG_TRY(dev_alloc(d, &d.rec, h.n));
    CUDA_TRY(cudaMemcpyAsync(d.rec, rec.data(), h.n * sizeof(VRec), cudaMemcpyHostToDevice, s));
    {
        const uint64_t words = (h.n + 31) / 32;
        const uint64_t nw = (words + kAdvanceWords - 1) / kAdvanceWords * kAdvanceWords;
        std::vector<uint32_t> deg(nw * 32, 0);
#pragma omp parallel for schedule(static)
        for (int64_t v = 0; v < (int64_t)h.n; ++v) deg[v] = (uint32_t)(h.vlist[v + 1] - h.vlist[v]);
        EFG_TRY(dev_alloc(d, &d.deg32, nw * 32));
        CUDA_TRY(cudaMemcpyAsync(d.deg32, deg.data(), nw * 32 * 4, cudaMemcpyHostToDevice, s));
        CUDA_TRY(cudaStreamSynchronize(s));
    }
    EFG_TRY(dev_alloc(d, &d.vlist, h.n + 1));
    CUDA_TRY(cudaMemcpyAsync(d.vlist, h.vlist.data(), (h.n + 1) * 8, cudaMemcpyHostToDevice, s));
    if (!h.weights.empty()) {
        EFG_TRY(dev_alloc(d, &d.weights, h.m));
        CUDA_TRY(cudaMemcpyAsync(d.weights, h.weights.data(), h.m * 4, cudaMemcpyHostToDevice, s));
    }

    // traversal workspace
    const uint64_t words = (h.n + 31) / 32;
    d.nwords = (words + kAdvanceWords - 1) / kAdvanceWords * kAdvanceWords;
    d.status_blocks = d.nwords / kAdvanceWords;
    EFG_TRY(dev_alloc(d, &d.vis, d.nwords));
    EFG_TRY(dev_alloc(d, &d.prev, d.nwords));
    EFG_TRY(dev_alloc(d, &d.queue, h.n));
    d.max_tiles = (h.m + (uint64_t)kVertexWork * h.n) / kTileWork + 2;
    EFG_TRY(dev_alloc(d, &d.tiles, d.max_tiles));
    EFG_TRY(dev_alloc(d, &d.depth, h.n));
    EFG_TRY(dev_alloc(d, &d.status, 4 * d.status_blocks));
    CUDA_TRY(cudaMemsetAsync(d.status, 0, 4 * d.status_blocks * 8, s));
    EFG_TRY(dev_alloc(d, &d.ctrl, 1));
    CUDA_TRY(cudaMemsetAsync(d.ctrl, 0, sizeof(LevelCtrl), s));
    CUDA_TRY(cudaMallocHost(reinterpret_cast<void **>(&d.ctrl_host), sizeof(LevelCtrl)));
    d.expand_blocks = d.num_sms * expand_occupancy(kModeVisit);
    CUDA_TRY(cudaStreamSynchronize(s));
    return EFG_OK;
}

struct Ctx {
    DeviceGraph &d;
    cudaStream_t s;
    uint32_t parity;
};

uint32_t g_epoch = 0;

int kshift_of(uint32_t k)
{
    if (k == 0 || (k & (k - 1))) return -1;
    return __builtin_ctz(k);
}  // parity source for the decoupled look-back status

efg_status run_advance(DeviceGraph &d, int32_t *depth, int32_t depth_value)
{
    AdvanceArgs a;
    a.vis = d.vis;
    a.prev = d.prev;
    a.rec = d.rec;
    a.deg32 = d.deg32;
    a.depth = depth;
    a.queue = d.queue;
    a.tiles = d.tiles;
    a.status = d.status;
    a.ctrl = d.ctrl;
    a.nwords = d.nwords;
    a.nblocks = d.status_blocks;
    a.depth_value = depth_value;
    a.parity = (g_epoch++) & 1u;
    a.k = d.k;
    a.kshift = kshift_of(d.k);
    CUDA_TRY(launch_advance(a, static_cast<cudaStream_t>(d.stream)));
    return EFG_OK;
}

efg_status run_expand(DeviceGraph &d, int mode, uint32_t *out)
{
    ExpandArgs a;
    a.data = d.data;
    a.rec = d.rec;
    a.queue = d.queue;
    a.tiles = d.tiles;
    a.ctrl = d.ctrl;
    a.vis = d.vis;
    a.out = out;
    a.k = d.k;
    a.kshift = kshift_of(d.k);
    const int blocks = d.num_sms * expand_occupancy(mode);
    CUDA_TRY(launch_expand(mode, a, blocks, static_cast<cudaStream_t>(d.stream)));
    return EFG_OK;
}

efg_status read_ctrl(DeviceGraph &d, LevelCtrl &c)
{
    cudaStream_t s = static_cast<cudaStream_t>(d.stream);
    CUDA_TRY(cudaMemcpyAsync(d.ctrl_host, d.ctrl, sizeof(LevelCtrl), cudaMemcpyDeviceToHost, s));
    CUDA_TRY(cudaStreamSynchronize(s));
    c = *d.ctrl_host;
    return EFG_OK;
}

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

extern "C" efg_status efg_build(uint64_t n, uint64_t m, const uint32_t *src, const uint32_t *dst,
                                const efg_build_opts *opts, efg_graph **out)
{
    clear_error();
    if (!out) return set_error(EFG_EINVAL, "efg_build: out is NULL");
    *out = nullptr;
    efg_build_opts o;
    if (opts)
        o = *opts;
    else
        efg_default_opts(&o);
    if (n == 0 || n > 0xFFFFFFFFull) return set_error(EFG_EINVAL, "efg_build: need 1 <= n <= 2^32-1");
    if (m && (!src || !dst)) return set_error(EFG_EINVAL, "efg_build: src/dst is NULL");
    if (o.dist) return set_error(EFG_ENOTSUP, "efg_build: multi-GPU partition not built into this library");
    efg_graph *g = new (std::nothrow) efg_graph();
    if (!g) return set_error(EFG_ENOMEM, "efg_build: handle allocation failed");
    efg_status st = build_host(n, m, src, dst, o, g->host);
    if (st != EFG_OK) {
        delete g;
        return st;
    }
    if (o.device >= 0) {
        st = upload(g, o);
        if (st != EFG_OK) {
            free_device(g->dev);
            delete g;
            return st;
        }
        g->on_device = true;
    }
    *out = g;
    return EFG_OK;
}

extern "C" void efg_free(efg_graph *g)
{
    if (!g) return;
    if (g->on_device) free_device(g->dev);
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

extern "C" efg_status efg_decode(efg_graph *g, uint32_t v0, uint32_t v1, uint32_t *out)
{
    clear_error();
    EFG_TRY(check_handle(g));
    const HostEFG &h = g->host;
    if (v0 > v1 || v1 > h.n) return set_error(EFG_ERANGE, "efg_decode: bad vertex range");
    const uint64_t cnt = h.vlist[v1] - h.vlist[v0];
    if (cnt == 0) return EFG_OK;
    if (!out) return set_error(EFG_EINVAL, "efg_decode: out is NULL");
    DeviceGraph &d = g->dev;
    CUDA_TRY(cudaSetDevice(d.device));
    cudaStream_t s = static_cast<cudaStream_t>(d.stream);
    const bool out_dev = is_device_ptr(out);
    uint32_t *od = out;
    if (!out_dev) EFG_TRY(dev_alloc(d, &od, cnt));
    efg_status st = EFG_OK;
    do {
        if (cudaMemsetAsync(d.vis, 0, d.nwords * 4, s) != cudaSuccess ||
            cudaMemsetAsync(d.prev, 0, d.nwords * 4, s) != cudaSuccess ||
            launch_set_range_bits(d.vis, v0, v1, s) != cudaSuccess) {
            st = set_error(EFG_ECUDA, std::string("efg_decode: ") + cudaGetErrorString(cudaGetLastError()));
            break;
        }
        if ((st = run_advance(d, d.depth, 0)) != EFG_OK) break;
        if ((st = run_expand(d, kModeDecode, od)) != EFG_OK) break;
        if (!out_dev && cudaMemcpyAsync(out, od, cnt * 4, cudaMemcpyDeviceToHost, s) != cudaSuccess) {
            st = set_error(EFG_ECUDA, "efg_decode: copy-out failed");
            break;
        }
        cudaError_t e = cudaStreamSynchronize(s);
        if (e != cudaSuccess) st = set_error(EFG_ECUDA, std::string("efg_decode: ") + cudaGetErrorString(e));
    } while (0);
    if (!out_dev) {
        cudaFree(od);
        d.device_bytes -= cnt * 4;
    }
    return st;
}

extern "C" efg_status efg_bfs(efg_graph *g, uint32_t source, int32_t *depth, uint32_t *parent, efg_stats *st)
{
    clear_error();
    EFG_TRY(check_handle(g));
    DeviceGraph &d = g->dev;
    if (source >= d.n) return set_error(EFG_ERANGE, "efg_bfs: source >= n");
    if (!depth) return set_error(EFG_EINVAL, "efg_bfs: depth is NULL");
    CUDA_TRY(cudaSetDevice(d.device));
    cudaStream_t s = static_cast<cudaStream_t>(d.stream);
    const bool depth_dev = is_device_ptr(depth);
    int32_t *dd = depth_dev ? depth : d.depth;
    uint32_t *pd = nullptr;
    bool parent_dev = false;
    if (parent) {
        parent_dev = is_device_ptr(parent);
        if (!parent_dev && !d.parent) EFG_TRY(dev_alloc(d, &d.parent, d.n));
        pd = parent_dev ? parent : d.parent;
    }
    const int mode = parent ? kModeVisitParent : kModeVisit;

    cudaEvent_t ev0, ev1;
    CUDA_TRY(cudaEventCreate(&ev0));
    CUDA_TRY(cudaEventCreate(&ev1));
    std::vector<cudaEvent_t> lev;  // expand start/stop pairs
    uint32_t launches = 0;

    CUDA_TRY(cudaEventRecord(ev0, s));
    CUDA_TRY(cudaMemsetAsync(d.vis, 0, d.nwords * 4, s));
    CUDA_TRY(cudaMemsetAsync(d.prev, 0, d.nwords * 4, s));
    CUDA_TRY(cudaMemsetAsync(dd, 0xFF, d.n * 4, s));
    if (pd) {
        CUDA_TRY(cudaMemsetAsync(pd, 0xFF, d.n * 4, s));
        CUDA_TRY(launch_fill_u32(pd + source, source, 1, s));
        ++launches;
    }
    CUDA_TRY(launch_set_range_bits(d.vis, source, source + 1, s));
    EFG_TRY(run_advance(d, dd, 0));
    launches += 2;

    uint64_t edges = 0, reached = 0;
    uint32_t level = 0;
    std::vector<uint64_t> lf, le;
    for (;;) {
        LevelCtrl c;
        EFG_TRY(read_ctrl(d, c));
        if (c.nf == 0) break;
        reached += c.nf;
        edges += c.ne;
        lf.push_back(c.nf);
        le.push_back(c.ne);
        cudaEvent_t a, b;
        CUDA_TRY(cudaEventCreate(&a));
        CUDA_TRY(cudaEventCreate(&b));
        lev.push_back(a);
        lev.push_back(b);
        CUDA_TRY(cudaEventRecord(a, s));
        EFG_TRY(run_expand(d, mode, pd));
        CUDA_TRY(cudaEventRecord(b, s));
        EFG_TRY(run_advance(d, dd, (int32_t)level + 1));
        launches += 2;
        ++level;
    }
    CUDA_TRY(cudaEventRecord(ev1, s));
    if (!depth_dev) CUDA_TRY(cudaMemcpyAsync(depth, dd, d.n * 4, cudaMemcpyDeviceToHost, s));
    if (parent && !parent_dev) CUDA_TRY(cudaMemcpyAsync(parent, pd, d.n * 4, cudaMemcpyDeviceToHost, s));
    CUDA_TRY(cudaStreamSynchronize(s));

    float total_ms = 0.f, exp_ms = 0.f;
    cudaEventElapsedTime(&total_ms, ev0, ev1);
    std::vector<float> per(level, 0.f);
    for (uint32_t i = 0; i < level; ++i) {
        cudaEventElapsedTime(&per[i], lev[2 * i], lev[2 * i + 1]);
        exp_ms += per[i];
    }
    for (auto e : lev) cudaEventDestroy(e);
    cudaEventDestroy(ev0);
    cudaEventDestroy(ev1);
    if (st) {
        st->levels = level;
        st->edges_traversed = edges;
        st->vertices_reached = reached;
        st->device_ms = total_ms;
        st->expand_ms = exp_ms;
        st->expand_launches = level;
        st->kernel_launches = launches;
        uint64_t bytes = 0;  // filled by the Python side from the host arrays
        st->expand_bytes = bytes;
        for (uint32_t i = 0; i < std::min(level, st->level_cap); ++i) {
            if (st->level_frontier) st->level_frontier[i] = lf[i];
            if (st->level_edges) st->level_edges[i] = le[i];
            if (st->level_expand_ms) st->level_expand_ms[i] = per[i];
        }
    }
    return EFG_OK;
}

extern "C" efg_status efg_sssp(efg_graph *g, uint32_t, float *, efg_stats *)
{
    clear_error();
    EFG_TRY(check_handle(g));
    return set_error(EFG_ENOTSUP, "efg_sssp: not implemented yet");
}

extern "C" efg_status efg_pagerank(efg_graph *g, double, uint32_t, double *, efg_stats *)
{
    clear_error();
    EFG_TRY(check_handle(g));
    return set_error(EFG_ENOTSUP, "efg_pagerank: not implemented yet");
}

extern "C" efg_status efg_get_unique_id(uint8_t id[128])
{
    (void)id;
    return set_error(EFG_ENOTSUP, "efg_get_unique_id: NCCL transport not built");
}

extern "C" efg_status efg_dist_init(int, int, const uint8_t *, int, efg_dist **out)
{
    if (out) *out = nullptr;
    return set_error(EFG_ENOTSUP, "efg_dist_init: NCCL transport not built");
}

extern "C" void efg_dist_free(efg_dist *) {}

extern "C" efg_status efg_partition(uint64_t n, const uint64_t *vlist, const uint64_t *offsets, int world,
                                    uint64_t *bounds)
{
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
