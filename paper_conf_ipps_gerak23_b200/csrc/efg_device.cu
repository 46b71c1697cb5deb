// efg_device.cu — device side of a handle: upload of the packed EFG, the
// traversal workspace, and the level-synchronous driver.
//
// Per BFS level the driver runs two kernels (efg_kernels.cu):
//   expand  (a4 a5 a6)  ->  frontier (a7, then the next level's a1 a2 a3 a4)
// Two drivers share them:
//   * graph mode (default): the level loop is one CUDA graph with a
//     conditional WHILE node; frontier_kernel's last block sets the condition
//     (frontier non-empty) on the device, so a whole BFS costs one graph launch
//     and no host round trip per level;
//   * host mode (efg_set_option EFG_OPT_LEVEL_LOOP = 1): the host launches each
//     level, reads the frontier size back, and brackets every expand launch
//     with CUDA events (the per-kernel timing bench.py reports for the roofline).
#include <cuda_runtime.h>

#include <algorithm>
#include <cstdio>
#include <cstddef>
#include <cstdlib>
#include <cstring>
#include <string>
#include <vector>

#include "efg_internal.h"
#include "efg_kernels.cuh"

namespace efg {

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

int kshift_of(uint32_t k)
{
    if (k == 0 || (k & (k - 1))) return -1;
    return __builtin_ctz(k);
}

cudaStream_t stream_of(const DeviceGraph &d) { return static_cast<cudaStream_t>(d.stream); }

// The chunk length of the device copy.  The expand kernel stages one chunk's
// lower fields in a kStageBytes buffer (<= 512 elements of <= 31 bits fit) and
// stores the chunk index in kCcBits of the descriptor; a format quantum k
// (any k >= 0 is a valid EFG) outside those limits — k = 0 (no
// pointers), k > 512, or ceil(deg/k) >= 2^kCcBits — is served by re-sampling
// the forward pointers at kMaxDeviceQuantum for the device (reading R3).
uint32_t device_quantum(uint32_t k, uint64_t maxdeg)
{
    if (k >= 1 && k <= kMaxDeviceQuantum && (maxdeg + k - 1) / k < (1ull << kCcBits)) return k;
    return kMaxDeviceQuantum;
}

// Device EF data with forward pointers every kd elements (fwd[j] =
// select1((j+1)kd - 1) - ((j+1)kd - 1), the high part of that element): the
// lower and upper sections are copied unchanged, the pointers are recomputed by
// a select1 scan over the upper bits of each list.
void resample_forward_pointers(const HostEFG &h, uint32_t kd, std::vector<uint8_t> &data,
                               std::vector<uint64_t> &offsets)
{
    const uint64_t n = h.n;
    offsets.assign(n + 1, 0);
    for (uint64_t v = 0; v < n; ++v) {
        const uint64_t dv = h.vlist[v + 1] - h.vlist[v];
        const uint64_t hf = h.k ? 4 * (dv / h.k) : 0;
        offsets[v + 1] = offsets[v] + (h.offsets[v + 1] - h.offsets[v]) - hf + 4 * (dv / kd);
    }
    data.assign(offsets[n], 0);
#pragma omp parallel for schedule(dynamic, 1024)
    for (int64_t v = 0; v < (int64_t)n; ++v) {
        const uint64_t dv = h.vlist[v + 1] - h.vlist[v];
        if (!dv) continue;
        const uint64_t hf = h.k ? 4 * (dv / h.k) : 0;
        const uint64_t body = h.offsets[v + 1] - h.offsets[v] - hf;  // lower + upper bytes
        const uint64_t F = dv / kd, lower = (dv * h.nlb[v] + 7) / 8;
        uint8_t *out = data.data() + offsets[v];
        std::memcpy(out + 4 * F, h.data.data() + h.offsets[v] + hf, body);
        const uint8_t *up = out + 4 * F + lower;
        const uint64_t U = body - lower;
        uint64_t ones = 0, target = kd - 1, j = 0;
        for (uint64_t b = 0; b < U && j < F; ++b) {
            const uint32_t byte = up[b], pc = (uint32_t)__builtin_popcount(byte);
            while (j < F && ones + pc > target) {  // element `target` has its stop bit in this byte
                uint32_t t = byte;
                for (uint64_t r = target - ones; r; --r) t &= t - 1;
                const uint32_t f = (uint32_t)(b * 8 + (uint64_t)__builtin_ctz(t) - target);
                std::memcpy(out + 4 * j, &f, 4);
                ++j;
                target += kd;
            }
            ones += pc;
        }
    }
}

// skip level for the lane-per-chunk threshold: visited prefix >= n / div (3;
// n / 8 cost C4 5 %, same-box)
// (EFG_LPC_SKIP_DIV: tuning only)
uint64_t lpc_skip_div()
{
    static const uint64_t div = [] {
        const char *e = std::getenv("EFG_LPC_SKIP_DIV");
        const long v = e ? std::atol(e) : 0;
        return (uint64_t)(v >= 1 ? v : 3);
    }();
    return div;
}

ExpandArgs expand_args(DeviceGraph &d, uint32_t *out)
{
    ExpandArgs a;
    a.data = d.data;
    a.chunks = d.chunks;
    a.cvtx = d.cvtx;
    a.tiles = d.tiles;
    a.deg32 = d.deg32;
    a.ctrl = d.ctrl;
    a.vis = d.vis;
    a.out = out;
    a.out_base = 0;
    a.stats = d.stats;
    a.vlist = d.vlist;
    a.weights = d.weights;
    a.dist = d.fbuf;
    a.rank = d.dbuf;
    a.next = d.dbuf ? d.dbuf + d.n : nullptr;
    a.contrib = d.dbuf ? d.dbuf + 2 * d.n + 1 : nullptr;
    a.max_stats = kMaxLevelStats;
    a.hot_words = (uint32_t)std::min<uint64_t>(kHotWords, d.nwords) & ~3u;
    a.k = d.k;
    a.pskip = d.prefix_skip ? 1u : 0u;
    a.variant = (uint32_t)d.expand_variant;
    a.lpc_skip_vpre = (uint32_t)(d.n / lpc_skip_div());
    return a;
}

FrontierArgs frontier_args(DeviceGraph &d, cudaGraphConditionalHandle cond, bool consume = false)
{
    FrontierArgs a;
    a.cond_global = 0;
    a.consume = consume ? 1 : 0;
    a.vis = d.vis;
    a.prev = d.prev;
    a.iso = d.iso;
    a.depth_stored = (d.old_of_new && !consume) ? d.depth_st : nullptr;
    a.depth_stored_only = d.old_of_new ? 1 : 0;
    a.deg32 = d.deg32;
    a.umax = d.umax;
    a.skipw = d.skipw;
#ifdef EFG_NO_LSKIP
    a.lskip = 0;  // tuning experiment: record-level skip only
#else
    a.lskip = (d.prefix_skip && !consume) ? ((d.expand_variant & 32) ? 2u : 1u) : 0u;
#endif
    a.rec = d.rec;
    a.chunks = d.chunks;
    a.cvtx = d.cvtx;
    a.tiles = d.tiles;
    a.ctrl = d.ctrl;
    a.status = d.status;
    a.barrier = reinterpret_cast<unsigned long long *>(d.status + 5 * kMaxGrid);
    a.big = d.big;
    a.trace = d.trace;
    a.stats = d.stats;
    a.max_stats = kMaxLevelStats;
    a.k = d.k;
    a.kshift = kshift_of(d.k);
    a.cond = cond;
    a.nwords = d.nwords;
    a.words_per_block = d.words_per_block;
    a.own_lo_w = d.own_lo_w;
    a.own_hi_w = d.own_hi_w;
    return a;
}

// level end + next plan: one launch (every block resident, see frontier_kernel)
efg_status launch_level_end(DeviceGraph &d, cudaGraphConditionalHandle cond, cudaStream_t s,
                            bool consume = false, bool cond_global = false, bool need_cvtx = true,
                            bool start = false)
{
    FrontierArgs fa = frontier_args(d, cond, consume);
    // a traversal's first plan has no visited prefix to skip by (decode and
    // PageRank mark their whole vertex range visited to plan it)
    if (start) fa.lskip = 0;
    fa.cond_global = cond_global ? 1 : 0;
    if (!need_cvtx) fa.cvtx = nullptr;  // plain BFS: the expand never reads the chunk's vertex
    CUDA_TRY(launch_frontier(fa, (unsigned)((d.nwords + d.words_per_block - 1) / d.words_per_block), s));
    return EFG_OK;
}

// expand launch of one level (BFS modes); with the frontier-order study variant
// the level's descriptors are first permuted into chunks_shuf
cudaError_t launch_level_expand(DeviceGraph &d, int mode, cudaStream_t s)
{
    ExpandArgs a = expand_args(d, nullptr);
    if ((d.expand_variant & 4) && d.chunks_shuf) {
        const cudaError_t e = launch_shuffle_chunks(d.chunks, mode == kModeVisit ? nullptr : d.cvtx, d.chunks_shuf,
                                                    d.cvtx_shuf, d.ctrl, d.num_sms * 8, s);
        if (e != cudaSuccess) return e;
        a.chunks = d.chunks_shuf;
        a.cvtx = d.cvtx_shuf;
    }
    return launch_expand(mode, a, d.num_sms * expand_occupancy(mode), s);
}

PeerArgs peer_args(DeviceGraph &d, int op)
{
    PeerArgs a;
    a.peers = d.peer_ptrs;
    a.local = d.peer_region;
    a.bounds = d.xchg_bounds;
    a.vis = d.vis;
    a.prev = d.prev;
    a.fault = &d.ctrl->fault;
    a.epoch = &d.ctrl->peer_epoch;
    a.sparse_levels = &d.ctrl->xchg_sparse;
    a.nwords = d.nwords;
    a.world = d.peer_world;
    a.rank = d.peer_rank;
    a.op = op;
    return a;
}

// the three peer-exchange launches of one level (publish, owner OR + broadcast, unpack)
efg_status launch_peer_exchange(DeviceGraph &d, cudaStream_t s)
{
    for (int op : {0, 3, 1, 4, 2}) CUDA_TRY(launch_peer(peer_args(d, op), d.num_sms, s));
    return EFG_OK;
}

// a handle of a 1-D row partition (efg_build_opts.row_lo / row_hi)
bool partitioned(const efg_graph *g) { return !(g->host.row_lo == 0 && g->host.row_hi == g->host.n); }

// Build (once per handle and mode) the graph:
//   while (frontier) { expand; frontier }                          (modes 0, 1)
//   while (global new) { expand; peer exchange; frontier }         (mode 2: partitioned)
constexpr int kLoopPartitioned = 2;
efg_status build_loop_graph(DeviceGraph &d, int mode)
{
    if (d.loop_exec[mode]) return EFG_OK;
    const bool part = mode == kLoopPartitioned;
    const int emode = part ? (int)kModeVisit : mode;
    cudaGraph_t g;
    CUDA_TRY(cudaGraphCreate(&g, 0));
    cudaGraphConditionalHandle cond;
    CUDA_TRY(cudaGraphConditionalHandleCreate(&cond, g, 1, cudaGraphCondAssignDefault));
    cudaGraphNodeParams cp = {};
    cp.type = cudaGraphNodeTypeConditional;
    cp.conditional.handle = cond;
    cp.conditional.type = cudaGraphCondTypeWhile;
    cp.conditional.size = 1;
    cudaGraphNode_t node;
    CUDA_TRY(cudaGraphAddNode(&node, g, nullptr, 0, &cp));
    cudaGraph_t body = cp.conditional.phGraph_out[0];
    cudaStream_t cs;
    CUDA_TRY(cudaStreamCreateWithFlags(&cs, cudaStreamNonBlocking));
    CUDA_TRY(cudaStreamBeginCaptureToGraph(cs, body, nullptr, nullptr, 0, cudaStreamCaptureModeRelaxed));
    cudaError_t e1 = launch_level_expand(d, emode, cs);
    efg_status st = e1 == cudaSuccess ? EFG_OK : EFG_ECUDA;
    if (st == EFG_OK && part) st = launch_peer_exchange(d, cs);
    if (st == EFG_OK) st = launch_level_end(d, cond, cs, false, part, emode != kModeVisit);
    cudaGraph_t captured;
    cudaError_t e2 = cudaStreamEndCapture(cs, &captured);
    cudaStreamDestroy(cs);
    if (e1 != cudaSuccess || st != EFG_OK || e2 != cudaSuccess) {
        cudaGraphDestroy(g);
        return set_error(EFG_ECUDA, std::string("loop graph capture failed: ") +
                                        cudaGetErrorString(e1 != cudaSuccess ? e1 : e2));
    }
    cudaGraphExec_t exec;
    CUDA_TRY(cudaGraphInstantiate(&exec, g, 0));
    d.loop_graph[mode] = g;
    d.loop_exec[mode] = exec;
    return EFG_OK;
}

}  // namespace

void device_drop_graphs(DeviceGraph &d)
{
    if (d.device >= 0) cudaSetDevice(d.device);
    for (int m = 0; m < DeviceGraph::kLoopGraphs; ++m) {
        if (d.loop_exec[m]) cudaGraphExecDestroy(d.loop_exec[m]);
        if (d.loop_graph[m]) cudaGraphDestroy(d.loop_graph[m]);
        d.loop_exec[m] = nullptr;
        d.loop_graph[m] = nullptr;
    }
}

void device_free(DeviceGraph &d)
{
    device_drop_graphs(d);
    device_peer_close(d);
    if (d.data_host)
        cudaFreeHost(d.data_host);  // out-of-core: d.data is its device mapping
    else
        cudaFree(d.data);
    cudaFree(d.rec);
    cudaFree(d.deg32);
    cudaFree(d.umax);
    cudaFree(d.skipw);
    cudaFree(d.depth8);
    if (d.depth8_host) cudaFreeHost(d.depth8_host);
    for (int c = 0; c < kD2HChunks; ++c)
        if (d.d2h_ev[c]) cudaEventDestroy(d.d2h_ev[c]);
    cudaFree(d.iso);
    cudaFree(d.vlist);
    cudaFree(d.weights);
    cudaFree(d.vis);
    cudaFree(d.prev);
    cudaFree(d.tiles);
    cudaFree(d.chunks);
    cudaFree(d.cvtx);
    cudaFree(d.chunks_shuf);
    cudaFree(d.cvtx_shuf);
    cudaFree(d.depth);
    cudaFree(d.parent);
    cudaFree(d.parent2);
    cudaFree(d.old_of_new);
    cudaFree(d.new_of_old);
    cudaFree(d.depth_st);
    cudaFree(d.status);
    cudaFree(d.big);
    cudaFree(d.trace);
    cudaFree(d.stats);
    cudaFree(d.xchg_bounds);
    cudaFree(d.ctrl);
    cudaFree(d.peer_region);
    cudaFree(d.fbuf);
    cudaFree(d.dbuf);
    if (d.ctrl_host) cudaFreeHost(d.ctrl_host);
    if (d.stats_host) cudaFreeHost(d.stats_host);
    d = DeviceGraph{};
}

efg_status device_upload(efg_graph *g, const efg_build_opts &o)
{
    DeviceGraph &d = g->dev;
    const HostEFG &h = g->host;
    CUDA_TRY(cudaSetDevice(o.device));
    d.device = o.device;
    d.stream = o.stream;
    d.n = h.n;
    d.k = h.k;
    cudaStream_t s = stream_of(d);
    cudaDeviceProp prop;
    CUDA_TRY(cudaGetDeviceProperties(&prop, o.device));
    d.num_sms = prop.multiProcessorCount;

    // the expand kernel stages select1(i) - i (< 2 * degree) in 27 bits
    uint64_t maxdeg = 0;
    for (uint64_t v = 0; v < h.n; ++v) maxdeg = std::max<uint64_t>(maxdeg, h.vlist[v + 1] - h.vlist[v]);
    if (maxdeg >= (1ull << 26))
        return set_error(EFG_ENOTSUP, "efg_build: a vertex degree >= 2^26 is not supported on the device");

    // device chunk quantum (reading R3): the format's k when every
    // chunk fits the kernel's staging buffer and chunk-index field, else the
    // forward pointers are re-sampled at kMaxDeviceQuantum for the device copy
    d.k = device_quantum(h.k, maxdeg);
    std::vector<uint8_t> rdata;       // re-sampled EF data (k != d.k), else empty
    std::vector<uint64_t> roffsets;   // its per-vertex offsets
    if (d.k != h.k) resample_forward_pointers(h, d.k, rdata, roffsets);
    const std::vector<uint8_t> &ddata = d.k != h.k ? rdata : h.data;
    const std::vector<uint64_t> &doffsets = d.k != h.k ? roffsets : h.offsets;

    // EF data, padded so 32-bit word reads past the last list stay in bounds
    d.data_bytes = ddata.size();
    if (d.data_bytes >= (1ull << kOffBits))
        return set_error(EFG_ENOTSUP, "efg_build: EF data of 1 TiB or more is not supported on the device");
    const uint64_t padded = ((d.data_bytes + 64) + 15) & ~15ull;
    // out-of-core: keep `data` in pinned, mapped host memory when
    // asked to, or when it does not fit the device's free memory next to the
    // per-vertex arrays and the traversal workspace (~ 64 B per vertex + 20 B
    // per chunk descriptor, estimated)
    bool host_resident = (o.flags & EFG_HOST_RESIDENT) != 0;
    if (!host_resident) {
        size_t fr = 0, tot = 0;
        CUDA_TRY(cudaMemGetInfo(&fr, &tot));
        const uint64_t rest = 64 * h.n + 20 * (h.n + h.m / d.k + 1) + (256ull << 20);
        host_resident = padded + rest > fr;
    }
    if (host_resident) {
        CUDA_TRY(cudaHostAlloc(reinterpret_cast<void **>(&d.data_host), padded,
                               cudaHostAllocMapped | cudaHostAllocPortable));
        std::memset(d.data_host + d.data_bytes, 0, padded - d.data_bytes);
        if (d.data_bytes) std::memcpy(d.data_host, ddata.data(), d.data_bytes);
        CUDA_TRY(cudaHostGetDevicePointer(reinterpret_cast<void **>(&d.data), d.data_host, 0));
    } else {
        EFG_TRY(dev_alloc(d, &d.data, padded));
        CUDA_TRY(cudaMemsetAsync(d.data, 0, padded, s));
        if (d.data_bytes) CUDA_TRY(cudaMemcpyAsync(d.data, ddata.data(), d.data_bytes, cudaMemcpyHostToDevice, s));
        CUDA_TRY(cudaStreamSynchronize(s));  // ddata may be a temporary
    }

    // bitmap geometry
    const uint64_t words = (h.n + 31) / 32;
    d.nwords = (words + kBitmapAlign - 1) / kBitmapAlign * kBitmapAlign;
    d.own_lo_w = h.row_lo / 32;
    d.own_hi_w = (h.row_hi + 31) / 32;

    // packed vertex records (one 16-byte load per frontier vertex) and degrees
    std::vector<VRec> rec(h.n);
    std::vector<uint32_t> deg(d.nwords * 32, 0);
#pragma omp parallel for schedule(static)
    for (int64_t v = 0; v < (int64_t)h.n; ++v) {
        const uint64_t dv = h.vlist[v + 1] - h.vlist[v];
        const uint32_t l = h.nlb[v];
        const uint64_t size = doffsets[v + 1] - doffsets[v];
        const uint64_t fwd = d.k ? 4 * (dv / d.k) : 0;
        const uint64_t lower = (dv * l + 7) / 8;
        VRec r;
        r.off_l = (doffsets[v] & kOffMask) | ((uint64_t)l << kOffBits);
        r.deg = (uint32_t)dv;
        r.ubytes = (uint32_t)(dv ? size - fwd - lower : 0);
        rec[v] = r;
        deg[v] = (uint32_t)dv;
    }
    EFG_TRY(dev_alloc(d, &d.rec, h.n));
    CUDA_TRY(cudaMemcpyAsync(d.rec, rec.data(), h.n * sizeof(VRec), cudaMemcpyHostToDevice, s));
    EFG_TRY(dev_alloc(d, &d.deg32, d.nwords * 32));
    CUDA_TRY(cudaMemcpyAsync(d.deg32, deg.data(), d.nwords * 32 * 4, cudaMemcpyHostToDevice, s));
    EFG_TRY(dev_alloc(d, &d.umax, d.nwords * 32));
    EFG_TRY(dev_alloc(d, &d.skipw, d.nwords));
    CUDA_TRY(cudaMemsetAsync(d.umax, 0, d.nwords * 32 * 4, s));
    CUDA_TRY(cudaMemcpyAsync(d.umax, h.umax.data(), h.n * 4, cudaMemcpyHostToDevice, s));
    {
        std::vector<uint32_t> iso(d.nwords, 0);
        // never probed: padding ids and vertices without an in-edge (directed
        // sinks are probed although their out-degree is 0)
        for (uint64_t v = 0; v < d.nwords * 32; ++v)
            if (v >= h.n || !h.has_in[v]) iso[v >> 5] |= 1u << (v & 31);
        EFG_TRY(dev_alloc(d, &d.iso, d.nwords));
        CUDA_TRY(cudaMemcpyAsync(d.iso, iso.data(), d.nwords * 4, cudaMemcpyHostToDevice, s));
        CUDA_TRY(cudaStreamSynchronize(s));
    }
    EFG_TRY(dev_alloc(d, &d.vlist, h.n + 1));
    CUDA_TRY(cudaMemcpyAsync(d.vlist, h.vlist.data(), (h.n + 1) * 8, cudaMemcpyHostToDevice, s));
    if (!h.old_of_new.empty()) {
        EFG_TRY(dev_alloc(d, &d.old_of_new, h.n));
        CUDA_TRY(cudaMemcpyAsync(d.old_of_new, h.old_of_new.data(), h.n * 4, cudaMemcpyHostToDevice, s));
        EFG_TRY(dev_alloc(d, &d.new_of_old, h.n));
        CUDA_TRY(cudaMemcpyAsync(d.new_of_old, h.new_of_old.data(), h.n * 4, cudaMemcpyHostToDevice, s));
        EFG_TRY(dev_alloc(d, &d.depth_st, h.n));
    }
    if (!h.weights.empty()) {
        EFG_TRY(dev_alloc(d, &d.weights, h.m));
        CUDA_TRY(cudaMemcpyAsync(d.weights, h.weights.data(), h.m * 4, cudaMemcpyHostToDevice, s));
    }

    // traversal workspace
    EFG_TRY(dev_alloc(d, &d.vis, d.nwords));
    EFG_TRY(dev_alloc(d, &d.prev, d.nwords));
    // a level has at most one chunk per frontier vertex plus one per k elements
    const uint64_t rows = (h.row_hi > h.row_lo) ? h.row_hi - h.row_lo : h.n;
    d.max_chunks = rows + h.m / d.k + 1;
    d.max_tiles = (h.m + (uint64_t)kChunkWork * d.max_chunks) / kTileWork + 2;
    EFG_TRY(dev_alloc(d, &d.tiles, d.max_tiles + 1));
    EFG_TRY(dev_alloc(d, &d.chunks, d.max_chunks));
    EFG_TRY(dev_alloc(d, &d.cvtx, d.max_chunks));
    EFG_TRY(dev_alloc(d, &d.depth, h.n));
    EFG_TRY(dev_alloc(d, &d.status, 5 * kMaxGrid + 1));  // + the grid-barrier counter
    CUDA_TRY(cudaMemsetAsync(d.status, 0, (5 * kMaxGrid + 1) * 8, s));
    if (std::getenv("EFG_FRONTIER_TRACE")) EFG_TRY(dev_alloc(d, &d.trace, 8 * kMaxGrid));
    // lists planned grid-wide: more than one chunk (deg > k) or more than one
    // tile of work (deg > kTileWork - kChunkWork)
    {
        const uint64_t q = std::min<uint64_t>(d.k, kTileWork - kChunkWork);
        d.max_big = std::min<uint64_t>(rows, h.m / q + 1);
        EFG_TRY(dev_alloc(d, &d.big, d.max_big));
    }
    EFG_TRY(dev_alloc(d, &d.stats, kMaxLevelStats));
    EFG_TRY(dev_alloc(d, &d.ctrl, 1));
    CUDA_TRY(cudaMemsetAsync(d.ctrl, 0, sizeof(LevelCtrl), s));
    CUDA_TRY(cudaMallocHost(reinterpret_cast<void **>(&d.ctrl_host), sizeof(LevelCtrl)));
    CUDA_TRY(cudaMallocHost(reinterpret_cast<void **>(&d.stats_host), kMaxLevelStats * sizeof(LevelStat)));
    // persistent grids of the frontier kernels: 2 blocks per SM, whole bitmap words
    d.frontier_blocks = (unsigned)std::min<uint64_t>((1024 / kFrontierThreads) * (uint64_t)d.num_sms, kMaxGrid);
    if (const char *e = std::getenv("EFG_FRONTIER_BLOCKS"))  // tuning knob (blocks of compact / plan)
        d.frontier_blocks = (unsigned)std::max(1, std::min(atoi(e), (int)kMaxGrid));
    const uint64_t per = (d.nwords + d.frontier_blocks - 1) / d.frontier_blocks;
    d.words_per_block = (per + kFrontierThreads - 1) / kFrontierThreads * kFrontierThreads;
    // frontier_kernel blocks wait on their predecessors: the whole grid must be resident
    const uint64_t grid = (d.nwords + d.words_per_block - 1) / d.words_per_block;
    const int occ = frontier_occupancy();
    if (occ <= 0 || grid > (uint64_t)occ * d.num_sms)
        return set_error(EFG_ECUDA, "frontier_kernel grid (" + std::to_string(grid) + " blocks) exceeds the resident limit (" +
                                        std::to_string(occ) + " per SM)");
    CUDA_TRY(cudaStreamSynchronize(s));
    return EFG_OK;
}

// Start a traversal: reset the bitmaps, mark [v0, v1), run the level-0 frontier
// kernels.  depth: device buffer receiving the level numbers.
static efg_status start_traversal(DeviceGraph &d, uint64_t v0, uint64_t v1, int32_t *depth,
                                  uint32_t *parent, uint32_t &launches)
{
    cudaStream_t s = stream_of(d);
    CUDA_TRY(cudaMemsetAsync(d.vis, 0, d.nwords * 4, s));
    CUDA_TRY(cudaMemsetAsync(d.prev, 0, d.nwords * 4, s));
    InitArgs ia;
    ia.ctrl = d.ctrl;
    ia.vis = d.vis;
    ia.depth = depth;
    ia.parent = parent;
    ia.v0 = v0;
    ia.v1 = v1;
    CUDA_TRY(launch_init(ia, s));
    EFG_TRY(launch_level_end(d, 0, s, false, false, true, true));
    launches += 2;
    return EFG_OK;
}

efg_status device_decode(efg_graph *g, uint32_t v0, uint32_t v1, uint32_t *out)
{
    const HostEFG &h = g->host;
    DeviceGraph &d = g->dev;
    const uint64_t cnt = h.vlist[v1] - h.vlist[v0];
    CUDA_TRY(cudaSetDevice(d.device));
    cudaStream_t s = stream_of(d);
    const bool out_dev = is_device_ptr(out);
    uint32_t *od = out;
    if (!out_dev) EFG_TRY(dev_alloc(d, &od, cnt));
    efg_status st = EFG_OK;
    uint32_t launches = 0;
    do {
        if ((st = start_traversal(d, v0, v1, d.depth, nullptr, launches)) != EFG_OK) break;
        const int blocks = d.num_sms * expand_occupancy(kModeDecode);
        ExpandArgs ea = expand_args(d, od);
        ea.out_base = h.vlist[v0];
        cudaError_t e = launch_expand(kModeDecode, ea, blocks, s);
        if (e == cudaSuccess && !out_dev) e = cudaMemcpyAsync(out, od, cnt * 4, cudaMemcpyDeviceToHost, s);
        if (e == cudaSuccess) e = cudaStreamSynchronize(s);
        if (e != cudaSuccess) st = set_error(EFG_ECUDA, std::string("efg_decode: ") + cudaGetErrorString(e));
    } while (0);
    if (!out_dev) {
        cudaFree(od);
        d.device_bytes -= std::max<uint64_t>(cnt, 1) * 4;
    }
    return st;
}

efg_status device_bfs(efg_graph *g, uint32_t source, int32_t *depth, uint32_t *parent, efg_stats *st)
{
    DeviceGraph &d = g->dev;
    CUDA_TRY(cudaSetDevice(d.device));
    cudaStream_t s = stream_of(d);
    const bool depth_dev = is_device_ptr(depth);
    int32_t *dd = depth_dev ? depth : d.depth;
    uint32_t *pd = nullptr;     // parent buffer the kernels write (stored ids)
    uint32_t *pout = nullptr;   // parent in input ids on the device
    bool parent_dev = false;
    const bool relabel = d.old_of_new != nullptr;
    if (parent) {
        parent_dev = is_device_ptr(parent);
        if ((relabel || !parent_dev) && !d.parent) EFG_TRY(dev_alloc(d, &d.parent, d.n));
        if (relabel && !parent_dev && !d.parent2) EFG_TRY(dev_alloc(d, &d.parent2, d.n));
        pd = (parent_dev && !relabel) ? parent : d.parent;
        pout = parent_dev ? parent : (relabel ? d.parent2 : d.parent);
    }
    // partitioned handle: the BFS is collective over the peer exchange (every
    // rank calls efg_bfs with the same source; each level = expand own rows,
    // exchange the new bits, level end over the global bitmap)
    const bool part = partitioned(g);
    if (part && !d.peer_ptrs)
        return set_error(EFG_ESTATE, "efg_bfs: a partitioned handle runs a collective BFS over the peer exchange: "
                                     "call efg_peer_alloc / efg_peer_open first (or drive the levels with "
                                     "efg_bfs_begin / efg_bfs_expand / efg_xchg_* / efg_bfs_finish_level)");
    if (part && parent)
        return set_error(EFG_ENOTSUP, "efg_bfs: parents are not available on a partitioned handle");
    if ((d.expand_variant & 4) && !d.chunks_shuf) {  // frontier-order study buffers
        EFG_TRY(dev_alloc(d, &d.chunks_shuf, d.max_chunks));
        EFG_TRY(dev_alloc(d, &d.cvtx_shuf, d.max_chunks));
    }
    const int emode = parent ? kModeVisitParent : kModeVisit;  // expand mode
    const int mode = part ? kLoopPartitioned : emode;            // loop graph
    const bool graph_mode = d.level_loop == 0;
    if (graph_mode) EFG_TRY(build_loop_graph(d, mode));

    // device outputs and no statistics: enqueue the whole BFS on the handle's
    // stream and return (stream-ordered, like cudaMemcpyAsync); back-to-back
    // calls then run without a host round trip in between
    if (graph_mode && !st && depth_dev && (!parent || parent_dev)) {
        uint32_t launches = 0;
        if (relabel)
            CUDA_TRY(cudaMemsetAsync(d.depth_st, 0xFF, d.n * 4, s));
        else
            CUDA_TRY(cudaMemsetAsync(dd, 0xFF, d.n * 4, s));
        if (pd) CUDA_TRY(cudaMemsetAsync(pd, 0xFF, d.n * 4, s));
        EFG_TRY(start_traversal(d, source, (uint64_t)source + 1, dd, pd, launches));
        CUDA_TRY(cudaGraphLaunch(d.loop_exec[mode], s));
        if (relabel) CUDA_TRY(launch_map_depth(d.depth_st, d.new_of_old, dd, d.n, s));
        if (parent && relabel) CUDA_TRY(launch_map_parent(pd, d.old_of_new, pout, d.n, s));
        return EFG_OK;
    }

    cudaEvent_t ev0, ev1;
    CUDA_TRY(cudaEventCreate(&ev0));
    CUDA_TRY(cudaEventCreate(&ev1));
    std::vector<cudaEvent_t> lev;  // host mode: expand start, expand end, level end
    uint32_t launches = 0;

    CUDA_TRY(cudaEventRecord(ev0, s));
    if (relabel)
        CUDA_TRY(cudaMemsetAsync(d.depth_st, 0xFF, d.n * 4, s));  // gathered into dd at the end
    else
        CUDA_TRY(cudaMemsetAsync(dd, 0xFF, d.n * 4, s));
    if (pd) CUDA_TRY(cudaMemsetAsync(pd, 0xFF, d.n * 4, s));
    EFG_TRY(start_traversal(d, source, (uint64_t)source + 1, dd, pd, launches));

    std::vector<uint64_t> lf, le;
    std::vector<float> lms;
    uint32_t levels = 0;
    if (graph_mode) {
        CUDA_TRY(cudaGraphLaunch(d.loop_exec[mode], s));
        if (relabel) CUDA_TRY(launch_map_depth(d.depth_st, d.new_of_old, dd, d.n, s));
        CUDA_TRY(cudaEventRecord(ev1, s));
        CUDA_TRY(cudaMemcpyAsync(d.ctrl_host, d.ctrl, sizeof(LevelCtrl), cudaMemcpyDeviceToHost, s));
        CUDA_TRY(cudaStreamSynchronize(s));
        levels = d.ctrl_host->nlevels;
        if (d.ctrl_host->fault)
            return set_error(EFG_ECUDA, "a grid or peer barrier timed out (grid not co-resident, or a rank "
                                        "missing from the collective); sticky until efg_free");
        const uint32_t ns = std::min(levels, kMaxLevelStats);
        if (ns) {
            CUDA_TRY(cudaMemcpyAsync(d.stats_host, d.stats, ns * sizeof(LevelStat), cudaMemcpyDeviceToHost, s));
            CUDA_TRY(cudaStreamSynchronize(s));
        }
        for (uint32_t i = 0; i < ns; ++i) {
            lf.push_back(d.stats_host[i].nf);
            le.push_back(d.stats_host[i].ne);
            const LevelStat &x = d.stats_host[i];
            lms.push_back(x.t1 > x.t0 ? (float)((double)(x.t1 - x.t0) * 1e-6) : 0.f);
        }
        launches += (part ? 7 : 2) * levels + (relabel ? 1 : 0);
    } else {
        for (;;) {
            CUDA_TRY(cudaMemcpyAsync(d.ctrl_host, d.ctrl, sizeof(LevelCtrl), cudaMemcpyDeviceToHost, s));
            CUDA_TRY(cudaStreamSynchronize(s));
            const LevelCtrl c = *d.ctrl_host;
            if (c.fault)
                return set_error(EFG_ECUDA, "a grid or peer barrier timed out (grid not co-resident, or a rank "
                                            "missing from the collective); sticky until efg_free");
            if ((part ? c.nnew : c.nf) == 0) break;  // partitioned: the global new count
            if (std::getenv("EFG_DEBUG_LEVELS")) {  // plan statistics of the level about to be expanded
                fprintf(stderr, "efg-level L=%u nf=%llu ne=%llu nchunks=%llu nwork=%llu ntiles=%llu vpre_used=%u"
                        " prev-batches lpc=%llu rec=%llu chunks %llu/%llu elems %llu/%llu lpc-slots %llu words %llu\n",
                        levels, (unsigned long long)c.nf, (unsigned long long)c.ne, (unsigned long long)c.nchunks,
                        (unsigned long long)c.nwork, (unsigned long long)c.ntiles, c.vpre_used, c.bstat[0],
                        c.bstat[1], c.bstat[2], c.bstat[3], c.bstat[4], c.bstat[5], c.bstat[6], c.bstat[7]);
                CUDA_TRY(cudaMemsetAsync(reinterpret_cast<char *>(d.ctrl) + offsetof(LevelCtrl, bstat), 0,
                                         sizeof(c.bstat), s));
            }
            lf.push_back(c.nf);
            le.push_back(c.ne);
            cudaEvent_t a, b;
            CUDA_TRY(cudaEventCreate(&a));
            CUDA_TRY(cudaEventCreate(&b));
            lev.push_back(a);
            lev.push_back(b);
            cudaEvent_t ec;
            CUDA_TRY(cudaEventCreate(&ec));
            lev.push_back(ec);
            CUDA_TRY(cudaEventRecord(a, s));
            CUDA_TRY(launch_level_expand(d, emode, s));
            CUDA_TRY(cudaEventRecord(b, s));
            if (part) EFG_TRY(launch_peer_exchange(d, s));
            EFG_TRY(launch_level_end(d, 0, s, false, false, emode != kModeVisit));
            CUDA_TRY(cudaEventRecord(ec, s));
            launches += part ? 7 : 2;
            if (d.trace) {  // debug: phase end times of frontier_kernel, max over blocks (us after the first start)
                const unsigned nb = (unsigned)((d.nwords + d.words_per_block - 1) / d.words_per_block);
                std::vector<unsigned long long> t(8 * nb);
                CUDA_TRY(cudaMemcpyAsync(t.data(), d.trace, t.size() * 8, cudaMemcpyDeviceToHost, s));
                CUDA_TRY(cudaStreamSynchronize(s));
                unsigned long long t0 = ~0ull, mx[8] = {0};
                for (unsigned b = 0; b < nb; ++b) {
                    t0 = std::min(t0, t[8 * b]);
                    for (int p = 0; p < 8; ++p) mx[p] = std::max(mx[p], t[8 * b + p]);
                }
                fprintf(stderr, "frontier-trace L=%u nf=%llu:", levels, (unsigned long long)0);
                for (int p = 0; p < 8; ++p) fprintf(stderr, " %.1f", (double)(mx[p] - t0) * 1e-3);
                fprintf(stderr, "\n");
            }
            ++levels;
        }
        if (relabel) {
            CUDA_TRY(launch_map_depth(d.depth_st, d.new_of_old, dd, d.n, s));
            ++launches;
        }
        CUDA_TRY(cudaEventRecord(ev1, s));
    }
    if (parent && relabel) CUDA_TRY(launch_map_parent(pd, d.old_of_new, pout, d.n, s));
    uint64_t d2h = 0;
    // a host depth array crosses PCIe as 4 bits per vertex when every depth
    // is < 15 (code = depth + 1, 0 = unreached), else as one byte per vertex
    // when every depth is < 127 ([-1, 126]); the host widens it
    // (efg_host_widen.cpp) chunk by chunk as the chunks land
    int narrow = 0;  // 4 or 8 bits per vertex, 0 = int32 copy
    if (!depth_dev && d.n >= 4096) narrow = levels < 15 ? 4 : levels < 127 ? 8 : 0;  // depth <= levels; levels is final here
    // chunk c: vertices [cv(c), cv(c+1)), multiples of 8 (one 4-bit word = 8 vertices)
    auto cv = [&](int c) -> uint64_t {
        return c == kD2HChunks ? d.n : (((d.n + 7) / 8) * c / kD2HChunks) * 8;
    };
    if (narrow) {
        if (!d.depth8) EFG_TRY(dev_alloc(d, &d.depth8, d.n + 8));
        if (!d.depth8_host) CUDA_TRY(cudaMallocHost(reinterpret_cast<void **>(&d.depth8_host), d.n + 8));
        if (!d.d2h_ev[0])
            for (int c = 0; c < kD2HChunks; ++c) CUDA_TRY(cudaEventCreateWithFlags(&d.d2h_ev[c], cudaEventDisableTiming));
        if (narrow == 4)
            CUDA_TRY(launch_pack4(dd, reinterpret_cast<uint32_t *>(d.depth8), d.n, s));
        else
            CUDA_TRY(launch_pack8(dd, d.depth8, d.n, s));
        // chunked copy: the host widens chunk c while chunks > c are in flight
        for (int c = 0; c < kD2HChunks; ++c) {
            const uint64_t b0 = narrow == 4 ? cv(c) / 2 : cv(c);
            const uint64_t b1 = narrow == 4 ? (cv(c + 1) + 7) / 8 * 4 : cv(c + 1);
            if (b1 > b0)
                CUDA_TRY(cudaMemcpyAsync(d.depth8_host + b0, d.depth8 + b0, b1 - b0, cudaMemcpyDeviceToHost, s));
            CUDA_TRY(cudaEventRecord(d.d2h_ev[c], s));
            d2h += b1 - b0;
        }
    } else if (!depth_dev) {
        CUDA_TRY(cudaMemcpyAsync(depth, dd, d.n * 4, cudaMemcpyDeviceToHost, s));
        d2h += d.n * 4;
    }
    if (parent && !parent_dev) {
        CUDA_TRY(cudaMemcpyAsync(parent, pout, d.n * 4, cudaMemcpyDeviceToHost, s));
        d2h += d.n * 4;
    }
    if (narrow) {
        for (int c = 0; c < kD2HChunks; ++c) {
            CUDA_TRY(cudaEventSynchronize(d.d2h_ev[c]));
            const uint64_t v0 = cv(c), v1 = cv(c + 1);
            if (v1 <= v0) continue;
            if (narrow == 4)
                host_widen_u4_i32(reinterpret_cast<const uint32_t *>(d.depth8_host) + v0 / 8, depth + v0,
                                  (int64_t)(v1 - v0));
            else
                host_widen_i8_i32(d.depth8_host + v0, depth + v0, (int64_t)(v1 - v0));
        }
    }
    CUDA_TRY(cudaStreamSynchronize(s));

    float total_ms = 0.f;
    cudaEventElapsedTime(&total_ms, ev0, ev1);
    std::vector<float> ems(levels, 0.f);
    if (!graph_mode) {
        lms.assign(levels, 0.f);
        for (uint32_t i = 0; i < levels; ++i) {
            cudaEventElapsedTime(&lms[i], lev[3 * i], lev[3 * i + 1]);
            cudaEventElapsedTime(&ems[i], lev[3 * i + 1], lev[3 * i + 2]);
        }
    }
    for (auto e : lev) cudaEventDestroy(e);
    cudaEventDestroy(ev0);
    cudaEventDestroy(ev1);
    if (st) {
        uint64_t edges = 0, reached = 0;
        float exp_ms = 0.f;
        for (size_t i = 0; i < lf.size(); ++i) {
            reached += lf[i];
            edges += le[i];
            exp_ms += lms[i];
        }
        if (graph_mode) {  // exact even past kMaxLevelStats levels
            reached = d.ctrl_host->total_nf;
            edges = d.ctrl_host->total_ne;
        }
        st->levels = levels;
        st->edges_traversed = edges;
        st->vertices_reached = reached;
        st->device_ms = total_ms;
        st->expand_ms = exp_ms;
        st->expand_launches = levels;
        st->kernel_launches = launches;
        st->expand_bytes = 0;
        st->d2h_bytes = d2h;
        st->xchg_sparse_levels = part ? d.ctrl_host->xchg_sparse : 0u;
        for (uint32_t i = 0; i < std::min<uint32_t>((uint32_t)lf.size(), st->level_cap); ++i) {
            if (st->level_frontier) st->level_frontier[i] = lf[i];
            if (st->level_edges) st->level_edges[i] = le[i];
            if (st->level_expand_ms) st->level_expand_ms[i] = lms[i];
            if (st->level_end_ms && i < ems.size()) st->level_end_ms[i] = ems[i];
        }
    }
    return EFG_OK;
}

// ---------------------------------------------------------------------------
// Stepwise driver of the 1-D partitioned BFS (efg.h "multi-GPU").
// ---------------------------------------------------------------------------
efg_status device_step_begin(efg_graph *g, uint32_t source, int32_t *depth)
{
    DeviceGraph &d = g->dev;
    CUDA_TRY(cudaSetDevice(d.device));
    cudaStream_t s = stream_of(d);
    if (!is_device_ptr(depth)) return set_error(EFG_EINVAL, "efg_bfs_begin: depth must be a device pointer");
    d.step_levels = 0;
    d.step_reached = d.step_edges = 0;
    d.step_lf.clear();
    d.step_le.clear();
    d.step_depth = depth;
    if (d.old_of_new)
        CUDA_TRY(cudaMemsetAsync(d.depth_st, 0xFF, d.n * 4, s));
    else
        CUDA_TRY(cudaMemsetAsync(depth, 0xFF, d.n * 4, s));
    uint32_t launches = 0;
    EFG_TRY(start_traversal(d, source, (uint64_t)source + 1, depth, nullptr, launches));
    d.step_launches = launches;
    CUDA_TRY(cudaMemcpyAsync(d.ctrl_host, d.ctrl, sizeof(LevelCtrl), cudaMemcpyDeviceToHost, s));
    CUDA_TRY(cudaStreamSynchronize(s));
    d.step_lf.push_back(d.ctrl_host->nf);
    d.step_le.push_back(d.ctrl_host->ne);
    return EFG_OK;
}

efg_status device_step_expand(efg_graph *g)
{
    DeviceGraph &d = g->dev;
    CUDA_TRY(cudaSetDevice(d.device));
    const int blocks = d.num_sms * expand_occupancy(kModeVisit);
    CUDA_TRY(launch_expand(kModeVisit, expand_args(d, nullptr), blocks, stream_of(d)));
    ++d.step_levels;
    ++d.step_launches;
    return EFG_OK;
}

efg_status device_step_finish(efg_graph *g, uint64_t *global_new)
{
    DeviceGraph &d = g->dev;
    CUDA_TRY(cudaSetDevice(d.device));
    cudaStream_t s = stream_of(d);
    EFG_TRY(launch_level_end(d, 0, s, false, false, false));  // the stepwise expand is plain BFS
    ++d.step_launches;
    CUDA_TRY(cudaMemcpyAsync(d.ctrl_host, d.ctrl, sizeof(LevelCtrl), cudaMemcpyDeviceToHost, s));
    CUDA_TRY(cudaStreamSynchronize(s));
    const LevelCtrl c = *d.ctrl_host;
    if (c.fault) return set_error(EFG_ECUDA, "partitioned level: a grid or peer barrier timed out");
    if (c.nnew == 0 && d.old_of_new) {  // traversal over: depth back to input ids
        CUDA_TRY(launch_map_depth(d.depth_st, d.new_of_old, d.step_depth, d.n, s));
        ++d.step_launches;
        CUDA_TRY(cudaStreamSynchronize(s));
    }
    if (c.nnew) {
        d.step_lf.push_back(c.nf);
        d.step_le.push_back(c.ne);
    }
    if (global_new) *global_new = c.nnew;
    return EFG_OK;
}

efg_status device_step_end(efg_graph *g, efg_stats *st)
{
    DeviceGraph &d = g->dev;
    if (!st) return EFG_OK;
    uint64_t reached = 0, edges = 0;
    for (size_t i = 0; i < d.step_lf.size(); ++i) {
        reached += d.step_lf[i];
        edges += d.step_le[i];
    }
    std::memset(st, 0, offsetof(efg_stats, level_cap));
    st->levels = d.step_levels;
    st->edges_traversed = edges;      // this rank's rows
    st->vertices_reached = reached;   // this rank's rows
    st->expand_launches = d.step_levels;
    st->kernel_launches = d.step_launches;
    st->xchg_sparse_levels = d.ctrl_host->xchg_sparse;
    for (uint32_t i = 0; i < std::min<uint32_t>((uint32_t)d.step_lf.size(), st->level_cap); ++i) {
        if (st->level_frontier) st->level_frontier[i] = d.step_lf[i];
        if (st->level_edges) st->level_edges[i] = d.step_le[i];
    }
    return EFG_OK;
}

// ---------------------------------------------------------------------------
// Peer-memory exchange (efg.h "multi-GPU", peer_kernel in efg_kernels.cu).
// ---------------------------------------------------------------------------
void device_peer_close(DeviceGraph &d)
{
    device_drop_graphs(d);  // a captured partitioned loop refers to the peer table
    for (int p = 0; p < kPeerMaxWorld; ++p)
        if (d.peer_ipc[p]) {
            cudaIpcCloseMemHandle(d.peer_ipc[p]);
            d.peer_ipc[p] = nullptr;
        }
    cudaFree(d.peer_ptrs);
    d.peer_ptrs = nullptr;
    d.peer_world = 0;
    d.peer_rank = -1;
}

efg_status device_peer_alloc(efg_graph *g, int world, void **region, uint8_t *ipc_handle)
{
    DeviceGraph &d = g->dev;
    CUDA_TRY(cudaSetDevice(d.device));
    cudaStream_t s = stream_of(d);
    CUDA_TRY(cudaStreamSynchronize(s));
    device_peer_close(d);
    if (!d.peer_region) {
        // its own allocation: an IPC handle maps exactly this region
        EFG_TRY(dev_alloc(d, &d.peer_region, peer_region_words(d.nwords)));
    }
    CUDA_TRY(cudaMemset(d.peer_region, 0, peer_region_words(d.nwords) * 4));  // flags = epoch 0
    CUDA_TRY(cudaMemset(&d.ctrl->peer_epoch, 0, sizeof(uint32_t)));           // exchange counter
    d.peer_alloc_world = world;
    if (region) *region = d.peer_region;
    if (ipc_handle) {
        cudaIpcMemHandle_t h;
        CUDA_TRY(cudaIpcGetMemHandle(&h, d.peer_region));
        static_assert(sizeof(h) == EFG_IPC_HANDLE_BYTES, "cudaIpcMemHandle_t size");
        std::memcpy(ipc_handle, &h, sizeof(h));
    }
    return EFG_OK;
}

efg_status device_peer_open(efg_graph *g, int world, int rank, const uint64_t *bounds, const uint8_t *ipc_handles,
                            void *const *regions)
{
    DeviceGraph &d = g->dev;
    CUDA_TRY(cudaSetDevice(d.device));
    cudaStream_t s = stream_of(d);
    if (!d.peer_region || d.peer_alloc_world != world)
        return set_error(EFG_ESTATE, "efg_peer_open: call efg_peer_alloc with the same world first");
    if (bounds[0] != 0 || bounds[world] != d.n)
        return set_error(EFG_EINVAL, "efg_peer_open: bounds must span [0, n)");
    for (int r = 0; r < world; ++r)
        if (bounds[r + 1] < bounds[r] || bounds[r] % 64)
            return set_error(EFG_EINVAL, "efg_peer_open: bounds must be non-decreasing multiples of 64");
    device_peer_close(d);
    std::vector<uint32_t *> ptrs(world);
    for (int p = 0; p < world; ++p) {
        if (p == rank) {
            ptrs[p] = d.peer_region;
        } else if (regions) {
            ptrs[p] = static_cast<uint32_t *>(regions[p]);
        } else {
            cudaIpcMemHandle_t h;
            std::memcpy(&h, ipc_handles + (size_t)p * EFG_IPC_HANDLE_BYTES, sizeof(h));
            void *ptr = nullptr;
            const cudaError_t e = cudaIpcOpenMemHandle(&ptr, h, cudaIpcMemLazyEnablePeerAccess);
            if (e != cudaSuccess) {
                cudaGetLastError();
                device_peer_close(d);
                return set_error(EFG_ECUDA, std::string("efg_peer_open: cudaIpcOpenMemHandle(rank ") +
                                                std::to_string(p) + "): " + cudaGetErrorString(e));
            }
            d.peer_ipc[p] = ptr;
            ptrs[p] = static_cast<uint32_t *>(ptr);
        }
    }
    EFG_TRY(dev_alloc(d, &d.peer_ptrs, (uint64_t)world));
    CUDA_TRY(cudaMemcpyAsync(d.peer_ptrs, ptrs.data(), world * sizeof(uint32_t *), cudaMemcpyHostToDevice, s));
    if ((uint64_t)world + 1 > d.xchg_bounds_cap) {
        cudaFree(d.xchg_bounds);
        d.xchg_bounds = nullptr;
        EFG_TRY(dev_alloc(d, &d.xchg_bounds, (uint64_t)world + 1));
        d.xchg_bounds_cap = (uint64_t)world + 1;
    }
    CUDA_TRY(cudaMemcpyAsync(d.xchg_bounds, bounds, (world + 1) * 8, cudaMemcpyHostToDevice, s));
    CUDA_TRY(cudaStreamSynchronize(s));
    d.peer_world = world;
    d.peer_rank = rank;
    return EFG_OK;
}

efg_status device_xchg_peer(efg_graph *g)
{
    DeviceGraph &d = g->dev;
    if (!d.peer_ptrs) return set_error(EFG_ESTATE, "efg_xchg_peer: call efg_peer_open first");
    CUDA_TRY(cudaSetDevice(d.device));
    EFG_TRY(launch_peer_exchange(d, stream_of(d)));
    d.step_launches += 5;
    return EFG_OK;
}

efg_status device_xchg_peer_phase(efg_graph *g, int phase)
{
    DeviceGraph &d = g->dev;
    if (!d.peer_ptrs) return set_error(EFG_ESTATE, "efg_xchg_peer_phase: call efg_peer_open first");
    CUDA_TRY(cudaSetDevice(d.device));
    cudaStream_t s = stream_of(d);
    CUDA_TRY(launch_peer(peer_args(d, phase), d.num_sms, s));
    CUDA_TRY(cudaStreamSynchronize(s));
    d.step_launches += 1;
    return EFG_OK;
}

efg_status device_xchg(efg_graph *g, int op, int world, const uint64_t *bounds, uint64_t slice_words,
                       uint32_t *out, const uint32_t *in)
{
    DeviceGraph &d = g->dev;
    CUDA_TRY(cudaSetDevice(d.device));
    cudaStream_t s = stream_of(d);
    if (op != 1) {
        if ((uint64_t)world + 1 > d.xchg_bounds_cap) {
            cudaFree(d.xchg_bounds);
            d.xchg_bounds = nullptr;
            EFG_TRY(dev_alloc(d, &d.xchg_bounds, (uint64_t)world + 1));
            d.xchg_bounds_cap = (uint64_t)world + 1;
        }
        CUDA_TRY(cudaMemcpyAsync(d.xchg_bounds, bounds, (world + 1) * 8, cudaMemcpyHostToDevice, s));
    }
    XchgArgs a;
    a.op = op;
    a.world = world;
    a.S = slice_words;
    a.bounds = d.xchg_bounds;
    a.vis = d.vis;
    a.prev = d.prev;
    a.out = out;
    a.in = in;
    CUDA_TRY(launch_xchg(a, s));
    ++d.step_launches;
    return EFG_OK;
}

// ---------------------------------------------------------------------------
// SSSP (§VI-F): frontier Bellman-Ford over the compressed graph.  The
// relaxed vertices of an iteration are marked in the visited bitmap, which the
// next compact consumes as the next frontier (and resets).
// ---------------------------------------------------------------------------
efg_status device_sssp(efg_graph *g, uint32_t source, float *dist, efg_stats *st)
{
    DeviceGraph &d = g->dev;
    CUDA_TRY(cudaSetDevice(d.device));
    cudaStream_t s = stream_of(d);
    if (!d.fbuf) EFG_TRY(dev_alloc(d, &d.fbuf, d.n));
    const bool dist_dev = is_device_ptr(dist);
    uint32_t *out = dist_dev && !d.old_of_new ? reinterpret_cast<uint32_t *>(dist) : nullptr;
    cudaEvent_t ev0, ev1;
    CUDA_TRY(cudaEventCreate(&ev0));
    CUDA_TRY(cudaEventCreate(&ev1));
    CUDA_TRY(cudaEventRecord(ev0, s));
    CUDA_TRY(launch_fill(reinterpret_cast<uint32_t *>(d.fbuf), 0x7F800000u, d.n, s));  // +inf
    CUDA_TRY(cudaMemsetAsync(d.fbuf + source, 0, 4, s));
    CUDA_TRY(cudaMemsetAsync(d.vis, 0, d.nwords * 4, s));
    InitArgs ia;
    ia.ctrl = d.ctrl;
    ia.vis = d.vis;
    ia.depth = nullptr;
    ia.parent = nullptr;
    ia.v0 = source;
    ia.v1 = (uint64_t)source + 1;
    CUDA_TRY(launch_init(ia, s));
    EFG_TRY(launch_level_end(d, 0, s, true));
    const int blocks = d.num_sms * expand_occupancy(kModeSssp);
    uint32_t iters = 0;
    uint64_t relax_edges = 0;
    for (;;) {
        CUDA_TRY(cudaMemcpyAsync(d.ctrl_host, d.ctrl, sizeof(LevelCtrl), cudaMemcpyDeviceToHost, s));
        CUDA_TRY(cudaStreamSynchronize(s));
        if (d.ctrl_host->nf == 0) break;
        relax_edges += d.ctrl_host->ne;
        CUDA_TRY(launch_expand(kModeSssp, expand_args(d, nullptr), blocks, s));
        EFG_TRY(launch_level_end(d, 0, s, true));
        ++iters;
    }
    uint32_t *dst = out;
    if (!dst) {  // stage: relabel and / or copy to the host
        if (!d.parent2) EFG_TRY(dev_alloc(d, &d.parent2, d.n));
        dst = d.parent2;
    }
    if (d.old_of_new || dst != reinterpret_cast<uint32_t *>(d.fbuf))
        CUDA_TRY(launch_gather32(reinterpret_cast<uint32_t *>(d.fbuf), d.new_of_old, dst, d.n, s));
    CUDA_TRY(cudaEventRecord(ev1, s));
    if (!dist_dev) CUDA_TRY(cudaMemcpyAsync(dist, dst, d.n * 4, cudaMemcpyDeviceToHost, s));
    else if (dst != reinterpret_cast<uint32_t *>(dist))
        CUDA_TRY(cudaMemcpyAsync(dist, dst, d.n * 4, cudaMemcpyDeviceToDevice, s));
    CUDA_TRY(cudaStreamSynchronize(s));
    float ms = 0.f;
    cudaEventElapsedTime(&ms, ev0, ev1);
    cudaEventDestroy(ev0);
    cudaEventDestroy(ev1);
    if (st) {
        std::memset(st, 0, offsetof(efg_stats, level_cap));
        st->levels = iters;
        st->edges_traversed = relax_edges;
        st->device_ms = ms;
        st->expand_launches = iters;
    }
    return EFG_OK;
}

// ---------------------------------------------------------------------------
// PageRank (§VI-F; 50 iterations P:201; reading C21): every vertex is
// active; the frontier/tile plan of "all vertices" is built once and reused.
// ---------------------------------------------------------------------------
efg_status device_pagerank(efg_graph *g, double damping, uint32_t iters, double *rank, efg_stats *st)
{
    DeviceGraph &d = g->dev;
    CUDA_TRY(cudaSetDevice(d.device));
    cudaStream_t s = stream_of(d);
    if (!d.dbuf) EFG_TRY(dev_alloc(d, &d.dbuf, 3 * d.n + 1));
    double *r = d.dbuf, *next = d.dbuf + d.n, *dsum = d.dbuf + 2 * d.n, *contrib = d.dbuf + 2 * d.n + 1;
    // pull (no atomics per edge) where every list is also the vertex's in-list:
    // symmetric graphs on a whole-graph handle; push otherwise
    const bool pull = g->host.symmetric && g->host.row_lo == 0 && g->host.row_hi == g->host.n && d.pr_pull;
    const int pmode = pull ? kModePrPull : kModePagerank;
    const bool rank_dev = is_device_ptr(rank);
    cudaEvent_t ev0, ev1;
    CUDA_TRY(cudaEventCreate(&ev0));
    CUDA_TRY(cudaEventCreate(&ev1));
    CUDA_TRY(cudaEventRecord(ev0, s));
    CUDA_TRY(launch_fill_f64(r, 1.0 / (double)d.n, d.n, s));
    CUDA_TRY(cudaMemsetAsync(next, 0, d.n * 8, s));
    uint32_t launches = 0;
    EFG_TRY(start_traversal(d, 0, d.n, d.depth, nullptr, launches));  // frontier = every vertex
    const int blocks = d.num_sms * expand_occupancy(pmode);
    if (pull) CUDA_TRY(launch_pr_contrib(r, d.deg32, contrib, d.n, s));
    for (uint32_t it = 0; it < iters; ++it) {
        CUDA_TRY(cudaMemsetAsync(dsum, 0, 8, s));
        CUDA_TRY(launch_pr_dangling(r, d.deg32, d.n, dsum, s));
        CUDA_TRY(launch_expand(pmode, expand_args(d, nullptr), blocks, s));
        CUDA_TRY(launch_pr_update(r, next, d.n, damping, dsum, pull ? contrib : nullptr, d.deg32, s));
    }
    // ranks back to input ids (next[] is free scratch now)
    double *src = r;
    if (d.old_of_new) {
        CUDA_TRY(launch_gather64(r, d.new_of_old, next, d.n, s));
        src = next;
    }
    CUDA_TRY(cudaEventRecord(ev1, s));
    CUDA_TRY(cudaMemcpyAsync(rank, src, d.n * 8, rank_dev ? cudaMemcpyDeviceToDevice : cudaMemcpyDeviceToHost, s));
    CUDA_TRY(cudaStreamSynchronize(s));
    float ms = 0.f;
    cudaEventElapsedTime(&ms, ev0, ev1);
    cudaEventDestroy(ev0);
    cudaEventDestroy(ev1);
    if (st) {
        std::memset(st, 0, offsetof(efg_stats, level_cap));
        st->levels = iters;
        st->edges_traversed = (uint64_t)iters * g->host.m;
        st->device_ms = ms;
        st->expand_launches = iters;
    }
    return EFG_OK;
}

}  // namespace efg
