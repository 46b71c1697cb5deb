// efg_kernels.cu — hand-written sm_100a kernels of the EFG BFS hot path.
//
// Steps and where they live, per BFS level:
//   a4 locate compressed bit ranges + a5 EF element decode + a6 visit
//      -> expand_kernel (persistent, warp per work tile)
//   a7 level end: visited-bitmap diff -> sorted next frontier queue + depth
//      -> compact_kernel (reduce-then-scan over the bitmap)
//   a1 degree lookup + a2 exclusive scan of per-vertex work + a3 partition
//      into tiles -> plan_kernel (reduce-then-scan over the queue)
// init_kernel starts a traversal (source bit, per-call state).
//
// Paper anchors: Alg. 1 (§III-B), scans/searches (§III-C),
// load-balanced partitioning (§VI-A, Fig. 4), single/partial/multi-list
// decompression (§VI-B..D, Alg. 2, Figs. 5-7), forward pointers
// (P:157-163), EFG layout (§V).  What differs from the paper's Titan Xp
// design is listed in DESIGN.md §"Differences from the paper".
#include <cuda_runtime.h>

#include <algorithm>
#include <cstdint>

#include "efg_kernels.cuh"

namespace efg {

namespace {

constexpr uint32_t FULL = 0xffffffffu;

// --------------------------------------------------------------------------
// warp / block primitives (§III-C: exclusive scan, bounded search)
// --------------------------------------------------------------------------
__device__ __forceinline__ uint32_t lane_id() { return threadIdx.x & 31; }

__device__ __forceinline__ unsigned long long globaltimer()
{
    unsigned long long t;
    asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
    return t;
}

__device__ __forceinline__ uint32_t warp_excl_u32(uint32_t x, uint32_t &total)
{
    uint32_t inc = x;
#pragma unroll
    for (int d = 1; d < 32; d <<= 1) {
        const uint32_t y = __shfl_up_sync(FULL, inc, d);
        if ((int)lane_id() >= d) inc += y;
    }
    total = __shfl_sync(FULL, inc, 31);
    return inc - x;
}

__device__ __forceinline__ uint64_t warp_excl_u64(uint64_t x, uint64_t &total)
{
    uint64_t inc = x;
#pragma unroll
    for (int d = 1; d < 32; d <<= 1) {
        const uint64_t y = __shfl_up_sync(FULL, inc, d);
        if ((int)lane_id() >= d) inc += y;
    }
    total = __shfl_sync(FULL, inc, 31);
    return inc - x;
}

__device__ __forceinline__ uint64_t warp_sum_u64(uint64_t x)
{
#pragma unroll
    for (int d = 16; d; d >>= 1) x += __shfl_xor_sync(FULL, x, d);
    return x;
}

// binsearch_maxle over a non-decreasing key held one per lane (key of lane 0
// must be <= g): the largest lane t with key_t <= g; among equal keys the last
// (reading C13).  5 shuffle steps, every lane may search a different g.
__device__ __forceinline__ int warp_maxle_u32(uint32_t key, uint32_t g)
{
    int lo = 0;
#pragma unroll
    for (int step = 16; step; step >>= 1) {
        const int cand = lo + step;
        const uint32_t kc = __shfl_sync(FULL, key, cand);
        if (kc <= g) lo = cand;
    }
    return lo;
}

__device__ __forceinline__ uint32_t ldg_u32(const uint32_t *p) { return __ldg(p); }

// uint32 little-endian at an arbitrary byte offset of the 4-byte aligned data
__device__ __forceinline__ uint32_t ld_u32_unaligned(const uint32_t *data32, uint64_t byteoff)
{
    const uint64_t w = byteoff >> 2;
    const uint32_t lo = ldg_u32(data32 + w);
    const uint32_t hi = ldg_u32(data32 + w + 1);
    return __funnelshift_r(lo, hi, (uint32_t)(byteoff & 3) * 8);
}




// Chunk length CH = k (forward-pointer quantum), or 2^40 when k = 0 (lists are
// never split).  Divisions by CH use a shift when k is a power of two (the
// paper's k = 512), the generic 64-bit divide otherwise.
struct ChunkLen {
    uint64_t ch;
    int shift;  // log2(ch) or -1
    __device__ __forceinline__ uint64_t div(uint64_t x) const { return shift >= 0 ? x >> shift : x / ch; }
};

__device__ __forceinline__ ChunkLen make_chunk(uint32_t k, int kshift)
{
    ChunkLen c;
    c.ch = k ? k : (1ull << 40);
    c.shift = k ? kshift : 40;
    return c;
}

// Entry of tile t whose boundary t*T falls inside vertex q's work range
// [W, W + kVertexWork + d): the first chunk whose start is >= t*T (chunk 0
// starts at W, chunk c > 0 at W + kVertexWork + c*k), or the next vertex.
__device__ __forceinline__ TileEntry tile_entry(uint64_t t, uint64_t q, uint64_t W, uint64_t d,
                                                const ChunkLen &cl)
{
    const uint64_t ch = cl.ch, A = kVertexWork;
    const uint64_t o = t * kTileWork - W;
    TileEntry te;
    if (o == 0) {
        te.fi = (uint32_t)q;
        te.chunk = 0;
        te.w = W;
        return te;
    }
    uint64_t c = o > A ? cl.div(o - A + ch - 1) : 1;
    if (c == 0) c = 1;
    if (c * ch < d) {
        te.fi = (uint32_t)q;
        te.chunk = (uint32_t)c;
        te.w = W + A + c * ch;
    } else {
        te.fi = (uint32_t)(q + 1);
        te.chunk = 0;
        te.w = W + A + d;
    }
    return te;
}

// --------------------------------------------------------------------------
// Cross-block exclusive prefix for the two frontier scans (a2, a7).  A block
// publishes its aggregate as one 64-bit word tag << 40 | value (value < 2^40),
// with tag = the per-launch sequence number, so no clearing pass and no fence
// are needed (the value travels in the same single-copy-atomic word as its
// tag).  The block then sums the aggregates of ALL its predecessors with every
// load issued at once (grids are at most 2 x #SMs blocks), i.e. one or two L2
// round trips instead of a look-back chain.
// --------------------------------------------------------------------------
__device__ __forceinline__ uint64_t ld_relaxed_u64(const uint64_t *p)
{
    uint64_t v;
    asm volatile("ld.relaxed.gpu.global.u64 %0, [%1];" : "=l"(v) : "l"(p) : "memory");
    return v;
}

__device__ __forceinline__ void st_relaxed_u64(uint64_t *p, uint64_t v)
{
    asm volatile("st.relaxed.gpu.global.u64 [%0], %1;" ::"l"(p), "l"(v) : "memory");
}

constexpr int kTagShift = 40;
constexpr uint64_t kTagVal = (1ull << kTagShift) - 1;

// warp 0: publish `agg` for block b and return the sum over blocks < b
__device__ uint64_t publish_and_prefix(uint64_t *st, uint32_t b, uint32_t tag, uint64_t agg)
{
    const uint32_t lane = lane_id();
    const uint64_t t = (uint64_t)(tag & 0xffffffu);
    if (lane == 0) st_relaxed_u64(st + b, (t << kTagShift) | agg);
    uint64_t acc = 0;
    for (uint32_t base = 0; base < b; base += 32 * 8) {
        uint64_t w[8];
#pragma unroll
        for (int u = 0; u < 8; ++u) {
            const uint32_t idx = base + u * 32 + lane;
            w[u] = idx < b ? ld_relaxed_u64(st + idx) : (t << kTagShift);
        }
#pragma unroll
        for (int u = 0; u < 8; ++u) {
            const uint32_t idx = base + u * 32 + lane;
            while ((w[u] >> kTagShift) != t) w[u] = ld_relaxed_u64(st + idx);
            acc += w[u] & kTagVal;
        }
    }
    return warp_sum_u64(acc);
}

// block-wide exclusive scan of a u64 (256 threads); returns the block total in `total`
template <int NT>
__device__ __forceinline__ uint64_t block_excl_u64(uint64_t x, uint64_t &total, uint64_t *s_warp)
{
    const uint32_t lane = lane_id(), wid = threadIdx.x >> 5;
    uint64_t wt;
    const uint64_t ex = warp_excl_u64(x, wt);
    if (lane == 31) s_warp[wid] = wt;
    __syncthreads();
    uint64_t pre = 0, tot = 0;
#pragma unroll
    for (int w = 0; w < NT / 32; ++w) {
        const uint64_t v = s_warp[w];
        if (w < (int)wid) pre += v;
        tot += v;
    }
    __syncthreads();
    total = tot;
    return pre + ex;
}

__device__ __forceinline__ uint64_t block_sum_u64(uint64_t x, uint64_t *s_warp)
{
    uint64_t tot;
    block_excl_u64<kFrontierThreads>(x, tot, s_warp);
    return tot;
}

// --------------------------------------------------------------------------
// init_kernel: per-call state (level 0, a fresh tag) and the start set:
// BFS marks the source (Alg. 1 initial frontier), decode marks [v0, v1).
// --------------------------------------------------------------------------
__global__ void init_kernel(InitArgs a)
{
    if (blockIdx.x == 0 && threadIdx.x == 0) {
        a.ctrl->depth = a.depth;
        a.ctrl->parent = a.parent;
        a.ctrl->level = 0;
        a.ctrl->xlevel = 0;
        a.ctrl->seq = a.ctrl->seq + 1;
        a.ctrl->nlevels = 0;
        a.ctrl->nnew = 0;
        a.ctrl->total_nf = 0;
        a.ctrl->total_ne = 0;
        if (a.parent) a.parent[a.v0] = (uint32_t)a.v0;
    }
    const uint64_t w0 = a.v0 >> 5, w1 = (a.v1 + 31) >> 5;
    for (uint64_t w = w0 + blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; w < w1;
         w += (uint64_t)gridDim.x * blockDim.x) {
        uint32_t m = FULL;
        if (w == (a.v0 >> 5)) m &= FULL << (a.v0 & 31);
        if (w == ((a.v1 - 1) >> 5) && (a.v1 & 31)) m &= (1u << (a.v1 & 31)) - 1;
        a.vis[w] |= m;
    }
}

// --------------------------------------------------------------------------
// compact_kernel: a7 level end.  new = vis & ~prev; the new vertices, in
// increasing id order, become the next frontier queue (sorted for free, in
// place of the paper's partial radix sort); depth[new] = level.
// Reduce-then-scan over a persistent grid.  A block's word range is split into
// one contiguous run per warp.  Pass 1 counts (coalesced word loads); the
// cross-block prefix places the block, the per-warp counts place the warps;
// pass 2 walks 32 words at a time: a warp scan of the popcounts gives each
// word's queue offset and, word by word, lane b writes bit b's vertex, so the
// queue and depth stores are coalesced.  No block barrier inside the loops.
// --------------------------------------------------------------------------
__global__ void __launch_bounds__(kFrontierThreads) compact_kernel(CompactArgs a)
{
    constexpr int NT = kFrontierThreads, NW = NT / 32;
    __shared__ uint64_t s_warp[NW];
    __shared__ uint64_t s_wcnt[NW];
    __shared__ uint64_t s_pre;

    const uint32_t tid = threadIdx.x, lane = tid & 31, wid = tid >> 5, b = blockIdx.x;
    const LevelCtrl *ctrl = a.ctrl;
    const uint32_t tag = ctrl->seq;
    const int32_t level = (int32_t)ctrl->level;
    int32_t *depth = ctrl->depth;
    const uint64_t lo = (uint64_t)b * a.words_per_block;
    const uint64_t hi = min(lo + a.words_per_block, a.nwords);
    const uint64_t per_w = (a.words_per_block + NW - 1) / NW;
    const uint64_t wlo = min(lo + wid * per_w, hi), whi = min(wlo + per_w, hi);

    // pass 1: count (queue = owned words only; nnew = every row); 4 loads in flight
    uint64_t cnt = 0, all = 0;
    for (uint64_t w0 = wlo + lane; w0 < whi; w0 += 128) {
        uint32_t c[4];
#pragma unroll
        for (int u = 0; u < 4; ++u) {
            const uint64_t w = w0 + 32 * u;
            c[u] = w < whi ? __popc(a.consume ? a.vis[w] : (a.vis[w] & ~a.prev[w])) : 0u;
        }
#pragma unroll
        for (int u = 0; u < 4; ++u) {
            const uint64_t w = w0 + 32 * u;
            all += c[u];
            if (w >= a.own_lo_w && w < a.own_hi_w) cnt += c[u];
        }
    }
    cnt = warp_sum_u64(cnt);
    all = warp_sum_u64(all);
    if (lane == 0) {
        s_wcnt[wid] = cnt;
        s_warp[wid] = all;
    }
    __syncthreads();
    if (wid == 0) {
        const uint64_t bc = lane < NW ? s_wcnt[lane] : 0, ba = lane < NW ? s_warp[lane] : 0;
        const uint64_t blk = warp_sum_u64(bc), blk_all = warp_sum_u64(ba);
        if (lane == 0 && blk_all) atomicAdd(reinterpret_cast<unsigned long long *>(&a.ctrl->nnew), blk_all);
        const uint64_t pre = publish_and_prefix(a.status, b, tag, blk);
        if (lane == 0) {
            s_pre = pre;
            if (b == gridDim.x - 1) a.ctrl->nf = pre + blk;
        }
    }
    __syncthreads();
    uint64_t base = s_pre;
    for (uint32_t w = 0; w < wid; ++w) base += s_wcnt[w];

    // pass 2: queue + depth
    const uint32_t lt = (1u << lane) - 1;
    for (uint64_t w0 = wlo; w0 < whi; w0 += 32) {
        const uint64_t w = w0 + lane;
        uint32_t nb = 0;
        if (w < whi) {
            const uint32_t x = a.vis[w];
            if (a.consume) {  // SSSP: the relaxed set itself is the next frontier; reset it
                nb = x;
                if (x) a.vis[w] = 0;
            } else {
                const uint32_t p = a.prev[w];
                nb = x & ~p;
                if (nb) a.prev[w] = x;
            }
        }
        const bool own = w >= a.own_lo_w && w < a.own_hi_w;
        const uint32_t nq = own ? nb : 0u;
        uint32_t tq;
        const uint32_t off = warp_excl_u32(__popc(nq), tq);
        uint32_t todo = __ballot_sync(FULL, nb != 0);
        while (todo) {
            const int j = __ffs(todo) - 1;
            todo &= todo - 1;
            const uint32_t nbw = __shfl_sync(FULL, nb, j);
            const uint32_t nqw = __shfl_sync(FULL, nq, j);
            const uint32_t offj = __shfl_sync(FULL, off, j);
            if ((nbw >> lane) & 1) {
                const uint32_t v = (uint32_t)((w0 + j) * 32 + lane);
                if (a.depth_stored) a.depth_stored[v] = level;  // stored-id order (coalesced)
                if (!a.depth_stored_only && depth) depth[v] = level;
                if (nqw) a.queue[base + offj + __popc(nqw & lt)] = v;
            }
        }
        base += tq;
    }
}

// --------------------------------------------------------------------------
// Exchange kernels of the 1-D partitioned BFS.  Slices are the
// owners' bitmap word ranges [bw[h], bw[h+1]), padded to S words.
//   pack:   send[h*S + i] = (vis & ~prev)[bw[h] + i]      (this rank's new bits)
//   reduce: mine[i] = OR_p recv[p*S + i]                    (owner ORs P slices)
//   unpack: vis[bw[h] + i] |= gathered[h*S + i]            (global new bits)
// --------------------------------------------------------------------------
__global__ void xchg_kernel(XchgArgs a)
{
    const uint64_t total = (uint64_t)(a.op == 1 ? 1 : a.world) * a.S;
    for (uint64_t t = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; t < total;
         t += (uint64_t)gridDim.x * blockDim.x) {
        if (a.op == 1) {
            uint32_t m = 0;
            for (int p = 0; p < a.world; ++p) m |= a.in[(uint64_t)p * a.S + t];
            a.out[t] = m;
            continue;
        }
        const int h = (int)(t / a.S);
        const uint64_t i = t - (uint64_t)h * a.S;
        const uint64_t w0 = a.bounds[h] / 32, w1 = (a.bounds[h + 1] + 31) / 32;
        const uint64_t w = w0 + i;
        if (a.op == 0)
            a.out[t] = w < w1 ? (a.vis[w] & ~a.prev[w]) : 0u;
        else if (w < w1 && a.in[t])
            a.vis[w] |= a.in[t];
    }
}

// --------------------------------------------------------------------------
// plan_kernel: a1 + a2 + a3.  For the sorted frontier queue: degree lookup
// (a1), exclusive scan of the per-vertex work kVertexWork + deg (a2), and the
// tile table (a3: each tile of kTileWork units gets its first chunk, the
// Fig. 4 maxle rule applied once per tile).  Same reduce-then-scan scheme as
// compact_kernel, over the frontier index range.  The last block publishes
// the level totals, records per-level statistics and, in graph mode, sets the
// loop condition (frontier non-empty).
// --------------------------------------------------------------------------
__global__ void __launch_bounds__(kFrontierThreads) plan_kernel(PlanArgs a)
{
    constexpr int NT = kFrontierThreads, NW = NT / 32;
    __shared__ uint64_t s_wwork[NW];
    __shared__ uint64_t s_pre;

    const uint32_t tid = threadIdx.x, lane = tid & 31, wid = tid >> 5, b = blockIdx.x;
    LevelCtrl *ctrl = a.ctrl;
    const uint32_t tag = ctrl->seq;
    const uint64_t nf = ctrl->nf;
    const ChunkLen cl = make_chunk(a.k, a.kshift);
    const uint64_t A = kVertexWork;
    const uint64_t per = (nf + gridDim.x - 1) / gridDim.x;
    const uint64_t lo = min((uint64_t)b * per, nf), hi = min(lo + per, nf);
    const uint64_t per_w = (per + NW - 1) / NW;
    const uint64_t qlo = min(lo + wid * per_w, hi), qhi = min(qlo + per_w, hi);

    // pass 1: work of the warp's range (a1 degree lookup), 4 lookups in flight
    uint64_t wk = 0;
    for (uint64_t i0 = qlo + lane; i0 < qhi; i0 += 128) {
        uint32_t q[4];
#pragma unroll
        for (int u = 0; u < 4; ++u) q[u] = i0 + 32 * u < qhi ? a.queue[i0 + 32 * u] : 0u;
#pragma unroll
        for (int u = 0; u < 4; ++u)
            if (i0 + 32 * u < qhi) wk += A + __ldg(a.deg32 + q[u]);
    }
    wk = warp_sum_u64(wk);
    if (lane == 0) s_wwork[wid] = wk;
    __syncthreads();
    if (wid == 0) {
        const uint64_t blk = warp_sum_u64(lane < NW ? s_wwork[lane] : 0);
        const uint64_t pre = publish_and_prefix(a.status, b, tag, blk);
        if (lane == 0) {
            s_pre = pre;
            if (b == gridDim.x - 1) {
                const uint64_t nwork = pre + blk;
                const uint32_t lvl = ctrl->level;
                ctrl->nwork = nwork;
                ctrl->ne = nwork - A * nf;
                ctrl->ntiles = (nwork + kTileWork - 1) / kTileWork;
                ctrl->xlevel = lvl;
                if (nf) {
                    ctrl->nlevels = lvl + 1;
                    ctrl->total_nf += nf;
                    ctrl->total_ne += nwork - A * nf;
                    if (a.stats && lvl < a.max_stats) {
                        a.stats[lvl].nf = nf;
                        a.stats[lvl].ne = nwork - A * nf;
                        a.stats[lvl].t0 = ~0ull;
                        a.stats[lvl].t1 = 0;
                    }
                }
                if (a.cond) cudaGraphSetConditional(a.cond, nf ? 1u : 0u);
            }
        }
    }
    __syncthreads();
    uint64_t run = s_pre;
    for (uint32_t w = 0; w < wid; ++w) run += s_wwork[w];

    // pass 2: exclusive scan of the work (a2) and the tile table (a3); the next
    // 32 degrees are fetched while the current ones are scanned
    uint32_t dn = qlo + lane < qhi ? __ldg(a.deg32 + a.queue[qlo + lane]) : 0u;
    for (uint64_t i0 = qlo; i0 < qhi; i0 += 32) {
        const uint64_t i = i0 + lane;
        const uint64_t d = dn;
        if (i0 + 32 < qhi) dn = i + 32 < qhi ? __ldg(a.deg32 + a.queue[i + 32]) : 0u;
        uint64_t tot;
        const uint64_t W = run + warp_excl_u64(i < qhi ? A + d : 0, tot);
        // tiles whose boundary t*T falls in this group's work window
        // [W_0, W_0 + tot): lanes take consecutive tiles, each finds its vertex
        // by maxle over the group's W (Fig. 4 rule inside the warp)
        const uint64_t wstart = __shfl_sync(FULL, W, 0);
        const uint64_t tfirst = (wstart + kTileWork - 1) / kTileWork;
        const uint64_t tend = (wstart + tot + kTileWork - 1) / kTileWork;
        const uint32_t wrel = i < qhi ? (uint32_t)(W - wstart) : 0xffffffffu;  // < tot <= 2^32
        for (uint64_t t0 = tfirst; t0 < tend; t0 += 32) {
            const uint64_t t = t0 + lane;
            const uint32_t key = t < tend ? (uint32_t)(t * kTileWork - wstart) : 0u;
            const int j = warp_maxle_u32(wrel, key);
            const uint64_t jW = __shfl_sync(FULL, W, j), jd = __shfl_sync(FULL, d, j);
            if (t < tend) a.tiles[t] = tile_entry(t, i0 + j, jW, jd, cl);
        }
        run += tot;
    }
}

// --------------------------------------------------------------------------
// expand_kernel: a4 + a5 + a6 (P:137-177 generalised, Alg. 1 lines 3-6)
//
// Persistent: one CTA of kExpandThreads per SM, one warp per work tile.  A
// tile's work is a run of "chunks": k-aligned pieces of frontier lists
// (P:157), so every chunk starts right after a forward pointer and needs no
// select to find its first bit.  Chunks are taken 32 at a time ("batch"; many
// short lists per warp: the multi-list case).  The batch's
// upper-bit words are laid end to end and processed 32 words per step (one
// aligned 32-bit word per lane, coalesced; the next step's word is loaded
// before the current one is used):
//   popcount + warp exclusive scan -> rank of each word's first stop bit (the
//                                     segmented scan of P:171-177; segments are
//                                     chunks, whose element prefix is subtracted)
//   set-bit enumeration (ffs)       -> select1(i) - i per element, staged in
//                                     shared memory by element slot (Alg. 2's
//                                     select step, without its byte LUT)
//   balanced pass, element e on lane e%32, kVisitBatch in flight, branch-free
//                                   -> lower bits by a funnel shift of two
//                                     coalesced words, x = hi << l | lo, visit.
// Visit: the first hot_words*32 vertex ids (the highest-degree vertices when the
// graph was built with EFG_REORDER_DEGREE) have a per-CTA shared-memory copy of
// their visited bits, loaded at kernel start (a snapshot of the level start,
// updated by this CTA's own discoveries).  A set bit there answers the probe
// without touching L1/L2; otherwise the global bitmap is probed and the
// atomicOr decides (stale reads are benign).
// --------------------------------------------------------------------------
struct SlotGeom {
    uint64_t A0, A1, U0;  // absolute bit range of the chunk's upper bits; upper start
    uint32_t wb, eb;      // exclusive word / element prefix within the batch
    uint64_t r0;          // rank of the chunk's first element in its list
};

struct alignas(16) SlotMeta {
    uint64_t lb;     // lower-bit address of batch element e: lb + e*l (modular)
    uint32_t l;      // lower bits per element
    uint32_t lmask;  // (1 << l) - 1
};

struct WarpSmem {
    // per element of the step: (select1(i) - i) << 5 | chunk slot.  select1(i) - i
    // = x >> l < 2 * deg, and degrees are < 2^26 (checked at build), so it fits.
    uint32_t hs[kExpandStage];
    SlotGeom geom[32];
    SlotMeta meta[32];
    uint64_t aux[32];           // parent: source vertex; decode: output index base;
                                // SSSP: weight index base; PageRank: share (double bits)
    float aux2[32];             // SSSP: dist of the chunk's source vertex
};

struct WordLd {
    uint32_t word;
    int s;
    uint64_t wi;
};

__device__ __forceinline__ WordLd load_word(const uint32_t *data32, const SlotGeom *geom,
                                            uint32_t wb, uint32_t g, uint32_t W)
{
    WordLd r;
    r.s = warp_maxle_u32(wb, g);
    r.word = 0;
    r.wi = 0;
    if (g < W) {
        const SlotGeom &sg = geom[r.s];
        const uint64_t w0 = sg.A0 >> 5, wl = (sg.A1 - 1) >> 5;
        r.wi = w0 + (g - sg.wb);
        uint32_t word = ldg_u32(data32 + r.wi);
        if (r.wi == w0) word &= FULL << (uint32_t)(sg.A0 & 31);
        if (r.wi == wl) {
            const uint32_t hb = (uint32_t)(sg.A1 - wl * 32);  // 1..32 valid bits
            if (hb < 32) word &= (1u << hb) - 1;
        }
        r.word = word;
    }
    return r;
}

// Lane l of a step handles the 16-bit half (l & 1) of batch word g0 + (l >> 1).
__device__ __forceinline__ WordLd load_half(const uint32_t *data32, const SlotGeom *geom, uint32_t wb,
                                            uint32_t lane, uint32_t g0, uint32_t W)
{
    WordLd r = load_word(data32, geom, wb, g0 + (lane >> 1), W);
    r.word = (lane & 1) ? (r.word >> 16) : (r.word & 0xffffu);
    return r;
}

__device__ __forceinline__ void prefetch_l2(const void *p)
{
    asm volatile("prefetch.global.L2 [%0];" ::"l"(p));
}

constexpr int kVisitBatch = 2;  // decoded elements per lane whose probes are in flight together

template <int MODE>
__global__ void __launch_bounds__(kExpandThreads, 1) expand_kernel(ExpandArgs a)
{
    extern __shared__ __align__(16) uint8_t smem_raw[];
    uint32_t *s_hot = reinterpret_cast<uint32_t *>(smem_raw);
    WarpSmem *ws_all = reinterpret_cast<WarpSmem *>(smem_raw + kHotWords * 4);

    const uint32_t lane = lane_id(), wid = threadIdx.x >> 5;
    WarpSmem &ws = ws_all[wid];
    const uint64_t ntiles = a.ctrl->ntiles, nf = a.ctrl->nf, nwork = a.ctrl->nwork;
    const uint32_t xl = a.ctrl->xlevel;  // index of the level being expanded
    uint32_t *parent = MODE == kModeVisitParent ? a.ctrl->parent : nullptr;
    const uint32_t hot_limit = a.hot_words * 32;  // vertex ids below this use s_hot
    constexpr bool kBfs = MODE == kModeVisit || MODE == kModeVisitParent;
    if (MODE != kModeDecode) {
        if (threadIdx.x == 0 && a.stats && xl < a.max_stats) atomicMin(&a.stats[xl].t0, globaltimer());
        if (blockIdx.x == 0 && threadIdx.x == 0) {
            a.ctrl->level = xl + 1;  // depth of the vertices this launch discovers
            a.ctrl->seq = a.ctrl->seq + 1;
            a.ctrl->nnew = 0;
        }
    }
    if (kBfs) {
        // level-start snapshot of the hot visited words
        const uint4 *src = reinterpret_cast<const uint4 *>(a.vis);
        uint4 *dst = reinterpret_cast<uint4 *>(s_hot);
        for (uint32_t i = threadIdx.x; i < a.hot_words / 4; i += blockDim.x) dst[i] = src[i];
        __syncthreads();
    }
    const uint32_t *data32 = reinterpret_cast<const uint32_t *>(a.data);
    const ChunkLen cl = make_chunk(a.k, a.kshift);
    const uint64_t CH = cl.ch;
    const uint64_t A = kVertexWork;
    const uint64_t gw = (uint64_t)blockIdx.x * kExpandWarps + wid;
    const uint64_t nwarps = (uint64_t)gridDim.x * kExpandWarps;

    for (uint64_t tile = gw; tile < ntiles; tile += nwarps) {
        const TileEntry te = a.tiles[tile];
        uint64_t fi = te.fi, c0 = te.chunk, P = te.w;
        const uint64_t Pend = min((tile + 1) * (uint64_t)kTileWork, nwork);

        while (P < Pend && fi < nf) {
            // ---- a1 (gather): up to 32 frontier vertices, one per lane ----
            const uint64_t fv = fi + lane;
            uint32_t v = 0, deg = 0, ubytes = 0;
            uint64_t offl = 0;
            if (fv < nf) {
                v = a.queue[fv];
                const uint4 r = __ldg(reinterpret_cast<const uint4 *>(a.rec + v));
                offl = ((uint64_t)r.y << 32) | r.x;
                deg = r.z;
                ubytes = r.w;
            }
            const uint64_t first = lane == 0 ? c0 : 0;
            const uint64_t nch = deg ? cl.div(deg + CH - 1) : 0;
            const uint32_t nrem = (uint32_t)(nch > first ? nch - first : 0);
            // work still ahead of this vertex (from its first remaining chunk on)
            const uint64_t wrem = fv < nf ? (first == 0 ? A + deg : deg - first * CH) : 0;
            uint32_t totc;
            const uint32_t cb = warp_excl_u32(nrem, totc);
            uint64_t totw;
            const uint64_t wbv = warp_excl_u64(wrem, totw);
            // W_v of each vertex (work position of its chunk 0)
            const uint64_t Wv = P + wbv - (first ? A + first * CH : 0);
            if (totc == 0) {  // 32 empty lists
                fi += 32;
                c0 = 0;
                P += totw;
                continue;
            }

            // ---- chunk slot t = lane -> owning vertex lane j (maxle, C13) ----
            const int j = warp_maxle_u32(cb, lane);
            const uint32_t deg_j = __shfl_sync(FULL, deg, j);
            const uint64_t offl_j = __shfl_sync(FULL, offl, j);
            const uint32_t ub_j = __shfl_sync(FULL, ubytes, j);
            const uint32_t cb_j = __shfl_sync(FULL, cb, j);
            const uint64_t Wv_j = __shfl_sync(FULL, Wv, j);
            const uint32_t v_j = __shfl_sync(FULL, v, j);
            const uint64_t nch_j = __shfl_sync(FULL, nch, j);
            const uint64_t cc = (j == 0 ? c0 : 0) + (lane - cb_j);
            const uint64_t r0 = cc * CH;
            const uint64_t cstart = Wv_j + (cc ? A + cc * CH : 0);
            const bool valid = lane < totc && cstart < Pend;
            const uint32_t count = __popc(__ballot_sync(FULL, valid));
            if (count == 0) break;

            // ---- a4: bit ranges of the chunk (forward pointers) ----
            uint32_t nwd = 0, nel = 0;
            uint64_t A0 = 0, A1 = 0, U0 = 0, lbase = 0;
            uint32_t l = 0;
            if (valid) {
                const uint64_t off = offl_j & kOffMask;
                l = (uint32_t)(offl_j >> kOffBits);
                const uint64_t F = a.k ? cl.div(deg_j) : 0;
                const uint64_t L = ((uint64_t)deg_j * l + 7) >> 3;
                lbase = (off + 4 * F) * 8;
                U0 = (off + 4 * F + L) * 8;
                const uint64_t r1 = min(r0 + CH, (uint64_t)deg_j);
                nel = (uint32_t)(r1 - r0);
                const uint64_t b0 = cc ? (uint64_t)ld_u32_unaligned(data32, off + 4 * (cc - 1)) + r0 : 0;
                const uint64_t b1 = r1 < deg_j ? (uint64_t)ld_u32_unaligned(data32, off + 4 * cc) + r1
                                               : 8ull * ub_j;
                A0 = U0 + b0;
                A1 = U0 + b1;
                nwd = (uint32_t)(((A1 - 1) >> 5) - (A0 >> 5) + 1);
            }
            uint32_t W, NE;
            const uint32_t wb = warp_excl_u32(nwd, W);
            const uint32_t ebt = warp_excl_u32(nel, NE);
            (void)NE;
            if (valid) {
                ws.geom[lane] = SlotGeom{A0, A1, U0, wb, ebt, r0};
                SlotMeta m;
                m.lb = lbase + (r0 - (uint64_t)ebt) * l;  // modular: rank = r0 + (e - ebt)
                m.l = l;
                m.lmask = l ? (FULL >> (32 - l)) : 0u;
                ws.meta[lane] = m;
                // pull the chunk's lower and upper bits toward L2 ahead of the word steps
                {
                    const uint64_t lb0 = (lbase + r0 * l) >> 3, lb1 = (lbase + (r0 + nel) * l + 7) >> 3;
                    for (uint64_t q = lb0 & ~127ull; q < lb1; q += 128) prefetch_l2(a.data + q);
                    for (uint64_t q = (A0 >> 3) & ~127ull; q < ((A1 + 7) >> 3); q += 128) prefetch_l2(a.data + q);
                }
                if (MODE == kModeVisitParent) ws.aux[lane] = v_j;
                if (MODE == kModeSssp) {  // weights are stored in CSR order: index vlist[u] + rank
                    ws.aux[lane] = a.vlist[v_j] + r0 - ebt;
                    ws.aux2[lane] = a.dist[v_j];
                }
                if (MODE == kModePagerank) {  // push r(u)/deg(u) along every edge
                    const double share = a.rank[v_j] / (double)deg_j;
                    ws.aux[lane] = (uint64_t)__double_as_longlong(share);
                }
                // decode: CSR position of the chunk's first element E_v + r0, E_v = W_v - A*q_v
                if (MODE == kModeDecode) ws.aux[lane] = Wv_j - A * (fi + (uint64_t)j) + r0 - ebt;
            }
            // state after this batch: continue after the last valid chunk
            {
                const int tl = (int)count - 1;
                const uint64_t last_cc = __shfl_sync(FULL, cc, tl);
                const uint64_t last_nch = __shfl_sync(FULL, nch_j, tl);
                const int last_j = __shfl_sync(FULL, j, tl);
                const uint64_t last_W = __shfl_sync(FULL, Wv_j, tl);
                const uint32_t last_deg = __shfl_sync(FULL, deg_j, tl);
                if (last_cc + 1 < last_nch) {
                    fi += last_j;
                    c0 = last_cc + 1;
                    P = last_W + A + c0 * CH;
                } else {
                    fi += last_j + 1;
                    c0 = 0;
                    P = last_W + A + last_deg;
                }
            }
            __syncwarp();

            // ---- a5 + a6: 16 upper-bit words per step, one 16-bit half per lane ----
            uint32_t run = 0;
            WordLd nxt = load_half(data32, ws.geom, wb, lane, 0, W);
            for (uint32_t g0 = 0; g0 < W; g0 += 16) {
                const WordLd cur = nxt;
                if (g0 + 16 < W) nxt = load_half(data32, ws.geom, wb, lane, g0 + 16, W);
                uint32_t tot;
                const uint32_t ep = warp_excl_u32(__popc(cur.word), tot);
                // set-bit enumeration: select1(i) - i of every element, by slot
                if (cur.word) {
                    const SlotGeom &sg = ws.geom[cur.s];
                    const uint64_t rank = sg.r0 + run + ep - sg.eb;  // rank of the first set bit
                    // hi = hb + p (p = bit within the half), hb -= 1 per bit
                    // hi of the bit at position b with e = its slot: hbe + b - e
                    const uint32_t hbe = (uint32_t)(cur.wi * 32 + (lane & 1) * 16 - sg.U0 - rank) + ep;
                    const uint32_t w = cur.word;
                    const uint32_t sc = (uint32_t)cur.s;
                    uint32_t e = ep;
                    // uniform 16-step scan of the half-word (no lane waits on the
                    // densest half of the warp, unlike an ffs loop)
#pragma unroll
                    for (int b = 0; b < 16; ++b) {
                        if ((w >> b) & 1) {
                            ws.hs[e] = ((hbe + b - e) << 5) | sc;
                            ++e;
                        }
                    }
                }
                __syncwarp();
                // balanced pass: element e on lane e % 32, kVisitBatch in flight,
                // written branch-free (slots past the step are computed and masked)
                for (uint32_t base = 0; base < tot; base += 32 * kVisitBatch) {
                    uint32_t xv[kVisitBatch], sv[kVisitBatch];
                    bool ok[kVisitBatch];
#pragma unroll
                    for (int u = 0; u < kVisitBatch; ++u) {
                        const uint32_t e = base + u * 32 + lane;
                        ok[u] = e < tot;
                        const uint32_t es = ok[u] ? e : 0;
                        const uint32_t hsv = ws.hs[es];
                        const uint32_t hi = hsv >> 5;
                        sv[u] = hsv & 31;
                        const SlotMeta m = ws.meta[sv[u]];
                        const uint64_t ba = m.lb + (uint64_t)(run + es) * m.l;
                        const uint32_t *p = data32 + (ba >> 5);
                        const uint32_t lo =
                            __funnelshift_r(ldg_u32(p), ldg_u32(p + 1), (uint32_t)(ba & 31)) & m.lmask;
                        xv[u] = (hi << m.l) | lo;  // (select1(i) - i) << l | lower[i]
                    }
                    if (MODE == kModeDecode) {
#pragma unroll
                        for (int u = 0; u < kVisitBatch; ++u)
                            if (ok[u]) a.out[ws.aux[sv[u]] + run + base + u * 32 + lane] = xv[u];
                    } else if (MODE == kModeSssp) {
                        // relax: d' = fl32(dist(u) + w), single rounding (reading C20)
                        float nd[kVisitBatch], cd[kVisitBatch];
#pragma unroll
                        for (int u = 0; u < kVisitBatch; ++u) {
                            nd[u] = INFINITY;
                            cd[u] = 0.f;
                            if (ok[u]) {
                                const float w = __ldg(a.weights + ws.aux[sv[u]] + run + base + u * 32 + lane);
                                nd[u] = __fadd_rn(ws.aux2[sv[u]], w);
                                cd[u] = a.dist[xv[u]];
                            }
                        }
#pragma unroll
                        for (int u = 0; u < kVisitBatch; ++u) {
                            if (ok[u] && nd[u] < cd[u]) {  // non-negative floats order like their bits
                                const int old = atomicMin(reinterpret_cast<int *>(a.dist) + xv[u], __float_as_int(nd[u]));
                                if (__float_as_int(nd[u]) < old) atomicOr(a.vis + (xv[u] >> 5), 1u << (xv[u] & 31));
                            }
                        }
                    } else if (MODE == kModePagerank) {
#pragma unroll
                        for (int u = 0; u < kVisitBatch; ++u)
                            if (ok[u]) atomicAdd(a.next + xv[u], __longlong_as_double((long long)ws.aux[sv[u]]));
                    } else {
                        // Alg. 1 line 3: hot ids answer from shared memory
                        bool need[kVisitBatch], hot[kVisitBatch];
#pragma unroll
                        for (int u = 0; u < kVisitBatch; ++u) {
                            hot[u] = ok[u] && xv[u] < hot_limit;
                            const uint32_t hw = hot[u] ? s_hot[xv[u] >> 5] : 0u;
                            need[u] = ok[u] && !((hw >> (xv[u] & 31)) & 1);
                        }
                        uint32_t gwd[kVisitBatch];
#pragma unroll
                        for (int u = 0; u < kVisitBatch; ++u) gwd[u] = need[u] ? a.vis[xv[u] >> 5] : FULL;
                        bool act = false;
#pragma unroll
                        for (int u = 0; u < kVisitBatch; ++u) act |= need[u];
                        if (__any_sync(FULL, act)) {  // most probes of a heavy level stop here
#pragma unroll
                            for (int u = 0; u < kVisitBatch; ++u) {
                                const uint32_t bit = 1u << (xv[u] & 31);
                                if (!(gwd[u] & bit)) {  // line 4 (stale reads are benign: the atomic decides)
                                    if (MODE == kModeVisit) {
                                        atomicOr(a.vis + (xv[u] >> 5), bit);
                                    } else {
                                        const uint32_t old = atomicOr(a.vis + (xv[u] >> 5), bit);
                                        if (!(old & bit)) parent[xv[u]] = (uint32_t)ws.aux[sv[u]];
                                    }
                                }
                                if (need[u] && hot[u]) atomicOr(s_hot + (xv[u] >> 5), bit);
                            }
                        }
                    }
                }
                __syncwarp();
                run += tot;
            }
        }
    }
    if (MODE != kModeDecode && threadIdx.x == 0 && a.stats && xl < a.max_stats)
        atomicMax(&a.stats[xl].t1, globaltimer());
}

// PageRank (reading C21): D = sum of rank over degree-0 vertices; then
// r'(v) = (1-d)/N + d * (next(v) + D/N), next(v) = 0.  fp64 throughout.
__global__ void pr_dangling_kernel(const double *rank, const uint32_t *deg32, uint64_t n, double *dsum)
{
    double acc = 0.0;
    for (uint64_t v = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; v < n; v += (uint64_t)gridDim.x * blockDim.x)
        if (deg32[v] == 0) acc += rank[v];
#pragma unroll
    for (int d = 16; d; d >>= 1) acc += __shfl_xor_sync(FULL, acc, d);
    if ((threadIdx.x & 31) == 0 && acc != 0.0) atomicAdd(dsum, acc);
}

__global__ void pr_update_kernel(double *rank, double *next, uint64_t n, double damping, const double *dsum)
{
    const double base = (1.0 - damping) / (double)n, dn = *dsum / (double)n;
    for (uint64_t v = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; v < n; v += (uint64_t)gridDim.x * blockDim.x) {
        rank[v] = base + damping * (next[v] + dn);
        next[v] = 0.0;
    }
}

__global__ void fill_kernel(uint32_t *p, uint32_t val, uint64_t n)
{
    for (uint64_t i = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; i < n; i += (uint64_t)gridDim.x * blockDim.x)
        p[i] = val;
}

__global__ void fill_f64_kernel(double *p, double val, uint64_t n)
{
    for (uint64_t i = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; i < n; i += (uint64_t)gridDim.x * blockDim.x)
        p[i] = val;
}

// out[v] = stored[new_of_old[v]] for 32- or 64-bit values (relabelled graphs)
__global__ void gather32_kernel(const uint32_t *stored, const uint32_t *new_of_old, uint32_t *out, uint64_t n)
{
    for (uint64_t v = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; v < n; v += (uint64_t)gridDim.x * blockDim.x)
        out[v] = stored[new_of_old ? new_of_old[v] : v];
}

__global__ void gather64_kernel(const double *stored, const uint32_t *new_of_old, double *out, uint64_t n)
{
    for (uint64_t v = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; v < n; v += (uint64_t)gridDim.x * blockDim.x)
        out[v] = stored[new_of_old ? new_of_old[v] : v];
}

// depth_out[old_of_new[i]] = depth_stored[i] as a gather over input ids:
// depth_out[v] = depth_stored[new_of_old[v]] (coalesced stores).
__global__ void map_depth_kernel(const int32_t *stored, const uint32_t *new_of_old, int32_t *out, uint64_t n)
{
    for (uint64_t v = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; v < n; v += (uint64_t)gridDim.x * blockDim.x)
        out[v] = stored[new_of_old[v]];
}

__global__ void map_parent_kernel(const uint32_t *pin, const uint32_t *old_of_new, uint32_t *pout, uint64_t n)
{
    for (uint64_t i = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; i < n; i += (uint64_t)gridDim.x * blockDim.x) {
        const uint32_t p = pin[i];
        pout[old_of_new[i]] = p == FULL ? FULL : old_of_new[p];
    }
}

}  // namespace

static unsigned grid_for(uint64_t n) { return (unsigned)std::max<uint64_t>(1, std::min<uint64_t>((n + 255) / 256, 148 * 16)); }

cudaError_t launch_pr_dangling(const double *rank, const uint32_t *deg32, uint64_t n, double *dsum, cudaStream_t s)
{
    pr_dangling_kernel<<<grid_for(n), 256, 0, s>>>(rank, deg32, n, dsum);
    return cudaGetLastError();
}

cudaError_t launch_pr_update(double *rank, double *next, uint64_t n, double damping, const double *dsum,
                             cudaStream_t s)
{
    pr_update_kernel<<<grid_for(n), 256, 0, s>>>(rank, next, n, damping, dsum);
    return cudaGetLastError();
}

cudaError_t launch_fill(uint32_t *p, uint32_t val, uint64_t n, cudaStream_t s)
{
    fill_kernel<<<grid_for(n), 256, 0, s>>>(p, val, n);
    return cudaGetLastError();
}

cudaError_t launch_fill_f64(double *p, double val, uint64_t n, cudaStream_t s)
{
    fill_f64_kernel<<<grid_for(n), 256, 0, s>>>(p, val, n);
    return cudaGetLastError();
}

cudaError_t launch_gather32(const uint32_t *stored, const uint32_t *new_of_old, uint32_t *out, uint64_t n,
                            cudaStream_t s)
{
    gather32_kernel<<<grid_for(n), 256, 0, s>>>(stored, new_of_old, out, n);
    return cudaGetLastError();
}

cudaError_t launch_gather64(const double *stored, const uint32_t *new_of_old, double *out, uint64_t n,
                            cudaStream_t s)
{
    gather64_kernel<<<grid_for(n), 256, 0, s>>>(stored, new_of_old, out, n);
    return cudaGetLastError();
}

cudaError_t launch_map_depth(const int32_t *stored, const uint32_t *new_of_old, int32_t *out, uint64_t n,
                             cudaStream_t s)
{
    const unsigned blocks = (unsigned)std::max<uint64_t>(1, std::min<uint64_t>((n + 255) / 256, 148 * 16));
    map_depth_kernel<<<blocks, 256, 0, s>>>(stored, new_of_old, out, n);
    return cudaGetLastError();
}

cudaError_t launch_map_parent(const uint32_t *pin, const uint32_t *old_of_new, uint32_t *pout, uint64_t n,
                              cudaStream_t s)
{
    const unsigned blocks = (unsigned)std::max<uint64_t>(1, std::min<uint64_t>((n + 255) / 256, 148 * 16));
    map_parent_kernel<<<blocks, 256, 0, s>>>(pin, old_of_new, pout, n);
    return cudaGetLastError();
}

size_t expand_smem_bytes() { return (size_t)kHotWords * 4 + (size_t)kExpandWarps * sizeof(WarpSmem); }

static cudaError_t expand_set_attrs()
{
    static bool done = false;
    if (done) return cudaSuccess;
    const int bytes = (int)expand_smem_bytes();
    cudaError_t e = cudaFuncSetAttribute(expand_kernel<kModeVisit>, cudaFuncAttributeMaxDynamicSharedMemorySize, bytes);
    if (e == cudaSuccess)
        e = cudaFuncSetAttribute(expand_kernel<kModeVisitParent>, cudaFuncAttributeMaxDynamicSharedMemorySize, bytes);
    if (e == cudaSuccess)
        e = cudaFuncSetAttribute(expand_kernel<kModeDecode>, cudaFuncAttributeMaxDynamicSharedMemorySize, bytes);
    if (e == cudaSuccess)
        e = cudaFuncSetAttribute(expand_kernel<kModeSssp>, cudaFuncAttributeMaxDynamicSharedMemorySize, bytes);
    if (e == cudaSuccess)
        e = cudaFuncSetAttribute(expand_kernel<kModePagerank>, cudaFuncAttributeMaxDynamicSharedMemorySize, bytes);
    if (e == cudaSuccess) done = true;
    return e;
}

int expand_occupancy(int mode)
{
    (void)mode;
    return 1;  // one CTA per SM (shared-memory resident hot bitmap)
}

cudaError_t launch_expand(int mode, const ExpandArgs &a, int blocks, cudaStream_t s)
{
    cudaError_t e = expand_set_attrs();
    if (e != cudaSuccess) return e;
    const size_t sm = expand_smem_bytes();
    switch (mode) {
    case kModeVisit:
        expand_kernel<kModeVisit><<<blocks, kExpandThreads, sm, s>>>(a);
        break;
    case kModeVisitParent:
        expand_kernel<kModeVisitParent><<<blocks, kExpandThreads, sm, s>>>(a);
        break;
    case kModeSssp:
        expand_kernel<kModeSssp><<<blocks, kExpandThreads, sm, s>>>(a);
        break;
    case kModePagerank:
        expand_kernel<kModePagerank><<<blocks, kExpandThreads, sm, s>>>(a);
        break;
    default:
        expand_kernel<kModeDecode><<<blocks, kExpandThreads, sm, s>>>(a);
        break;
    }
    return cudaGetLastError();
}

cudaError_t launch_init(const InitArgs &a, cudaStream_t s)
{
    const uint64_t words = ((a.v1 + 31) >> 5) - (a.v0 >> 5);
    const unsigned blocks = (unsigned)std::max<uint64_t>(1, std::min<uint64_t>((words + 255) / 256, 4096));
    init_kernel<<<blocks, 256, 0, s>>>(a);
    return cudaGetLastError();
}

cudaError_t launch_compact(const CompactArgs &a, unsigned blocks, cudaStream_t s)
{
    compact_kernel<<<blocks, kFrontierThreads, 0, s>>>(a);
    return cudaGetLastError();
}

cudaError_t launch_xchg(const XchgArgs &a, cudaStream_t s)
{
    const uint64_t total = (uint64_t)(a.op == 1 ? 1 : a.world) * a.S;
    const unsigned blocks = (unsigned)std::max<uint64_t>(1, std::min<uint64_t>((total + 255) / 256, 148 * 8));
    xchg_kernel<<<blocks, 256, 0, s>>>(a);
    return cudaGetLastError();
}

cudaError_t launch_plan(const PlanArgs &a, unsigned blocks, cudaStream_t s)
{
    plan_kernel<<<blocks, kFrontierThreads, 0, s>>>(a);
    return cudaGetLastError();
}

}  // namespace efg
