// efg_kernels.cu — hand-written sm_100a kernels of the EFG BFS hot path.
//
// Steps and where they live:
//   a7 level end + a1 frontier materialisation/degree lookup + a2 exclusive scan
//      + a3 load-balanced partition  -> advance_kernel (one pass over the
//      visited bitmap; single-pass decoupled look-back scan; writes the sorted
//      next-frontier queue and the edge-tile table)
//   a4 locate compressed bit ranges + a5 EF element decode + a6 visit
//      -> expand_kernel (persistent, warp per edge tile)
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
constexpr int kWarps = kExpandThreads / 32;

// --------------------------------------------------------------------------
// warp / block primitives (§III-C: exclusive scan, bounded search)
// --------------------------------------------------------------------------
__device__ __forceinline__ uint32_t lane_id() { return threadIdx.x & 31; }

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

__device__ __forceinline__ void st_release_u64(uint64_t *p, uint64_t v)
{
    asm volatile("st.release.gpu.global.u64 [%0], %1;" ::"l"(p), "l"(v) : "memory");
}

__device__ __forceinline__ uint64_t ld_acquire_u64(const uint64_t *p)
{
    uint64_t v;
    asm volatile("ld.acquire.gpu.global.u64 %0, [%1];" : "=l"(v) : "l"(p) : "memory");
    return v;
}

constexpr uint64_t kFlagAgg = 1ull << 62;
constexpr uint64_t kFlagIncl = 2ull << 62;
constexpr uint64_t kValMask = (1ull << 62) - 1;

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

// Cross-block exclusive prefix for the advance scan (a2).  Every block
// publishes its aggregate pair (frontier count, work) as two 64-bit words
// flag | value (same flag in both, so no fence is needed: each value travels in
// the same single-copy-atomic word as its flag).  A block then sums the
// aggregates of ALL its predecessors directly, 32 lanes x several independent
// loads per step: latency is a couple of L2 round trips regardless of the block
// index, instead of a look-back chain that grows with the grid when every
// block is resident at once.
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

__device__ void prefix_of_block(const uint64_t *st, uint64_t b, uint64_t &ex_c, uint64_t &ex_w)
{
    const uint32_t lane = lane_id();
    uint64_t c_acc = 0, w_acc = 0;
    for (uint64_t base = 0; base < b; base += 32 * 4) {
        uint64_t c[4], w[4];
#pragma unroll
        for (int u = 0; u < 4; ++u) {
            const uint64_t idx = base + u * 32 + lane;
            c[u] = kFlagAgg;
            w[u] = kFlagAgg;
            if (idx < b) {
                c[u] = ld_relaxed_u64(st + 2 * idx);
                w[u] = ld_relaxed_u64(st + 2 * idx + 1);
            }
        }
#pragma unroll
        for (int u = 0; u < 4; ++u) {
            const uint64_t idx = base + u * 32 + lane;
            while (idx < b && ((c[u] >> 62) == 0 || (w[u] >> 62) == 0)) {
                c[u] = ld_relaxed_u64(st + 2 * idx);
                w[u] = ld_relaxed_u64(st + 2 * idx + 1);
            }
            c_acc += c[u] & kValMask;
            w_acc += w[u] & kValMask;
        }
    }
    ex_c = warp_sum_u64(c_acc);
    ex_w = warp_sum_u64(w_acc);
}

// --------------------------------------------------------------------------
// advance_kernel: a7 + a1 + a2 + a3
//   new = vis & ~prev per 32-vertex word; depth[new] = level; sorted queue of
//   the new frontier; per-vertex degree (a1) scanned (a2) into work offsets
//   W_v = sum over earlier frontier vertices of (kVertexWork + deg); tiles of
//   kTileWork units -> first owned chunk (a3: the Fig. 4 maxle rule applied
//   once per tile, with boundaries snapped to k-aligned chunk starts).
//   Vertex v occupies work [W_v, W_v + kVertexWork + deg_v); its chunk 0
//   starts at W_v, chunk c > 0 at W_v + kVertexWork + c*k.
//   Layout: a block covers kAdvanceWords bitmap words; thread t owns
//   kAdvanceRounds consecutive words (one 16-byte load per bitmap).  Degrees
//   come from the compact deg32 array: a word with many new bits loads its 32
//   degrees as eight 16-byte loads, a sparse word loads per bit.
// --------------------------------------------------------------------------
struct HubItem {
    uint64_t q, w, d;
};

__device__ __forceinline__ void write_tiles(TileEntry *tiles, uint64_t q, uint64_t W, uint64_t d,
                                            const ChunkLen &cl, uint64_t w_begin, uint64_t w_step)
{
    const uint64_t ch = cl.ch;
    const uint64_t T = kTileWork, A = kVertexWork;
    for (uint64_t t = (W + T - 1) / T + w_begin; t * T < W + A + d; t += w_step) {
        const uint64_t o = t * T - W;
        TileEntry te;
        if (o == 0) {
            te.fi = (uint32_t)q;
            te.chunk = 0;
            te.w = W;
        } else {
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
        }
        tiles[t] = te;
    }
}

// Tile entries for one frontier vertex; long lists are queued for the whole block.
__device__ __noinline__ void place_tiles(TileEntry *tiles, uint64_t q, uint64_t W, uint64_t d,
                                         const ChunkLen &cl, HubItem *hub, uint32_t *nhub, uint32_t cap)
{
    if (d >= 8ull * kTileWork) {
        const uint32_t slot = atomicAdd(nhub, 1u);
        if (slot < cap) {
            hub[slot] = HubItem{q, W, d};
            return;
        }
    }
    write_tiles(tiles, q, W, d, cl, 0, 1);
}

// exact warp sum of a value < 2^48 with two 32-bit REDUX instructions
__device__ __forceinline__ uint64_t warp_sum_small(uint64_t x)
{
    const uint32_t hi = __reduce_add_sync(FULL, (uint32_t)(x >> 16));
    const uint32_t lo = __reduce_add_sync(FULL, (uint32_t)(x & 0xffff));
    return ((uint64_t)hi << 16) + lo;
}

constexpr int kAdvGroup = 8;  // bitmap words whose degree loads are in flight together

// Pop up to kAdvGroup set bits (word indices) from a warp-uniform mask.
__device__ __forceinline__ int pop_words(uint32_t &mask, int (&j)[kAdvGroup])
{
    int n = 0;
#pragma unroll
    for (int u = 0; u < kAdvGroup; ++u) {
        j[u] = 0;
        if (mask) {
            j[u] = __ffs(mask) - 1;
            mask &= mask - 1;
            n = u + 1;
        }
    }
    return n;
}

__global__ void __launch_bounds__(kAdvanceThreads, 3) advance_kernel(AdvanceArgs a)
{
    constexpr int NW = kAdvanceThreads / 32;
    constexpr int R = kAdvanceRounds;
    constexpr int kHubCap = 256;
    __shared__ uint32_t s_wcnt[NW];
    __shared__ uint64_t s_wwork[NW];
    __shared__ uint64_t s_block_q, s_block_w;
    __shared__ HubItem s_hub[kHubCap];
    __shared__ uint32_t s_nhub;

    const uint32_t tid = threadIdx.x, lane = tid & 31, wid = tid >> 5;
    const uint64_t b = blockIdx.x;
    const ChunkLen cl = make_chunk(a.k, a.kshift);
    const uint64_t A = kVertexWork;
    const uint32_t lt = (1u << lane) - 1;
    // words of (warp, round r): rbase(r) + 0..31, lane j owns word rbase(r) + j
    const uint64_t wbase = b * (uint64_t)kAdvanceWords + (uint64_t)wid * 32 * R;

    if (tid == 0) s_nhub = 0;

    // ---- pass 1: new bits (a7), depth, per-word (count, work) via a1 ----
    uint32_t nb[R], wc[R];
    uint64_t ww[R];
#pragma unroll
    for (int r = 0; r < R; ++r) {
        const uint64_t rb = wbase + (uint64_t)r * 32;
        const uint32_t x = a.vis[rb + lane], p = a.prev[rb + lane];
        nb[r] = x & ~p;
        if (nb[r]) a.prev[rb + lane] = x;
        wc[r] = __popc(nb[r]);
        ww[r] = 0;
        uint32_t mask = __ballot_sync(FULL, nb[r] != 0);
        while (mask) {
            int j[kAdvGroup];
            pop_words(mask, j);
            uint32_t d[kAdvGroup], nbw[kAdvGroup];
#pragma unroll
            for (int u = 0; u < kAdvGroup; ++u) {
                nbw[u] = __shfl_sync(FULL, nb[r], j[u]);
                // lanes past the popped words see j = 0 duplicates: drop them
                if (u > 0 && j[u] == 0) nbw[u] = 0;
                d[u] = (nbw[u] >> lane & 1) ? __ldg(a.deg32 + (rb + j[u]) * 32 + lane) : 0;
            }
#pragma unroll
            for (int u = 0; u < kAdvGroup; ++u) {
                const bool bit = nbw[u] >> lane & 1;
                if (bit) a.depth[(rb + j[u]) * 32 + lane] = a.depth_value;
                const uint64_t s = warp_sum_small(bit ? A + d[u] : 0);
                if (nbw[u] && (int)lane == j[u]) ww[r] = s;
            }
        }
    }
    // warp totals -> block scan
    uint64_t tot_c = 0, tot_w = 0;
#pragma unroll
    for (int r = 0; r < R; ++r) {
        tot_c += __reduce_add_sync(FULL, wc[r]);
        tot_w += warp_sum_small(ww[r]);
    }
    if (lane == 0) {
        s_wcnt[wid] = (uint32_t)tot_c;
        s_wwork[wid] = tot_w;
    }
    __syncthreads();
    uint64_t pre_c = 0, pre_w = 0, blk_c = 0, blk_w = 0;
#pragma unroll
    for (int w = 0; w < NW; ++w) {
        if (w < (int)wid) {
            pre_c += s_wcnt[w];
            pre_w += s_wwork[w];
        }
        blk_c += s_wcnt[w];
        blk_w += s_wwork[w];
    }

    // ---- a2 across blocks ----
    uint64_t *st = a.status + (uint64_t)a.parity * 2 * a.nblocks;
    if (wid == 0) {
        if (lane == 0) {
            // clear this block's slots of the other parity for the next launch
            uint64_t *other = a.status + (uint64_t)(a.parity ^ 1) * 2 * a.nblocks;
            other[2 * b] = 0;
            other[2 * b + 1] = 0;
            st_relaxed_u64(st + 2 * b, kFlagAgg | blk_c);
            st_relaxed_u64(st + 2 * b + 1, kFlagAgg | blk_w);
        }
        uint64_t bq, bw;
        prefix_of_block(st, b, bq, bw);
        if (lane == 0) {
            s_block_q = bq;
            s_block_w = bw;
            if (b == a.nblocks - 1) {
                const uint64_t nf = bq + blk_c, nwork = bw + blk_w;
                a.ctrl->nf = nf;
                a.ctrl->nwork = nwork;
                a.ctrl->ne = nwork - A * nf;
                a.ctrl->ntiles = (nwork + kTileWork - 1) / kTileWork;
            }
        }
    }
    __syncthreads();

    // ---- pass 2: sorted queue (a7) + tile table (a3) ----
    uint64_t run_c = s_block_q + pre_c, run_w = s_block_w + pre_w;
#pragma unroll
    for (int r = 0; r < R; ++r) {
        const uint64_t rb = wbase + (uint64_t)r * 32;
        uint32_t tc;
        uint64_t tw;
        const uint64_t wq = run_c + warp_excl_u32(wc[r], tc);
        const uint64_t wwp = run_w + warp_excl_u64(ww[r], tw);
        run_c += tc;
        run_w += tw;
        uint32_t mask = __ballot_sync(FULL, nb[r] != 0);
        while (mask) {
            int j[kAdvGroup];
            pop_words(mask, j);
            uint32_t d[kAdvGroup], nbw[kAdvGroup];
#pragma unroll
            for (int u = 0; u < kAdvGroup; ++u) {
                nbw[u] = __shfl_sync(FULL, nb[r], j[u]);
                if (u > 0 && j[u] == 0) nbw[u] = 0;
                d[u] = (nbw[u] >> lane & 1) ? __ldg(a.deg32 + (rb + j[u]) * 32 + lane) : 0;
            }
#pragma unroll
            for (int u = 0; u < kAdvGroup; ++u) {
                const bool bit = nbw[u] >> lane & 1;
                const uint64_t q0 = __shfl_sync(FULL, wq, j[u]);
                const uint64_t w0 = __shfl_sync(FULL, wwp, j[u]);
                uint64_t dummy;
                const uint64_t wex = warp_excl_u64(bit ? A + d[u] : 0, dummy);
                if (bit) {
                    const uint64_t q = q0 + __popc(nbw[u] & lt);
                    const uint64_t W = w0 + wex;
                    a.queue[q] = (uint32_t)((rb + j[u]) * 32 + lane);
                    // does a tile boundary fall inside [W, W + A + d)?
                    if (((W + kTileWork - 1) & ~(uint64_t)(kTileWork - 1)) < W + A + d[u])
                        place_tiles(a.tiles, q, W, d[u], cl, s_hub, &s_nhub, kHubCap);
                }
            }
        }
    }
    __syncthreads();
    const uint32_t nhub = min(s_nhub, (uint32_t)kHubCap);
    for (uint32_t h = 0; h < nhub; ++h)
        write_tiles(a.tiles, s_hub[h].q, s_hub[h].w, s_hub[h].d, cl, tid, kAdvanceThreads);
}


// --------------------------------------------------------------------------
// expand_kernel: a4 + a5 + a6 (P:137-177 generalised, Alg. 1 lines 3-6)
//
// One warp per tile (persistent grid-stride over tiles).  A tile's work is a
// run of "chunks": k-aligned pieces of frontier lists, so every chunk
// starts right after a forward pointer and needs no select to find its first
// bit.  Chunks are taken 32 at a time ("batch"; many short lists per warp: the
// multi-list case).  The batch's upper-bit words are laid end to
// end and processed 32 words per step (one aligned 32-bit word per lane,
// coalesced; the next step's word is loaded before the current one is used):
//   popcount + warp exclusive scan  -> rank of each word's first stop bit
//                                      (the segmented scan of P:171-177: the
//                                      segments are chunks, whose element
//                                      prefix is subtracted)
//   per lane, serially over its word -> select1(i) - i by ffs-and-clear, the
//                                      lower bits from a bit buffer streamed
//                                      over the lower section, x = hi<<l | lo,
//                                      then the visits, kGroup probes in flight.
// --------------------------------------------------------------------------

constexpr int kGroup = 8;  // probes in flight per lane

struct SlotGeom {
    uint64_t A0, A1, U0;  // absolute bit range of the chunk's upper bits; upper start
    uint32_t wb, eb;      // exclusive word / element prefix within the batch
    uint64_t r0;          // rank of the chunk's first element in its list
};

struct SlotMeta {
    uint64_t lbase_l;  // absolute bit address of the lower section | l << 58
    int64_t rankoff;   // rank = rankoff + batch element index
    uint64_t aux;      // parent: source vertex; decode: output index base
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

template <int MODE>
__global__ void __launch_bounds__(kExpandThreads, 8) expand_kernel(ExpandArgs a)
{
    __shared__ SlotGeom s_geom[kWarps][32];
    __shared__ SlotMeta s_meta[kWarps][32];

    const uint32_t lane = lane_id(), wid = threadIdx.x >> 5;
    const uint64_t ntiles = a.ctrl->ntiles, nf = a.ctrl->nf, nwork = a.ctrl->nwork;
    const uint32_t *data32 = reinterpret_cast<const uint32_t *>(a.data);
    const ChunkLen cl = make_chunk(a.k, a.kshift);
    const uint64_t CH = cl.ch;
    const uint64_t A = kVertexWork;
    const uint64_t gw = (uint64_t)blockIdx.x * kWarps + wid;
    const uint64_t nwarps = (uint64_t)gridDim.x * kWarps;

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
                s_geom[wid][lane] = SlotGeom{A0, A1, U0, wb, ebt, r0};
                uint64_t aux = 0;
                if (MODE == kModeVisitParent) aux = v_j;
                if (MODE == kModeDecode) {
                    // CSR position of the chunk's first element: E_v + r0, E_v = W_v - A*q_v
                    const uint64_t qv = fi + (uint64_t)j;
                    aux = Wv_j - A * qv + r0 - ebt;
                }
                s_meta[wid][lane] = SlotMeta{lbase | ((uint64_t)l << kOffBits), (int64_t)r0 - (int64_t)ebt, aux};
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

            // ---- a5 + a6: 32 upper-bit words per step, one word per lane ----
            // Each lane decodes the elements whose stop bits lie in its word,
            // serially: select1(i) - i by ffs-and-clear, the lower bits from a
            // per-lane bit buffer streamed over the chunk's lower section, then
            // the visit.  Lanes start at ranks given by the warp scan of the
            // words' popcounts.
            uint32_t run = 0;
            WordLd nxt = load_word(data32, s_geom[wid], wb, lane, W);
            for (uint32_t g0 = 0; g0 < W; g0 += 32) {
                const WordLd cur = nxt;
                if (g0 + 32 < W) nxt = load_word(data32, s_geom[wid], wb, g0 + 32 + lane, W);
                uint32_t tot;
                const uint32_t ep = warp_excl_u32(__popc(cur.word), tot);
                if (cur.word) {
                    const SlotGeom &sg = s_geom[wid][cur.s];
                    const SlotMeta m = s_meta[wid][cur.s];
                    const uint64_t rank = sg.r0 + run + ep - sg.eb;         // rank of the first set bit
                    uint32_t hb = (uint32_t)(cur.wi * 32 - sg.U0 - rank);  // hi = hb + p - jj
                    const uint32_t ll = (uint32_t)(m.lbase_l >> kOffBits);
                    const uint32_t lmask = ll ? (0xffffffffu >> (32 - ll)) : 0u;
                    // lower-bit stream at bit lbase + rank*l (bit buffer `buf` holds nb bits)
                    const uint64_t lpos = (m.lbase_l & kOffMask) + rank * ll;
                    const uint32_t *lp = data32 + (lpos >> 5);
                    uint64_t buf = 0;
                    uint32_t nb = 64, pre = 0;
                    if (ll) {
                        const uint32_t sh = (uint32_t)(lpos & 31);
                        buf = (((uint64_t)ldg_u32(lp + 1) << 32) | ldg_u32(lp)) >> sh;
                        nb = 64 - sh;
                        pre = ldg_u32(lp + 2);
                        lp += 3;
                    }
                    uint64_t obase = m.aux + run + ep;  // decode: output index of the next element
                    uint32_t w = cur.word;
                    while (w) {
                        // decode up to kGroup elements, then resolve their probes together
                        uint32_t xs[kGroup];
                        uint32_t valid = 0;
#pragma unroll
                        for (int u = 0; u < kGroup; ++u) {
                            xs[u] = 0;
                            if (w) {
                                const uint32_t p = __ffs(w) - 1;
                                w &= w - 1;
                                const uint32_t hi = hb + p;  // select1(i) - i
                                hb -= 1;
                                uint32_t lo = 0;
                                if (ll) {
                                    if (nb < ll) {
                                        buf |= (uint64_t)pre << nb;
                                        nb += 32;
                                        pre = ldg_u32(lp++);
                                    }
                                    lo = (uint32_t)buf & lmask;
                                    buf >>= ll;
                                    nb -= ll;
                                }
                                xs[u] = (hi << ll) | lo;
                                valid |= 1u << u;
                            }
                        }
                        if (MODE == kModeDecode) {
#pragma unroll
                            for (int u = 0; u < kGroup; ++u)
                                if (valid >> u & 1) a.out[obase + u] = xs[u];
                            obase += __popc(valid);
                        } else {
                            uint32_t ws[kGroup];
#pragma unroll
                            for (int u = 0; u < kGroup; ++u)  // Alg. 1 line 3: probes in flight together
                                ws[u] = (valid >> u & 1) ? a.vis[xs[u] >> 5] : FULL;
#pragma unroll
                            for (int u = 0; u < kGroup; ++u) {
                                const uint32_t bit = 1u << (xs[u] & 31);
                                if (!(ws[u] & bit)) {  // stale reads are benign: the atomic decides
                                    if (MODE == kModeVisit) {
                                        atomicOr(a.vis + (xs[u] >> 5), bit);  // line 4
                                    } else {
                                        const uint32_t old = atomicOr(a.vis + (xs[u] >> 5), bit);
                                        if (!(old & bit)) a.out[xs[u]] = (uint32_t)m.aux;
                                    }
                                }
                            }
                        }
                    }
                }
                run += tot;
            }
        }
    }
}


__global__ void set_range_bits_kernel(uint32_t *vis, uint64_t v0, uint64_t v1)
{
    const uint64_t w0 = v0 >> 5, w1 = (v1 + 31) >> 5;
    for (uint64_t w = w0 + blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; w < w1;
         w += (uint64_t)gridDim.x * blockDim.x) {
        uint32_t m = FULL;
        if (w == (v0 >> 5)) m &= FULL << (v0 & 31);
        if (w == ((v1 - 1) >> 5) && (v1 & 31)) m &= (1u << (v1 & 31)) - 1;
        vis[w] |= m;
    }
}

__global__ void fill_u32_kernel(uint32_t *p, uint32_t val, uint64_t n)
{
    for (uint64_t i = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; i < n;
         i += (uint64_t)gridDim.x * blockDim.x)
        p[i] = val;
}

}  // namespace

int expand_occupancy(int mode)
{
    int nb = 0;
    switch (mode) {
    case kModeVisit:
        cudaOccupancyMaxActiveBlocksPerMultiprocessor(&nb, expand_kernel<kModeVisit>, kExpandThreads, 0);
        break;
    case kModeVisitParent:
        cudaOccupancyMaxActiveBlocksPerMultiprocessor(&nb, expand_kernel<kModeVisitParent>, kExpandThreads, 0);
        break;
    default:
        cudaOccupancyMaxActiveBlocksPerMultiprocessor(&nb, expand_kernel<kModeDecode>, kExpandThreads, 0);
        break;
    }
    return nb > 0 ? nb : 1;
}

cudaError_t launch_expand(int mode, const ExpandArgs &a, int blocks, cudaStream_t s)
{
    switch (mode) {
    case kModeVisit:
        expand_kernel<kModeVisit><<<blocks, kExpandThreads, 0, s>>>(a);
        break;
    case kModeVisitParent:
        expand_kernel<kModeVisitParent><<<blocks, kExpandThreads, 0, s>>>(a);
        break;
    default:
        expand_kernel<kModeDecode><<<blocks, kExpandThreads, 0, s>>>(a);
        break;
    }
    return cudaGetLastError();
}

cudaError_t launch_advance(const AdvanceArgs &a, cudaStream_t s)
{
    advance_kernel<<<(unsigned)a.nblocks, kAdvanceThreads, 0, s>>>(a);
    return cudaGetLastError();
}

cudaError_t launch_set_range_bits(uint32_t *vis, uint64_t v0, uint64_t v1, cudaStream_t s)
{
    if (v1 <= v0) return cudaSuccess;
    const uint64_t words = ((v1 + 31) >> 5) - (v0 >> 5);
    const unsigned blocks = (unsigned)std::min<uint64_t>((words + 255) / 256, 4096);
    set_range_bits_kernel<<<blocks, 256, 0, s>>>(vis, v0, v1);
    return cudaGetLastError();
}

cudaError_t launch_fill_u32(uint32_t *p, uint32_t val, uint64_t n, cudaStream_t s)
{
    if (!n) return cudaSuccess;
    const unsigned blocks = (unsigned)std::min<uint64_t>((n + 255) / 256, 148 * 16);
    fill_u32_kernel<<<blocks, 256, 0, s>>>(p, val, n);
    return cudaGetLastError();
}

}  // namespace efg
