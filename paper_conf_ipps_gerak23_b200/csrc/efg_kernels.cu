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
constexpr int kStage = 1024;  // max set bits in 32 words of 32 bits

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

// Warp-cooperative decoupled look-back: exclusive prefix of block b from the
// status words of its predecessors (each word: flag | value).
__device__ uint64_t lookback(const uint64_t *st, uint64_t b)
{
    const uint32_t lane = lane_id();
    uint64_t excl = 0;
    int64_t pred = (int64_t)b - 1;
    while (pred >= 0) {
        const int64_t idx = pred - (int64_t)lane;
        uint64_t s;
        for (;;) {
            s = idx >= 0 ? ld_acquire_u64(st + idx) : kFlagIncl;
            if (!__any_sync(FULL, (s >> 62) == 0)) break;
        }
        const uint32_t incl = __ballot_sync(FULL, (s >> 62) == 2);
        const int first = incl ? __ffs(incl) - 1 : 31;
        excl += warp_sum_u64((int)lane <= first ? (s & kValMask) : 0);
        if (incl) break;
        pred -= 32;
    }
    return excl;
}

// --------------------------------------------------------------------------
// advance_kernel: a7 + a1 + a2 + a3
//   new = vis & ~prev per 32-vertex word; depth[new] = level; sorted queue of
//   the new frontier; per-vertex degree (a1) scanned into edge offsets (a2);
//   edge tiles of kTileEdges -> first owned chunk (a3, Fig. 4 rule with
//   boundaries snapped to k-aligned chunk starts).
// --------------------------------------------------------------------------
struct HubItem {
    uint64_t q, e, d;
};

__device__ __forceinline__ void write_tiles(TileEntry *tiles, uint64_t q, uint64_t e, uint64_t d,
                                            uint64_t ch, uint64_t w_begin, uint64_t w_step)
{
    // tiles w with w*T in [e, e+d): first chunk start >= w*T
    const uint64_t T = kTileEdges;
    for (uint64_t w = (e + T - 1) / T + w_begin; w * T < e + d; w += w_step) {
        const uint64_t off = w * T - e;
        const uint64_t c = (off + ch - 1) / ch;
        TileEntry te;
        if (c * ch < d) {
            te.fi = (uint32_t)q;
            te.chunk = (uint32_t)c;
            te.e = e + c * ch;
        } else {
            te.fi = (uint32_t)(q + 1);
            te.chunk = 0;
            te.e = e + d;
        }
        tiles[w] = te;
    }
}

__global__ void __launch_bounds__(kAdvanceThreads) advance_kernel(AdvanceArgs a)
{
    constexpr int NW = kAdvanceThreads / 32;
    constexpr int kHubCap = 32;
    __shared__ uint32_t s_wcnt[NW];
    __shared__ uint64_t s_wedge[NW];
    __shared__ uint64_t s_block_q, s_block_e;
    __shared__ HubItem s_hub[kHubCap];
    __shared__ uint32_t s_nhub;

    const uint32_t tid = threadIdx.x, lane = tid & 31, wid = tid >> 5;
    const uint64_t b = blockIdx.x;
    const uint64_t wi = b * kAdvanceThreads + tid;
    const uint64_t ch = a.k ? a.k : (1ull << 40);

    if (tid == 0) s_nhub = 0;

    uint32_t x = 0, p = 0;
    if (wi < a.nwords) {
        x = a.vis[wi];
        p = a.prev[wi];
    }
    const uint32_t nb = x & ~p;
    if (nb) a.prev[wi] = x;

    // a1: degree lookup of the new frontier vertices (+ depth of the level)
    uint64_t edges = 0;
    for (uint32_t t = nb; t; t &= t - 1) {
        const uint64_t v = wi * 32 + (__ffs(t) - 1);
        edges += a.rec[v].deg;
        a.depth[v] = a.depth_value;
    }
    const uint32_t cnt = __popc(nb);

    // a2: block scan of (cnt, edges)
    uint32_t wtot_c;
    uint64_t wtot_e;
    const uint32_t ex_c = warp_excl_u32(cnt, wtot_c);
    const uint64_t ex_e = warp_excl_u64(edges, wtot_e);
    if (lane == 31) {
        s_wcnt[wid] = wtot_c;
        s_wedge[wid] = wtot_e;
    }
    __syncthreads();
    uint32_t pre_c = 0;
    uint64_t pre_e = 0, blk_c = 0, blk_e = 0;
#pragma unroll
    for (int w = 0; w < NW; ++w) {
        if (w < (int)wid) {
            pre_c += s_wcnt[w];
            pre_e += s_wedge[w];
        }
        blk_c += s_wcnt[w];
        blk_e += s_wedge[w];
    }

    // decoupled look-back across blocks (single pass)
    uint64_t *st_c = a.status + (uint64_t)(a.parity * 2 + 0) * a.nblocks;
    uint64_t *st_e = a.status + (uint64_t)(a.parity * 2 + 1) * a.nblocks;
    if (wid == 0) {
        if (lane == 0) {
            // clear this block's slots of the other parity for the next launch
            a.status[(uint64_t)((a.parity ^ 1) * 2 + 0) * a.nblocks + b] = 0;
            a.status[(uint64_t)((a.parity ^ 1) * 2 + 1) * a.nblocks + b] = 0;
            if (b == 0) {
                st_release_u64(st_c + b, kFlagIncl | blk_c);
                st_release_u64(st_e + b, kFlagIncl | blk_e);
            } else {
                st_release_u64(st_c + b, kFlagAgg | blk_c);
                st_release_u64(st_e + b, kFlagAgg | blk_e);
            }
        }
        uint64_t bq = 0, be = 0;
        if (b > 0) {
            bq = lookback(st_c, b);
            be = lookback(st_e, b);
            if (lane == 0) {
                st_release_u64(st_c + b, kFlagIncl | (bq + blk_c));
                st_release_u64(st_e + b, kFlagIncl | (be + blk_e));
            }
        }
        if (lane == 0) {
            s_block_q = bq;
            s_block_e = be;
            if (b == a.nblocks - 1) {
                const uint64_t nf = bq + blk_c, ne = be + blk_e;
                a.ctrl->nf = nf;
                a.ctrl->ne = ne;
                a.ctrl->ntiles = (ne + kTileEdges - 1) / kTileEdges;
            }
        }
    }
    __syncthreads();

    // a7 queue + a3 tile table
    uint64_t q = s_block_q + pre_c + ex_c;
    uint64_t e = s_block_e + pre_e + ex_e;
    for (uint32_t t = nb; t; t &= t - 1) {
        const uint64_t v = wi * 32 + (__ffs(t) - 1);
        const uint64_t d = a.rec[v].deg;
        a.queue[q] = (uint32_t)v;
        if (d) {
            bool done = false;
            if (d >= 64ull * kTileEdges) {  // hub: hand the tile writes to the whole block
                const uint32_t slot = atomicAdd(&s_nhub, 1u);
                if (slot < kHubCap) {
                    s_hub[slot] = HubItem{q, e, d};
                    done = true;
                }
            }
            if (!done) write_tiles(a.tiles, q, e, d, ch, 0, 1);
        }
        ++q;
        e += d;
    }
    __syncthreads();
    const uint32_t nhub = min(s_nhub, (uint32_t)kHubCap);
    for (uint32_t h = 0; h < nhub; ++h)
        write_tiles(a.tiles, s_hub[h].q, s_hub[h].e, s_hub[h].d, ch, tid, kAdvanceThreads);
}

// --------------------------------------------------------------------------
// expand_kernel: a4 + a5 + a6 (P:137-177 generalised, Alg. 1 lines 3-6)
//
// One warp per edge tile (persistent grid-stride over tiles).  A tile's work
// is a run of "chunks": k-aligned pieces of frontier lists, so every
// chunk starts at a forward pointer and needs no select to find its first bit.
// Chunks are taken 32 at a time ("batch"; several short lists per warp: the
// multi-list case).  The batch's upper-bit words are laid end to end
// and processed 32 words per step (one aligned 32-bit word per lane, coalesced):
//   popcount + warp exclusive scan  -> element slot of each word's first bit
//   set-bit enumeration (ffs)        -> select1(i) - i for every element
//                                       (staged in shared memory by rank)
//   balanced pass, one element per lane -> lower bits by a funnel shift of two
//                                       words, value = hi << l | lo, visit.
// --------------------------------------------------------------------------
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

template <int MODE>
__device__ __forceinline__ void visit(const ExpandArgs &a, uint32_t x, const SlotMeta &m,
                                      uint64_t ei)
{
    if (MODE == kModeDecode) {
        a.out[m.aux + ei] = x;
    } else {
        uint32_t *wp = a.vis + (x >> 5);
        const uint32_t bit = 1u << (x & 31);
        if (!(*wp & bit)) {  // Alg. 1 line 3 (stale reads are benign: the atomic decides)
            if (MODE == kModeVisit) {
                atomicOr(wp, bit);  // line 4; the advance pass finds the new bits
            } else {
                const uint32_t old = atomicOr(wp, bit);
                if (!(old & bit)) a.out[x] = (uint32_t)m.aux;
            }
        }
    }
}

template <int MODE>
__global__ void __launch_bounds__(kExpandThreads, 6) expand_kernel(ExpandArgs a)
{
    __shared__ uint32_t s_hi[kWarps][kStage];
    __shared__ uint8_t s_cs[kWarps][kStage];
    __shared__ SlotGeom s_geom[kWarps][32];
    __shared__ SlotMeta s_meta[kWarps][32];

    const uint32_t lane = lane_id(), wid = threadIdx.x >> 5;
    const uint64_t ntiles = a.ctrl->ntiles, nf = a.ctrl->nf, ne = a.ctrl->ne;
    const uint32_t *data32 = reinterpret_cast<const uint32_t *>(a.data);
    const uint64_t CH = a.k ? a.k : (1ull << 40);
    const uint64_t gw = (uint64_t)blockIdx.x * kWarps + wid;
    const uint64_t nwarps = (uint64_t)gridDim.x * kWarps;

    for (uint64_t tile = gw; tile < ntiles; tile += nwarps) {
        const TileEntry te = a.tiles[tile];
        uint64_t fi = te.fi, c0 = te.chunk, E = te.e;
        const uint64_t Eend = min((tile + 1) * (uint64_t)kTileEdges, ne);

        while (E < Eend && fi < nf) {
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
            const uint64_t nch = deg ? (deg + CH - 1) / CH : 0;
            const uint32_t nrem = (uint32_t)(nch > first ? nch - first : 0);
            const uint64_t erem = nrem ? deg - first * CH : 0;
            uint32_t totc;
            const uint32_t cb = warp_excl_u32(nrem, totc);
            uint64_t tote;
            const uint64_t eb = warp_excl_u64(erem, tote);
            if (totc == 0) {  // 32 empty lists
                fi += 32;
                c0 = 0;
                continue;
            }

            // ---- a3 (within tile): chunk slot t = lane -> owning vertex lane j ----
            const int j = warp_maxle_u32(cb, lane);
            const uint32_t deg_j = __shfl_sync(FULL, deg, j);
            const uint64_t offl_j = __shfl_sync(FULL, offl, j);
            const uint32_t ub_j = __shfl_sync(FULL, ubytes, j);
            const uint32_t cb_j = __shfl_sync(FULL, cb, j);
            const uint64_t eb_j = __shfl_sync(FULL, eb, j);
            const uint32_t v_j = __shfl_sync(FULL, v, j);
            const uint64_t nch_j = __shfl_sync(FULL, nch, j);
            const uint64_t cc = (j == 0 ? c0 : 0) + (lane - cb_j);
            const uint64_t r0 = cc * CH;
            const uint64_t chunk_e = E + eb_j + (uint64_t)(lane - cb_j) * CH;
            const bool valid = lane < totc && chunk_e < Eend;
            const uint32_t count = __popc(__ballot_sync(FULL, valid));
            if (count == 0) break;

            // ---- a4: bit ranges of the chunk (forward pointers) ----
            uint32_t nwd = 0, nel = 0;
            uint64_t A0 = 0, A1 = 0, U0 = 0, lbase = 0;
            uint32_t l = 0;
            if (valid) {
                const uint64_t off = offl_j & kOffMask;
                l = (uint32_t)(offl_j >> kOffBits);
                const uint64_t F = a.k ? deg_j / a.k : 0;
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
                if (MODE == kModeDecode) aux = chunk_e - ebt;
                s_meta[wid][lane] = SlotMeta{lbase | ((uint64_t)l << kOffBits), (int64_t)r0 - (int64_t)ebt, aux};
            }
            // state after this batch: continue after the last valid chunk
            {
                const int tl = (int)count - 1;
                const uint64_t last_cc = __shfl_sync(FULL, cc, tl);
                const uint64_t last_nch = __shfl_sync(FULL, nch_j, tl);
                const int last_j = __shfl_sync(FULL, j, tl);
                const uint64_t last_end = __shfl_sync(FULL, chunk_e, tl) + __shfl_sync(FULL, nel, tl);
                if (last_cc + 1 < last_nch) {
                    fi += last_j;
                    c0 = last_cc + 1;
                } else {
                    fi += last_j + 1;
                    c0 = 0;
                }
                E = last_end;
            }
            __syncwarp();

            // ---- a5 + a6: 32 upper-bit words per step ----
            uint32_t run = 0;
            for (uint32_t g0 = 0; g0 < W; g0 += 32) {
                const uint32_t g = g0 + lane;
                const int s = warp_maxle_u32(wb, g);
                uint32_t word = 0;
                uint64_t wi = 0;
                if (g < W) {
                    const SlotGeom &sg = s_geom[wid][s];
                    const uint64_t w0 = sg.A0 >> 5, wl = (sg.A1 - 1) >> 5;
                    wi = w0 + (g - sg.wb);
                    word = ldg_u32(data32 + wi);
                    if (wi == w0) word &= FULL << (uint32_t)(sg.A0 & 31);
                    if (wi == wl) {
                        const uint32_t hb = (uint32_t)(sg.A1 - wl * 32);  // 1..32 valid bits
                        if (hb < 32) word &= (1u << hb) - 1;
                    }
                }
                uint32_t tot;
                const uint32_t ep = warp_excl_u32(__popc(word), tot);
                if (word) {
                    const SlotGeom &sg = s_geom[wid][s];
                    const uint64_t rank = sg.r0 + run + ep - sg.eb;  // rank of the first set bit
                    const uint64_t hb = wi * 32 - sg.U0 - rank;      // hi = hb + p - jj
                    uint32_t w = word, jj = 0;
                    while (w) {
                        const uint32_t p = __ffs(w) - 1;
                        w &= w - 1;
                        s_hi[wid][ep + jj] = (uint32_t)(hb + p - jj);  // select1(i) - i
                        s_cs[wid][ep + jj] = (uint8_t)s;
                        ++jj;
                    }
                }
                __syncwarp();
                for (uint32_t e = lane; e < tot; e += 32) {
                    const uint32_t hi = s_hi[wid][e];
                    const SlotMeta m = s_meta[wid][s_cs[wid][e]];
                    const uint32_t ll = (uint32_t)(m.lbase_l >> kOffBits);
                    uint32_t lo = 0;
                    if (ll) {
                        const uint64_t rank = (uint64_t)(m.rankoff + (int64_t)(run + e));
                        const uint64_t ba = (m.lbase_l & kOffMask) + rank * ll;
                        const uint64_t bw = ba >> 5;
                        lo = __funnelshift_r(ldg_u32(data32 + bw), ldg_u32(data32 + bw + 1),
                                             (uint32_t)(ba & 31)) &
                             ((1u << ll) - 1);
                    }
                    visit<MODE>(a, (hi << ll) | lo, m, run + e);
                }
                __syncwarp();
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
