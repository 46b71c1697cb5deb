// efg_kernels.cu — hand-written sm_100a kernels of the EFG BFS hot path.
//
// Steps and where they live, per BFS level:
//   a4 locate compressed bit ranges + a5 EF element decode + a6 visit
//      -> expand_kernel (persistent, warp per work tile)
//   a7 level end: visited-bitmap diff -> sorted next frontier queue + depth,
//   fused with the next level's a1 degree lookup + a2 exclusive scan of
//   per-vertex work + a3 partition into tiles + a4 chunk descriptors
//      -> frontier_kernel (reduce-then-scan over the bitmap)
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
    // Kogge-Stone scan; the shuffle's in-range predicate guards the add (no compare)
    uint32_t inc = x;
#pragma unroll
    for (int d = 1; d < 32; d <<= 1)
        asm volatile("{\n\t.reg .u32 t;\n\t.reg .pred p;\n\t"
                     "shfl.sync.up.b32 t|p, %0, %1, 0, -1;\n\t"
                     "@p add.u32 %0, %0, t;\n\t}"
                     : "+r"(inc)
                     : "r"(d));
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

// position (0..31) of the set bit of rank kk (0-based, kk < popc(w)) of w:
// five popcount halvings (the in-word part of select1)
__device__ __forceinline__ uint32_t select_in_word(uint32_t w, uint32_t kk)
{
    uint32_t pos = 0;
#pragma unroll
    for (uint32_t sh = 16; sh; sh >>= 1) {
        const uint32_t c = __popc(w & ((1u << sh) - 1));
        const bool up = kk >= c;
        kk -= up ? c : 0u;
        w = up ? w >> sh : w;
        pos += up ? sh : 0u;
    }
    return pos;
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

// relaxed gpu-scope accesses (cross-block words of the persistent frontier grid)
__device__ __forceinline__ uint64_t ld_relaxed_u64(const uint64_t *p)
{
    uint64_t v;
    asm volatile("ld.relaxed.gpu.global.u64 %0, [%1];" : "=l"(v) : "l"(p) : "memory");
    return v;
}

__device__ __forceinline__ uint32_t ld_relaxed_u32(const uint32_t *p)
{
    uint32_t v;
    asm volatile("ld.relaxed.gpu.global.u32 %0, [%1];" : "=r"(v) : "l"(p) : "memory");
    return v;
}

__device__ __forceinline__ void st_relaxed_u64(uint64_t *p, uint64_t v)
{
    asm volatile("st.relaxed.gpu.global.u64 [%0], %1;" ::"l"(p), "l"(v) : "memory");
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
        a.ctrl->vmin2[0] = FULL;
        a.ctrl->vmin2[1] = FULL;
        a.ctrl->vpre_used = 0;
        a.ctrl->xchg_sparse = 0;
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
// Peer-memory exchange (SURVEY §8(e) "B200-native upgrade"): the same OR-reduce
// to owners + all-gather as pack / all-to-all / reduce / all-gather / unpack,
// with no collective library and no intermediate slices: owners read every
// rank's published new bits straight from its HBM over NVLink and store the
// OR into every rank's result buffer.  Five launches per level, in stream
// order on each rank (the barriers are one-block kernels, the data ops never
// spin):
//   op 0  publish:  pub[w] = vis[w] & ~prev[w]                 (local)
//                   + the non-zero words as a (word, bits) list while they
//                     number <= cap (warp-aggregated appends)
//   op 3  barrier e
//   op 1  every rank reads all ranks' list counts (same decision everywhere):
//         sparse (every count <= cap): vis[w] |= bits for the entries of the
//           OTHER ranks' lists (one pass, no owner step, traffic ~ discoveries)
//         dense: for owned words w: m = OR_p pub_p[w]; res_p[w] = m for all p
//   op 4  barrier e+1
//   op 2  dense: vis[w] |= res[w] (local); both: reset this rank's count
// Barrier e: block 0 stores e into flags[rank] of every rank (release, system
// scope), every block waits until all of its own flags reach e (acquire).
// Reuse is safe without more barriers: a rank republishes (op 0 of the next
// level) only after its barrier e+1, which every rank passes only after all
// ops 1 (the readers of pub) completed; owners write res (op 1 of the next
// level) only after barrier e+2, i.e. after every rank's op 2 read it.
// A wait longer than 4 s (a rank that never arrives) raises *fault and gives
// up instead of holding the device.
// --------------------------------------------------------------------------
__device__ __forceinline__ bool peer_barrier(const PeerArgs &a, uint32_t e)
{
    if (blockIdx.x == 0 && threadIdx.x < (unsigned)a.world) {
        __threadfence_system();
        uint32_t *f = a.peers[threadIdx.x] + a.rank;
        asm volatile("st.release.sys.global.u32 [%0], %1;" ::"l"(f), "r"(e) : "memory");
    }
    __shared__ int ok;
    if (threadIdx.x == 0) ok = 1;
    __syncthreads();
    if (threadIdx.x < (unsigned)a.world) {
        const uint32_t *f = a.local + threadIdx.x;
        const unsigned long long t0 = globaltimer();
        for (uint32_t it = 0;; ++it) {
            uint32_t cur;
            asm volatile("ld.acquire.sys.global.u32 %0, [%1];" : "=r"(cur) : "l"(f) : "memory");
            if ((int32_t)(cur - e) >= 0) break;
            __nanosleep(64);
            if ((it & 255) == 255 && globaltimer() - t0 > 4000000000ull) {
                atomicExch(a.fault, 1u);
                ok = 0;
                break;
            }
        }
    }
    __syncthreads();
    return ok != 0;
}

__global__ void peer_kernel(PeerArgs a)
{
    const uint64_t pub = kPeerFlagWords, res = kPeerFlagWords + peer_pad(a.nwords);
    const uint64_t sp = peer_sp_off(a.nwords), lst = sp + kPeerSpWords;
    const uint32_t cap = (uint32_t)peer_list_cap(a.nwords);
    const uint64_t stride = (uint64_t)gridDim.x * blockDim.x;
    const uint64_t t0 = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x;
    if (a.op == 0) {
        // whole warps iterate together (the list appends are warp-aggregated)
        const uint64_t tw = t0 & ~31ull;
        const uint32_t lane = threadIdx.x & 31;
        for (uint64_t w0 = tw; w0 < a.nwords; w0 += stride) {
            const uint64_t w = w0 + lane;
            const uint32_t m = w < a.nwords ? a.vis[w] & ~a.prev[w] : 0u;
            if (w < a.nwords) a.local[pub + w] = m;
            const uint32_t bal = __ballot_sync(FULL, m != 0);
            if (bal && __ldcg(a.local + sp) <= cap) {  // (past cap the level is dense: stop appending)
                uint32_t base = 0;
                if (lane == 0) base = atomicAdd(a.local + sp, (uint32_t)__popc(bal));
                base = __shfl_sync(FULL, base, 0) + __popc(bal & ((1u << lane) - 1));
                if (m && base < cap) {
                    a.local[lst + 2 * (uint64_t)base] = (uint32_t)w;
                    a.local[lst + 2 * (uint64_t)base + 1] = m;
                }
            }
        }
        // barrier epochs of this exchange: E - 1 (before op 1) and E (before
        // op 2), E = the counter after this increment (a device counter, so a
        // captured level loop advances it every iteration; every rank runs the
        // same number of exchanges, so the counters agree)
        if (blockIdx.x == 0 && threadIdx.x == 0) *a.epoch += 2;
        return;
    }
    if (a.op == 3 || a.op == 4) {  // the barrier alone, one block (op 3: epoch E - 1, op 4: E)
        const uint32_t E = *a.epoch;
        peer_barrier(a, a.op == 3 ? E - 1 : E);
        return;
    }
    if (a.op == 1) {
        // the decision: every rank sees the same published counts
        __shared__ uint32_t s_cnt[kPeerMaxWorld];
        __shared__ int s_sparse;
        if (threadIdx.x == 0) s_sparse = 1;
        __syncthreads();
        if (threadIdx.x < (unsigned)a.world) {
            s_cnt[threadIdx.x] = __ldcv(a.peers[threadIdx.x] + sp);
            if (s_cnt[threadIdx.x] > cap) s_sparse = 0;
        }
        __syncthreads();
        if (s_sparse) {
            if (blockIdx.x == 0 && threadIdx.x == 0) {
                a.local[sp + 1] = 1;
                *a.sparse_levels += 1;
            }
            for (int p = 0; p < a.world; ++p) {
                if (p == a.rank) continue;  // its own bits are in vis already
                const uint32_t *l = a.peers[p] + lst;
                for (uint64_t i = t0; i < s_cnt[p]; i += stride) {
                    const uint32_t w = __ldcv(l + 2 * i), m = __ldcv(l + 2 * i + 1);
                    atomicOr(a.vis + w, m);
                }
            }
            __threadfence_system();
            return;
        }
        if (blockIdx.x == 0 && threadIdx.x == 0) a.local[sp + 1] = 0;
        const uint64_t w0 = a.bounds[a.rank] / 32, w1 = (a.bounds[a.rank + 1] + 31) / 32;
        for (uint64_t w = w0 + t0; w < w1; w += stride) {
            uint32_t m = 0;
            for (int p = 0; p < a.world; ++p) m |= __ldcv(a.peers[p] + pub + w);
            for (int p = 0; p < a.world; ++p) __stcg(a.peers[p] + res + w, m);
        }
        __threadfence_system();
        return;
    }
    // op 2 (every peer has passed its op 1: the list and its count may be reused)
    const bool sparse = __ldcv(a.local + sp + 1) != 0;
    __syncthreads();
    if (blockIdx.x == 0 && threadIdx.x == 0) a.local[sp] = 0;
    if (sparse) return;
    for (uint64_t w = t0; w < a.nwords; w += stride) {
        const uint32_t m = __ldcv(a.local + res + w);
        if (m) a.vis[w] |= m;
    }
}

// --------------------------------------------------------------------------
// frontier_kernel: the level end (a7) fused with the next level's plan
// (a1 + a2 + a3 + a4), one launch per level.
//
//   a7  new = vis & ~prev: the new vertices, in increasing id order, become
//       the next frontier queue (sorted for free, in place of the paper's
//       partial radix sort); depth[new] = level;
//   a1  degree lookup (compact deg32 of each new vertex, then its 16-byte
//       record);
//   a2  exclusive scans of the per-vertex chunk count and work (kChunkWork
//       per k-aligned chunk + one unit per element);
//   a4  one ChunkDesc per k-aligned chunk;
//   a3  the tile table: tile t (work [tT, (t+1)T)) starts at the first chunk
//       whose work position is >= tT (the Fig. 4 maxle rule, once per tile).
//
// Persistent grid (every block resident: blocks wait on each other).  Phases:
//   0   (list skip on the level's own prefix, lskip = 2) each warp finds the
//       first vertex of its bitmap groups neither visited nor isolated, the
//       minimum is reduced over the grid, grid barrier;
//   1   a warp counts the new vertices of its bitmap word run, their work and
//       chunks (degree loads coalesced: lanes over the bits of a word);
//       the per-block aggregates are published, a grid barrier, then each
//       block sums its predecessors' (one warp per aggregate) and per-warp
//       sums place every warp;
//   2a  the warp writes its queue segment, depth, prev and, per queue entry,
//       the exclusive work and chunk prefixes (warp scans over the bits of
//       each word);
//   --  grid barrier;
//   2b  32-entry groups of the whole queue, grid-stride (balanced however the
//       new vertices cluster in id space): a list of one chunk writes its
//       descriptor and at most one tile boundary; longer lists are appended
//       to a BigList table;
//   --  grid barrier;
//   3   one BigList per warp: its descriptors and tile boundaries (lanes over
//       chunks / tiles), so hub lists are spread over the grid.
// The visited prefix (smallest vertex neither visited nor of degree 0) is
// reduced into ctrl->vmin2[level & 1], which the next expand reads; the
// other slot is reset for the following level end.
// --------------------------------------------------------------------------
// Grid-wide barrier of a persistent grid (every block resident): a 64-bit
// arrival counter that only grows (each barrier adds gridDim.x), release on
// arrival, acquire while polling with a short back-off.
// A barrier that has waited 4 s (a grid that is not co-resident, e.g. another
// kernel holding SMs forever) gives up and raises ctrl->fault, which the host
// reports as an error, instead of hanging the device.
__device__ __forceinline__ void grid_barrier(unsigned long long *count, uint32_t *fault)
{
    __syncthreads();
    if (threadIdx.x == 0) {
        __threadfence();
        unsigned long long old;
        asm volatile("atom.add.release.gpu.global.u64 %0, [%1], 1;" : "=l"(old) : "l"(count) : "memory");
        const unsigned long long target = (old / gridDim.x + 1) * gridDim.x;
        const unsigned long long t0 = globaltimer();
        for (uint32_t it = 0;; ++it) {
            unsigned long long cur;
            asm volatile("ld.acquire.gpu.global.u64 %0, [%1];" : "=l"(cur) : "l"(count) : "memory");
            if (cur >= target) break;
            __nanosleep(32);
            if ((it & 1023) == 1023 && globaltimer() - t0 > 4000000000ull) {
                atomicExch(fault, 1u);
                break;
            }
        }
        __threadfence();
    }
    __syncthreads();
}

// sums of the published per-block aggregates over blocks [0, b) and over all
// blocks (warp-wide; every lane gets both); 8 loads per lane in flight
__device__ __forceinline__ void sum_published(const uint64_t *agg, uint32_t b, uint64_t &pre, uint64_t &tot)
{
    uint64_t p = 0, t = 0;
    for (uint32_t i0 = 0; i0 < gridDim.x; i0 += 256) {
        uint64_t v[8];
#pragma unroll
        for (int u = 0; u < 8; ++u) {
            const uint32_t i = i0 + u * 32 + lane_id();
            v[u] = i < gridDim.x ? __ldcg(agg + i) : 0;
        }
#pragma unroll
        for (int u = 0; u < 8; ++u) {
            const uint32_t i = i0 + u * 32 + lane_id();
            t += v[u];
            p += i < b ? v[u] : 0;
        }
    }
    pre = warp_sum_u64(p);
    tot = warp_sum_u64(t);
}

// exclusive warp scans of N independent u32 values per lane, interleaved (N
// shuffle chains in flight instead of one)
template <int N>
__device__ __forceinline__ void warp_excl_u32_n(uint32_t (&x)[N], uint32_t (&total)[N])
{
    uint32_t inc[N];
#pragma unroll
    for (int i = 0; i < N; ++i) inc[i] = x[i];
#pragma unroll
    for (int d = 1; d < 32; d <<= 1) {
#pragma unroll
        for (int i = 0; i < N; ++i) {
            const uint32_t y = __shfl_up_sync(FULL, inc[i], d);
            if ((int)lane_id() >= d) inc[i] += y;
        }
    }
#pragma unroll
    for (int i = 0; i < N; ++i) {
        total[i] = __shfl_sync(FULL, inc[i], 31);
        x[i] = inc[i] - x[i];
    }
}

__global__ void __launch_bounds__(kFrontierThreads, 1024 / kFrontierThreads) frontier_kernel(FrontierArgs a)
{
    constexpr int NT = kFrontierThreads, NW = NT / 32;
    __shared__ uint64_t s_q[NW], s_wk[NW], s_ch[NW], s_sk[NW], s_bg[NW], s_all[NW];
    __shared__ uint64_t s_pre[5], s_tot[5];
    __shared__ uint32_t s_skw[NW][32];  // phase 1, sparse groups: skipped lists of each word

    const uint32_t tid = threadIdx.x, lane = tid & 31, wid = tid >> 5, b = blockIdx.x;
#define FTRACE(p)                                                      \
    do {                                                               \
        if (a.trace && tid == 0) a.trace[b * 8 + (p)] = globaltimer(); \
    } while (0)
    FTRACE(0);
    LevelCtrl *ctrl = a.ctrl;
    const uint32_t level = ctrl->level;
    int32_t *depth = ctrl->depth;
    if (b == 0 && tid == 0) {  // slots of the next level end
        ctrl->vmin2[(level & 1) ^ 1] = FULL;
    }
    const ChunkLen cl = make_chunk(a.k, a.kshift);
    const uint64_t CH = cl.ch, CW = kChunkWork;
    // warp gw owns the 32-word groups gw, gw + G, ... of the bitmap (round
    // robin: a dense id range, e.g. relabelled hubs, is spread over the grid);
    // its queue segment is contiguous, in group order
    const uint32_t G = gridDim.x * NW;
    const uint32_t gw = b * NW + wid;
    const uint64_t WG = 32ull * G;  // words between a warp's groups
    const uint32_t lt = (1u << lane) - 1;
#ifndef EFG_KB
#define EFG_KB 4
#endif
    constexpr int kB = EFG_KB;  // pass 1: non-empty words whose degree loads are in flight together
#ifndef EFG_P1_SPARSE
#define EFG_P1_SPARSE 4
#endif

    // ---- 1: count, work and chunks of the warp's new (owned) vertices ----
    // BFS list skip: a list whose largest neighbour is below the visited
    // prefix the last expand used (a lower bound of the next one) cannot
    // discover anything: it is neither planned nor expanded (its degree still
    // counts in the level's edges, reading C18)
    // lskip == 2: the level's own visited prefix (phase 0: the smallest vertex
    // neither visited nor isolated after this level's expand, reduced over the
    // grid before the counting) — at a discovery level's end the prefix jumps,
    // and the previous one would keep lists planned that cannot discover anything
    uint32_t vmin = FULL;  // smallest vertex of this warp's range that is neither visited nor isolated
    uint32_t vlow = 0;
    if (a.lskip == 2) {
        for (uint64_t w0 = 32ull * gw; w0 < a.nwords; w0 += WG) {  // the warp's first group with a zero
            const uint64_t w = w0 + lane;
            const uint32_t un = w < a.nwords ? ~(__ldcg(a.vis + w) | a.iso[w]) : 0u;
            const uint32_t zm = __ballot_sync(FULL, un != 0);
            if (zm) {
                const uint32_t cand = (uint32_t)(w * 32) + (un ? (uint32_t)__ffs(un) - 1 : 0u);
                vmin = __shfl_sync(FULL, cand, __ffs(zm) - 1);
                break;
            }
        }
        if (lane == 0 && vmin != FULL) atomicMin(&ctrl->vmin2[level & 1], vmin);
        grid_barrier(a.barrier, &ctrl->fault);
        vlow = __ldcg(&ctrl->vmin2[level & 1]);
        vmin = FULL;  // already reduced
    } else if (a.lskip) {
        vlow = ctrl->vpre_used;
    }
    const bool vmin_done = a.lskip == 2;
    uint32_t cq = 0, all = 0, ch = 0;  // lane partials
    uint64_t wk = 0, sk = 0;
    uint32_t bg = 0;  // lists planned grid-wide (phase 3)
    for (uint64_t w0 = 32ull * gw; w0 < a.nwords; w0 += WG) {
        const uint64_t w = w0 + lane;
        uint32_t nb = 0, nq = 0;
        if (w < a.nwords) {
            const uint32_t x = a.vis[w];
            nb = a.consume ? x : (x & ~a.prev[w]);
            if (!a.consume && !vmin_done && vmin == FULL) {
                const uint32_t un = ~(x | a.iso[w]);
                if (un) vmin = (uint32_t)(w * 32) + (__ffs(un) - 1);
            }
            nq = (w >= a.own_lo_w && w < a.own_hi_w) ? nb : 0u;
        }
        all += __popc(nb);
        cq += __popc(nq);
        // a1: degrees of the new vertices, lanes over the bits of each non-empty
        // word (one coalesced 128-byte load per word)
        uint32_t todo = __ballot_sync(FULL, nq != 0);
        const uint32_t gq = __reduce_add_sync(FULL, __popc(nq));
        if (kFrontierSparse && gq && EFG_P1_SPARSE * gq <= 32u * (uint32_t)__popc(todo)) {
            // sparsely filled words (<= 32 / EFG_P1_SPARSE new vertices per non-empty word): lanes
            // over the group's new vertices instead (32 per slot, kB slots of
            // loads in flight — a word per step would leave most lanes idle and
            // serialise one memory round trip per few vertices)
            uint32_t t_;
            const uint32_t gex = warp_excl_u32(__popc(nq), t_);
            if (vlow) s_skw[wid][lane] = 0;
            __syncwarp();
            for (uint32_t cursor = 0; cursor < gq; cursor += 32u * kB) {
                uint32_t dv[kB], uv[kB];
#pragma unroll
                for (int u = 0; u < kB; ++u) {
                    dv[u] = 0;
                    uv[u] = FULL;
                    const uint32_t t = cursor + 32u * u + lane;
                    if (cursor + 32u * u < gq) {  // warp-uniform
                        const int j = warp_maxle_u32(gex, t < gq ? t : 0u);
                        const uint32_t bits = __shfl_sync(FULL, nq, j);
                        const uint32_t r = t - __shfl_sync(FULL, gex, j);
                        if (t < gq) {
                            const uint32_t bit = select_in_word(bits, r);
                            const uint64_t v = (w0 + j) * 32 + bit;
                            dv[u] = __ldg(a.deg32 + v);
                            if (vlow) {
                                uv[u] = __ldg(a.umax + v);
                                if (uv[u] < vlow) atomicOr(&s_skw[wid][j], 1u << bit);
                            }
                        }
                    }
                }
#pragma unroll
                for (int u = 0; u < kB; ++u) {
                    const uint32_t d = dv[u];
                    if (uv[u] < vlow) {  // skipped list
                        sk += d;
                        continue;
                    }
                    const uint32_t nch = d ? (uint32_t)cl.div((uint64_t)d + CH - 1) : 0u;
                    wk += (uint64_t)nch * CW + d;
                    ch += nch;
                    bg += (nch > 1 || (uint64_t)nch * CW + d > kTileWork) ? 1u : 0u;
                }
            }
            if (vlow) {
                __syncwarp();
                if (nq) a.skipw[w] = s_skw[wid][lane];
                __syncwarp();
            }
            todo = 0;
        }
        while (todo) {
            uint32_t dv[kB], uv[kB], jv[kB];
#pragma unroll
            for (int u = 0; u < kB; ++u) {
                dv[u] = 0;
                uv[u] = FULL;
                jv[u] = 32;
                if (todo) {
                    const int j = __ffs(todo) - 1;
                    todo &= todo - 1;
                    jv[u] = j;
                    const uint32_t bits = __shfl_sync(FULL, nq, j);
                    if ((bits >> lane) & 1) {
                        dv[u] = __ldg(a.deg32 + (w0 + j) * 32 + lane);
                        if (vlow) uv[u] = __ldg(a.umax + (w0 + j) * 32 + lane);
                    }
                }
            }
#pragma unroll
            for (int u = 0; u < kB; ++u) {
                const uint32_t d = dv[u];
                if (vlow) {  // skipped lists of this word -> skipw (phase 2 drops them)
                    const uint32_t sm = __ballot_sync(FULL, uv[u] < vlow);
                    if (lane == 0 && jv[u] < 32) a.skipw[w0 + jv[u]] = sm;
                }
                if (uv[u] < vlow) {  // skipped list (vlow = 0: never)
                    sk += d;
                    continue;
                }
                const uint32_t nch = d ? (uint32_t)cl.div((uint64_t)d + CH - 1) : 0u;
                wk += (uint64_t)nch * CW + d;
                ch += nch;
                bg += (nch > 1 || (uint64_t)nch * CW + d > kTileWork) ? 1u : 0u;
            }
        }
    }
    const uint64_t cqw = warp_sum_u64(cq), allw = warp_sum_u64(all), chw = warp_sum_u64(ch);
    wk = warp_sum_u64(wk);
    sk = warp_sum_u64(sk);
    const uint64_t bgw = warp_sum_u64(bg);
#pragma unroll
    for (int d = 16; d; d >>= 1) vmin = min(vmin, __shfl_xor_sync(FULL, vmin, d));
    if (lane == 0) {
        s_q[wid] = cqw;
        s_all[wid] = allw;
        s_wk[wid] = wk;
        s_ch[wid] = chw;
        s_sk[wid] = sk;
        s_bg[wid] = bgw;
        if (vmin != FULL) atomicMin(&ctrl->vmin2[level & 1], vmin);
    }
    __syncthreads();
    FTRACE(1);
    // publish the block's aggregates (frontier vertices, work units, chunks,
    // skipped-list edges), barrier, then every block sums its predecessors'
    // (region r by warp r)
    if (wid < 5) {
        const uint64_t *src = wid == 0 ? s_q : (wid == 1 ? s_wk : (wid == 2 ? s_ch : (wid == 3 ? s_sk : s_bg)));
        const uint64_t agg = warp_sum_u64(lane < NW ? src[lane] : 0);
        if (lane == 0) st_relaxed_u64(a.status + wid * kMaxGrid + b, agg);
    } else if (wid == 5) {
        const uint64_t blk_all = warp_sum_u64(lane < NW ? s_all[lane] : 0);
        if (lane == 0 && blk_all) atomicAdd(reinterpret_cast<unsigned long long *>(&ctrl->nnew), blk_all);
    }
    grid_barrier(a.barrier, &ctrl->fault);
    if (wid < 5) {
        uint64_t pre, tot;
        sum_published(a.status + wid * kMaxGrid, b, pre, tot);
        if (lane == 0) {
            s_pre[wid] = pre;
            s_tot[wid] = tot;
        }
    }
    __syncthreads();
    const uint64_t nf = s_tot[0];
    // tile size of this level (a3): 2 x kTileWork on levels with plenty of work
    // (longer batches of short lists per warp), kTileWork otherwise (enough
    // tiles for every expand warp on small levels).  Lists of <= kTileWork
    // units cross at most one tile boundary either way (phase 2).
    const uint32_t TWs = (31 - __builtin_clz(kTileWork)) + (s_tot[1] >= kTileBigMinWork ? 1 : 0);
    const uint64_t TW = 1ull << TWs;  // a power of two: tile index = work position >> TWs
    if (b == gridDim.x - 1 && tid == 0) {  // level totals
        const uint64_t nwork = s_tot[1], nchunks = s_tot[2];
        const uint64_t ne = nwork - CW * nchunks + s_tot[3];  // every frontier list's edges
        const uint64_t ntiles = (nwork + TW - 1) >> TWs;
        ctrl->nf = nf;
        ctrl->nwork = nwork;
        ctrl->nchunks = nchunks;
        ctrl->ne = ne;
        ctrl->ntiles = ntiles;
        ctrl->xlevel = level;
        a.tiles[ntiles] = (uint32_t)nchunks;  // sentinel: end of the last tile
        if (nf) {
            ctrl->nlevels = level + 1;
            ctrl->total_nf += nf;
            ctrl->total_ne += ne;
            if (a.stats && level < a.max_stats) {
                a.stats[level].nf = nf;
                a.stats[level].ne = ne;
                a.stats[level].t0 = ~0ull;
                a.stats[level].t1 = 0;
            }
        }
        if (a.cond) {
            // loop while the next frontier is non-empty: this rank's owned part
            // (whole graph), or the global new set (partitioned: identical on
            // every rank after the exchange, so all ranks stop together); a
            // timed-out grid or peer barrier ends the loop (sticky fault)
            const uint64_t more = a.cond_global ? __ldcg(&ctrl->nnew) : nf;
            cudaGraphSetConditional(a.cond, (more && !__ldcg(&ctrl->fault)) ? 1u : 0u);
        }
    }
    FTRACE(2);
    uint64_t run = s_pre[1];
    uint32_t crun = (uint32_t)s_pre[2];  // chunks of a level < 2^32 (n + m/k)
    uint32_t brun = (uint32_t)s_pre[4];  // this warp's first BigList entry (no atomics)
    const uint32_t nbig = (uint32_t)s_tot[4];
    for (uint32_t w = 0; w < wid; ++w) {
        brun += (uint32_t)s_bg[w];
        run += s_wk[w];
        crun += (uint32_t)s_ch[w];
    }

    // ---- 2: depth, prev and the plan of the warp's new vertices, word by
    // word (lanes over bits): record loads (a1), work / chunk prefixes (a2),
    // descriptors (a4) and tile boundaries (a3) of single-chunk lists; longer
    // lists go to the BigList table (phase 3) ----
    const bool narrow = a.k == 0 || a.k >= 32;  // per-lane work < 2^27: 32-bit scans
#ifndef EFG_KS
#define EFG_KS 3
#endif
    constexpr int kS = EFG_KS;                    // slots (words, or 32-vertex groups) planned together
    for (uint64_t w0 = 32ull * gw; w0 < a.nwords; w0 += WG) {
        const uint64_t w = w0 + lane;
        uint32_t nb = 0, skw = 0;
        if (w < a.nwords) {
            // lists skipped in phase 1 are not planned (a word's mask is valid
            // wherever phase 1 saw owned new bits, i.e. wherever it is used)
            if (vlow) skw = a.skipw[w];
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
        const uint32_t nq = own ? nb & ~skw : 0u;
        uint32_t todo = __ballot_sync(FULL, nb != 0);
        // a slot = up to 32 new vertices, one per lane, in id order: the bits of
        // one non-empty word (dense groups: 32 consecutive records, coalesced),
        // or, when the group's non-empty words are sparsely filled, the next 32
        // new vertices of the whole group (compacted: a lane finds its word by
        // maxle over the words' popcount prefix, then its bit by select)
        const uint32_t gtot = __reduce_add_sync(FULL, __popc(nb));
        const bool sparse = kFrontierSparse && 4 * gtot <= 32u * (uint32_t)__popc(todo);
        uint32_t gex = 0;  // exclusive popcount prefix of the group's words (sparse slots only)
        if (sparse) {
            uint32_t t;
            gex = warp_excl_u32(__popc(nb), t);
        }
        uint32_t cursor = 0;
        while (sparse ? cursor < gtot : todo != 0) {
            uint32_t vv[kS], bq[kS], wl[kS], nc[kS];
            bool pl[kS];
            uint4 rv[kS];
#pragma unroll
            for (int u = 0; u < kS; ++u) {
                bool isnew = false;
                pl[u] = false;
                vv[u] = 0;
                rv[u] = make_uint4(0, 0, 0, 0);
                if (sparse) {
                    const uint32_t t = cursor + lane;
                    if (cursor < gtot) {
                        const int j = warp_maxle_u32(gex, t < gtot ? t : 0u);
                        const uint32_t bits = __shfl_sync(FULL, nb, j), qb = __shfl_sync(FULL, nq, j);
                        const uint32_t r = t - __shfl_sync(FULL, gex, j);
                        if (t < gtot) {
                            const uint32_t bit = select_in_word(bits, r);
                            vv[u] = (uint32_t)((w0 + j) * 32 + bit);
                            isnew = true;
                            pl[u] = (qb >> bit) & 1;
                        }
                        cursor += 32;
                    }
                } else if (todo) {
                    const int j = __ffs(todo) - 1;
                    todo &= todo - 1;
                    const uint32_t qb = __shfl_sync(FULL, nq, j), bb = __shfl_sync(FULL, nb, j);
                    vv[u] = (uint32_t)((w0 + j) * 32 + lane);
                    isnew = (bb >> lane) & 1;
                    pl[u] = (qb >> lane) & 1;
                }
                bq[u] = __ballot_sync(FULL, pl[u]);
                if (pl[u]) rv[u] = __ldg(reinterpret_cast<const uint4 *>(a.rec + vv[u]));
                if (isnew) {
                    if (a.depth_stored) a.depth_stored[vv[u]] = (int32_t)level;  // stored-id order
                    if (!a.depth_stored_only && depth) depth[vv[u]] = (int32_t)level;
                }
            }
            // per-list work nch*CW + d < 2^31.1 (deg < 2^26); the 32-lane sums fit
            // 32 bits when k >= 32 (< 2^27 per list), else the work is scanned
            // as (w >> 5, w & 31)
            uint32_t wlo[kS], wt[kS], wtlo[kS], ct[kS];
#pragma unroll
            for (int u = 0; u < kS; ++u) {
                const uint32_t d = rv[u].z;
                nc[u] = d ? (uint32_t)cl.div((uint64_t)d + CH - 1) : 0u;
                const uint32_t wv = nc[u] * (uint32_t)CW + d;
                wl[u] = narrow ? wv : wv >> 5;
                wlo[u] = narrow ? 0u : wv & 31;
            }
            warp_excl_u32_n<kS>(wl, wt);
            if (!narrow) warp_excl_u32_n<kS>(wlo, wtlo);
            uint32_t cex[kS];
            bool one = true;  // every list of these words is one chunk (or empty)
#pragma unroll
            for (int u = 0; u < kS; ++u) {
                one = one && nc[u] <= 1;
                cex[u] = nc[u];
            }
            if (__all_sync(FULL, one)) {
#pragma unroll
                for (int u = 0; u < kS; ++u) {
                    const uint32_t hm = __ballot_sync(FULL, nc[u] != 0);
                    ct[u] = __popc(hm);
                    cex[u] = __popc(hm & lt);
                }
            } else {
                warp_excl_u32_n<kS>(cex, ct);
            }
#pragma unroll
            for (int u = 0; u < kS; ++u) {
                if (!bq[u]) continue;  // warp-uniform
                const bool mine = pl[u];
                const uint32_t d = rv[u].z, ub = rv[u].w, nch = nc[u];
                const uint64_t off_l = ((uint64_t)rv[u].y << 32) | rv[u].x;
                const uint64_t W = run + (narrow ? (uint64_t)wl[u] : ((uint64_t)wl[u] << 5) + wlo[u]);
                const uint32_t C = crun + cex[u];
                const uint64_t wlen = (uint64_t)nch * CW + d;
                const bool big = mine && (nch > 1 || wlen > kTileWork);
                if (mine && !big) {
                    if (nch == 1) {  // a4: the list's only chunk (cc = 0)
                        *reinterpret_cast<uint4 *>(a.chunks + C) = make_uint4(rv[u].x, rv[u].y, d, ub);
                        if (a.cvtx) a.cvtx[C] = vv[u];
                    }
                    // a3: a tile boundary t*T inside [W, W + wlen) starts at this chunk or the next
                    const uint64_t t = (W + TW - 1) >> TWs;
                    if (t * TW < W + wlen) a.tiles[t] = C + (t * TW > W ? 1u : 0u);
                }
                const uint32_t bm = __ballot_sync(FULL, big);
                if (bm) {
                    const uint32_t base = brun;
                    brun += __popc(bm);
                    if (big) {
                        BigList bl;
                        bl.W = W;
                        bl.cstart = C;
                        bl.off_l = off_l;
                        bl.deg = d;
                        bl.ubytes = ub;
                        bl.v = vv[u];
                        bl.nch = nch;
                        a.big[base + __popc(bm & lt)] = bl;
                    }
                }
                run += narrow ? (uint64_t)wt[u] : ((uint64_t)wt[u] << 5) + wtlo[u];
                crun += ct[u];
            }
        }
    }
    FTRACE(5);
    if (nbig == 0) return;  // grid-uniform: no long list this level
    grid_barrier(a.barrier, &ctrl->fault);
    FTRACE(6);

    // ---- 3: the long lists, one per lane (lists of > 8 chunks or tiles: one
    // per warp, lanes over chunks / tiles): descriptors and the tile
    // boundaries of the list's window (Fig. 4 rule) ----
    const bool udiv = a.k && CW + CH < (1ull << 31);  // 32-bit chunk division (rel < 2^31.1 - CW - CH)
    const uint32_t CWH = (uint32_t)(CW + CH);
    auto tile_chunk = [&](uint32_t rel, uint32_t nch) -> uint32_t {
        // chunk c of a list starts at W + c*(CW + k): first chunk at or after W + rel
        uint32_t c = rel ? 1u : 0u;
        if (udiv && nch > 1) c = min((rel + CWH - 1) / CWH, nch);
        return c;
    };
    // entry e = gw + G*(lane + 32*i): consecutive entries (neighbouring ids,
    // i.e. similar degrees: the relabelled hubs come together) go to
    // different warps
    for (uint64_t e0 = gw; e0 < nbig; e0 += 32ull * G) {
        const uint64_t e = e0 + (uint64_t)lane * G;
        uint64_t W = 0, cs = 0, off_l = 0;
        uint32_t d = 0, ub = 0, v = 0, nch = 0;
        if (e < nbig) {
            const BigList *bp = a.big + e;
            W = __ldcg(&bp->W);
            cs = __ldcg(&bp->cstart);
            off_l = __ldcg(&bp->off_l);
            d = __ldcg(&bp->deg);
            ub = __ldcg(&bp->ubytes);
            v = __ldcg(&bp->v);
            nch = __ldcg(&bp->nch);
        }
        const uint64_t wl = (uint64_t)nch * CW + d;
        const uint64_t t_lo = (W + TW - 1) >> TWs, t_hi = (W + wl + TW - 1) >> TWs;
        const bool huge = nch > 8 || t_hi - t_lo > 8;
        if (!huge) {
            for (uint32_t j = 0; j < nch; ++j) {
                const uint64_t oc = off_l | ((uint64_t)j << kCcShift);
                *reinterpret_cast<uint4 *>(a.chunks + cs + j) = make_uint4((uint32_t)oc, (uint32_t)(oc >> 32), d, ub);
                if (a.cvtx) a.cvtx[cs + j] = v;
            }
            for (uint64_t t = t_lo; t < t_hi; ++t)
                a.tiles[t] = (uint32_t)(cs + tile_chunk((uint32_t)(t * TW - W), nch));
        }
        uint32_t hm = __ballot_sync(FULL, huge);
        while (hm) {
            const int o = __ffs(hm) - 1;
            hm &= hm - 1;
            const uint64_t oW = __shfl_sync(FULL, W, o), ocs = __shfl_sync(FULL, cs, o);
            const uint64_t ooff = __shfl_sync(FULL, off_l, o);
            const uint32_t od = __shfl_sync(FULL, d, o), oub = __shfl_sync(FULL, ub, o);
            const uint32_t ov = __shfl_sync(FULL, v, o), onch = __shfl_sync(FULL, nch, o);
            for (uint32_t j = lane; j < onch; j += 32) {
                const uint64_t oc = ooff | ((uint64_t)j << kCcShift);
                *reinterpret_cast<uint4 *>(a.chunks + ocs + j) = make_uint4((uint32_t)oc, (uint32_t)(oc >> 32), od, oub);
                if (a.cvtx) a.cvtx[ocs + j] = ov;
            }
            const uint64_t owl = (uint64_t)onch * CW + od;
            const uint64_t ot_lo = (oW + TW - 1) >> TWs, ot_hi = (oW + owl + TW - 1) >> TWs;
            for (uint64_t t = ot_lo + lane; t < ot_hi; t += 32)
                a.tiles[t] = (uint32_t)(ocs + tile_chunk((uint32_t)(t * TW - oW), onch));
        }
    }
    FTRACE(7);
#undef FTRACE
}

// --------------------------------------------------------------------------
// expand_kernel: a4 + a5 + a6 (P:137-177 generalised, Alg. 1 lines 3-6)
//
// Persistent: one CTA of kExpandWarps warps per SM; a warp takes tiles
// gw, gw + #warps, ...  A tile's chunks (frontier_kernel descriptors) are cut into
// batches of <= 32 chunks whose compressed bytes fit one staging buffer.  Per
// batch the warp
//   (producer)  a4: locates each chunk's bits from the forward pointers
//               (Fig. 6: a chunk starts right after pointer cc-1, so
//               no select is needed) and stages the lower fields and upper
//               words into shared memory with TMA bulk copies (cp.async.bulk,
//               completion on a per-buffer mbarrier), one batch ahead of the
//               decoder (double buffering); BFS chunk skip: a chunk whose
//               last element (high part = its forward pointer) is below
//               the visited prefix becomes an empty slot, nothing staged;
//   (rounds)    lays the batch's upper-bit words end to end (kRoundWords per
//               round), masks each chunk's first/last word and keeps the
//               non-zero words as 16-byte records {word, hi base, lower-field
//               base, l | slot} (bases relative to the record's first stop bit)
//               with the kept-element prefix of each (the segmented scan of
//               P:171-177, segments = chunks); BFS prefix skip: a word whose
//               ids are all below the visited prefix vpre gets no record;
//   (decode)    a5: splits the round's kept elements evenly over the lanes; a
//               lane finds select1 of its first element once (maxle over the
//               record prefix, Fig. 4 rule, then an in-word select) and walks
//               its run serially: the next set bit (bfind on the reversed word)
//               gives select1(i) - i, the lower field is a funnel shift of two
//               shared-memory words, x = hi << l | lo; an exhausted word is
//               refilled from the next record without a branch (every record
//               has a set bit);
//   (visit)     a6: kU elements per lane in flight: ids below vpre are known
//               visited (register compare), the others probe the global bitmap
//               and atomicOr decides (stale reads are benign, C16); SSSP relax,
//               PageRank push / pull and decode use the same walk.
// --------------------------------------------------------------------------
struct SlotP {        // one chunk of the batch being decoded (shared memory)
    uint32_t lsmb;    // shared-window bit address of element e's lower field = lsmb + e*l (mod 2^32)
    uint32_t lflags;  // l | (A0 & 31) << 8 | ((A1 - 1) & 31) << 16 | staged-upper << 24
    uint32_t HB;      // hi = 32*g + p - e + HB  (g batch word, p bit in word, e batch element)
    uint32_t eb;      // first batch element of the chunk
    uint32_t wb;      // first batch word of the chunk
    uint32_t nwd;     // upper-bit words of the chunk
    uint64_t usrc;    // staged: stage-area word index of batch word wb; else global word index
    uint64_t aux;     // parent: v; decode / SSSP: CSR position of the chunk's first element; PR: share bits
    float aux2;       // SSSP: dist of the chunk's source vertex
    uint32_t pad;
};
static_assert(sizeof(SlotP) == 48, "SlotP");

struct WarpSmem {
    uint32_t stage[2][kStageBytes / 4];   // TMA staging buffers (16-byte aligned)
    uint4 wrec[kRoundWords];              // non-zero words of the round: {word, 32g + HB, lsmb, l | slot << 8}
    uint32_t wpre[kRoundWords];           // batch element index of each record's first stop bit
    SlotP slot[32];
    uint64_t mbar[2];
};

constexpr size_t kExpandSmem = (size_t)kHotWords * 4 + (size_t)kExpandWarps * sizeof(WarpSmem);
static_assert(kExpandSmem <= 232448, "expand kernel shared memory exceeds 227 KB");
static_assert(sizeof(WarpSmem) % 16 == 0, "WarpSmem alignment");

__device__ __forceinline__ uint32_t smem_u32(const void *p)
{
    return static_cast<uint32_t>(__cvta_generic_to_shared(p));
}

__device__ __forceinline__ void mbar_init(uint64_t *bar, uint32_t count)
{
    asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(smem_u32(bar)), "r"(count) : "memory");
}

__device__ __forceinline__ void mbar_arrive_expect_tx(uint64_t *bar, uint32_t bytes)
{
    asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(smem_u32(bar)), "r"(bytes)
                 : "memory");
}

__device__ __forceinline__ void mbar_wait(uint64_t *bar, uint32_t parity)
{
    const uint32_t addr = smem_u32(bar);
    uint32_t done = 0;
    while (!done) {
        asm volatile(
            "{\n\t.reg .pred p;\n\t"
            "mbarrier.try_wait.parity.shared::cta.b64 p, [%1], %2;\n\t"
            "selp.u32 %0, 1, 0, p;\n\t}"
            : "=r"(done)
            : "r"(addr), "r"(parity)
            : "memory");
    }
}

__device__ __forceinline__ uint32_t lds_u32(uint32_t addr)
{
    uint32_t v;
    asm volatile("ld.shared.u32 %0, [%1];" : "=r"(v) : "r"(addr));
    return v;
}

// leading zeros of a non-zero word in one instruction (bfind.shiftamt)
__device__ __forceinline__ uint32_t clz_nz(uint32_t x)
{
    uint32_t d;
    asm("bfind.shiftamt.u32 %0, %1;" : "=r"(d) : "r"(x));
    return d;
}

// funnel shift right with the shift amount taken mod 32 (no masking instruction)
__device__ __forceinline__ uint32_t shf_r_wrap(uint32_t lo, uint32_t hi, uint32_t sh)
{
    uint32_t d;
    asm("shf.r.wrap.b32 %0, %1, %2, %3;" : "=r"(d) : "r"(lo), "r"(hi), "r"(sh));
    return d;
}

// TMA bulk copy global -> shared (16-byte aligned addresses, size a multiple of 16)
__device__ __forceinline__ void bulk_g2s(void *dst, const void *src, uint32_t bytes, uint64_t *bar)
{
    asm volatile("cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];"
                 ::"r"(smem_u32(dst)), "l"(src), "r"(bytes), "r"(smem_u32(bar))
                 : "memory");
}

__device__ __forceinline__ void fence_proxy_async()
{
    asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
}

// Producer output of one batch: per lane = per chunk slot (registers), plus
// the batch totals (warp-uniform).
struct Batch {
    uint32_t cnt, ne, nw, buf;   // chunks, elements, upper words, staging buffer
    uint32_t lsmb, lflags, HB, eb, wb, nwd, v, cc;
    uint32_t nel;                // elements of this lane's chunk
    bool lpc;                    // warp-uniform: decode lane-per-chunk (see expand_kernel)
    uint64_t usrc;
};

// largest power of two below kRoundWords: the maxle search over a round's records
constexpr uint32_t kSearchStep = kRoundWords <= 1 ? 0u : (1u << (31 - __builtin_clz(kRoundWords - 1)));

constexpr bool kUseHot = kHotWords > 4;  // shared-memory visited snapshot compiled in

#ifndef EFG_KU
#define EFG_KU 4
#endif
constexpr int kU = EFG_KU;  // elements per lane whose probes are in flight together
#ifndef EFG_CHUNK_SKIP
#define EFG_CHUNK_SKIP 1
#endif
constexpr bool kChunkSkip = EFG_CHUNK_SKIP;  // BFS: k-chunks wholly below the visited prefix are not staged
#ifndef EFG_LPC
#define EFG_LPC 1
#endif
constexpr bool kLpc = EFG_LPC;  // lane-per-chunk decode of balanced batches (no word records)
#ifndef EFG_SPAN_STAGE
#define EFG_SPAN_STAGE 1
#endif
constexpr bool kSpanStage = EFG_SPAN_STAGE;  // one bulk copy per batch when the chunks' bytes are adjacent
#ifndef EFG_FAST_SINGLE
#define EFG_FAST_SINGLE 1
#endif
constexpr bool kFastSingle = EFG_FAST_SINGLE;  // producer fast path for batches of whole short lists
#ifndef EFG_LPC_BITSKIP
#define EFG_LPC_BITSKIP 1
#endif
constexpr bool kLpcBitSkip = EFG_LPC_BITSKIP;  // lane-per-chunk: skip the below-vpre stop bits of the first kept word
constexpr uint64_t kMaxSuperTile = 16;           // tiles per super-tile at most (work assignment)

template <int MODE>
__global__ void __launch_bounds__(kExpandThreads, 1) expand_kernel(ExpandArgs a)
{
    extern __shared__ __align__(128) uint8_t smem_raw[];
    WarpSmem *ws_all = reinterpret_cast<WarpSmem *>(smem_raw);
    uint32_t *s_hot = reinterpret_cast<uint32_t *>(smem_raw + (size_t)kExpandWarps * sizeof(WarpSmem));

    const uint32_t lane = lane_id(), wid = threadIdx.x >> 5;
    WarpSmem &ws = ws_all[wid];
    const uint64_t ntiles = a.ctrl->ntiles;
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
    if (lane == 0) {
        mbar_init(&ws.mbar[0], 1);
        mbar_init(&ws.mbar[1], 1);
    }
    if (kBfs && kUseHot) {
        // level-start snapshot of the hot visited words
        const uint4 *src = reinterpret_cast<const uint4 *>(a.vis);
        uint4 *dst = reinterpret_cast<uint4 *>(s_hot);
        for (uint32_t i = threadIdx.x; i < a.hot_words / 4; i += blockDim.x) dst[i] = src[i];
    }
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
    __syncthreads();

    const uint8_t *data = a.data;
    const uint32_t *data32 = reinterpret_cast<const uint32_t *>(a.data);
    const uint32_t *st32 = &ws.stage[0][0];
    const uint32_t sbits = smem_u32(st32) * 8;  // shared-window bit address of the staging area
    const uint32_t vpre = kBfs ? a.ctrl->vmin2[xl & 1] : 0u;  // ids below it are visited (or never probed)
    const bool pskip = kBfs && a.pskip && vpre != 0;              // warp-uniform
    // lane-per-chunk threshold (busy element slots >= 2/lpcf of 32 x the longest
    // chunk): halved on skip levels (visited prefix past n/3: most elements are
    // stepped over word by word, so a lane's chunk costs little whatever its
    // length, while a record round is paid in full)
    const uint32_t lpcf = (pskip && (a.variant & 64) && vpre >= a.lpc_skip_vpre) ? 4u : 2u;
    if (blockIdx.x == 0 && threadIdx.x == 0) a.ctrl->vpre_used = pskip ? vpre : 0u;
    const uint64_t gw = (uint64_t)blockIdx.x * kExpandWarps + wid;
    const uint64_t nwarps = (uint64_t)gridDim.x * kExpandWarps;
    const uint64_t CH = a.k ? a.k : (1ull << 40);
    const bool kpow2 = a.k && !(a.k & (a.k - 1));
    const uint32_t kshift = kpow2 ? (uint32_t)__ffs(a.k) - 1 : 0u;

    // producer cursor: chunks [cnext, cend) of the current tile
    // work assignment: super-tiles of ST consecutive tiles dealt round robin to
    // the warps; a warp's batches run across the tile boundaries inside a
    // super-tile (fewer part-filled batches), and round robin keeps regions
    // of the id space spread over the grid.  ST grows with the level's tile
    // count (>= 4 super-tiles per warp) up to kMaxSuperTile.
    uint64_t ST = 1;
    if (a.variant & 16) {
        ST = ntiles / (4 * nwarps);
        ST = ST < 1 ? 1 : (ST > kMaxSuperTile ? kMaxSuperTile : ST);
    }
    const uint64_t nst = (ntiles + ST - 1) / ST;
    uint64_t tile = gw;  // super-tile index
    uint64_t cnext = 0, cend = 0;
    if (tile < nst) {
        cnext = a.tiles[tile * ST];
        cend = a.tiles[tile * ST + ST < ntiles ? tile * ST + ST : ntiles];
    }
    uint32_t phase = 0;  // bit b: parity of the next wait on buffer b
    uint32_t nbuf = 0;   // buffer of the next produced batch

    // ---- producer: descriptors -> chunk bit ranges (a4) -> staged bytes ----
    auto produce = [&](Batch &B) -> bool {
        while (cnext >= cend) {
            tile += nwarps;
            if (tile >= nst) return false;
            cnext = a.tiles[tile * ST];
            cend = a.tiles[tile * ST + ST < ntiles ? tile * ST + ST : ntiles];
        }
        const uint64_t c = cnext + lane;
        const bool valid = c < cend;
        uint4 d0 = make_uint4(0, 0, 0, 0);
        if (valid) d0 = *reinterpret_cast<const uint4 *>(a.chunks + c);
        // fast path: every chunk of the batch is a whole short list (deg < k:
        // no forward pointers, cc = 0, bytes [lower][upper] contiguous)
        // with a stageable upper section — the common case on the levels that
        // expand millions of small lists.  One span copy stages them all.
        // (a list whose bytes + alignment slack exceed a buffer takes the general path)
        const uint32_t lsec = ((d0.z * ((d0.y >> (kOffBits - 32)) & 63)) + 7) >> 3;
        if (kFastSingle && (a.variant & 2) &&
            __all_sync(FULL, !valid || ((uint64_t)d0.z < CH && d0.w <= kUpperStageMax &&
                                        lsec + d0.w + 40 <= kStageBytes))) {
            const uint64_t off = (((uint64_t)d0.y << 32) | d0.x) & kOffMask;
            const uint32_t l = (d0.y >> (kOffBits - 32)) & 63, deg = d0.z, ub = d0.w;
            const uint64_t U0b = off + ((deg * l + 7) >> 3);  // byte address of the upper section
            const uint64_t rs = off & ~15ull;                  // staged range: the whole list + 8 B
            const uint64_t re = (U0b + ub + 8 + 15) & ~15ull;  // (two-word lower windows), 16-B aligned
            const uint64_t S = __shfl_sync(FULL, rs, 0);       // lane 0 is valid (cnext < cend)
            uint32_t E = valid ? ((rs >= S && re - S < (1ull << 30)) ? (uint32_t)(re - S) : (1u << 30)) : 0u;
#pragma unroll
            for (int d = 1; d < 32; d <<= 1) {
                const uint32_t t = __shfl_up_sync(FULL, E, d);
                if ((int)lane >= d) E = max(E, t);
            }
            const bool fits = valid && E <= kStageBytes;
            const uint32_t cnt = __popc(__ballot_sync(FULL, fits));
            // sparse frontiers leave gaps between the lists: when packing the
            // lists one after the other would fit more of them, take the
            // general path (which then stages them per chunk)
            uint32_t tsum;
            const uint32_t ssum = warp_excl_u32(valid ? (uint32_t)(re - rs) : 0u, tsum);
            const uint32_t cnt_sum = __popc(__ballot_sync(FULL, valid && ssum + (uint32_t)(re - rs) <= kStageBytes));
            if (cnt >= cnt_sum) {
                B.cnt = cnt;
                const uint32_t buf = nbuf;
                B.buf = buf;
                nbuf ^= 1;
                const uint64_t A0 = U0b * 8, A1 = A0 + 8ull * ub;
                const uint32_t nel = fits ? deg : 0u;
                const uint32_t nwd = fits ? (uint32_t)(((A1 - 1) >> 5) - (A0 >> 5) + 1) : 0u;
                uint32_t t;  // < 2^15 elements (32 lists of < 512), < 2^16 words (32 x <= 241)
                const uint32_t ex = warp_excl_u32(nel | nwd << 16, t);
                B.eb = ex & 0xffffu;
                B.wb = ex >> 16;
                B.ne = t & 0xffffu;
                B.nw = t >> 16;
                B.nwd = nwd;
                B.nel = nel;
                B.cc = 0;
                B.v = (MODE != kModeVisit && valid) ? a.cvtx[c] : 0u;
                B.lpc = kLpc && (a.variant & 1) && lpcf * B.ne >= 32 * __reduce_max_sync(FULL, nel);
                const uint32_t sbase = buf * kStageBytes;
                B.lsmb = sbits + 8 * (sbase + (uint32_t)(off - S)) - B.eb * l;
                B.lflags = l | ((uint32_t)(A0 & 31) << 8) | ((uint32_t)((A1 - 1) & 31) << 16) | (1u << 24);
                B.HB = 0u - 32u * B.wb - (uint32_t)(A0 & 31) + B.eb;
                B.usrc = (sbase + (uint32_t)((A0 >> 5) * 4 - S)) >> 2;
                cnext += B.cnt;
                const uint32_t tot_b = __shfl_sync(FULL, E, B.cnt - 1);
                __syncwarp();
                if (lane == 0) {
                    mbar_arrive_expect_tx(&ws.mbar[buf], tot_b);
                    fence_proxy_async();
                    bulk_g2s(reinterpret_cast<uint8_t *>(&ws.stage[0][0]) + sbase, data + S, tot_b, &ws.mbar[buf]);
                }
                return true;
            }
        }
        uint64_t lb = 0, A0 = 0, A1 = 0;
        uint32_t l = 0, nel = 0, hib = 0, v = 0, cc = 0;
        bool skipc = false;  // an empty slot: no elements, no words, no bytes
        if (valid) {
            const uint64_t offl = ((uint64_t)d0.y << 32) | d0.x;
            const uint64_t off = offl & kOffMask;
            const uint32_t deg = d0.z, ubytes = d0.w;
            l = (uint32_t)(offl >> kOffBits) & 63;
            cc = (uint32_t)(offl >> kCcShift);
            if (MODE != kModeVisit) v = a.cvtx[c];
            const uint64_t F = a.k ? (kpow2 ? (uint64_t)(deg >> kshift) : (uint64_t)deg / a.k) : 0;  // forward pointers (C8)
            const uint64_t Lb = ((uint64_t)deg * l + 7) >> 3;            // lower section bytes
            const uint64_t lbase = (off + 4 * F) * 8;
            const uint64_t U0 = (off + 4 * F + Lb) * 8;
            const uint64_t r0 = (uint64_t)cc * CH;
            const uint64_t r1 = min(r0 + CH, (uint64_t)deg);
            // chunk cc starts right after element r0-1, whose stop bit is
            // fwd[cc-1] + r0 - 1; it ends after element r1-1 (C14)
            hib = cc ? ld_u32_unaligned(data32, off + 4 * (uint64_t)(cc - 1)) : 0u;
            const uint32_t fwdc = r1 < deg ? ld_u32_unaligned(data32, off + 4 * (uint64_t)cc) : 0u;
            const uint64_t b1 = r1 < deg ? (uint64_t)fwdc + r1 : 8ull * ubytes;
            // BFS chunk skip: fwd[cc] is the high part of the chunk's last
            // element, so fwd[cc] < vpre >> l puts every element of the chunk
            // below the visited prefix: nothing to stage, decode or probe
            skipc = kChunkSkip && pskip && r1 < deg && fwdc < (vpre >> l);
            nel = skipc ? 0u : (uint32_t)(r1 - r0);
            lb = lbase + r0 * l;
            A0 = U0 + (cc ? (uint64_t)hib + r0 : 0);
            A1 = U0 + b1;
        }
        // byte ranges: lower fields [lg0, lg1) (+8 bytes for the two-word window),
        // upper words [ug0, ug1), both 16-byte aligned supersets
        uint64_t lg0 = 0, lg1 = 0, ug0 = 0, ug1 = 0;
        uint32_t bytes = 0, lsz = 0;
        bool ustage = false, merged = false;
        uint32_t nwd = 0;
        if (valid && !skipc) {
            if (l) {
                lg0 = (lb >> 3) & ~15ull;
                lg1 = ((((lb + (uint64_t)nel * l - 1) >> 5) * 4 + 8) + 15) & ~15ull;
            }
            ug0 = ((A0 >> 5) * 4) & ~15ull;
            ug1 = ((((A1 - 1) >> 5) * 4 + 4) + 15) & ~15ull;
            nwd = (uint32_t)(((A1 - 1) >> 5) - (A0 >> 5) + 1);
            ustage = ug1 - ug0 <= kUpperStageMax;
            merged = l && ustage && ug0 >= lg0 && ug0 <= lg1 + 16;
            lsz = (uint32_t)(lg1 - lg0);
            bytes = merged ? (uint32_t)(max(lg1, ug1) - lg0) : lsz + (ustage ? (uint32_t)(ug1 - ug0) : 0u);
        }
        // Two staging layouts; the one that fits more chunks wins:
        //   sum:  each chunk's ranges packed one after the other (one or two
        //         bulk copies per chunk; a lane issues its own);
        //   span: ONE bulk copy of [S, E), the byte span of consecutive chunks
        //         whose staged bytes are single ranges — frontier lists in id
        //         order are laid out in increasing offset order, so on
        //         dense levels the span is the chunks' bytes plus small gaps,
        //         without per-chunk 16-byte rounding
        uint32_t tb;
        const uint32_t sb = warp_excl_u32(bytes, tb);
        const bool fits_sum = valid && sb + bytes <= kStageBytes;
        const uint64_t rs = l ? lg0 : ug0;  // this lane's single range [rs, rs + bytes)
        const uint32_t hm = __ballot_sync(FULL, valid && bytes);
        const uint64_t S = hm ? __shfl_sync(FULL, rs, __ffs(hm) - 1) : 0ull;
        uint32_t E = 0;  // span end relative to S, inclusive max over lanes <= this one
        if (valid && bytes) E = (rs >= S && rs + bytes - S < (1ull << 30)) ? (uint32_t)(rs + bytes - S) : (1u << 30);
#pragma unroll
        for (int d = 1; d < 32; d <<= 1) {
            const uint32_t t = __shfl_up_sync(FULL, E, d);
            if ((int)lane >= d) E = max(E, t);
        }
        const bool fits_span = valid && E <= kStageBytes;
        const bool one = __all_sync(FULL, !(valid && l && ustage && !merged));
        const uint32_t cnt_sum = __popc(__ballot_sync(FULL, fits_sum));
        const uint32_t cnt_span = __popc(__ballot_sync(FULL, fits_span));
        const bool span = kSpanStage && (a.variant & 2) && one && cnt_span >= cnt_sum;  // warp-uniform
        const bool fits = span ? fits_span : fits_sum;
        B.cnt = span ? cnt_span : cnt_sum;  // a prefix of the lanes; >= 1 (one chunk always fits)
        const uint32_t buf = nbuf;
        B.buf = buf;
        nbuf ^= 1;
        uint32_t tot_e, tot_w;
        if (kpow2 && a.k <= 1024 && __all_sync(FULL, !fits || nwd < 2048)) {
            // one scan for both: a batch holds < 2^15 elements (32 chunks of <= 512)
            // and, with every chunk under 2048 words, < 2^16 words
            uint32_t t;
            const uint32_t ex = warp_excl_u32(fits ? (nel | nwd << 16) : 0u, t);
            B.eb = ex & 0xffffu;
            B.wb = ex >> 16;
            tot_e = t & 0xffffu;
            tot_w = t >> 16;
        } else {
            B.eb = warp_excl_u32(fits ? nel : 0u, tot_e);
            B.wb = warp_excl_u32(fits ? nwd : 0u, tot_w);
        }
        const uint32_t tot_b = __shfl_sync(FULL, span ? E : sb + bytes, B.cnt - 1);  // bytes of the fitting prefix
        B.ne = tot_e;
        B.nw = tot_w;
        B.nwd = nwd;
        B.v = v;
        B.cc = cc;
        B.nel = fits ? nel : 0u;
        // lane-per-chunk decode when the lanes' chunks are balanced enough:
        // >= 50 % of the warp's element slots busy (the degree relabelling puts
        // lists of similar length next to each other in the frontier)
        B.lpc = kLpc && (a.variant & 1) && lpcf * tot_e >= 32 * __reduce_max_sync(FULL, B.nel);
        // stage-area byte offset of this chunk's first staged byte
        const uint32_t base = buf * kStageBytes + (span ? (bytes ? (uint32_t)(rs - S) : 0u) : sb);
        const uint32_t lsm = sbits + (l ? base * 8 + (uint32_t)(lb - lg0 * 8) : buf * kStageBytes * 8);
        B.lsmb = lsm - B.eb * l;
        B.lflags = l | ((uint32_t)(A0 & 31) << 8) | ((uint32_t)((A1 - 1) & 31) << 16) | (ustage ? 1u << 24 : 0u);
        B.HB = hib - 32u * B.wb - (uint32_t)(A0 & 31) + B.eb;
        if (ustage) {
            const uint32_t ub = merged ? base + (uint32_t)(ug0 - lg0) : base + lsz;
            B.usrc = (ub + (uint32_t)((A0 >> 5) * 4 - ug0)) >> 2;
        } else {
            B.usrc = A0 >> 5;
        }
        cnext += B.cnt;
        // stage (the buffer was last read by the decoder two batches ago)
        __syncwarp();
        if (lane == 0) mbar_arrive_expect_tx(&ws.mbar[buf], tot_b);
        __syncwarp();
        if (span) {
            if (lane == 0 && tot_b) {
                fence_proxy_async();
                bulk_g2s(reinterpret_cast<uint8_t *>(&ws.stage[0][0]) + buf * kStageBytes, data + S, tot_b,
                         &ws.mbar[buf]);
            }
        } else if (fits) {
            fence_proxy_async();
            uint8_t *dst = reinterpret_cast<uint8_t *>(&ws.stage[0][0]) + base;
            if (merged) {
                bulk_g2s(dst, data + lg0, bytes, &ws.mbar[buf]);
            } else {
                if (lsz) bulk_g2s(dst, data + lg0, lsz, &ws.mbar[buf]);
                if (ustage) bulk_g2s(dst + lsz, data + ug0, (uint32_t)(ug1 - ug0), &ws.mbar[buf]);
            }
        }
        return true;
    };

    // ---- a6 (and the other modes' visit functors) for kU decoded elements ----
        auto visit = [&](const uint32_t (&xv)[kU], const uint32_t (&sv)[kU], const uint32_t (&ev)[kU],
                         int cntu, uint32_t &pr_slot, double &pr_acc) {
            if (MODE == kModeDecode) {
#pragma unroll
                for (int u = 0; u < kU; ++u)
                    if (u < cntu) a.out[ws.slot[sv[u]].aux + (ev[u] - ws.slot[sv[u]].eb)] = xv[u];
            } else if (MODE == kModeSssp) {
                // relax: d' = fl32(dist(u) + w), single rounding (reading C20)
                float nd[kU], cd[kU];
#pragma unroll
                for (int u = 0; u < kU; ++u) {
                    nd[u] = INFINITY;
                    cd[u] = 0.f;
                    if (u < cntu) {
                        const SlotP &sp = ws.slot[sv[u]];
                        nd[u] = __fadd_rn(sp.aux2, __ldg(a.weights + sp.aux + (ev[u] - sp.eb)));
                        cd[u] = a.dist[xv[u]];
                    }
                }
#pragma unroll
                for (int u = 0; u < kU; ++u) {
                    if (u < cntu && nd[u] < cd[u]) {  // non-negative floats order like their bits
                        const int old = atomicMin(reinterpret_cast<int *>(a.dist) + xv[u], __float_as_int(nd[u]));
                        if (__float_as_int(nd[u]) < old) atomicOr(a.vis + (xv[u] >> 5), 1u << (xv[u] & 31));
                    }
                }
            } else if (MODE == kModePrPull) {
                // pull (symmetric graphs): the lane sums contrib[u] = r(u)/deg(u) of its
                // run's neighbours and adds the sum once per list it leaves
                double cv[kU];
#pragma unroll
                for (int u = 0; u < kU; ++u) cv[u] = u < cntu ? __ldg(a.contrib + xv[u]) : 0.0;
#pragma unroll
                for (int u = 0; u < kU; ++u) {
                    if (u < cntu) {
                        if (sv[u] != pr_slot) {
                            if (pr_slot != FULL) atomicAdd(a.next + ws.slot[pr_slot].aux, pr_acc);
                            pr_slot = sv[u];
                            pr_acc = 0.0;
                        }
                        pr_acc += cv[u];
                    }
                }
            } else if (MODE == kModePagerank) {
#pragma unroll
                for (int u = 0; u < kU; ++u)
                    if (u < cntu)
                        atomicAdd(a.next + xv[u], __longlong_as_double((long long)ws.slot[sv[u]].aux));
            } else {
                // Alg. 1 line 3: hot ids answer from shared memory
                // ids below vpre are known visited without a memory access
                bool need[kU];
#pragma unroll
                for (int u = 0; u < kU; ++u) {
                    need[u] = u < cntu && xv[u] >= vpre;
                    if (kUseHot) {
                        const uint32_t hw = (need[u] && xv[u] < hot_limit) ? s_hot[xv[u] >> 5] : 0u;
                        need[u] = need[u] && !((hw >> (xv[u] & 31)) & 1);
                    }
                }
                uint32_t gv[kU];
#pragma unroll
                for (int u = 0; u < kU; ++u) gv[u] = need[u] ? a.vis[xv[u] >> 5] : FULL;
                uint32_t hit = 1;
#pragma unroll
                for (int u = 0; u < kU; ++u) hit &= shf_r_wrap(gv[u], gv[u], xv[u]);
                const bool miss = !(hit & 1);
                if (!__any_sync(__activemask(), miss)) return;  // most probes of a heavy level end here
#pragma unroll
                for (int u = 0; u < kU; ++u) {
                    const uint32_t bit = 1u << (xv[u] & 31);
                    if (!(gv[u] & bit)) {  // line 4 (the atomic decides)
                        if (MODE == kModeVisit) {
                            atomicOr(a.vis + (xv[u] >> 5), bit);
                        } else {
                            const uint32_t old = atomicOr(a.vis + (xv[u] >> 5), bit);
                            if (!(old & bit)) parent[xv[u]] = (uint32_t)ws.slot[sv[u]].aux;
                        }
                        if (kUseHot && xv[u] < hot_limit) atomicOr(s_hot + (xv[u] >> 5), bit);
                    }
                }
            }
        };

    Batch cur, nxt;
    bool have = produce(cur);
    while (have) {
        // slot table of the current batch (its producer registers are about to be reused)
        const uint32_t cnt = cur.cnt, NW = cur.nw, buf = cur.buf;
#ifdef EFG_BATCH_STATS
        // [0/1] batches lane-per-chunk / records, [2/3] their chunks, [4/5] their
        // elements, [6] 32 x longest chunk summed over the LPC batches, [7] words
        if (lane == 0) {
            const int r = cur.lpc ? 0 : 1;
            atomicAdd(&a.ctrl->bstat[r], 1ull);
            atomicAdd(&a.ctrl->bstat[2 + r], (unsigned long long)cnt);
            atomicAdd(&a.ctrl->bstat[4 + r], (unsigned long long)cur.ne);
            atomicAdd(&a.ctrl->bstat[7], (unsigned long long)NW);
        }
        {
            const uint32_t mx = __reduce_max_sync(FULL, lane < cnt ? cur.nel : 0u);
            if (lane == 0 && cur.lpc) atomicAdd(&a.ctrl->bstat[6], 32ull * mx);
        }
#endif
        if (lane < cnt) {
            SlotP sp;
            sp.lsmb = cur.lsmb;
            sp.lflags = cur.lflags;
            sp.HB = cur.HB;
            sp.eb = cur.eb;
            sp.wb = cur.wb;
            sp.nwd = cur.nwd;
            sp.usrc = cur.usrc;
            sp.aux = 0;
            sp.aux2 = 0.f;
            sp.pad = 0;
            const uint64_t r0 = (uint64_t)cur.cc * CH;
            if (MODE == kModeVisitParent) sp.aux = cur.v;
            if (MODE == kModeDecode) sp.aux = a.vlist[cur.v] + r0 - a.out_base;
            if (MODE == kModeSssp) {
                sp.aux = a.vlist[cur.v] + r0;
                sp.aux2 = a.dist[cur.v];
            }
            if (MODE == kModePrPull) sp.aux = cur.v;  // the list's vertex gathers its neighbours' shares
            if (MODE == kModePagerank) {  // push r(u)/deg(u) along every edge
                const double share = a.rank[cur.v] / (double)a.deg32[cur.v];
                sp.aux = (uint64_t)__double_as_longlong(share);
            }
            ws.slot[lane] = sp;
        }
        const uint32_t cwb = lane < cnt ? cur.wb : 0xffffffffu;  // slot word starts, for maxle
        // stage the next batch while this one is decoded
        have = produce(nxt);
        __syncwarp();
        mbar_wait(&ws.mbar[buf], (phase >> buf) & 1);
        phase ^= 1u << buf;

        if (cur.lpc) {
            // ---- lane-per-chunk: lane i walks chunk i of the batch serially
            // from the staged bytes (a5): the next stop bit of its upper words
            // gives select1(j) - j, its lower field the low bits; no word
            // records, no lane-start search.  With the prefix skip the lane
            // first steps over whole words whose last stop bit is below
            // vpre >> l (their elements are visited; P:157's pointers already
            // dropped whole chunks) ----
            if (lane < cnt && cur.nel) {
                const uint32_t nel = cur.nel, l = cur.lflags & 63, lmask = (1u << l) - 1;
                const uint32_t a0s = (cur.lflags >> 8) & 31, a1s = (cur.lflags >> 16) & 31;
                const bool staged = (cur.lflags >> 24) & 1;
                const uint32_t nwd = cur.nwd, ebase = cur.eb;
                const uint64_t usrc = cur.usrc;
                uint32_t la = cur.lsmb + ebase * l;          // lower field of element j
                uint32_t hcur = cur.HB + 32u * cur.wb - ebase;  // hi = hcur + p - j for a stop bit at p of word gl
                uint32_t gl = 0, j = 0;
                auto word = [&](uint32_t g) -> uint32_t {
                    uint32_t w = staged ? st32[usrc + g] : ldg_u32(data32 + usrc + g);
                    if (g == 0) w &= FULL << a0s;
                    if (g == nwd - 1) w &= FULL >> (31 - a1s);
                    return w;
                };
                uint32_t w = word(0);
                if (pskip) {
                    const uint32_t h0 = vpre >> l;
                    // whole words whose last stop bit has a high part below h0
                    while (gl + 1 < nwd) {
                        const uint32_t pc = __popc(w);
                        if (pc && hcur + (31 - __clz(w)) - (j + pc - 1) >= h0) break;
                        j += pc;
                        la += pc * l;
                        ++gl;
                        hcur += 32;
                        w = word(gl);
                    }
                    // inside the first kept word: the stop bit of element j + k at
                    // position p has high part hcur + p - (j + k) = hcur - j + (zeros
                    // of w below p), so the elements below h0 are the set bits
                    // below zero number D - 1 of w, D = h0 + j - hcur (select0)
                    const int32_t D = (int32_t)(h0 + j - hcur);
                    if (kLpcBitSkip && (a.variant & 8) && D > 0 && D <= 32 - __popc(w)) {
                        const uint32_t zpos = select_in_word(~w, (uint32_t)D - 1);
                        const uint32_t below = w & ((1u << zpos) - 1);  // zpos < 32: w has a zero there
                        const uint32_t cnt = __popc(below);
                        w ^= below;
                        j += cnt;
                        la += cnt * l;
                    }
                }
                uint32_t uw = __brev(w);  // reversed: the next stop bit is the leading one
                uint32_t e = ebase + j;
                auto decode1 = [&](uint32_t &x) {
                    while (uw == 0) {
                        ++gl;
                        hcur += 32;
                        uw = __brev(word(gl));
                    }
                    const uint32_t p = clz_nz(uw);
                    uw ^= 0x80000000u >> p;
                    const uint32_t hi = hcur + p - j;  // select1(j) - j
                    const uint32_t ad = (la >> 3) & ~3u;
                    const uint32_t lo = shf_r_wrap(lds_u32(ad), lds_u32(ad + 4), la) & lmask;
                    x = (hi << l) | lo;
                    la += l;
                    ++j;
                    ++e;
                };
                uint32_t pr_slot = FULL;  // PageRank pull partial sum (one list per lane)
                double pr_acc = 0.0;
                for (; j + kU <= nel;) {
                    uint32_t xv[kU], sv[kU], ev[kU];
#pragma unroll
                    for (int u = 0; u < kU; ++u) {
                        ev[u] = e;
                        sv[u] = lane;
                        decode1(xv[u]);
                    }
                    visit(xv, sv, ev, kU, pr_slot, pr_acc);
                }
                if (j < nel) {
                    uint32_t xv[kU], sv[kU], ev[kU];
                    const int cntu = (int)(nel - j);
#pragma unroll
                    for (int u = 0; u < kU; ++u) {
                        xv[u] = 0;
                        sv[u] = lane;
                        ev[u] = e;
                        if (u < cntu) decode1(xv[u]);
                    }
                    visit(xv, sv, ev, cntu, pr_slot, pr_acc);
                }
                if (MODE == kModePrPull && pr_slot != FULL) atomicAdd(a.next + ws.slot[pr_slot].aux, pr_acc);
            }
            __syncwarp();
            cur = nxt;
            continue;
        }

        uint32_t Er0 = 0;  // batch element index at the round start
        for (uint32_t ga = 0; ga < NW; ga += kRoundWords) {
            const uint32_t nw = min(kRoundWords, NW - ga);
            // ---- round words: mask, popcount prefix, records ----
            // BFS prefix skip: a word whose stop bits all have a high part
            // below vpre >> l holds only ids below the visited prefix (lists
            // are sorted): no record, so those elements are neither decoded
            // nor probed (their bytes are staged all the same)
            uint32_t run = Er0, krun = 0, nrec = 0;
#pragma unroll
            for (uint32_t j = 0; j < kRoundWords / 32; ++j) {
                if (j * 32 >= nw) break;
                const uint32_t gl = j * 32 + lane;
                const uint32_t g = ga + gl;
                const int sl = warp_maxle_u32(cwb, gl < nw ? g : 0u);
                uint32_t wd = 0;
                const SlotP &sp = ws.slot[sl];
                if (gl < nw) {
                    const uint64_t idx = sp.usrc + (g - sp.wb);
                    wd = (sp.lflags >> 24) ? st32[idx] : ldg_u32(data32 + idx);
                    if (g == sp.wb) wd &= FULL << ((sp.lflags >> 8) & 31);
                    if (g == sp.wb + sp.nwd - 1) wd &= FULL >> (31 - ((sp.lflags >> 16) & 31));
                }
                const uint32_t pc = __popc(wd);
                uint32_t tot;
                const uint32_t ex = warp_excl_u32(pc, tot);
                const uint32_t l = sp.lflags & 63;
                // stop bit at p, j-th of the record: high part hb + p - j = select1(i) - i
                const uint32_t hb = 32 * g + sp.HB - (run + ex);
                bool keep = wd != 0;
                uint32_t kex = ex, ktot = tot;  // kept-element prefix (= all without the skip)
                const uint32_t nzm = __ballot_sync(FULL, wd != 0);
                if (pskip) {
                    keep = keep && hb + (31 - __clz(wd)) - (pc - 1) >= (vpre >> l);
                    const uint32_t km0 = __ballot_sync(FULL, keep);
                    if (km0 == 0) {  // every word of these 32 skipped
                        kex = 0;
                        ktot = 0;
                    } else if (km0 != nzm) {  // some skipped: scan the kept popcounts
                        kex = warp_excl_u32(keep ? pc : 0u, ktot);
                    }
                }
                const uint32_t km = __ballot_sync(FULL, keep);
                if (keep) {
                    const uint32_t k = nrec + __popc(km & ((1u << lane) - 1));
                    ws.wrec[k] = make_uint4(__brev(wd), hb, sp.lsmb + (run + ex) * l, l | ((uint32_t)sl << 8));
                    ws.wpre[k] = krun + kex;
                }
                run += tot;
                krun += ktot;
                nrec += __popc(km);
            }
            __syncwarp();
            const uint32_t Er1 = run;
            const uint32_t NK = krun;  // kept elements of the round
            uint32_t c = (uint32_t)(((uint64_t)lane * NK) >> 5);
            const uint32_t c1 = (uint32_t)(((uint64_t)(lane + 1) * NK) >> 5);
            if (c < c1) {
                // ---- lane start: record of kept element c (maxle) + in-word select ----
                uint32_t k = 0;
#pragma unroll
                for (uint32_t step = kSearchStep; step; step >>= 1)
                    if (k + step < nrec && ws.wpre[k + step] <= c) k += step;
                // records hold bit-reversed words: the lowest remaining stop bit is the
                // leading one (clz), so no bit reversal per element
                uint4 r = ws.wrec[k];
                uint32_t j = c - ws.wpre[k];  // rank of the lane's first element in its record
                if (j) r.x &= FULL >> select_in_word(__brev(r.x), j);  // drop j stop bits
                uint32_t l = r.w & 63, lmask = (1u << l) - 1;
                uint32_t e = Er0 + c;  // batch element index (modes without the skip keep every record)
                uint32_t pr_slot = FULL;  // PageRank pull: slot being summed and its partial sum
                double pr_acc = 0.0;

                // one element: next stop bit -> select1(i) - i, lower field, value
                auto decode = [&](uint32_t &x, uint32_t &slot_of) {
                    if (r.x == 0) {  // next record (always has a stop bit)
                        ++k;
                        r = ws.wrec[k];
                        j = 0;
                        l = r.w & 63;
                        lmask = (1u << l) - 1;
                    }
                    const uint32_t p = clz_nz(r.x);
                    r.x ^= 0x80000000u >> p;
                    const uint32_t hi = r.y + p - j;  // select1(i) - i
                    const uint32_t la = r.z + j * l;
                    const uint32_t ad = (la >> 3) & ~3u;
                    const uint32_t lo = shf_r_wrap(lds_u32(ad), lds_u32(ad + 4), la) & lmask;
                    x = (hi << l) | lo;  // (select1(i) - i) << l | lower[i]
                    slot_of = r.w >> 8;
                    ++j;
                    ++e;
                };

                // main loop: kU elements per step, no per-element guards
                for (; c + kU <= c1; c += kU) {
                    uint32_t xv[kU], sv[kU], ev[kU];
#pragma unroll
                    for (int u = 0; u < kU; ++u) {
                        ev[u] = e;
                        decode(xv[u], sv[u]);
                    }
                    visit(xv, sv, ev, kU, pr_slot, pr_acc);
                }
                // tail: < kU elements
                if (c < c1) {
                    uint32_t xv[kU], sv[kU], ev[kU];
                    const int cntu = (int)(c1 - c);
#pragma unroll
                    for (int u = 0; u < kU; ++u) {
                        xv[u] = 0;
                        sv[u] = 0;
                        ev[u] = e;
                        if (u < cntu) decode(xv[u], sv[u]);
                    }
                    visit(xv, sv, ev, cntu, pr_slot, pr_acc);
                }
                if (MODE == kModePrPull && pr_slot != FULL) atomicAdd(a.next + ws.slot[pr_slot].aux, pr_acc);
            }
            __syncwarp();
            Er0 = Er1;
        }
        cur = nxt;
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

__global__ void pr_update_kernel(double *rank, double *next, uint64_t n, double damping, const double *dsum,
                                 double *contrib, const uint32_t *deg32)
{
    const double base = (1.0 - damping) / (double)n, dn = *dsum / (double)n;
    for (uint64_t v = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; v < n; v += (uint64_t)gridDim.x * blockDim.x) {
        const double r = base + damping * (next[v] + dn);
        rank[v] = r;
        next[v] = 0.0;
        if (contrib) contrib[v] = deg32[v] ? r / (double)deg32[v] : 0.0;  // pull: next iteration's shares
    }
}

__global__ void pr_contrib_kernel(const double *rank, const uint32_t *deg32, double *contrib, uint64_t n)
{
    for (uint64_t v = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; v < n; v += (uint64_t)gridDim.x * blockDim.x)
        contrib[v] = deg32[v] ? rank[v] / (double)deg32[v] : 0.0;
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

// host depth transfer: one byte per vertex (every depth in [-1, 126])
__global__ void pack8_kernel(const int32_t *in, int8_t *out, uint64_t n)
{
    for (uint64_t i = (blockIdx.x * (uint64_t)blockDim.x + threadIdx.x) * 4; i < n; i += (uint64_t)gridDim.x * blockDim.x * 4) {
        if (i + 4 <= n) {
            const int4 v = *reinterpret_cast<const int4 *>(in + i);
            const uint32_t b = (uint32_t)(uint8_t)v.x | (uint32_t)(uint8_t)v.y << 8 | (uint32_t)(uint8_t)v.z << 16 |
                               (uint32_t)(uint8_t)v.w << 24;
            *reinterpret_cast<uint32_t *>(out + i) = b;
        } else {
            for (uint64_t j = i; j < n; ++j) out[j] = (int8_t)in[j];
        }
    }
}

__global__ void map_parent_kernel(const uint32_t *pin, const uint32_t *old_of_new, uint32_t *pout, uint64_t n)
{
    for (uint64_t i = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; i < n; i += (uint64_t)gridDim.x * blockDim.x) {
        const uint32_t p = pin[i];
        pout[old_of_new[i]] = p == FULL ? FULL : old_of_new[p];
    }
}

// frontier-order study: the level's chunks in a pseudo-random order (an
// "arbitrary order" frontier), same tiles (index ranges)
__global__ void shuffle_chunks_kernel(const ChunkDesc *in, const uint32_t *cvin, ChunkDesc *out, uint32_t *cvout,
                                      const LevelCtrl *ctrl)
{
    const uint64_t N = ctrl->nchunks;
    for (uint64_t c = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; c < N; c += (uint64_t)gridDim.x * blockDim.x) {
        const uint64_t d = (c * 2654435761ull + 12345ull) % N;
        out[d] = in[c];
        if (cvin) cvout[d] = cvin[c];
    }
}

}  // namespace

cudaError_t launch_shuffle_chunks(const ChunkDesc *in, const uint32_t *cvin, ChunkDesc *out, uint32_t *cvout,
                                  const LevelCtrl *ctrl, int blocks, cudaStream_t s)
{
    shuffle_chunks_kernel<<<blocks, 256, 0, s>>>(in, cvin, out, cvout, ctrl);
    return cudaGetLastError();
}

static unsigned grid_for(uint64_t n) { return (unsigned)std::max<uint64_t>(1, std::min<uint64_t>((n + 255) / 256, 148 * 16)); }

cudaError_t launch_pr_dangling(const double *rank, const uint32_t *deg32, uint64_t n, double *dsum, cudaStream_t s)
{
    pr_dangling_kernel<<<grid_for(n), 256, 0, s>>>(rank, deg32, n, dsum);
    return cudaGetLastError();
}

cudaError_t launch_pr_update(double *rank, double *next, uint64_t n, double damping, const double *dsum,
                             double *contrib, const uint32_t *deg32, cudaStream_t s)
{
    pr_update_kernel<<<grid_for(n), 256, 0, s>>>(rank, next, n, damping, dsum, contrib, deg32);
    return cudaGetLastError();
}

cudaError_t launch_pr_contrib(const double *rank, const uint32_t *deg32, double *contrib, uint64_t n, cudaStream_t s)
{
    pr_contrib_kernel<<<grid_for(n), 256, 0, s>>>(rank, deg32, contrib, n);
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

// host depth transfer in 4-bit codes (every depth < 15): out word g holds
// depth + 1 of vertices 8g .. 8g+7 (low nibble first; 0 = unreached)
__global__ void pack4_kernel(const int32_t *in, uint32_t *out, uint64_t n)
{
    const uint64_t G = (n + 7) / 8;
    for (uint64_t g = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; g < G; g += (uint64_t)gridDim.x * blockDim.x) {
        const uint64_t i = 8 * g;
        uint32_t w = 0;
        if (i + 8 <= n) {
            const int4 a = *reinterpret_cast<const int4 *>(in + i);
            const int4 b = *reinterpret_cast<const int4 *>(in + i + 4);
            w = ((uint32_t)(a.x + 1) & 15u) | ((uint32_t)(a.y + 1) & 15u) << 4 | ((uint32_t)(a.z + 1) & 15u) << 8 |
                ((uint32_t)(a.w + 1) & 15u) << 12 | ((uint32_t)(b.x + 1) & 15u) << 16 |
                ((uint32_t)(b.y + 1) & 15u) << 20 | ((uint32_t)(b.z + 1) & 15u) << 24 | ((uint32_t)(b.w + 1) & 15u) << 28;
        } else {
            for (uint64_t j = i; j < n; ++j) w |= ((uint32_t)(in[j] + 1) & 15u) << (4 * (j - i));
        }
        out[g] = w;
    }
}

cudaError_t launch_pack4(const int32_t *in, uint32_t *out, uint64_t n, cudaStream_t s)
{
    const unsigned blocks = (unsigned)std::max<uint64_t>(1, std::min<uint64_t>((n / 8 + 255) / 256, 148 * 8));
    pack4_kernel<<<blocks, 256, 0, s>>>(in, out, n);
    return cudaGetLastError();
}

cudaError_t launch_pack8(const int32_t *in, int8_t *out, uint64_t n, cudaStream_t s)
{
    const unsigned blocks = (unsigned)std::max<uint64_t>(1, std::min<uint64_t>((n / 4 + 255) / 256, 148 * 8));
    pack8_kernel<<<blocks, 256, 0, s>>>(in, out, n);
    return cudaGetLastError();
}

cudaError_t launch_map_parent(const uint32_t *pin, const uint32_t *old_of_new, uint32_t *pout, uint64_t n,
                              cudaStream_t s)
{
    const unsigned blocks = (unsigned)std::max<uint64_t>(1, std::min<uint64_t>((n + 255) / 256, 148 * 16));
    map_parent_kernel<<<blocks, 256, 0, s>>>(pin, old_of_new, pout, n);
    return cudaGetLastError();
}

size_t expand_smem_bytes() { return kExpandSmem; }

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
    if (e == cudaSuccess)
        e = cudaFuncSetAttribute(expand_kernel<kModePrPull>, cudaFuncAttributeMaxDynamicSharedMemorySize, bytes);
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
    case kModePrPull:
        expand_kernel<kModePrPull><<<blocks, kExpandThreads, sm, s>>>(a);
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

int frontier_occupancy()
{
    int nb = 0;
    if (cudaOccupancyMaxActiveBlocksPerMultiprocessor(&nb, frontier_kernel, kFrontierThreads, 0) != cudaSuccess) {
        cudaGetLastError();
        return 0;
    }
    return nb;
}

cudaError_t launch_frontier(const FrontierArgs &a, unsigned blocks, cudaStream_t s)
{
    frontier_kernel<<<blocks, kFrontierThreads, 0, s>>>(a);
    return cudaGetLastError();
}

cudaError_t launch_xchg(const XchgArgs &a, cudaStream_t s)
{
    const uint64_t total = (uint64_t)(a.op == 1 ? 1 : a.world) * a.S;
    const unsigned blocks = (unsigned)std::max<uint64_t>(1, std::min<uint64_t>((total + 255) / 256, 148 * 8));
    xchg_kernel<<<blocks, 256, 0, s>>>(a);
    return cudaGetLastError();
}

cudaError_t launch_peer(const PeerArgs &a, int max_blocks, cudaStream_t s)
{
    // the barrier ops spin in ONE block (a rank waiting for the others holds
    // one block's worth of an SM, which matters when ranks share a device);
    // the data ops never wait
    const unsigned blocks = (a.op == 3 || a.op == 4)
                                ? 1u
                                : (unsigned)std::max<uint64_t>(1, std::min<uint64_t>((a.nwords + 255) / 256,
                                                                                     (uint64_t)max_blocks));
    peer_kernel<<<blocks, 256, 0, s>>>(a);
    return cudaGetLastError();
}


}  // namespace efg
