// efg_kernels.cuh — launchers for the sm_100a kernels (efg_kernels.cu).
#pragma once

#include <cuda_runtime.h>

#include "efg_internal.h"

namespace efg {

enum ExpandMode : int {
    kModeVisit = 0,        // BFS: visited-bitmap probe + atomicOr (Alg. 1 lines 3-4)
    kModeVisitParent = 1,  // BFS with parents (winner of the atomicOr writes parent)
    kModeDecode = 2,       // efg_decode: store the decoded value in CSR order
    kModeSssp = 3,         // SSSP relax: atomicMin on fp32 dist, mark relaxed vertices
    kModePagerank = 4,     // PageRank push: next[v] += r(u)/deg(u)
    kModePrPull = 5,       // PageRank pull (symmetric graphs): next[u] += sum of contrib[v] over u's list
};

struct ExpandArgs {
    const uint8_t *data;       // EF data (device, 4-byte aligned, padded)
    const ChunkDesc *chunks;   // chunk descriptors of the level (frontier_kernel)
    const uint32_t *cvtx;      // source vertex of each chunk (modes other than plain BFS)
    const uint32_t *tiles;     // tile table: first chunk of tile t (ntiles + 1 entries)
    const uint32_t *deg32;     // degrees (PageRank share)
    LevelCtrl *ctrl;           // nf, ne, ntiles of this level; parent pointer; level
    uint32_t *vis;             // visited bitmap (modes 0, 1)
    uint32_t *out;             // decode output (mode 2): CSR positions minus out_base
    uint64_t out_base;
    LevelStat *stats;          // per-level statistics (device) or null
    const uint64_t *vlist;     // SSSP: CSR offsets (weight index)
    const float *weights;      // SSSP: weights in CSR order
    float *dist;               // SSSP: distances (stored ids)
    const double *rank;        // PageRank: current ranks (stored ids)
    double *next;              // PageRank: accumulated pushes
    const double *contrib;     // PageRank pull: r(v)/deg(v) per vertex
    uint32_t max_stats;
    uint32_t hot_words;        // bitmap words with a shared-memory snapshot (multiple of 4)
    uint32_t k;                // forward-pointer quantum (chunk length); 0 = none
    uint32_t pskip;            // BFS: skip upper words whose ids are all below the visited prefix
    uint32_t lpc_skip_vpre;    // visited prefix from which a level counts as a skip level (n / 3)
    uint32_t variant;          // EFG_OPT_EXPAND_VARIANT: bit 0 lane-per-chunk decode, bit 1 span staging
};

struct InitArgs {
    LevelCtrl *ctrl;
    uint32_t *vis;
    int32_t *depth;            // depth buffer of this call (device)
    uint32_t *parent;          // parent buffer of this call (device) or null
    uint64_t v0, v1;           // start set [v0, v1)
};

struct XchgArgs {
    int op;                        // 0 pack, 1 reduce, 2 unpack
    int world;
    uint64_t S;                    // slice words
    const uint64_t *bounds;        // device copy of the vertex bounds (world+1)
    uint32_t *vis;
    const uint32_t *prev;
    uint32_t *out;
    const uint32_t *in;
};

// Peer-memory exchange (efg_xchg_peer): every rank's region, mapped into every
// rank (CUDA IPC over NVLink / NVSwitch, or plain pointers on one device), is
//   [flags: kPeerFlagWords u32 | pub: peer_pad(nwords) u32 | res: peer_pad(nwords) u32 |
//    sp: kPeerSpWords u32 | list: 2 * peer_list_cap(nwords) u32]
// flags[p] = the last barrier epoch rank p signalled to this rank; sp[0] = the
// number of non-zero words this rank published (its sparse list: (word, bits)
// pairs, complete while sp[0] <= cap); sp[1] = this rank's decision for the
// current exchange (1 sparse, 0 dense).
constexpr int kPeerMaxWorld = 64;
constexpr uint64_t kPeerFlagWords = 64;
constexpr uint64_t kPeerSpWords = 32;
__host__ __device__ inline uint64_t peer_pad(uint64_t nwords) { return (nwords + 31) & ~31ull; }
// sparse-level exchange: at most 1/32 of the words non-zero on every rank
__host__ __device__ inline uint64_t peer_list_cap(uint64_t nwords) { return peer_pad(nwords) / 32 + 32; }
__host__ __device__ inline uint64_t peer_sp_off(uint64_t nwords) { return kPeerFlagWords + 2 * peer_pad(nwords); }
__host__ __device__ inline uint64_t peer_region_words(uint64_t nwords)
{
    return peer_sp_off(nwords) + kPeerSpWords + 2 * peer_list_cap(nwords);
}

struct PeerArgs {
    uint32_t *const *peers;        // device array [world]: region base of every rank (own included)
    uint32_t *local;               // this rank's region
    const uint64_t *bounds;        // device copy of the vertex bounds (world+1)
    uint32_t *vis;
    const uint32_t *prev;
    uint32_t *fault;               // LevelCtrl.fault: a barrier wait timed out
    uint64_t nwords;
    uint32_t *epoch;               // device exchange counter (LevelCtrl.peer_epoch): op 0 adds 2,
                                   // ops 1 and 2 wait on barrier epochs counter-1 and counter
    uint32_t *sparse_levels;       // LevelCtrl.xchg_sparse: exchanges that took the sparse path
    int world, rank;
    int op;                        // 0 publish, 1 owner OR + broadcast, 2 unpack, 3 / 4 barrier (one block)
};

struct FrontierArgs {           // level end (a7) + next level plan (a1-a4), one launch
    uint32_t *vis, *prev;      // visited bitmap now / at the previous level end
    const uint32_t *iso;       // degree-0 vertices (never probed): count as visited for the visited prefix
    int32_t *depth_stored;     // depth by stored id (relabelled graphs)
    int depth_stored_only;     // 1: depth_stored is the only depth output (relabelled graphs)
    int consume;               // 1: frontier = vis itself, vis reset (SSSP relaxed set)
    const uint32_t *deg32;     // degrees (pass 1)
    const uint32_t *umax;      // largest neighbour of each list
    uint32_t lskip;            // BFS: lists whose largest neighbour is below the visited prefix are not planned
                               // (1: ctrl->vpre_used, the previous level's; 2: this level's, phase 0)
    uint32_t *skipw;           // scratch (nwords): per bitmap word, the skipped lists (phase 1 -> phase 2)
    const VRec *rec;           // vertex records (pass 2)
    ChunkDesc *chunks;         // out: chunk descriptors
    uint32_t *cvtx;            // out: source vertex of each chunk, or null (plain BFS never reads it)
    uint32_t *tiles;           // out: first chunk of each tile (+ sentinel)
    LevelCtrl *ctrl;           // in: level, seq, depth ptr; out: nf, ne, nwork, nchunks, ntiles, xlevel, vmin2
    uint64_t *status;          // five per-block aggregate regions of kMaxGrid words
    unsigned long long *barrier;  // grid-barrier arrival counter (grows by gridDim.x per barrier)
    BigList *big;              // scratch: lists planned by the whole grid
    unsigned long long *trace; // debug (EFG_FRONTIER_TRACE): per block, 8 phase timestamps, or null
    LevelStat *stats;
    uint32_t max_stats;
    uint32_t k;
    int32_t kshift;
    cudaGraphConditionalHandle cond;  // graph-mode loop condition, 0 = host loop
    int cond_global;                  // 1: loop while the global new count (ctrl->nnew) is non-zero
                                      // (partitioned traversal), 0: while this rank's frontier is
    uint64_t nwords, words_per_block;
    uint64_t own_lo_w, own_hi_w;  // owned bitmap words: only these enter the frontier
};

cudaError_t launch_expand(int mode, const ExpandArgs &a, int blocks, cudaStream_t s);
cudaError_t launch_init(const InitArgs &a, cudaStream_t s);
cudaError_t launch_frontier(const FrontierArgs &a, unsigned blocks, cudaStream_t s);
int frontier_occupancy();  // resident frontier_kernel blocks per SM (its grid must fit: blocks spin on predecessors)
cudaError_t launch_xchg(const XchgArgs &a, cudaStream_t s);
cudaError_t launch_peer(const PeerArgs &a, int max_blocks, cudaStream_t s);
int expand_occupancy(int mode);
size_t expand_smem_bytes();
// pout[old_of_new[i]] = pin[i] == ~0u ? ~0u : old_of_new[pin[i]]  (parents back to input ids)
cudaError_t launch_pr_dangling(const double *rank, const uint32_t *deg32, uint64_t n, double *dsum, cudaStream_t s);
cudaError_t launch_pr_update(double *rank, double *next, uint64_t n, double damping, const double *dsum,
                             double *contrib, const uint32_t *deg32, cudaStream_t s);
cudaError_t launch_pr_contrib(const double *rank, const uint32_t *deg32, double *contrib, uint64_t n, cudaStream_t s);
cudaError_t launch_fill(uint32_t *p, uint32_t val, uint64_t n, cudaStream_t s);
cudaError_t launch_fill_f64(double *p, double val, uint64_t n, cudaStream_t s);
cudaError_t launch_gather32(const uint32_t *stored, const uint32_t *new_of_old, uint32_t *out, uint64_t n,
                            cudaStream_t s);
cudaError_t launch_gather64(const double *stored, const uint32_t *new_of_old, double *out, uint64_t n,
                            cudaStream_t s);
cudaError_t launch_map_depth(const int32_t *stored, const uint32_t *new_of_old, int32_t *out, uint64_t n,
                             cudaStream_t s);
cudaError_t launch_pack8(const int32_t *in, int8_t *out, uint64_t n, cudaStream_t s);  // n % 4 handled
cudaError_t launch_pack4(const int32_t *in, uint32_t *out, uint64_t n, cudaStream_t s);  // n % 8 handled
// frontier-order study: out[pi(c)] = in[c] for the
// level's chunk descriptors, pi(c) = (c * 2654435761 + 12345) mod nchunks (a
// bijection: the multiplier is prime and larger than any chunk count it meets)
cudaError_t launch_shuffle_chunks(const ChunkDesc *in, const uint32_t *cvin, ChunkDesc *out, uint32_t *cvout,
                                  const LevelCtrl *ctrl, int blocks, cudaStream_t s);
cudaError_t launch_map_parent(const uint32_t *pin, const uint32_t *old_of_new, uint32_t *pout, uint64_t n,
                              cudaStream_t s);

}  // namespace efg
