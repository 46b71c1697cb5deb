// efg_internal.h — internal structures shared by the host builder
// (efg_builder.cpp), the C-ABI glue (efg_api.cu) and the kernels (efg_kernels.cu).
// Not part of the ABI.  Citations: PAPER.md "P:<line> §<section>".
#pragma once

#include <cstdint>
#include <cstddef>
#include <string>
#include <vector>

#include <cuda_runtime.h>

#include "efg.h"

namespace efg {

// ---------------------------------------------------------------------------
// Host-side EFG (§V): the four arrays of the format.
// ---------------------------------------------------------------------------
struct HostEFG {
    uint64_t n = 0;                 // vertices
    uint64_t m = 0;                 // directed edges (post symmetrise/dedup)
    uint64_t m_input = 0;
    uint32_t k = 512;               // forward-pointer quantum
    std::vector<uint64_t> vlist;    // n+1  (degree = vlist[v+1]-vlist[v])
    std::vector<uint8_t> nlb;       // n    num_lower_bits
    std::vector<uint64_t> offsets;  // n+1  exclusive sum of per-vertex byte sizes
    std::vector<uint8_t> data;      // offsets[n] bytes (+ padding on device)
    std::vector<float> weights;     // m (CSR order) or empty
    std::vector<uint32_t> old_of_new, new_of_old;  // EFG_REORDER_DEGREE relabelling (else empty)
    std::vector<uint8_t> has_in;    // n: vertex has an in-edge (stored ids; all rows)
    std::vector<uint32_t> umax;     // n: largest neighbour (list's last element, P:218 u), 0 if empty
    uint64_t fwd_bytes = 0, lower_bytes = 0, upper_bytes = 0, apriori_bits = 0;
    uint64_t row_lo = 0, row_hi = 0;
    bool symmetric = false;         // built with EFG_SYMMETRIZE: out-lists = in-lists
    double build_seconds = 0.0;
};

// Elias-Fano parameters of one list (readings C1-C4, C7, C8).
struct ListGeom {
    uint32_t l;        // lower bits per element
    uint64_t fwd;      // bytes of forward pointers = 4*floor(n/k)
    uint64_t lower;    // bytes of lower bits = ceil(n*l/8)
    uint64_t upper;    // bytes of upper bits = ceil(((u>>l)+n)/8)
};

ListGeom list_geom(uint64_t n, uint64_t u, uint32_t k);

// Builder (efg_builder.cpp).  Returns EFG_OK or an error with set_error().
efg_status build_host(uint64_t n, uint64_t m, const uint32_t *src, const uint32_t *dst,
                      const efg_build_opts &o, HostEFG &out);
efg_status build_host_stream(uint64_t n, uint64_t m, efg_edge_gen_fn gen, void *user, int weighted,
                             const efg_build_opts &o, HostEFG &out);
// On-disk EFG (efg_io.cpp).
efg_status save_host(const HostEFG &h, const char *path);
efg_status load_host(const char *path, HostEFG &h);

// ---------------------------------------------------------------------------
// Device layout
// ---------------------------------------------------------------------------
// Packed 16-byte vertex record: one aligned 128-bit load gives everything the
// frontier step a1 needs (degree, data offset, l, upper-section length).
struct alignas(16) VRec {
    uint64_t off_l;   // bits 0..39: offsets[v] (byte offset in data); bits 40..45: l; 46..63: 0
    uint32_t deg;     // vlist[v+1]-vlist[v]
    uint32_t ubytes;  // upper-bits section length in bytes
};
static_assert(sizeof(VRec) == 16, "VRec must be 16 bytes");

constexpr int kOffBits = 40;                            // data byte offsets < 2^40 (1 TiB)
constexpr uint64_t kOffMask = (1ull << kOffBits) - 1;
constexpr int kCcShift = 46;                            // ChunkDesc: chunk index above l
constexpr int kCcBits = 64 - kCcShift;                  // chunk index field: cc < 2^18
constexpr uint32_t kMaxDeviceQuantum = 512;             // largest device chunk (its lower fields fit a staging buffer)

// Chunk descriptor (step a1, written by frontier_kernel, read by expand_kernel):
// one k-aligned piece of a frontier vertex's list.  The expand
// kernel derives the chunk's bit ranges from it and the forward pointers (a4).
struct alignas(16) ChunkDesc {
    uint64_t off_l_cc;  // the list's VRec.off_l (offset: 40 bits, l: bits 40-45) | chunk index cc << 46
                        // (rank of the chunk's first element r0 = cc*k; device_upload picks the
                        // device quantum k so that ceil(deg/k) < 2^kCcBits for every list)
    uint32_t deg;       // list length
    uint32_t ubytes;    // upper-bits section bytes of the list
};
static_assert(sizeof(ChunkDesc) == 16, "ChunkDesc must be 16 bytes");
// The chunk's source vertex lives in a parallel array (cvtx), read only by the
// modes that need it (parents, decode, SSSP, PageRank): a BFS moves 16 B per chunk.

// Level control block (device), written by the advance kernel.
struct LevelCtrl {
    uint64_t nf;        // frontier size for the next expand
    uint64_t ne;        // edges out of that frontier (E_L)
    uint64_t ntiles;    // ceil(nwork / kTileWork)
    uint64_t nwork;     // work units = ne + kChunkWork * nchunks
    uint64_t nchunks;   // chunk descriptors of the level
    int32_t *depth;     // depth buffer of the current call
    uint32_t *parent;   // parent buffer of the current call, or null
    uint32_t level;     // depth assigned by the next frontier_kernel
    uint32_t xlevel;    // index of the level the next expand processes
    uint32_t seq;       // tag of the cross-block prefix words of this level
    uint32_t nlevels;   // levels expanded so far
    uint64_t nnew;      // vertices discovered in the last level (all rows; partitioned runs)
    uint64_t total_nf;  // sum of frontier sizes (= vertices reached)
    uint64_t total_ne;  // sum of E_L (= edges traversed, reading C18)
    uint32_t vmin2[2];  // frontier_kernel of level L: smallest vertex neither visited nor isolated, in
                        // slot L & 1 (atomicMin); the expand of level L reads it as its visited prefix
    uint32_t vpre_used; // visited prefix the last BFS expand used (0: none); lower bound for the next level end
    uint32_t fault;     // a frontier_kernel grid barrier timed out (sticky; reported by the host)
    uint32_t peer_epoch;  // peer exchange counter (efg_xchg_peer / partitioned efg_bfs): +2 per exchange
    uint32_t xchg_sparse; // exchanges of the current traversal that took the sparse path
    unsigned long long bstat[8];  // debug builds (EFG_BATCH_STATS): expand batch counters of the last level
};

// A frontier list whose chunk descriptors and tile boundaries are written by
// the whole grid rather than by the warp that planned it (frontier_kernel):
// lists of more than one chunk or more than one tile of work.
struct BigList {
    uint64_t W;       // work position of the list's first unit
    uint64_t cstart;  // index of its first chunk descriptor
    uint64_t off_l;   // VRec.off_l
    uint32_t deg, ubytes, v, nch;
};
static_assert(sizeof(BigList) == 40, "BigList");

// Per-level statistics written on the device (graph mode has no host loop).
struct LevelStat {
    uint64_t nf, ne;                 // frontier size and its edges
    unsigned long long t0, t1;       // expand kernel start / end (%globaltimer, ns)
};
constexpr uint32_t kMaxLevelStats = 4096;

// expand_kernel: one CTA per SM, kExpandWarps warps; each warp owns two
// staging buffers (TMA double buffering) and a word-round workspace.
#ifndef EFG_EXPAND_THREADS
#define EFG_EXPAND_THREADS 768
#endif
constexpr int kExpandThreads = EFG_EXPAND_THREADS;
constexpr int kExpandWarps = kExpandThreads / 32;
#ifndef EFG_STAGE_BYTES
#define EFG_STAGE_BYTES 2560
#endif
constexpr uint32_t kStageBytes = EFG_STAGE_BYTES;       // one staging buffer (>= the largest single chunk)
// upper-bit regions larger than this are read from global memory; a chunk's
// lower fields take at most 512*23/8 + 24 bytes (n*2^l <= u < 2^32), so one
// chunk always fits a staging buffer
constexpr uint32_t kUpperStageMax = (kStageBytes - 1536 - 64) < 1024 ? ((kStageBytes - 1536 - 64) & ~15u) : 1024u;
static_assert(kStageBytes >= 2048, "staging buffer too small for one chunk");
#ifndef EFG_ROUND_WORDS
#define EFG_ROUND_WORDS 64
#endif
constexpr uint32_t kRoundWords = EFG_ROUND_WORDS;        // upper-bit words decoded per round
#ifndef EFG_HOT_WORDS
#define EFG_HOT_WORDS 4
#endif
constexpr uint32_t kHotWords = EFG_HOT_WORDS;     // > 4: shared-memory visited snapshot of the first 32*kHotWords ids (off: vpre covers the visited prefix)
#ifndef EFG_FRONTIER_THREADS
#define EFG_FRONTIER_THREADS 256
#endif
constexpr int kFrontierThreads = EFG_FRONTIER_THREADS;  // frontier_kernel (8 warps; 1024 threads per SM)
constexpr int kBitmapAlign = 1024;           // bitmap words are padded to a multiple of this
// Step a3 partitions "work units" rather than bare edges: a chunk costs
// kChunkWork units (descriptor, staging, set-up) plus one per element, so a
// tile of kTileWork units holds at most kTileWork/kChunkWork chunks.
#ifndef EFG_TILE_WORK
#define EFG_TILE_WORK 2048
#endif
constexpr uint32_t kTileWork = EFG_TILE_WORK;         // work units per tile (a3)
static_assert((kTileWork & (kTileWork - 1)) == 0, "kTileWork: a power of two (tile indices by shifts)");
constexpr uint32_t kChunkWork = 32;          // per-chunk overhead in work units
#ifndef EFG_FRONTIER_SPARSE
#define EFG_FRONTIER_SPARSE 1
#endif
constexpr bool kFrontierSparse = EFG_FRONTIER_SPARSE;  // frontier_kernel phase 2: compacted slots for sparse groups
#ifndef EFG_TILE_BIG_MIN_WORK
#define EFG_TILE_BIG_MIN_WORK (1ull << 27)
#endif
constexpr uint64_t kTileBigMinWork = EFG_TILE_BIG_MIN_WORK;  // levels with this much work use 2 x kTileWork tiles

constexpr unsigned kMaxGrid = 4096;
constexpr int kD2HChunks = 8;               // host depth transfer pipeline depth

struct DeviceGraph {
    int device = -1;
    void *stream = nullptr;            // cudaStream_t
    uint64_t n = 0, nwords = 0;        // nwords = ceil(n/32) rounded up
    uint32_t k = 512;
    uint8_t *data = nullptr;           // EF data + padding (device address; mapped host memory when out-of-core)
    uint8_t *data_host = nullptr;      // out-of-core (EFG_HOST_RESIDENT): the pinned host allocation behind `data`
    uint64_t data_bytes = 0;
    VRec *rec = nullptr;               // n records
    uint32_t *deg32 = nullptr;         // n degrees (padded to the bitmap size)
    uint32_t *umax = nullptr;          // n largest neighbour per list (padded to the bitmap size)
    uint32_t *skipw = nullptr;         // frontier_kernel scratch: skipped lists per bitmap word
    int8_t *depth8 = nullptr;          // host depth transfer: 1 byte per vertex (device) ...
    int8_t *depth8_host = nullptr;     // ... and its pinned host staging buffer
    cudaEvent_t d2h_ev[8] = {};        // chunked depth8 copy: one event per chunk
    uint32_t *iso = nullptr;           // bitmap of the degree-0 vertices and the padding (nwords)
    uint64_t *vlist = nullptr;         // n+1 (SSSP weight indexing / decode)
    float *weights = nullptr;          // m or null
    // traversal workspace
    uint32_t *vis = nullptr;           // visited bitmap (nwords)
    uint32_t *prev = nullptr;          // visited bitmap at the end of the last level
    uint32_t *tiles = nullptr;         // tile table: first chunk of each tile (max_tiles + 1)
    uint64_t max_tiles = 0;
    ChunkDesc *chunks = nullptr;       // chunk descriptors of the level (max_chunks)
    uint32_t *cvtx = nullptr;          // source vertex of each chunk (max_chunks)
    uint64_t max_chunks = 0;
    ChunkDesc *chunks_shuf = nullptr;  // frontier-order study (EFG_OPT_EXPAND_VARIANT bit 2): permuted
    uint32_t *cvtx_shuf = nullptr;     // copies of chunks / cvtx, lazily allocated
    int32_t *depth = nullptr;          // internal depth (n)
    uint32_t *parent = nullptr;        // internal parent (n), lazily allocated
    uint32_t *parent2 = nullptr;       // parent in input ids (reordered graphs), lazily
    uint32_t *old_of_new = nullptr;    // EFG_REORDER_DEGREE relabelling (n) or null
    uint32_t *new_of_old = nullptr;    // its inverse (n) or null
    int32_t *depth_st = nullptr;       // depth by stored id (relabelled graphs)
    int32_t *step_depth = nullptr;     // stepwise traversal: caller's depth buffer
    uint64_t *status = nullptr;        // frontier_kernel: 5 x [kMaxGrid] per-block aggregates + barrier counter
    BigList *big = nullptr;
    unsigned long long *trace = nullptr;  // debug: frontier_kernel phase timestamps            // frontier_kernel: multi-chunk / multi-tile lists of a level
    uint64_t max_big = 0;
    LevelStat *stats = nullptr;        // per-level statistics (kMaxLevelStats)
    unsigned frontier_blocks = 0;      // grid of frontier_kernel
    uint64_t words_per_block = 0;
    LevelCtrl *ctrl = nullptr;         // device control block
    LevelCtrl *ctrl_host = nullptr;    // pinned mirror
    float *fbuf = nullptr;             // SSSP distance (n) lazily
    double *dbuf = nullptr;            // PageRank buffers lazily (3n)
    uint64_t device_bytes = 0;
    int num_sms = 148;
    LevelStat *stats_host = nullptr;   // pinned mirror of stats
    int level_loop = 0;                // 0 = CUDA graph (device loop), 1 = host loop + events
    int prefix_skip = 1;               // EFG_OPT_PREFIX_SKIP
    int pr_pull = 1;                   // EFG_OPT_PAGERANK_PULL
    int expand_variant = 107;          // EFG_OPT_EXPAND_VARIANT (bits 0, 1, 3, 5, 6)
    static constexpr int kLoopGraphs = 3;                 // visit, visit+parent, partitioned visit
    cudaGraph_t loop_graph[kLoopGraphs] = {};
    cudaGraphExec_t loop_exec[kLoopGraphs] = {};
    uint64_t own_lo_w = 0, own_hi_w = 0;   // bitmap words of the owned rows (frontier filter)
    uint64_t *xchg_bounds = nullptr;       // device copy of the partition bounds
    uint64_t xchg_bounds_cap = 0;
    // peer-memory exchange (efg_peer_alloc / efg_peer_open / efg_xchg_peer)
    uint32_t *peer_region = nullptr;       // this rank's region (own cudaMalloc: IPC-exportable)
    uint32_t **peer_ptrs = nullptr;        // device array [peer_world] of region bases
    void *peer_ipc[64] = {};               // IPC-opened peer bases (closed on free)
    int peer_world = 0, peer_rank = -1;
    int peer_alloc_world = 0;
    // stepwise (partitioned) traversal state
    uint32_t step_levels = 0;
    uint32_t step_launches = 0;            // kernels this stepwise BFS launched (efg_stats.kernel_launches)
    uint64_t step_reached = 0, step_edges = 0;
    std::vector<uint64_t> step_lf, step_le;
};

}  // namespace efg

struct efg_graph {
    efg::HostEFG host;
    efg::DeviceGraph dev;
    bool on_device = false;
};

// device side (efg_device.cu)
namespace efg {
efg_status device_upload(efg_graph *g, const efg_build_opts &o);
void device_drop_graphs(DeviceGraph &d);  // captured level loops (rebuilt on next use)
void device_free(DeviceGraph &d);
efg_status device_decode(efg_graph *g, uint32_t v0, uint32_t v1, uint32_t *out);
efg_status device_bfs(efg_graph *g, uint32_t source, int32_t *depth, uint32_t *parent, efg_stats *st);
efg_status device_sssp(efg_graph *g, uint32_t source, float *dist, efg_stats *st);
efg_status device_pagerank(efg_graph *g, double damping, uint32_t iters, double *rank, efg_stats *st);
efg_status device_step_begin(efg_graph *g, uint32_t source, int32_t *depth);
efg_status device_step_expand(efg_graph *g);
efg_status device_step_finish(efg_graph *g, uint64_t *global_new);
efg_status device_step_end(efg_graph *g, efg_stats *st);
// op 0 = pack (out = send), 1 = reduce (in = recv, out = mine), 2 = unpack (in = gathered)
efg_status device_peer_alloc(efg_graph *g, int world, void **region, uint8_t *ipc_handle);
efg_status device_peer_open(efg_graph *g, int world, int rank, const uint64_t *bounds, const uint8_t *ipc_handles,
                            void *const *regions);
efg_status device_xchg_peer(efg_graph *g);
efg_status device_xchg_peer_phase(efg_graph *g, int phase);
void device_peer_close(DeviceGraph &d);
efg_status device_xchg(efg_graph *g, int op, int world, const uint64_t *bounds, uint64_t slice_words,
                       uint32_t *out, const uint32_t *in);
}  // namespace efg

// host widening of the compact depth transfer (efg_host_widen.cpp): dst[i] = src[i], OpenMP
namespace efg {
void host_widen_i8_i32(const int8_t *src, int32_t *dst, int64_t n);
// dst[i] = nibble i of src (8 per word, low nibble first) - 1; n vertices from a word boundary
void host_widen_u4_i32(const uint32_t *src, int32_t *dst, int64_t n);
}  // namespace efg

// error handling (efg_error.cpp)
namespace efg {
efg_status set_error(efg_status s, const std::string &msg);
void clear_error();
}  // namespace efg
