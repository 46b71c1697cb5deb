/*
 * efg.h — C ABI of the B200-native Elias-Fano graph (EFG) traversal library
 * (libefg.so).  Implements the data-parallel hot path of
 *   P. Gera, H. Kim, "Traversing Large Compressed Graphs on GPUs", IPDPS'23
 * cited as "P:<line> §<section>" against the extracted text PAPER.md, and
 * SURVEY.md §8(b) for the boundary.
 *
 * Conventions for every call
 *   - Plain C types only.  Sizes are element counts unless stated.
 *   - Every call returns efg_status; on failure efg_last_error() returns a
 *     thread-local, NUL-terminated message that stays valid until the next call
 *     on the same thread.  No call aborts, throws, or leaves a partial handle.
 *   - Output pointers marked "host or device" are classified with
 *     cudaPointerGetAttributes: device (or managed) pointers are written by the
 *     GPU in stream order, host pointers are filled by a device->host copy
 *     before the call returns.
 *   - A handle is not safe for concurrent calls from several threads; distinct
 *     handles are independent.  All GPU work of a handle is issued on the
 *     stream given at build time, and every call synchronises that stream
 *     before returning (results are complete on return) — except the
 *     enqueue-only form of efg_bfs (device outputs, st == NULL) and the
 *     partitioned step calls, which are stream-ordered (see each call).
 *   - A device-side barrier that times out (efg_bfs, the peer exchange) sets a
 *     sticky fault in the handle; every later synchronous call on it returns
 *     EFG_ECUDA.
 */
#ifndef EFG_H
#define EFG_H

#include <stddef.h>
#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

typedef enum efg_status {
    EFG_OK = 0,
    EFG_EINVAL = 1,  /* null pointer, n == 0, n > 2^32-1, bad option            */
    EFG_ERANGE = 2,  /* a vertex id >= n (input edge, source, vertex range)      */
    EFG_ENOMEM = 3,  /* host or device allocation failed                         */
    EFG_ECUDA = 4,   /* a CUDA runtime error (message in efg_last_error)         */
    EFG_ENCCL = 5,   /* a NCCL error (multi-GPU)                                 */
    EFG_ENOTSUP = 6, /* the operation is not available on this handle            */
    EFG_ESTATE = 7,  /* handle in the wrong state (e.g. host-only handle)        */
    EFG_EIO = 8      /* efg_save / efg_load: a file that cannot be written / read */
} efg_status;

/* efg_build_opts.flags (SURVEY §8(c) readings C11, C12) */
#define EFG_SYMMETRIZE 0x1u       /* add (d,s) for every input (s,d): "_sym" graphs  */
#define EFG_DEDUP 0x2u            /* keep one copy of each directed (s,d)                   */
#define EFG_DROP_SELF_LOOPS 0x4u  /* remove (v,v)                                           */
#define EFG_REORDER_DEGREE 0x8u   /* relabel vertices by degree (descending, ties by id) before
                                   * encoding: the reordering preprocessing of P:246-258 in its
                                   * simplest form.  Traversal inputs/outputs (source, depth,
                                   * parent, dist, rank) stay in INPUT ids; efg_export and
                                   * efg_decode describe the relabelled graph, whose relabelling
                                   * efg_export_perm returns. */
#define EFG_HOST_RESIDENT 0x10u   /* out-of-core EFG (§I, §VIII-B): the EF
                                   * `data` array stays in pinned host memory mapped into
                                   * the device's address space; the traversal kernels stage it
                                   * over the host link (zero-copy) while the vertex records,
                                   * bitmaps and work plan stay in HBM.  Without this flag the
                                   * same happens automatically when `data` does not fit the
                                   * device's free memory (efg_info_t.data_location). */
#define EFG_DEFAULT_FLAGS (EFG_SYMMETRIZE | EFG_DEDUP | EFG_DROP_SELF_LOOPS)

typedef struct efg_graph efg_graph; /* opaque: host EFG arrays + device copy */

typedef struct efg_build_opts {
    /* Forward-pointer quantum k (§VI-C; k = 512 in the paper's
     * experiments).  0 disables forward pointers.  Default 512.  Any k
     * is accepted: the host arrays (efg_export) use k; the device copy splits
     * lists into k-element chunks when 1 <= k <= 512 and every list has fewer
     * than 2^18 chunks, else it re-samples the pointers every 512 elements
     * (efg_info_t.device_quantum).  Results do not depend on k. */
    uint32_t fwd_quantum;
    /* EFG_* flags above.  Default EFG_DEFAULT_FLAGS. */
    uint32_t flags;
    /* CUDA device ordinal for the device copy; -1 = host-only handle (builder
     * output only: efg_info / efg_export work, traversals return EFG_ESTATE). */
    int32_t device;
    /* Host threads for the builder; 0 = OpenMP default. */
    uint32_t n_threads;
    /* cudaStream_t for all device work of this handle; NULL = legacy default. */
    void *stream;
    /* Optional per-input-edge fp32 weights (SSSP; uncompressed).
     * NULL = unweighted.  Weights of duplicate (s,d) pairs: the minimum is kept.
     * With EFG_SYMMETRIZE the reverse edge gets the same weight. */
    const float *weights;
    /* 1-D row partition: when row_hi > row_lo this handle encodes
     * and uploads only the lists of rows [row_lo, row_hi) (e.g. a range from
     * efg_partition); all other vertices keep empty lists.  Every rank passes
     * the same edge list.  0, 0 = the whole graph. */
    uint64_t row_lo, row_hi;
} efg_build_opts;

/* Fill *o with the defaults above (k = 512, EFG_DEFAULT_FLAGS, device 0). */
void efg_default_opts(efg_build_opts *o);

/*
 * efg_build — edge list -> CSR -> EFG (§III-D, §V).
 *   n           number of vertices, 1 <= n <= 2^32-1; ids are 0..n-1
 *   m           number of input edges
 *   src, dst    host arrays of m vertex ids (caller-owned, read-only; they may
 *               be freed after the call returns)
 *   opts        NULL = defaults
 *   out         receives the new handle (NULL on failure)
 * Each vertex's neighbour list is sorted ascending, de-duplicated and
 * stripped of self-loops per flags, then Elias-Fano encoded per P:81-96 with
 * l = max{0, floor(log2(u/n))}, u = the list's last element (readings C1-C3),
 * laid out as [forward pointers (uint32 LE)][lower bits][upper bits], each
 * section byte-aligned, LSB-first within bytes (readings C6-C8).  The four
 * arrays of P:113 (vlist, num_lower_bits, offsets, data) stay on the host
 * (efg_export) and, if opts->device >= 0, are uploaded in a packed device
 * layout.
 * Errors: EFG_EINVAL (null pointers, n == 0, n > 2^32-1), EFG_ERANGE (an id >=
 * n), EFG_ENOMEM, EFG_ECUDA.
 */
efg_status efg_build(uint64_t n, uint64_t m, const uint32_t *src, const uint32_t *dst,
                     const efg_build_opts *opts, efg_graph **out);

/*
 * efg_build_stream — efg_build over edges produced on demand instead of held in
 * caller arrays (a rank builds only its rows of a graph larger
 * than host memory allows as an edge list, e.g. RMAT-29/ef32, BASELINE
 * configs[4]).
 *   gen(user, first, count, src, dst, w) must write samples [first, first +
 *   count) of the edge list into src[0..count), dst[0..count) and, when
 *   `weighted` != 0, w[0..count) (else w is NULL).  It is called from one
 *   thread at a time, chunk by chunk in increasing `first`, TWICE over [0, m)
 *   (a counting pass, then a scatter pass), and must return the same samples
 *   both times (e.g. a counter-based generator).  Its buffers belong to the
 *   library and are only valid during the call.
 *   n, opts, out: as efg_build (opts->weights is ignored; weights come from gen).
 * Memory: the builder holds the adjacency of the materialised rows only — the
 * owned rows of a row-range handle (row_lo/row_hi) without EFG_REORDER_DEGREE;
 * every row otherwise (the relabelling needs every degree) — never the edge
 * list: 4 bytes per directed entry (8 when weighted) plus the EFG.
 * The result equals efg_build on the concatenated samples.
 * Errors: as efg_build.
 */
typedef void (*efg_edge_gen_fn)(void *user, uint64_t first, uint64_t count, uint32_t *src, uint32_t *dst,
                                float *w);
efg_status efg_build_stream(uint64_t n, uint64_t m, efg_edge_gen_fn gen, void *user, int weighted,
                            const efg_build_opts *opts, efg_graph **out);

/*
 * efg_save / efg_load — the on-disk EFG: a built graph written once and loaded
 * without rebuilding (the builder's minutes on C3-C5 become a file read).
 * The file holds a fixed header (magic "EFGRAPH1", version, n, m, k, row
 * range, section byte totals, the length of every array) followed by the
 * P:113 arrays vlist (u64[n+1]), num_lower_bits (u8[n]), offsets (u64[n+1]),
 * data (u8[offsets[n]]), then the builder's derived arrays: largest neighbour
 * (u32[n]), in-edge flags (u8[n]), the EFG_REORDER_DEGREE relabelling
 * (u32[n] twice, or absent) and the CSR-order weights (f32[m], or absent).
 * Native byte order (little-endian on every supported host).
 *   efg_save: g may be host-only or on a device; the host arrays are written.
 *   efg_load: opts->device / stream / flags & EFG_HOST_RESIDENT apply as in
 *     efg_build (NULL: defaults, device 0); the other options are the file's.
 *     The loaded handle equals the saved one (efg_export, efg_export_perm,
 *     every traversal).
 * Errors: EFG_EINVAL (null argument), EFG_EIO (open / write / read failure,
 * not an EFG file, other version, inconsistent header, truncated file), then
 * as efg_build for the upload.
 */
efg_status efg_save(const efg_graph *g, const char *path);
efg_status efg_load(const char *path, const efg_build_opts *opts, efg_graph **out);

/* Release everything the handle owns (host and device).  NULL-safe. */
void efg_free(efg_graph *g);

typedef struct efg_info_t {
    uint64_t n;              /* vertices                                           */
    uint64_t m;              /* directed edges after symmetrise/dedup (= vlist[n]) */
    uint64_t m_input;        /* input edges as given                               */
    uint32_t fwd_quantum;    /* k                                                  */
    uint32_t device;         /* CUDA ordinal, or 0xFFFFFFFF for host-only          */
    uint64_t data_bytes;     /* sum of per-vertex sizes = offsets[n]               */
    uint64_t fwd_bytes;      /* forward-pointer sections                           */
    uint64_t lower_bytes;    /* lower-bits sections                                */
    uint64_t upper_bytes;    /* upper-bits sections                                */
    uint64_t apriori_bits;   /* sum over lists of n*l + n + (u >> l)  */
    uint64_t vertex_bytes;   /* host vertex arrays: vlist 8 + offsets 8 + nlb 1     */
    uint64_t device_bytes;   /* device memory held by the handle                   */
    uint64_t row_lo, row_hi; /* owned row range (whole graph: 0, n)                */
    double build_seconds;    /* host builder wall time                             */
    uint32_t device_quantum; /* chunk length of the device copy: fwd_quantum when  *
                              * 1 <= k <= 512 and ceil(deg/k) < 2^18 for every    *
                              * list, else 512 (the device copy's forward         *
                              * pointers are re-sampled; the host arrays keep k)  */
    uint32_t data_location;  /* 0: EF data in device memory (HBM); 1: pinned host  *
                              * memory mapped into the device (out-of-core)       */
} efg_info_t;

efg_status efg_info(const efg_graph *g, efg_info_t *info);

/* Copy the P:113 arrays to caller-owned host buffers (any may be NULL):
 * vlist[n+1] (uint64), num_lower_bits[n] (uint8), offsets[n+1] (uint64),
 * data[offsets[n]] (uint8).  For a partitioned handle these describe the
 * owned row range (vertices outside it have empty lists). */
efg_status efg_export(const efg_graph *g, uint64_t *vlist, uint8_t *num_lower_bits,
                      uint64_t *offsets, uint8_t *data);

/* Copy the relabelling of an EFG_REORDER_DEGREE handle: old_of_new[i] = input id
 * of stored vertex i (n entries, caller-owned host buffer).  Without the flag
 * the identity is written. */
efg_status efg_export_perm(const efg_graph *g, uint32_t *old_of_new);

/*
 * efg_decode — GPU decode of the neighbour lists of vertices [v0, v1) into
 * CSR order: out[vlist[v] - vlist[v0] + i] = x_i of v (§IV-A), using
 * the same frontier/partition/decode kernels as efg_bfs (the BFS visit step is
 * replaced by a store).  out: host or device, vlist[v1]-vlist[v0] entries.
 * Errors: EFG_ERANGE (v0 > v1 or v1 > n), EFG_ESTATE (host-only handle).
 */
efg_status efg_decode(efg_graph *g, uint32_t v0, uint32_t v1, uint32_t *out);

/* Per-call statistics (all fields except level_cap / arrays are outputs). */
typedef struct efg_stats {
    uint32_t levels;           /* BFS levels expanded (frontiers processed)          */
    uint32_t level_cap;        /* in: capacity of the per-level arrays (0 = none)    */
    uint64_t edges_traversed;  /* sum of deg(f) over every expanded frontier vertex  */
    uint64_t vertices_reached; /* vertices with depth >= 0                           */
    float device_ms;           /* device time of the traversal (CUDA events)         */
    float expand_ms;           /* device time inside the expand+decode kernel        */
    uint32_t expand_launches;  /* number of expand+decode launches                   */
    uint32_t kernel_launches;  /* all kernels launched by the call                   */
    uint64_t expand_bytes;     /* reserved, 0 (bench.py derives the algorithmic     *
                                *  bytes from efg_export sizes and the levels)      */
    uint64_t *level_frontier;  /* in/out: |F_L| per level (level_cap entries)        */
    uint64_t *level_edges;     /* in/out: E_L = sum of frontier degrees per level    */
    float *level_expand_ms;    /* in/out: expand kernel time per level, or NULL      */
    float *level_end_ms;       /* in/out: level-end + plan kernel time per level     *
                                *         (host loop only, CUDA events), or NULL     */
    uint64_t d2h_bytes;        /* out: device->host bytes the call moved for host    *
                                *       outputs (a host depth array travels as one   *
                                *       byte per vertex when every depth < 127)      */
    uint32_t xchg_sparse_levels; /* out (partitioned BFS over the peer exchange):    *
                                  *  levels whose exchange took the sparse path      */
} efg_stats;

/*
 * efg_bfs — level-synchronous top-down BFS from `source` over the compressed
 * graph (Alg. 1; frontier partition P:125-135; in-kernel decode
 * P:137-177).  depth[v] = hop distance from source, -1 if unreachable
 * (reading C15).  parent (nullable): some neighbour u with depth[u] ==
 * depth[v]-1 (any valid one, reading C28); parent[source] = source; unreached
 * 0xFFFFFFFF.  depth / parent: host or device, n entries, caller-allocated.
 * Partitioned handle (row_lo/row_hi): the call is COLLECTIVE
 * over the peer exchange opened with efg_peer_alloc / efg_peer_open — every
 * rank calls it with the same source; each level expands the rank's own rows,
 * ORs the new bits over peer memory (efg_xchg_peer) and ends the level over
 * the now-global bitmap, so every rank receives the full depth array.  The
 * loop ends on the device when the global new count is 0 (identical on every
 * rank).  Without an open peer exchange it returns EFG_ESTATE (drive the
 * levels with efg_bfs_begin / expand / xchg_* / finish_level instead);
 * parent != NULL returns EFG_ENOTSUP.  st then counts this rank's rows.
 * Completion: with device outputs (depth and parent, if any) and st == NULL
 * the call only enqueues the BFS on the handle's stream (efg_build_opts
 * stream) and returns; the outputs are valid once that stream is
 * synchronised (stream order, as cudaMemcpyAsync).  A barrier time-out in
 * that form is reported by the next synchronous call.  Otherwise it returns
 * with the outputs written.
 * Errors: EFG_ERANGE (source >= n), EFG_ESTATE, EFG_ENOTSUP, EFG_ECUDA.
 */
efg_status efg_bfs(efg_graph *g, uint32_t source, int32_t *depth, uint32_t *parent,
                   efg_stats *st);

/*
 * efg_sssp — single-source shortest paths with the build-time weights (P:185
 * §VI-F): frontier Bellman-Ford, relaxed vertices marked in a bitmap, fp32
 * distances with single-rounding adds (dist[u] + w, no contraction; reading
 * C20).  dist: host or device, n entries; unreached = +inf.
 * Errors: EFG_EINVAL (graph built without weights), EFG_ERANGE, EFG_ESTATE,
 * EFG_ENOTSUP (partitioned handle).
 */
efg_status efg_sssp(efg_graph *g, uint32_t source, float *dist, efg_stats *st);

/*
 * efg_pagerank — PageRank over the compressed graph (§VI-F; capped at
 * `iters` iterations, 50 in the paper P:201).  Reading C21: r0 = 1/N,
 * r' = (1-d)/N + d*(sum_{u in N(v)} r(u)/deg(u) + D/N), D = rank mass on
 * degree-0 vertices, exactly `iters` iterations, fp64 accumulation.
 * rank: host or device, n doubles.
 * Errors: EFG_EINVAL, EFG_ESTATE, EFG_ENOTSUP (partitioned handle).
 */
efg_status efg_pagerank(efg_graph *g, double damping, uint32_t iters, double *rank,
                        efg_stats *st);

/* Options (efg_set_option). */
#define EFG_OPT_LEVEL_LOOP 1 /* 0 (default): the BFS level loop runs on the device as one
                              * CUDA graph with a conditional WHILE node (no host round trip
                              * per level); 1: host-driven loop that reads the frontier size
                              * each level and times every expand launch with CUDA events. */
#define EFG_OPT_PREFIX_SKIP 2 /* 1 (default): BFS expand drops upper-bit words whose elements
                               * are all below the visited prefix vpre (every id < vpre is
                               * visited or has no in-edge; lists are sorted, so such words
                               * form a prefix of each list): those ids are neither decoded
                               * nor probed; their bytes are still staged.  0: every element
                               * is decoded and probed (the paper's expansion, Alg. 1).
                               * Results are identical either way. */
#define EFG_OPT_PAGERANK_PULL 3 /* 1 (default): efg_pagerank on a symmetric whole-graph handle
                                 * gathers r(u)/deg(u) over each vertex's own list (one fp64
                                 * atomic per list run instead of one per edge); 0 (and every
                                 * directed or row-range handle): push along every edge with
                                 * fp64 atomicAdd.  Same sums, other order (C21). */

#define EFG_OPT_EXPAND_VARIANT 4 /* tuning / A-B switch of the expand kernel, bit mask (default 107):
                                  * bit 0: batches of balanced chunks are decoded lane-per-chunk
                                  * (each lane walks its own chunk) instead of by word records
                                  * split evenly over the lanes; bit 1: a batch of adjacent chunks
                                  * is staged by one bulk copy of its byte span; bit 2: frontier-
                                  * order study — BFS expands each level's chunks in
                                  * a pseudo-random ("arbitrary") order instead of the bitmap's
                                  * id order; bit 3: a lane-per-chunk lane steps over the stop
                                  * bits below the visited prefix inside its first kept word
                                  * (select0) instead of decoding them; bit 4: tiles are dealt
                                  * to the warps in super-tiles of consecutive tiles; bit 5: the
                                  * level-end list skip uses the visited prefix of the level just
                                  * expanded (one more grid barrier) instead of the previous one;
                                  * bit 6: on skip levels (visited prefix >= n/3) a batch goes
                                  * lane-per-chunk from 25 % busy element slots instead of 50 %.
                                  * Values 0..127.  Results are identical for every value. */

/* Set a per-handle option.  Errors: EFG_EINVAL (unknown option / value),
 * EFG_ESTATE (host-only handle). */
efg_status efg_set_option(efg_graph *g, int option, int64_t value);

/* ---- multi-GPU: 1-D row partition, per-level exchange ----
 *
 * One process per GPU; rank r's handle holds rows [bounds[r], bounds[r+1]).
 * A partitioned BFS is driven level by level (all ranks in lock step):
 *   efg_bfs_begin                 source, level 0
 *   repeat:
 *     efg_bfs_expand              decode + visit the rank's own frontier rows
 *                                 (discoveries land in the rank's full-width
 *                                 visited bitmap)
 *     efg_xchg_pack               slice h of this rank's new bits -> send[h*S ..]
 *     (caller) all-to-all         send -> recv   (e.g. torch.distributed over NCCL)
 *     efg_xchg_reduce             OR of the P received slices -> mine[0..S)
 *     (caller) all-gather         mine -> gathered[P*S]
 *     efg_xchg_unpack             visited |= gathered (same global bitmap on all ranks)
 *     efg_bfs_finish_level        next frontier = new owned vertices, depth of all
 *                                 new vertices; returns the GLOBAL new count
 *   until the global new count is 0;  efg_bfs_end.
 * The library provides every computation; the caller only moves bytes.  S =
 * slice length in 32-bit words (the largest owner range, see efg_xchg_geometry).
 * All buffers are device pointers on the handle's device; calls are ordered on
 * the handle's stream (efg_bfs_finish_level synchronises it).
 */

/* bounds[world+1] vertex boundaries (multiples of 64, bounds[world] = n).
 * Writes the slice length S in 32-bit words (max over ranks). */
efg_status efg_xchg_geometry(const efg_graph *g, int world, const uint64_t *bounds, uint64_t *slice_words);

efg_status efg_bfs_begin(efg_graph *g, uint32_t source, int32_t *depth_device);
efg_status efg_bfs_expand(efg_graph *g);
efg_status efg_xchg_pack(efg_graph *g, int world, const uint64_t *bounds, uint64_t slice_words,
                         uint32_t *send);
efg_status efg_xchg_reduce(efg_graph *g, int world, uint64_t slice_words, const uint32_t *recv,
                           uint32_t *mine);
efg_status efg_xchg_unpack(efg_graph *g, int world, const uint64_t *bounds, uint64_t slice_words,
                           const uint32_t *gathered);
efg_status efg_bfs_finish_level(efg_graph *g, uint64_t *global_new);
efg_status efg_bfs_end(efg_graph *g, efg_stats *st);

/* ---- multi-GPU exchange over peer memory (NVLink / NVSwitch), no NCCL ----
 *
 * The same per-level exchange as pack / all-to-all / reduce / all-gather /
 * unpack (owners OR the P ranks' new bits of their rows, every
 * rank receives the OR of every owner), done by the library's kernels reading
 * and writing the other ranks' HBM directly.  Level loop:
 *   efg_bfs_expand; efg_xchg_peer; efg_bfs_finish_level
 * Setup, once per handle and partition (collective: every rank, same world):
 *   efg_peer_alloc   allocates this rank's exchange region (cudaMalloc, 4 *
 *                    (96 + 2 * W + 2 * (W / 32 + 32)) bytes with W =
 *                    ceil32(ceil(n/32)), owned by the handle, zeroed) and
 *                    returns its device address and its 64-byte CUDA IPC
 *                    handle; either may be NULL.
 *   (caller)         all-gathers the handles (e.g. torch.distributed) — or, for
 *                    several handles on one device in one process, the addresses.
 *   efg_peer_open    maps the other ranks' regions: ipc_handles = world * 64
 *                    bytes (rank order; cudaIpcOpenMemHandle with lazy peer
 *                    access), or regions = world device addresses (same
 *                    process); exactly one of the two is non-NULL.  bounds as in
 *                    efg_xchg_geometry (bounds[0] = 0, bounds[world] = n).
 *   efg_xchg_peer    enqueues the exchange on the handle's stream (five
 *                    kernels: publish, barrier, owner OR + broadcast, barrier,
 *                    unpack; the cross-rank barriers over flags in the regions
 *                    spin in one block each) and returns.  Every rank must call
 *                    it once per level.  Sparse levels: when no
 *                    rank has more than W/32 + 32 non-zero words of new bits,
 *                    every rank ORs the others' published (word, bits) lists
 *                    into its bitmap instead (no owner step, traffic in
 *                    proportion to the discoveries); all ranks take the same
 *                    decision from the published counts.
 *   efg_xchg_peer_phase  the same exchange without the device barriers, one
 *                    phase per call (0 publish, 1 owner OR + broadcast, 2
 *                    unpack), each synchronising the handle's stream before it
 *                    returns: the CALLER orders the phases across ranks with a
 *                    host barrier after every phase (no kernel waits for
 *                    another rank — the form for ranks time-sharing one GPU,
 *                    whose cross-rank spinning kernels nothing schedules
 *                    together).  Errors as efg_xchg_peer, EFG_EINVAL for a bad
 *                    phase.
 * Ranks that share one device must use distinct non-blocking streams (the
 * barrier kernels of one rank wait for the others' kernels).  A barrier that
 * waits more than 4 s gives up; the next efg_bfs_finish_level then returns
 * EFG_ECUDA.  efg_free unmaps and frees everything.
 * Errors: EFG_EINVAL (bad world / rank / bounds / pointers), EFG_ESTATE (open
 * before alloc, exchange before open, host-only handle), EFG_ECUDA.
 */
#define EFG_IPC_HANDLE_BYTES 64
efg_status efg_peer_alloc(efg_graph *g, int world, void **region, uint8_t *ipc_handle);
efg_status efg_peer_open(efg_graph *g, int world, int rank, const uint64_t *bounds, const uint8_t *ipc_handles,
                         void *const *regions);
efg_status efg_xchg_peer(efg_graph *g);
efg_status efg_xchg_peer_phase(efg_graph *g, int phase);

/*
 * efg_partition — the 1-D row partition (efg_build_opts.row_lo / row_hi):
 * rank r owns vertices [bounds[r], bounds[r+1]).  Boundaries balance
 * sum(offsets bytes) + 29 bytes per vertex and are multiples
 * of 64 (so bitmap words have one owner).  bounds: world+1 entries.
 * Host-only computation over the P:113 vlist/offsets arrays of the whole graph.
 */
efg_status efg_partition(uint64_t n, const uint64_t *vlist, const uint64_t *offsets, int world,
                         uint64_t *bounds);

/* Thread-local message for the last failing call on this thread ("" if none). */
const char *efg_last_error(void);

/* Library version string. */
const char *efg_version(void);

#ifdef __cplusplus
}
#endif
#endif /* EFG_H */
