/*
 * oracle/oracle.c — TEST INFRASTRUCTURE ONLY.
 *
 * A plain, slow, single-threaded CPU implementation of what the EFG hot path
 * computes, written from PAPER.md (Gera & Kim, "Traversing Large Compressed
 * Graphs on GPUs", IPDPS'23).  Citations are "P:<line> §<section>".
 *
 * Only tests/, __graft_entry__.smoke() and bench.py's cpu_baseline / reference
 * leg may load this library.  It shares no code, header, table or constant with
 * the product (paper_conf_ipps_gerak23_b200/) and never calls it.
 *
 * Contents (each function cites the passage it follows):
 *   or_csr_*        CSR construction (§III-D) with the DESIGN.md readings
 *                   C11 (drop duplicates and self-loops) and C12 (symmetrise).
 *   or_bfs          BFS depth by its plain definition: FIFO queue BFS
 *                   (Alg. 1 semantics, §III-B).  depth = hop distance.
 *   or_bfs_bounded  the same BFS stopped after a budget of scanned edges
 *                   (bench.py reference arm: a bounded sample per step).
 *   or_ef_*         Elias-Fano list encoding / naive decoding (§IV,
 *                   Fig. 2, forward pointers P:157 §VI-C, EFG layout
 *                   P:111-117 §V), step by step in the order of SURVEY §8(c).
 *   or_efg_*        whole-graph EFG arrays vlist/num_lower_bits/offsets/data
 *                   (P:113).
 *   or_maxle        binsearch_maxle (§III-C, Fig. 4) written as a
 *                   linear scan: index of the largest value <= key, last of ties.
 *   or_sssp         fp32 Dijkstra (binary heap) for SSSP (§VI-F).
 *   or_pagerank     fp64 power iteration for PageRank (P:185, 50 its P:201).
 *
 * Every function here is pinned by tests in tests/test_oracle_*.py against the
 * paper's worked examples (Figs. 2-6), closed forms and brute force.
 */
#include <stdint.h>
#include <stdlib.h>
#include <string.h>
#include <math.h>

/* ------------------------------------------------------------------------- */
/* CSR (§III-D): vlist[|V|+1] row offsets, elist[|E|] column indices. */
/* ------------------------------------------------------------------------- */

typedef struct {
    uint64_t n, m;
    uint64_t *vlist;
    uint32_t *elist;
} or_csr;

static int cmp_u32(const void *a, const void *b)
{
    uint32_t x = *(const uint32_t *)a, y = *(const uint32_t *)b;
    return (x > y) - (x < y);
}

/* Build a CSR from an edge list.
 * symmetrize (C12): the directed multiset contains (s,d) and (d,s).
 * drop_self  (C11): remove (v,v).   dedup (C11): keep one copy of each (s,d).
 * Neighbour lists are sorted ascending (EF needs sorted lists).
 * Returns NULL if an id is >= n or on allocation failure. */
or_csr *or_csr_build(uint64_t n, uint64_t m_in, const uint32_t *src, const uint32_t *dst,
                     int symmetrize, int dedup, int drop_self)
{
    for (uint64_t e = 0; e < m_in; ++e)
        if (src[e] >= n || dst[e] >= n) return NULL;

    or_csr *g = (or_csr *)calloc(1, sizeof(or_csr));
    if (!g) return NULL;
    g->n = n;
    uint64_t *cnt = (uint64_t *)calloc(n + 1, sizeof(uint64_t));
    if (!cnt) { free(g); return NULL; }

    /* count out-degree of the directed multiset */
    for (uint64_t e = 0; e < m_in; ++e) {
        cnt[src[e]]++;
        if (symmetrize) cnt[dst[e]]++;
    }
    uint64_t *start = (uint64_t *)malloc((n + 1) * sizeof(uint64_t));
    if (!start) { free(cnt); free(g); return NULL; }
    start[0] = 0;
    for (uint64_t v = 0; v < n; ++v) start[v + 1] = start[v] + cnt[v];
    uint64_t total = start[n];
    uint32_t *tmp = (uint32_t *)malloc((total ? total : 1) * sizeof(uint32_t));
    if (!tmp) { free(start); free(cnt); free(g); return NULL; }

    /* bucket by source (counting sort) */
    for (uint64_t v = 0; v < n; ++v) cnt[v] = start[v];
    for (uint64_t e = 0; e < m_in; ++e) {
        tmp[cnt[src[e]]++] = dst[e];
        if (symmetrize) tmp[cnt[dst[e]]++] = src[e];
    }

    /* sort each list, then drop self-loops and duplicates, compacting in place */
    g->vlist = (uint64_t *)malloc((n + 1) * sizeof(uint64_t));
    if (!g->vlist) { free(tmp); free(start); free(cnt); free(g); return NULL; }
    uint64_t w = 0;
    g->vlist[0] = 0;
    for (uint64_t v = 0; v < n; ++v) {
        uint64_t a = start[v], b = start[v + 1];
        qsort(tmp + a, (size_t)(b - a), sizeof(uint32_t), cmp_u32);
        for (uint64_t i = a; i < b; ++i) {
            uint32_t x = tmp[i];
            if (drop_self && x == (uint32_t)v) continue;
            if (dedup && w > g->vlist[v] && tmp[w - 1] == x) continue;
            tmp[w++] = x;
        }
        g->vlist[v + 1] = w;
    }
    g->m = w;
    g->elist = (uint32_t *)realloc(tmp, (w ? w : 1) * sizeof(uint32_t));
    if (!g->elist) g->elist = tmp;
    free(start);
    free(cnt);
    return g;
}

uint64_t or_csr_n(const or_csr *g) { return g->n; }
uint64_t or_csr_m(const or_csr *g) { return g->m; }
const uint64_t *or_csr_vlist(const or_csr *g) { return g->vlist; }
const uint32_t *or_csr_elist(const or_csr *g) { return g->elist; }

void or_csr_free(or_csr *g)
{
    if (!g) return;
    free(g->vlist);
    free(g->elist);
    free(g);
}

/* ------------------------------------------------------------------------- */
/* BFS depth, plain definition (Alg. 1; output reading C15):         */
/* depth[v] = number of edges on a shortest path source -> v, -1 unreached.  */
/* Single-threaded FIFO queue.  Returns the number of reached vertices.      */
/* ------------------------------------------------------------------------- */
uint64_t or_bfs(uint64_t n, const uint64_t *vlist, const uint32_t *elist, uint32_t source,
                int32_t *depth)
{
    for (uint64_t v = 0; v < n; ++v) depth[v] = -1;
    if (source >= n) return 0;
    uint32_t *q = (uint32_t *)malloc((n ? n : 1) * sizeof(uint32_t));
    if (!q) return 0;
    uint64_t head = 0, tail = 0;
    depth[source] = 0;
    q[tail++] = source;
    while (head < tail) {
        uint32_t u = q[head++];
        for (uint64_t e = vlist[u]; e < vlist[u + 1]; ++e) {
            uint32_t v = elist[e];
            if (depth[v] < 0) {
                depth[v] = depth[u] + 1;
                q[tail++] = v;
            }
        }
    }
    free(q);
    return tail;
}

/* Bounded sample of the same FIFO BFS (bench.py reference arm only: a timed
 * step must stay within seconds on the largest configs).  Identical to or_bfs
 * except that it stops dequeuing once the adjacency entries scanned reach
 * max_edges (the current vertex's list is always finished).  Every depth it
 * assigns is final (a FIFO BFS assigns a vertex's depth once, at discovery),
 * so depth[] is or_bfs's depth on the discovered vertices and -1 elsewhere.
 * *edges_scanned = adjacency entries scanned (= sum of the degrees of the
 * dequeued vertices).  Returns the number of dequeued vertices. */
uint64_t or_bfs_bounded(uint64_t n, const uint64_t *vlist, const uint32_t *elist, uint32_t source,
                        int32_t *depth, uint64_t max_edges, uint64_t *edges_scanned)
{
    for (uint64_t v = 0; v < n; ++v) depth[v] = -1;
    *edges_scanned = 0;
    if (source >= n) return 0;
    uint32_t *q = (uint32_t *)malloc((n ? n : 1) * sizeof(uint32_t));
    if (!q) return 0;
    uint64_t head = 0, tail = 0, scanned = 0;
    depth[source] = 0;
    q[tail++] = source;
    while (head < tail && scanned < max_edges) {
        uint32_t u = q[head++];
        for (uint64_t e = vlist[u]; e < vlist[u + 1]; ++e) {
            uint32_t v = elist[e];
            if (depth[v] < 0) {
                depth[v] = depth[u] + 1;
                q[tail++] = v;
            }
        }
        scanned += vlist[u + 1] - vlist[u];
    }
    free(q);
    *edges_scanned = scanned;
    return head;
}

/* ------------------------------------------------------------------------- */
/* Elias-Fano list encoding (§IV; layout P:113-115 §V; forward        */
/* pointers P:157 §VI-C).  Steps follow SURVEY §8(c) "EFG encoding, step by   */
/* step" with readings C1-C10.                          */
/* ------------------------------------------------------------------------- */

/* Step 2: l = max{0, floor(log2(u/n))} (C1 log base 2, C2 u = last
 * element, C3 integer division).  Computed by repeated doubling so that no
 * floating point enters an integer decision. */
uint32_t or_ef_lower_bits(uint64_t n, uint64_t u)
{
    if (n == 0) return 0;
    uint64_t q = u / n;           /* floor(u/n); floor(log2(u/n)) = floor(log2(floor(u/n))) */
    if (q == 0) return 0;         /* u < n */
    uint32_t l = 0;
    while ((q >> 1) != 0) { q >>= 1; ++l; }
    return l;
}

/* Section sizes in bytes (C7: [fwd][lower][upper], each byte aligned).
 *   fwd   = 4 * floor(n/k)                (C8, uint32 pointers; k = 0 -> none)
 *   lower = ceil(n*l / 8)
 *   upper = ceil(((u >> l) + n) / 8)      (C4; n stop bits + (u>>l) zeros)  */
void or_ef_sections(uint64_t n, uint64_t u, uint32_t k, uint64_t *fwd_bytes,
                    uint64_t *lower_bytes, uint64_t *upper_bytes)
{
    uint32_t l = or_ef_lower_bits(n, u);
    *fwd_bytes = (n && k) ? 4 * (n / k) : 0;
    *lower_bytes = n ? (n * l + 7) / 8 : 0;
    *upper_bytes = n ? (((u >> l) + n) + 7) / 8 : 0;
}

static inline void set_bit(uint8_t *p, uint64_t q) { p[q >> 3] |= (uint8_t)(1u << (q & 7)); }
static inline int get_bit(const uint8_t *p, uint64_t q) { return (p[q >> 3] >> (q & 7)) & 1; }

/* Encode one sorted list x[0..n-1] into out (zeroed by this function).
 * Returns the byte size S = fwd + lower + upper and writes l. */
uint64_t or_ef_encode_list(const uint32_t *x, uint64_t n, uint32_t k, uint8_t *out, uint32_t *l_out)
{
    if (n == 0) { *l_out = 0; return 0; }                     /* step 1 (C10) */
    uint64_t u = x[n - 1];                                     /* step 2 (C2) */
    uint32_t l = or_ef_lower_bits(n, u);
    uint64_t fb, lb, ub;
    or_ef_sections(n, u, k, &fb, &lb, &ub);
    memset(out, 0, (size_t)(fb + lb + ub));
    /* step 3: forward pointers fwd[j] = x[(j+1)k-1] >> l  (= select1(i) - i) */
    if (k) {
        for (uint64_t j = 0; j < n / k; ++j) {
            uint32_t f = (uint32_t)(x[(j + 1) * k - 1] >> l);
            out[4 * j + 0] = (uint8_t)(f);
            out[4 * j + 1] = (uint8_t)(f >> 8);
            out[4 * j + 2] = (uint8_t)(f >> 16);
            out[4 * j + 3] = (uint8_t)(f >> 24);
        }
    }
    /* step 4: lower bits of x[i] at bit offset i*l, LSB first (C6) */
    uint8_t *lower = out + fb;
    for (uint64_t i = 0; i < n; ++i)
        for (uint32_t b = 0; b < l; ++b)
            if ((x[i] >> b) & 1u) set_bit(lower, i * l + b);
    /* step 5: upper bits — unary gaps with a 1 stop bit: bit (x[i]>>l) + i */
    uint8_t *upper = lower + lb;
    for (uint64_t i = 0; i < n; ++i) set_bit(upper, (x[i] >> l) + i);
    *l_out = l;
    return fb + lb + ub;                                       /* step 6 */
}

/* select_1(i): position of the i-th (0-indexed) set bit of the upper-bits
 * array, found by walking bits from position 0 (§IV-A definition). */
uint64_t or_ef_select1(const uint8_t *enc, uint64_t n, uint32_t l, uint32_t k, uint64_t i)
{
    uint64_t fb = k ? 4 * (n / k) : 0;
    const uint8_t *upper = enc + fb + (n * l + 7) / 8;
    uint64_t seen = 0;
    for (uint64_t pos = 0;; ++pos) {
        if (get_bit(upper, pos)) {
            if (seen == i) return pos;
            ++seen;
        }
    }
}

/* Naive decode (§IV-A): x_i = ((select_1(i) - i) << l) | lower[i].
 * One left-to-right walk of the upper bits yields select_1(0), select_1(1), ...
 * in order; lower[i] is read bit by bit at offset i*l. */
void or_ef_decode_list(const uint8_t *enc, uint64_t n, uint32_t l, uint32_t k, uint32_t *out)
{
    uint64_t fb = k ? 4 * (n / k) : 0;
    const uint8_t *lower = enc + fb;
    const uint8_t *upper = lower + (n * l + 7) / 8;
    uint64_t i = 0;
    for (uint64_t pos = 0; i < n; ++pos) {
        if (!get_bit(upper, pos)) continue;
        uint64_t hi = pos - i;                    /* select_1(i) - i */
        uint64_t lo = 0;
        for (uint32_t b = 0; b < l; ++b) lo |= (uint64_t)get_bit(lower, i * l + b) << b;
        out[i] = (uint32_t)((hi << l) | lo);
        ++i;
    }
}

/* Read forward pointer j (uint32 little endian, C8). */
uint32_t or_ef_fwd(const uint8_t *enc, uint64_t j)
{
    return (uint32_t)enc[4 * j] | ((uint32_t)enc[4 * j + 1] << 8) |
           ((uint32_t)enc[4 * j + 2] << 16) | ((uint32_t)enc[4 * j + 3] << 24);
}

/* ------------------------------------------------------------------------- */
/* Whole-graph EFG arrays (§V): vlist (= CSR vlist), num_lower_bits,    */
/* offsets = exclusive prefix sum of per-vertex byte sizes, data.             */
/* ------------------------------------------------------------------------- */

/* offsets[0..n] and the total data size; data itself by or_efg_encode. */
uint64_t or_efg_offsets(uint64_t n, const uint64_t *vlist, const uint32_t *elist, uint32_t k,
                        uint64_t *offsets)
{
    offsets[0] = 0;
    for (uint64_t v = 0; v < n; ++v) {
        uint64_t deg = vlist[v + 1] - vlist[v];
        uint64_t s = 0;
        if (deg) {
            uint64_t fb, lb, ub;
            or_ef_sections(deg, elist[vlist[v + 1] - 1], k, &fb, &lb, &ub);
            s = fb + lb + ub;
        }
        offsets[v + 1] = offsets[v] + s;                      /* step 7 */
    }
    return offsets[n];
}

/* Encode every list into data[offsets[v] .. offsets[v+1]); writes nlb[v]. */
void or_efg_encode(uint64_t n, const uint64_t *vlist, const uint32_t *elist, uint32_t k,
                   const uint64_t *offsets, uint8_t *nlb, uint8_t *data)
{
    for (uint64_t v = 0; v < n; ++v) {
        uint32_t l = 0;
        uint64_t deg = vlist[v + 1] - vlist[v];
        uint64_t s = or_ef_encode_list(elist + vlist[v], deg, k, data + offsets[v], &l);
        (void)s;
        nlb[v] = (uint8_t)l;
    }
}

/* Decode every list of vertices [v0, v1) into out (CSR order). */
void or_efg_decode_range(const uint64_t *vlist, const uint8_t *nlb, const uint64_t *offsets,
                         const uint8_t *data, uint32_t k, uint64_t v0, uint64_t v1, uint32_t *out)
{
    uint64_t base = vlist[v0];
    for (uint64_t v = v0; v < v1; ++v) {
        uint64_t deg = vlist[v + 1] - vlist[v];
        if (deg) or_ef_decode_list(data + offsets[v], deg, nlb[v], k, out + (vlist[v] - base));
    }
}

/* ------------------------------------------------------------------------- */
/* binsearch_maxle (§III-C; Fig. 4): the index of the largest      */
/* value <= key; among equal values the last one (reading C13).  Written as a */
/* linear scan so it is its own definition.                                   */
/* ------------------------------------------------------------------------- */
int64_t or_maxle(const uint64_t *a, uint64_t len, uint64_t key)
{
    int64_t best = -1;
    for (uint64_t i = 0; i < len; ++i)
        if (a[i] <= key) best = (int64_t)i;
    return best;
}

/* Exclusive scan: out[0] = 0, out[i+1] = out[i] + a[i]. */
void or_exclusive_scan(const uint64_t *a, uint64_t len, uint64_t *out)
{
    out[0] = 0;
    for (uint64_t i = 0; i < len; ++i) out[i + 1] = out[i] + a[i];
}

/* ------------------------------------------------------------------------- */
/* SSSP (§VI-F): single-source shortest paths with non-negative fp32    */
/* weights.  Plain Dijkstra with a binary heap; tentative distances are the   */
/* fp32 sum d[u] + w (reading C20 / DESIGN.md: left-fold fp32 path sums).      */
/* w is indexed like elist (CSR order).  Unreached -> +inf.                   */
/* ------------------------------------------------------------------------- */
typedef struct { float d; uint32_t v; } hent;

static void heap_push(hent *h, uint64_t *sz, hent x)
{
    uint64_t i = (*sz)++;
    while (i > 0) {
        uint64_t p = (i - 1) / 2;
        if (h[p].d <= x.d) break;
        h[i] = h[p];
        i = p;
    }
    h[i] = x;
}

static hent heap_pop(hent *h, uint64_t *sz)
{
    hent top = h[0];
    hent x = h[--(*sz)];
    uint64_t i = 0;
    for (;;) {
        uint64_t c = 2 * i + 1;
        if (c >= *sz) break;
        if (c + 1 < *sz && h[c + 1].d < h[c].d) ++c;
        if (h[c].d >= x.d) break;
        h[i] = h[c];
        i = c;
    }
    h[i] = x;
    return top;
}

int or_sssp(uint64_t n, const uint64_t *vlist, const uint32_t *elist, const float *w,
            uint32_t source, float *dist)
{
    for (uint64_t v = 0; v < n; ++v) dist[v] = INFINITY;
    if (source >= n) return -1;
    uint64_t cap = vlist[n] + 1, sz = 0;
    hent *h = (hent *)malloc(cap * sizeof(hent));
    uint8_t *done = (uint8_t *)calloc(n, 1);
    if (!h || !done) { free(h); free(done); return -1; }
    dist[source] = 0.0f;
    heap_push(h, &sz, (hent){0.0f, source});
    while (sz) {
        hent t = heap_pop(h, &sz);
        if (done[t.v]) continue;
        done[t.v] = 1;
        for (uint64_t e = vlist[t.v]; e < vlist[t.v + 1]; ++e) {
            volatile float nd = dist[t.v] + w[e];     /* one fp32 rounding, no contraction */
            uint32_t v = elist[e];
            if (nd < dist[v]) {
                dist[v] = nd;
                heap_push(h, &sz, (hent){nd, v});
            }
        }
    }
    free(h);
    free(done);
    return 0;
}

/* ------------------------------------------------------------------------- */
/* PageRank (§VI-F, 50 iterations P:201), reading C21:                  */
/*   r0 = 1/N;  r'(v) = (1-d)/N + d * ( sum_{u in N(v)} r(u)/deg(u) + D/N )    */
/* with D = sum of r over deg-0 vertices; exactly `iters` iterations; fp64.    */
/* The graph is symmetric, so in-neighbours = out-neighbours = elist lists.    */
/* Written as the push form the paper describes: each u adds r(u)/deg(u) to    */
/* every neighbour.                                                            */
/* ------------------------------------------------------------------------- */
void or_pagerank(uint64_t n, const uint64_t *vlist, const uint32_t *elist, double damping,
                 uint32_t iters, double *rank)
{
    double *next = (double *)malloc((n ? n : 1) * sizeof(double));
    for (uint64_t v = 0; v < n; ++v) rank[v] = 1.0 / (double)n;
    for (uint32_t it = 0; it < iters; ++it) {
        double dangling = 0.0;
        for (uint64_t v = 0; v < n; ++v) next[v] = 0.0;
        for (uint64_t u = 0; u < n; ++u) {
            uint64_t deg = vlist[u + 1] - vlist[u];
            if (deg == 0) { dangling += rank[u]; continue; }
            double share = rank[u] / (double)deg;
            for (uint64_t e = vlist[u]; e < vlist[u + 1]; ++e) next[elist[e]] += share;
        }
        for (uint64_t v = 0; v < n; ++v)
            rank[v] = (1.0 - damping) / (double)n + damping * (next[v] + dangling / (double)n);
    }
    free(next);
}
