// efg_builder.cpp — host-side EFG builder (north_star (a)).
//
// edge source --(symmetrise, "_sym")--> directed multiset
//             --(bucket by source, sort each list, drop self-loops/duplicates:
//                readings C11/C12)--> CSR vlist/elist (§III-D)
//             --(per-vertex Elias-Fano, §IV, layout P:111-117 §V,
//                forward pointers P:157 §VI-C)--> vlist, num_lower_bits, offsets, data
//
// The edge source is either caller arrays (efg_build) or a generator callback
// that produces any sample range on demand (efg_build_stream): the builder then
// reads the edges in chunks, twice (a counting pass and a scatter pass), and
// never holds the edge list — on a row-range handle it holds only the owned
// rows' adjacency, which is what makes RMAT-29 shards (BASELINE configs[4])
// fit a host.
//
// Two encoding passes as the paper notes the size is known a priori:
// pass 1 computes every list's byte size from (n, u, k) alone, an exclusive scan
// gives `offsets`, pass 2 encodes all lists in parallel (OpenMP).
#include <omp.h>

#include <algorithm>
#include <chrono>
#include <cstring>
#include <memory>
#include <new>
#include <vector>

#include "efg_internal.h"

namespace efg {

ListGeom list_geom(uint64_t n, uint64_t u, uint32_t k)
{
    ListGeom g{0, 0, 0, 0};
    if (n == 0) return g;                                  // reading C10
    const uint64_t q = u / n;                              // reading C3 (integer u/n)
    g.l = q ? (uint32_t)(63 - __builtin_clzll(q)) : 0u;    // floor(log2(u/n)), C1
    g.fwd = k ? 4ull * (n / k) : 0ull;                     // C8: uint32 per pointer
    g.lower = (n * g.l + 7) / 8;                           // P:89 lower-bits array
    g.upper = ((u >> g.l) + n + 7) / 8;                    // C4: n stop bits + (u>>l) zeros
    return g;
}

namespace {

// Exclusive scan in place over a[0..len) with a[len] = total (a has len+1 slots).
void exclusive_scan_inplace(uint64_t *a, uint64_t len)
{
    uint64_t run = 0;
    for (uint64_t i = 0; i < len; ++i) {
        uint64_t x = a[i];
        a[i] = run;
        run += x;
    }
    a[len] = run;
}

inline uint32_t float_key(float w)
{
    uint32_t b;
    std::memcpy(&b, &w, 4);
    return b;  // weights are >= 0, so the IEEE bit pattern orders like the value
}

// Adjacency entries: the neighbour id alone (unweighted), or neighbour << 32 |
// weight key (weighted: sorting then orders by neighbour, ties by weight, so the
// first copy of a duplicate carries the minimum weight).
inline uint32_t nbr_of(uint32_t a) { return a; }
inline uint32_t nbr_of(uint64_t a) { return (uint32_t)(a >> 32); }
inline uint32_t make_entry(uint32_t /*tag*/, uint32_t nb, uint32_t) { return nb; }
inline uint64_t make_entry(uint64_t /*tag*/, uint32_t nb, uint32_t wk) { return ((uint64_t)nb << 32) | wk; }

// Encode one sorted, duplicate-free list x[0..n) at `out` (pre-zeroed).
void encode_list(const uint32_t *x, uint64_t n, uint32_t k, const ListGeom &g, uint8_t *out)
{
    const uint32_t l = g.l;
    // forward pointers: fwd[j] = x[(j+1)k-1] >> l  (= select1(i) - i)
    if (k) {
        const uint64_t F = n / k;
        for (uint64_t j = 0; j < F; ++j) {
            const uint32_t f = x[(j + 1) * k - 1] >> l;
            std::memcpy(out + 4 * j, &f, 4);  // little endian host
        }
    }
    // lower bits: element i occupies bits [i*l, (i+1)*l), LSB first (C6)
    uint8_t *lower = out + g.fwd;
    if (l) {
        const uint64_t mask = (1ull << l) - 1;
        uint64_t acc = 0;
        uint32_t nb = 0;
        uint64_t p = 0;
        for (uint64_t i = 0; i < n; ++i) {
            acc |= ((uint64_t)x[i] & mask) << nb;
            nb += l;
            while (nb >= 8) {
                lower[p++] = (uint8_t)acc;
                acc >>= 8;
                nb -= 8;
            }
        }
        if (nb) lower[p++] = (uint8_t)acc;
    }
    // upper bits: stop bit of element i at position (x[i] >> l) + i
    uint8_t *upper = lower + g.lower;
    for (uint64_t i = 0; i < n; ++i) {
        const uint64_t pos = ((uint64_t)(x[i] >> l)) + i;
        upper[pos >> 3] |= (uint8_t)(1u << (pos & 7));
    }
}

// The edges, chunk by chunk: caller arrays (one chunk) or a generator.
struct EdgeSource {
    uint64_t m = 0;
    const uint32_t *src = nullptr, *dst = nullptr;
    const float *w = nullptr;
    efg_edge_gen_fn gen = nullptr;
    void *user = nullptr;
    bool weighted = false;
    uint64_t chunk = 1ull << 26;
    std::vector<uint32_t> bs, bd;
    std::vector<float> bw;

    // f(const uint32_t *s, const uint32_t *d, const float *w, uint64_t count, uint64_t first)
    template <class F>
    void for_each(F &&f)
    {
        if (!gen) {
            f(src, dst, w, m, 0);
            return;
        }
        const uint64_t cz = std::min<uint64_t>(chunk, std::max<uint64_t>(m, 1));
        bs.resize(cz);
        bd.resize(cz);
        if (weighted) bw.resize(cz);
        for (uint64_t first = 0; first < m; first += cz) {
            const uint64_t cnt = std::min<uint64_t>(cz, m - first);
            gen(user, first, cnt, bs.data(), bd.data(), weighted ? bw.data() : nullptr);
            f(bs.data(), bd.data(), weighted ? bw.data() : nullptr, cnt, first);
        }
    }
};

template <class T>
efg_status build_lists(uint64_t n, EdgeSource &es, const efg_build_opts &o, HostEFG &out)
{
    const bool sym = o.flags & EFG_SYMMETRIZE;
    const bool dedup = o.flags & EFG_DEDUP;
    const bool noself = o.flags & EFG_DROP_SELF_LOOPS;
    const bool weighted = es.weighted;
    const bool reorder = o.flags & EFG_REORDER_DEGREE;
    const uint32_t k = o.fwd_quantum;
    const bool part = o.row_hi > o.row_lo;
    const uint64_t lo = part ? std::min<uint64_t>(o.row_lo, n) : 0, hi = part ? std::min<uint64_t>(o.row_hi, n) : n;
    // rows whose adjacency is materialised: the owned range, or every row when
    // the degree relabelling needs the whole graph's degrees
    const uint64_t mlo = (part && !reorder) ? lo : 0, mhi = (part && !reorder) ? hi : n;

    // ---- pass A: validate ids, count the materialised rows' entries, and
    // mark vertices with an in-edge (any row; never probed otherwise) ----
    std::vector<uint64_t> start(n + 1, 0);
    std::vector<uint8_t> has_in(n, 0);
    uint64_t bad = 0;
    es.for_each([&](const uint32_t *s, const uint32_t *d, const float *, uint64_t cnt, uint64_t) {
        uint64_t b = 0;
#pragma omp parallel for reduction(+ : b) schedule(static)
        for (int64_t e = 0; e < (int64_t)cnt; ++e) {
            const uint32_t u = s[e], v = d[e];
            if (u >= n || v >= n) {
                ++b;
                continue;
            }
            if (u == v) {
                if (noself) continue;
            } else {
                has_in[v] = 1;  // benign same-value races
                if (sym) has_in[u] = 1;
            }
            if (u >= mlo && u < mhi) __atomic_fetch_add(&start[u], 1ull, __ATOMIC_RELAXED);
            if (sym && v >= mlo && v < mhi) __atomic_fetch_add(&start[v], 1ull, __ATOMIC_RELAXED);
        }
        bad += b;
    });
    if (bad) return set_error(EFG_ERANGE, "efg_build: " + std::to_string(bad) + " edge endpoints >= n");
    exclusive_scan_inplace(start.data(), n);
    const uint64_t total = start[n];

    // ---- pass B: bucket by source (order inside a bucket is fixed by the sort below) ----
    std::unique_ptr<uint64_t[]> cur(new uint64_t[n]);
    std::memcpy(cur.get(), start.data(), n * sizeof(uint64_t));
    std::unique_ptr<T[]> tmp(new T[total ? total : 1]);
    es.for_each([&](const uint32_t *s, const uint32_t *d, const float *w, uint64_t cnt, uint64_t) {
#pragma omp parallel for schedule(static)
        for (int64_t e = 0; e < (int64_t)cnt; ++e) {
            const uint32_t u = s[e], v = d[e];
            if (noself && u == v) continue;
            const uint32_t wk = (weighted && w) ? float_key(w[e]) : 0u;
            if (u >= mlo && u < mhi) tmp[__atomic_fetch_add(&cur[u], 1ull, __ATOMIC_RELAXED)] = make_entry(T(), v, wk);
            if (sym && v >= mlo && v < mhi)
                tmp[__atomic_fetch_add(&cur[v], 1ull, __ATOMIC_RELAXED)] = make_entry(T(), u, wk);
        }
    });
    cur.reset();

    // ---- sort each list; drop duplicates (keep the min weight) ----
    std::vector<uint64_t> deg(n + 1, 0);
#pragma omp parallel for schedule(dynamic, 512)
    for (int64_t v = 0; v < (int64_t)n; ++v) {
        T *a = tmp.get() + start[v];
        const uint64_t len = start[v + 1] - start[v];
        std::sort(a, a + len);
        uint64_t w = 0;
        for (uint64_t i = 0; i < len; ++i) {
            if (dedup && w && nbr_of(a[w - 1]) == nbr_of(a[i])) continue;
            a[w++] = a[i];
        }
        deg[v] = w;
    }
    // optional relabelling by degree (descending, ties by id): the
    // reordering preprocessing of P:246-258 / P:35 in its simplest form.
    // Results are reported in input ids.
    if (reorder) {
        uint64_t maxd = 0;
#pragma omp parallel for reduction(max : maxd)
        for (int64_t v = 0; v < (int64_t)n; ++v) maxd = std::max<uint64_t>(maxd, deg[v]);
        std::vector<uint64_t> bucket(maxd + 2, 0);
        for (uint64_t v = 0; v < n; ++v) bucket[maxd - deg[v]]++;
        exclusive_scan_inplace(bucket.data(), maxd + 1);
        out.old_of_new.resize(n);
        out.new_of_old.resize(n);
        for (uint64_t v = 0; v < n; ++v) {  // stable: ascending id within a degree
            const uint64_t i = bucket[maxd - deg[v]]++;
            out.old_of_new[i] = (uint32_t)v;
            out.new_of_old[v] = (uint32_t)i;
        }
        std::vector<uint64_t> start2(n + 1, 0), deg2(n + 1, 0);
        for (uint64_t i = 0; i < n; ++i) deg2[i] = deg[out.old_of_new[i]];
        for (uint64_t i = 0; i < n; ++i) start2[i + 1] = start2[i] + deg2[i];
        std::unique_ptr<T[]> tmp2(new T[start2[n] ? start2[n] : 1]);
        const uint32_t *nof = out.new_of_old.data();
#pragma omp parallel for schedule(dynamic, 512)
        for (int64_t i = 0; i < (int64_t)n; ++i) {
            const uint64_t v = out.old_of_new[i];
            const T *a = tmp.get() + start[v];
            T *b = tmp2.get() + start2[i];
            for (uint64_t t = 0; t < deg2[i]; ++t) {
                if constexpr (sizeof(T) == 4)
                    b[t] = nof[a[t]];
                else
                    b[t] = ((uint64_t)nof[(uint32_t)(a[t] >> 32)] << 32) | (uint32_t)a[t];
            }
            std::sort(b, b + deg2[i]);
        }
        tmp.swap(tmp2);
        start.swap(start2);
        deg.swap(deg2);
        std::vector<uint8_t> hin(n);
        for (uint64_t v = 0; v < n; ++v) hin[nof[v]] = has_in[v];
        has_in.swap(hin);
    }
    out.has_in.swap(has_in);
    // partition: keep only the owned rows' lists
    for (uint64_t v = 0; v < n; ++v)
        if (v < lo || v >= hi) deg[v] = 0;
    out.vlist.assign(deg.begin(), deg.end());
    exclusive_scan_inplace(out.vlist.data(), n);
    out.m = out.vlist[n];
    out.n = n;
    out.m_input = es.m;
    out.k = k;
    out.row_lo = lo;
    out.symmetric = sym;
    out.row_hi = hi;

    // ---- pass 1: a-priori sizes -> offsets ----
    if (weighted) out.weights.resize(out.m);
    out.nlb.assign(n, 0);
    out.umax.assign(n, 0);
    out.offsets.assign(n + 1, 0);
    uint64_t fb = 0, lb = 0, ub = 0, ab = 0;
#pragma omp parallel for schedule(dynamic, 1024) reduction(+ : fb, lb, ub, ab)
    for (int64_t v = 0; v < (int64_t)n; ++v) {
        const uint64_t d = deg[v];
        if (!d) continue;
        const T *a = tmp.get() + start[v];
        const uint32_t u = nbr_of(a[d - 1]);
        const ListGeom g = list_geom(d, u, k);
        out.nlb[v] = (uint8_t)g.l;
        out.umax[v] = u;
        out.offsets[v] = g.fwd + g.lower + g.upper;
        fb += g.fwd;
        lb += g.lower;
        ub += g.upper;
        ab += d * g.l + d + ((uint64_t)u >> g.l);
    }
    exclusive_scan_inplace(out.offsets.data(), n);
    out.fwd_bytes = fb;
    out.lower_bytes = lb;
    out.upper_bytes = ub;
    out.apriori_bits = ab;

    // ---- pass 2: encode (parallel over vertices) ----
    out.data.assign(out.offsets[n], 0);
#pragma omp parallel
    {
        std::vector<uint32_t> x;
#pragma omp for schedule(dynamic, 1024)
        for (int64_t v = 0; v < (int64_t)n; ++v) {
            const uint64_t d = deg[v];
            if (!d) continue;
            const T *a = tmp.get() + start[v];
            x.resize(d);
            for (uint64_t i = 0; i < d; ++i) x[i] = nbr_of(a[i]);
            if (weighted) {
                float *wo = out.weights.data() + out.vlist[v];
                for (uint64_t i = 0; i < d; ++i) {
                    const uint32_t b = (uint32_t)(uint64_t)a[i];
                    std::memcpy(&wo[i], &b, 4);
                }
            }
            const ListGeom g = list_geom(d, x[d - 1], k);
            encode_list(x.data(), d, k, g, out.data.data() + out.offsets[v]);
        }
    }
    return EFG_OK;
}

efg_status build_from(uint64_t n, EdgeSource &es, const efg_build_opts &o, HostEFG &out)
{
    const auto t0 = std::chrono::steady_clock::now();
    if (o.n_threads) omp_set_num_threads((int)o.n_threads);
    efg_status st;
    try {
        st = es.weighted ? build_lists<uint64_t>(n, es, o, out) : build_lists<uint32_t>(n, es, o, out);
    } catch (const std::bad_alloc &) {
        return set_error(EFG_ENOMEM, "efg_build: host allocation failed");
    }
    out.build_seconds = std::chrono::duration<double>(std::chrono::steady_clock::now() - t0).count();
    return st;
}

}  // namespace

efg_status build_host(uint64_t n, uint64_t m, const uint32_t *src, const uint32_t *dst,
                      const efg_build_opts &o, HostEFG &out)
{
    EdgeSource es;
    es.m = m;
    es.src = src;
    es.dst = dst;
    es.w = o.weights;
    es.weighted = o.weights != nullptr;
    return build_from(n, es, o, out);
}

efg_status build_host_stream(uint64_t n, uint64_t m, efg_edge_gen_fn gen, void *user, int weighted,
                             const efg_build_opts &o, HostEFG &out)
{
    EdgeSource es;
    es.m = m;
    es.gen = gen;
    es.user = user;
    es.weighted = weighted != 0;
    return build_from(n, es, o, out);
}

}  // namespace efg
