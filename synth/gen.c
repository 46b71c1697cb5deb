/*
 * synth/gen.c — seeded synthetic INPUT generators (edge lists, permutations,
 * source samples, edge weights).  Shared by the oracle tests, the GPU parity
 * tests and bench.py.  This file holds none of the method's arithmetic: no
 * Elias-Fano coding, no CSR construction, no traversal.  It only draws random
 * numbers from a counter-based generator (splitmix64), so every array it
 * produces is a pure function of (parameters, seed) and is identical across
 * processes, thread counts and machines.
 *
 * Workload shapes follow DESIGN.md "Input recipe":
 *   - synth_rmat:     Graph500 Kronecker/R-MAT, (a,b,c,d)=(.57,.19,.19,.05),
 *                     no per-level noise (PAPER.md P:69,
 *                     kron graphs from GAP [16]).
 *   - synth_uniform:  Erdos-Renyi style uniform endpoints (urnd_26).
 *   - synth_chunglu:  Chung-Lu power-law (Twitter-shaped C3).
 *   - synth_web:      host-block locality graph (web-shaped C4).
 *   - synth_permutation: random relabelling ("random ordering").
 *   - synth_weights:  symmetric fp32 weights in (0,1].
 */
#include <stdint.h>
#include <stddef.h>
#include <math.h>

static inline uint64_t sm64(uint64_t x)
{
    /* splitmix64 finaliser (Steele, Lea, Flood 2014) */
    x += 0x9E3779B97F4A7C15ull;
    x = (x ^ (x >> 30)) * 0xBF58476D1CE4E5B9ull;
    x = (x ^ (x >> 27)) * 0x94D049BB133111EBull;
    return x ^ (x >> 31);
}

/* counter-based stream: value number `j` of stream `i` under `seed` */
static inline uint64_t draw(uint64_t seed, uint64_t i, uint64_t j)
{
    return sm64(sm64(seed * 0xD1B54A32D192ED03ull + i) ^ (j * 0x9E3779B97F4A7C15ull + 0x632BE59BD9B4E019ull));
}

/* uniform double in [0,1) with 53 random bits */
static inline double unif(uint64_t r) { return (double)(r >> 11) * (1.0 / 9007199254740992.0); }

uint64_t synth_splitmix64(uint64_t x) { return sm64(x); }
uint64_t synth_draw(uint64_t seed, uint64_t i, uint64_t j) { return draw(seed, i, j); }

/* R-MAT / Kronecker edge sampler: for each of `scale` bit levels (MSB first)
 * pick a quadrant with probabilities a, b, c, 1-a-b-c.  `m` undirected samples. */
static void rmat_range(int scale, uint64_t first, uint64_t m, double a, double b, double c, uint64_t seed,
                       uint32_t *src, uint32_t *dst)
{
    const double ab = a + b, abc = a + b + c;
#pragma omp parallel for schedule(static)
    for (int64_t i = 0; i < (int64_t)m; ++i) {
        const uint64_t e = first + (uint64_t)i;
        uint32_t u = 0, v = 0;
        /* draw(seed, e, lvl) with the per-sample part hoisted (same values) */
        const uint64_t h = sm64(seed * 0xD1B54A32D192ED03ull + e);
        for (int lvl = 0; lvl < scale; ++lvl) {
            double r = unif(sm64(h ^ ((uint64_t)lvl * 0x9E3779B97F4A7C15ull + 0x632BE59BD9B4E019ull)));
            uint32_t ub, vb;
            if (r < a)        { ub = 0; vb = 0; }
            else if (r < ab)  { ub = 0; vb = 1; }
            else if (r < abc) { ub = 1; vb = 0; }
            else              { ub = 1; vb = 1; }
            u = (u << 1) | ub;
            v = (v << 1) | vb;
        }
        src[i] = u;
        dst[i] = v;
    }
}

void synth_rmat(int scale, uint64_t m, double a, double b, double c, uint64_t seed,
                uint32_t *src, uint32_t *dst)
{
    rmat_range(scale, 0, m, a, b, c, seed, src, dst);
}

/* uniform random endpoints in [0,n) */
void synth_uniform(uint64_t n, uint64_t m, uint64_t seed, uint32_t *src, uint32_t *dst)
{
#pragma omp parallel for schedule(static)
    for (int64_t e = 0; e < (int64_t)m; ++e) {
        src[e] = (uint32_t)((__uint128_t)draw(seed, (uint64_t)e, 0) * n >> 64);
        dst[e] = (uint32_t)((__uint128_t)draw(seed, (uint64_t)e, 1) * n >> 64);
    }
}

/* random permutation of [0,n): sort-free "random keys" would need a sort, so use
 * a sequential Fisher-Yates driven by the counter stream (deterministic). */
void synth_permutation(uint64_t n, uint64_t seed, uint32_t *perm)
{
    for (uint64_t i = 0; i < n; ++i) perm[i] = (uint32_t)i;
    for (uint64_t i = n; i > 1; --i) {
        uint64_t j = (uint64_t)((__uint128_t)draw(seed, i, 7) * i >> 64);
        uint32_t t = perm[i - 1]; perm[i - 1] = perm[j]; perm[j] = t;
    }
}

/* relabel endpoints in place: x -> perm[x] */
void synth_apply_permutation(uint64_t m, const uint32_t *perm, uint32_t *src, uint32_t *dst)
{
#pragma omp parallel for schedule(static)
    for (int64_t e = 0; e < (int64_t)m; ++e) {
        src[e] = perm[src[e]];
        dst[e] = perm[dst[e]];
    }
}

/* Chung-Lu style power law: endpoint ids drawn from a Zipf-like law by inverse
 * CDF on a continuous approximation p(x) ~ (x+1)^-alpha over [0,n), then
 * relabelled by independent permutations (caller applies).  A fraction `rho` of
 * samples reuses an earlier sample reversed (reciprocity). */
static inline uint32_t zipf_draw(uint64_t n, double alpha, double r)
{
    /* inverse CDF of density ~ (x+1)^-alpha on [0, n) (alpha != 1) */
    double one_m = 1.0 - alpha;
    double hi = pow((double)n + 1.0, one_m) - 1.0;
    double x = pow(1.0 + r * hi, 1.0 / one_m) - 1.0;
    uint64_t xi = (uint64_t)x;
    if (xi >= n) xi = n - 1;
    return (uint32_t)xi;
}

static void chunglu_range(uint64_t n, uint64_t first, uint64_t m, double alpha_src, double alpha_dst,
                          double rho, uint64_t seed, uint32_t *src, uint32_t *dst)
{
#pragma omp parallel for schedule(static)
    for (int64_t i = 0; i < (int64_t)m; ++i) {
        const uint64_t e = first + (uint64_t)i;
        uint64_t r0 = draw(seed, e, 0);
        if (e > 0 && unif(r0) < rho) {
            /* reciprocal copy of an earlier sample (index drawn from [0,e)) */
            uint64_t j = (uint64_t)((__uint128_t)draw(seed, e, 1) * e >> 64);
            uint32_t u = zipf_draw(n, alpha_src, unif(draw(seed, j, 2)));
            uint32_t v = zipf_draw(n, alpha_dst, unif(draw(seed, j, 3)));
            src[i] = v; dst[i] = u;
        } else {
            src[i] = zipf_draw(n, alpha_src, unif(draw(seed, e, 2)));
            dst[i] = zipf_draw(n, alpha_dst, unif(draw(seed, e, 3)));
        }
    }
}

void synth_chunglu(uint64_t n, uint64_t m, double alpha_src, double alpha_dst, double rho,
                   uint64_t seed, uint32_t *src, uint32_t *dst)
{
    chunglu_range(n, 0, m, alpha_src, alpha_dst, rho, seed, src, dst);
}

/* Web-shaped locality graph.  Vertices are grouped into contiguous "hosts" of
 * Pareto-distributed size (mean ~ host_mean).  Each sample picks a uniform source
 * u; with prob p_intra its target lies in u's host at a geometric offset, with
 * prob p_near in a host at a geometric host offset, otherwise it points to the
 * first page of a Zipf-popular host.  host_start[] (n_hosts+1) is provided by
 * the caller from synth_web_hosts.  Ids are locality-ordered; callers permute
 * for the "random ordering" variant. */
uint64_t synth_web_hosts(uint64_t n, double pareto_alpha, double xm, uint64_t cap, uint64_t seed,
                         uint64_t *host_start, uint64_t max_hosts)
{
    uint64_t h = 0, pos = 0;
    while (pos < n && h < max_hosts) {
        double r = unif(draw(seed, h, 11));
        /* Pareto(xm, alpha) size: mean xm * alpha / (alpha - 1) (~100 pages for
         * xm = 33.3, alpha = 1.5: SURVEY §8(d) C4) */
        double s = xm * pow(1.0 - r, -1.0 / pareto_alpha);
        uint64_t sz = (uint64_t)s;
        if (sz < 1) sz = 1;
        if (sz > cap) sz = cap;
        if (pos + sz > n) sz = n - pos;
        host_start[h++] = pos;
        pos += sz;
    }
    host_start[h] = n;
    return h;
}

static inline int64_t geom_off(double p, double r)
{
    /* geometric(p) >= 1 magnitude */
    return 1 + (int64_t)floor(log(1.0 - r) / log(1.0 - p));
}

static void web_range(uint64_t n, uint64_t first, uint64_t m, const uint64_t *host_start, uint64_t n_hosts,
                      const uint32_t *host_of, double p_intra, double p_near, double zipf_alpha,
                      uint64_t seed, uint32_t *src, uint32_t *dst)
{
#pragma omp parallel for schedule(static)
    for (int64_t i = 0; i < (int64_t)m; ++i) {
        const int64_t e = (int64_t)(first + (uint64_t)i);
        uint64_t u = (uint64_t)((__uint128_t)draw(seed, (uint64_t)e, 0) * n >> 64);
        uint64_t h = host_of[u];
        double kind = unif(draw(seed, (uint64_t)e, 1));
        double r2 = unif(draw(seed, (uint64_t)e, 2));
        int sgn = (draw(seed, (uint64_t)e, 3) & 1) ? 1 : -1;
        uint64_t v;
        if (kind < p_intra) {
            uint64_t lo = host_start[h], hi = host_start[h + 1];
            int64_t off = geom_off(0.03, r2) * sgn;
            int64_t t = (int64_t)u + off;
            uint64_t span = hi - lo;
            /* reflect into [lo, hi) */
            int64_t rel = t - (int64_t)lo;
            rel %= (int64_t)span; if (rel < 0) rel += (int64_t)span;
            v = lo + (uint64_t)rel;
        } else if (kind < p_intra + p_near) {
            int64_t off = geom_off(0.05, r2) * sgn;
            int64_t th = (int64_t)h + off;
            th %= (int64_t)n_hosts; if (th < 0) th += (int64_t)n_hosts;
            uint64_t lo = host_start[th], hi = host_start[th + 1];
            v = lo + (uint64_t)((__uint128_t)draw(seed, (uint64_t)e, 4) * (hi - lo) >> 64);
        } else {
            uint64_t th = zipf_draw(n_hosts, zipf_alpha, r2);
            uint64_t lo = host_start[th], hi = host_start[th + 1];
            if (draw(seed, (uint64_t)e, 5) & 1) v = lo;
            else v = lo + (uint64_t)((__uint128_t)draw(seed, (uint64_t)e, 4) * (hi - lo) >> 64);
        }
        src[i] = (uint32_t)u;
        dst[i] = (uint32_t)v;
    }
}

void synth_web(uint64_t n, uint64_t m, const uint64_t *host_start, uint64_t n_hosts,
               const uint32_t *host_of, double p_intra, double p_near, double zipf_alpha,
               uint64_t seed, uint32_t *src, uint32_t *dst)
{
    web_range(n, 0, m, host_start, n_hosts, host_of, p_intra, p_near, zipf_alpha, seed, src, dst);
}

/* host_of[v] for v in [0,n) given host_start */
void synth_web_host_of(uint64_t n_hosts, const uint64_t *host_start, uint32_t *host_of)
{
#pragma omp parallel for schedule(dynamic, 1024)
    for (int64_t h = 0; h < (int64_t)n_hosts; ++h)
        for (uint64_t v = host_start[h]; v < host_start[h + 1]; ++v) host_of[v] = (uint32_t)h;
}

/* Symmetric fp32 edge weight in (0,1], exactly representable (k * 2^-24),
 * a function of the unordered pair {u,v}. */
static inline float weight_of(uint64_t seed, uint32_t u, uint32_t v)
{
    uint64_t lo = u < v ? u : v, hi = u < v ? v : u;
    uint64_t r = sm64(seed ^ ((lo << 32) | hi));
    return (float)((double)((r >> 40) + 1) * (1.0 / 16777216.0));
}

void synth_weights(uint64_t m, const uint32_t *src, const uint32_t *dst, uint64_t seed, float *w)
{
#pragma omp parallel for schedule(static)
    for (int64_t e = 0; e < (int64_t)m; ++e) w[e] = weight_of(seed, src[e], dst[e]);
}

float synth_weight_pair(uint64_t seed, uint32_t u, uint32_t v) { return weight_of(seed, u, v); }

/* ------------------------------------------------------------------------- */
/* Range generation for streamed builds (efg_build_stream): a context names a */
/* config's generator; synth_gen_range writes samples [first, first+count),   */
/* identical to the same indices of the whole-array generator, then the       */
/* optional relabelling and the optional weights.  Matches efg_edge_gen_fn.   */
/* ------------------------------------------------------------------------- */
typedef struct synth_gen_ctx {
    int kind;                 /* 0 rmat, 1 chunglu, 2 web, 3 uniform */
    int scale;
    uint64_t n, seed;
    double a, b, c;           /* rmat */
    double alpha_src, alpha_dst, rho;  /* chunglu */
    const uint64_t *host_start;        /* web */
    uint64_t n_hosts;
    const uint32_t *host_of;
    double p_intra, p_near, zipf_alpha;
    const uint32_t *perm;     /* relabelling x -> perm[x], or NULL */
    uint64_t wseed;           /* weight seed (weights written when w != NULL) */
} synth_gen_ctx;

void synth_gen_range(void *vctx, uint64_t first, uint64_t count, uint32_t *src, uint32_t *dst, float *w)
{
    const synth_gen_ctx *g = (const synth_gen_ctx *)vctx;
    switch (g->kind) {
    case 0: rmat_range(g->scale, first, count, g->a, g->b, g->c, g->seed, src, dst); break;
    case 1: chunglu_range(g->n, first, count, g->alpha_src, g->alpha_dst, g->rho, g->seed, src, dst); break;
    case 2: web_range(g->n, first, count, g->host_start, g->n_hosts, g->host_of, g->p_intra, g->p_near,
                      g->zipf_alpha, g->seed, src, dst); break;
    default:
#pragma omp parallel for schedule(static)
        for (int64_t i = 0; i < (int64_t)count; ++i) {
            const uint64_t e = first + (uint64_t)i;
            src[i] = (uint32_t)((__uint128_t)draw(g->seed, e, 0) * g->n >> 64);
            dst[i] = (uint32_t)((__uint128_t)draw(g->seed, e, 1) * g->n >> 64);
        }
    }
    if (g->perm) synth_apply_permutation(count, g->perm, src, dst);
    if (w) synth_weights(count, src, dst, g->wseed, w);
}
