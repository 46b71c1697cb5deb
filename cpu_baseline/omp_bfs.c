/*
 * cpu_baseline/omp_bfs.c — the optional all-core CPU baseline of BASELINE.md
 * ("CPU-baseline plan"): a level-synchronous top-down BFS over an uncompressed
 * CSR with OpenMP, reported next to the single-core oracle by bench.py.  It is
 * a baseline, not a reference: tests check it against the oracle's depths.  It
 * shares no code with the oracle or the product.
 *
 * Each level: threads take frontier vertices in dynamic chunks, claim
 * undiscovered neighbours with a compare-and-swap on depth (-1 -> L+1), append
 * them to a thread-local buffer, and the buffers are concatenated into the
 * next frontier.  Returns the number of reached vertices.
 */
#include <stdint.h>
#include <stdlib.h>
#include <string.h>
#include <omp.h>

uint64_t cb_bfs_omp(uint64_t n, const uint64_t *vlist, const uint32_t *elist, uint32_t source, int32_t *depth,
                    int threads)
{
    if (threads > 0) omp_set_num_threads(threads);
#pragma omp parallel for schedule(static)
    for (int64_t v = 0; v < (int64_t)n; ++v) depth[v] = -1;
    if (source >= n) return 0;
    uint32_t *cur = (uint32_t *)malloc(n * sizeof(uint32_t));
    uint32_t *nxt = (uint32_t *)malloc(n * sizeof(uint32_t));
    if (!cur || !nxt) { free(cur); free(nxt); return 0; }
    uint64_t ncur = 1, reached = 1;
    cur[0] = source;
    depth[source] = 0;
    int32_t level = 0;
    while (ncur) {
        uint64_t nnext = 0;
#pragma omp parallel
        {
            uint32_t *buf = (uint32_t *)malloc(4096 * sizeof(uint32_t));
            uint64_t nb = 0;
#pragma omp for schedule(dynamic, 64)
            for (int64_t i = 0; i < (int64_t)ncur; ++i) {
                const uint32_t u = cur[i];
                for (uint64_t e = vlist[u]; e < vlist[u + 1]; ++e) {
                    const uint32_t v = elist[e];
                    if (__atomic_load_n(&depth[v], __ATOMIC_RELAXED) >= 0) continue;
                    int32_t expect = -1;
                    if (__atomic_compare_exchange_n(&depth[v], &expect, level + 1, 0, __ATOMIC_RELAXED,
                                                    __ATOMIC_RELAXED)) {
                        buf[nb++] = v;
                        if (nb == 4096) {
                            const uint64_t at = __atomic_fetch_add(&nnext, nb, __ATOMIC_RELAXED);
                            memcpy(nxt + at, buf, nb * sizeof(uint32_t));
                            nb = 0;
                        }
                    }
                }
            }
            if (nb) {
                const uint64_t at = __atomic_fetch_add(&nnext, nb, __ATOMIC_RELAXED);
                memcpy(nxt + at, buf, nb * sizeof(uint32_t));
            }
            free(buf);
        }
        uint32_t *t = cur; cur = nxt; nxt = t;
        ncur = nnext;
        reached += nnext;
        ++level;
    }
    free(cur);
    free(nxt);
    return reached;
}
