/*
 * omp_bfs.c -- OpenMP level-synchronous top-down BFS on all host cores: the parallel CPU baseline
 * SURVEY 8(d) d1/d3 asks to time beside the GPU ("plus an OpenMP level-synchronous BFS on all host
 * cores").  Context for bench.py only -- it is neither the oracle (oracle/oracle.c is the parity
 * reference) nor part of the product path, and nothing else loads it.
 *
 * Level t: every thread takes frontier vertices, claims unvisited neighbours with a
 * compare-and-swap on depth (-1 -> t+1) and appends winners to a thread-local buffer; the buffers
 * are concatenated into the next frontier.  Depths equal the FIFO BFS's (levels are unique).
 */
#include <stdint.h>
#include <stdlib.h>
#include <string.h>
#include <omp.h>

int omp_bfs(int64_t n, const int64_t *off, const int32_t *col, int32_t src, int32_t *depth) {
    if (n <= 0 || src < 0 || src >= n) return -2;
    int32_t *cur = (int32_t *)malloc((size_t)n * sizeof(int32_t));
    int32_t *nxt = (int32_t *)malloc((size_t)n * sizeof(int32_t));
    if (!cur || !nxt) { free(cur); free(nxt); return -1; }
#pragma omp parallel for schedule(static)
    for (int64_t v = 0; v < n; ++v) depth[v] = -1;
    depth[src] = 0;
    cur[0] = src;
    int64_t ncur = 0 + 1;
    int32_t lvl = 0;
    while (ncur > 0) {
        int64_t nn = 0;
#pragma omp parallel
        {
            int32_t buf[1024];
            int nb = 0;
#pragma omp for schedule(dynamic, 64)
            for (int64_t i = 0; i < ncur; ++i) {
                const int32_t u = cur[i];
                for (int64_t e = off[u]; e < off[u + 1]; ++e) {
                    const int32_t v = col[e];
                    if (depth[v] < 0 && __sync_bool_compare_and_swap(&depth[v], -1, lvl + 1)) {
                        buf[nb++] = v;
                        if (nb == 1024) {
                            int64_t p = __atomic_fetch_add(&nn, nb, __ATOMIC_RELAXED);
                            memcpy(nxt + p, buf, sizeof(int32_t) * nb);
                            nb = 0;
                        }
                    }
                }
            }
            if (nb) {
                int64_t p = __atomic_fetch_add(&nn, nb, __ATOMIC_RELAXED);
                memcpy(nxt + p, buf, sizeof(int32_t) * nb);
            }
        }
        int32_t *t = cur; cur = nxt; nxt = t;
        ncur = nn;
        ++lvl;
    }
    free(cur); free(nxt);
    return 0;
}

int omp_threads(void) { return omp_get_max_threads(); }
