/*
 * gen.c -- seeded synthetic graph generators shared by the oracle side and the CUDA side.
 *
 * This module holds NO arithmetic of the method (no BFS/SSSP/CC/PR/BC, no features, no selector).
 * It only draws inputs: R-MAT/Kronecker edge tuples, a 2D road-like grid, a Chung-Lu power-law
 * graph, and symmetric integer edge weights, then builds a CSR (symmetrise, drop self-loops,
 * dedupe, sort adjacency ascending).  All graphs are undirected as in the paper: "All graphs were
 * transformed into undirected ones" (Sec. 5.1 footnote 3).
 *
 * Randomness is counter-based (splitmix64, Vigna), so every draw is a pure function of
 * (seed, stream, index): results do not depend on thread count or evaluation order.
 *   splitmix64(x): z = x + 0x9E3779B97F4A7C15; z = (z^(z>>30))*0xBF58476D1CE4E5B9;
 *                  z = (z^(z>>27))*0x94D049BB133111EB; return z^(z>>31)
 *
 * Recipes:
 *   R-MAT  : Graph500 (a,b,c,d)=(.57,.19,.19,.05), ef*2^scale tuples, no noise, random vertex
 *            permutation (Fisher-Yates with the same counter RNG).
 *   grid   : W x H 4-neighbour grid, row-major ids.
 *   weights: w(u,v) = 1 + splitmix64((min(u,v)*N + max(u,v)) ^ seed) mod maxw
 *   ChungLu: P(i) ~ (i+i0)^(-1/(gamma-1)), `pairs` endpoint pairs by inverse-CDF sampling,
 *            random permutation.
 */
#include <stdint.h>
#include <stdlib.h>
#include <string.h>
#include <math.h>

#define GOLDEN 0x9E3779B97F4A7C15ULL

static inline uint64_t splitmix64(uint64_t x) {
    uint64_t z = x + GOLDEN;
    z = (z ^ (z >> 30)) * 0xBF58476D1CE4E5B9ULL;
    z = (z ^ (z >> 27)) * 0x94D049BB133111EBULL;
    return z ^ (z >> 31);
}
/* idx-th output of the splitmix64 stream keyed by (seed, stream) */
static inline uint64_t crng(uint64_t seed, uint64_t stream, uint64_t idx) {
    uint64_t key = splitmix64(seed ^ (stream * 0xD1B54A32D192ED03ULL));
    return splitmix64(key + idx * GOLDEN);
}
static inline double u01(uint64_t r) { return (double)(r >> 11) * (1.0 / 9007199254740992.0); }

uint64_t gen_splitmix64(uint64_t x) { return splitmix64(x); }

/* OpenMP threads of the generators (0 = all cores).  torchrun exports OMP_NUM_THREADS=1 to every
 * rank; bench.py gives each rank its share of the host cores for its slice of C5 instead. */
#ifdef _OPENMP
#include <omp.h>
#endif
void gen_set_threads(int k) {
#ifdef _OPENMP
    omp_set_num_threads(k > 0 ? k : omp_get_num_procs());
#else
    (void)k;
#endif
}

typedef struct {
    int64_t n, nnz;
    int64_t *off;   /* n+1 */
    int32_t *col;   /* nnz */
    uint32_t *w;    /* nnz or NULL */
} gen_csr;

void gen_free(gen_csr *g) {
    free(g->off); free(g->col); free(g->w);
    g->off = NULL; g->col = NULL; g->w = NULL;
}

static int cmp_i32(const void *a, const void *b) {
    int32_t x = *(const int32_t *)a, y = *(const int32_t *)b;
    return (x > y) - (x < y);
}

/* Build a symmetric, loop-free, deduplicated CSR with ascending rows from m undirected tuples. */
static int build_csr(int64_t n, int64_t m, const uint32_t *U, const uint32_t *V, gen_csr *out) {
    int64_t *cnt = (int64_t *)calloc((size_t)n + 1, sizeof(int64_t));
    if (!cnt) return -1;
    for (int64_t k = 0; k < m; ++k) {
        if (U[k] == V[k]) continue;
        cnt[U[k] + 1]++; cnt[V[k] + 1]++;
    }
    for (int64_t i = 0; i < n; ++i) cnt[i + 1] += cnt[i];
    int64_t tot = cnt[n];
    int32_t *col = (int32_t *)malloc((size_t)(tot ? tot : 1) * sizeof(int32_t));
    int64_t *pos = (int64_t *)malloc((size_t)n * sizeof(int64_t));
    if (!col || !pos) { free(cnt); free(col); free(pos); return -1; }
    memcpy(pos, cnt, (size_t)n * sizeof(int64_t));
    for (int64_t k = 0; k < m; ++k) {
        uint32_t u = U[k], v = V[k];
        if (u == v) continue;
        col[pos[u]++] = (int32_t)v;
        col[pos[v]++] = (int32_t)u;
    }
    free(pos);
    int64_t *deg = (int64_t *)malloc((size_t)n * sizeof(int64_t));
    if (!deg) { free(cnt); free(col); return -1; }
#pragma omp parallel for schedule(dynamic, 1024)
    for (int64_t i = 0; i < n; ++i) {
        int32_t *r = col + cnt[i];
        int64_t len = cnt[i + 1] - cnt[i];
        if (len > 1) qsort(r, (size_t)len, sizeof(int32_t), cmp_i32);
        int64_t k = 0;
        for (int64_t j = 0; j < len; ++j)
            if (k == 0 || r[j] != r[k - 1]) r[k++] = r[j];
        deg[i] = k;
    }
    int64_t *off = (int64_t *)malloc(((size_t)n + 1) * sizeof(int64_t));
    if (!off) { free(cnt); free(col); free(deg); return -1; }
    off[0] = 0;
    for (int64_t i = 0; i < n; ++i) off[i + 1] = off[i] + deg[i];
    int64_t nnz = off[n];
    int32_t *c2 = (int32_t *)malloc((size_t)(nnz ? nnz : 1) * sizeof(int32_t));
    if (!c2) { free(cnt); free(col); free(deg); free(off); return -1; }
#pragma omp parallel for schedule(dynamic, 4096)
    for (int64_t i = 0; i < n; ++i)
        memcpy(c2 + off[i], col + cnt[i], (size_t)deg[i] * sizeof(int32_t));
    free(cnt); free(col); free(deg);
    out->n = n; out->nnz = nnz; out->off = off; out->col = c2; out->w = NULL;
    return 0;
}

/* Fisher-Yates permutation of [0,n) drawn from the counter RNG (stream 2). */
static uint32_t *make_perm(int64_t n, uint64_t seed) {
    uint32_t *p = (uint32_t *)malloc((size_t)(n ? n : 1) * sizeof(uint32_t));
    if (!p) return NULL;
    for (int64_t i = 0; i < n; ++i) p[i] = (uint32_t)i;
    for (int64_t i = n - 1; i > 0; --i) {
        uint64_t j = crng(seed, 2, (uint64_t)i) % (uint64_t)(i + 1);
        uint32_t t = p[i]; p[i] = p[j]; p[j] = t;
    }
    return p;
}

int gen_rmat(int scale, int edgefactor, double a, double b, double c, uint64_t seed,
             int permute, gen_csr *out) {
    if (scale < 1 || scale > 30 || edgefactor < 1) return -2;
    int64_t n = (int64_t)1 << scale;
    int64_t m = (int64_t)edgefactor * n;
    uint32_t *U = (uint32_t *)malloc((size_t)m * sizeof(uint32_t));
    uint32_t *V = (uint32_t *)malloc((size_t)m * sizeof(uint32_t));
    if (!U || !V) { free(U); free(V); return -1; }
    double ab = a + b, abc = a + b + c;
#pragma omp parallel for schedule(static)
    for (int64_t k = 0; k < m; ++k) {
        uint32_t u = 0, v = 0;
        for (int l = 0; l < scale; ++l) {
            double r = u01(crng(seed, 1, (uint64_t)k * (uint64_t)scale + (uint64_t)l));
            uint32_t bu, bv;
            if (r < a) { bu = 0; bv = 0; }
            else if (r < ab) { bu = 0; bv = 1; }
            else if (r < abc) { bu = 1; bv = 0; }
            else { bu = 1; bv = 1; }
            u = (u << 1) | bu; v = (v << 1) | bv;
        }
        U[k] = u; V[k] = v;
    }
    if (permute) {
        uint32_t *p = make_perm(n, seed);
        if (!p) { free(U); free(V); return -1; }
#pragma omp parallel for schedule(static)
        for (int64_t k = 0; k < m; ++k) { U[k] = p[U[k]]; V[k] = p[V[k]]; }
        free(p);
    }
    int rc = build_csr(n, m, U, V, out);
    free(U); free(V);
    return rc;
}

/* The l-th R-MAT tuple of gen_rmat (before the permutation). */
static inline void rmat_tuple(int scale, double a, double ab, double abc, uint64_t seed, int64_t k,
                              uint32_t *pu, uint32_t *pv) {
    uint32_t u = 0, v = 0;
    for (int l = 0; l < scale; ++l) {
        double r = u01(crng(seed, 1, (uint64_t)k * (uint64_t)scale + (uint64_t)l));
        uint32_t bu, bv;
        if (r < a) { bu = 0; bv = 0; }
        else if (r < ab) { bu = 0; bv = 1; }
        else if (r < abc) { bu = 1; bv = 0; }
        else { bu = 1; bv = 1; }
        u = (u << 1) | bu; v = (v << 1) | bv;
    }
    *pu = u; *pv = v;
}

/* Rows [vb, ve) of exactly the graph gen_rmat builds (same tuples, permutation, symmetrisation,
 * loop removal and per-row dedupe), with offsets rebased to 0 (out->n = ve - vb rows, columns are
 * global ids).  No tuple array is held: the tuples are regenerated twice (count, then fill), so
 * memory is the slice's CSR plus the permutation.  This is how each rank of the partitioned C5
 * runs builds only its own rows, and with [0, n) a memory-light parallel builder of
 * the whole graph. */
int gen_rmat_slice(int scale, int edgefactor, double a, double b, double c, uint64_t seed,
                   int permute, int64_t vb, int64_t ve, gen_csr *out) {
    if (scale < 1 || scale > 30 || edgefactor < 1) return -2;
    const int64_t n = (int64_t)1 << scale, m = (int64_t)edgefactor * n;
    if (vb < 0 || ve > n || vb > ve) return -2;
    const int64_t rows = ve - vb;
    const double ab = a + b, abc = a + b + c;
    uint32_t *p = permute ? make_perm(n, seed) : NULL;
    if (permute && !p) return -1;
    int64_t *cnt = (int64_t *)calloc((size_t)rows + 1, sizeof(int64_t));
    if (!cnt) { free(p); return -1; }
#pragma omp parallel for schedule(static)
    for (int64_t k = 0; k < m; ++k) {
        uint32_t u, v;
        rmat_tuple(scale, a, ab, abc, seed, k, &u, &v);
        if (p) { u = p[u]; v = p[v]; }
        if (u == v) continue;
        if ((int64_t)u >= vb && (int64_t)u < ve) __atomic_fetch_add(&cnt[u - vb + 1], 1, __ATOMIC_RELAXED);
        if ((int64_t)v >= vb && (int64_t)v < ve) __atomic_fetch_add(&cnt[v - vb + 1], 1, __ATOMIC_RELAXED);
    }
    for (int64_t i = 0; i < rows; ++i) cnt[i + 1] += cnt[i];
    const int64_t tot = cnt[rows];
    int32_t *col = (int32_t *)malloc((size_t)(tot ? tot : 1) * sizeof(int32_t));
    int64_t *pos = (int64_t *)malloc((size_t)(rows ? rows : 1) * sizeof(int64_t));
    if (!col || !pos) { free(p); free(cnt); free(col); free(pos); return -1; }
    memcpy(pos, cnt, (size_t)rows * sizeof(int64_t));
#pragma omp parallel for schedule(static)
    for (int64_t k = 0; k < m; ++k) {
        uint32_t u, v;
        rmat_tuple(scale, a, ab, abc, seed, k, &u, &v);
        if (p) { u = p[u]; v = p[v]; }
        if (u == v) continue;
        if ((int64_t)u >= vb && (int64_t)u < ve) col[__atomic_fetch_add(&pos[u - vb], 1, __ATOMIC_RELAXED)] = (int32_t)v;
        if ((int64_t)v >= vb && (int64_t)v < ve) col[__atomic_fetch_add(&pos[v - vb], 1, __ATOMIC_RELAXED)] = (int32_t)u;
    }
    free(p);
    free(pos);
    int64_t *deg = (int64_t *)malloc((size_t)(rows ? rows : 1) * sizeof(int64_t));
    if (!deg) { free(cnt); free(col); return -1; }
#pragma omp parallel for schedule(dynamic, 1024)
    for (int64_t i = 0; i < rows; ++i) {
        int32_t *r = col + cnt[i];
        int64_t len = cnt[i + 1] - cnt[i];
        if (len > 1) qsort(r, (size_t)len, sizeof(int32_t), cmp_i32);
        int64_t k = 0;
        for (int64_t j = 0; j < len; ++j)
            if (k == 0 || r[j] != r[k - 1]) r[k++] = r[j];
        deg[i] = k;
    }
    int64_t *off = (int64_t *)malloc(((size_t)rows + 1) * sizeof(int64_t));
    if (!off) { free(cnt); free(col); free(deg); return -1; }
    off[0] = 0;
    for (int64_t i = 0; i < rows; ++i) off[i + 1] = off[i] + deg[i];
    /* compact in place: rows move only towards lower addresses (off[i] <= cnt[i]) */
    for (int64_t i = 0; i < rows; ++i)
        if (off[i] != cnt[i]) memmove(col + off[i], col + cnt[i], (size_t)deg[i] * sizeof(int32_t));
    free(cnt); free(deg);
    out->n = rows; out->nnz = off[rows]; out->off = off; out->col = col; out->w = NULL;
    return 0;
}

int gen_grid(int64_t width, int64_t height, gen_csr *out) {
    if (width < 1 || height < 1) return -2;
    int64_t n = width * height;
    int64_t *off = (int64_t *)malloc(((size_t)n + 1) * sizeof(int64_t));
    if (!off) return -1;
    off[0] = 0;
    for (int64_t i = 0; i < height; ++i)
        for (int64_t j = 0; j < width; ++j) {
            int64_t d = (i > 0) + (j > 0) + (j + 1 < width) + (i + 1 < height);
            off[i * width + j + 1] = off[i * width + j] + d;
        }
    int64_t nnz = off[n];
    int32_t *col = (int32_t *)malloc((size_t)(nnz ? nnz : 1) * sizeof(int32_t));
    if (!col) { free(off); return -1; }
#pragma omp parallel for schedule(static)
    for (int64_t i = 0; i < height; ++i)
        for (int64_t j = 0; j < width; ++j) {
            int64_t id = i * width + j, p = off[id];
            if (i > 0) col[p++] = (int32_t)(id - width);
            if (j > 0) col[p++] = (int32_t)(id - 1);
            if (j + 1 < width) col[p++] = (int32_t)(id + 1);
            if (i + 1 < height) col[p++] = (int32_t)(id + width);
        }
    out->n = n; out->nnz = nnz; out->off = off; out->col = col; out->w = NULL;
    return 0;
}

int gen_chung_lu(int64_t n, int64_t pairs, double gamma, double i0, uint64_t seed, gen_csr *out) {
    if (n < 2 || pairs < 0 || gamma <= 1.0) return -2;
    double *cdf = (double *)malloc((size_t)n * sizeof(double));
    if (!cdf) return -1;
    double ex = -1.0 / (gamma - 1.0), s = 0.0;
    for (int64_t i = 0; i < n; ++i) { s += pow((double)i + i0, ex); cdf[i] = s; }
    for (int64_t i = 0; i < n; ++i) cdf[i] /= s;
    cdf[n - 1] = 1.0;
    uint32_t *U = (uint32_t *)malloc((size_t)(pairs ? pairs : 1) * sizeof(uint32_t));
    uint32_t *V = (uint32_t *)malloc((size_t)(pairs ? pairs : 1) * sizeof(uint32_t));
    uint32_t *p = make_perm(n, seed);
    if (!U || !V || !p) { free(cdf); free(U); free(V); free(p); return -1; }
#pragma omp parallel for schedule(static)
    for (int64_t k = 0; k < pairs; ++k) {
        for (int e = 0; e < 2; ++e) {
            double r = u01(crng(seed, 3, 2 * (uint64_t)k + (uint64_t)e));
            int64_t lo = 0, hi = n - 1;           /* first i with cdf[i] > r */
            while (lo < hi) { int64_t mid = (lo + hi) / 2; if (cdf[mid] > r) hi = mid; else lo = mid + 1; }
            if (e == 0) U[k] = p[lo]; else V[k] = p[lo];
        }
    }
    free(cdf); free(p);
    int rc = build_csr(n, pairs, U, V, out);
    free(U); free(V);
    return rc;
}

/* Symmetric hash weights in [1, maxw]: w(u,v) = 1 + splitmix64((min*N+max) ^ seed) % maxw. */
int gen_hash_weights(gen_csr *g, uint64_t seed, uint32_t maxw) {
    if (maxw < 1) return -2;
    uint32_t *w = (uint32_t *)malloc((size_t)(g->nnz ? g->nnz : 1) * sizeof(uint32_t));
    if (!w) return -1;
    uint64_t N = (uint64_t)g->n;
#pragma omp parallel for schedule(dynamic, 4096)
    for (int64_t u = 0; u < g->n; ++u)
        for (int64_t e = g->off[u]; e < g->off[u + 1]; ++e) {
            uint64_t v = (uint64_t)g->col[e];
            uint64_t lo = (uint64_t)u < v ? (uint64_t)u : v, hi = (uint64_t)u < v ? v : (uint64_t)u;
            w[e] = 1u + (uint32_t)(splitmix64((lo * N + hi) ^ seed) % maxw);
        }
    free(g->w);
    g->w = w;
    return 0;
}
