/*
 * oracle.c -- plain, slow, obviously-correct CPU reference for GSWITCH's frontier-step hot path.
 *
 * TEST INFRASTRUCTURE ONLY.  Only tests/, __graft_entry__.smoke() and bench.py's cpu_baseline /
 * --impl reference legs may load or call this library.  The product path (the CUDA library under
 * paper_conf_ppopp_menglts19_b200/csrc) shares no code, header, table or helper with this file,
 * and neither side includes or links the other.
 *
 * Every function computes the plain definition of what the method computes,
 * in the textbook order.  Citations are PAPER.md line numbers ("P:nnn").  Everything is single-
 * threaded except the per-vertex loops of orc_pr and orc_dpr, which OpenMP spreads over vertices:
 * each vertex's sum is still computed by one thread in ascending in-edge order and the dangling
 * mass / activation counts stay serial, so the result is bit-identical to the serial loop
 * (tests/test_oracle.py checks 1 thread vs all); this only makes full-size checks (C3 Delta-PR,
 * C5 PageRank) finish in minutes.  orc_set_threads(k) pins the thread count (0 = OpenMP default).
 *
 *   orc_bfs          FIFO-queue BFS depths                    P:262-263 ([7]); Fig. 11
 *   orc_bfs_features per-level Va/Ea/Via/Eia of the BFS        Table 1; record R P:948-951
 *   orc_sssp         binary-heap Dijkstra (lazy deletion)      P:264-265 ([42]); footnote 2 P:411-413
 *   orc_cc           union-find, labels = min vertex id        P:263-264 ([53]); north_star
 *   orc_pr           fp64 power iteration, dangling mass       P:264 ([11]); SURVEY Q9
 *   orc_dpr          Delta-PageRank, fp64, threshold eps       P:386-388 ([19]); Fig. 3; DESIGN R16
 *   orc_bc           Brandes, sigma u64, delta fp64            P:265-266 ([47],[10] P:1584-1585)
 *   orc_attrs        dataset attributes N,M,dbar,sd,rd,GI,Her  Table 1; [29]
 *   orc_ratios       Vap,Eap,Viap,Eiap,cd from counts          Table 1; record R P:948-951
 *
 * Parity pins (tests/test_oracle.py): brute force on tiny graphs (Floyd-Warshall, transitive
 * closure, dense Google matrix, explicit shortest-path enumeration), closed forms (grid depth i+j,
 * regular-graph PR = 1/N, exact-rational star/path PR, path/star BC), invariants (Graph500 BFS
 * checks, SSSP triangle/tightness, PR mass conservation, CC label checks, Brandes sum identity) and
 * the record-R arithmetic for the feature ratios.  orc_ratios' r_cd is NOT computed here
 * ("parity unpinned": the printed 137.7 in record R is not recoverable).
 */
#include <stdint.h>
#include <stdlib.h>
#include <string.h>
#include <math.h>
#ifdef _OPENMP
#include <omp.h>
#endif

#define ORC_OK 0
#define ORC_ENOMEM (-1)
#define ORC_EINVAL (-2)
#define ORC_EOVERFLOW (-3)

void orc_set_threads(int k) {
#ifdef _OPENMP
    omp_set_num_threads(k > 0 ? k : omp_get_num_procs());
#else
    (void)k;
#endif
}

int orc_threads(void) {
#ifdef _OPENMP
    return omp_get_max_threads();
#else
    return 1;
#endif
}

/* ---------------------------------------------------------------- BFS (FIFO) */
int orc_bfs(int64_t n, const int64_t *off, const int32_t *col, int32_t src, int32_t *depth) {
    if (n <= 0 || src < 0 || src >= n) return ORC_EINVAL;
    int32_t *q = (int32_t *)malloc((size_t)n * sizeof(int32_t));
    if (!q) return ORC_ENOMEM;
    for (int64_t v = 0; v < n; ++v) depth[v] = -1;          /* unvisited: level < 0 (Fig. 11) */
    int64_t head = 0, tail = 0;
    depth[src] = 0;                                          /* source level 0 */
    q[tail++] = src;
    while (head < tail) {
        int32_t u = q[head++];
        for (int64_t e = off[u]; e < off[u + 1]; ++e) {
            int32_t v = col[e];
            if (depth[v] < 0) {                              /* emit(u) = level+1 */
                depth[v] = depth[u] + 1;
                q[tail++] = v;
            }
        }
    }
    free(q);
    return ORC_OK;
}

/*
 * Per-iteration runtime characteristics of level-synchronous BFS (Table 1).
 * Iteration t has active set F_t = {v : depth[v] == t}.  "Inactive" = not yet visited when
 * iteration t starts = {v : depth[v] > t or depth[v] == -1}  (record R: N - Va - Via = Fixed).
 *   Va[t] = |F_t|, Ea[t] = sum_{v in F_t} deg(v), Via[t] = |inactive|, Eia[t] = sum deg(inactive).
 * Returns the number of iterations L (levels 0..L-1 have Va > 0), or a negative error.
 */
int64_t orc_bfs_features(int64_t n, const int64_t *off, const int32_t *col, int32_t src,
                         int64_t *Va, int64_t *Ea, int64_t *Via, int64_t *Eia, int64_t max_levels) {
    int32_t *depth = (int32_t *)malloc((size_t)n * sizeof(int32_t));
    if (!depth) return ORC_ENOMEM;
    int rc = orc_bfs(n, off, col, src, depth);
    if (rc) { free(depth); return rc; }
    int64_t L = 0;
    for (int64_t v = 0; v < n; ++v) if (depth[v] + 1 > L) L = depth[v] + 1;
    if (L > max_levels) { free(depth); return ORC_EINVAL; }
    for (int64_t t = 0; t < L; ++t) {
        int64_t va = 0, ea = 0, via = 0, eia = 0;
        for (int64_t v = 0; v < n; ++v) {
            int64_t d = off[v + 1] - off[v];
            if (depth[v] == t) { va++; ea += d; }
            else if (depth[v] < 0 || depth[v] > t) { via++; eia += d; }
        }
        Va[t] = va; Ea[t] = ea; Via[t] = via; Eia[t] = eia;
    }
    free(depth);
    return L;
}

/* ---------------------------------------------------------------- SSSP (Dijkstra) */
typedef struct { uint64_t d; int32_t v; } hitem;

static void heap_push(hitem *h, int64_t *sz, hitem x) {
    int64_t i = (*sz)++;
    while (i > 0) {
        int64_t p = (i - 1) / 2;
        if (h[p].d <= x.d) break;
        h[i] = h[p]; i = p;
    }
    h[i] = x;
}
static hitem heap_pop(hitem *h, int64_t *sz) {
    hitem top = h[0], x = h[--(*sz)];
    int64_t i = 0;
    for (;;) {
        int64_t c = 2 * i + 1;
        if (c >= *sz) break;
        if (c + 1 < *sz && h[c + 1].d < h[c].d) c++;
        if (h[c].d >= x.d) break;
        h[i] = h[c]; i = c;
    }
    if (*sz > 0) h[i] = x;
    return top;
}

/* dist[s]=0; dist[v] = min over paths of sum w; UINT32_MAX if unreachable.  u64 internally. */
int orc_sssp(int64_t n, const int64_t *off, const int32_t *col, const uint32_t *w, int32_t src,
             uint32_t *dist) {
    if (n <= 0 || src < 0 || src >= n || !w) return ORC_EINVAL;
    uint64_t *D = (uint64_t *)malloc((size_t)n * sizeof(uint64_t));
    int64_t cap = off[n] + 1;
    hitem *h = (hitem *)malloc((size_t)cap * sizeof(hitem));
    if (!D || !h) { free(D); free(h); return ORC_ENOMEM; }
    for (int64_t v = 0; v < n; ++v) D[v] = UINT64_MAX;
    int64_t sz = 0;
    D[src] = 0;
    heap_push(h, &sz, (hitem){0, src});
    while (sz > 0) {
        hitem it = heap_pop(h, &sz);
        if (it.d != D[it.v]) continue;                       /* lazy deletion */
        for (int64_t e = off[it.v]; e < off[it.v + 1]; ++e) {
            uint64_t nd = it.d + (uint64_t)w[e];
            int32_t v = col[e];
            if (nd < D[v]) { D[v] = nd; heap_push(h, &sz, (hitem){nd, v}); }
        }
    }
    int rc = ORC_OK;
    for (int64_t v = 0; v < n; ++v) {
        if (D[v] == UINT64_MAX) dist[v] = UINT32_MAX;
        else if (D[v] >= UINT32_MAX) { rc = ORC_EOVERFLOW; dist[v] = UINT32_MAX; }
        else dist[v] = (uint32_t)D[v];
    }
    free(D); free(h);
    return rc;
}

/* ---------------------------------------------------------------- CC (union-find) */
static int32_t uf_find(int32_t *p, int32_t x) {
    while (p[x] != x) { p[x] = p[p[x]]; x = p[x]; }          /* path halving */
    return x;
}

/* label[v] = min{u : u connected to v} */
int orc_cc(int64_t n, const int64_t *off, const int32_t *col, int32_t *label) {
    if (n < 0) return ORC_EINVAL;
    int32_t *p = (int32_t *)malloc((size_t)(n ? n : 1) * sizeof(int32_t));
    int32_t *sz = (int32_t *)malloc((size_t)(n ? n : 1) * sizeof(int32_t));
    int32_t *mn = (int32_t *)malloc((size_t)(n ? n : 1) * sizeof(int32_t));
    if (!p || !sz || !mn) { free(p); free(sz); free(mn); return ORC_ENOMEM; }
    for (int64_t v = 0; v < n; ++v) { p[v] = (int32_t)v; sz[v] = 1; }
    for (int64_t u = 0; u < n; ++u)
        for (int64_t e = off[u]; e < off[u + 1]; ++e) {
            int32_t a = uf_find(p, (int32_t)u), b = uf_find(p, col[e]);
            if (a == b) continue;
            if (sz[a] < sz[b]) { int32_t t = a; a = b; b = t; }   /* union by size */
            p[b] = a; sz[a] += sz[b];
        }
    for (int64_t v = 0; v < n; ++v) mn[v] = INT32_MAX;
    for (int64_t v = 0; v < n; ++v) {
        int32_t r = uf_find(p, (int32_t)v);
        if ((int32_t)v < mn[r]) mn[r] = (int32_t)v;
    }
    for (int64_t v = 0; v < n; ++v) label[v] = mn[uf_find(p, (int32_t)v)];
    free(p); free(sz); free(mn);
    return ORC_OK;
}

/* ---------------------------------------------------------------- PageRank (fp64) */
/*
 * pr_0 = 1/N.  For t < T:  D_t = sum_{deg_out(u)=0} pr_t(u)
 *   pr_{t+1}(v) = (1-d)/N + d * ( sum_{u in N_in(v)} pr_t(u)/deg_out(u) + D_t/N )
 * In-neighbours from the CSC (csc_off/csc_col); out-degree from the CSR offsets.  For the
 * symmetric graphs of every config CSC == CSR.  Pull order: ascending position in the CSC row.
 */
int orc_pr(int64_t n, const int64_t *csr_off, const int64_t *csc_off, const int32_t *csc_col,
           double d, int32_t iters, double *pr) {
    if (n <= 0 || iters < 0) return ORC_EINVAL;
    double *nxt = (double *)malloc((size_t)n * sizeof(double));
    if (!nxt) return ORC_ENOMEM;
    double N = (double)n;
    for (int64_t v = 0; v < n; ++v) pr[v] = 1.0 / N;
    for (int32_t t = 0; t < iters; ++t) {
        double D = 0.0;
        for (int64_t u = 0; u < n; ++u)
            if (csr_off[u + 1] == csr_off[u]) D += pr[u];
#pragma omp parallel for schedule(dynamic, 4096)
        for (int64_t v = 0; v < n; ++v) {
            double s = 0.0;
            for (int64_t e = csc_off[v]; e < csc_off[v + 1]; ++e) {
                int32_t u = csc_col[e];
                s += pr[u] / (double)(csr_off[u + 1] - csr_off[u]);
            }
            nxt[v] = (1.0 - d) / N + d * (s + D / N);
        }
        memcpy(pr, nxt, (size_t)n * sizeof(double));
    }
    free(nxt);
    return ORC_OK;
}

/* ---------------------------------------------------------------- Delta-PageRank (fp64) */
/*
 * Delta-PageRank ([19]; Fig. 3 "Iteration No. of Delta-PR"), reading R16.
 * Each vertex holds a rank r and an unpropagated residual delta.  With M(w,v) = 1/deg_out(v) for
 * every edge v->w (no dangling teleport), the fixed point is x = (1-d)/N 1 + d M x, and
 *   delta_0(v) = (1-d)/N,  r_0 = 0;   iteration t:
 *     A_t = { v : delta_t(v) > eps }                                     (Filter: active set)
 *     r(v) += delta_t(v)                                 for v in A_t
 *     delta_{t+1}(w) = [w not in A_t] delta_t(w) + sum_{v in A_t, v->w} d delta_t(v)/deg_out(v)
 *                                                                         (Expand)
 *   stop when A_t is empty or after max_iters iterations.
 * Invariant: x = r + (I - dM)^{-1} delta, so 0 <= x - r and ||x - r||_1 <= ||delta||_1/(1-d).
 * eps < 0 makes every vertex active every iteration: r is then the Neumann partial sum
 * sum_{k<T} (dM)^k (1-d)/N 1.  Sums in ascending in-edge order (csc_off/csc_col).
 * iters_out: iterations executed (the last, empty A_t is not counted).
 */
int orc_dpr(int64_t n, const int64_t *csr_off, const int64_t *csc_off, const int32_t *csc_col,
            double d, double eps, int32_t max_iters, double *r, int32_t *iters_out) {
    if (n <= 0 || max_iters < 0) return ORC_EINVAL;
    double *delta = (double *)malloc((size_t)n * sizeof(double));
    double *nxt = (double *)malloc((size_t)n * sizeof(double));
    char *act = (char *)malloc((size_t)n);
    if (!delta || !nxt || !act) { free(delta); free(nxt); free(act); return ORC_ENOMEM; }
    for (int64_t v = 0; v < n; ++v) { r[v] = 0.0; delta[v] = (1.0 - d) / (double)n; }
    int32_t t = 0;
    for (; t < max_iters; ++t) {
        int64_t na = 0;
        for (int64_t v = 0; v < n; ++v) { act[v] = delta[v] > eps; na += act[v]; }
        if (na == 0) break;
        for (int64_t v = 0; v < n; ++v)
            if (act[v]) r[v] += delta[v];
#pragma omp parallel for schedule(dynamic, 4096)
        for (int64_t w = 0; w < n; ++w) {
            double s = 0.0;
            for (int64_t e = csc_off[w]; e < csc_off[w + 1]; ++e) {
                int32_t v = csc_col[e];
                if (act[v]) s += d * delta[v] / (double)(csr_off[v + 1] - csr_off[v]);
            }
            nxt[w] = (act[w] ? 0.0 : delta[w]) + s;
        }
        memcpy(delta, nxt, (size_t)n * sizeof(double));
    }
    if (iters_out) *iters_out = t;
    free(delta); free(nxt); free(act);
    return ORC_OK;
}

/* ---------------------------------------------------------------- BC (Brandes) */
/*
 * bc[v] = sum_{s in S, s != v} delta_s(v),
 * delta_s(v) = sum_{w : v in pred_s(w)} sigma_sv/sigma_sw * (1 + delta_s(w)).
 * sigma exact in u64 (returns ORC_EOVERFLOW if any sigma >= 2^63), delta in fp64.  No
 * normalisation, no halving for undirected graphs.
 */
int orc_bc(int64_t n, const int64_t *off, const int32_t *col, const int32_t *sources, int32_t nsrc,
           double *bc) {
    if (n <= 0 || nsrc < 0) return ORC_EINVAL;
    int32_t *depth = (int32_t *)malloc((size_t)n * sizeof(int32_t));
    int32_t *stack = (int32_t *)malloc((size_t)n * sizeof(int32_t));
    uint64_t *sigma = (uint64_t *)malloc((size_t)n * sizeof(uint64_t));
    double *delta = (double *)malloc((size_t)n * sizeof(double));
    if (!depth || !stack || !sigma || !delta) {
        free(depth); free(stack); free(sigma); free(delta); return ORC_ENOMEM;
    }
    int rc = ORC_OK;
    for (int64_t v = 0; v < n; ++v) bc[v] = 0.0;
    for (int32_t k = 0; k < nsrc; ++k) {
        int32_t s = sources[k];
        if (s < 0 || s >= n) { rc = ORC_EINVAL; break; }
        for (int64_t v = 0; v < n; ++v) { depth[v] = -1; sigma[v] = 0; delta[v] = 0.0; }
        int64_t head = 0, tail = 0;
        depth[s] = 0; sigma[s] = 1; stack[tail++] = s;
        while (head < tail) {                                 /* BFS, stack = visit order */
            int32_t u = stack[head++];
            for (int64_t e = off[u]; e < off[u + 1]; ++e) {
                int32_t v = col[e];
                if (depth[v] < 0) { depth[v] = depth[u] + 1; stack[tail++] = v; }
                if (depth[v] == depth[u] + 1) {
                    if (sigma[v] > (UINT64_C(1) << 63) - 1 - sigma[u]) rc = ORC_EOVERFLOW;
                    sigma[v] += sigma[u];
                }
            }
        }
        for (int64_t i = tail - 1; i >= 0; --i) {             /* dependency accumulation */
            int32_t w = stack[i];
            for (int64_t e = off[w]; e < off[w + 1]; ++e) {
                int32_t v = col[e];
                if (depth[v] == depth[w] - 1)
                    delta[v] += (double)sigma[v] / (double)sigma[w] * (1.0 + delta[w]);
            }
            if (w != s) bc[w] += delta[w];
        }
    }
    free(depth); free(stack); free(sigma); free(delta);
    return rc;
}

/* ---------------------------------------------------------------- features */
static int cmp_i64(const void *a, const void *b) {
    int64_t x = *(const int64_t *)a, y = *(const int64_t *)b;
    return (x > y) - (x < y);
}

/*
 * Dataset attributes (Table 1), out[0..6] = N, M, dbar, sigma_d, r_d, Gini, H_er.
 *   M = nnz/2 (undirected edges; record R: dbar = 2M/N = 28.2), dbar = 2M/N,
 *   sigma_d = population standard deviation of deg, r_d = (d_max - d_min)/dbar,
 *   Gini = sum_i (2i - N - 1) d_(i) / (N sum d)   over ascending d_(1..N)  ([29]),
 *   H_er = -sum_i (d_i/2M) ln(d_i/2M) / ln N      (0 ln 0 = 0)            ([29]).
 */
int orc_attrs(int64_t n, const int64_t *off, double *out) {
    if (n <= 0) return ORC_EINVAL;
    int64_t *d = (int64_t *)malloc((size_t)n * sizeof(int64_t));
    if (!d) return ORC_ENOMEM;
    int64_t sum = 0, dmin = INT64_MAX, dmax = 0;
    for (int64_t v = 0; v < n; ++v) {
        d[v] = off[v + 1] - off[v]; sum += d[v];
        if (d[v] < dmin) dmin = d[v];
        if (d[v] > dmax) dmax = d[v];
    }
    double N = (double)n, twoM = (double)sum, dbar = twoM / N;
    double var = 0.0;
    for (int64_t v = 0; v < n; ++v) var += ((double)d[v] - dbar) * ((double)d[v] - dbar);
    var /= N;
    double H = 0.0;
    for (int64_t v = 0; v < n; ++v)
        if (d[v] > 0) { double p = (double)d[v] / twoM; H -= p * log(p); }
    qsort(d, (size_t)n, sizeof(int64_t), cmp_i64);
    double g = 0.0;
    for (int64_t i = 1; i <= n; ++i) g += (double)(2 * i - n - 1) * (double)d[i - 1];
    out[0] = N;
    out[1] = twoM / 2.0;
    out[2] = dbar;
    out[3] = sqrt(var);
    out[4] = dbar > 0 ? (double)(dmax - dmin) / dbar : 0.0;
    out[5] = sum > 0 ? g / (N * twoM) : 0.0;
    out[6] = (sum > 0 && n > 1) ? H / log(N) : 0.0;
    free(d);
    return ORC_OK;
}

/* Ratios of Table 1: out = Vap, Eap, Viap, Eiap, cd. */
void orc_ratios(int64_t N, int64_t M, int64_t Va, int64_t Ea, int64_t Via, int64_t Eia, double *out) {
    out[0] = (double)Va / (double)N;
    out[1] = (double)Ea / (2.0 * (double)M);
    out[2] = (double)Via / (double)N;
    out[3] = (double)Eia / (2.0 * (double)M);
    out[4] = Va > 0 ? (double)Ea / (double)Va : 0.0;
}
