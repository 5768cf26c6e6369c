/*
 * gsw.h -- C ABI of the B200-native GSWITCH frontier-step library (libgsw.so).
 *
 * What it computes.  GSWITCH standardises a BSP graph algorithm as a two-phase per-iteration
 * process: "The filtering step (Filter) generates the active set and updates their private data;
 * then the expansion step (Expand) processes all the neighbors of the generated active set"
 * (Sec. 2.1).  An algorithm "terminates with no more active elements"
 * (P:251-252).  Every iteration the library extracts runtime features (Table 1), runs
 * a decision-tree selector over the five patterns in the order direction -> load balance ->
 * active-set format -> stepping -> fusion and executes the selected Filter/Expand
 * variant.  All of this runs on the device inside one persistent kernel per run;
 * the host is crossed only at entry and at the final synchronisation.
 *
 * Conventions (all functions):
 *   - Vertex ids are int32 in [0, n).  n < 2^31, nnz < 2^32 (else GSW_EOVERFLOW).
 *   - Array arguments may be HOST or DEVICE pointers: the library classifies every pointer with
 *     cudaPointerGetAttributes and copies host data in / results out on the handle's stream.
 *   - Every call is synchronous: it returns after its work on the handle's stream completed, so
 *     outputs and stats are valid on return.
 *   - The library never aborts.  A non-OK status leaves a message in gsw_last_error() (thread
 *     local).  CUDA errors map to GSW_ECUDA, NCCL errors to GSW_ENCCL.
 *   - A handle is not thread-safe: one call at a time per handle.  Separate handles on separate
 *     streams are independent.
 *   - Memory: the library allocates no device memory of its own.  The caller queries
 *     gsw_workspace_size(), allocates one device buffer (e.g. a torch uint8 tensor) and passes it
 *     to gsw_graph_create(); the graph copy and all per-run scratch live in it.  The caller keeps
 *     it alive until gsw_graph_destroy().
 */
#ifndef GSW_H
#define GSW_H

#include <stddef.h>
#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

typedef enum {
    GSW_OK = 0,
    GSW_EINVAL = 1,          /* bad argument (null pointer, source out of range, bad CSR ...)   */
    GSW_ENOMEM = 2,          /* workspace too small                                             */
    GSW_ECUDA = 3,           /* a CUDA runtime/driver call or kernel failed                     */
    GSW_ENCCL = 4,           /* an NCCL call failed                                             */
    GSW_EUNSUPPORTED = 5,    /* forced configuration not valid for this algorithm               */
    GSW_EOVERFLOW = 6        /* sizes or path lengths exceed the 32-bit internal representation */
} gsw_status;

typedef struct gsw_graph_s *gsw_graph;

/* CSR (out-edges) or CSC (in-edges).  Caller-owned; copied by gsw_graph_create. */
typedef struct {
    int64_t n;                    /* vertices                                                  */
    int64_t nnz;                  /* directed entries (= 2x undirected edges for symmetric)    */
    const int64_t *row_offsets;   /* n+1, non-decreasing, row_offsets[0]=0, [n]=nnz            */
    const int32_t *col_indices;   /* nnz, each in [0,n)                                        */
    const uint32_t *weights;      /* nnz or NULL; required by gsw_sssp                         */
} gsw_csr;

/* ---- pattern candidates (Sec. 3).  0 = AUTO (selector decides each iteration) ---- */
enum { GSW_AUTO = 0 };
/* Pattern 1, direction */
enum { GSW_PUSH = 1, GSW_PULL = 2 };
/* Pattern 2, active-set format */
enum { GSW_BITMAP = 1, GSW_QUEUE = 2, GSW_SORTED_QUEUE = 3 };
/* Pattern 3, load balance; THREAD = naive one-thread-per-vertex (north_star) */
enum { GSW_LB_THREAD = 1, GSW_LB_TWC = 2, GSW_LB_WM = 3, GSW_LB_CM = 4, GSW_LB_STRICT = 5 };
/* Pattern 4, stepping: SSSP priority threshold control.
 *   INCREASE/DECREASE/REMAIN pin the per-iteration decision of the dynamic controller;
 *   STATIC = classic delta-stepping with fixed delta0 (theta += delta0 when the near set empties);
 *   UNORDERED = Bellman-Ford (theta = infinity).                                                  */
enum { GSW_STEP_INCREASE = 1, GSW_STEP_DECREASE = 2, GSW_STEP_REMAIN = 3,
       GSW_STEP_STATIC = 4, GSW_STEP_UNORDERED = 5 };
/* Pattern 5, kernel fusion */
enum { GSW_STANDALONE = 1, GSW_FUSED = 2 };

typedef struct {
    int32_t direction;      /* AUTO | GSW_PUSH | GSW_PULL                                     */
    int32_t format;         /* AUTO | GSW_BITMAP | GSW_QUEUE | GSW_SORTED_QUEUE               */
    int32_t load_balance;   /* AUTO | GSW_LB_*                                                */
    int32_t stepping;       /* AUTO | GSW_STEP_*  (ignored by all algorithms but SSSP)        */
    int32_t fusion;         /* AUTO | GSW_STANDALONE | GSW_FUSED                              */
    uint32_t delta0;        /* SSSP threshold step; 0 = c*wbar/dbar with c=32     */
} gsw_config;

/* One record per iteration (the paper's per-iteration feedback). */
typedef struct {
    int32_t iteration;
    int32_t direction, format, load_balance, stepping, fusion;   /* the executed variant     */
    int64_t Va, Ea, Via, Eia;     /* runtime characteristics of the active set (Table 1)       */
    int64_t edges;                /* adjacency entries read by this iteration's Expand          */
    uint32_t theta;               /* SSSP priority threshold in force (0 for other algorithms) */
    float filter_us, expand_us;   /* device time of the Filter and Expand phases (%globaltimer)*/
    int32_t ctas;                 /* CTAs that executed the iteration: the persistent grid, or 1
                                     in the CTA-resident tier for tiny active sets */
} gsw_iter_record;

typedef struct {
    int32_t iterations;           /* BSP iterations executed (summed over sources for BC)      */
    float gpu_ms;                 /* device time of the run, CUDA events on the handle stream  */
    int64_t edges_touched;        /* adjacency entries read by Expand (summed over iterations)  */
    int64_t bytes_alg;            /* algorithmic HBM bytes (roofline model D0)      */
    gsw_iter_record *records;     /* optional HOST buffer of max_records entries, or NULL      */
    int32_t max_records;          /* records beyond this many are counted but not stored        */
} gsw_run_stats;

/* Bytes of device workspace gsw_graph_create needs for a graph of this size. */
gsw_status gsw_workspace_size(int64_t n, int64_t nnz, int32_t has_weights, int32_t has_csc,
                              size_t *bytes);

/*
 * Copy a CSR (and optionally a separate CSC for directed graphs; NULL = symmetric, the CSC is the
 * CSR -- all paper inputs are undirected) into the workspace, converting offsets to u32,
 * and compute the dataset attributes of Table 1 (N, M, dbar, sigma_d, r_d, Gini, H_er, P:752-759,
 * "computed only once while loading the data").
 *   workspace: DEVICE buffer of >= gsw_workspace_size() bytes, 256-byte aligned.
 *   cuda_stream: cudaStream_t (NULL = legacy default stream) used by every call on the handle.
 * Errors: GSW_EINVAL (nulls, n<=0, nnz mismatch), GSW_ENOMEM (workspace too small),
 *         GSW_EOVERFLOW (n >= 2^31 or nnz >= 2^32).  The CSR contents are not validated beyond
 *         offsets[0]==0 and offsets[n]==nnz (use gsw_graph_validate).
 */
gsw_status gsw_graph_create(const gsw_csr *csr, const gsw_csr *csc, void *workspace,
                            size_t ws_bytes, void *cuda_stream, gsw_graph *out);
gsw_status gsw_graph_destroy(gsw_graph g);
/* Full device-side check: monotone offsets and every column in range (GSW_EINVAL otherwise). */
gsw_status gsw_graph_validate(gsw_graph g);

/* Dataset attributes of Table 1, out[0..6] = N, M, dbar, sigma_d, r_d, Gini, H_er. */
gsw_status gsw_graph_attributes(gsw_graph g, double out[7]);

/*
 * Pin pattern choices for every iteration of later runs on this handle (NULL = full autotune).
 * Each non-AUTO field overrides the selector.  Unsupported combinations return
 * GSW_EUNSUPPORTED at run time:
 *   - PR: fusion is ignored (every vertex is active every iteration);
 *   - BC backward sweep always pulls; forcing applies to the forward (sigma) phase;
 *   - Delta-PR (gsw_dpr): only the direction is honoured (push or pull every iteration).
 * Pinning any field also disables the CTA-resident ("solo") tier of BFS/SSSP, so a forced run
 * executes exactly the pinned patterns.  Environment knobs read at each run (calibration only):
 * GSW_SELECTOR=trees (BFS: learned CART trees instead of the hand-set rules), GSW_SOLO_E /
 * GSW_SOLO_V (solo-tier thresholds; GSW_SOLO_E=0 disables it), GSW_SSSP_LAW (stepping law),
 * GSW_DPR_PULL_K (Delta-PR: pull iff K*Ea > nnz, default 2), GSW_PR_CACHE (PageRank hub-cache
 * entries), GSW_PR_BLOCKED / GSW_PR_BLOCKS (row-tier / source-blocked PageRank), GSW_MINB_BFS_FIXED /
 * GSW_MINB_SSSP_FIXED (disable the per-graph residency choice), GSW_DIST_LOOKAHEAD (levels the
 * partitioned host loop runs ahead of its done-flag poll), GSW_PHASES=1 (BFS init / loop / output
 * device times on stderr), GSW_CC_SWITCH=k (autotuned gsw_cc: label-propagation iterations before
 * it hands over to hooking, default 12, 0 = never), GSW_TEAM=k (BFS: clustered launch whose first
 * k-CTA cluster runs the small levels, road-like graphs, default off), GSW_CLUSTER=k (run a
 * persistent kernel as ONE k-CTA cluster, barrier.cluster as its grid barrier), GSW_GRID_CTAS=k
 * (persistent grid of k CTAs), GSW_DIST_GRAPH=0|1 (partitioned BFS level loop as a CUDA graph;
 * default on for loopback / one NCCL rank), GSW_DIST_HUBFIRST=0 / GSW_DIST_PR_HUBORDER=0
 * (partitioned create-time row reordering / PageRank hub-order layout off), GSW_RELABEL_KEYS64=1
 * (graph create: the 64-bit key sort instead of the symmetric pair sort).
 */
gsw_status gsw_force_config(gsw_graph g, const gsw_config *cfg);

/* BFS from `source` (Fig. 11).  depth[v] = hop distance, depth[source]=0,
 * -1 if unreachable.  depth: n int32, host or device.                                        */
gsw_status gsw_bfs(gsw_graph g, int32_t source, int32_t *depth, gsw_run_stats *stats);

/* SSSP with dynamic stepping (footnote 2 P:411-413).  Requires weights.
 * dist[v] = shortest-path length (uint32), UINT32_MAX if unreachable.  GSW_EOVERFLOW if
 * max_w * (n-1) >= 2^32-1.                                                                    */
gsw_status gsw_sssp(gsw_graph g, int32_t source, uint32_t *dist, gsw_run_stats *stats);

/* Connected components: label[v] = min vertex id of v's component.               */
gsw_status gsw_cc(gsw_graph g, int32_t *label, gsw_run_stats *stats);

/* Connected components by hooking + pointer jumping: the edge-centric GPU CC the paper compares
 * its CC against (Soman et al. [53], reading Q8).  Each iteration sweeps
 * every edge and hangs the tree with the larger root id below the other root (atomicMin on packed
 * (caller id, internal id) parent pointers), then compresses every pointer to its root; it stops
 * after a sweep in which no hook succeeded.  Output identical to gsw_cc: label[v] = min vertex id
 * of v's component.  label: n int32, host or device.  gsw_force_config's load_balance selects the
 * sweep's mapping (AUTO: THREAD when the degree range r_d <= 16, else STRICT); its other fields
 * are ignored.  stats->records: one per iteration,
 * Va = successful hooks, edges = adjacency entries swept.
 * Errors: GSW_EINVAL (NULL label), GSW_EUNSUPPORTED (distributed handle).                     */
gsw_status gsw_cc_hook(gsw_graph g, int32_t *label, gsw_run_stats *stats);

/* PageRank power iteration: pr_0 = 1/N, exactly `iters` iterations of
 *   pr'(v) = (1-d)/N + d * (sum_{u->v} pr(u)/deg_out(u) + D/N),  D = sum of dangling pr.
 * rank: n doubles, host or device.                                                            */
gsw_status gsw_pr(gsw_graph g, double damping, int32_t iters, double *rank, gsw_run_stats *stats);

/* Delta-PageRank (P:386-388 [19]; Fig. 3; reading R16).  Residual
 * propagation with an active set: delta_0 = (1-d)/N, r_0 = 0; each iteration the vertices with
 * delta(v) > eps = tol*(1-d)/N add delta(v) to r(v) and push d*delta(v)/deg_out(v) to their
 * out-neighbours' residuals; the run ends when no vertex is active (or after max_iters).  The
 * fixed point x solves x = (1-d)/N + d * sum_{u->v} x(u)/deg_out(u) (no dangling teleport: a
 * vertex without out-edges keeps its mass), and the result satisfies 0 <= x - rank and
 * ||x - rank||_1 <= tol.  Per iteration the selector picks push (queue of active vertices, fp64
 * atomics) or pull (in-edge reduction) from the active-edge count;
 * gsw_force_config's direction pins it, its other fields are ignored.
 *   tol: >= 0, finite (0 = run until residuals underflow or max_iters).
 *   max_iters: 1 .. 65536 (per-iteration records live in the workspace).   rank: n doubles, host or device.
 * stats->iterations counts non-empty iterations; records carry Va/Ea and the direction run.
 * Errors: GSW_EINVAL (bad arguments), GSW_EUNSUPPORTED (distributed handle, forced direction
 * other than push/pull).                                                                      */
gsw_status gsw_dpr(gsw_graph g, double damping, double tol, int32_t max_iters, double *rank,
                   gsw_run_stats *stats);

/* Betweenness centrality (Brandes): bc[v] = sum_{s in sources, s != v} delta_s(v),
 * unnormalised.  sources: nsrc int32 on the HOST.  bc: n doubles, host or device.              */
gsw_status gsw_bc(gsw_graph g, const int32_t *sources, int32_t nsrc, double *bc,
                  gsw_run_stats *stats);

/* ---------------------------------------------------------------------------------------------
 * Multi-GPU: 1D vertex partition (the paper itself is single-GPU).  Rank r of p owns
 * the vertex slice [r*S, min(n,(r+1)*S)) with S = gsw_dist_slice(n, p) (a multiple of 64, equal
 * for every rank as collectives need equal counts).  Every write lands on an owned vertex, so no
 * cross-GPU atomics are needed.
 *   BFS level: the rank expands into its owned slice of the next frontier bitmap (push: the
 *     column slice "global source -> owned targets" built at create; pull: the owned rows, i.e.
 *     in-edges of owned vertices, with early exit), then an in-place all-gather of the bitmap
 *     slices (n/8 bytes) and an all-reduce of (Va, Ea, edges) give every rank the same frontier;
 *     a device kernel on every rank evaluates the same direction rule on those global counts.
 *   PageRank iteration: owned rows pull the replicated fp32 contributions pr/deg; all-gather of
 *     the contribution slices (n*4 bytes) + all-reduce of the dangling mass.
 *   CC iteration: min-label propagation with the pointer-jumping shortcut label[label[v]] on the
 *     replicated labels; all-gather of the label slices + all-reduce of the change count.
 *   BC source (Brandes): forward levels pull sigma over in-neighbours at the previous depth,
 *     backward levels pull omega = (1 + delta) / sigma over successors; the owned slices of the
 *     replicated depth / sigma / omega arrays are all-gathered after every level.
 *   SSSP round (weighted graphs): near/far with a static step delta0 (gsw_config.delta0, else
 *     32*wbar/dbar; forced UNORDERED = Bellman-Ford): the near set is all-gathered as a bitmap,
 *     frontier vertices relax their column slices into owned distances (atomicMin), and the
 *     distance slices are all-gathered after every round.
 * The host never waits per iteration (NCCL / loopback): it polls the device's done flag two
 * iterations behind the stream.  Supported on distributed handles: gsw_bfs, gsw_pr, gsw_cc,
 * gsw_sssp, gsw_bc (gsw_dpr, gsw_app_* return GSW_EUNSUPPORTED); gsw_force_config's direction pins the BFS direction,
 * its stepping (UNORDERED) and delta0 the SSSP step.
 * Outputs of NCCL / host-staged handles cover the OWNED slice only; loopback outputs all n.
 * Three exchange backends run the same kernels:
 *   NCCL (one process per GPU; NCCL is dlopen'ed, a missing library gives GSW_ENCCL),
 *   loopback (p virtual ranks on one GPU, exchange = the shared replicated buffers),
 *   host-staged (caller callbacks, e.g. torch.distributed over gloo; several processes may share
 *     a GPU; one host round trip per exchange).
 * ------------------------------------------------------------------------------------------- */
/* Slice size S for n vertices over p ranks. */
int64_t gsw_dist_slice(int64_t n, int32_t nranks);
/* Fill 128 bytes with a new ncclUniqueId (call on one rank, broadcast the bytes to the others). */
gsw_status gsw_dist_unique_id(void *id128);
/* Workspace bytes for a partition of n_global vertices with nnz_owned adjacency entries. */
gsw_status gsw_dist_workspace_size(int64_t n_global, int64_t nnz_owned, int32_t nranks, size_t *bytes);
/* The same with edge weights (needed by gsw_sssp on partitioned handles) and/or for loopback mode
 * (loopback != 0: nnz_owned is the whole graph's nnz, nranks the number of virtual parts). */
gsw_status gsw_dist_workspace_size_weighted(int64_t n_global, int64_t nnz_owned, int32_t nranks, int32_t has_weights,
                                            int32_t loopback, size_t *bytes);
/* NCCL mode (one process per GPU).  owned: the rows of the owned slice -- owned->n = number of
 * owned vertices, row_offsets start at 0, col_indices are GLOBAL ids (symmetric graph).
 * nccl_id128 may be NULL only when nranks == 1 (a private communicator is created; the
 * collectives still run).  Collective over all ranks (same call order on every rank).
 * Errors: GSW_EINVAL (slice size mismatch), GSW_ENCCL (communicator creation failed). */
gsw_status gsw_graph_create_dist(const gsw_csr *owned, int64_t n_global, const void *nccl_id128,
                                 int32_t nranks, int32_t rank, void *workspace, size_t ws_bytes,
                                 void *cuda_stream, gsw_graph *out);
/* Host-staged exchange: the library copies its slice / counters to pinned host memory, calls
 * these callbacks (every rank in the same order, like a collective), and copies the result back.
 * Each returns 0 on success.
 *   allgather(user, send, recv, bytes): recv (nranks*bytes) = every rank's send, in rank order;
 *   allreduce_u64 / allreduce_f64(user, buf, count): in-place element-wise sum over the ranks. */
typedef struct {
    void *user;
    int (*allgather)(void *user, const void *send, void *recv, size_t bytes);
    int (*allreduce_u64)(void *user, uint64_t *buf, size_t count);
    int (*allreduce_f64)(void *user, double *buf, size_t count);
} gsw_exchange;
/* Same arguments as gsw_graph_create_dist (workspace: gsw_dist_workspace_size), exchange through
 * `exchange` (copied; its function pointers must stay valid until gsw_graph_destroy). */
gsw_status gsw_graph_create_dist_host(const gsw_csr *owned, int64_t n_global, const gsw_exchange *exchange,
                                      int32_t nranks, int32_t rank, void *workspace, size_t ws_bytes,
                                      void *cuda_stream, gsw_graph *out);
/* Loopback mode: `nparts` virtual ranks of the full symmetric graph on THIS GPU, exchanging
 * through device memory in stream order (the same partitioned kernels as NCCL mode; used to test
 * the partitioned path on one GPU).  Outputs cover all n vertices. */
gsw_status gsw_dist_loopback_workspace_size(int64_t n, int64_t nnz, int32_t nparts, size_t *bytes);
gsw_status gsw_graph_create_partitioned(const gsw_csr *csr, int32_t nparts, void *workspace,
                                        size_t ws_bytes, void *cuda_stream, gsw_graph *out);

/* ---------------------------------------------------------------------------------------------
 * User-programmable front-end (Sec. 4.2, Fig. 11): the paper's
 * filter / emit / comp / compAtomic functions as a header-only C++ policy template
 * (include/gsw_app.cuh, gsw::app::run) driven by the same persistent engine, pattern candidates
 * and selector.  These two entry points are BFS and SSSP written with it (csrc/app.cu); they
 * return exactly what gsw_bfs / gsw_sssp return (same arguments, outputs and errors), including
 * under gsw_force_config (direction / format / load balance / fusion; SSSP stepping STATIC /
 * UNORDERED, otherwise the dynamic law).
 * ------------------------------------------------------------------------------------------- */
gsw_status gsw_app_bfs(gsw_graph g, int32_t source, int32_t *depth, gsw_run_stats *stats);
gsw_status gsw_app_sssp(gsw_graph g, int32_t source, uint32_t *dist, gsw_run_stats *stats);

/* Thread-local message for the last non-OK status of this thread. */
const char *gsw_last_error(void);
/* Library version string. */
const char *gsw_version(void);

#ifdef __cplusplus
}
#endif
#endif /* GSW_H */
