"""Brute-force definitions on tiny graphs (<= ~12 vertices), used to pin the oracle.

Each function computes its quantity by a route different from the oracle's algorithm:
Floyd-Warshall instead of BFS/Dijkstra, transitive closure instead of union-find, the dense
Google matrix instead of the sparse pull, and explicit shortest-path pair counting instead of
Brandes' recursion.
"""
import numpy as np

INF = np.iinfo(np.int64).max // 4


def edge_list(g):
    for u in range(g.n):
        for e in range(g.off[u], g.off[u + 1]):
            yield u, int(g.col[e]), e


def floyd(g, weighted: bool):
    n = g.n
    D = np.full((n, n), INF, dtype=np.int64)
    for i in range(n):
        D[i, i] = 0
    for u, v, e in edge_list(g):
        w = int(g.w[e]) if weighted else 1
        D[u, v] = min(D[u, v], w)
    for k in range(n):
        D = np.minimum(D, D[:, k:k + 1] + D[k:k + 1, :])
    return D


def bfs_depth(g, s):
    d = floyd(g, False)[s]
    return np.where(d >= INF, -1, d).astype(np.int32)


def sssp_dist(g, s):
    d = floyd(g, True)[s]
    return np.where(d >= INF, np.iinfo(np.uint32).max, d).astype(np.uint32)


def cc_labels(g):
    n = g.n
    R = np.eye(n, dtype=bool)
    for u, v, _ in edge_list(g):
        R[u, v] = True
    for k in range(n):                       # transitive closure (Warshall)
        R = R | (R[:, k:k + 1] & R[k:k + 1, :])
    return np.array([int(np.argmax(R[v])) for v in range(n)], dtype=np.int32)


def pagerank_dense(g, d=0.85, iters=20):
    """x_{t+1} = G x_t with the dense Google matrix
    G = d * (A^T Dinv + (1/N) 1 z^T) + (1-d)/N 1 1^T, z = indicator of dangling vertices."""
    n = g.n
    A = np.zeros((n, n))
    for u, v, _ in edge_list(g):
        A[u, v] += 1.0
    deg = A.sum(1)
    P = np.zeros((n, n))
    for u in range(n):
        if deg[u] > 0:
            P[:, u] = A[u] / deg[u]
        else:
            P[:, u] = 1.0 / n
    G = d * P + (1 - d) / n
    x = np.full(n, 1.0 / n)
    for _ in range(iters):
        x = G @ x
    return x


def dpr_fixed_point(g, d=0.85):
    """Exact fixed point of Delta-PageRank's linear system (DESIGN R16), by a dense solve:
    (I - d A^T Dinv) x = (1-d)/N 1, dangling columns zero (no teleport of their mass)."""
    n = g.n
    A = np.zeros((n, n))
    for u, v, _ in edge_list(g):
        A[u, v] += 1.0
    deg = A.sum(1)
    M = np.zeros((n, n))
    for u in range(n):
        if deg[u] > 0:
            M[:, u] = A[u] / deg[u]
    return np.linalg.solve(np.eye(n) - d * M, np.full(n, (1 - d) / n))


def path_counts(g):
    """dist[s,t] (hops) and sigma[s,t] (# shortest paths, counting parallel edges) for all pairs
    via dynamic programming over hop length."""
    n = g.n
    A = np.zeros((n, n), dtype=object)
    for u, v, _ in edge_list(g):
        A[u, v] += 1
    dist = np.full((n, n), -1, dtype=np.int64)
    sigma = np.zeros((n, n), dtype=object)
    for s in range(n):
        cur = np.zeros(n, dtype=object)
        cur[s] = 1
        dist[s, s] = 0
        sigma[s, s] = 1
        for k in range(1, n):
            nxt = np.zeros(n, dtype=object)
            for u in range(n):
                if cur[u]:
                    for v in range(n):
                        if A[u, v]:
                            nxt[v] += cur[u] * A[u, v]
            # walks of length k that are shortest paths
            fresh = np.zeros(n, dtype=object)
            for v in range(n):
                if nxt[v] and dist[s, v] < 0:
                    dist[s, v] = k
                    sigma[s, v] = nxt[v]
                    fresh[v] = nxt[v]
            cur = fresh
            if not any(fresh):
                break
    return dist, sigma


def bc_pairs(g, sources):
    """bc[v] = sum_{s in S} sum_{t != s, v} sigma_st(v)/sigma_st  (pair-dependency definition)."""
    dist, sigma = path_counts(g)
    n = g.n
    bc = np.zeros(n)
    for s in sources:
        for t in range(n):
            if t == s or dist[s, t] < 0:
                continue
            for v in range(n):
                if v in (s, t) or dist[s, v] < 0 or dist[v, t] < 0:
                    continue
                if dist[s, v] + dist[v, t] == dist[s, t]:
                    bc[v] += float(sigma[s, v] * sigma[v, t]) / float(sigma[s, t])
    return bc


def random_graph(rng, n, p, weighted=False, maxw=9):
    edges = [(u, v) for u in range(n) for v in range(u + 1, n) if rng.random() < p]
    import gen
    w = None
    if weighted:
        w = [int(rng.integers(1, maxw + 1)) for _ in edges]
    if not edges:
        return gen.from_edges(n, np.zeros((0, 2), np.int64), weights=[] if weighted else None)
    return gen.from_edges(n, edges, weights=w)
