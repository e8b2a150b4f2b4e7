"""Independent checks used to pin the oracle (tests only; none of this is imported by the product).

Each helper is a *different* computation from the oracle's Dijkstra: brute-force Floyd-Warshall,
closed forms, union-find components and the Bellman optimality certificate.
"""
import numpy as np

INF = 0x3FFFFFFF


def brute_fw(n, src, dst, w):
    """Textbook Floyd-Warshall [9] on the adjacency matrix, int64, vectorised over k."""
    D = np.full((n, n), np.iinfo(np.int64).max // 4, dtype=np.int64)
    np.fill_diagonal(D, 0)
    for u, v, x in zip(np.asarray(src), np.asarray(dst), np.asarray(w)):
        if x < D[u, v]:
            D[u, v] = D[v, u] = x
    for k in range(n):
        D = np.minimum(D, D[:, k, None] + D[None, k, :])
    D[D >= np.iinfo(np.int64).max // 8] = INF
    return D


def batched_fw(D):
    """Floyd-Warshall over a stack of (G, n, n) int64 matrices (big = no edge)."""
    n = D.shape[1]
    for k in range(n):
        D = np.minimum(D, D[:, :, k, None] + D[:, None, k, :])
    return D


def components(n, src, dst):
    """Union-find component labels."""
    parent = np.arange(n)

    def find(x):
        while parent[x] != x:
            parent[x] = parent[parent[x]]
            x = parent[x]
        return x

    for u, v in zip(np.asarray(src), np.asarray(dst)):
        a, b = find(int(u)), find(int(v))
        if a != b:
            parent[max(a, b)] = min(a, b)
    return np.array([find(x) for x in range(n)])


def bellman_certificate(S, rows, n, src, dst, w):
    """True iff S[rows] are exact shortest-path distances: d(s,s)=0, every arc is
    relaxed (d(s,t) <= d(s,u)+w), every finite d(s,t), t != s, is attained by some arc, and INF
    entries only where t is unreachable (relaxation forces every reachable entry finite)."""
    S = np.asarray(S, dtype=np.int64)
    rows = np.asarray(rows)
    u = np.concatenate([src, dst]).astype(np.int64)
    v = np.concatenate([dst, src]).astype(np.int64)
    ww = np.concatenate([w, w]).astype(np.int64)
    keep = u != v
    u, v, ww = u[keep], v[keep], ww[keep]
    if not np.all(S[np.arange(len(rows)), rows] == 0):
        return False
    ok = True
    for i in range(len(rows)):
        d = S[i]
        du = d[u]
        fin = du < INF
        cand = np.where(fin, du + ww, np.iinfo(np.int64).max)
        if np.any(d[v] > cand):
            return False
        best = np.full(n, np.iinfo(np.int64).max, dtype=np.int64)
        np.minimum.at(best, v, cand)
        need = (d < INF)
        need[rows[i]] = False
        if np.any(best[need] != d[need]):
            ok = False
            break
        if np.any(d > INF) or np.any(d < 0):
            return False
    return ok
