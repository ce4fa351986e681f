"""Small-graph builders, brute-force references and exact certificates (test helpers).

Nothing here is used by the product; these are the independent pins the oracle
is checked against (and, at full size, the GPU output too).
"""
from __future__ import annotations

import numpy as np

INF32 = np.uint32(0xFFFFFFFF)


def csr_from_edges(n, edges, weights=None, symmetric=False):
    """CSR (row_ptr int64, col int32, w uint32) from (u, v[, w]) edges; duplicates keep the min weight."""
    best = {}
    for i, (u, v) in enumerate(edges):
        if u == v:
            continue
        w = 1 if weights is None else int(weights[i])
        pairs = [(u, v), (v, u)] if symmetric else [(u, v)]
        for a, b in pairs:
            if (a, b) not in best or w < best[(a, b)]:
                best[(a, b)] = w
    keys = sorted(best)
    rp = np.zeros(n + 1, dtype=np.int64)
    for a, _ in keys:
        rp[a + 1] += 1
    rp = np.cumsum(rp)
    ci = np.array([b for _, b in keys], dtype=np.int32)
    w = np.array([best[k] for k in keys], dtype=np.uint32)
    return rp, ci, w


def bellman_ford(n, rp, ci, w, s):
    """O(n m) textbook Bellman-Ford with Python ints."""
    INF = float("inf")
    d = [INF] * n
    d[s] = 0
    src = np.repeat(np.arange(n), np.diff(rp)).tolist()
    dst = ci.tolist()
    ww = w.tolist()
    for _ in range(max(n - 1, 1)):
        changed = False
        for u, v, x in zip(src, dst, ww):
            if d[u] + x < d[v]:
                d[v] = d[u] + x
                changed = True
        if not changed:
            break
    return np.array([0xFFFFFFFF if x == INF else x for x in d], dtype=np.uint32)


def floyd_warshall(n, rp, ci, w, s):
    D = np.full((n, n), np.inf)
    np.fill_diagonal(D, 0)
    for u in range(n):
        for k in range(rp[u], rp[u + 1]):
            D[u, ci[k]] = min(D[u, ci[k]], float(w[k]))
    for k in range(n):
        D = np.minimum(D, D[:, k:k + 1] + D[k:k + 1, :])
    row = D[s]
    return np.where(np.isinf(row), 0xFFFFFFFF, row).astype(np.uint32)


def certify_sssp(rp, ci, w, s, dist):
    """Exact O(m) certificate: dist[s]=0, every edge feasible, every finite
    v != s has a tight in-edge, unreachable <=> INF.  With w >= 1 this implies dist == delta."""
    rp = np.asarray(rp, np.int64)
    n = len(rp) - 1
    dist = np.asarray(dist, np.uint32)
    if dist[s] != 0:
        return "dist[source] != 0"
    src = np.repeat(np.arange(n, dtype=np.int64), np.diff(rp))
    du = dist[src].astype(np.int64)
    dv = dist[ci].astype(np.int64)
    ww = np.asarray(w, np.int64)
    fin = dist[src] != INF32
    if np.any(dv[fin] > du[fin] + ww[fin]):
        return "infeasible edge"
    tight = fin & (dv == du + ww)
    has = np.zeros(n, dtype=bool)
    has[np.asarray(ci)[tight]] = True
    need = (dist != INF32)
    need[s] = False
    if np.any(need & ~has):
        return "finite vertex without a tight in-edge"
    # unreachable must have no finite in-neighbour (feasibility covers it: dv=INF > du+w)
    return None


def certify_bfs(rp, ci, s, level):
    lv = np.asarray(level, np.int64)
    d = np.where(lv < 0, 0xFFFFFFFF, lv).astype(np.uint32)
    return certify_sssp(rp, ci, np.ones(len(ci), np.uint32), s, d)


def csr_np(n, u, v, symmetric=True):
    """Vectorised CSR build (sorted rows, no self-loops, duplicates merged) from edge arrays;
    symmetric adds (v, u).  For large adversarial graphs where csr_from_edges is too slow."""
    u = np.asarray(u, np.int64)
    v = np.asarray(v, np.int64)
    keep = u != v
    u, v = u[keep], v[keep]
    if symmetric:
        u, v = np.concatenate([u, v]), np.concatenate([v, u])
    key = np.unique(u * n + v)
    rows, cols = key // n, key % n
    rp = np.zeros(n + 1, np.int64)
    np.add.at(rp, rows + 1, 1)
    return np.cumsum(rp), cols.astype(np.int32)


def pair_weights(rp, ci):
    """Symmetric weights 1..255 keyed by the unordered pair (test-side recipe)."""
    n = len(rp) - 1
    src = np.repeat(np.arange(n, dtype=np.int64), np.diff(rp))
    a, b = np.minimum(src, ci), np.maximum(src, ci)
    return ((a * 2654435761 + b * 40503) % 255 + 1).astype(np.uint32)
