"""Pins for oracle.sssp (Dijkstra) and oracle.bfs (PAPER.md P5@10183, P11@2218, P5@11591).

Independent of oracle/orc.c: the CLRS Fig. 24.6 worked example
(tests/golden/sssp_clrs_24_6.txt), Bellman-Ford and Floyd-Warshall brute force
on 200 random tiny graphs, scipy.sparse.csgraph, closed forms (path, star,
complete, grid, binary tree), BFS == unit-weight SSSP, and the exact O(m)
shortest-path certificate on R-MAT graphs.
"""
import os

import numpy as np
import pytest
import scipy.sparse as sp
from scipy.sparse import csgraph

import inlgen
import oracle
from graphs import INF32, bellman_ford, certify_bfs, certify_sssp, csr_from_edges, floyd_warshall

GOLDEN = os.path.join(os.path.dirname(__file__), "golden")


def test_clrs_worked_example():
    edges, ws, want = [], [], {}
    src = None
    for line in open(os.path.join(GOLDEN, "sssp_clrs_24_6.txt")):
        f = line.split("#")[0].split()
        if not f:
            continue
        if f[0] == "edge":
            edges.append((int(f[1]), int(f[2])))
            ws.append(int(f[3]))
        elif f[0] == "source":
            src = int(f[1])
        elif f[0] == "dist":
            want[int(f[1])] = int(f[2])
    rp, ci, w = csr_from_edges(5, edges, ws)
    d = oracle.sssp(rp, ci, w, src)
    assert d.tolist() == [want[v] for v in range(5)]


def _random_graph(rng):
    n = int(rng.integers(1, 65))
    kind = rng.integers(0, 5)
    if kind == 0:  # sparse random, possibly disconnected
        m = int(rng.integers(0, 3 * n + 1))
        edges = [(int(rng.integers(n)), int(rng.integers(n))) for _ in range(m)]
    elif kind == 1:  # path
        edges = [(i, i + 1) for i in range(n - 1)]
    elif kind == 2:  # star
        edges = [(0, i) for i in range(1, n)]
    elif kind == 3:  # complete
        edges = [(i, j) for i in range(n) for j in range(n) if i != j]
    else:  # dense random
        edges = [(i, j) for i in range(n) for j in range(n) if rng.random() < 0.3]
    ws = rng.integers(1, 256, size=len(edges))
    sym = bool(rng.integers(0, 2))
    return n, edges, ws, sym


@pytest.mark.parametrize("seed", range(200))
def test_dijkstra_equals_bellman_ford_and_floyd_warshall(seed):
    rng = np.random.default_rng(seed)
    n, edges, ws, sym = _random_graph(rng)
    rp, ci, w = csr_from_edges(n, edges, ws, symmetric=sym)
    s = int(rng.integers(n))
    d = oracle.sssp(rp, ci, w, s)
    assert np.array_equal(d, bellman_ford(n, rp, ci, w, s))
    assert np.array_equal(d, floyd_warshall(n, rp, ci, w, s))
    assert certify_sssp(rp, ci, w, s, d) is None
    # BFS == SSSP with unit weights
    lv = oracle.bfs(rp, ci, s)
    du = oracle.sssp(rp, ci, np.ones_like(w), s)
    assert np.array_equal(np.where(lv < 0, INF32, lv).astype(np.uint32), du)


def test_scipy_csgraph_on_rmat():
    g = inlgen.host_build(12, 16, seed=1, flags=inlgen.SYMMETRIC)
    w = inlgen.weights_host(g.row_ptr, g.col_idx)
    A = sp.csr_matrix((w.astype(np.float64), g.col_idx, g.row_ptr), shape=(g.n_rows, g.n_global))
    for s in inlgen.sources(g.row_ptr, 4):
        d = oracle.sssp(g.row_ptr, g.col_idx, w, s)
        ref = csgraph.dijkstra(A, directed=True, indices=s)
        assert np.array_equal(d, np.where(np.isinf(ref), INF32, ref).astype(np.uint32))
        lv = oracle.bfs(g.row_ptr, g.col_idx, s)
        ref = csgraph.shortest_path(A, directed=True, unweighted=True, indices=s)
        assert np.array_equal(lv, np.where(np.isinf(ref), -1, ref).astype(np.int32))
        assert certify_sssp(g.row_ptr, g.col_idx, w, s, d) is None
        assert certify_bfs(g.row_ptr, g.col_idx, s, lv) is None


def test_path_prefix_sums():
    n = 50
    ws = np.arange(1, n)
    rp, ci, w = csr_from_edges(n, [(i, i + 1) for i in range(n - 1)], ws)
    assert oracle.sssp(rp, ci, w, 0).tolist() == np.concatenate([[0], np.cumsum(ws)]).tolist()
    assert oracle.bfs(rp, ci, 0).tolist() == list(range(n))
    assert oracle.bfs(rp, ci, 10).tolist() == [-1] * 10 + list(range(n - 10))


def test_bfs_closed_forms():
    n = 20
    rp, ci, _ = csr_from_edges(n, [(0, i) for i in range(1, n)], symmetric=True)
    assert oracle.bfs(rp, ci, 0).tolist() == [0] + [1] * (n - 1)
    assert oracle.bfs(rp, ci, 3).tolist() == [1] + [2] * 2 + [0] + [2] * (n - 4)
    rp, ci, _ = csr_from_edges(n, [(i, j) for i in range(n) for j in range(n)], symmetric=True)
    assert oracle.bfs(rp, ci, 5).tolist() == [1] * 5 + [0] + [1] * (n - 6)
    R, Cc = 7, 9  # 2-D grid: Manhattan distance
    idx = lambda r, c: r * Cc + c
    e = [(idx(r, c), idx(r, c + 1)) for r in range(R) for c in range(Cc - 1)] + \
        [(idx(r, c), idx(r + 1, c)) for r in range(R - 1) for c in range(Cc)]
    rp, ci, _ = csr_from_edges(R * Cc, e, symmetric=True)
    lv = oracle.bfs(rp, ci, idx(2, 3))
    assert lv.tolist() == [abs(r - 2) + abs(c - 3) for r in range(R) for c in range(Cc)]
    n = 127  # complete binary tree
    rp, ci, _ = csr_from_edges(n, [((i - 1) // 2, i) for i in range(1, n)], symmetric=True)
    assert oracle.bfs(rp, ci, 0).tolist() == [int(np.floor(np.log2(i + 1))) for i in range(n)]


def test_isolated_source_and_single_vertex():
    rp, ci, w = csr_from_edges(4, [(1, 2), (2, 3)], [5, 6], symmetric=True)
    assert oracle.sssp(rp, ci, w, 0).tolist() == [0, 0xFFFFFFFF, 0xFFFFFFFF, 0xFFFFFFFF]
    assert oracle.bfs(rp, ci, 0).tolist() == [0, -1, -1, -1]
    rp = np.zeros(2, np.int64)
    assert oracle.sssp(rp, np.zeros(0, np.int32), np.zeros(0, np.uint32), 0).tolist() == [0]


def test_certificate_rejects_wrong_distances():
    g = inlgen.host_build(9, 16, seed=1, flags=inlgen.SYMMETRIC)
    w = inlgen.weights_host(g.row_ptr, g.col_idx)
    s = inlgen.sources(g.row_ptr, 1)[0]
    d = oracle.sssp(g.row_ptr, g.col_idx, w, s)
    reach = np.nonzero((d != INF32) & (np.arange(len(d)) != s))[0]
    bad = d.copy()
    bad[reach[0]] += 1
    assert certify_sssp(g.row_ptr, g.col_idx, w, s, bad) is not None
    bad = d.copy()
    bad[reach[1]] -= 1
    assert certify_sssp(g.row_ptr, g.col_idx, w, s, bad) is not None
