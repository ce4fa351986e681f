"""Pins for oracle.pagerank (PAPER.md P5@9262, P5@9781; reading R1 in DESIGN.md).

Independent of oracle/orc.c: total mass 1 after every step, the closed form of
the symmetric star (tests/golden/pagerank_star.txt), uniform fixed points of
vertex-transitive graphs, the edgeless graph, and 20 steps of the dense Google
matrix power iteration in numpy.
"""
import os

import numpy as np
import pytest

import inlgen
import oracle

GOLDEN = os.path.join(os.path.dirname(__file__), "golden")


def _in_csr(n, edges):
    """in-edge CSR (rows = destinations) and out-degrees from a directed edge list."""
    edges = sorted(set((u, v) for u, v in edges if u != v), key=lambda e: (e[1], e[0]))
    rp = np.zeros(n + 1, dtype=np.int64)
    for _, v in edges:
        rp[v + 1] += 1
    rp = np.cumsum(rp)
    ci = np.array([u for u, _ in edges], dtype=np.int32)
    od = np.zeros(n, dtype=np.int32)
    for u, _ in edges:
        od[u] += 1
    return rp, ci, od


def _google_power(n, edges, d, iters):
    """Dense column-stochastic Google matrix, dangling columns uniform."""
    G = np.zeros((n, n))
    od = np.zeros(n)
    E = set((u, v) for u, v in edges if u != v)
    for u, v in E:
        od[u] += 1
    for u, v in E:
        G[v, u] = 1.0 / od[u]
    for u in range(n):
        if od[u] == 0:
            G[:, u] = 1.0 / n
    M = d * G + (1 - d) / n * np.ones((n, n))
    p = np.full(n, 1.0 / n)
    for _ in range(iters):
        p = M @ p
    return p


def test_star_closed_form_golden():
    vals = {}
    for line in open(os.path.join(GOLDEN, "pagerank_star.txt")):
        line = line.split("#")[0].strip()
        if line:
            k, v = line.split("=")
            vals[k.strip()] = float(v)
    k, d, t = int(vals["k"]), vals["d"], int(vals["t"])
    n = k + 1
    edges = [(0, i) for i in range(1, n)] + [(i, 0) for i in range(1, n)]
    rp, ci, od = _in_csr(n, edges)
    for it in range(t + 1):
        r = oracle.pagerank(n, rp, ci, od, d, it)
        ps = ((1 - d) / n + d) / (1 + d)
        ph = ps + (-d) ** it * (1.0 / n - ps)
        assert abs(r[0] - ph) < 1e-15
        np.testing.assert_allclose(r[1:], (1 - ph) / k, rtol=0, atol=1e-15)
    assert abs(r[0] - vals["p_hub"]) < 1e-8


@pytest.mark.parametrize("n", [1, 2, 5, 64])
def test_cycle_and_complete_are_uniform(n):
    cyc = [(i, (i + 1) % n) for i in range(n)]
    comp = [(i, j) for i in range(n) for j in range(n) if i != j]
    for edges in (cyc, comp):
        rp, ci, od = _in_csr(n, edges)
        r = oracle.pagerank(n, rp, ci, od, 0.85, 20)
        np.testing.assert_allclose(r, 1.0 / n, rtol=1e-14)


def test_edgeless_all_dangling_is_uniform_and_zero_iterations():
    n = 10
    rp, ci, od = _in_csr(n, [])
    np.testing.assert_allclose(oracle.pagerank(n, rp, ci, od, 0.85, 20), 0.1, rtol=1e-15)
    g = inlgen.host_build(8, 16, seed=4, flags=inlgen.TRANSPOSE)
    np.testing.assert_array_equal(oracle.pagerank(g.n_global, g.row_ptr, g.col_idx, g.out_degree, 0.85, 0),
                                  np.full(g.n_global, 1.0 / g.n_global))


@pytest.mark.parametrize("seed", range(12))
def test_dense_google_matrix_power_iteration(seed):
    rng = np.random.default_rng(100 + seed)
    n = int(rng.integers(2, 40))
    p = rng.random() * 0.3
    edges = [(u, v) for u in range(n) for v in range(n) if u != v and rng.random() < p]
    rp, ci, od = _in_csr(n, edges)
    for d in (0.85, 0.5):
        r = oracle.pagerank(n, rp, ci, od, d, 20)
        np.testing.assert_allclose(r, _google_power(n, edges, d, 20), rtol=1e-13, atol=1e-16)


def test_mass_is_one_every_iteration_on_rmat():
    g = inlgen.host_build(11, 16, seed=1, flags=inlgen.TRANSPOSE)
    for it in (1, 2, 5, 20):
        r = oracle.pagerank(g.n_global, g.row_ptr, g.col_idx, g.out_degree, 0.85, it)
        assert abs(r.sum() - 1.0) < 1e-12
        assert (r > 0).all()


def test_out_degree_matches_in_csr_columns():
    g = inlgen.host_build(10, 16, seed=2, flags=inlgen.TRANSPOSE)
    assert np.array_equal(np.bincount(g.col_idx, minlength=g.n_global), g.out_degree)


def test_fixed_point_matches_linear_solve():
    rng = np.random.default_rng(5)
    n = 30
    edges = [(u, v) for u in range(n) for v in range(n) if u != v and rng.random() < 0.1]
    rp, ci, od = _in_csr(n, edges)
    d = 0.85
    r = oracle.pagerank(n, rp, ci, od, d, 200)
    # p = d (G p) + (1-d)/n 1 with G column-stochastic (dangling uniform)
    G = np.zeros((n, n))
    for u, v in set(edges):
        G[v, u] = 1.0 / od[u]
    for u in range(n):
        if od[u] == 0:
            G[:, u] = 1.0 / n
    p = np.linalg.solve(np.eye(n) - d * G, np.full(n, (1 - d) / n))
    np.testing.assert_allclose(r, p, rtol=1e-12)


def test_openmp_context_line_is_bit_identical():
    import inlgen
    g = inlgen.host_build(13, 16, seed=inlgen.SEED_GRAPH, flags=inlgen.TRANSPOSE)
    a = oracle.pagerank_par(g.n_global, g.row_ptr, g.col_idx, g.out_degree, 0.85, 20)
    b = oracle.pagerank(g.n_global, g.row_ptr, g.col_idx, g.out_degree, 0.85, 20)
    assert np.array_equal(a, b)
