"""Pins for oracle.bc (Brandes betweenness, reading R10) — nothing here calls orc_bc's
recurrence: closed forms, an identity over all pairs, and a brute force that counts
shortest paths as walks of length d(s, t) (matrix powers).

PAPER.md P5@8318: BC "is equal to the number of shortest paths from all nodes to all
others that pass through that node" — pair dependencies sigma_st(v) / sigma_st summed
over ordered pairs (s, t), s != v != t.
"""
import numpy as np
import pytest
import scipy.sparse as sp
from scipy.sparse.csgraph import shortest_path

import oracle
from graphs import csr_from_edges


def brute_bc(n, rp, ci, sources=None):
    A = np.zeros((n, n), dtype=object)
    for u in range(n):
        for k in range(rp[u], rp[u + 1]):
            A[u, ci[k]] = 1
    D = np.full((n, n), -1, dtype=np.int64)
    sig = np.zeros((n, n), dtype=object)  # walks of length D[s,t] = shortest paths
    P = np.identity(n, dtype=object)
    for d in range(n):
        newly = (P != 0) & (D < 0)
        D[newly] = d
        sig[newly] = P[newly]
        P = P.dot(A)
    bc = np.zeros(n)
    src = range(n) if sources is None else sources
    for s in src:
        for t in range(n):
            if t == s or D[s, t] < 0:
                continue
            for v in range(n):
                if v in (s, t) or D[s, v] < 0 or D[v, t] < 0:
                    continue
                if D[s, v] + D[v, t] == D[s, t]:
                    bc[v] += float(sig[s, v] * sig[v, t]) / float(sig[s, t])
    return bc


def test_path_closed_form():
    n = 9
    rp, ci, _ = csr_from_edges(n, [(i, i + 1) for i in range(n - 1)], symmetric=True)
    b = oracle.bc(rp, ci)
    assert np.array_equal(b, [2.0 * i * (n - 1 - i) for i in range(n)])


def test_star_and_complete():
    k = 7
    rp, ci, _ = csr_from_edges(k + 1, [(0, i) for i in range(1, k + 1)], symmetric=True)
    b = oracle.bc(rp, ci)
    assert b[0] == k * (k - 1) and np.all(b[1:] == 0)
    n = 6
    rp, ci, _ = csr_from_edges(n, [(i, j) for i in range(n) for j in range(i + 1, n)], symmetric=True)
    assert np.all(oracle.bc(rp, ci) == 0)


@pytest.mark.parametrize("n", [7, 8])
def test_cycle_closed_form(n):
    rp, ci, _ = csr_from_edges(n, [(i, (i + 1) % n) for i in range(n)], symmetric=True)
    k = n // 2
    per = k * (k - 1) if n % 2 else (k - 1) ** 2
    assert np.allclose(oracle.bc(rp, ci), per, rtol=0, atol=1e-12)


def test_sum_identity_random():
    """sum_v bc(v) = sum over reachable ordered pairs of (d(s,t) - 1) (every shortest path
    has d - 1 interior vertices), with distances from scipy."""
    rng = np.random.default_rng(7)
    for trial in range(20):
        n = int(rng.integers(5, 60))
        m = int(rng.integers(n, 4 * n))
        e = [(int(rng.integers(n)), int(rng.integers(n))) for _ in range(m)]
        sym = bool(trial % 2)
        rp, ci, _ = csr_from_edges(n, e, symmetric=sym)
        A = sp.csr_matrix((np.ones(len(ci)), ci, rp), shape=(n, n))
        D = shortest_path(A, unweighted=True, directed=True)
        fin = np.isfinite(D) & (D > 0)
        assert abs(oracle.bc(rp, ci).sum() - (D[fin] - 1).sum()) <= 1e-9 * max(1.0, (D[fin] - 1).sum())


def test_brute_force_random_small():
    rng = np.random.default_rng(11)
    for trial in range(60):
        n = int(rng.integers(2, 12))
        m = int(rng.integers(0, 3 * n))
        e = [(int(rng.integers(n)), int(rng.integers(n))) for _ in range(m)]
        rp, ci, _ = csr_from_edges(n, e, symmetric=bool(trial % 3))
        ref = brute_bc(n, rp, ci)
        assert np.allclose(oracle.bc(rp, ci), ref, rtol=1e-12, atol=1e-12)
        srcs = sorted(set(int(x) for x in rng.integers(0, n, size=3)))
        assert np.allclose(oracle.bc(rp, ci, srcs), brute_bc(n, rp, ci, srcs), rtol=1e-12, atol=1e-12)


def test_rejects_bad_sources():
    rp, ci, _ = csr_from_edges(3, [(0, 1)], symmetric=True)
    with pytest.raises(RuntimeError):
        oracle.bc(rp, ci, [3])
    assert oracle.bc(np.zeros(1, np.int64), np.zeros(0, np.int32)).size == 0
