"""Pins for oracle.spmv (SpMV over CSR, PAPER.md P5@10072, P5@10497).

Each pin is independent of oracle/orc.c: closed forms (identity, diagonal,
permutation, row sums), exact integer arithmetic in Python ints, and a dense
numpy / scipy.sparse product.  A dropped term, a wrong index or a transposed
operand in the oracle fails at least one of them.
"""
import numpy as np
import pytest
import scipy.sparse as sp

import inlgen
import oracle


def _csr(dense):
    m = sp.csr_matrix(dense)
    m.sort_indices()
    return m.indptr.astype(np.int64), m.indices.astype(np.int32), m.data.astype(np.float32)


def test_identity_gives_x_bit_exact():
    n = 257
    rp = np.arange(n + 1, dtype=np.int64)
    ci = np.arange(n, dtype=np.int32)
    val = np.ones(n, dtype=np.float32)
    x = inlgen.vector_host(n)
    y = oracle.spmv(rp, ci, val, x)
    assert np.array_equal(y, x.astype(np.float64))


def test_diagonal_is_one_rounded_product():
    n = 300
    rp = np.arange(n + 1, dtype=np.int64)
    ci = np.arange(n, dtype=np.int32)
    d = inlgen.vector_host(n, seed=11) * np.float32(3.0)
    x = inlgen.vector_host(n, seed=12)
    y = oracle.spmv(rp, ci, d, x)
    # the product of two fp32 values is exact in fp64 (24+24 < 53 mantissa bits)
    assert np.array_equal(y, d.astype(np.float64) * x.astype(np.float64))


def test_permutation_permutes_x():
    n = 1000
    rng = np.random.default_rng(7)
    perm = rng.permutation(n).astype(np.int32)
    rp = np.arange(n + 1, dtype=np.int64)
    x = inlgen.vector_host(n, seed=13)
    y = oracle.spmv(rp, perm, np.ones(n, np.float32), x)
    assert np.array_equal(y, x[perm].astype(np.float64))


def test_empty_rows_are_zero_and_empty_matrix():
    rp = np.array([0, 0, 2, 2, 2, 3], dtype=np.int64)
    ci = np.array([1, 4, 0], dtype=np.int32)
    val = np.array([2.0, 3.0, 5.0], dtype=np.float32)
    x = np.array([1.0, 10.0, 100.0, 1000.0, 10000.0], dtype=np.float32)
    y = oracle.spmv(rp, ci, val, x)
    assert y.tolist() == [0.0, 2 * 10.0 + 3 * 10000.0, 0.0, 0.0, 5.0]
    assert oracle.spmv(np.zeros(1, np.int64), np.zeros(0, np.int32), np.zeros(0, np.float32),
                       np.zeros(0, np.float32)).shape == (0,)


def test_integer_values_exact_against_python_ints():
    g = inlgen.host_build(10, 16, seed=3)
    val = inlgen.values_host(g.row_ptr, g.col_idx, mode=1)
    x = inlgen.vector_host(g.n_global, mode=1)
    y = oracle.spmv(g.row_ptr, g.col_idx, val, x)
    vi = val.astype(np.int64).tolist()
    xi = x.astype(np.int64).tolist()
    ci = g.col_idx.tolist()
    rp = g.row_ptr.tolist()
    for i in range(g.n_rows):
        s = 0
        for k in range(rp[i], rp[i + 1]):
            s += vi[k] * xi[ci[k]]
        assert y[i] == s


@pytest.mark.parametrize("seed", range(6))
def test_dense_brute_force(seed):
    rng = np.random.default_rng(seed)
    n, m = int(rng.integers(1, 300)), int(rng.integers(1, 300))
    dense = (rng.random((n, m)) < rng.random() * 0.3) * rng.random((n, m))
    dense = dense.astype(np.float32)
    rp, ci, val = _csr(dense)
    x = rng.random(m).astype(np.float32)
    y = oracle.spmv(rp, ci, val, x)
    ref = dense.astype(np.float64) @ x.astype(np.float64)
    np.testing.assert_allclose(y, ref, rtol=1e-13, atol=0)


def test_rmat_against_scipy_and_row_sums():
    g = inlgen.host_build(12, 16, seed=1)
    val = inlgen.values_host(g.row_ptr, g.col_idx)
    x = inlgen.vector_host(g.n_global)
    y = oracle.spmv(g.row_ptr, g.col_idx, val, x)
    A = sp.csr_matrix((val.astype(np.float64), g.col_idx, g.row_ptr), shape=(g.n_rows, g.n_global))
    np.testing.assert_allclose(y, A @ x.astype(np.float64), rtol=1e-13, atol=0)
    ones = np.ones(g.n_global, dtype=np.float32)
    rs = oracle.spmv(g.row_ptr, g.col_idx, val, ones)
    np.testing.assert_allclose(rs, np.add.reduceat(np.r_[val.astype(np.float64), 0], g.row_ptr[:-1])
                               * (np.diff(g.row_ptr) > 0), rtol=1e-13)


def test_openmp_context_line_is_bit_identical():
    """The "CPU-parallel" context line (oracle/orc_par.c) only splits the row loop."""
    import inlgen
    g = inlgen.host_build(14, 16, seed=inlgen.SEED_GRAPH)
    val = inlgen.values_host(g.row_ptr, g.col_idx)
    x = inlgen.vector_host(g.n_global)
    assert np.array_equal(oracle.spmv_par(g.row_ptr, g.col_idx, val, x), oracle.spmv(g.row_ptr, g.col_idx, val, x))
    assert oracle.par_threads() >= 1
