"""CPU tests of the CSR loaders and the CiteSeer-shaped generator (input side, SURVEY §8a row
a1: "a CSR generator and loader"; PAPER.md P11@2099 CSR encoding, P5@12491-13052 CiteSeer).

Pins: hand-written MatrixMarket files with duplicates / self-loops / comments against an
expected CSR written out by hand, scipy.io.mmread on a clean file, SYMMETRIC / TRANSPOSE
orientation, .inlcsr round trips (with values and out-degrees) and malformed-file errors, and
the generator's shape (n, entries, degree range and mean of PAPER.md's CiteSeer)."""
import os

import numpy as np
import pytest
import scipy.io
import scipy.sparse as sp

import inlgen

MTX_GENERAL = """%%MatrixMarket matrix coordinate real general
% a comment
4 5 7
1 2 1.5
1 2 9.0
2 2 3.0
3 1 -2.0
1 5 0.25
4 4 7.0
3 3 1.0
"""


def _write(tmp_path, name, txt):
    p = os.path.join(tmp_path, name)
    with open(p, "w") as f:
        f.write(txt)
    return p


def test_mtx_general_duplicates_selfloops(tmp_path):
    g = inlgen.load_mtx(_write(tmp_path, "a.mtx", MTX_GENERAL))
    # rows: 0 -> {1: 1.5 (first of the duplicate pair), 4: 0.25}; 1 -> {} (self-loop);
    # 2 -> {0: -2.0} (self-loop (2,2) dropped); 3 -> {} (self-loop)
    assert g.n_global == 5 and g.n_rows == 4
    assert g.row_ptr.tolist() == [0, 2, 2, 3, 3]
    assert g.col_idx.tolist() == [1, 4, 0]
    assert g.val.tolist() == [1.5, 0.25, -2.0]


def test_mtx_matches_scipy_on_clean_file(tmp_path):
    rng = np.random.default_rng(3)
    n = 60
    A = sp.random(n, n, density=0.1, random_state=rng, format="coo", dtype=np.float32)
    A.setdiag(0)
    A.eliminate_zeros()
    p = os.path.join(tmp_path, "r.mtx")
    scipy.io.mmwrite(p, A)
    g = inlgen.load_mtx(p)
    B = sp.csr_matrix(scipy.io.mmread(p)).astype(np.float32)
    B.sort_indices()
    assert np.array_equal(g.row_ptr, B.indptr.astype(np.int64))
    assert np.array_equal(g.col_idx, B.indices.astype(np.int32))
    assert np.array_equal(g.val, B.data.astype(np.float32))


def test_mtx_symmetric_storage_and_flags(tmp_path):
    txt = "%%MatrixMarket matrix coordinate pattern symmetric\n4 4 3\n2 1\n3 1\n4 3\n"
    p = _write(tmp_path, "s.mtx", txt)
    g = inlgen.load_mtx(p)
    A = sp.csr_matrix((np.ones(len(g.col_idx)), g.col_idx, g.row_ptr), shape=(4, 4)).toarray()
    assert np.array_equal(A, A.T) and A.sum() == 6 and g.val is None
    # a general pattern file + SYMMETRIC flag gives the same graph
    q = _write(tmp_path, "g.mtx", "%%MatrixMarket matrix coordinate pattern general\n4 4 3\n2 1\n1 3\n4 3\n")
    h = inlgen.load_mtx(q, inlgen.SYMMETRIC)
    assert np.array_equal(h.row_ptr, g.row_ptr) and np.array_equal(h.col_idx, g.col_idx)
    # TRANSPOSE: in-CSR (rows = destinations) + out-degrees of the directed file
    t = inlgen.load_mtx(q, inlgen.TRANSPOSE)
    At = sp.csr_matrix((np.ones(len(t.col_idx)), t.col_idx, t.row_ptr), shape=(4, 4)).toarray()
    Ad = np.zeros((4, 4))
    Ad[1, 0] = Ad[0, 2] = Ad[3, 2] = 1
    assert np.array_equal(At, Ad.T)
    assert t.out_degree.tolist() == Ad.sum(axis=1).astype(int).tolist()


@pytest.mark.parametrize("txt", [
    "not a header\n1 1 0\n",
    "%%MatrixMarket matrix array real general\n2 2\n1\n2\n3\n4\n",
    "%%MatrixMarket matrix coordinate complex general\n2 2 1\n1 2 1 1\n",
    "%%MatrixMarket matrix coordinate real general\n2 2 2\n1 2 1.0\n",       # truncated
    "%%MatrixMarket matrix coordinate real general\n2 2 1\n3 1 1.0\n",       # out of range
])
def test_mtx_errors(tmp_path, txt):
    with pytest.raises(RuntimeError):
        inlgen.load_mtx(_write(tmp_path, "bad.mtx", txt))


def test_mtx_transpose_needs_square(tmp_path):
    with pytest.raises(RuntimeError):
        inlgen.load_mtx(_write(tmp_path, "a.mtx", MTX_GENERAL), inlgen.TRANSPOSE)


def test_inlcsr_round_trip(tmp_path):
    g = inlgen.host_build(12, 16, seed=inlgen.SEED_GRAPH, flags=inlgen.TRANSPOSE)
    g.val = inlgen.values_host(g.row_ptr, g.col_idx)
    p = os.path.join(tmp_path, "g.inlcsr")
    inlgen.save_inlcsr(p, g)
    h = inlgen.load_inlcsr(p)
    assert (h.n_global, h.n_rows, h.row_begin) == (g.n_global, g.n_rows, g.row_begin)
    assert np.array_equal(h.row_ptr, g.row_ptr) and np.array_equal(h.col_idx, g.col_idx)
    assert np.array_equal(h.val, g.val) and np.array_equal(h.out_degree, g.out_degree)
    # a row block without values / out-degrees
    b = inlgen.host_build(10, 16, seed=inlgen.SEED_GRAPH, row_begin=100, row_end=300)
    inlgen.save_inlcsr(p, b)
    c = inlgen.load_inlcsr(p)
    assert c.row_begin == 100 and c.n_rows == 200 and c.val is None and c.out_degree is None
    assert np.array_equal(c.col_idx, b.col_idx)


def test_inlcsr_rejects_malformed(tmp_path):
    g = inlgen.host_build(8, 8, seed=inlgen.SEED_GRAPH)
    p = os.path.join(tmp_path, "g.inlcsr")
    inlgen.save_inlcsr(p, g)
    raw = open(p, "rb").read()
    for bad in (raw[:-5], b"XXXXXXXX" + raw[8:], raw[:8 + 40 + 8] + (2**40).to_bytes(8, "little") + raw[8 + 40 + 16:]):
        q = os.path.join(tmp_path, "bad.inlcsr")
        open(q, "wb").write(bad)
        with pytest.raises(RuntimeError):
            inlgen.load_inlcsr(q)


def test_powerlaw_small_shape_and_determinism():
    g = inlgen.powerlaw_build(5000, 1, 300, 20.0, seed=7)
    h = inlgen.powerlaw_build(5000, 1, 300, 20.0, seed=7)
    assert np.array_equal(g.row_ptr, h.row_ptr) and np.array_equal(g.col_idx, h.col_idx)
    deg = np.diff(g.row_ptr)
    assert deg.max() <= 300 and abs(deg.mean() - 20.0) < 1.0
    A = sp.csr_matrix((np.ones(len(g.col_idx)), g.col_idx, g.row_ptr), shape=(5000, 5000))
    assert (A != A.T).nnz == 0 and A.diagonal().sum() == 0  # symmetric, no self-loops
    assert all(np.all(np.diff(g.col_idx[g.row_ptr[i]:g.row_ptr[i + 1]]) > 0) for i in range(0, 5000, 97))


@pytest.mark.slow
def test_citeseer_like_shape():
    """PAPER.md P5@12491-13052: 434,102 nodes, degree 1..1,188, mean 73.9 (~32.1 M CSR entries)."""
    g = inlgen.citeseer_like()
    deg = np.diff(g.row_ptr)
    assert g.n_global == 434102
    assert deg.max() <= 1188 and np.mean(deg >= 1) > 0.999
    assert abs(deg.mean() - 73.9) / 73.9 < 0.02
    assert abs(len(g.col_idx) - 32.1e6) / 32.1e6 < 0.02


def test_wikivote_like_shape():
    """PAPER.md P5@13172-13524: Wiki-vote, 7,115 nodes, 103,689 edges, mean outdegree 14.6,
    at most 893 (symmetric stand-in, R7)."""
    g = inlgen.wikivote_like()
    deg = np.diff(g.row_ptr)
    assert g.n_global == 7115
    assert deg.min() >= 1 and deg.max() <= 893
    assert abs(deg.mean() - 14.6) / 14.6 < 0.02
    assert abs(len(g.col_idx) - 103689) / 103689 < 0.02
    assert np.array_equal(inlgen.wikivote_like().col_idx, g.col_idx)  # seeded
