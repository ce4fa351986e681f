"""The seeded input generator (host side): Philox known answers, the relabel
bijection, CSR invariants, and an independent numpy rebuild of the CSR from the
raw R-MAT tuples."""
import numpy as np
import pytest

import inlgen


def test_philox_known_answers():
    # Random123 kat_vectors, philox4x32_10
    assert inlgen.philox([0, 0, 0, 0], [0, 0]) == [0x6627E8D5, 0xE169C58D, 0xBC57AC4C, 0x9B00DBD8]
    assert inlgen.philox([0xFFFFFFFF] * 4, [0xFFFFFFFF] * 2) == [0x408F276D, 0x41C83B0E, 0xA20BC7C6,
                                                                0x6D5451FD]
    assert inlgen.philox([0x243F6A88, 0x85A308D3, 0x13198A2E, 0x03707344], [0xA4093822, 0x299F31D0]) == \
        [0xD16CFE09, 0x94FDCCEB, 0x5001E420, 0x24126EA1]


@pytest.mark.parametrize("scale", [1, 2, 3, 7, 12, 16])
def test_relabel_is_bijection(scale):
    n = 1 << scale
    img = np.array([inlgen.relabel(x, scale) for x in range(n)]) if scale <= 12 else None
    if img is None:
        xs = np.random.default_rng(0).choice(n, 4096, replace=False)
        ys = [inlgen.relabel(int(x), scale) for x in xs]
        assert len(set(ys)) == len(ys) and max(ys) < n
    else:
        assert sorted(img.tolist()) == list(range(n))


@pytest.mark.parametrize("flags", [0, inlgen.SYMMETRIC, inlgen.TRANSPOSE])
def test_csr_matches_numpy_rebuild_from_tuples(flags):
    scale, ef = 10, 16
    g = inlgen.host_build(scale, ef, seed=9, flags=flags)
    u, v = inlgen.rmat_tuples(scale, 9, 0, ef << scale)
    keep = u != v
    u, v = u[keep], v[keep]
    if flags & inlgen.SYMMETRIC:
        u, v = np.r_[u, v], np.r_[v, u]
    if flags & inlgen.TRANSPOSE:
        u, v = v, u
    keys = np.unique(u * (1 << scale) + v)
    rows, cols = keys >> scale, keys & ((1 << scale) - 1)
    assert g.nnz == len(keys)
    assert np.array_equal(g.col_idx, cols.astype(np.int32))
    assert np.array_equal(g.row_ptr, np.searchsorted(rows, np.arange((1 << scale) + 1)))


def test_csr_invariants_and_shape():
    g = inlgen.host_build(12, 16, seed=1)
    rp, ci = g.row_ptr, g.col_idx
    assert rp[0] == 0 and np.all(np.diff(rp) >= 0)
    rows = np.repeat(np.arange(g.n_rows), np.diff(rp))
    assert np.all(ci != rows)  # no self-loops
    same = rows[1:] == rows[:-1]
    assert np.all(ci[1:][same] > ci[:-1][same])  # sorted, unique
    # R-MAT shape at scale 12 (SURVEY §8 preamble: ~53.5K directed nnz, max degree ~900)
    assert 50_000 < g.nnz < 56_000
    assert 500 < np.diff(rp).max() < 2000
    s = inlgen.host_build(12, 16, seed=1, flags=inlgen.SYMMETRIC)
    A = set(zip(np.repeat(np.arange(s.n_rows), np.diff(s.row_ptr)).tolist(), s.col_idx.tolist()))
    assert all((b, a) in A for a, b in A)


def test_row_range_slices_the_full_graph():
    full = inlgen.host_build(9, 16, seed=5, flags=inlgen.SYMMETRIC)
    part = inlgen.host_build(9, 16, seed=5, flags=inlgen.SYMMETRIC, row_begin=100, row_end=300)
    lo, hi = full.row_ptr[100], full.row_ptr[300]
    assert np.array_equal(part.row_ptr, full.row_ptr[100:301] - lo)
    assert np.array_equal(part.col_idx, full.col_idx[lo:hi])


def test_weights_symmetric_in_range_and_values():
    g = inlgen.host_build(10, 16, seed=1, flags=inlgen.SYMMETRIC)
    w = inlgen.weights_host(g.row_ptr, g.col_idx)
    assert w.min() >= 1 and w.max() <= 255
    rows = np.repeat(np.arange(g.n_rows), np.diff(g.row_ptr))
    d = {(a, b): x for a, b, x in zip(rows.tolist(), g.col_idx.tolist(), w.tolist())}
    assert all(d[(b, a)] == x for (a, b), x in d.items())
    v = inlgen.values_host(g.row_ptr, g.col_idx)
    assert v.min() >= 0 and v.max() < 1 and len(np.unique(v)) > 0.9 * len(v)
    vi = inlgen.values_host(g.row_ptr, g.col_idx, mode=1)
    assert vi.min() >= 1 and vi.max() <= 255 and np.all(vi == np.round(vi))
    x = inlgen.vector_host(1000, mode=1)
    assert x.min() >= 0 and x.max() <= 15
    # values keyed by (row, col): a row-range build gets identical values
    part = inlgen.host_build(10, 16, seed=1, flags=inlgen.SYMMETRIC, row_begin=10, row_end=20)
    vp = inlgen.values_host(part.row_ptr, part.col_idx, row_begin=10)
    assert np.array_equal(vp, v[g.row_ptr[10]:g.row_ptr[20]])
