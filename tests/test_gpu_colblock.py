"""GPU parity of the column-blocked deferred bin (colblock.cuh) vs the oracle.

Opt-in (INL_BINS_COLBLOCK).  Rows of degree > max(t_warp, mult * blocks) are summed per column block from a
shared-memory copy of x and combined in block order.  Small block widths
(INL_CB_K, read when a plan is built) force many blocks at test sizes; every
case spans several blocks, partial last blocks and CTA-share boundaries.
Bar: integer-valued SpMV bit-exact; fp32 max relative error <= 1e-5 (SpMV and
PageRank); partition (row-block) invariance bit-exact for integer data.
"""
import numpy as np
import pytest
import torch

import inlgen
import oracle
from paper_conf_icpp_liwb15_b200 import inl

pytestmark = pytest.mark.gpu
RTOL = 1e-5
CB = inl.BINS_COLBLOCK


def dev(a):
    return torch.from_numpy(np.ascontiguousarray(a)).cuda()


def rel_err(y, ref):
    y = np.asarray(y, np.float64)
    nz = ref != 0
    assert np.all(y[~nz] == 0)
    return float(np.max(np.abs(y[nz] - ref[nz]) / np.abs(ref[nz]))) if nz.any() else 0.0


@pytest.fixture(scope="module")
def ctx():
    return inl.Ctx(0)


@pytest.fixture(scope="module")
def g14():
    return inlgen.host_build(14, 16, seed=inlgen.SEED_GRAPH)


def spmv(ctx, g, val, x, bins, row_begin=0, n_rows=None):
    rp, ci, v = g.row_ptr, g.col_idx, val
    if n_rows is not None:  # a row block, as one rank of inl_partition_rows holds it
        lo, hi = rp[row_begin], rp[row_begin + n_rows]
        rp, ci, v = rp[row_begin:row_begin + n_rows + 1] - lo, ci[lo:hi], val[lo:hi]
    A = inl.Csr(dev(rp), dev(ci), g.n_global, row_begin)
    plan = inl.Plan(ctx, A, bins)
    y = torch.full((A.n_rows,), float("nan"), device="cuda")
    inl.spmv(ctx, A, dev(v), dev(x), y, plan)
    torch.cuda.synchronize()
    return y.cpu().numpy(), plan.info()


@pytest.mark.parametrize("K,mult,t_warp", [(256, 1, 32), (1000, 2, 64), (4096, 1, 16), (64, 4, 128)])
def test_spmv_colblock_integer_bit_exact(ctx, g14, monkeypatch, K, mult, t_warp):
    monkeypatch.setenv("INL_CB_K", str(K))
    monkeypatch.setenv("INL_CB_MULT", str(mult))
    val = inlgen.values_host(g14.row_ptr, g14.col_idx, mode=1)
    x = inlgen.vector_host(g14.n_global, mode=1)
    ref = oracle.spmv(g14.row_ptr, g14.col_idx, val, x)
    y, info = spmv(ctx, g14, val, x, inl.bins(t_thread=4, t_warp=t_warp, t_block=max(t_warp, 512), grid_chunk=96, flags=CB))
    assert info["cb_rows"] > 0 and info["cb_width"] == (K & ~3)
    assert info["cb_runs"] > info["cb_rows"]  # rows span several blocks
    assert np.array_equal(y.astype(np.float64), ref)


@pytest.mark.parametrize("K", [256, 2052])
def test_spmv_colblock_uniform(ctx, g14, monkeypatch, K):
    monkeypatch.setenv("INL_CB_K", str(K))
    monkeypatch.setenv("INL_CB_MULT", "1")
    val = inlgen.values_host(g14.row_ptr, g14.col_idx)
    x = inlgen.vector_host(g14.n_global)
    ref = oracle.spmv(g14.row_ptr, g14.col_idx, val, x)
    y, info = spmv(ctx, g14, val, x, inl.bins(t_warp=32, flags=CB))
    assert info["cb_rows"] > 0
    assert rel_err(y, ref) <= RTOL


def test_spmv_colblock_deterministic_and_partition_invariant(ctx, g14, monkeypatch):
    monkeypatch.setenv("INL_CB_K", "512")
    monkeypatch.setenv("INL_CB_MULT", "1")
    val = inlgen.values_host(g14.row_ptr, g14.col_idx)
    x = inlgen.vector_host(g14.n_global)
    b = inl.bins(t_warp=32, flags=CB)
    y0, _ = spmv(ctx, g14, val, x, b)
    y1, _ = spmv(ctx, g14, val, x, b)
    assert np.array_equal(y0, y1)  # run to run
    # row blocks (integer data: exact sums, so any difference would be a wrong entry)
    val = inlgen.values_host(g14.row_ptr, g14.col_idx, mode=1)
    x = inlgen.vector_host(g14.n_global, mode=1)
    y0, _ = spmv(ctx, g14, val, x, b)
    n = g14.n_rows
    half = (n // 2 + 127) // 128 * 128
    ya, ia = spmv(ctx, g14, val, x, b, 0, half)
    yb, ib = spmv(ctx, g14, val, x, b, half, n - half)
    assert ia["cb_rows"] > 0 and ib["cb_rows"] > 0
    assert np.array_equal(np.concatenate([ya, yb]), y0)


def test_spmv_colblock_is_opt_in(ctx, g14, monkeypatch):
    monkeypatch.setenv("INL_CB_K", "256")
    val = inlgen.values_host(g14.row_ptr, g14.col_idx, mode=1)
    x = inlgen.vector_host(g14.n_global, mode=1)
    ref = oracle.spmv(g14.row_ptr, g14.col_idx, val, x)
    y, info = spmv(ctx, g14, val, x, inl.bins(t_warp=32))
    assert info["cb_rows"] == 0
    assert np.array_equal(y.astype(np.float64), ref)


@pytest.mark.parametrize("K", [128, 1000])
def test_pagerank_colblock(ctx, monkeypatch, K):
    monkeypatch.setenv("INL_CB_K", str(K))
    monkeypatch.setenv("INL_CB_MULT", "1")
    t = inlgen.host_build(14, 16, seed=inlgen.SEED_GRAPH, flags=inlgen.TRANSPOSE)
    A = inl.Csr(dev(t.row_ptr), dev(t.col_idx), t.n_global)
    plan = inl.Plan(ctx, A, inl.bins(t_warp=32, flags=CB))
    r = torch.empty(t.n_global, device="cuda")
    inl.pagerank(ctx, A, dev(t.out_degree), r, 0.85, 20, plan)
    ref = oracle.pagerank(t.n_global, t.row_ptr, t.col_idx, t.out_degree, 0.85, 20)
    got = r.cpu().numpy().astype(np.float64)
    assert np.max(np.abs(got - ref) / ref) <= RTOL
    assert abs(got.sum() - 1.0) < 1e-4
    r2 = torch.empty_like(r)
    inl.pagerank(ctx, A, dev(t.out_degree), r2, 0.85, 20, plan)
    assert torch.equal(r, r2)
