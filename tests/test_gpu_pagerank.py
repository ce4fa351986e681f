"""GPU parity: inl_pagerank (CUDA through the C-ABI) vs oracle.pagerank (fp64).

Bar: max relative error <= 1e-5 (fp32) after 20 iterations, d = 0.85."""
import numpy as np
import pytest
import torch

import inlgen
import oracle
from paper_conf_icpp_liwb15_b200 import inl

pytestmark = pytest.mark.gpu
RTOL = 1e-5


def dev(a):
    return torch.from_numpy(np.ascontiguousarray(a)).cuda()


@pytest.fixture(scope="module")
def ctx():
    return inl.Ctx(0)


def run(ctx, g_rp, g_ci, od, n, iters=20, d=0.85, b=None, use_plan=True):
    A = inl.Csr(dev(g_rp), dev(g_ci), n)
    r = torch.full((n,), float("nan"), device="cuda")
    plan = inl.Plan(ctx, A, b) if use_plan else None
    inl.pagerank(ctx, A, dev(od), r, d, iters, plan)
    torch.cuda.synchronize()
    return r.cpu().numpy().astype(np.float64)


@pytest.mark.parametrize("kw", [dict(), dict(t_thread=-1, t_warp=128, t_block=128, grid_chunk=64),
                                dict(t_thread=32, t_warp=64, t_block=1024, grid_chunk=1000, cta_threads=512)])
def test_cfg1_matches_oracle(ctx, kw):
    g = inlgen.host_build(12, 16, seed=inlgen.SEED_GRAPH, flags=inlgen.TRANSPOSE)
    ref = oracle.pagerank(g.n_global, g.row_ptr, g.col_idx, g.out_degree, 0.85, 20)
    r = run(ctx, g.row_ptr, g.col_idx, g.out_degree, g.n_global, b=inl.bins(**kw))
    assert np.max(np.abs(r - ref) / ref) <= RTOL
    assert abs(r.sum() - 1.0) < 1e-5


@pytest.mark.parametrize("iters", [0, 1, 2, 7])
def test_iteration_counts_and_transient_plan(ctx, iters):
    g = inlgen.host_build(10, 16, seed=3, flags=inlgen.TRANSPOSE)
    ref = oracle.pagerank(g.n_global, g.row_ptr, g.col_idx, g.out_degree, 0.85, iters)
    r = run(ctx, g.row_ptr, g.col_idx, g.out_degree, g.n_global, iters=iters, use_plan=False)
    assert np.max(np.abs(r - ref) / ref) <= RTOL


def test_star_closed_form(ctx):
    k, d = 7, 0.85
    n = k + 1
    # in-CSR of the symmetric star: hub 0 <- leaves, leaf i <- hub
    rp = np.array([0, k] + [k + i for i in range(1, k + 1)], np.int64)
    ci = np.array(list(range(1, n)) + [0] * k, np.int32)
    od = np.array([k] + [1] * k, np.int32)
    r = run(ctx, rp, ci, od, n, iters=20, d=d)
    assert abs(r[0] - 0.45623827) < 1e-6


def test_damping_zero_and_edgeless(ctx):
    g = inlgen.host_build(9, 16, seed=2, flags=inlgen.TRANSPOSE)
    r = run(ctx, g.row_ptr, g.col_idx, g.out_degree, g.n_global, d=0.0)
    np.testing.assert_allclose(r, 1.0 / g.n_global, rtol=1e-6)
    n = 100
    r = run(ctx, np.zeros(n + 1, np.int64), np.zeros(0, np.int32), np.zeros(n, np.int32), n)
    np.testing.assert_allclose(r, 0.01, rtol=1e-6)


def test_bad_damping_rejected(ctx):
    g = inlgen.host_build(6, 4, seed=2, flags=inlgen.TRANSPOSE)
    with pytest.raises(inl.InlError):
        run(ctx, g.row_ptr, g.col_idx, g.out_degree, g.n_global, d=1.0)


def test_scale18_against_oracle(ctx):
    g = inlgen.dev_build(18, 16, seed=inlgen.SEED_GRAPH, flags=inlgen.TRANSPOSE)
    A = inl.Csr(g["row_ptr"], g["col_idx"], g["n_global"])
    r = torch.empty(g["n_global"], device="cuda")
    inl.pagerank(ctx, A, g["out_degree"], r, 0.85, 20, inl.Plan(ctx, A))
    ref = oracle.pagerank(g["n_global"], g["row_ptr"].cpu().numpy(), g["col_idx"].cpu().numpy(),
                          g["out_degree"].cpu().numpy(), 0.85, 20)
    rr = r.cpu().numpy().astype(np.float64)
    assert np.max(np.abs(rr - ref) / ref) <= RTOL
