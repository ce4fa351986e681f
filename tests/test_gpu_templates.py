"""GPU parity of the paper's load-balancing templates (templates.cu) vs the oracle.

dual-queue (Fig. 1(b), P5@2074), dbuf-global and dbuf-shared (Fig. 1(c), P5@2717,
P5@3623) for SpMV, over lbTHRES (P5@332) and CTA sizes (P5@11808, P11@1656).
Bar: integer-valued SpMV bit-exact; fp32 max relative error <= 1e-5.
"""
import numpy as np
import pytest
import torch

import inlgen
import oracle
from graphs import csr_from_edges
from paper_conf_icpp_liwb15_b200 import inl

pytestmark = pytest.mark.gpu
TPL = {"dual_queue": inl.BINS_TPL_DUAL_QUEUE, "dbuf_global": inl.BINS_TPL_DBUF_GLOBAL,
       "dbuf_shared": inl.BINS_TPL_DBUF_SHARED}


def dev(a):
    return torch.from_numpy(np.ascontiguousarray(a)).cuda()


@pytest.fixture(scope="module")
def ctx():
    return inl.Ctx(0)


@pytest.fixture(scope="module")
def g14():
    return inlgen.host_build(14, 16, seed=inlgen.SEED_GRAPH)


def run(ctx, rp, ci, n, val, x, flags, lbt, cta):
    A = inl.Csr(dev(rp), dev(ci), n)
    plan = inl.Plan(ctx, A, inl.bins(t_thread=lbt if lbt > 0 else -1, t_warp=max(lbt, 16),
                                      t_block=max(lbt, 16), cta_threads=cta, flags=flags))
    y = torch.full((len(rp) - 1,), float("nan"), device="cuda")
    inl.spmv(ctx, A, dev(val), dev(x), y, plan)
    torch.cuda.synchronize()
    return y.cpu().numpy().astype(np.float64)


@pytest.mark.parametrize("name", sorted(TPL))
@pytest.mark.parametrize("lbt,cta", [(0, 64), (8, 192), (32, 256), (128, 64), (1024, 1024)])
def test_template_integer_bit_exact(ctx, g14, name, lbt, cta):
    val = inlgen.values_host(g14.row_ptr, g14.col_idx, mode=1)
    x = inlgen.vector_host(g14.n_global, mode=1)
    ref = oracle.spmv(g14.row_ptr, g14.col_idx, val, x)
    y = run(ctx, g14.row_ptr, g14.col_idx, g14.n_global, val, x, TPL[name], lbt, cta)
    assert np.array_equal(y, ref)


@pytest.mark.parametrize("name", sorted(TPL))
def test_template_uniform_and_star(ctx, g14, name):
    val = inlgen.values_host(g14.row_ptr, g14.col_idx)
    x = inlgen.vector_host(g14.n_global)
    ref = oracle.spmv(g14.row_ptr, g14.col_idx, val, x)
    y = run(ctx, g14.row_ptr, g14.col_idx, g14.n_global, val, x, TPL[name], 32, 192)
    nz = ref != 0
    assert np.all(y[~nz] == 0) and np.max(np.abs(y[nz] - ref[nz]) / ref[nz]) <= 1e-5
    # one row far above lbTHRES among empty and short rows
    n = 5000
    e = [(0, i) for i in range(1, n)] + [(i, (i * 7) % n) for i in range(2, n, 3)]
    rp, ci, w = csr_from_edges(n, e, np.ones(len(e), np.uint32), symmetric=False)
    v = (np.arange(len(ci)) % 5 + 1).astype(np.float32)
    xx = (np.arange(n) % 3).astype(np.float32)
    assert np.array_equal(run(ctx, rp, ci, n, v, xx, TPL[name], 16, 64), oracle.spmv(rp, ci, v, xx))


@pytest.mark.parametrize("name", ["thread_only", "dual_queue", "dbuf_global", "dbuf_shared"])
@pytest.mark.parametrize("lbt", [8, 64])
def test_pagerank_templates(ctx, name, lbt):
    """PageRank through the paper's templates / its T1 baseline (template study, one GPU) vs the
    20-iteration oracle, <= 1e-5."""
    g = inlgen.host_build(14, 16, seed=inlgen.SEED_GRAPH, flags=inlgen.TRANSPOSE)
    A = inl.Csr(dev(g.row_ptr), dev(g.col_idx), g.n_global)
    fl = inl.BINS_THREAD_ONLY if name == "thread_only" else TPL[name]
    plan = inl.Plan(ctx, A, inl.bins(t_thread=lbt, t_warp=max(lbt, 16), t_block=max(lbt, 16), cta_threads=64,
                                     flags=fl))
    r = torch.empty(g.n_global, device="cuda")
    inl.pagerank(ctx, A, dev(g.out_degree), r, 0.85, 20, plan)
    ref = oracle.pagerank(g.n_global, g.row_ptr, g.col_idx, g.out_degree, 0.85, 20)
    assert np.max(np.abs(r.cpu().numpy().astype(np.float64) - ref) / ref) <= 1e-5


def test_template_flag_combinations(ctx, g14):
    A = inl.Csr(dev(g14.row_ptr), dev(g14.col_idx), g14.n_global)
    # more than one template, or a template with another flag: rejected when the plan is made
    for fl in (inl.BINS_TPL_DBUF_SHARED | inl.BINS_TPL_DUAL_QUEUE, inl.BINS_TPL_DUAL_QUEUE | inl.BINS_TPL_DBUF_GLOBAL,
               inl.BINS_TPL_DBUF_SHARED | inl.BINS_TPL_DBUF_GLOBAL, inl.BINS_TPL_DBUF_GLOBAL | inl.BINS_THREAD_ONLY):
        with pytest.raises(RuntimeError):
            inl.Plan(ctx, A, inl.bins(flags=fl))


@pytest.mark.parametrize("name", ["dbuf_global", "dbuf_shared", "dual_queue"])
@pytest.mark.parametrize("lbt", [0, 8, 32, 1024])
def test_frontier_templates_bit_exact(ctx, name, lbt):
    """SSSP / BFS through the paper's templates (plain frontier Bellman-Ford / top-down BFS)."""
    g = inlgen.host_build(12, 16, seed=inlgen.SEED_GRAPH, flags=inlgen.SYMMETRIC)
    w = inlgen.weights_host(g.row_ptr, g.col_idx)
    A = inl.Csr(dev(g.row_ptr), dev(g.col_idx), g.n_global)
    plan = inl.Plan(ctx, A, inl.bins(t_thread=lbt if lbt > 0 else -1, t_warp=max(lbt, 16), t_block=max(lbt, 16),
                                      flags=TPL[name]))
    for s in inlgen.sources(g.row_ptr, 3):
        d = torch.zeros(g.n_global, dtype=torch.int32, device="cuda")
        inl.sssp(ctx, A, dev(w.view(np.int32)), s, d, plan)
        assert np.array_equal(d.cpu().numpy().view(np.uint32), oracle.sssp(g.row_ptr, g.col_idx, w, s))
        lv = torch.zeros(g.n_global, dtype=torch.int32, device="cuda")
        inl.bfs(ctx, A, s, lv, plan)
        assert np.array_equal(lv.cpu().numpy(), oracle.bfs(g.row_ptr, g.col_idx, s))


def test_dual_queue_frontier_hub_and_empty(ctx):
    """Dual-queue on the frontier: a hub far above lbTHRES (large queue, one CTA) next to a path,
    and an isolated source (empty queues)."""
    n = 30000
    e = [(0, i) for i in range(1, n - 100)] + [(i, i + 1) for i in range(n - 101, n - 1)]
    rp, ci, w = csr_from_edges(n, e, np.arange(len(e)) % 255 + 1, symmetric=True)
    A = inl.Csr(dev(rp), dev(ci), n)
    plan = inl.Plan(ctx, A, inl.bins(t_thread=32, flags=inl.BINS_TPL_DUAL_QUEUE))
    for s in (0, n - 1, 5):
        d = torch.zeros(n, dtype=torch.int32, device="cuda")
        inl.sssp(ctx, A, dev(w.view(np.int32)), s, d, plan)
        assert np.array_equal(d.cpu().numpy().view(np.uint32), oracle.sssp(rp, ci, w, s))
        lv = torch.zeros(n, dtype=torch.int32, device="cuda")
        inl.bfs(ctx, A, s, lv, plan)
        assert np.array_equal(lv.cpu().numpy(), oracle.bfs(rp, ci, s))
    rp, ci, w = csr_from_edges(6, [(1, 2), (2, 3)], [5, 6], symmetric=True)
    A = inl.Csr(dev(rp), dev(ci), 6)
    d = torch.zeros(6, dtype=torch.int32, device="cuda")
    inl.sssp(ctx, A, dev(w.view(np.int32)), 0, d, inl.Plan(ctx, A, inl.bins(t_thread=1, flags=inl.BINS_TPL_DUAL_QUEUE)))
    assert d.cpu().numpy().view(np.uint32).tolist() == [0] + [0xFFFFFFFF] * 5
