"""GPU parity: inl_bc (CUDA through the C-ABI) vs oracle.bc (Brandes, fp64 CPU).

Bar: fp64 on both sides; the sums differ only in order (thread-serial rows follow the
oracle's order, warp / CTA rows use fixed trees), so max relative error <= 1e-9 and
vertices of zero betweenness exactly 0.  Path counts are integers (exact in fp64).
"""
import numpy as np
import pytest
import torch

import inlgen
import oracle
from graphs import csr_from_edges
from paper_conf_icpp_liwb15_b200 import inl

pytestmark = pytest.mark.gpu
RTOL = 1e-9


def dev(a):
    return torch.from_numpy(np.ascontiguousarray(a)).cuda()


@pytest.fixture(scope="module")
def ctx():
    return inl.Ctx(0)


@pytest.fixture(params=["level", "src"])
def mode(request, monkeypatch):
    """Both non-template paths: level-synchronous, source-parallel (bc.cu)."""
    monkeypatch.setenv("INL_BC_MODE", request.param)
    return request.param


def gpu_bc(ctx, rp, ci, n, sources):
    out = torch.full((n,), float("nan"), dtype=torch.float64, device="cuda")
    st = inl.bc(ctx, inl.Csr(dev(rp), dev(ci), n), sources, out)
    return out.cpu().numpy(), st


def check(got, ref):
    z = ref == 0
    assert np.all(got[z] == 0), "zero betweenness must be exactly 0"
    if (~z).any():
        assert np.max(np.abs(got[~z] - ref[~z]) / ref[~z]) <= RTOL


def test_closed_forms(ctx, mode):
    n = 40
    rp, ci, _ = csr_from_edges(n, [(i, i + 1) for i in range(n - 1)], symmetric=True)
    got, _ = gpu_bc(ctx, rp, ci, n, range(n))
    assert np.array_equal(got, [2.0 * i * (n - 1 - i) for i in range(n)])
    k = 5000  # hub above the warp bin: CTA-mapped (global delayed buffer) in both phases
    rp, ci, _ = csr_from_edges(k + 1, [(0, i) for i in range(1, k + 1)], symmetric=True)
    got, _ = gpu_bc(ctx, rp, ci, k + 1, range(0, k + 1, 7))
    ref = oracle.bc(rp, ci, range(0, k + 1, 7))
    check(got, ref)
    assert got[0] == ref[0]  # integer-valued for a star
    n = 30
    rp, ci, _ = csr_from_edges(n, [(i, j) for i in range(n) for j in range(i + 1, n)], symmetric=True)
    assert np.all(gpu_bc(ctx, rp, ci, n, range(n))[0] == 0)


def test_cfg1_exact_all_sources(ctx, mode):
    g = inlgen.host_build(12, 16, seed=inlgen.SEED_GRAPH, flags=inlgen.SYMMETRIC)
    got, st = gpu_bc(ctx, g.row_ptr, g.col_idx, g.n_global, range(g.n_global))
    check(got, oracle.bc(g.row_ptr, g.col_idx))
    assert st["iterations"] >= g.n_global


def test_directed_and_repeatable(ctx, mode):
    g = inlgen.host_build(13, 16, seed=inlgen.SEED_GRAPH)  # directed R-MAT
    srcs = inlgen.sources(g.row_ptr, 16)
    got, _ = gpu_bc(ctx, g.row_ptr, g.col_idx, g.n_global, srcs)
    check(got, oracle.bc(g.row_ptr, g.col_idx, srcs))
    again, _ = gpu_bc(ctx, g.row_ptr, g.col_idx, g.n_global, srcs)
    assert np.array_equal(got, again)


def test_scale16_sources(ctx, mode):
    g = inlgen.host_build(16, 16, seed=inlgen.SEED_GRAPH, flags=inlgen.SYMMETRIC)
    srcs = inlgen.sources(g.row_ptr, 8)
    got, _ = gpu_bc(ctx, g.row_ptr, g.col_idx, g.n_global, srcs)
    check(got, oracle.bc(g.row_ptr, g.col_idx, srcs))


def test_random_small_and_edge_cases(ctx, mode):
    rng = np.random.default_rng(3)
    for trial in range(30):
        n = int(rng.integers(1, 40))
        e = [(int(rng.integers(n)), int(rng.integers(n))) for _ in range(int(rng.integers(0, 4 * n)))]
        rp, ci, _ = csr_from_edges(n, e, symmetric=bool(trial % 2))
        srcs = sorted(set(int(v) for v in rng.integers(0, n, size=5)))
        got, _ = gpu_bc(ctx, rp, ci, n, srcs)
        check(got, oracle.bc(rp, ci, srcs))
    rp, ci, _ = csr_from_edges(4, [(1, 2)], symmetric=True)
    got, _ = gpu_bc(ctx, rp, ci, 4, [])  # no sources: zeros
    assert np.all(got == 0)
    out = np.full(4, np.nan)  # host output buffer
    inl.bc(ctx, inl.Csr(rp, ci, 4), [0, 1], out)
    assert np.all(out == 0)
    with pytest.raises(RuntimeError):
        gpu_bc(ctx, rp, ci, 4, [4])


def test_pull_steps_with_symmetric_plan(ctx, monkeypatch):
    """With a plan that verified symmetry, large frontiers are expanded by pull steps."""
    monkeypatch.setenv("INL_BC_MODE", "level")
    g = inlgen.host_build(15, 16, seed=inlgen.SEED_GRAPH, flags=inlgen.SYMMETRIC)
    A = inl.Csr(dev(g.row_ptr), dev(g.col_idx), g.n_global)
    plan = inl.Plan(ctx, A)
    assert plan.info()["symmetric"] == 1
    srcs = inlgen.sources(g.row_ptr, 6)
    out = torch.empty(g.n_global, dtype=torch.float64, device="cuda")
    inl.bc(ctx, A, srcs, out, plan)
    got = out.cpu().numpy()
    check(got, oracle.bc(g.row_ptr, g.col_idx, srcs))
    plain, _ = gpu_bc(ctx, g.row_ptr, g.col_idx, g.n_global, srcs)  # push-only path
    check(got, plain)
    d = inlgen.host_build(13, 16, seed=inlgen.SEED_GRAPH)  # directed: plan must not pull
    Ad = inl.Csr(dev(d.row_ptr), dev(d.col_idx), d.n_global)
    pd = inl.Plan(ctx, Ad)
    out = torch.empty(d.n_global, dtype=torch.float64, device="cuda")
    s = inlgen.sources(d.row_ptr, 4)
    inl.bc(ctx, Ad, s, out, pd)
    check(out.cpu().numpy(), oracle.bc(d.row_ptr, d.col_idx, s))


TEMPLATES = {"thread_only": inl.BINS_THREAD_ONLY, "dual_queue": inl.BINS_TPL_DUAL_QUEUE,
             "dbuf_global": inl.BINS_TPL_DBUF_GLOBAL, "dbuf_shared": inl.BINS_TPL_DBUF_SHARED}


def tpl_bc(ctx, h, srcs, flags, lbt, cta=192):
    A = inl.Csr(dev(h.row_ptr), dev(h.col_idx), h.n_global)
    plan = inl.Plan(ctx, A, inl.bins(t_thread=lbt, cta_threads=cta, flags=flags))
    out = torch.full((h.n_global,), float("nan"), dtype=torch.float64, device="cuda")
    st = inl.bc(ctx, A, srcs, out, plan)
    return out.cpu().numpy(), st


@pytest.mark.parametrize("name", sorted(TEMPLATES))
@pytest.mark.parametrize("lbt", [1, 32, 1024])
def test_templates_wikivote_shaped(ctx, name, lbt):
    """Fig. 6 BC bars: the paper's templates (and T1) over lbTHRES on the Wiki-vote-shaped
    graph; thread-serial vertices and CTA-tree vertices both appear at lbt 1 and 32."""
    h = inlgen.wikivote_like()
    srcs = inlgen.sources(h.row_ptr, 6)
    got, st = tpl_bc(ctx, h, srcs, TEMPLATES[name], lbt)
    check(got, oracle.bc(h.row_ptr, h.col_idx, srcs))
    assert st["iterations"] >= len(srcs)


@pytest.mark.parametrize("name", sorted(TEMPLATES))
def test_templates_star_path_and_directed(ctx, name):
    k = 3000  # the hub is block-mapped under every template but T1
    rp, ci, _ = csr_from_edges(k + 1, [(0, i) for i in range(1, k + 1)], symmetric=True)
    h = inlgen.HostGraph(k + 1, 0, rp, ci)
    srcs = list(range(0, k + 1, 97))
    got, _ = tpl_bc(ctx, h, srcs, TEMPLATES[name], 16, 128)
    ref = oracle.bc(rp, ci, srcs)
    check(got, ref)
    n = 50
    rp, ci, _ = csr_from_edges(n, [(i, i + 1) for i in range(n - 1)], symmetric=True)
    got, _ = tpl_bc(ctx, inlgen.HostGraph(n, 0, rp, ci), range(n), TEMPLATES[name], 1, 64)
    assert np.array_equal(got, [2.0 * i * (n - 1 - i) for i in range(n)])
    d = inlgen.host_build(13, 16, seed=inlgen.SEED_GRAPH)  # directed R-MAT
    s = inlgen.sources(d.row_ptr, 4)
    got, _ = tpl_bc(ctx, d, s, TEMPLATES[name], 32, 256)
    check(got, oracle.bc(d.row_ptr, d.col_idx, s))


# ---- source-parallel BC (one CTA per source; bc.cu k_bc_src) -------------------------------

@pytest.fixture
def src_mode(monkeypatch):
    monkeypatch.setenv("INL_BC_MODE", "src")


def test_source_parallel_wikivote_auto(ctx):
    """Many sources on the Wiki-vote-shaped graph: the auto choice is the source-parallel
    kernel (state in shared memory), one launch pair, no host sync per level."""
    h = inlgen.wikivote_like()
    srcs = inlgen.sources(h.row_ptr, 300)
    got, st = gpu_bc(ctx, h.row_ptr, h.col_idx, h.n_global, srcs)
    assert st["launches"] == 2 and st["host_syncs"] == 0
    check(got, oracle.bc(h.row_ptr, h.col_idx, srcs))
    again, _ = gpu_bc(ctx, h.row_ptr, h.col_idx, h.n_global, srcs)
    assert np.array_equal(got, again)  # static source -> CTA assignment, CTA-ordered reduction
    g = inlgen.host_build(18, 16, seed=inlgen.SEED_GRAPH, flags=inlgen.SYMMETRIC)
    s8 = inlgen.sources(g.row_ptr, 8)  # few sources on a larger graph: level-synchronous
    got, st2 = gpu_bc(ctx, g.row_ptr, g.col_idx, g.n_global, s8)
    assert st2["launches"] > 2
    check(got, oracle.bc(g.row_ptr, g.col_idx, s8))


def test_source_parallel_closed_forms(ctx, src_mode):
    n = 40
    rp, ci, _ = csr_from_edges(n, [(i, i + 1) for i in range(n - 1)], symmetric=True)
    got, st = gpu_bc(ctx, rp, ci, n, range(n))
    assert np.array_equal(got, [2.0 * i * (n - 1 - i) for i in range(n)])
    assert st["iterations"] == sum(max(i, n - 1 - i) + 1 for i in range(n))
    k = 5000  # hub: warp-mapped inside the CTA in both sweeps
    rp, ci, _ = csr_from_edges(k + 1, [(0, i) for i in range(1, k + 1)], symmetric=True)
    got, _ = gpu_bc(ctx, rp, ci, k + 1, range(0, k + 1, 7))
    ref = oracle.bc(rp, ci, range(0, k + 1, 7))
    check(got, ref)
    assert got[0] == ref[0]


@pytest.mark.parametrize("scale", [13, 14])  # 13: state in shared memory; 14: global slices
def test_source_parallel_rmat(ctx, src_mode, scale):
    for flags in (0, inlgen.SYMMETRIC):
        g = inlgen.host_build(scale, 16, seed=inlgen.SEED_GRAPH, flags=flags)
        srcs = inlgen.sources(g.row_ptr, 200)
        got, st = gpu_bc(ctx, g.row_ptr, g.col_idx, g.n_global, srcs)
        check(got, oracle.bc(g.row_ptr, g.col_idx, srcs))
        assert st["launches"] == 2


def test_source_parallel_edge_cases(ctx, src_mode):
    rng = np.random.default_rng(5)
    for trial in range(20):
        n = int(rng.integers(1, 40))
        e = [(int(rng.integers(n)), int(rng.integers(n))) for _ in range(int(rng.integers(0, 4 * n)))]
        rp, ci, _ = csr_from_edges(n, e, symmetric=bool(trial % 2))
        srcs = [int(v) for v in rng.integers(0, n, size=7)]  # repeats allowed
        got, _ = gpu_bc(ctx, rp, ci, n, srcs)
        check(got, oracle.bc(rp, ci, srcs))
    rp, ci, _ = csr_from_edges(5, [], symmetric=True)  # edgeless: every source isolated
    got, st = gpu_bc(ctx, rp, ci, 5, range(5))
    assert np.all(got == 0) and st["iterations"] == 5
