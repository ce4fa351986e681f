"""Parity at BASELINE.json's full sizes, in the launch configuration bench.py times (plans,
default bins).

* cfg3 SSSP / BFS (R-MAT scale 23, symmetric, w in 1..255): all 9 sources (8 seeded + the
  max-degree vertex) through the exact O(m) shortest-path certificate of tests/graphs.py
  (feasible edges + a tight in-edge for every finite vertex => dist equals the true
  distances, for weights >= 1), evaluated with torch on the GPU (test-side arithmetic on the
  library's outputs); the first 2 sources also bit-exact against oracle Dijkstra / BFS.
* cfg5 BFS (R-MAT scale 26, symmetric, 2.1 B entries): 8 seeded sources, certificate
  evaluated over row ranges.
* cfg4 PageRank (R-MAT scale 25 in-CSR, 528 M entries, 20 iterations): element-wise against
  the oracle's 20 fp64 iterations (SURVEY §8d "Scale of the oracle runs").
"""
import numpy as np
import pytest
import torch

import inlgen
from paper_conf_icpp_liwb15_b200 import inl

pytestmark = pytest.mark.gpu
INF = 0xFFFFFFFF


@pytest.fixture(scope="module")
def ctx():
    return inl.Ctx(0)


def certify_gpu(rp, ci, w, s, dist, chunk=1 << 28):
    """Exact certificate for dist (int64 tensor, INF = unreachable) from source s, evaluated
    over row ranges of <= ~chunk entries (scale 26 has 2.1 B entries).  w = None: unit weights."""
    n = rp.numel() - 1
    nnz = int(rp[-1])
    assert int(dist[s]) == 0
    has = torch.zeros(n, dtype=torch.bool, device=rp.device)
    cuts = torch.searchsorted(rp, torch.arange(0, nnz + chunk, chunk, device=rp.device, dtype=torch.int64))
    cuts = sorted(set([0, n] + [min(int(c), n) for c in cuts.tolist()]))
    for r0, r1 in zip(cuts[:-1], cuts[1:]):
        k0, k1 = int(rp[r0]), int(rp[r1])
        if k1 == k0:
            continue
        deg = rp[r0 + 1:r1 + 1] - rp[r0:r1]
        src = torch.repeat_interleave(torch.arange(r0, r1, device=rp.device, dtype=torch.int64), deg)
        du = dist[src]
        v = ci[k0:k1].long()
        dv = dist[v]
        ww = 1 if w is None else w[k0:k1].long()
        fin = du != INF
        assert not bool(((dv > du + ww) & fin).any()), "infeasible edge"
        tight = fin & (dv == du + ww)
        has[v[tight]] = True
        del src, du, v, dv, fin, tight
    need = dist != INF
    need[s] = False
    assert not bool((need & ~has).any()), "finite vertex without a tight in-edge"


def _levels_as_dist(lv):
    lvl = lv.long()
    return torch.where(lvl < 0, torch.full_like(lvl, INF), lvl)


def test_certificate_rejects_wrong_answers(ctx):
    """The certificate itself: perturbed distances / levels must fail it."""
    g = inlgen.dev_build(14, 16, seed=inlgen.SEED_GRAPH, flags=inlgen.SYMMETRIC)
    rp, ci = g["row_ptr"], g["col_idx"]
    n = g["n_global"]
    w = inlgen.weights_dev(rp, ci)
    wl = w.view(torch.int32).long() & 0xFFFFFFFF
    A = inl.Csr(rp, ci, n)
    s = inlgen.sources(rp.cpu().numpy(), 1)[0]
    d = torch.empty(n, dtype=torch.int32, device="cuda")
    inl.sssp(ctx, A, w, s, d)
    dist = d.long() & 0xFFFFFFFF
    certify_gpu(rp, ci, wl, s, dist, chunk=1 << 16)
    fin = torch.nonzero((dist != INF) & (dist > 0)).flatten()
    for delta in (-1, 1):
        bad = dist.clone()
        bad[fin[len(fin) // 2]] += delta
        with pytest.raises(AssertionError):
            certify_gpu(rp, ci, wl, s, bad, chunk=1 << 16)


def test_cfg3_sssp_bfs_all_sources(ctx):
    """cfg3, the bench's plan: all 9 sources certified; the first 2 equal the oracle."""
    import oracle
    g = inlgen.dev_build(23, 16, seed=inlgen.SEED_GRAPH, flags=inlgen.SYMMETRIC)
    rp, ci = g["row_ptr"], g["col_idx"]
    n = g["n_global"]
    w = inlgen.weights_dev(rp, ci)
    wl = w.view(torch.int32).long() & 0xFFFFFFFF
    A = inl.Csr(rp, ci, n)
    plan = inl.Plan(ctx, A)
    assert plan.info()["symmetric"] == 1  # BFS runs direction-optimizing, as in the bench
    rph = rp.cpu().numpy()
    srcs = inlgen.sources(rph, 8)
    assert len(srcs) == 9
    cih = wh = None
    for i, s in enumerate(srcs):
        d = torch.empty(n, dtype=torch.int32, device="cuda")
        inl.sssp(ctx, A, w, s, d, plan)
        dist = d.long() & 0xFFFFFFFF
        certify_gpu(rp, ci, wl, s, dist)
        lv = torch.empty(n, dtype=torch.int32, device="cuda")
        inl.bfs(ctx, A, s, lv, plan)
        certify_gpu(rp, ci, None, s, _levels_as_dist(lv))
        assert int((lv >= 0).sum()) == int((d != -1).sum())  # same reached set
        if i < 2:
            if cih is None:
                cih, wh = ci.cpu().numpy(), w.cpu().numpy().view(np.uint32)
            assert np.array_equal(d.cpu().numpy().view(np.uint32), oracle.sssp(rph, cih, wh, s)), s
            assert np.array_equal(lv.cpu().numpy(), oracle.bfs(rph, cih, s)), s


def test_cfg5_bfs_scale26_certificate(ctx):
    """cfg5, the bench's plan: 8 seeded sources' levels certified exactly."""
    g = inlgen.dev_build(26, 16, seed=inlgen.SEED_GRAPH, flags=inlgen.SYMMETRIC)
    rp, ci = g["row_ptr"], g["col_idx"]
    n = g["n_global"]
    A = inl.Csr(rp, ci, n)
    plan = inl.Plan(ctx, A)
    assert plan.info()["symmetric"] == 1
    srcs = inlgen.sources(rp.cpu().numpy(), 8)[:8]
    lv = torch.empty(n, dtype=torch.int32, device="cuda")
    reached = []
    for s in srcs:
        inl.bfs(ctx, A, s, lv, plan)
        certify_gpu(rp, ci, None, s, _levels_as_dist(lv))
        reached.append(int((lv >= 0).sum()))
    assert min(reached) > n // 4  # the giant component
    del plan, A, g, rp, ci, lv
    torch.cuda.empty_cache()


def test_cfg4_pagerank_against_20_iteration_oracle(ctx):
    """cfg4, the bench's plan: PR^20 element-wise vs the oracle's 20 fp64 iterations (reading
    R1), max relative error <= 1e-5; mass 1."""
    import oracle
    g = inlgen.dev_build(25, 16, seed=inlgen.SEED_GRAPH, flags=inlgen.TRANSPOSE)
    rp, ci, od = g["row_ptr"], g["col_idx"], g["out_degree"]
    n = g["n_global"]
    A = inl.Csr(rp, ci, n)
    plan = inl.Plan(ctx, A)
    r20 = torch.empty(n, device="cuda")
    inl.pagerank(ctx, A, od, r20, 0.85, 20, plan)
    p20 = r20.cpu().numpy().astype(np.float64)
    rph, cih, odh = rp.cpu().numpy(), ci.cpu().numpy(), od.cpu().numpy()
    del plan, A, g, rp, ci, od, r20
    torch.cuda.empty_cache()
    ref = oracle.pagerank(n, rph, cih, odh, 0.85, 20)
    assert abs(ref.sum() - 1.0) < 1e-9 and abs(p20.sum() - 1.0) < 1e-4
    err = np.abs(p20 - ref) / ref
    assert err.max() <= 1e-5, (int(err.argmax()), float(err.max()))
