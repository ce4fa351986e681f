"""Parity at BASELINE.json's full sizes, in the launch configuration bench.py times (plans,
default bins), where the oracle cannot run whole: exact certificates and one-step checks.

* SSSP / BFS, cfg3 graph (R-MAT scale 23, symmetric, w in 1..255): the O(m) shortest-path
  certificate of tests/graphs.py (feasible edges + a tight in-edge for every finite vertex
  => dist equals the true distances, for weights >= 1), evaluated with torch on the GPU
  (test-side arithmetic only, on the library's outputs).
* PageRank, cfg4 graph (R-MAT scale 25 in-CSR, 20 iterations): PR^20 from the library must
  equal one oracle-style step (reading R1, fp64) applied to the library's own PR^19 at
  sampled pages (the highest in-degree pages + random ones), and the mass must be 1.
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


def certify_gpu(rp, ci, w, s, dist):
    """Exact certificate for dist (int64 tensor, INF = unreachable) from source s."""
    n = rp.numel() - 1
    deg = (rp[1:] - rp[:-1])
    src = torch.repeat_interleave(torch.arange(n, device=rp.device, dtype=torch.int32), deg)
    du = dist[src.long()]
    dv = dist[ci.long()]
    fin = du != INF
    ww = w.long()
    assert int(dist[s]) == 0
    assert not bool(((dv > du + ww) & fin).any()), "infeasible edge"
    tight = fin & (dv == du + ww)
    has = torch.zeros(n, dtype=torch.bool, device=rp.device)
    has[ci.long()[tight]] = True
    need = dist != INF
    need[s] = False
    assert not bool((need & ~has).any()), "finite vertex without a tight in-edge"
    del src, du, dv, fin, tight


def test_cfg3_sssp_bfs_certificate(ctx):
    g = inlgen.dev_build(23, 16, seed=inlgen.SEED_GRAPH, flags=inlgen.SYMMETRIC)
    rp, ci = g["row_ptr"], g["col_idx"]
    w = inlgen.weights_dev(rp, ci)
    A = inl.Csr(rp, ci, g["n_global"])
    plan = inl.Plan(ctx, A)
    assert plan.info()["symmetric"] == 1  # BFS runs direction-optimizing, as in the bench
    s = inlgen.sources(rp.cpu().numpy(), 1)[0]
    d = torch.empty(g["n_global"], dtype=torch.int32, device="cuda")
    inl.sssp(ctx, A, w, s, d, plan)
    dist = d.view(torch.int32).long() & 0xFFFFFFFF
    certify_gpu(rp, ci, w.view(torch.int32).long() & 0xFFFFFFFF, s, dist)
    lv = torch.empty(g["n_global"], dtype=torch.int32, device="cuda")
    inl.bfs(ctx, A, s, lv, plan)
    lvl = torch.where(lv < 0, torch.full_like(lv, -1), lv).long()
    lvl = torch.where(lvl < 0, torch.full_like(lvl, INF), lvl)
    certify_gpu(rp, ci, torch.ones_like(ci), s, lvl)
    assert int((lv >= 0).sum()) == int((d != -1).sum())  # same reached set


def test_cfg4_pagerank_one_step_and_mass(ctx):
    g = inlgen.dev_build(25, 16, seed=inlgen.SEED_GRAPH, flags=inlgen.TRANSPOSE)
    rp, ci, od = g["row_ptr"], g["col_idx"], g["out_degree"]
    n = g["n_global"]
    A = inl.Csr(rp, ci, n)
    plan = inl.Plan(ctx, A)
    r19 = torch.empty(n, device="cuda")
    r20 = torch.empty(n, device="cuda")
    inl.pagerank(ctx, A, od, r19, 0.85, 19, plan)
    inl.pagerank(ctx, A, od, r20, 0.85, 20, plan)
    torch.cuda.synchronize()
    p19 = r19.cpu().numpy().astype(np.float64)
    p20 = r20.cpu().numpy().astype(np.float64)
    odh = od.cpu().numpy()
    assert abs(p20.sum() - 1.0) < 1e-4
    d = 0.85
    D = p19[odh == 0].sum()
    indeg = (rp[1:] - rp[:-1]).cpu().numpy()
    rng = np.random.default_rng(5)
    sample = np.unique(np.concatenate([np.argsort(-indeg)[:200], rng.integers(0, n, 1800)]))
    rph = rp.cpu().numpy()
    for v in sample:
        cols = ci[int(rph[v]):int(rph[v + 1])].cpu().numpy()
        s = float(np.sum(p19[cols] / odh[cols])) if cols.size else 0.0
        ref = (1 - d) / n + d * (s + D / n)
        assert abs(p20[v] - ref) / ref <= 1e-5, (int(v), p20[v], ref)
