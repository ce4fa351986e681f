"""GPU parity: inl_sssp / inl_bfs (CUDA through the C-ABI) vs oracle Dijkstra / queue BFS.

Bar: bit-exact distances and levels (unique answers), every source; larger graphs
add the exact O(m) certificate (tests/graphs.py) for every source."""
import numpy as np
import pytest
import torch

import inlgen
import oracle
from graphs import certify_bfs, certify_sssp, csr_from_edges
from paper_conf_icpp_liwb15_b200 import inl

pytestmark = pytest.mark.gpu


def dev(a):
    return torch.from_numpy(np.ascontiguousarray(a)).cuda()


@pytest.fixture(scope="module")
def ctx():
    return inl.Ctx(0)


@pytest.fixture(scope="module")
def cfg1():
    g = inlgen.host_build(12, 16, seed=inlgen.SEED_GRAPH, flags=inlgen.SYMMETRIC)
    w = inlgen.weights_host(g.row_ptr, g.col_idx)
    return g, w


def gpu_sssp(ctx, rp, ci, w, n, s, b=None):
    A = inl.Csr(dev(rp), dev(ci), n)
    d = torch.zeros(n, dtype=torch.int32, device="cuda")
    plan = inl.Plan(ctx, A, b) if b is not None else None
    st = inl.sssp(ctx, A, dev(w.view(np.int32)), s, d, plan)
    return d.cpu().numpy().view(np.uint32), st


def gpu_bfs(ctx, rp, ci, n, s, b=None):
    A = inl.Csr(dev(rp), dev(ci), n)
    lv = torch.zeros(n, dtype=torch.int32, device="cuda")
    plan = inl.Plan(ctx, A, b) if b is not None else None
    st = inl.bfs(ctx, A, s, lv, plan)
    return lv.cpu().numpy(), st


BINS = [None, dict(t_thread=-1, t_warp=32, t_block=128, grid_chunk=64),
        dict(t_thread=1, t_warp=128, t_block=256, grid_chunk=64), dict(flags=inl.BINS_THREAD_ONLY),
        dict(t_thread=64, t_warp=128, t_block=4096, grid_chunk=1000),
        dict(flags=inl.BINS_SSSP_DEVLOOP),  # device-driven near-far step loop
        dict(t_thread=1, t_warp=32, t_block=128, grid_chunk=64, flags=inl.BINS_SSSP_DEVLOOP)]


@pytest.mark.parametrize("loop", ["graph", "host"])
@pytest.mark.parametrize("bi", range(len(BINS)))
def test_cfg1_all_sources_bit_exact(ctx, cfg1, bi, loop, monkeypatch):
    monkeypatch.setenv("INL_SSSP_LOOP", loop)
    g, w = cfg1
    b = inl.bins(**BINS[bi]) if BINS[bi] is not None else None
    for s in inlgen.sources(g.row_ptr, 8):
        d, st = gpu_sssp(ctx, g.row_ptr, g.col_idx, w, g.n_global, s, b)
        assert np.array_equal(d, oracle.sssp(g.row_ptr, g.col_idx, w, s))
        assert st["iterations"] >= 1
        lv, st = gpu_bfs(ctx, g.row_ptr, g.col_idx, g.n_global, s, b)
        assert np.array_equal(lv, oracle.bfs(g.row_ptr, g.col_idx, s))


def test_small_graph_edge_cases(ctx):
    rp, ci, w = csr_from_edges(6, [(1, 2), (2, 3), (3, 1)], [5, 6, 7], symmetric=True)
    d, _ = gpu_sssp(ctx, rp, ci, w, 6, 0)  # isolated source
    assert d.tolist() == [0] + [0xFFFFFFFF] * 5
    lv, _ = gpu_bfs(ctx, rp, ci, 6, 1)
    assert lv.tolist() == [-1, 0, 1, 1, -1, -1]
    rp = np.zeros(2, np.int64)
    d, _ = gpu_sssp(ctx, rp, np.zeros(0, np.int32), np.zeros(0, np.uint32), 1, 0)
    assert d.tolist() == [0]
    # a star whose hub has degree far above every threshold (grid bin), path tail
    n = 30000
    e = [(0, i) for i in range(1, n - 100)] + [(i, i + 1) for i in range(n - 101, n - 1)]
    rp, ci, w = csr_from_edges(n, e, np.arange(len(e)) % 255 + 1, symmetric=True)
    for s in (0, n - 1, 5):
        d, _ = gpu_sssp(ctx, rp, ci, w, n, s)
        assert np.array_equal(d, oracle.sssp(rp, ci, w, s))
        lv, _ = gpu_bfs(ctx, rp, ci, n, s)
        assert np.array_equal(lv, oracle.bfs(rp, ci, s))


@pytest.mark.parametrize("loop", ["graph", "graph-list", "graph-trace", "dyn", "dyn-bits"])
def test_devloop_edge_cases_and_certificate(ctx, loop, monkeypatch, tmp_path):
    """The device-driven near-far loop: one CUDA-graph launch per source (default: bitmap
    frontier; graph-list: the queue-counter worklists, INL_SSSP_FRONTIER=list; graph-trace: with
    the per-step %globaltimer trace and improvement counter) or stream launches with host polling
    (INL_SSSP_LOOP=dyn; dyn-bits: the graph loop's bitmap step kernels), vs the host-driven loop."""
    trace = None
    if loop == "graph-list":
        monkeypatch.setenv("INL_SSSP_FRONTIER", "list")
        loop = "graph"
    elif loop == "graph-trace":
        trace = tmp_path / "trace.txt"
        monkeypatch.setenv("INL_SSSP_TRACE", str(trace))
        monkeypatch.setenv("INL_SSSP_TRACE_MARKS", "1")
        loop = "graph"
    elif loop == "dyn-bits":
        monkeypatch.setenv("INL_SSSP_DYN_BITS", "1")
        loop = "dyn"
    monkeypatch.setenv("INL_SSSP_LOOP", loop)
    b = inl.bins(flags=inl.BINS_SSSP_DEVLOOP)
    rp, ci, w = csr_from_edges(6, [(1, 2), (2, 3), (3, 1)], [5, 6, 7], symmetric=True)
    d, st = gpu_sssp(ctx, rp, ci, w, 6, 0, b)  # isolated source
    assert d.tolist() == [0] + [0xFFFFFFFF] * 5 and st["host_syncs"] >= 1
    n = 30000
    e = [(0, i) for i in range(1, n - 100)] + [(i, i + 1) for i in range(n - 101, n - 1)]
    rp, ci, w = csr_from_edges(n, e, np.arange(len(e)) % 255 + 1, symmetric=True)
    for s in (0, n - 1, 5):
        d, _ = gpu_sssp(ctx, rp, ci, w, n, s, b)
        assert np.array_equal(d, oracle.sssp(rp, ci, w, s))
    g = inlgen.host_build(16, 16, seed=inlgen.SEED_GRAPH, flags=inlgen.SYMMETRIC)
    w = inlgen.weights_host(g.row_ptr, g.col_idx)
    for s in inlgen.sources(g.row_ptr, 3):
        d, st = gpu_sssp(ctx, g.row_ptr, g.col_idx, w, g.n_global, s, b)
        assert certify_sssp(g.row_ptr, g.col_idx, w, s, d) is None
        monkeypatch.setenv("INL_SSSP_LOOP", "host")
        ref, st0 = gpu_sssp(ctx, g.row_ptr, g.col_idx, w, g.n_global, s, inl.bins())
        monkeypatch.setenv("INL_SSSP_LOOP", loop)
        assert np.array_equal(d, ref)
        assert st["launches"] > 0 and st["host_syncs"] < st0["host_syncs"]
        if loop == "graph":
            assert st["host_syncs"] == 1
    if trace is not None:  # one block per call; per step: 6 stamps, nF, nsplit, relaxed / marked counters, pieces
        rows = [list(map(int, l.split())) for l in trace.read_text().splitlines() if not l.startswith("#")]
        assert rows and all(len(r) == 14 for r in rows)
        last = [r for r in rows if r[1] and r[5]]
        assert all(r[2] >= r[1] and r[5] >= r[4] for r in last)  # stamps in kernel order
        assert max(r[11] for r in rows) > 0 and max(r[12] for r in rows) > 0  # relaxed, improved


def test_host_buffers(ctx, cfg1):
    g, w = cfg1
    s = inlgen.sources(g.row_ptr, 1)[0]
    d = np.zeros(g.n_global, np.uint32)
    inl.sssp(ctx, inl.Csr(g.row_ptr, g.col_idx, g.n_global), w, s, d)
    assert np.array_equal(d, oracle.sssp(g.row_ptr, g.col_idx, w, s))
    lv = np.zeros(g.n_global, np.int32)
    inl.bfs(ctx, inl.Csr(g.row_ptr, g.col_idx, g.n_global), s, lv)
    assert np.array_equal(lv, oracle.bfs(g.row_ptr, g.col_idx, s))


def test_scale18_certificate_all_sources(ctx):
    g = inlgen.dev_build(18, 16, seed=inlgen.SEED_GRAPH, flags=inlgen.SYMMETRIC)
    rp, ci = g["row_ptr"], g["col_idx"]
    w = inlgen.weights_dev(rp, ci)
    A = inl.Csr(rp, ci, g["n_global"])
    plan = inl.Plan(ctx, A)
    rph, cih, wh = rp.cpu().numpy(), ci.cpu().numpy(), w.cpu().numpy().view(np.uint32)
    srcs = inlgen.sources(rph, 8)
    for i, s in enumerate(srcs):
        d = torch.zeros(g["n_global"], dtype=torch.int32, device="cuda")
        inl.sssp(ctx, A, w, s, d, plan)
        dh = d.cpu().numpy().view(np.uint32)
        assert certify_sssp(rph, cih, wh, s, dh) is None
        lv = torch.zeros(g["n_global"], dtype=torch.int32, device="cuda")
        inl.bfs(ctx, A, s, lv, plan)
        lvh = lv.cpu().numpy()
        assert certify_bfs(rph, cih, s, lvh) is None
        if i < 2:
            assert np.array_equal(dh, oracle.sssp(rph, cih, wh, s))
            assert np.array_equal(lvh, oracle.bfs(rph, cih, s))


def test_directed_graph_with_plan(ctx):
    """Bottom-up BFS steps need rows to list predecessors: the plan enables them only for a
    symmetric CSR; a directed R-MAT through a plan must still match the oracle."""
    g = inlgen.host_build(14, 16, seed=inlgen.SEED_GRAPH)  # directed
    A = inl.Csr(dev(g.row_ptr), dev(g.col_idx), g.n_global)
    plan = inl.Plan(ctx, A)
    assert plan.info()["symmetric"] == 0
    for s in inlgen.sources(g.row_ptr, 4):
        lv = torch.zeros(g.n_global, dtype=torch.int32, device="cuda")
        inl.bfs(ctx, A, s, lv, plan)
        assert np.array_equal(lv.cpu().numpy(), oracle.bfs(g.row_ptr, g.col_idx, s))
    gs = inlgen.host_build(14, 16, seed=inlgen.SEED_GRAPH, flags=inlgen.SYMMETRIC)
    assert inl.Plan(ctx, inl.Csr(dev(gs.row_ptr), dev(gs.col_idx), gs.n_global)).info()["symmetric"] == 1


# ---- adversarial shapes for the grid-bin (dbuf-global) buffer (ADVICE high) ----
def _dense_band_graph(n=20000, picks=700, seed=11):
    """Every vertex of degree ~1025..2048: each one just above t_warp = 1024, so a frontier of
    them emits one grid piece per ~1.1K edges (the worst case of the capacity bound)."""
    from graphs import csr_np
    rng = np.random.default_rng(seed)
    u = np.repeat(np.arange(n), picks)
    v = rng.integers(0, n, n * picks)
    return csr_np(n, u, v)


def test_grid_buffer_dense_band_fresh_ctx_no_plan():
    from graphs import pair_weights
    rp, ci = _dense_band_graph()
    deg = np.diff(rp)
    assert np.mean((deg > 1024) & (deg <= 2048)) > 0.95
    w = pair_weights(rp, ci)
    c = inl.Ctx(0)  # fresh ctx: nothing pre-grown by an earlier plan
    for s in (0, 17, 19999):
        d, _ = gpu_sssp(c, rp, ci, w, len(rp) - 1, s)
        assert np.array_equal(d, oracle.sssp(rp, ci, w, s))
        lv, _ = gpu_bfs(c, rp, ci, len(rp) - 1, s)
        assert np.array_equal(lv, oracle.bfs(rp, ci, s))


def test_grid_buffer_complete_bipartite_no_plan():
    from graphs import csr_np, pair_weights
    k = 1100
    a = np.repeat(np.arange(k), k)
    b = np.tile(np.arange(k, 2 * k), k)
    rp, ci = csr_np(2 * k, a, b)
    w = pair_weights(rp, ci)
    c = inl.Ctx(0)
    for s in (0, k, 2 * k - 1):
        lv, _ = gpu_bfs(c, rp, ci, 2 * k, s)
        assert np.array_equal(lv, oracle.bfs(rp, ci, s))
        d, _ = gpu_sssp(c, rp, ci, w, 2 * k, s)
        assert np.array_equal(d, oracle.sssp(rp, ci, w, s))


@pytest.mark.parametrize("lbt", [8, 32])
def test_dbuf_global_template_default_t_block(ctx, lbt):
    """INL_BINS_TPL_DBUF_GLOBAL with lbTHRES = t_thread and the DEFAULT t_block: every vertex
    above lbTHRES goes to the global buffer (inl.h documents this path)."""
    g = inlgen.host_build(16, 16, seed=inlgen.SEED_GRAPH, flags=inlgen.SYMMETRIC)
    w = inlgen.weights_host(g.row_ptr, g.col_idx)
    b = inl.bins(t_thread=lbt, flags=inl.BINS_TPL_DBUF_GLOBAL)
    for s in inlgen.sources(g.row_ptr, 3):
        d, _ = gpu_sssp(ctx, g.row_ptr, g.col_idx, w, g.n_global, s, b)
        assert np.array_equal(d, oracle.sssp(g.row_ptr, g.col_idx, w, s))
        lv, _ = gpu_bfs(ctx, g.row_ptr, g.col_idx, g.n_global, s, b)
        assert np.array_equal(lv, oracle.bfs(g.row_ptr, g.col_idx, s))
    rp, ci = _dense_band_graph(n=4000, picks=600)
    wb = inlgen.weights_host(rp, ci)
    d, _ = gpu_sssp(ctx, rp, ci, wb, len(rp) - 1, 0, b)
    assert np.array_equal(d, oracle.sssp(rp, ci, wb, 0))


def test_bfs_bottom_up_entered_twice(ctx):
    """Two dense clusters joined by a long path: BFS goes bottom-up in the first cluster,
    top-down along the path, and bottom-up again in the second — the second entry starts from
    the plan's static degree bins, most of whose vertices (the first cluster) are visited and
    must be skipped.  Levels bit-exact against the oracle, with the direction switches taken."""
    rng = np.random.default_rng(7)
    na, npath = 6000, 120
    n = 2 * na + npath
    e = set()
    for base in (0, na + npath):  # two clusters: random graph, mean degree ~24, plus a few hubs
        for _ in range(na * 12):
            u, v = rng.integers(0, na, 2)
            if u != v:
                e.add((base + int(min(u, v)), base + int(max(u, v))))
        for h in range(8):
            for v in rng.choice(na, 400, replace=False):
                if int(v) != h:
                    e.add((base + min(h, int(v)), base + max(h, int(v))))
    chain = [na - 1] + list(range(na, na + npath)) + [na + npath]
    e.update((a, b) for a, b in zip(chain[:-1], chain[1:]))
    rp, ci, _ = csr_from_edges(n, sorted(e), symmetric=True)
    for s in (0, 17, n - 1):
        lv, st = gpu_bfs(ctx, rp, ci, n, s, inl.bins())
        assert np.array_equal(lv, oracle.bfs(rp, ci, s))
        assert st["iterations"] > npath
