"""GPU: the multi-GPU row-block product path under oracle parity on ONE device.

P row-block contexts join a loopback communicator (inl_comm_init_loopback, loopback.cu)
that stands in for NCCL behind the same exchange calls; each rank runs in its own host
thread on its own stream, exactly like the ranks of a torchrun job.  Every rank's CSR is
its block of inl_partition_rows (row_begin != 0 for every rank but 0), so the kernels'
row-block paths run: the local gather and its allgather (SpMV, PageRank's contribution
compaction over P blocks), SSSP's synchronous rounds with allreduce-min and
k_sssp_collect, BFS's allreduce-max byte map and k_bfs_apply.

Bars: BFS levels and SSSP distances bit-exact vs the oracle on every rank;
SpMV bit-exact for integer-valued data and <= 1e-5 relative for U[0,1) data; PageRank
<= 1e-5 vs orc_pagerank; replicated outputs identical on every rank.
"""
import threading

import numpy as np
import pytest
import torch

import inlgen
import oracle
from paper_conf_icpp_liwb15_b200 import inl

pytestmark = pytest.mark.gpu


def dev(a):
    return torch.from_numpy(np.ascontiguousarray(a)).cuda()


def block(rp, ci, lo, hi, extra=None):
    """Rows [lo, hi) of a host CSR as a local CSR (rebased row_ptr, global columns)."""
    s, e = int(rp[lo]), int(rp[hi])
    out = [rp[lo:hi + 1] - s, ci[s:e]]
    if extra is not None:
        out.append(extra[s:e])
    return out


def run_ranks(P, fn, timeout=900):
    """fn(rank, ctx) on P loopback ranks, one thread + stream each; returns the results."""
    grp = inl.LoopGroup(P)
    streams = [torch.cuda.Stream() for _ in range(P)]
    ctxs = []
    for r in range(P):
        with torch.cuda.stream(streams[r]):
            c = inl.Ctx(0)
            c.comm_init_loopback(grp, r)
            ctxs.append(c)
    torch.cuda.synchronize()
    res, errs = [None] * P, []

    def work(r):
        try:
            torch.cuda.set_device(0)
            with torch.cuda.stream(streams[r]):
                res[r] = fn(r, ctxs[r])
            streams[r].synchronize()
        except Exception as e:  # noqa: BLE001 — reported below
            errs.append((r, repr(e)))

    th = [threading.Thread(target=work, args=(r,)) for r in range(P)]
    for t in th:
        t.start()
    for t in th:
        t.join(timeout)
    assert not any(t.is_alive() for t in th), "a loopback rank hung"
    torch.cuda.synchronize()
    for c in ctxs:
        c.close()
    grp.close()
    return res, errs


PS = [2, 3, 8]


@pytest.fixture(scope="module")
def g12_dir():
    return inlgen.host_build(12, 16, seed=inlgen.SEED_GRAPH)


@pytest.fixture(scope="module")
def g12_sym():
    g = inlgen.host_build(12, 16, seed=inlgen.SEED_GRAPH, flags=inlgen.SYMMETRIC)
    return g, inlgen.weights_host(g.row_ptr, g.col_idx)


@pytest.fixture(scope="module")
def g18_sym():
    g = inlgen.host_build(18, 16, seed=inlgen.SEED_GRAPH, flags=inlgen.SYMMETRIC)
    return g, inlgen.weights_host(g.row_ptr, g.col_idx)


def _spmv_ranks(P, g, val, x, use_plan):
    n = g.n_global
    b = inl.partition_rows(n, P)

    def fn(r, ctx):
        rp, ci, v = block(g.row_ptr, g.col_idx, b[r], b[r + 1], val)
        A = inl.Csr(dev(rp), dev(ci), n, b[r])
        plan = inl.Plan(ctx, A) if use_plan else None
        xl, vl = dev(x), dev(v)
        y = torch.empty(A.n_rows, device="cuda")
        inl.spmv(ctx, A, vl, xl, y, plan)
        yg = torch.empty(n, device="cuda")
        inl.spmv_allgather(ctx, A, vl, xl, yg, plan)
        return y.cpu().numpy(), yg.cpu().numpy()
    res, errs = run_ranks(P, fn)
    assert not errs, errs
    return b, res


@pytest.mark.parametrize("P", PS)
@pytest.mark.parametrize("use_plan", [True, False])
def test_spmv_integer_bit_exact(g12_dir, P, use_plan):
    g = g12_dir
    val = inlgen.values_host(g.row_ptr, g.col_idx, mode=1)
    x = inlgen.vector_host(g.n_global, mode=1)
    ref = oracle.spmv(g.row_ptr, g.col_idx, val, x)
    b, res = _spmv_ranks(P, g, val, x, use_plan)
    for r, (y, yg) in enumerate(res):
        assert np.array_equal(y.astype(np.float64), ref[b[r]:b[r + 1]])
        assert np.array_equal(yg.astype(np.float64), ref)


@pytest.mark.parametrize("P", PS)
def test_spmv_float_within_1e5(P):
    g = inlgen.host_build(18, 16, seed=inlgen.SEED_GRAPH)
    val = inlgen.values_host(g.row_ptr, g.col_idx)
    x = inlgen.vector_host(g.n_global)
    ref = oracle.spmv(g.row_ptr, g.col_idx, val, x)
    _, res = _spmv_ranks(P, g, val, x, True)
    nz = ref != 0
    for _, yg in res:
        yy = yg.astype(np.float64)
        assert np.all(yy[~nz] == 0)
        assert np.max(np.abs(yy[nz] - ref[nz]) / ref[nz]) <= 1e-5
    assert all(np.array_equal(res[0][1], yg) for _, yg in res)  # replicated: identical bytes


@pytest.mark.parametrize("P", PS)
@pytest.mark.parametrize("scale", [12, 18])
@pytest.mark.parametrize("subblocks", [1, 4, 16])
def test_pagerank(P, scale, subblocks, monkeypatch):
    """subblocks = row sub-blocks per rank of the pipelined exchange (pagerank.cu): 1 = one
    allgather after the gather; 4 (default) and 16 (several empty sub-blocks at scale 12)
    overlap sub-block k's allgather, on the ctx's comm stream, with the later gathers."""
    monkeypatch.setenv("INL_PR_SUBBLOCKS", str(subblocks))
    g = inlgen.host_build(scale, 16, seed=inlgen.SEED_GRAPH, flags=inlgen.TRANSPOSE)
    n = g.n_global
    ref = oracle.pagerank(n, g.row_ptr, g.col_idx, g.out_degree, 0.85, 20)
    b = inl.partition_rows(n, P)

    def fn(r, ctx):
        rp, ci = block(g.row_ptr, g.col_idx, b[r], b[r + 1])
        A = inl.Csr(dev(rp), dev(ci), n, b[r])
        out = torch.empty(n, device="cuda")
        inl.pagerank(ctx, A, dev(g.out_degree), out, 0.85, 20, inl.Plan(ctx, A))
        return out.cpu().numpy()
    res, errs = run_ranks(P, fn)
    assert not errs, errs
    for pr in res:
        assert np.max(np.abs(pr.astype(np.float64) - ref) / ref) <= 1e-5
        assert np.array_equal(pr, res[0])


def _frontier_ranks(P, g, w, sources, use_plan=True):
    n = g.n_global
    b = inl.partition_rows(n, P)

    def fn(r, ctx):
        rp, ci, wl = block(g.row_ptr, g.col_idx, b[r], b[r + 1], w)
        A = inl.Csr(dev(rp), dev(ci), n, b[r])
        plan = inl.Plan(ctx, A) if use_plan else None
        wd = dev(wl.view(np.int32))
        out = []
        for s in sources:
            d = torch.empty(n, dtype=torch.int32, device="cuda")
            inl.sssp(ctx, A, wd, s, d, plan)
            lv = torch.empty(n, dtype=torch.int32, device="cuda")
            inl.bfs(ctx, A, s, lv, plan)
            out.append((d.cpu().numpy().view(np.uint32), lv.cpu().numpy()))
        return out
    res, errs = run_ranks(P, fn)
    assert not errs, errs
    return res


@pytest.mark.parametrize("P", PS)
@pytest.mark.parametrize("exchange", ["fused", "collective"])
def test_sssp_bfs_cfg1_bit_exact(g12_sym, P, exchange, monkeypatch):
    """exchange = fused: NEXT-1 (BFS bits set in the owners' bitmaps, SSSP improvements
    sent to the owners, peer memory; the default); collective: the r01 byte-map allreduce-max /
    dense allreduce-min over the whole vector."""
    if exchange == "collective":
        monkeypatch.setenv("INL_BFS_EXCHANGE", "bytemap")
        monkeypatch.setenv("INL_SSSP_EXCHANGE", "dense")
    g, w = g12_sym
    srcs = inlgen.sources(g.row_ptr, 8)
    res = _frontier_ranks(P, g, w, srcs)
    for i, s in enumerate(srcs):
        dref = oracle.sssp(g.row_ptr, g.col_idx, w, s)
        lref = oracle.bfs(g.row_ptr, g.col_idx, s)
        for r in range(P):
            assert np.array_equal(res[r][i][0], dref), (r, s)
            assert np.array_equal(res[r][i][1], lref), (r, s)


@pytest.mark.parametrize("P", PS)
def test_sssp_bfs_scale18_bit_exact(g18_sym, P):
    g, w = g18_sym
    srcs = inlgen.sources(g.row_ptr, 2)
    res = _frontier_ranks(P, g, w, srcs, use_plan=P != 3)  # P = 3: transient bins
    for i, s in enumerate(srcs):
        dref = oracle.sssp(g.row_ptr, g.col_idx, w, s)
        lref = oracle.bfs(g.row_ptr, g.col_idx, s)
        for r in range(P):
            assert np.array_equal(res[r][i][0], dref), (r, s)
            assert np.array_equal(res[r][i][1], lref), (r, s)


def test_failing_rank_releases_its_peers(g12_sym):
    """A rank whose call fails aborts the group: its peer fails too instead of hanging."""
    g, w = g12_sym
    n = g.n_global
    b = inl.partition_rows(n, 2)

    def fn(r, ctx):
        rp, ci, wl = block(g.row_ptr, g.col_idx, b[r], b[r + 1], w)
        A = inl.Csr(dev(rp), dev(ci), n, b[r])
        d = torch.empty(n, dtype=torch.int32, device="cuda")
        inl.sssp(ctx, A, dev(wl.view(np.int32)), n + 5 if r == 1 else 0, d)  # rank 1: bad source
    _, errs = run_ranks(2, fn, timeout=120)
    assert sorted(r for r, _ in errs) == [0, 1]
    assert any("INL_ERR_NCCL" in e for _, e in errs) and any("INVALID_ARGUMENT" in e for _, e in errs)


def test_row_block_checks(g12_dir):
    """A block that does not match inl_partition_rows for the rank is rejected."""
    g = g12_dir
    n = g.n_global
    b = inl.partition_rows(n, 2)

    def fn(r, ctx):
        lo, hi = (b[1], b[2]) if r == 0 else (b[0], b[1])  # swapped blocks
        rp, ci = block(g.row_ptr, g.col_idx, lo, hi)
        A = inl.Csr(dev(rp), dev(ci), n, lo)
        y = torch.empty(n, device="cuda")
        inl.spmv_allgather(ctx, A, dev(np.ones(A.nnz, np.float32)), dev(np.ones(n, np.float32)), y)
    _, errs = run_ranks(2, fn, timeout=120)
    assert len(errs) == 2 and all("INVALID_ARGUMENT" in e or "NCCL" in e for _, e in errs)


@pytest.mark.parametrize("P", [2, 8])
def test_exchange_volume_fused_vs_collective(g18_sym, P, monkeypatch):
    """NEXT-1's exchange volume against the r01 collectives, per rank and BFS / SSSP call
    (inl_stats.exchange_bytes): same results, and the record lands in the test log."""
    g, w = g18_sym
    s = inlgen.sources(g.row_ptr, 1)[0]
    n = g.n_global
    b = inl.partition_rows(n, P)
    vols = {}
    for mode in ("fused", "collective"):
        if mode == "collective":
            monkeypatch.setenv("INL_BFS_EXCHANGE", "bytemap")
            monkeypatch.setenv("INL_SSSP_EXCHANGE", "dense")

        def fn(r, ctx):
            rp, ci, wl = block(g.row_ptr, g.col_idx, b[r], b[r + 1], w)
            A = inl.Csr(dev(rp), dev(ci), n, b[r])
            d = torch.empty(n, dtype=torch.int32, device="cuda")
            st_s = inl.sssp(ctx, A, dev(wl.view(np.int32)), s, d)
            lv = torch.empty(n, dtype=torch.int32, device="cuda")
            st_b = inl.bfs(ctx, A, s, lv)
            return d.cpu().numpy(), lv.cpu().numpy(), st_s["exchange_bytes"], st_b["exchange_bytes"]
        res, errs = run_ranks(P, fn)
        assert not errs, errs
        vols[mode] = (max(r[2] for r in res), max(r[3] for r in res))
        assert np.array_equal(res[0][0].view(np.uint32), oracle.sssp(g.row_ptr, g.col_idx, w, s))
        assert np.array_equal(res[0][1], oracle.bfs(g.row_ptr, g.col_idx, s))
    print(f"\nexchange bytes per rank, scale 18, P={P}: SSSP fused {vols['fused'][0]} vs dense "
          f"{vols['collective'][0]}; BFS fused {vols['fused'][1]} vs byte map {vols['collective'][1]}")
    assert vols["fused"][0] > 0 and vols["fused"][1] > 0
