"""GPU: the row-block (multi-GPU) code path exercised on one GPU with a 1-rank NCCL
communicator — synchronous SSSP with allreduce-min, BFS with the allreduce-max
byte map, PageRank with the allgather of contributions — against the oracle."""
import numpy as np
import pytest
import torch

import inlgen
import oracle
from paper_conf_icpp_liwb15_b200 import inl

pytestmark = pytest.mark.gpu


def dev(a):
    return torch.from_numpy(np.ascontiguousarray(a)).cuda()


@pytest.fixture(scope="module")
def dctx():
    c = inl.Ctx(0)
    c.comm_init(1, 0)
    return c


def test_dist_sssp_bfs_match_oracle(dctx):
    g = inlgen.host_build(12, 16, seed=inlgen.SEED_GRAPH, flags=inlgen.SYMMETRIC)
    w = inlgen.weights_host(g.row_ptr, g.col_idx)
    A = inl.Csr(dev(g.row_ptr), dev(g.col_idx), g.n_global)
    for s in inlgen.sources(g.row_ptr, 4):
        d = torch.zeros(g.n_global, dtype=torch.int32, device="cuda")
        inl.sssp(dctx, A, dev(w.view(np.int32)), s, d)
        assert np.array_equal(d.cpu().numpy().view(np.uint32), oracle.sssp(g.row_ptr, g.col_idx, w, s))
        lv = torch.zeros(g.n_global, dtype=torch.int32, device="cuda")
        inl.bfs(dctx, A, s, lv)
        assert np.array_equal(lv.cpu().numpy(), oracle.bfs(g.row_ptr, g.col_idx, s))


def test_dist_pagerank_matches_oracle(dctx):
    g = inlgen.host_build(12, 16, seed=inlgen.SEED_GRAPH, flags=inlgen.TRANSPOSE)
    A = inl.Csr(dev(g.row_ptr), dev(g.col_idx), g.n_global)
    r = torch.empty(g.n_global, device="cuda")
    inl.pagerank(dctx, A, dev(g.out_degree), r, 0.85, 20, inl.Plan(dctx, A))
    ref = oracle.pagerank(g.n_global, g.row_ptr, g.col_idx, g.out_degree, 0.85, 20)
    rr = r.cpu().numpy().astype(np.float64)
    assert np.max(np.abs(rr - ref) / ref) <= 1e-5


def test_dist_spmv_allgather_and_exchange(dctx):
    """inl_spmv_allgather and the NEXT-1 exchange (CUDA IPC handle exchange over NCCL) on a
    1-rank communicator: same results as the oracle; no bytes cross ranks at P = 1."""
    g = inlgen.host_build(12, 16, seed=inlgen.SEED_GRAPH)
    val = inlgen.values_host(g.row_ptr, g.col_idx, mode=1)
    x = inlgen.vector_host(g.n_global, mode=1)
    A = inl.Csr(dev(g.row_ptr), dev(g.col_idx), g.n_global)
    y = torch.empty(g.n_global, device="cuda")
    inl.spmv_allgather(dctx, A, dev(val), dev(x), y)
    assert np.array_equal(y.cpu().numpy().astype(np.float64), oracle.spmv(g.row_ptr, g.col_idx, val, x))
    s = inlgen.host_build(12, 16, seed=inlgen.SEED_GRAPH, flags=inlgen.SYMMETRIC)
    w = inlgen.weights_host(s.row_ptr, s.col_idx)
    As = inl.Csr(dev(s.row_ptr), dev(s.col_idx), s.n_global)
    src = inlgen.sources(s.row_ptr, 1)[0]
    d = torch.zeros(s.n_global, dtype=torch.int32, device="cuda")
    st = inl.sssp(dctx, As, dev(w.view(np.int32)), src, d)
    assert np.array_equal(d.cpu().numpy().view(np.uint32), oracle.sssp(s.row_ptr, s.col_idx, w, src))
    lv = torch.zeros(s.n_global, dtype=torch.int32, device="cuda")
    sb = inl.bfs(dctx, As, src, lv)
    assert np.array_equal(lv.cpu().numpy(), oracle.bfs(s.row_ptr, s.col_idx, src))
    assert st["exchange_bytes"] == 0 and sb["exchange_bytes"] == 0
