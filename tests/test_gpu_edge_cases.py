"""GPU: degenerate inputs through the C-ABI (SURVEY §8b conventions: n_global == 0 and nnz == 0
are valid no-ops; bad arguments are INL_ERR_INVALID_ARGUMENT, never a crash)."""
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
def ctx():
    return inl.Ctx(0)


def test_empty_matrix(ctx):
    rp = np.zeros(1, np.int64)
    A = inl.Csr(dev(rp), torch.zeros(0, dtype=torch.int32, device="cuda"), 0)
    e = torch.zeros(0, device="cuda")
    inl.spmv(ctx, A, e, e, e)
    inl.spmv_allgather(ctx, A, e, e, e)
    inl.pagerank(ctx, A, torch.zeros(0, dtype=torch.int32, device="cuda"), e, 0.85, 20)
    out = torch.zeros(0, dtype=torch.int64, device="cuda")
    for m in (inl.TREE_FLAT, inl.TREE_LEVELS):
        inl.tree_descendants(ctx, A, torch.zeros(0, dtype=torch.int32, device="cuda"), out, 0, m)
    with pytest.raises(inl.InlError):  # source out of range
        inl.bfs(ctx, A, 0, torch.zeros(0, dtype=torch.int32, device="cuda"))


def test_edgeless_graph(ctx):
    n = 1000
    rp = np.zeros(n + 1, np.int64)
    A = inl.Csr(dev(rp), torch.zeros(0, dtype=torch.int32, device="cuda"), n)
    y = torch.full((n,), 7.0, device="cuda")
    inl.spmv(ctx, A, torch.zeros(0, device="cuda"), torch.ones(n, device="cuda"), y, inl.Plan(ctx, A))
    assert float(y.abs().max()) == 0.0
    r = torch.empty(n, device="cuda")
    inl.pagerank(ctx, A, torch.zeros(n, dtype=torch.int32, device="cuda"), r, 0.85, 20)
    assert np.allclose(r.cpu().numpy(), 1.0 / n, rtol=1e-6)  # all dangling: uniform
    d = torch.empty(n, dtype=torch.int32, device="cuda")
    inl.sssp(ctx, A, torch.zeros(0, dtype=torch.int32, device="cuda"), 17, d)
    dh = d.cpu().numpy().view(np.uint32)
    assert dh[17] == 0 and np.all(np.delete(dh, 17) == 0xFFFFFFFF)
    lv = torch.empty(n, dtype=torch.int32, device="cuda")
    inl.bfs(ctx, A, 999, lv)
    assert lv[999].item() == 0 and int((lv >= 0).sum()) == 1


def test_bad_arguments_are_errors_not_crashes(ctx):
    g = inlgen.host_build(8, 8, seed=inlgen.SEED_GRAPH)
    A = inl.Csr(dev(g.row_ptr), dev(g.col_idx), g.n_global)
    y = torch.empty(A.n_rows, device="cuda")
    with pytest.raises(inl.InlError):
        inl.spmv(ctx, A, None, torch.ones(g.n_global, device="cuda"), y)  # val NULL
    with pytest.raises(inl.InlError):
        inl.pagerank(ctx, A, dev(np.ones(g.n_global, np.int32)), y, 1.5, 3)  # damping out of range
    with pytest.raises(inl.InlError):
        inl.Plan(ctx, A, inl.bins(t_warp=8))  # t_warp below 16
    with pytest.raises(inl.InlError):
        inl.spmv_allgather(ctx, inl.Csr(dev(g.row_ptr[:11] - g.row_ptr[0]), dev(g.col_idx[:int(g.row_ptr[10])]),
                                        g.n_global, 5), torch.ones(int(g.row_ptr[10]), device="cuda"),
                           torch.ones(g.n_global, device="cuda"), torch.empty(g.n_global, device="cuda"))
    # the ctx stays usable after errors
    inl.spmv(ctx, A, dev(inlgen.values_host(g.row_ptr, g.col_idx)), dev(inlgen.vector_host(g.n_global)), y)
    ref = oracle.spmv(g.row_ptr, g.col_idx, inlgen.values_host(g.row_ptr, g.col_idx), inlgen.vector_host(g.n_global))
    nz = ref != 0
    yy = y.cpu().numpy().astype(np.float64)
    assert np.max(np.abs(yy[nz] - ref[nz]) / ref[nz]) <= 1e-5
