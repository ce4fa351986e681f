"""Small end-to-end run of every op through the C-ABI (used under compute-sanitizer)."""
import os
import sys

import numpy as np
import torch

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
sys.path.insert(0, os.path.join(ROOT, "tests"))
import inlgen  # noqa: E402
from paper_conf_icpp_liwb15_b200 import inl  # noqa: E402


def dev(a):
    return torch.from_numpy(np.ascontiguousarray(a)).cuda()


def main():
    ctx = inl.Ctx(0)
    g = inlgen.host_build(10, 16, seed=1)
    A = inl.Csr(dev(g.row_ptr), dev(g.col_idx), g.n_global)
    y = torch.empty(A.n_rows, device="cuda")
    for b in (None, inl.bins(t_thread=2, t_warp=32, t_block=64, grid_chunk=48)):
        inl.spmv(ctx, A, dev(inlgen.values_host(g.row_ptr, g.col_idx)), dev(inlgen.vector_host(g.n_global)), y,
                 inl.Plan(ctx, A, b))
    inl.spmv(ctx, A, dev(inlgen.values_host(g.row_ptr, g.col_idx)), dev(inlgen.vector_host(g.n_global)), y)
    t = inlgen.host_build(10, 16, seed=1, flags=inlgen.TRANSPOSE)
    At = inl.Csr(dev(t.row_ptr), dev(t.col_idx), t.n_global)
    r = torch.empty(t.n_global, device="cuda")
    inl.pagerank(ctx, At, dev(t.out_degree), r, 0.85, 5, inl.Plan(ctx, At))
    s = inlgen.host_build(12, 16, seed=1, flags=inlgen.SYMMETRIC)
    As = inl.Csr(dev(s.row_ptr), dev(s.col_idx), s.n_global)
    w = dev(inlgen.weights_host(s.row_ptr, s.col_idx).view(np.int32))
    d = torch.empty(s.n_global, dtype=torch.int32, device="cuda")
    src = inlgen.sources(s.row_ptr, 1)[0]
    inl.sssp(ctx, As, w, src, d)
    inl.bfs(ctx, As, src, d)
    ps = inl.Plan(ctx, As)  # symmetric plan: BFS bottom-up steps, BC pull steps
    inl.bfs(ctx, As, src, d, ps)
    inl.sssp(ctx, As, w, src, d, inl.Plan(ctx, As, inl.bins(flags=inl.BINS_SSSP_DEVLOOP)))
    for fl in (inl.BINS_TPL_DBUF_SHARED, inl.BINS_TPL_DBUF_GLOBAL, inl.BINS_TPL_DUAL_QUEUE, inl.BINS_THREAD_ONLY):
        pt = inl.Plan(ctx, As, inl.bins(t_thread=16, t_warp=16, t_block=16, flags=fl))
        inl.sssp(ctx, As, w, src, d, pt)
        inl.bfs(ctx, As, src, d, pt)
    bc = torch.empty(s.n_global, dtype=torch.float64, device="cuda")
    srcs = inlgen.sources(s.row_ptr, 3)
    os.environ["INL_BC_MODE"] = "level"
    inl.bc(ctx, As, srcs, bc)
    inl.bc(ctx, As, srcs, bc, ps)  # pull steps
    os.environ["INL_BC_MODE"] = "src"
    inl.bc(ctx, As, srcs, bc)  # source-parallel, state in shared memory
    s14 = inlgen.host_build(14, 8, seed=1, flags=inlgen.SYMMETRIC)
    A14 = inl.Csr(dev(s14.row_ptr), dev(s14.col_idx), s14.n_global)
    b14 = torch.empty(s14.n_global, dtype=torch.float64, device="cuda")
    inl.bc(ctx, A14, inlgen.sources(s14.row_ptr, 3), b14)  # source-parallel, global state
    del os.environ["INL_BC_MODE"]
    for fl in (inl.BINS_TPL_DBUF_SHARED, inl.BINS_TPL_DBUF_GLOBAL, inl.BINS_TPL_DUAL_QUEUE, inl.BINS_THREAD_ONLY):
        inl.bc(ctx, As, srcs, bc, inl.Plan(ctx, As, inl.bins(t_thread=16, cta_threads=128, flags=fl)))
    # the paper's templates and the column-blocked bin (small blocks: several per row)
    val, x = dev(inlgen.values_host(g.row_ptr, g.col_idx)), dev(inlgen.vector_host(g.n_global))
    for fl in (inl.BINS_TPL_DUAL_QUEUE, inl.BINS_TPL_DBUF_GLOBAL, inl.BINS_TPL_DBUF_SHARED):
        inl.spmv(ctx, A, val, x, y, inl.Plan(ctx, A, inl.bins(t_thread=16, t_warp=16, t_block=16, cta_threads=64,
                                                               flags=fl)))
    os.environ["INL_CB_K"] = "128"
    os.environ["INL_CB_MULT"] = "1"
    inl.spmv(ctx, A, val, x, y, inl.Plan(ctx, A, inl.bins(t_warp=16, flags=inl.BINS_COLBLOCK)))
    inl.pagerank(ctx, At, dev(t.out_degree), r, 0.85, 3, inl.Plan(ctx, At, inl.bins(t_warp=16, flags=inl.BINS_COLBLOCK)))
    # grid-bin buffer at its worst case: every vertex just above t_warp, fresh ctx, no plan;
    # and dbuf-global with lbTHRES = 32 and the default t_block
    from graphs import csr_np
    rng = np.random.default_rng(3)
    nb = 2400
    brp, bci = csr_np(nb, np.repeat(np.arange(nb), 560), rng.integers(0, nb, nb * 560))
    Ab = inl.Csr(dev(brp), dev(bci), nb)
    wb = dev(inlgen.weights_host(brp, bci).view(np.int32))
    db = torch.empty(nb, dtype=torch.int32, device="cuda")
    c2 = inl.Ctx(0)
    inl.bfs(c2, Ab, 0, db)
    inl.sssp(c2, Ab, wb, 0, db)
    pg = inl.Plan(c2, Ab, inl.bins(t_thread=32, flags=inl.BINS_TPL_DBUF_GLOBAL))
    inl.bfs(c2, Ab, 0, db, pg)
    inl.sssp(c2, Ab, wb, 0, db, pg)
    torch.cuda.synchronize()
    print("sanitize driver ok")


if __name__ == "__main__":
    main()
