"""world_size-2 CPU tests (gloo) of the multi-GPU row-block path.

The product's N > 1 path itself (libinl's row-block kernels and its exchange, NCCL or the
one-device loopback communicator) runs under oracle parity in tests/test_gpu_loopback.py
(P = 2, 3, 8 on one B200).  What can run here, without a GPU, is its host side — the NCCL unique-id bootstrap through libinl and
torch.distributed, the row-block partition (inl_partition_rows) and per-rank CSR
slices (inlgen row ranges) — and step-by-step models of the three exchange
protocols, with gloo standing in for NCCL, checked against the single-process
oracle:
  * PageRank: allgather of the contribution slice + the rank's dangling partial,
    summed in rank order (pagerank.cu);
  * SSSP: synchronous relaxation of the owned rows, allreduce-min over dist with a
    trailing "no change" word, next frontier = owned vertices whose distance dropped
    (frontier.cu sssp_run);
  * BFS: allreduce-max over an n-byte next map with a trailing flag byte, new levels
    applied on every rank, owned new vertices form the next frontier (bfs_run).
"""
import os
import socket

import numpy as np
import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp

import inlgen
import oracle

WORLD = 2


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _run(fn, *args):
    port = _free_port()
    ctx = mp.get_context("spawn")
    q = ctx.SimpleQueue()
    procs = [ctx.Process(target=_worker, args=(r, port, fn, args, q)) for r in range(WORLD)]
    for p in procs:
        p.start()
    for p in procs:
        p.join(120)
    res = [q.get() for _ in range(WORLD)]
    for p in procs:
        assert p.exitcode == 0, f"rank exited with {p.exitcode}"
    errs = [r for r in res if r != "ok"]
    assert not errs, errs


def _worker(rank, port, fn, args, q):
    import sys
    root = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
    sys.path.insert(0, root)
    sys.path.insert(0, os.path.join(root, "tests"))
    try:
        dist.init_process_group("gloo", init_method=f"tcp://127.0.0.1:{port}", rank=rank, world_size=WORLD)
        globals()[fn](rank, *args)
        dist.barrier()
        dist.destroy_process_group()
        q.put("ok")
    except Exception as e:  # report instead of hanging the peer
        import traceback
        q.put(f"rank {rank}: {e!r}\n{traceback.format_exc()}")


# ---------------------------------------------------------------------------------------
def _uid(rank):
    from paper_conf_icpp_liwb15_b200 import inl
    uid = inl.broadcast_unique_id(rank)
    t = torch.from_numpy(uid.astype(np.int64))
    g = [torch.zeros_like(t) for _ in range(WORLD)]
    dist.all_gather(g, t)
    assert all(torch.equal(g[0], x) for x in g) and int(g[0].abs().sum()) > 0


def test_nccl_unique_id_bootstrap():
    _run("_uid")


def _slices(rank, scale):
    from paper_conf_icpp_liwb15_b200 import inl
    n = 1 << scale
    b = inl.partition_rows(n, WORLD)
    full = inlgen.host_build(scale, 16, seed=1, flags=inlgen.SYMMETRIC)
    part = inlgen.host_build(scale, 16, seed=1, flags=inlgen.SYMMETRIC, row_begin=b[rank], row_end=b[rank + 1])
    lo, hi = full.row_ptr[b[rank]], full.row_ptr[b[rank + 1]]
    assert np.array_equal(part.row_ptr, full.row_ptr[b[rank]:b[rank + 1] + 1] - lo)
    assert np.array_equal(part.col_idx, full.col_idx[lo:hi])
    nnz = torch.tensor([part.nnz], dtype=torch.int64)
    dist.all_reduce(nnz)
    assert int(nnz) == full.nnz


def test_row_blocks_cover_the_graph():
    _run("_slices", 10)


# ---------------------------------------------------------------------------------------
def _pagerank(rank, scale, iters):
    from paper_conf_icpp_liwb15_b200 import inl
    g = inlgen.host_build(scale, 16, seed=1, flags=inlgen.TRANSPOSE)
    n = g.n_global
    b = inl.partition_rows(n, WORLD)
    B = b[1] - b[0]
    r0, r1 = b[rank], b[rank + 1]
    od = g.out_degree.astype(np.float64)
    rp, ci = g.row_ptr, g.col_idx
    d = 0.85
    pr0 = 1.0 / n
    c = np.where(od > 0, pr0 / np.maximum(od, 1), 0.0)  # replicated contributions
    D = float((od == 0).sum()) * pr0
    rank_vec = None
    for t in range(iters):
        base = (1 - d) / n + d * D / n
        s = np.array([c[ci[rp[v]:rp[v + 1]]].sum() for v in range(r0, r1)])
        pr = base + d * s
        cl = np.zeros(B)
        cl[:r1 - r0] = np.where(od[r0:r1] > 0, pr / np.maximum(od[r0:r1], 1), 0.0)
        dl = float(pr[od[r0:r1] == 0].sum())
        parts = [torch.zeros(B, dtype=torch.float64) for _ in range(WORLD)]
        dist.all_gather(parts, torch.from_numpy(cl))
        dparts = [torch.zeros(1, dtype=torch.float64) for _ in range(WORLD)]
        dist.all_gather(dparts, torch.tensor([dl], dtype=torch.float64))
        c = torch.cat(parts).numpy()[:n]
        D = sum(float(x) for x in dparts)  # rank order: deterministic
        rk = np.zeros(B)
        rk[:r1 - r0] = pr
        rparts = [torch.zeros(B, dtype=torch.float64) for _ in range(WORLD)]
        dist.all_gather(rparts, torch.from_numpy(rk))
        rank_vec = torch.cat(rparts).numpy()[:n]
    ref = oracle.pagerank(n, rp, ci, g.out_degree, d, iters)
    np.testing.assert_allclose(rank_vec, ref, rtol=1e-12)


def test_pagerank_allgather_protocol():
    _run("_pagerank", 9, 6)


def _sssp(rank, scale, src_i):
    from paper_conf_icpp_liwb15_b200 import inl
    g = inlgen.host_build(scale, 16, seed=1, flags=inlgen.SYMMETRIC)
    w = inlgen.weights_host(g.row_ptr, g.col_idx)
    n = g.n_global
    b = inl.partition_rows(n, WORLD)
    r0, r1 = b[rank], b[rank + 1]
    s = inlgen.sources(g.row_ptr, 4)[src_i]
    INF = 0xFFFFFFFF
    D = np.full(n + 1, INF, dtype=np.int64)  # dist ++ "no change" word
    D[s] = 0
    prev = D[r0:r1].copy()
    front = [s - r0] if r0 <= s < r1 else []
    rounds = 0
    while True:
        D[n] = 1
        for u in front:  # relax the owned frontier into the local copy (asynchronous inside)
            gu = r0 + u
            for k in range(g.row_ptr[gu], g.row_ptr[gu + 1]):
                v, nd = g.col_idx[k], D[gu] + int(w[k])
                if nd < D[v]:
                    D[v] = nd
                    D[n] = 0
        t = torch.from_numpy(D)
        dist.all_reduce(t, op=dist.ReduceOp.MIN)
        D = t.numpy().copy()
        rounds += 1
        if D[n] == 1:
            break
        changed = np.nonzero(D[r0:r1] < prev)[0]
        prev = D[r0:r1].copy()
        front = list(changed)
    ref = oracle.sssp(g.row_ptr, g.col_idx, w, s)
    assert np.array_equal(D[:n].astype(np.uint32), ref)
    assert rounds >= 2


def test_sssp_allreduce_min_protocol():
    _run("_sssp", 9, 0)
    _run("_sssp", 8, 3)


def _bfs(rank, scale, src_i):
    from paper_conf_icpp_liwb15_b200 import inl
    g = inlgen.host_build(scale, 16, seed=1, flags=inlgen.SYMMETRIC)
    n = g.n_global
    b = inl.partition_rows(n, WORLD)
    r0, r1 = b[rank], b[rank + 1]
    s = inlgen.sources(g.row_ptr, 4)[src_i]
    level = np.full(n, -1, dtype=np.int64)
    level[s] = 0
    visited = np.zeros(n, dtype=bool)
    visited[s] = True
    front = [s - r0] if r0 <= s < r1 else []
    L = 0
    while True:
        nxt = np.zeros(n + 1, dtype=np.uint8)
        for u in front:
            gu = r0 + u
            for v in g.col_idx[g.row_ptr[gu]:g.row_ptr[gu + 1]]:
                if not visited[v]:
                    nxt[v] = 1
                    nxt[n] = 1
        t = torch.from_numpy(nxt)
        dist.all_reduce(t, op=dist.ReduceOp.MAX)
        nxt = t.numpy()
        if nxt[n] == 0:
            break
        new = np.nonzero((nxt[:n] == 1) & (level < 0))[0]
        level[new] = L + 1
        visited[new] = True
        front = [v - r0 for v in new if r0 <= v < r1]
        L += 1
    assert np.array_equal(level.astype(np.int32), oracle.bfs(g.row_ptr, g.col_idx, s))


def test_bfs_allreduce_max_protocol():
    _run("_bfs", 10, 0)
    _run("_bfs", 9, 4)
