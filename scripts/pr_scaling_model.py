"""PageRank strong-scaling projection for SURVEY §8e's >= 5x gate (R-MAT scale 25, 20 iterations,
P = 1, 2, 4, 8) from ONE GPU — a model grounded in measurements, not a multi-GPU measurement
(this sandbox gives one GPU per call):

  gather(P):   PageRank's measured k_gather time per iteration at P = 1 (kernel timer), scaled
               by the measured ratio of a rank's share of a gather-shaped kernel: inl_spmv over
               row block 0 of inl_partition_rows(n, P) of the same in-CSR (unit values) —
               how a rank's gather time falls with its block;
  over:        the rest of a P = 1 iteration (x_hot copy, dangling sum, base), kept whole;
  X(P):        the allgather of one iteration's compacted contributions: each rank receives
               (P-1) * Bc * 4 bytes (Bc = the largest rank's pages with out-links), at the
               measured 770 GB/s NVLink peer-copy bandwidth per direction
               (/opt/skills/guides/B200_PROFILING.md);
  T(P) = gather(P) + over + X(P) / K (the pipelined exchange hides all but the last of its
         K = 4 sub-blocks);  speedup = T(1) / T(P).

usage: python scripts/pr_scaling_model.py > profiles/r02/pr_scaling_model.jsonl
"""
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import torch  # noqa: E402

import inlgen  # noqa: E402
from paper_conf_icpp_liwb15_b200 import inl  # noqa: E402

NVLINK_GBS = 770.0  # measured peer copy per direction (B200_PROFILING.md)
K = 4


def timed(fn, reps=10):
    for _ in range(3):
        fn()
    torch.cuda.synchronize()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record()
    for _ in range(reps):
        fn()
    e1.record()
    torch.cuda.synchronize()
    return e0.elapsed_time(e1) / reps


def main():
    torch.cuda.set_device(0)
    ctx = inl.Ctx(0)
    g = inlgen.dev_build(25, 16, seed=inlgen.SEED_GRAPH, flags=inlgen.TRANSPOSE)
    rp, ci, od = g["row_ptr"], g["col_idx"], g["out_degree"]
    n = g["n_global"]
    # the measured full PageRank at P = 1 (20 iterations) and its gather share (kernel timer)
    A = inl.Csr(rp, ci, n)
    plan = inl.Plan(ctx, A)
    r = torch.empty(n, device="cuda")
    inl.pagerank(ctx, A, od, r, 0.85, 20, plan)
    ctx.ktimer_enable(True)
    pr_ms = timed(lambda: inl.pagerank(ctx, A, od, r, 0.85, 20, plan), reps=3) / 20
    nl, gms = ctx.ktimer_read("k_gather")
    ctx.ktimer_enable(False)
    gather1 = gms / nl
    over = pr_ms - gather1
    x = torch.rand(n, device="cuda")
    nd = (od > 0).int()
    comp1 = None
    for P in (1, 2, 4, 8):
        b = inl.partition_rows(n, P)
        k0, k1 = int(rp[b[0]]), int(rp[b[1]])
        Ab = inl.Csr((rp[b[0]:b[1] + 1] - k0).contiguous(), ci[k0:k1], n, b[0])
        pb = inl.Plan(ctx, Ab)
        ones = torch.ones(k1 - k0, device="cuda")
        y = torch.empty(b[1] - b[0], device="cuda")
        comp = timed(lambda: inl.spmv(ctx, Ab, ones, x, y, pb))
        comp1 = comp1 or comp
        gather = gather1 * comp / comp1
        Bc = max(int(nd[b[q]:b[q + 1]].sum()) for q in range(P))
        x_ms = (P - 1) * Bc * 4 / (NVLINK_GBS * 1e9) * 1e3
        T = gather + over + x_ms / K
        print(json.dumps({"P": P, "rows_per_rank": b[1] - b[0], "nnz_rank0": k1 - k0,
                          "measured_pagerank_ms_per_iter_P1": round(pr_ms, 4),
                          "measured_gather_ms_per_iter_P1": round(gather1, 4),
                          "measured_block_gather_proxy_ms": round(comp, 4), "gather_ms": round(gather, 4),
                          "overhead_ms": round(over, 4), "exchange_bytes_per_rank": (P - 1) * Bc * 4,
                          "exchange_ms_at_770GBs": round(x_ms, 4), "model_ms_per_iter": round(T, 4),
                          "model_speedup": round(pr_ms / T, 2),
                          "kind": "projection (model), not a multi-GPU measurement"}), flush=True)
        del pb, Ab


if __name__ == "__main__":
    main()
