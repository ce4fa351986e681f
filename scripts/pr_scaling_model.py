"""PageRank strong-scaling projection for SURVEY §8e's >= 5x gate (R-MAT scale 25, 20 iterations,
P = 1, 2, 4, 8) from ONE GPU — a model grounded in measurements, not a multi-GPU measurement
(this sandbox gives one GPU per call):

  compute(P):  the measured time of one PageRank-shaped gather (inl_spmv with unit values over
               the in-CSR) on row block 0 of inl_partition_rows(n, P) — a rank's share of one
               iteration's gather;
  X(P):        the allgather of one iteration's compacted contributions: each rank receives
               (P-1) * Bc * 4 bytes (Bc = the largest rank's pages with out-links), at the
               measured 770 GB/s NVLink peer-copy bandwidth per direction
               (/opt/skills/guides/B200_PROFILING.md);
  T(P) = compute(P) + X(P) / K (the pipelined exchange hides all but the last of its K = 4
         sub-blocks) + the measured per-iteration overhead at P = 1;  speedup = T(1) / T(P).

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
    # the measured full PageRank at P = 1 (20 iterations) and its gather share
    A = inl.Csr(rp, ci, n)
    plan = inl.Plan(ctx, A)
    r = torch.empty(n, device="cuda")
    pr_ms = timed(lambda: inl.pagerank(ctx, A, od, r, 0.85, 20, plan), reps=3) / 20
    x = torch.rand(n, device="cuda")
    t1 = None
    for P in (1, 2, 4, 8):
        b = inl.partition_rows(n, P)
        k0, k1 = int(rp[b[0]]), int(rp[b[1]])
        Ab = inl.Csr((rp[b[0]:b[1] + 1] - k0).contiguous(), ci[k0:k1], n, b[0])
        pb = inl.Plan(ctx, Ab)
        ones = torch.ones(k1 - k0, device="cuda")
        y = torch.empty(b[1] - b[0], device="cuda")
        comp = timed(lambda: inl.spmv(ctx, Ab, ones, x, y, pb))
        # pages with out-links per rank block (the compacted exchange)
        nd = (od > 0).int()
        Bc = max(int(nd[b[q]:b[q + 1]].sum()) for q in range(P))
        x_ms = (P - 1) * Bc * 4 / (NVLINK_GBS * 1e9) * 1e3
        if P == 1:
            over = pr_ms - comp  # x_hot copy, dangling sum, base: per iteration at P = 1
            t1 = pr_ms
        T = comp + x_ms / K + over
        print(json.dumps({"P": P, "rows_per_rank": b[1] - b[0], "nnz_rank0": k1 - k0,
                          "measured_pagerank_ms_per_iter_P1": round(pr_ms, 4), "compute_ms": round(comp, 4),
                          "exchange_bytes_per_rank": (P - 1) * Bc * 4, "exchange_ms_at_770GBs": round(x_ms, 4),
                          "overhead_ms": round(over, 4), "model_ms_per_iter": round(T, 4),
                          "model_speedup": round(t1 / T, 2), "kind": "projection (model), not a multi-GPU measurement"}),
              flush=True)
        del pb, Ab


if __name__ == "__main__":
    main()
