"""Tree descendants / heights study on B200 (the paper's Fig. 7 / 8 and their
(c) tables): regular depth-4 trees with outdegree 32..512, then outdegree 512 with sparsity 0..4.
Per configuration and problem: the flat template (thread per node, atomics up the parent chain)
and the level-synchronous pull, time per call (CUDA events, mean of --reps), atomics, kernel
launches, and the speedup over the serial CPU oracle (the paper's baseline is "the better one
between recursive and iterative serial CPU code"; here: the oracle's bottom-up loop, 1 core).
One JSON line per (config, problem, method); results parity-checked against the oracle.

usage: python scripts/tree_study.py [--reps 5] > profiles/r02/tree_study.jsonl
"""
import argparse
import json
import os
import sys
import time

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import numpy as np  # noqa: E402
import torch  # noqa: E402

import inlgen  # noqa: E402
import oracle  # noqa: E402
from paper_conf_icpp_liwb15_b200 import inl  # noqa: E402


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--reps", type=int, default=5)
    ap.add_argument("--depth", type=int, default=4)
    a = ap.parse_args()
    torch.cuda.set_device(0)
    stream = torch.cuda.Stream(0)
    torch.cuda.set_stream(stream)
    ctx = inl.Ctx(0)
    configs = [(d, 0) for d in (32, 64, 128, 256, 512)] + [(512, s) for s in (1, 2, 3, 4)]
    for d, sp in configs:
        t = inlgen.tree_build(a.depth, d, sp)
        n = t.n_global
        T = inl.Csr(torch.from_numpy(t.row_ptr).cuda(), torch.from_numpy(t.col_idx).cuda(), n)
        par = torch.from_numpy(t.parent).cuda()
        out = torch.empty(n, dtype=torch.int64, device="cuda")
        for prob, fn, ofn in (("descendants", inl.tree_descendants, oracle.tree_descendants),
                              ("heights", inl.tree_heights, oracle.tree_heights)):
            t0 = time.perf_counter()
            ref = ofn(t.row_ptr, t.col_idx, 0)
            cpu_ms = (time.perf_counter() - t0) * 1e3
            for method, name in ((inl.TREE_FLAT, "flat (thread per node, atomics)"),
                                 (inl.TREE_LEVELS, "levels (pull, one launch per level)")):
                st = fn(ctx, T, par, out, 0, method)  # warm-up
                torch.cuda.synchronize()
                assert np.array_equal(out.cpu().numpy(), ref), (d, sp, prob, name)
                e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
                e0.record(stream)
                for _ in range(a.reps):
                    st = fn(ctx, T, par, out, 0, method)
                e1.record(stream)
                torch.cuda.synchronize()
                ms = e0.elapsed_time(e1) / a.reps
                print(json.dumps({"outdegree": d, "sparsity": sp, "depth": a.depth, "nodes": n, "problem": prob,
                                  "method": name, "ms": round(ms, 4), "atomics": st["atomics"],
                                  "launches": st["launches"], "cpu_oracle_ms": round(cpu_ms, 2),
                                  "speedup_vs_cpu": round(cpu_ms / ms, 2)}), flush=True)
        del T, par, out
        torch.cuda.empty_cache()


if __name__ == "__main__":
    main()
