"""One SSSP source at the bench configuration (R-MAT scale 23 symmetric, w in 1..255) after a
warm-up source, for ncu launch lists of the per-step kernels (run with INL_SSSP_LOOP=host so
every step is a stream launch).  Prints the stats of the measured source.

usage: INL_SSSP_LOOP=host ncu --metrics ... python scripts/sssp_steps.py [--scale 23] [--source-index 1]
"""
import argparse
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import torch  # noqa: E402

import bench  # noqa: E402
import inlgen  # noqa: E402
from paper_conf_icpp_liwb15_b200 import inl  # noqa: E402


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--scale", type=int, default=23)
    ap.add_argument("--source-index", type=int, default=1)
    ap.add_argument("--op", choices=["sssp", "bfs"], default="sssp")
    ap.add_argument("--no-warmup", action="store_true", help="run only the measured source (ncu launch indices start at its first step)")
    a = ap.parse_args()
    torch.cuda.set_device(0)
    ctx = inl.Ctx(0)
    W = bench.build_workload(a.op, a.scale, 16, 1, 0, torch)
    g = W["g"]
    A = inl.Csr(g["row_ptr"], g["col_idx"], g["n_global"])
    plan = inl.Plan(ctx, A)
    srcs = inlgen.sources(g["row_ptr"].cpu().numpy(), 9)
    d = torch.empty(g["n_global"], dtype=torch.int32, device="cuda")
    for s in ((srcs[a.source_index],) if a.no_warmup else (srcs[0], srcs[a.source_index])):
        if a.op == "sssp":
            st = inl.sssp(ctx, A, W["w"], s, d, plan)
        else:
            st = inl.bfs(ctx, A, s, d, plan)
    torch.cuda.synchronize()
    print(json.dumps({"source": srcs[a.source_index], **st}))


if __name__ == "__main__":
    main()
