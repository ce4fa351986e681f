"""PageRank template study (the paper's Fig. 6 PageRank bars and Table II PageRank row) on the
CiteSeer-shaped graph or R-MAT: the thread-mapped baseline T1, dual-queue, dbuf-global and
dbuf-shared over lbTHRES, beside the default pull gather.  One JSON line per variant: ms per
PageRank iteration (20 iterations, CUDA events), speedup over T1, max relative difference to
the default's ranks.

usage: python scripts/template_study_pr.py [--graph citeseer|rmat] [--scale 22] [--only NAME[:LBT]]
"""
import argparse
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import torch  # noqa: E402

import inlgen  # noqa: E402
from paper_conf_icpp_liwb15_b200 import inl  # noqa: E402


def citeseer_in_csr():
    """The CiteSeer-shaped graph (symmetric: its in-CSR is itself; out-degree = degree)."""
    cache = os.environ.get("INL_CITESEER_CACHE", "/tmp/inl_citeseer_seed1.inlcsr")
    if os.path.exists(cache):
        h = inlgen.load_inlcsr(cache)
    else:
        h = inlgen.citeseer_like()
        inlgen.save_inlcsr(cache, h)
    rp = torch.from_numpy(h.row_ptr).cuda()
    ci = torch.from_numpy(h.col_idx).cuda()
    od = (rp[1:] - rp[:-1]).int()
    return h.n_global, rp, ci, od


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--graph", choices=["rmat", "citeseer"], default="citeseer")
    ap.add_argument("--scale", type=int, default=22)
    ap.add_argument("--only", type=str, default="")
    ap.add_argument("--iterations", type=int, default=20)
    a = ap.parse_args()
    torch.cuda.set_device(0)
    stream = torch.cuda.Stream(0)
    torch.cuda.set_stream(stream)
    ctx = inl.Ctx(0)
    if a.graph == "citeseer":
        n, rp, ci, od = citeseer_in_csr()
    else:
        g = inlgen.dev_build(a.scale, 16, seed=inlgen.SEED_GRAPH, flags=inlgen.TRANSPOSE)
        n, rp, ci, od = g["n_global"], g["row_ptr"], g["col_idx"], g["out_degree"]
    A = inl.Csr(rp, ci, n)
    variants = [("thread_only (T1)", dict(cta_threads=192, flags=inl.BINS_THREAD_ONLY), None)]
    for name, fl in (("dual_queue", inl.BINS_TPL_DUAL_QUEUE), ("dbuf_global", inl.BINS_TPL_DBUF_GLOBAL),
                     ("dbuf_shared", inl.BINS_TPL_DBUF_SHARED)):
        for lbt in (32, 64, 256, 1024):
            variants.append((name, dict(t_thread=lbt, t_warp=max(lbt, 16), t_block=max(lbt, 16), cta_threads=64,
                                        flags=fl), lbt))
    variants.append(("default (pull gather)", dict(), None))
    if a.only:
        nm, _, lb = a.only.partition(":")
        variants = [v for v in variants if v[0].startswith(nm) and (not lb or str(v[2]) == lb)]
    r = torch.empty(n, device="cuda")
    ref, t1 = None, None
    for name, kw, lbt in variants:
        plan = inl.Plan(ctx, A, inl.bins(**kw))
        inl.pagerank(ctx, A, od, r, 0.85, a.iterations, plan)
        torch.cuda.synchronize()
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record(stream)
        inl.pagerank(ctx, A, od, r, 0.85, a.iterations, plan)
        e1.record(stream)
        torch.cuda.synchronize()
        ms = e0.elapsed_time(e1) / a.iterations
        if ref is None:
            ref = r.clone()
        err = float(((r - ref).abs() / ref.abs()).max().item())
        if t1 is None:
            t1 = ms
        print(json.dumps({"template": name, "lbTHRES": lbt, "bins": kw, "ms_per_iteration": round(ms, 4),
                          "speedup_vs_T1": round(t1 / ms, 2), "max_rel_diff_vs_T1": err, "graph": a.graph,
                          "n": n, "nnz": int(rp[-1])}), flush=True)
        del plan


if __name__ == "__main__":
    main()
