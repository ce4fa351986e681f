"""Template study for SSSP on B200 (the paper's Fig. 5 / Table I application): R-MAT scale 23
symmetric, w in 1..255, the thread-mapped baseline T1 (plain frontier Bellman-Ford, [5]) and
the paper's dbuf-shared / dbuf-global templates over lbTHRES (same algorithm), beside this
build's default (flat CTA windows + grid pieces, near-far delta).  One JSON line per variant:
mean time per source over `--sources` seeded sources (CUDA events on the ctx stream).

usage: python scripts/template_study_sssp.py [--scale 23] [--sources 3] > profiles/r01/template_study_sssp.jsonl
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


def citeseer_workload(op, torch):
    """The CiteSeer-shaped synthetic graph (n = 434,102, ~32.1 M CSR entries, degree 1..1,188,
    mean 73.9; inlgen.citeseer_like) on the GPU with the recipe's values / x / weights."""
    import inlgen
    cache = os.environ.get("INL_CITESEER_CACHE", "/tmp/inl_citeseer_seed1.inlcsr")  # regenerated if absent
    if os.path.exists(cache):
        h = inlgen.load_inlcsr(cache)
    else:
        h = inlgen.citeseer_like()
        inlgen.save_inlcsr(cache, h)
    rp = torch.from_numpy(h.row_ptr).cuda()
    ci = torch.from_numpy(h.col_idx).cuda()
    g = {"n_global": h.n_global, "row_begin": 0, "row_ptr": rp, "col_idx": ci, "out_degree": None}
    W = {"g": g, "n": h.n_global}
    if op == "spmv":
        W["val"] = inlgen.values_dev(rp, ci)
        W["x"] = inlgen.vector_dev(h.n_global)
    else:
        W["w"] = inlgen.weights_dev(rp, ci)
    torch.cuda.synchronize()
    return W


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--graph", choices=["rmat", "citeseer"], default="rmat",
                    help="citeseer: the CiteSeer-shaped graph of PAPER.md P5@12491 (inlgen.citeseer_like)")
    ap.add_argument("--scale", type=int, default=23)
    ap.add_argument("--sources", type=int, default=3)
    ap.add_argument("--only", type=str, default="", help="NAME[:LBT] — run one variant (for ncu)")
    a = ap.parse_args()
    torch.cuda.set_device(0)
    stream = torch.cuda.Stream(0)
    torch.cuda.set_stream(stream)
    ctx = inl.Ctx(0)
    W = citeseer_workload("sssp", torch) if a.graph == "citeseer" else bench.build_workload("sssp", a.scale, 16, 1, 0, torch)
    g = W["g"]
    A = inl.Csr(g["row_ptr"], g["col_idx"], g["n_global"])
    srcs = inlgen.sources(g["row_ptr"].cpu().numpy(), a.sources)[: a.sources]
    d = torch.empty(A.n_global, dtype=torch.int32, device="cuda")
    ref = {}
    variants = [("thread_only (T1)", dict(flags=inl.BINS_THREAD_ONLY), None)]
    for name, fl in (("dual_queue", inl.BINS_TPL_DUAL_QUEUE), ("dbuf_shared", inl.BINS_TPL_DBUF_SHARED),
                     ("dbuf_global", inl.BINS_TPL_DBUF_GLOBAL)):
        for lbt in (32, 64, 128, 256, 1024):
            variants.append((name, dict(t_thread=lbt, t_warp=max(lbt, 16), t_block=max(lbt, 16), flags=fl), lbt))
    variants.append(("default (flat + grid, near-far)", dict(), None))
    if a.only:
        nm, _, lb = a.only.partition(":")
        variants = [v for v in variants if v[0].startswith(nm) and (not lb or str(v[2]) == lb)]
    t1 = None
    for name, kw, lbt in variants:
        plan = inl.Plan(ctx, A, inl.bins(**kw))
        inl.sssp(ctx, A, W["w"], srcs[0], d, plan)  # warm-up
        torch.cuda.synchronize()
        tot, relax = 0.0, 0
        for s in srcs:
            e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            e0.record(stream)
            st = inl.sssp(ctx, A, W["w"], s, d, plan)
            e1.record(stream)
            torch.cuda.synchronize()
            tot += e0.elapsed_time(e1)
            relax += st["edges_relaxed"]
            h = hash(d.cpu().numpy().tobytes())
            assert ref.setdefault(s, h) == h, "distances differ between variants"
        ms = tot / len(srcs)
        if t1 is None:
            t1 = ms
        print(json.dumps({"template": name, "lbTHRES": lbt, "bins": kw, "ms_per_source": round(ms, 4),
                          "speedup_vs_T1": round(t1 / ms, 2), "relaxations": relax // len(srcs),
                          "scale": a.scale, "graph": a.graph, "sources": srcs}), flush=True)
        del plan


if __name__ == "__main__":
    main()
