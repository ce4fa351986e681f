"""Template study on B200 (the paper's Fig. 4 / Table II experiment):
SpMV on the cfg2 matrix (R-MAT scale 22, ef 16) with the paper's templates — thread-mapped
baseline (T1), dual-queue, dbuf-global, dbuf-shared — over lbTHRES and CTA sizes, beside the
default fused gather and its own threshold sweep.  One JSON line per variant:
time per SpMV (mean of timed runs, CUDA events on the ctx stream), GTEPS, speedup over T1.

usage: python scripts/template_study.py [--scale 22] [--reps 10] > profiles/r01/template_study.jsonl
"""
import argparse
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import torch  # noqa: E402

import bench  # noqa: E402
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
    ap.add_argument("--scale", type=int, default=22)
    ap.add_argument("--reps", type=int, default=10)
    ap.add_argument("--quick", action="store_true")
    ap.add_argument("--only", type=str, default="", help="NAME[:LBT[:CTA]] — run one variant (for ncu)")
    a = ap.parse_args()
    torch.cuda.set_device(0)
    stream = torch.cuda.Stream(0)
    torch.cuda.set_stream(stream)
    ctx = inl.Ctx(0)
    W = citeseer_workload("spmv", torch) if a.graph == "citeseer" else bench.build_workload("spmv", a.scale, 16, 1, 0, torch)
    g = W["g"]
    A = inl.Csr(g["row_ptr"], g["col_idx"], g["n_global"])
    y = torch.empty(A.n_rows, device="cuda")
    ref = None

    def timed(bins):
        nonlocal ref
        plan = inl.Plan(ctx, A, bins)
        for _ in range(3):
            inl.spmv(ctx, A, W["val"], W["x"], y, plan)
        torch.cuda.synchronize()
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record(stream)
        for _ in range(a.reps):
            inl.spmv(ctx, A, W["val"], W["x"], y, plan)
        e1.record(stream)
        torch.cuda.synchronize()
        ms = e0.elapsed_time(e1) / a.reps
        if ref is None:
            ref = y.clone()
        err = float(((y - ref).abs() / ref.abs().clamp_min(1e-30)).max().item())
        del plan
        return ms, err

    variants = [("thread_only (T1)", dict(cta_threads=192, flags=inl.BINS_THREAD_ONLY), None, 192)]
    lbts = [32, 128, 1024] if a.quick else [32, 64, 128, 192, 256, 1024]
    ctas = [64, 192] if a.quick else [64, 192, 256]
    for name, fl in (("dual_queue", inl.BINS_TPL_DUAL_QUEUE), ("dbuf_global", inl.BINS_TPL_DBUF_GLOBAL),
                     ("dbuf_shared", inl.BINS_TPL_DBUF_SHARED)):
        for lbt in lbts:
            for cta in ctas:
                variants.append((name, dict(t_thread=lbt, t_warp=max(lbt, 16), t_block=max(lbt, 16),
                                            cta_threads=cta, flags=fl), lbt, cta))
    for tt in ([-1, 8, 32] if a.quick else [-1, 2, 4, 8, 16, 32]):
        for tw in ([1024] if a.quick else [256, 1024, 4096]):
            variants.append(("fused (default kernel)", dict(t_thread=tt, t_warp=tw), tt, None))
    if a.only:
        nm, _, rest = a.only.partition(":")
        lb, _, ct = rest.partition(":")
        variants = [v for v in variants if v[0].startswith(nm) and (not lb or str(v[2]) == lb) and
                    (not ct or str(v[3]) == ct)]
    t1 = None
    nnz = A.nnz
    for name, kw, lbt, cta in variants:
        ms, err = timed(inl.bins(**kw))
        if t1 is None:
            t1 = ms
        print(json.dumps({"template": name, "lbTHRES": lbt, "cta": cta, "bins": kw, "ms": round(ms, 5),
                          "gteps": round(nnz / (ms * 1e-3) / 1e9, 2), "speedup_vs_T1": round(t1 / ms, 2),
                          "max_rel_diff_vs_T1": err, "scale": a.scale, "graph": a.graph, "nnz": nnz}), flush=True)


if __name__ == "__main__":
    main()
