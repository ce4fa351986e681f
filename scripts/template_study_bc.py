"""BC template study (the paper's Fig. 6 BC bars and Table II BC row) on the Wiki-vote-shaped
graph (inlgen.wikivote_like: n = 7,115, ~103.6 K CSR entries, degree 1..893 law, mean 14.6):
the thread-mapped baseline T1, dual-queue, dbuf-global and dbuf-shared over lbTHRES (both
sweeps of Brandes' BC through the same template), beside this build's two non-template paths:
level-synchronous (degree-binned levels, global pieces, pull steps when the plan finds the
graph symmetric) and source-parallel (one CTA per source, state in shared memory).  One JSON line per
variant: ms per source over `--sources` seeded sources (CUDA events), speedup over T1, max
relative difference of bc to T1's.

usage: python scripts/template_study_bc.py [--sources 256] [--only NAME[:LBT]] > profiles/r02/template_study_wikivote_bc.jsonl
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


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--sources", type=int, default=256)
    ap.add_argument("--only", type=str, default="")
    a = ap.parse_args()
    torch.cuda.set_device(0)
    stream = torch.cuda.Stream(0)
    torch.cuda.set_stream(stream)
    ctx = inl.Ctx(0)
    h = inlgen.wikivote_like()
    n = h.n_global
    A = inl.Csr(torch.from_numpy(h.row_ptr).cuda(), torch.from_numpy(h.col_idx).cuda(), n)
    srcs = inlgen.sources(h.row_ptr, a.sources)
    variants = [("thread_only (T1)", dict(cta_threads=192, flags=inl.BINS_THREAD_ONLY), None)]
    for name, fl in (("dual_queue", inl.BINS_TPL_DUAL_QUEUE), ("dbuf_global", inl.BINS_TPL_DBUF_GLOBAL),
                     ("dbuf_shared", inl.BINS_TPL_DBUF_SHARED)):
        for lbt in (32, 64, 256, 1024):
            variants.append((name, dict(t_thread=lbt, cta_threads=192, flags=fl), lbt))
    variants.append(("default level-synchronous (binned levels)", dict(), "level"))
    variants.append(("source-parallel (one CTA per source)", dict(), "src"))
    if a.only:
        nm, _, lb = a.only.partition(":")
        variants = [v for v in variants if v[0].startswith(nm) and (not lb or str(v[2]) == lb)]
    os.environ.pop("INL_BC_MODE", None)
    out = torch.empty(n, dtype=torch.float64, device="cuda")
    ref, t1 = None, None
    for name, kw, lbt in variants:
        if lbt in ("level", "src"):  # the two non-template paths (bc.cu)
            os.environ["INL_BC_MODE"] = lbt
        plan = inl.Plan(ctx, A, inl.bins(**kw))
        inl.bc(ctx, A, srcs, out, plan)  # warm-up (scratch sized for the source count)
        torch.cuda.synchronize()
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record(stream)
        st = inl.bc(ctx, A, srcs, out, plan)
        e1.record(stream)
        torch.cuda.synchronize()
        ms = e0.elapsed_time(e1) / len(srcs)
        if ref is None:
            ref = out.clone()
        nz = ref != 0
        err = float(((out[nz] - ref[nz]).abs() / ref[nz]).max().item()) if bool(nz.any()) else 0.0
        if t1 is None:
            t1 = ms
        print(json.dumps({"template": name, "lbTHRES": lbt, "bins": kw, "ms_per_source": round(ms, 4),
                          "speedup_vs_T1": round(t1 / ms, 2), "max_rel_diff_vs_T1": err,
                          "levels_per_source": st["iterations"] / len(srcs), "launches": st["launches"],
                          "graph": "wikivote_like", "n": n, "nnz": int(h.nnz), "sources": len(srcs)}), flush=True)
        del plan


if __name__ == "__main__":
    main()
