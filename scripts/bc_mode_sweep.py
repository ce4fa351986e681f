"""BC path choice (bc.cu bc_use_src): ms per source of the level-synchronous path and the
source-parallel path (one CTA per source) over graph size and source count.  One JSON line
per (graph, sources, mode).

usage: python scripts/bc_mode_sweep.py > profiles/r02/bc_mode_sweep.jsonl
"""
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import torch  # noqa: E402

import inlgen  # noqa: E402
from paper_conf_icpp_liwb15_b200 import inl  # noqa: E402


def main():
    torch.cuda.set_device(0)
    stream = torch.cuda.Stream(0)
    torch.cuda.set_stream(stream)
    ctx = inl.Ctx(0)
    graphs = [("wikivote_like", inlgen.wikivote_like())]
    for sc in (14, 16, 18, 20):
        graphs.append((f"rmat{sc}_sym", inlgen.host_build(sc, 16, seed=inlgen.SEED_GRAPH, flags=inlgen.SYMMETRIC)))
    for gname, h in graphs:
        A = inl.Csr(torch.from_numpy(h.row_ptr).cuda(), torch.from_numpy(h.col_idx).cuda(), h.n_global)
        plan = inl.Plan(ctx, A)
        out = torch.empty(h.n_global, dtype=torch.float64, device="cuda")
        for ns in (16, 74, 148, 592):
            srcs = inlgen.sources(h.row_ptr, ns)
            for mode in ("level", "src"):
                os.environ["INL_BC_MODE"] = mode
                try:
                    inl.bc(ctx, A, srcs, out, plan)  # warm-up: same source count (scratch sized)
                except inl.InlError as e:
                    print(json.dumps({"graph": gname, "n": h.n_global, "sources": len(srcs), "mode": mode,
                                      "skipped": str(e)}), flush=True)
                    continue
                torch.cuda.synchronize()
                e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
                e0.record(stream)
                st = inl.bc(ctx, A, srcs, out, plan)
                e1.record(stream)
                torch.cuda.synchronize()
                ms = e0.elapsed_time(e1)
                print(json.dumps({"graph": gname, "n": h.n_global, "nnz": int(h.nnz), "sources": len(srcs),
                                  "mode": mode, "ms": round(ms, 3), "ms_per_source": round(ms / len(srcs), 4),
                                  "launches": st["launches"]}), flush=True)
        del plan
    os.environ.pop("INL_BC_MODE", None)


if __name__ == "__main__":
    main()
