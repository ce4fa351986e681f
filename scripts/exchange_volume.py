"""NEXT-1 exchange volume on the loopback communicator (P row-block ranks on one B200):
per-rank bytes moved by one SSSP / BFS call with the fused peer-memory exchange against the
round-1 collectives (dense allreduce-min over distances, byte-map allreduce-max), from
inl_stats.exchange_bytes; both modes' outputs compared.  Timing on one device says nothing
about NVLink, so only volumes are reported.

usage: python scripts/exchange_volume.py [--scale 22] [--P 8] > profiles/r02/exchange_volume.jsonl
"""
import argparse
import json
import os
import sys
import threading

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import torch  # noqa: E402

import inlgen  # noqa: E402
from paper_conf_icpp_liwb15_b200 import inl  # noqa: E402


def run(P, g, w, s, mode):
    os.environ["INL_BFS_EXCHANGE"] = "bytemap" if mode == "collective" else "bits"
    os.environ["INL_SSSP_EXCHANGE"] = "dense" if mode == "collective" else "sparse"
    n = g["n_global"]
    b = inl.partition_rows(n, P)
    rp, ci = g["row_ptr"], g["col_idx"]
    grp = inl.LoopGroup(P)
    streams = [torch.cuda.Stream() for _ in range(P)]
    ctxs, blocks = [], []
    for r in range(P):
        with torch.cuda.stream(streams[r]):
            c = inl.Ctx(0)
            c.comm_init_loopback(grp, r)
            ctxs.append(c)
        k0, k1 = int(rp[b[r]]), int(rp[b[r + 1]])
        blocks.append((inl.Csr((rp[b[r]:b[r + 1] + 1] - k0).contiguous(), ci[k0:k1], n, b[r]), w[k0:k1]))
    torch.cuda.synchronize()
    out = [None] * P

    def work(r):
        torch.cuda.set_device(0)
        with torch.cuda.stream(streams[r]):
            A, wl = blocks[r]
            d = torch.empty(n, dtype=torch.int32, device="cuda")
            ss = inl.sssp(ctxs[r], A, wl, s, d)
            lv = torch.empty(n, dtype=torch.int32, device="cuda")
            sb = inl.bfs(ctxs[r], A, s, lv)
            streams[r].synchronize()
            out[r] = (d, lv, ss, sb)
    th = [threading.Thread(target=work, args=(r,)) for r in range(P)]
    for t in th:
        t.start()
    for t in th:
        t.join()
    torch.cuda.synchronize()
    return out


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--scale", type=int, default=22)
    ap.add_argument("--P", type=int, nargs="+", default=[2, 4, 8])
    a = ap.parse_args()
    torch.cuda.set_device(0)
    g = inlgen.dev_build(a.scale, 16, seed=inlgen.SEED_GRAPH, flags=inlgen.SYMMETRIC)
    w = inlgen.weights_dev(g["row_ptr"], g["col_idx"])
    s = inlgen.sources(g["row_ptr"].cpu().numpy(), 1)[0]
    n = g["n_global"]
    for P in a.P:
        res = {m: run(P, g, w, s, m) for m in ("fused", "collective")}
        same = all(torch.equal(res["fused"][r][0], res["collective"][r][0]) and
                   torch.equal(res["fused"][r][1], res["collective"][r][1]) for r in range(P))
        rec = {"scale": a.scale, "n": n, "nnz": int(g["row_ptr"][-1]), "P": P, "source": s, "same_results": same}
        for m in ("fused", "collective"):
            rec[f"sssp_{m}_bytes_per_rank"] = max(o[2]["exchange_bytes"] for o in res[m])
            rec[f"bfs_{m}_bytes_per_rank"] = max(o[3]["exchange_bytes"] for o in res[m])
            rec[f"sssp_{m}_rounds"] = res[m][0][2]["iterations"]
            rec[f"bfs_{m}_levels"] = res[m][0][3]["iterations"]
        print(json.dumps(rec), flush=True)


if __name__ == "__main__":
    main()
