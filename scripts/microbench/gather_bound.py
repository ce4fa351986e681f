"""Runs gather_bound.cu on the cfg2 matrix: original column order vs columns relabelled by
descending in-degree (hot columns dense).  Prints one line per variant."""
import ctypes as C
import os
import subprocess
import sys

import torch

ROOT = os.path.dirname(os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
sys.path.insert(0, ROOT)
import inlgen  # noqa: E402

here = os.path.dirname(os.path.abspath(__file__))
so = os.path.join(here, "gather_bound.so")
subprocess.check_call(["nvcc", "-gencode", "arch=compute_100a,code=sm_100a", "-O3", "-shared", "-Xcompiler", "-fPIC",
                       "-o", so, os.path.join(here, "gather_bound.cu")])
L = C.CDLL(so)
L.mb_run.argtypes = [C.c_void_p, C.c_void_p, C.c_int64, C.c_void_p, C.c_int, C.c_int, C.c_int, C.c_int,
                     C.POINTER(C.c_float)]
scale = int(sys.argv[1]) if len(sys.argv) > 1 else 22
g = inlgen.dev_build(scale, 16, seed=1)
col, n = g["col_idx"], g["n_global"]
val = inlgen.values_dev(g["row_ptr"], col)
x = inlgen.vector_dev(n)
nnz = col.numel() // 4 * 4
deg = torch.bincount(col.long(), minlength=n)
order = torch.argsort(deg, descending=True)
rank = torch.empty_like(order)
rank[order] = torch.arange(n, device=col.device)
col_hot = rank[col.long()].int()
ms = C.c_float()
bytes_stream = 8 * nnz
L.mb_run_hot.argtypes = [C.c_void_p, C.c_void_p, C.c_int64, C.c_void_p, C.c_void_p, C.c_int, C.c_int, C.c_int,
                         C.POINTER(C.c_float), C.c_int]
for K in (32768, 40960, 49152):
    hot = rank[col.long()] < K
    enc = torch.where(hot, -1 - rank[col.long()], col.long()).int()
    xhot = x[order[:K]].contiguous()
    for blk, un in ((1024, 1), (1024, 2), (1024, 4), (768, 4)):
        rc = L.mb_run_hot(enc.data_ptr(), val.data_ptr(), nnz, x.data_ptr(), xhot.data_ptr(), K, blk, 10, C.byref(ms), un)
        print(f"hot-smem K={K} block={blk} U={un}: rc={rc} {ms.value*1e3:8.1f} us  {bytes_stream/ms.value/1e6:8.1f} GB/s "
              f"(hot fraction {hot.float().mean().item():.3f})", flush=True)
for name, cc in (("orig", col), ("hot-relabel", col_hot)):
    for which, wname in ((0, "stream"), (2, "gather_u4")):
        for gm, blk in ((8, 256),):
            L.mb_run(cc.data_ptr(), val.data_ptr(), nnz, x.data_ptr(), which, gm, blk, 10, C.byref(ms))
            print(f"{name:12s} {wname:10s} grid={gm}x148 block={blk}: {ms.value*1e3:8.1f} us  "
                  f"{bytes_stream/ms.value/1e6:8.1f} GB/s (col+val only)", flush=True)
