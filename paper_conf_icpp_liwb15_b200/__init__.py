"""paper_conf_icpp_liwb15_b200 — B200-native (sm_100a) load-balanced irregular nested loops.

The hot path of Li, Wu, Becchi (ICPP 2015): the loop over CSR rows / vertices
with a variable-length inner loop over nonzeros / edges, load-balanced by
degree (thread / warp / block / grid bins), for SpMV, PageRank, SSSP and BFS.
All compute is in libinl.so (include/inl.h); `inl` is the ctypes binding.
"""
from . import inl  # noqa: F401
from .inl import Csr, Ctx, InlError, Plan, bfs, bins, pagerank, partition_rows, spmv, sssp  # noqa: F401

__all__ = ["inl", "Csr", "Ctx", "InlError", "Plan", "bfs", "bins", "pagerank", "partition_rows", "spmv", "sssp"]
