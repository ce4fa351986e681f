"""oracle — ctypes binding of liborc.so, the plain fp64 CPU ORACLE.

TEST INFRASTRUCTURE ONLY.  Only tests/, __graft_entry__.smoke() and bench.py
(the cpu_baseline leg and --impl reference) may import this module.  The
product package (paper_conf_icpp_liwb15_b200) never imports it, and it never
imports the product.  See oracle/orc.c for the passages each function follows.
"""
from __future__ import annotations

import ctypes as C
import os

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_LIB_PATH = os.path.join(_HERE, "liborc.so")
_lib = None


def lib() -> C.CDLL:
    global _lib
    if _lib is None:
        if not os.path.exists(_LIB_PATH):
            raise RuntimeError(f"{_LIB_PATH} missing: run `python scripts/build.py --only oracle`")
        L = C.CDLL(_LIB_PATH)
        vp, i64 = C.c_void_p, C.c_int64
        L.orc_version.restype = C.c_char_p
        L.orc_spmv.argtypes = [i64, vp, vp, vp, vp, vp]
        L.orc_pagerank.argtypes = [i64, vp, vp, vp, C.c_double, C.c_int32, vp]
        L.orc_sssp_dijkstra.argtypes = [i64, vp, vp, vp, i64, vp]
        L.orc_bfs.argtypes = [i64, vp, vp, i64, vp]
        L.orc_bc.argtypes = [i64, vp, vp, vp, i64, vp]
        L.orc_tree_descendants.argtypes = [i64, vp, vp, i64, vp]
        L.orc_tree_heights.argtypes = [i64, vp, vp, i64, vp]
        _lib = L
    return _lib


def _a(x, dt):
    x = np.ascontiguousarray(x, dtype=dt)
    return x, (x.ctypes.data if x.size else 0)


def _rc(rc, what):
    if rc != 0:
        raise RuntimeError(f"{what} returned {rc}")


_par = None


def par_lib() -> C.CDLL:
    """liborc_par.so: orc.c's SpMV / PageRank loops with the outer loop under OpenMP — the
    "CPU-parallel" context line of SURVEY §8d (bit-identical results; not a parity reference)."""
    global _par
    if _par is None:
        p = os.path.join(_HERE, "liborc_par.so")
        if not os.path.exists(p):
            raise RuntimeError(f"{p} missing: run `python scripts/build.py --only oracle`")
        L = C.CDLL(p)
        vp, i64 = C.c_void_p, C.c_int64
        L.orc_spmv_par.argtypes = [i64, vp, vp, vp, vp, vp]
        L.orc_pagerank_par.argtypes = [i64, vp, vp, vp, C.c_double, C.c_int32, vp]
        _par = L
    return _par


def par_threads() -> int:
    return int(par_lib().orc_par_threads())


def spmv_par(row_ptr, col_idx, val, x) -> np.ndarray:
    rp, prp = _a(row_ptr, np.int64)
    ci, pci = _a(col_idx, np.int32)
    va, pva = _a(val, np.float32)
    xx, pxx = _a(x, np.float32)
    n = len(rp) - 1
    y = np.empty(n, dtype=np.float64)
    _rc(par_lib().orc_spmv_par(n, prp, pci, pva, pxx, y.ctypes.data if n else 0), "orc_spmv_par")
    return y


def pagerank_par(n, in_row_ptr, in_col_idx, out_degree, damping=0.85, iterations=20) -> np.ndarray:
    rp, prp = _a(in_row_ptr, np.int64)
    ci, pci = _a(in_col_idx, np.int32)
    od, pod = _a(out_degree, np.int32)
    r = np.empty(n, dtype=np.float64)
    _rc(par_lib().orc_pagerank_par(n, prp, pci, pod, damping, iterations, r.ctypes.data if n else 0),
        "orc_pagerank_par")
    return r


def spmv(row_ptr, col_idx, val, x) -> np.ndarray:
    rp, prp = _a(row_ptr, np.int64)
    ci, pci = _a(col_idx, np.int32)
    va, pva = _a(val, np.float32)
    xx, pxx = _a(x, np.float32)
    n = len(rp) - 1
    y = np.empty(n, dtype=np.float64)
    _rc(lib().orc_spmv(n, prp, pci, pva, pxx, y.ctypes.data if n else 0), "orc_spmv")
    return y


def pagerank(n, in_row_ptr, in_col_idx, out_degree, damping=0.85, iterations=20) -> np.ndarray:
    rp, prp = _a(in_row_ptr, np.int64)
    ci, pci = _a(in_col_idx, np.int32)
    od, pod = _a(out_degree, np.int32)
    r = np.empty(n, dtype=np.float64)
    _rc(lib().orc_pagerank(n, prp, pci, pod, damping, iterations, r.ctypes.data if n else 0), "orc_pagerank")
    return r


def sssp(row_ptr, col_idx, w, source) -> np.ndarray:
    rp, prp = _a(row_ptr, np.int64)
    ci, pci = _a(col_idx, np.int32)
    ww, pww = _a(w, np.uint32)
    n = len(rp) - 1
    d = np.empty(n, dtype=np.uint32)
    _rc(lib().orc_sssp_dijkstra(n, prp, pci, pww, source, d.ctypes.data), "orc_sssp_dijkstra")
    return d


def bfs(row_ptr, col_idx, source) -> np.ndarray:
    rp, prp = _a(row_ptr, np.int64)
    ci, pci = _a(col_idx, np.int32)
    n = len(rp) - 1
    lv = np.empty(n, dtype=np.int32)
    _rc(lib().orc_bfs(n, prp, pci, source, lv.ctypes.data), "orc_bfs")
    return lv


def bc(row_ptr, col_idx, sources=None) -> np.ndarray:
    """Betweenness over the given sources (None = all vertices: exact BC), fp64."""
    rp, prp = _a(row_ptr, np.int64)
    ci, pci = _a(col_idx, np.int32)
    n = len(rp) - 1
    src = np.arange(n, dtype=np.int64) if sources is None else np.ascontiguousarray(sources, dtype=np.int64)
    out = np.empty(n, dtype=np.float64)
    _rc(lib().orc_bc(n, prp, pci, src.ctypes.data if src.size else 0, len(src), out.ctypes.data if n else 0),
        "orc_bc")
    return out


def tree_descendants(row_ptr, col_idx, root=0) -> np.ndarray:
    """desc[v] = 1 + sum of desc over v's children (children CSR), int64."""
    rp, prp = _a(row_ptr, np.int64)
    ci, pci = _a(col_idx, np.int32)
    n = len(rp) - 1
    out = np.empty(n, dtype=np.int64)
    _rc(lib().orc_tree_descendants(n, prp, pci, root, out.ctypes.data if n else 0), "orc_tree_descendants")
    return out


def tree_heights(row_ptr, col_idx, root=0) -> np.ndarray:
    """height[v] = 1 + max height over v's children (a leaf: 1), int64."""
    rp, prp = _a(row_ptr, np.int64)
    ci, pci = _a(col_idx, np.int32)
    n = len(rp) - 1
    out = np.empty(n, dtype=np.int64)
    _rc(lib().orc_tree_heights(n, prp, pci, root, out.ctypes.data if n else 0), "orc_tree_heights")
    return out
