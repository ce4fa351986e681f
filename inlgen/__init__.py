"""inlgen — seeded synthetic inputs (R-MAT CSR graphs, values, weights, vectors).

Input side only: this module holds none of the paper's method arithmetic.  It
is the one module both the oracle side (tests/, bench.py cpu_baseline) and the
CUDA side consume (DESIGN.md §4 "Input recipe").  Host builds return numpy
arrays; device builds return torch CUDA tensors (torch is plumbing here).
"""
from __future__ import annotations

import ctypes as C
import os

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_LIB_PATH = os.path.join(_HERE, "libinlgen.so")
SYMMETRIC = 1
TRANSPOSE = 2

# Seeds of the recipe (SURVEY.md §8c reading 7): graph, weights, values, x, sources.
SEED_GRAPH, SEED_WEIGHT, SEED_VALUE, SEED_X, SEED_SOURCE = 1, 2, 3, 4, 5

_lib = None


def lib() -> C.CDLL:
    global _lib
    if _lib is None:
        if not os.path.exists(_LIB_PATH):
            raise RuntimeError(f"{_LIB_PATH} missing: run `python scripts/build.py`")
        L = C.CDLL(_LIB_PATH)
        i64, i32, u64, vp = C.c_int64, C.c_int, C.c_uint64, C.c_void_p
        L.inlgen_last_error.restype = C.c_char_p
        L.inlgen_philox.argtypes = [vp, vp, vp]
        L.inlgen_relabel.argtypes = [u64, i32, u64]
        L.inlgen_relabel.restype = u64
        L.inlgen_rmat_tuples.argtypes = [i32, u64, u64, i64, vp, vp]
        L.inlgen_host_build.argtypes = [i32, i32, u64, i32, i64, i64, C.POINTER(vp)]
        L.inlgen_dev_build.argtypes = [i32, i32, u64, i32, i64, i64, vp, C.POINTER(vp)]
        L.inlgen_graph_info.argtypes = [vp] + [C.POINTER(i64)] * 4 + [C.POINTER(i32)]
        L.inlgen_graph_export.argtypes = [vp, vp, vp, vp, vp]
        L.inlgen_graph_free.argtypes = [vp]
        L.inlgen_graph_free.restype = None
        for nm in ("inlgen_weights_host", "inlgen_weights_dev"):
            getattr(L, nm).argtypes = [i64, i64, vp, vp, u64, vp] + ([vp] if nm.endswith("dev") else [])
        for nm in ("inlgen_values_host", "inlgen_values_dev"):
            getattr(L, nm).argtypes = [i64, i64, vp, vp, u64, i32, vp] + ([vp] if nm.endswith("dev") else [])
        L.inlgen_vector_host.argtypes = [i64, i64, u64, i32, vp]
        L.inlgen_load_mtx.argtypes = [C.c_char_p, i32, C.POINTER(vp)]
        L.inlgen_save_csr.argtypes = [C.c_char_p, vp]
        L.inlgen_load_csr.argtypes = [C.c_char_p, C.POINTER(vp)]
        L.inlgen_graph_from_csr.argtypes = [i64, i64, i64, vp, vp, vp, vp, C.POINTER(vp)]
        L.inlgen_graph_values.argtypes = [vp, vp]
        L.inlgen_powerlaw_build.argtypes = [i64, i32, i32, C.c_double, u64, i32, C.POINTER(vp)]
        L.inlgen_tree_build.argtypes = [i32, i32, i32, u64, C.POINTER(vp)]
        L.inlgen_graph_parent.argtypes = [vp, vp]
        L.inlgen_vector_dev.argtypes = [i64, i64, u64, i32, vp, vp]
        _lib = L
    return _lib


def _check(rc: int, what: str) -> None:
    if rc != 0:
        raise RuntimeError(f"{what} failed ({rc}): {lib().inlgen_last_error().decode()}")


def _p(a: np.ndarray) -> int:
    return a.ctypes.data if a.size else 0


def philox(ctr, key) -> list[int]:
    c = np.asarray(ctr, dtype=np.uint32)
    k = np.asarray(key, dtype=np.uint32)
    o = np.zeros(4, dtype=np.uint32)
    lib().inlgen_philox(c.ctypes.data, k.ctypes.data, o.ctypes.data)
    return [int(v) for v in o]


def relabel(x: int, scale: int, seed: int = SEED_GRAPH) -> int:
    return int(lib().inlgen_relabel(x, scale, seed))


def rmat_tuples(scale: int, seed: int, e_begin: int, count: int):
    u = np.empty(count, dtype=np.int64)
    v = np.empty(count, dtype=np.int64)
    _check(lib().inlgen_rmat_tuples(scale, seed, e_begin, count, _p(u), _p(v)), "inlgen_rmat_tuples")
    return u, v


class HostGraph:
    """CSR on the host: row_ptr int64 [n_rows+1], col_idx int32 [nnz] (global ids)."""

    def __init__(self, n_global, row_begin, row_ptr, col_idx, out_degree=None, scale=None, flags=0, val=None):
        self.n_global = int(n_global)
        self.row_begin = int(row_begin)
        self.row_ptr = row_ptr
        self.col_idx = col_idx
        self.out_degree = out_degree
        self.scale = scale
        self.flags = flags
        self.val = val  # fp32 values of a loaded matrix (None for generated graphs)

    @property
    def n_rows(self) -> int:
        return len(self.row_ptr) - 1

    @property
    def nnz(self) -> int:
        return int(self.row_ptr[-1])


def _info(g):
    vals = [C.c_int64() for _ in range(4)]
    od = C.c_int()
    _check(lib().inlgen_graph_info(g, *[C.byref(v) for v in vals], C.byref(od)), "inlgen_graph_info")
    return [v.value for v in vals] + [od.value]


def host_build(scale: int, edge_factor: int = 16, seed: int = SEED_GRAPH, flags: int = 0,
               row_begin: int = 0, row_end: int = -1) -> HostGraph:
    g = C.c_void_p()
    _check(lib().inlgen_host_build(scale, edge_factor, seed, flags, row_begin, row_end, C.byref(g)),
           "inlgen_host_build")
    try:
        n_global, n_rows, rb, nnz, _ = _info(g)
        rp = np.empty(n_rows + 1, dtype=np.int64)
        ci = np.empty(max(nnz, 0), dtype=np.int32)
        od = np.empty(n_global, dtype=np.int32) if flags & TRANSPOSE else None
        _check(lib().inlgen_graph_export(g, _p(rp), _p(ci), _p(od) if od is not None else 0, None),
               "inlgen_graph_export")
    finally:
        lib().inlgen_graph_free(g)
    return HostGraph(n_global, rb, rp, ci, od, scale, flags)


def _host_graph(g, flags=0, scale=None) -> HostGraph:
    """Export a library host graph handle into numpy arrays (and free the handle)."""
    try:
        n_global, n_rows, rb, nnz, _ = _info(g)
        rp = np.empty(n_rows + 1, dtype=np.int64)
        ci = np.empty(max(nnz, 0), dtype=np.int32)
        od = np.empty(n_global, dtype=np.int32) if flags & TRANSPOSE else None
        _check(lib().inlgen_graph_export(g, _p(rp), _p(ci), _p(od) if od is not None else 0, None),
               "inlgen_graph_export")
        val = np.empty(max(nnz, 0), dtype=np.float32)
        if lib().inlgen_graph_values(g, _p(val) if nnz else val.ctypes.data) != 0:
            val = None
    finally:
        lib().inlgen_graph_free(g)
    return HostGraph(n_global, rb, rp, ci, od, scale, flags, val)


def load_mtx(path: str, flags: int = 0) -> HostGraph:
    """MatrixMarket coordinate file -> host CSR (self-loops dropped, repeated pairs keep the first
    value, columns sorted; SYMMETRIC adds reverses, TRANSPOSE gives the in-CSR + out_degree)."""
    g = C.c_void_p()
    _check(lib().inlgen_load_mtx(os.fsencode(path), flags, C.byref(g)), "inlgen_load_mtx")
    return _host_graph(g, flags)


def save_inlcsr(path: str, g: HostGraph) -> None:
    """Write a host CSR (with its values / out_degree when present) as an .inlcsr file."""
    h = C.c_void_p()
    rp = np.ascontiguousarray(g.row_ptr, dtype=np.int64)
    ci = np.ascontiguousarray(g.col_idx, dtype=np.int32)
    val = None if g.val is None else np.ascontiguousarray(g.val, dtype=np.float32)
    od = None if g.out_degree is None else np.ascontiguousarray(g.out_degree, dtype=np.int32)
    _check(lib().inlgen_graph_from_csr(g.n_global, len(rp) - 1, g.row_begin, _p(rp), _p(ci) if ci.size else None,
                                       _p(val) if val is not None and val.size else None,
                                       _p(od) if od is not None and od.size else None, C.byref(h)),
           "inlgen_graph_from_csr")
    try:
        _check(lib().inlgen_save_csr(os.fsencode(path), h), "inlgen_save_csr")
    finally:
        lib().inlgen_graph_free(h)


def load_inlcsr(path: str) -> HostGraph:
    g = C.c_void_p()
    _check(lib().inlgen_load_csr(os.fsencode(path), C.byref(g)), "inlgen_load_csr")
    # out_degree travels in the file when it was saved with one
    n_global, n_rows, rb, nnz, _ = _info(g)
    try:
        rp = np.empty(n_rows + 1, dtype=np.int64)
        ci = np.empty(max(nnz, 0), dtype=np.int32)
        od = np.empty(max(n_global, 1), dtype=np.int32)
        rc = lib().inlgen_graph_export(g, _p(rp), _p(ci), od.ctypes.data, None)
        od = od[:n_global] if rc == 0 else None
        if rc != 0:
            _check(lib().inlgen_graph_export(g, _p(rp), _p(ci), None, None), "inlgen_graph_export")
        val = np.empty(max(nnz, 0), dtype=np.float32)
        if lib().inlgen_graph_values(g, val.ctypes.data) != 0:
            val = None
    finally:
        lib().inlgen_graph_free(g)
    return HostGraph(n_global, rb, rp, ci, od, None, TRANSPOSE if od is not None else 0, val)


def powerlaw_build(n: int, dmin: int, dmax: int, mean: float, seed: int = SEED_GRAPH) -> HostGraph:
    """Undirected configuration-model graph with a truncated power-law degree sequence."""
    g = C.c_void_p()
    _check(lib().inlgen_powerlaw_build(n, dmin, dmax, mean, seed, 0, C.byref(g)), "inlgen_powerlaw_build")
    return _host_graph(g, SYMMETRIC)


SEED_TREE = 6


def tree_build(depth: int, outdegree: int, sparsity: int = 0, seed: int = SEED_TREE) -> HostGraph:
    """Synthetic tree of PAPER.md §III.C (depth levels, outdegree, sparsity): the children CSR
    (level-order ids, root 0) with .parent (parent[0] = -1)."""
    g = C.c_void_p()
    _check(lib().inlgen_tree_build(depth, outdegree, sparsity, seed, C.byref(g)), "inlgen_tree_build")
    n_global = _info(g)[0]
    par = np.empty(max(n_global, 1), dtype=np.int32)
    _check(lib().inlgen_graph_parent(g, par.ctypes.data), "inlgen_graph_parent")
    h = _host_graph(g)
    h.parent = par[:n_global]
    return h


# PAPER.md P5@12491-13052: CiteSeer, 434,102 nodes, "16 million edges", degree 1..1,188, mean 73.9
CITESEER_N, CITESEER_DMIN, CITESEER_DMAX, CITESEER_MEAN = 434102, 1, 1188, 73.9


def citeseer_like(seed: int = SEED_GRAPH) -> HostGraph:
    """The CiteSeer-shaped synthetic graph of SURVEY §8f NEXT-2 (symmetric CSR)."""
    return powerlaw_build(CITESEER_N, CITESEER_DMIN, CITESEER_DMAX, CITESEER_MEAN, seed)


# PAPER.md P5@13172-13524: Wiki-vote, 7,115 nodes, 103,689 edges, outdegree 0..893, mean 14.6
# (reading R7: an undirected stand-in with the same n, entry count and degree range;
# the configuration model needs dmin >= 1)
WIKIVOTE_N, WIKIVOTE_DMIN, WIKIVOTE_DMAX, WIKIVOTE_MEAN = 7115, 1, 893, 14.6


def wikivote_like(seed: int = SEED_GRAPH) -> HostGraph:
    """The Wiki-vote-shaped synthetic graph of the BC template study (Fig. 6; symmetric CSR)."""
    return powerlaw_build(WIKIVOTE_N, WIKIVOTE_DMIN, WIKIVOTE_DMAX, WIKIVOTE_MEAN, seed)


def dev_build(scale: int, edge_factor: int = 16, seed: int = SEED_GRAPH, flags: int = 0,
              row_begin: int = 0, row_end: int = -1, device=None):
    """Device build (bit-identical to host_build); returns a dict of torch CUDA tensors."""
    import torch
    dev = torch.device("cuda", torch.cuda.current_device() if device is None else device)
    stream = torch.cuda.current_stream(dev).cuda_stream
    g = C.c_void_p()
    with torch.cuda.device(dev):
        _check(lib().inlgen_dev_build(scale, edge_factor, seed, flags, row_begin, row_end, stream,
                                      C.byref(g)), "inlgen_dev_build")
        try:
            n_global, n_rows, rb, nnz, _ = _info(g)
            rp = torch.empty(n_rows + 1, dtype=torch.int64, device=dev)
            ci = torch.empty(max(nnz, 1), dtype=torch.int32, device=dev)[:nnz]
            od = torch.empty(n_global, dtype=torch.int32, device=dev) if flags & TRANSPOSE else None
            _check(lib().inlgen_graph_export(g, rp.data_ptr(), ci.data_ptr(),
                                             od.data_ptr() if od is not None else 0, stream),
                   "inlgen_graph_export")
        finally:
            lib().inlgen_graph_free(g)
    return {"n_global": n_global, "row_begin": rb, "row_ptr": rp, "col_idx": ci, "out_degree": od,
            "scale": scale, "flags": flags}


def weights_host(row_ptr, col_idx, row_begin=0, seed=SEED_WEIGHT) -> np.ndarray:
    w = np.empty(len(col_idx), dtype=np.uint32)
    _check(lib().inlgen_weights_host(len(row_ptr) - 1, row_begin, _p(row_ptr), _p(col_idx), seed, _p(w)),
           "inlgen_weights_host")
    return w


def values_host(row_ptr, col_idx, row_begin=0, seed=SEED_VALUE, mode=0) -> np.ndarray:
    v = np.empty(len(col_idx), dtype=np.float32)
    _check(lib().inlgen_values_host(len(row_ptr) - 1, row_begin, _p(row_ptr), _p(col_idx), seed, mode,
                                    _p(v)), "inlgen_values_host")
    return v


def vector_host(n, begin=0, seed=SEED_X, mode=0) -> np.ndarray:
    x = np.empty(n, dtype=np.float32)
    _check(lib().inlgen_vector_host(n, begin, seed, mode, _p(x)), "inlgen_vector_host")
    return x


def _stream(t):
    import torch
    return torch.cuda.current_stream(t.device).cuda_stream


def weights_dev(row_ptr, col_idx, row_begin=0, seed=SEED_WEIGHT):
    import torch
    w = torch.empty(max(col_idx.numel(), 1), dtype=torch.int32, device=col_idx.device)[:col_idx.numel()]
    _check(lib().inlgen_weights_dev(row_ptr.numel() - 1, row_begin, row_ptr.data_ptr(), col_idx.data_ptr(),
                                    seed, w.data_ptr(), _stream(w)), "inlgen_weights_dev")
    return w  # uint32 bit pattern stored in an int32 tensor (weights are <= 255)


def values_dev(row_ptr, col_idx, row_begin=0, seed=SEED_VALUE, mode=0):
    import torch
    v = torch.empty(max(col_idx.numel(), 1), dtype=torch.float32, device=col_idx.device)[:col_idx.numel()]
    _check(lib().inlgen_values_dev(row_ptr.numel() - 1, row_begin, row_ptr.data_ptr(), col_idx.data_ptr(),
                                   seed, mode, v.data_ptr(), _stream(v)), "inlgen_values_dev")
    return v


def vector_dev(n, begin=0, seed=SEED_X, mode=0, device=None):
    import torch
    dev = torch.device("cuda", torch.cuda.current_device() if device is None else device)
    x = torch.empty(max(n, 1), dtype=torch.float32, device=dev)[:n]
    _check(lib().inlgen_vector_dev(n, begin, seed, mode, x.data_ptr(), _stream(x)), "inlgen_vector_dev")
    return x


def sources(row_ptr: np.ndarray, count: int = 8, seed: int = SEED_SOURCE) -> list[int]:
    """SURVEY §8c reading 7: `count` seeded vertices with degree > 0, plus the max-degree vertex."""
    deg = np.diff(row_ptr)
    cand = np.nonzero(deg > 0)[0]
    out = []
    if len(cand) == 0:
        return [0]
    i = 0
    while len(out) < count and i < 64 * count:
        r = philox([i, 0, 0, 6], [seed & 0xFFFFFFFF, seed >> 32])[0]
        v = int(cand[r % len(cand)])
        if v not in out:
            out.append(v)
        i += 1
    hub = int(np.argmax(deg))
    if hub not in out:
        out.append(hub)
    return out
