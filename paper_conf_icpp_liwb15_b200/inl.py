"""Thin ctypes binding of libinl.so (include/inl.h) — argument marshalling only.

Every step of the hot path runs in the library's sm_100a kernels; this module
only turns torch tensors / numpy arrays into pointers, passes the current
torch CUDA stream, and maps status codes to exceptions.  It never imports the
oracle and has no CPU fallback: if libinl.so is missing it raises.

Arrays may be CUDA tensors (the fast, asynchronous path for SpMV / PageRank)
or host arrays (numpy / CPU tensors; copied through the library's device
scratch — the end-to-end path).
"""
from __future__ import annotations

import ctypes as C
import os
from dataclasses import dataclass

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
LIB_PATH = os.environ.get("INL_LIB") or os.path.join(_HERE, "libinl.so")  # INL_LIB: A/B variant builds

INL_OK = 0
STATUS = {0: "INL_OK", 1: "INL_ERR_INVALID_ARGUMENT", 2: "INL_ERR_OUT_OF_MEMORY", 3: "INL_ERR_CUDA",
          4: "INL_ERR_NCCL", 5: "INL_ERR_NOT_INITIALIZED", 6: "INL_ERR_UNSUPPORTED", 7: "INL_ERR_INTERNAL"}
BINS_THREAD_ONLY = 1
BINS_COLBLOCK = 2
BINS_SSSP_DEVLOOP = 4
BINS_TPL_DUAL_QUEUE = 8
BINS_TPL_DBUF_GLOBAL = 16
BINS_TPL_DBUF_SHARED = 32
TREE_FLAT = 0    # the paper's flat template: thread per node, atomics up the parent chain
TREE_LEVELS = 1  # level-synchronous pull (B200 form of the hierarchical template)


class InlError(RuntimeError):
    def __init__(self, code: int, msg: str):
        super().__init__(f"{STATUS.get(code, code)}: {msg}")
        self.code = code


class CsrT(C.Structure):
    _fields_ = [("n_rows", C.c_int64), ("n_global", C.c_int64), ("row_begin", C.c_int64),
                ("nnz", C.c_int64), ("row_ptr", C.c_void_p), ("col_idx", C.c_void_p)]


class BinsT(C.Structure):
    _fields_ = [("t_thread", C.c_int32), ("t_warp", C.c_int32), ("t_block", C.c_int32),
                ("grid_chunk", C.c_int32), ("cta_threads", C.c_int32), ("flags", C.c_int32)]


class StatsT(C.Structure):
    _fields_ = [("iterations", C.c_int32), ("edges_relaxed", C.c_int64), ("frontier_total", C.c_int64),
                ("launches", C.c_int64), ("host_syncs", C.c_int64), ("exchange_bytes", C.c_int64)]


class PlanInfoT(C.Structure):
    _fields_ = [("n_tiles", C.c_int64), ("rows_thread", C.c_int64), ("rows_warp", C.c_int64),
                ("rows_block", C.c_int64), ("rows_grid", C.c_int64), ("nnz_thread", C.c_int64),
                ("nnz_warp", C.c_int64), ("nnz_block", C.c_int64), ("nnz_grid", C.c_int64),
                ("n_grid_chunks", C.c_int64), ("bins", BinsT), ("cb_rows", C.c_int64),
                ("cb_runs", C.c_int64), ("cb_nnz", C.c_int64), ("cb_width", C.c_int64),
                ("cb_threshold", C.c_int64), ("symmetric", C.c_int64)]


_lib = None


def lib() -> C.CDLL:
    """Load libinl.so (raises if it has not been built: there is no fallback)."""
    global _lib
    if _lib is None:
        if not os.path.exists(LIB_PATH):
            raise RuntimeError(f"{LIB_PATH} is missing: build it with `python scripts/build.py` "
                               "(the CUDA path has no CPU fallback)")
        L = C.CDLL(LIB_PATH)
        vp, i32, i64 = C.c_void_p, C.c_int32, C.c_int64
        L.inl_version.restype = C.c_char_p
        L.inl_status_string.restype = C.c_char_p
        L.inl_status_string.argtypes = [C.c_int]
        L.inl_last_error.restype = C.c_char_p
        L.inl_last_error.argtypes = [vp]
        L.inl_ctx_create.argtypes = [C.POINTER(vp), C.c_int, vp]
        L.inl_ctx_set_stream.argtypes = [vp, vp]
        L.inl_ctx_destroy.argtypes = [vp]
        L.inl_partition_rows.argtypes = [i64, i32, vp]
        L.inl_nccl_unique_id.argtypes = [vp]
        L.inl_comm_init.argtypes = [vp, vp, i32, i32]
        L.inl_loop_create.argtypes = [i32, C.POINTER(vp)]
        L.inl_loop_destroy.argtypes = [vp]
        L.inl_comm_init_loopback.argtypes = [vp, vp, i32]
        L.inl_spmv_allgather.argtypes = [vp, C.POINTER(CsrT), vp, vp, vp, vp]
        L.inl_plan_create.argtypes = [vp, C.POINTER(CsrT), C.POINTER(BinsT), C.POINTER(vp)]
        L.inl_plan_get_info.argtypes = [vp, C.POINTER(PlanInfoT)]
        L.inl_plan_destroy.argtypes = [vp]
        L.inl_csr_validate.argtypes = [vp, C.POINTER(CsrT)]
        L.inl_spmv.argtypes = [vp, C.POINTER(CsrT), vp, vp, vp, vp]
        L.inl_pagerank.argtypes = [vp, C.POINTER(CsrT), vp, C.c_float, i32, vp, vp]
        L.inl_sssp.argtypes = [vp, C.POINTER(CsrT), vp, i64, vp, C.POINTER(StatsT), vp]
        L.inl_bfs.argtypes = [vp, C.POINTER(CsrT), i64, vp, C.POINTER(StatsT), vp]
        L.inl_bc.argtypes = [vp, C.POINTER(CsrT), vp, i64, vp, C.POINTER(StatsT), vp]
        L.inl_tree_descendants.argtypes = [vp, C.POINTER(CsrT), vp, i64, i32, vp, C.POINTER(StatsT)]
        L.inl_tree_heights.argtypes = [vp, C.POINTER(CsrT), vp, i64, i32, vp, C.POINTER(StatsT)]
        L.inl_ktimer_enable.argtypes = [vp, i32]
        L.inl_ktimer_read.argtypes = [vp, C.c_char_p, C.POINTER(i64), C.POINTER(C.c_double)]
        for f in ("inl_ctx_create", "inl_ctx_set_stream", "inl_ctx_destroy", "inl_partition_rows",
                  "inl_nccl_unique_id", "inl_comm_init", "inl_loop_create", "inl_loop_destroy",
                  "inl_comm_init_loopback", "inl_spmv_allgather", "inl_tree_descendants", "inl_tree_heights",
                  "inl_plan_create", "inl_plan_get_info",
                  "inl_plan_destroy", "inl_csr_validate", "inl_spmv", "inl_pagerank", "inl_sssp", "inl_bfs",
                  "inl_ktimer_enable", "inl_ktimer_read"):
            getattr(L, f).restype = C.c_int
        _lib = L
    return _lib


def version() -> str:
    return lib().inl_version().decode()


def _check(rc: int, ctx=None) -> None:
    if rc != INL_OK:
        msg = lib().inl_last_error(ctx.handle if ctx is not None else None)
        raise InlError(rc, (msg or b"").decode())


def _ptr(a) -> int:
    if a is None:
        return 0
    if isinstance(a, np.ndarray):
        if not a.flags["C_CONTIGUOUS"]:
            raise ValueError("host arrays must be C-contiguous")
        return a.ctypes.data if a.size else 0
    import torch
    if isinstance(a, torch.Tensor):
        if not a.is_contiguous():
            raise ValueError("tensors must be contiguous")
        return a.data_ptr() if a.numel() else 0
    raise TypeError(f"unsupported array type {type(a)}")


def partition_rows(n: int, nranks: int) -> list[int]:
    """Row-block bounds (host only): bounds[p] = min(p * ceil(n/nranks), n)."""
    b = np.zeros(nranks + 1, dtype=np.int64)
    rc = lib().inl_partition_rows(n, nranks, b.ctypes.data)
    if rc != INL_OK:
        raise InlError(rc, lib().inl_last_error(None).decode())
    return [int(v) for v in b]


def broadcast_unique_id(rank: int, group=None, device=None) -> np.ndarray:
    """Rank 0 creates the NCCL unique id (inl_nccl_unique_id, no GPU needed) and every rank
    receives it through torch.distributed; without a process group, returns rank 0's id."""
    import torch
    import torch.distributed as dist
    uid = np.zeros(128, dtype=np.uint8)
    if rank == 0:
        rc = lib().inl_nccl_unique_id(uid.ctypes.data)
        if rc != INL_OK:
            raise InlError(rc, lib().inl_last_error(None).decode())
    if dist.is_available() and dist.is_initialized():
        t = torch.from_numpy(uid.copy())
        if dist.get_backend(group) == "nccl":
            t = t.cuda(device)
        dist.broadcast(t, src=0, group=group)
        uid = t.cpu().numpy().astype(np.uint8)
    return uid


class Ctx:
    """One library context per (process, device): stream, scratch, optional NCCL comm."""

    def __init__(self, device: int = 0):
        import torch
        self.device = int(device)
        h = C.c_void_p()
        stream = torch.cuda.current_stream(self.device).cuda_stream
        _check(lib().inl_ctx_create(C.byref(h), self.device, stream))
        self.handle = h
        self.nranks, self.rank = 1, 0

    def sync_stream(self) -> None:
        import torch
        lib().inl_ctx_set_stream(self.handle, torch.cuda.current_stream(self.device).cuda_stream)

    def comm_init(self, nranks: int, rank: int, group=None) -> None:
        """NCCL communicator; the unique id travels through torch.distributed (gloo or nccl)."""
        uid = broadcast_unique_id(rank, group, device=self.device)
        _check(lib().inl_comm_init(self.handle, uid.ctypes.data, nranks, rank), self)
        self.nranks, self.rank = nranks, rank

    def comm_init_loopback(self, group: "LoopGroup", rank: int) -> None:
        """Join a loopback group as `rank` (row-block contexts on one device)."""
        _check(lib().inl_comm_init_loopback(self.handle, group.handle, int(rank)), self)
        self.nranks, self.rank = group.nranks, int(rank)

    def ktimer_enable(self, on: bool = True) -> None:
        """Bracket the main kernels' launches with CUDA events (measurement only)."""
        _check(lib().inl_ktimer_enable(self.handle, 1 if on else 0), self)

    def ktimer_read(self, kernel: str) -> tuple[int, float]:
        """(launches, summed device ms) of `kernel` since ktimer_enable (syncs the stream)."""
        n, ms = C.c_int64(), C.c_double()
        _check(lib().inl_ktimer_read(self.handle, kernel.encode(), C.byref(n), C.byref(ms)), self)
        return int(n.value), float(ms.value)

    def close(self) -> None:
        if getattr(self, "handle", None):
            lib().inl_ctx_destroy(self.handle)
            self.handle = None

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass


class LoopGroup:
    """Host object of a loopback communicator for `nranks` contexts on one device
    (inl_loop_create).  Drive each member ctx from its own thread."""

    def __init__(self, nranks: int):
        h = C.c_void_p()
        rc = lib().inl_loop_create(int(nranks), C.byref(h))
        if rc != INL_OK:
            raise InlError(rc, "inl_loop_create")
        self.handle, self.nranks = h, int(nranks)

    def close(self) -> None:
        if getattr(self, "handle", None):
            lib().inl_loop_destroy(self.handle)
            self.handle = None

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass


@dataclass
class Csr:
    """A (local) CSR: row_ptr int64 [n_rows+1], col_idx int32 [nnz]; global ids."""
    row_ptr: object
    col_idx: object
    n_global: int
    row_begin: int = 0

    @property
    def n_rows(self) -> int:
        return int(self.row_ptr.shape[0]) - 1

    @property
    def nnz(self) -> int:
        return int(self.col_idx.shape[0])

    def struct(self) -> CsrT:
        return CsrT(self.n_rows, int(self.n_global), int(self.row_begin), self.nnz,
                    _ptr(self.row_ptr), _ptr(self.col_idx))


def bins(t_thread=0, t_warp=0, t_block=0, grid_chunk=0, cta_threads=0, flags=0) -> BinsT:
    return BinsT(t_thread, t_warp, t_block, grid_chunk, cta_threads, flags)


class Plan:
    """Degree bins of one device CSR on one ctx (reused across calls)."""

    def __init__(self, ctx: Ctx, A: Csr, b: BinsT | None = None):
        ctx.sync_stream()
        self.ctx, self.A = ctx, A
        self._s = A.struct()
        h = C.c_void_p()
        _check(lib().inl_plan_create(ctx.handle, C.byref(self._s), C.byref(b) if b is not None else None,
                                     C.byref(h)), ctx)
        self.handle = h

    def info(self) -> dict:
        i = PlanInfoT()
        _check(lib().inl_plan_get_info(self.handle, C.byref(i)), self.ctx)
        d = {f: getattr(i, f) for f, _ in PlanInfoT._fields_ if f != "bins"}
        d["bins"] = {f: getattr(i.bins, f) for f, _ in BinsT._fields_}
        return d

    def close(self) -> None:
        if getattr(self, "handle", None):
            lib().inl_plan_destroy(self.handle)
            self.handle = None

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass


def _plan_handle(plan):
    return plan.handle if plan is not None else None


def csr_validate(ctx: Ctx, A: Csr) -> None:
    ctx.sync_stream()
    s = A.struct()
    _check(lib().inl_csr_validate(ctx.handle, C.byref(s)), ctx)


def spmv(ctx: Ctx, A: Csr, val, x, y, plan: Plan | None = None):
    """y[i] = sum_k val[k] * x[col_idx[k]] over local row i (PAPER.md P5@10072)."""
    ctx.sync_stream()
    s = A.struct()
    _check(lib().inl_spmv(ctx.handle, C.byref(s), _ptr(val), _ptr(x), _ptr(y), _plan_handle(plan)), ctx)
    return y


def spmv_allgather(ctx: Ctx, A: Csr, val, x, y_global, plan: Plan | None = None):
    """y_global[n_global] = A * x replicated on every rank: this rank's row block, then the
    allgather of the blocks."""
    ctx.sync_stream()
    s = A.struct()
    _check(lib().inl_spmv_allgather(ctx.handle, C.byref(s), _ptr(val), _ptr(x), _ptr(y_global),
                                    _plan_handle(plan)), ctx)
    return y_global


def pagerank(ctx: Ctx, A_in: Csr, out_degree, rank, damping: float = 0.85, iterations: int = 20,
             plan: Plan | None = None):
    """PageRank pull over the in-edge CSR (PAPER.md P5@9262, P5@9781; reading R1)."""
    ctx.sync_stream()
    s = A_in.struct()
    _check(lib().inl_pagerank(ctx.handle, C.byref(s), _ptr(out_degree), C.c_float(damping), iterations,
                              _ptr(rank), _plan_handle(plan)), ctx)
    return rank


def sssp(ctx: Ctx, G: Csr, w, source: int, dist, plan: Plan | None = None) -> dict:
    """Single-source shortest paths (PAPER.md P5@10241); blocks until converged."""
    ctx.sync_stream()
    s = G.struct()
    st = StatsT()
    _check(lib().inl_sssp(ctx.handle, C.byref(s), _ptr(w), int(source), _ptr(dist), C.byref(st),
                          _plan_handle(plan)), ctx)
    return {"iterations": st.iterations, "edges_relaxed": st.edges_relaxed, "frontier_total": st.frontier_total,
            "launches": st.launches, "host_syncs": st.host_syncs,
            "exchange_bytes": st.exchange_bytes}


def bfs(ctx: Ctx, G: Csr, source: int, level, plan: Plan | None = None) -> dict:
    """Level-synchronous BFS (PAPER.md P5@11591); blocks until converged."""
    ctx.sync_stream()
    s = G.struct()
    st = StatsT()
    _check(lib().inl_bfs(ctx.handle, C.byref(s), int(source), _ptr(level), C.byref(st),
                         _plan_handle(plan)), ctx)
    return {"iterations": st.iterations, "edges_relaxed": st.edges_relaxed, "frontier_total": st.frontier_total,
            "launches": st.launches, "host_syncs": st.host_syncs,
            "exchange_bytes": st.exchange_bytes}


def bc(ctx: Ctx, G: Csr, sources, out, plan: Plan | None = None) -> dict:
    """Betweenness centrality over `sources` (PAPER.md P5@8318; reading R10): out[n_global]
    float64 (torch CUDA tensor or numpy), overwritten; blocks until done."""
    import numpy as np
    ctx.sync_stream()
    s = G.struct()
    src = np.ascontiguousarray(np.asarray(sources, dtype=np.int64))
    st = StatsT()
    _check(lib().inl_bc(ctx.handle, C.byref(s), src.ctypes.data if src.size else None, len(src), _ptr(out),
                        C.byref(st), _plan_handle(plan)), ctx)
    return {"iterations": st.iterations, "frontier_total": st.frontier_total, "launches": st.launches,
            "host_syncs": st.host_syncs}


def _tree(fn, ctx, T, parent, root, out, method):
    ctx.sync_stream()
    s = T.struct()
    st = StatsT()
    _check(fn(ctx.handle, C.byref(s), _ptr(parent), int(root), int(method), _ptr(out), C.byref(st)), ctx)
    return {"levels": st.iterations, "atomics": st.edges_relaxed, "launches": st.launches,
            "host_syncs": st.host_syncs}


def tree_descendants(ctx: Ctx, T: Csr, parent, out, root: int = 0, method: int = TREE_LEVELS) -> dict:
    """desc[v] = 1 + sum of desc over v's children (§II.C Fig. 3); out int64 [n]."""
    return _tree(lib().inl_tree_descendants, ctx, T, parent, root, out, method)


def tree_heights(ctx: Ctx, T: Csr, parent, out, root: int = 0, method: int = TREE_LEVELS) -> dict:
    """height[v] = 1 + max height over v's children, a leaf 1 (reading R14); out int64 [n]."""
    return _tree(lib().inl_tree_heights, ctx, T, parent, root, out, method)
