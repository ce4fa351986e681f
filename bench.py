#!/usr/bin/env python
"""bench.py — the driver's benchmark contract for the load-balanced irregular nested loop.

Default (N = 1): SpMV fp32 on R-MAT scale 22, edge factor 16 (BASELINE.json
configs[1]), one `inl_spmv` call per step on a cached plan (degree bins built
once, timed separately).  Prints ONE JSON line (rank 0).

  python bench.py [--gpus N] [--steps K] [--warmup W] [--op spmv|sssp|bfs|pagerank]
  python bench.py --impl reference ...   # the CPU oracle on the host cores (bounded sample)

Under torchrun (N > 1) every rank owns a row block (inl_partition_rows) of an
R-MAT graph whose scale grows with log2(N) so per-GPU work stays fixed (weak
scaling), or, with --strong, of the N = 1 graph (strong scaling: PageRank at
scale 25 is the north star's >= 5x gate).  SpMV needs no collective for one
product (x replicated; the headline value), and the line also reports the
product followed by the allgather of y (inl_spmv_allgather, the form an iterated
SpMV needs); SSSP/BFS/PageRank use the library's NCCL exchange.  Time = max over
ranks of CUDA-event time.
"""
from __future__ import annotations

import argparse
import json
import math
import os
import statistics
import subprocess
import sys
import tempfile
import time

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

METRIC = "GTEPS and achieved HBM GB/s (fraction of peak) for SpMV/SSSP at 1/2/4/8 B200"
FALLBACK_HBM = 6650.0


def parse():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=20)
    ap.add_argument("--warmup", type=int, default=5)
    ap.add_argument("--impl", choices=["inl", "reference"], default="inl")
    ap.add_argument("--op", choices=["spmv", "sssp", "bfs", "pagerank", "bc"], default="spmv")
    ap.add_argument("--scale", type=int, default=None, help="R-MAT scale at N=1 (default per op)")
    ap.add_argument("--edge-factor", type=int, default=16)
    ap.add_argument("--bins", type=str, default="", help="t_thread,t_warp,t_block,grid_chunk,cta")
    ap.add_argument("--thread-only", action="store_true", help="paper baseline T1 (no load balancing)")
    ap.add_argument("--colblock", action="store_true", help="long rows column-blocked (INL_BINS_COLBLOCK)")
    ap.add_argument("--bin-flags", type=int, default=0, help="extra inl_bins.flags (e.g. 4 = INL_BINS_SSSP_DEVLOOP)")
    ap.add_argument("--no-e2e", action="store_true")
    ap.add_argument("--no-cpu-baseline", action="store_true")
    ap.add_argument("--iterations", type=int, default=20, help="PageRank iterations")
    ap.add_argument("--strong", action="store_true", help="N > 1: keep the N = 1 graph (strong scaling)")
    ap.add_argument("--no-context", action="store_true", help="skip the cuSPARSE / OpenMP context lines")
    return ap.parse_args()


DEFAULT_SCALE = {"spmv": 22, "sssp": 23, "bfs": 23, "pagerank": 25, "bc": 20}


def peaks():
    p = os.path.join(ROOT, "MEASURED_PEAKS.json")
    if os.path.exists(p):
        d = json.load(open(p))
        return float(d["hbm_gbs"]), "measured (MEASURED_PEAKS.json hbm_gbs, copy r+w)"
    return FALLBACK_HBM, "fallback (B200_PROFILING.md 6.65 TB/s)"


class Clocks:
    """Samples nvidia-smi during the timed region (B200_PROFILING.md clocks line)."""

    Q = ("clocks.sm,clocks.max.sm,power.draw,clocks_event_reasons.active,clocks_event_reasons.hw_slowdown,"
         "clocks_event_reasons.hw_thermal_slowdown,clocks_event_reasons.sw_thermal_slowdown,"
         "clocks_event_reasons.sw_power_cap")

    def __init__(self, index: int):
        self.f = tempfile.NamedTemporaryFile("w+", suffix=".csv", delete=False)
        self.idx = index
        self.p = None

    def __enter__(self):
        try:
            self.p = subprocess.Popen(["nvidia-smi", "-i", str(self.idx), f"--query-gpu={self.Q}",
                                       "--format=csv,noheader,nounits", "-lms", "100"],
                                      stdout=self.f, stderr=subprocess.DEVNULL)
        except Exception:
            self.p = None
        time.sleep(0.3)
        return self

    def __exit__(self, *a):
        if self.p:
            self.p.terminate()
            try:
                self.p.wait(timeout=5)
            except Exception:
                self.p.kill()

    def summary(self):
        try:
            rows = [l.split(",") for l in open(self.f.name).read().strip().splitlines() if l.strip()]
            os.unlink(self.f.name)
        except Exception:
            return {"sm_mhz": None, "sm_max_mhz": None, "reasons": ["unavailable"]}
        sm, smax, reasons = [], [], set()
        names = ["hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown", "sw_power_cap"]
        for r in rows:
            r = [x.strip() for x in r]
            try:
                sm.append(float(r[0]))
                smax.append(float(r[1]))
            except ValueError:
                continue
            for nm, v in zip(names, r[4:8]):
                if v.lower() == "active":
                    reasons.add(nm)
        if not sm:
            return {"sm_mhz": None, "sm_max_mhz": None, "reasons": ["unavailable"]}
        load = [s for s in sm if s > 0.5 * max(sm)] or sm
        return {"sm_mhz": statistics.median(load), "sm_max_mhz": max(smax), "samples": len(sm),
                "reasons": sorted(reasons)}


def dist_env():
    rank = int(os.environ.get("RANK", "0"))
    world = int(os.environ.get("WORLD_SIZE", "1"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    return rank, world, local


def cpu_cores():
    try:
        return len(os.sched_getaffinity(0))
    except Exception:
        return os.cpu_count() or 1


# --------------------------------------------------------------------------------------------
# Workloads (inputs generated on the GPU by inlgen, bit-identical to the host generator)
# --------------------------------------------------------------------------------------------

def build_workload(op, scale, ef, world, rank, torch):
    import inlgen
    from paper_conf_icpp_liwb15_b200 import inl
    flags = {"spmv": 0, "pagerank": inlgen.TRANSPOSE, "sssp": inlgen.SYMMETRIC, "bfs": inlgen.SYMMETRIC,
             "bc": inlgen.SYMMETRIC}[op]
    n = 1 << scale
    b = inl.partition_rows(n, world)
    g = inlgen.dev_build(scale, ef, seed=inlgen.SEED_GRAPH, flags=flags, row_begin=b[rank], row_end=b[rank + 1])
    w = {"g": g, "bounds": b, "n": n, "flags": flags}
    if op == "spmv":
        w["val"] = inlgen.values_dev(g["row_ptr"], g["col_idx"], row_begin=b[rank])
        w["x"] = inlgen.vector_dev(n)
    elif op == "sssp":
        w["w"] = inlgen.weights_dev(g["row_ptr"], g["col_idx"], row_begin=b[rank])
    torch.cuda.synchronize()
    return w


def spmv_bytes(nnz, n_rows, n_global):
    """Algorithmic bytes of one SpMV: col+val, int64 row_ptr, x once, y."""
    return 8 * nnz + 8 * (n_rows + 1) + 4 * n_global + 4 * n_rows


def pagerank_bytes_per_iter(nnz, n_rows, n_global):
    """Per iteration: col, row_ptr, contribution gather once, outdeg, c' write."""
    return 4 * nnz + 8 * (n_rows + 1) + 4 * n_global + 4 * n_rows + 4 * n_rows


# --------------------------------------------------------------------------------------------

def run_inl(a):
    import torch
    import torch.distributed as dist
    import inlgen
    from paper_conf_icpp_liwb15_b200 import inl

    rank, world, local = dist_env()
    if world != a.gpus:
        raise SystemExit(f"--gpus {a.gpus} but WORLD_SIZE={world}")
    torch.cuda.set_device(local)
    if world > 1:
        dist.init_process_group("nccl", device_id=torch.device("cuda", local))
    scale0 = a.scale or DEFAULT_SCALE[a.op]
    # weak scaling: fixed rows/nnz per GPU; --strong: the same graph at every N
    scale = scale0 + (0 if a.strong else int(round(math.log2(world))))
    stream = torch.cuda.Stream(local)
    torch.cuda.set_stream(stream)
    ctx = inl.Ctx(local)
    if world > 1 or a.op != "spmv":
        if world > 1:
            ctx.comm_init(world, rank)
    W = build_workload(a.op, scale, a.edge_factor, world, rank, torch)
    g = W["g"]
    A = inl.Csr(g["row_ptr"], g["col_idx"], g["n_global"], g["row_begin"])
    bargs = [int(v) for v in a.bins.split(",")] if a.bins else []
    bb = inl.bins(*bargs, flags=(inl.BINS_THREAD_ONLY if a.thread_only else 0) |
                  (inl.BINS_COLBLOCK if a.colblock else 0) | a.bin_flags)
    t0 = time.perf_counter()
    plan = inl.Plan(ctx, A, bb)
    torch.cuda.synchronize()
    plan_ms = (time.perf_counter() - t0) * 1e3
    info = plan.info()
    nnz_local = A.nnz
    peak, peak_src = peaks()

    out = {}
    if a.op == "spmv":
        y = torch.empty(A.n_rows, device="cuda")
        step = lambda: inl.spmv(ctx, A, W["val"], W["x"], y, plan)  # noqa: E731
        units_local = nnz_local
        bytes_local = spmv_bytes(nnz_local, A.n_rows, A.n_global)
        # k_build_xhot + k_gather (+ k_cb + k_cb_combine when rows are column-blocked)
        launches_per_step = (1 if a.thread_only else 2) + (2 if info["cb_rows"] > 0 else 0)
    elif a.op == "pagerank":
        r = torch.empty(A.n_global, device="cuda")
        step = lambda: inl.pagerank(ctx, A, g["out_degree"], r, 0.85, a.iterations, plan)  # noqa: E731
        units_local = nnz_local * a.iterations
        bytes_local = pagerank_bytes_per_iter(nnz_local, A.n_rows, A.n_global) * a.iterations
        launches_per_step = None  # counted by the library's kernel timer below
    else:
        # seeded sources of degree > 0 (+ the max-degree vertex); under torchrun rank 0 picks
        # them from its row block (global ids: its row_begin is 0) and broadcasts them
        srcs = inlgen.sources(g["row_ptr"].cpu().numpy(), 8) if rank == 0 else []
        if world > 1:
            src_t = torch.full((16,), -1, dtype=torch.int64, device="cuda")
            if rank == 0:
                src_t[:len(srcs)] = torch.tensor(srcs, dtype=torch.int64)
            dist.broadcast(src_t, 0)
            srcs = [int(v) for v in src_t.tolist() if v >= 0]
        out_arr = torch.empty(A.n_global, dtype=torch.int32, device="cuda")
        bc_arr = torch.empty(A.n_global, dtype=torch.float64, device="cuda") if a.op == "bc" else None
        state = {"i": 0, "last": None}

        def step():
            s = srcs[state["i"] % len(srcs)]
            state["i"] += 1
            if a.op == "sssp":
                state["last"] = inl.sssp(ctx, A, W["w"], s, out_arr, plan)
            elif a.op == "bc":  # one source per step: forward BFS DAG + backward dependencies
                state["last"] = inl.bc(ctx, A, [s], bc_arr, plan)
            else:
                state["last"] = inl.bfs(ctx, A, s, out_arr, plan)
        units_local = None
        bytes_local = None
        launches_per_step = None

    for _ in range(max(a.warmup, 0)):
        step()
    torch.cuda.synchronize()
    if world > 1:
        dist.barrier()
    ev0, ev1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    reached = []
    # the dominant kernel(s), timed live by the library with events on its own stream
    kernels = (["k_gather", "k_gather_chunks", "k_cb", "k_cb_combine"] if a.op in ("spmv", "pagerank")
               else ["k_bc_fwd", "k_bc_bwd"] if a.op == "bc"
               else ["k_expand_flat", "k_expand_grid", "k_bfs_bottom_up", "k_bu_thread", "k_bu_small", "k_bu_warp", "k_bu_deep",
                     "k_sssp_split", "sssp_graph"])
    if a.thread_only:
        kernels = ["k_gather_thread_only"] if a.op == "spmv" else ["k_expand", "k_expand_grid"]
    ctx.ktimer_enable(True)
    with Clocks(local) as ck:
        torch.cuda.synchronize()
        ev0.record(stream)
        marks = []  # per-step boundaries (mean as the paper reports it, P5@9184, plus min / median)
        for _ in range(a.steps):
            step()
            e = torch.cuda.Event(enable_timing=True)
            e.record(stream)
            marks.append(e)
            if a.op in ("sssp", "bfs", "bc"):
                reached.append(state["last"])
        ev1.record(stream)
        torch.cuda.synchronize()
    ms = ev0.elapsed_time(ev1)
    per_step = [ev0.elapsed_time(marks[0])] + [marks[i - 1].elapsed_time(marks[i]) for i in range(1, len(marks))]
    k_launches, k_ms, k_used, k_each = 0, 0.0, [], {}
    for kn in kernels:
        nl, kms = ctx.ktimer_read(kn)
        k_launches += nl
        k_ms += kms
        if nl:
            k_used.append(kn)
            k_each[kn] = {"launches": nl, "ms_per_launch": round(kms / nl, 5)}
    if a.op == "pagerank":
        # per step: init + base0; per iteration: x_hot + gather (+ k_cb + combine); between
        # iterations: dangling sum + base
        cb_on = "k_cb" in k_used
        launches_per_step = 2 + a.iterations * (4 if cb_on else 2) + (a.iterations - 1) * 2
    ctx.ktimer_enable(False)
    if world > 1:
        t = torch.tensor([ms], device="cuda")
        dist.all_reduce(t, op=dist.ReduceOp.MAX)
        ms = float(t.item())
    ms_step = ms / a.steps

    if a.op in ("sssp", "bfs", "bc"):
        # m_reached = sum of degrees of reached vertices (directed CSR entries) per source
        tot_edges = 0
        for i in range(a.steps):
            s = srcs[i % len(srcs)]
            if a.op == "sssp":
                inl.sssp(ctx, A, W["w"], s, out_arr, plan)
                reached_mask = out_arr.view(torch.int32) != -1
            else:
                inl.bfs(ctx, A, s, out_arr, plan)
                reached_mask = out_arr >= 0
            deg = (g["row_ptr"][1:] - g["row_ptr"][:-1])
            lo = g["row_begin"]
            tot_edges += int(deg[reached_mask[lo:lo + A.n_rows]].sum().item())
        units_local = tot_edges
        if a.op == "bc":
            # every reached edge is scanned twice (forward, backward): col + level per scan;
            # per reached vertex: row_ptr twice, sigma, delta, bc, queue
            bytes_local = 16 * tot_edges + 64 * sum(r["frontier_total"] for r in reached)
            for r in reached:
                r["edges_relaxed"] = 2 * tot_edges // max(len(reached), 1)
        else:
            relax = sum(r["edges_relaxed"] for r in reached)
            # per examined edge: col_idx (+ the weight for SSSP); per frontier vertex: row_ptr pair,
            # queue entry, distance/level (bitmaps and dist stay L2-resident)
            bytes_local = (8 if a.op == "sssp" else 4) * relax + 16 * sum(r["frontier_total"] for r in reached)
        if all(r.get("launches", 0) > 0 for r in reached):  # counted by the library
            launches_per_step = sum(r["launches"] for r in reached) / len(reached)
        else:
            launches_per_step = 1 + max(r["iterations"] for r in reached) * 2

    if a.op in ("spmv", "pagerank"):  # per-step figures -> whole timed region
        units_local *= a.steps
        bytes_local *= a.steps
    ag = None
    if a.op == "spmv" and world > 1:  # the product followed by the allgather of y (replicated)
        yg = torch.empty(A.n_global, device="cuda")
        for _ in range(max(a.warmup, 1)):
            inl.spmv_allgather(ctx, A, W["val"], W["x"], yg, plan)
        torch.cuda.synchronize()
        dist.barrier()
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record(stream)
        for _ in range(a.steps):
            inl.spmv_allgather(ctx, A, W["val"], W["x"], yg, plan)
        e1.record(stream)
        torch.cuda.synchronize()
        t = torch.tensor([e0.elapsed_time(e1)], device="cuda")
        dist.all_reduce(t, op=dist.ReduceOp.MAX)
        ag = float(t.item())
    cnt = torch.tensor([int(units_local), int(bytes_local)], dtype=torch.int64, device="cuda")
    kt = torch.tensor([k_ms], dtype=torch.float64, device="cuda")
    if world > 1:
        dist.all_reduce(cnt)
        dist.all_reduce(kt, op=dist.ReduceOp.MAX)
    units_total, bytes_total = (int(v) for v in cnt.tolist())
    k_ms = float(kt.item())
    gteps = units_total / (ms * 1e-3) / 1e9
    # roofline of the dominant kernel: algorithmic bytes of the timed region / the summed
    # device time of that kernel's launches (max over ranks); the step adds the small
    # launches around it (x_hot copy, PageRank reductions, frontier bookkeeping)
    achieved_gbs = (bytes_total / world) / (k_ms * 1e-3) / 1e9 if k_ms > 0 else 0.0

    if rank == 0:
        out.update({
            "metric": METRIC, "value": round(gteps, 3), "unit": "GTEPS", "n_gpus": world,
            "steps": a.steps, "warmup": a.warmup, "ms_per_step": round(ms_step, 5),
            "ms_per_step_min": round(min(per_step), 5), "ms_per_step_median": round(statistics.median(per_step), 5),
            "higher_is_better": True, "scaling": "strong" if (a.strong and world > 1) else "weak", "vs_baseline": None, "dtype": "f32" if a.op in ("spmv", "pagerank") else "u32",
            "data": "synthetic (R-MAT A,B,C=.57,.19,.19, Philox seeds graph=1 val=3 x=4 w=2, generated on GPU)",
            "config": {"workload": {"spmv": "cfg2 SpMV fp32 R-MAT", "pagerank": "cfg4 PageRank R-MAT in-CSR",
                                    "sssp": "cfg3 SSSP R-MAT symmetric w in 1..255",
                                    "bfs": "cfg5 BFS R-MAT symmetric",
                                    "bc": "NEXT-3 betweenness R-MAT symmetric (one source per step)"}[a.op],
                       "op": a.op, "scale": scale, "edge_factor": a.edge_factor, "n": A.n_global,
                       "nnz_total": units_total // a.steps // (a.iterations if a.op == "pagerank" else 1) if a.op in ("spmv", "pagerank") else None,
                       "rows_per_gpu": A.n_rows, "parallelism": f"row-blocks x{world}",
                       "bins": info["bins"], "plan_ms": round(plan_ms, 3),
                       "l2": "inputs larger than L2 (CSR streamed once per step; L2 is 126 MB)",
                       "thread_only_baseline": bool(a.thread_only)},
            "gpu_launches": int(round(launches_per_step * a.steps)) if launches_per_step else None,
        })
        frac = achieved_gbs / peak
        out["roofline"] = {"bound": "hbm", "achieved": round(achieved_gbs, 1), "peak": peak, "unit": "GB/s",
                           "frac": round(frac, 4), "peak_source": peak_src,
                           "frac_of_8TBs": round(achieved_gbs / 8000.0, 4),
                           "kernel": "+".join(k_used or kernels), "kernels": k_each,
                           "kernel_launches": k_launches, "kernel_ms_per_launch": round(k_ms / max(k_launches, 1), 5),
                           "kernel_share_of_step": round(k_ms / ms, 4),
                           "alg_bytes_per_step_per_gpu": int(bytes_total / world / a.steps),
                           "traffic": traffic_lookup(a.op, scale, "_t1" if a.thread_only else "")}
        out["plan"] = info
        if ag is not None:
            out["with_allgather"] = {"value": round(units_total / (ag * 1e-3) / 1e9, 3), "unit": "GTEPS",
                                     "ms_per_step": round(ag / a.steps, 5),
                                     "what": "inl_spmv_allgather: local product + NCCL allgather of y (replicated)"}
    if a.op == "spmv" and not a.no_e2e:
        e2e = e2e_spmv(a, ctx, g, W, torch, world, rank)
        if rank == 0:
            out["e2e"] = e2e
    if a.op in ("sssp", "bfs", "bc") and rank == 0:
        out["config"]["sources"] = srcs
        out["config"]["iterations"] = [r["iterations"] for r in reached]
        out["config"]["relaxations_per_m_reached"] = round(sum(r["edges_relaxed"] for r in reached) / max(units_total, 1), 3)
        out["config"]["host_syncs_per_source"] = round(sum(r.get("host_syncs", 0) for r in reached) / max(len(reached), 1), 1)
    if rank == 0:
        out["clocks"] = ck.summary()
        if not a.no_cpu_baseline and world == 1:
            out["cpu_baseline"] = cpu_baseline(a.op, g, W, a, torch)
            if not a.no_context:
                ctxl = context_lines(a.op, g, W, a, torch, A)
                if ctxl:
                    out["context"] = ctxl
        print(json.dumps(out), flush=True)
    if world > 1:
        dist.barrier()
        dist.destroy_process_group()


def traffic_lookup(op, scale, variant=""):
    """ncu dram bytes per launch of this op's dominant kernel at this scale (profiles/traffic.json),
    keyed by op, scale and variant ("" = the default kernels, "_t1" = the thread-only baseline)."""
    p = os.path.join(ROOT, "profiles", "traffic.json")
    try:
        d = json.load(open(p))
        return d.get(f"{op}_s{scale}{variant}")
    except Exception:
        return None


def host_info():
    """nproc, CPU model and RAM of the box (the oracle's line records them)."""
    model, ram = None, None
    try:
        for line in open("/proc/cpuinfo"):
            if line.startswith("model name"):
                model = line.split(":", 1)[1].strip()
                break
        for line in open("/proc/meminfo"):
            if line.startswith("MemTotal"):
                ram = round(int(line.split()[1]) / 1024 / 1024, 1)
                break
    except Exception:
        pass
    return {"nproc": os.cpu_count(), "cpu_model": model, "ram_gb": ram}


def context_lines(op, g, W, a, torch, A):
    """Context only: the oracle loops under OpenMP on all host cores (bit-identical
    to the oracle) and, for SpMV, cuSPARSE's CSR SpMV on the same matrix (a library call, timed
    with CUDA events).  Neither is the product or the parity reference."""
    import oracle
    out = {}
    rp = g["row_ptr"].cpu().numpy()
    ci = g["col_idx"].cpu().numpy()
    try:
        if op == "spmv":
            val, x = W["val"].cpu().numpy(), W["x"].cpu().numpy()
            reps, t0 = 0, time.perf_counter()
            while reps < 3 or time.perf_counter() - t0 < 3.0:
                oracle.spmv_par(rp, ci, val, x)
                reps += 1
            dt = (time.perf_counter() - t0) / reps
            out["cpu_parallel"] = {"value": round(len(ci) / dt / 1e9, 4), "unit": "GTEPS", "ms": round(dt * 1e3, 2),
                                   "cores": oracle.par_threads(), "kind": "oracle loops under OpenMP (orc_par.c)"}
        elif op == "pagerank":
            t0 = time.perf_counter()
            oracle.pagerank_par(g["n_global"], rp, ci, g["out_degree"].cpu().numpy(), 0.85, 2)
            dt = (time.perf_counter() - t0) / 2
            out["cpu_parallel"] = {"value": round(len(ci) / dt / 1e9, 4), "unit": "GTEPS",
                                   "ms_per_iteration": round(dt * 1e3, 2), "cores": oracle.par_threads(),
                                   "kind": "oracle loops under OpenMP (orc_par.c), 2 iterations"}
    except Exception as e:  # context only: never fail the bench over it
        out["cpu_parallel"] = {"error": repr(e)[:200]}
    if op == "spmv":
        try:
            M = torch.sparse_csr_tensor(g["row_ptr"], g["col_idx"].long(), W["val"],
                                        size=(A.n_rows, A.n_global))
            for _ in range(3):
                torch.mv(M, W["x"])
            torch.cuda.synchronize()
            e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            e0.record()
            for _ in range(10):
                torch.mv(M, W["x"])
            e1.record()
            torch.cuda.synchronize()
            ms = e0.elapsed_time(e1) / 10
            out["cusparse_spmv"] = {"ms": round(ms, 4), "value": round(len(ci) / (ms * 1e-3) / 1e9, 2),
                                    "unit": "GTEPS", "what": "torch.mv on a CSR tensor (cuSPARSE SpMV, int64 "
                                    "indices), same matrix / x, CUDA events, 10 calls; library context only"}
            del M
        except Exception as e:
            out["cusparse_spmv"] = {"error": repr(e)[:200]}
    return out


def e2e_spmv(a, ctx, g, W, torch, world, rank):
    """Same metric through the public API with HOST (pinned) buffers: H2D of the CSR, values and
    x, a transient plan, the kernel, and D2H of y — all inside the timed region."""
    import torch.distributed as dist
    from paper_conf_icpp_liwb15_b200 import inl
    rp = g["row_ptr"].cpu().pin_memory()
    ci = g["col_idx"].cpu().pin_memory()
    val = W["val"].cpu().pin_memory()
    x = W["x"].cpu().pin_memory()
    y = torch.empty(rp.numel() - 1, dtype=torch.float32).pin_memory()
    A = inl.Csr(rp, ci, g["n_global"], g["row_begin"])
    steps = max(3, min(a.steps, 10))
    inl.spmv(ctx, A, val, x, y)  # warm-up
    torch.cuda.synchronize()
    if world > 1:
        dist.barrier()
    t0 = time.perf_counter()
    for _ in range(steps):
        inl.spmv(ctx, A, val, x, y)  # returns after y is back on the host
    dt = time.perf_counter() - t0
    t = torch.tensor([dt], device="cuda")
    nn = torch.tensor([float(ci.numel())], device="cuda")
    if world > 1:
        dist.all_reduce(t, op=dist.ReduceOp.MAX)
        dist.all_reduce(nn)
    dt = float(t.item())
    h2d = rp.numel() * 8 + ci.numel() * 4 + val.numel() * 4 + x.numel() * 4
    return {"value": round(float(nn.item()) * steps / dt / 1e9, 4), "unit": "GTEPS",
            "h2d_bytes_per_step": int(h2d), "d2h_bytes_per_step": int(y.numel() * 4),
            "ms_per_step": round(dt / steps * 1e3, 3), "steps": steps,
            "path": "inl_spmv(host pinned buffers, plan=NULL): H2D + binning + gather + D2H (wall clock, synchronous)"}


def cpu_baseline(op, g, W, a, torch, budget_s=10.0):
    """The oracle as it stands (single thread, fp64) on the host cores, bounded sample."""
    import oracle
    rp = g["row_ptr"].cpu().numpy()
    ci = g["col_idx"].cpu().numpy()
    if op == "spmv":
        val, x = W["val"].cpu().numpy(), W["x"].cpu().numpy()
        reps, t0 = 0, time.perf_counter()
        while True:
            oracle.spmv(rp, ci, val, x)
            reps += 1
            if time.perf_counter() - t0 > budget_s:
                break
        dt = time.perf_counter() - t0
        return {"value": round(len(ci) * reps / dt / 1e9, 5), "unit": "GTEPS", "cores": 1, "kind": "oracle",
                "sample": f"full cfg2 matrix ({len(ci)} nnz) x {reps} repetitions, {dt:.1f} s", **host_info()}
    if op == "pagerank":
        t0 = time.perf_counter()
        it = 2
        oracle.pagerank(g["n_global"], rp, ci, g["out_degree"].cpu().numpy(), 0.85, it)
        dt = time.perf_counter() - t0
        return {"value": round(len(ci) * it / dt / 1e9, 5), "unit": "GTEPS", "cores": 1, "kind": "oracle",
                "sample": f"{it} PageRank iterations on the full graph ({len(ci)} nnz), {dt:.1f} s", **host_info()}
    import inlgen
    src = inlgen.sources(rp, 1)[0]
    t0 = time.perf_counter()
    if op == "sssp":
        d = oracle.sssp(rp, ci, W["w"].cpu().numpy().view("uint32"), src)
        reached = d != 0xFFFFFFFF
    else:
        d = oracle.bfs(rp, ci, src)
        reached = d >= 0
        if op == "bc":
            oracle.bc(rp, ci, [src])
    dt = time.perf_counter() - t0
    m = int((rp[1:] - rp[:-1])[reached].sum())
    return {"value": round(m / dt / 1e9, 5), "unit": "GTEPS", "cores": 1, "kind": "oracle",
            "sample": f"1 source ({src}), m_reached={m}, {dt:.1f} s", **host_info()}


def run_reference(a):
    """--impl reference: the oracle (plain C, single thread) on the host cores, on this arm's
    workload and metric.  Rank 0 only; other ranks exit 0 without work."""
    rank, world, local = dist_env()
    if rank != 0:
        return
    import numpy as np
    import inlgen
    import oracle
    scale0 = a.scale or DEFAULT_SCALE[a.op]
    scale = scale0 + (0 if a.strong else int(round(math.log2(max(world, 1)))))
    # bounded: the host generator builds the graph for small scales; large ones use the GPU twin
    try:
        import torch
        have_gpu = torch.cuda.is_available()
    except Exception:
        have_gpu = False
    flags = {"spmv": 0, "pagerank": inlgen.TRANSPOSE, "sssp": inlgen.SYMMETRIC, "bfs": inlgen.SYMMETRIC,
             "bc": inlgen.SYMMETRIC}[a.op]
    if have_gpu:
        g = inlgen.dev_build(scale, a.edge_factor, seed=inlgen.SEED_GRAPH, flags=flags)
        rp, ci = g["row_ptr"].cpu().numpy(), g["col_idx"].cpu().numpy()
        od = g["out_degree"].cpu().numpy() if g["out_degree"] is not None else None
        n = g["n_global"]
    else:
        h = inlgen.host_build(scale, a.edge_factor, seed=inlgen.SEED_GRAPH, flags=flags)
        rp, ci, od, n = h.row_ptr, h.col_idx, h.out_degree, h.n_global
    if a.op == "spmv":
        val = inlgen.values_host(rp, ci)
        x = inlgen.vector_host(n)
        fn = lambda: oracle.spmv(rp, ci, val, x)  # noqa: E731
        units = len(ci)
        sample = "full cfg2 SpMV per step"
    elif a.op == "pagerank":
        fn = lambda: oracle.pagerank(n, rp, ci, od, 0.85, 1)  # noqa: E731
        units = len(ci)
        sample = "1 PageRank iteration of the full graph per step"
    else:
        src = inlgen.sources(rp, 1)[0]
        wts = inlgen.weights_host(rp, ci) if a.op == "sssp" else None
        fn = (lambda: oracle.sssp(rp, ci, wts, src)) if a.op == "sssp" else (lambda: oracle.bfs(rp, ci, src))
        d = fn()
        reached = (d != 0xFFFFFFFF) if a.op == "sssp" else (d >= 0)
        if a.op == "bc":
            fn = lambda: oracle.bc(rp, ci, [src])  # noqa: E731
        units = int(np.diff(rp)[reached].sum())
        sample = f"one full {a.op} from source {src} per step"
    for _ in range(max(a.warmup, 0)):
        fn()
    t0 = time.perf_counter()
    for _ in range(a.steps):
        fn()
    dt = time.perf_counter() - t0
    v = units * a.steps / dt / 1e9
    line = {"impl": "reference", "metric": METRIC, "value": round(v, 5), "unit": "GTEPS", "n_gpus": world,
            "steps": a.steps, "warmup": a.warmup, "ms_per_step": round(dt / a.steps * 1e3, 3),
            "higher_is_better": True, "scaling": "strong" if (a.strong and world > 1) else "weak", "vs_baseline": None, "dtype": "f64" if a.op in ("spmv", "pagerank") else "int64",
            "data": "synthetic (same R-MAT recipe and seeds as the inl arm)",
            "config": {"workload": {"spmv": "cfg2 SpMV fp32 R-MAT", "pagerank": "cfg4 PageRank R-MAT in-CSR",
                                    "sssp": "cfg3 SSSP R-MAT symmetric w in 1..255",
                                    "bfs": "cfg5 BFS R-MAT symmetric",
                                    "bc": "NEXT-3 betweenness R-MAT symmetric (one source per step)"}[a.op],
                       "op": a.op, "scale": scale, "edge_factor": a.edge_factor, "n": int(n), "nnz_total": int(len(ci))},
            "cpu_baseline": {"value": round(v, 5), "unit": "GTEPS", "cores": 1, "kind": "oracle", "sample": sample,
                             **host_info()},
            "e2e": {"value": round(v, 5), "unit": "GTEPS", "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0}}
    print(json.dumps(line), flush=True)


if __name__ == "__main__":
    args = parse()
    if args.impl == "reference":
        run_reference(args)
    else:
        run_inl(args)
