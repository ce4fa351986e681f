"""GPU parity: inl_spmv (CUDA, sm_100a, through the C-ABI) vs oracle.spmv (fp64 CPU).

Bar (BASELINE.json north_star): integer-valued SpMV bit-exact; fp32 U[0,1)
values max relative error <= 1e-5 vs fp64, rows with a zero reference exactly 0.
"""
import numpy as np
import pytest
import torch

import inlgen
import oracle
from paper_conf_icpp_liwb15_b200 import inl

pytestmark = pytest.mark.gpu
RTOL = 1e-5


def rel_err(y, ref):
    y = np.asarray(y, np.float64)
    nz = ref != 0
    assert np.all(y[~nz] == 0), "rows with a zero reference must be exactly 0"
    return float(np.max(np.abs(y[nz] - ref[nz]) / np.abs(ref[nz]))) if nz.any() else 0.0


def dev(a):
    return torch.from_numpy(np.ascontiguousarray(a)).cuda()


def run(ctx, rp, ci, n_global, val, x, plan_bins=None, row_begin=0, use_plan=True):
    A = inl.Csr(dev(rp), dev(ci), n_global, row_begin)
    y = torch.full((A.n_rows,), float("nan"), device="cuda")
    plan = inl.Plan(ctx, A, plan_bins) if use_plan else None
    inl.spmv(ctx, A, dev(val), dev(x), y, plan)
    torch.cuda.synchronize()
    return y.cpu().numpy(), plan


@pytest.fixture(scope="module")
def ctx():
    return inl.Ctx(0)


@pytest.fixture(scope="module")
def cfg1():
    g = inlgen.host_build(12, 16, seed=inlgen.SEED_GRAPH)
    return g


def test_cfg1_integer_values_bit_exact(ctx, cfg1):
    val = inlgen.values_host(cfg1.row_ptr, cfg1.col_idx, mode=1)
    x = inlgen.vector_host(cfg1.n_global, mode=1)
    ref = oracle.spmv(cfg1.row_ptr, cfg1.col_idx, val, x)
    y, _ = run(ctx, cfg1.row_ptr, cfg1.col_idx, cfg1.n_global, val, x)
    assert np.array_equal(y.astype(np.float64), ref)


def test_cfg1_uniform_values(ctx, cfg1):
    val = inlgen.values_host(cfg1.row_ptr, cfg1.col_idx)
    x = inlgen.vector_host(cfg1.n_global)
    ref = oracle.spmv(cfg1.row_ptr, cfg1.col_idx, val, x)
    y, plan = run(ctx, cfg1.row_ptr, cfg1.col_idx, cfg1.n_global, val, x)
    assert rel_err(y, ref) <= RTOL
    info = plan.info()
    assert info["rows_thread"] + info["rows_warp"] + info["rows_block"] + info["rows_grid"] == cfg1.n_rows
    assert info["nnz_thread"] + info["nnz_warp"] + info["nnz_block"] + info["nnz_grid"] == cfg1.nnz


SWEEP = [dict(), dict(t_thread=-1), dict(t_thread=1, t_warp=32, t_block=128, grid_chunk=32),
         dict(t_thread=32, t_warp=64, t_block=256, grid_chunk=240),
         dict(t_thread=4, t_warp=128, t_block=4096, grid_chunk=1008),
         dict(t_thread=8, t_warp=96, t_block=2048, grid_chunk=100), dict(grid_chunk=224),
         dict(t_thread=2, t_warp=48, t_block=128, grid_chunk=100000)]


@pytest.mark.parametrize("kw", SWEEP)
def test_threshold_sweep_invariance(ctx, cfg1, kw):
    """Every template variant re-maps the same loop nest (P5@2078-4753): same result."""
    val = inlgen.values_host(cfg1.row_ptr, cfg1.col_idx, mode=1)
    x = inlgen.vector_host(cfg1.n_global, mode=1)
    ref = oracle.spmv(cfg1.row_ptr, cfg1.col_idx, val, x)
    y, plan = run(ctx, cfg1.row_ptr, cfg1.col_idx, cfg1.n_global, val, x, inl.bins(**kw))
    assert np.array_equal(y.astype(np.float64), ref)
    valf = inlgen.values_host(cfg1.row_ptr, cfg1.col_idx)
    xf = inlgen.vector_host(cfg1.n_global)
    reff = oracle.spmv(cfg1.row_ptr, cfg1.col_idx, valf, xf)
    yf, _ = run(ctx, cfg1.row_ptr, cfg1.col_idx, cfg1.n_global, valf, xf, inl.bins(**kw))
    assert rel_err(yf, reff) <= RTOL


def test_thread_only_baseline_and_transient_plan(ctx, cfg1):
    val = inlgen.values_host(cfg1.row_ptr, cfg1.col_idx)
    x = inlgen.vector_host(cfg1.n_global)
    ref = oracle.spmv(cfg1.row_ptr, cfg1.col_idx, val, x)
    y, _ = run(ctx, cfg1.row_ptr, cfg1.col_idx, cfg1.n_global, val, x, inl.bins(flags=inl.BINS_THREAD_ONLY))
    assert rel_err(y, ref) <= RTOL
    y2, _ = run(ctx, cfg1.row_ptr, cfg1.col_idx, cfg1.n_global, val, x, use_plan=False)
    assert rel_err(y2, ref) <= RTOL
    y3, _ = run(ctx, cfg1.row_ptr, cfg1.col_idx, cfg1.n_global, val, x, use_plan=False)
    assert np.array_equal(y2, y3)  # deterministic: no float atomics


def test_host_buffers_end_to_end(ctx, cfg1):
    val = inlgen.values_host(cfg1.row_ptr, cfg1.col_idx)
    x = inlgen.vector_host(cfg1.n_global)
    y = np.full(cfg1.n_rows, np.nan, dtype=np.float32)
    A = inl.Csr(cfg1.row_ptr, cfg1.col_idx, cfg1.n_global)
    inl.spmv(ctx, A, val, x, y)
    yd, _ = run(ctx, cfg1.row_ptr, cfg1.col_idx, cfg1.n_global, val, x)
    assert np.array_equal(y, yd)  # same kernels, same bits
    assert rel_err(y, oracle.spmv(cfg1.row_ptr, cfg1.col_idx, val, x)) <= RTOL


def test_row_blocks_match_full(ctx, cfg1):
    """Row blocks (the multi-GPU partition): integer SpMV bit-identical to 1 GPU, fp32 within
    rounding (a row's segmented-sum order depends on where the tile/lane boundaries fall)."""
    val = inlgen.values_host(cfg1.row_ptr, cfg1.col_idx)
    x = inlgen.vector_host(cfg1.n_global)
    full, _ = run(ctx, cfg1.row_ptr, cfg1.col_idx, cfg1.n_global, val, x)
    for P in (2, 3, 8):
        b = inl.partition_rows(cfg1.n_rows, P)
        parts = []
        for p in range(P):
            lo, hi = cfg1.row_ptr[b[p]], cfg1.row_ptr[b[p + 1]]
            rp = cfg1.row_ptr[b[p]:b[p + 1] + 1] - lo
            yp, _ = run(ctx, rp, cfg1.col_idx[lo:hi], cfg1.n_global, val[lo:hi], x, row_begin=b[p])
            parts.append(yp)
        assert rel_err(np.concatenate(parts), full.astype(np.float64)) <= 1e-6
    vi = inlgen.values_host(cfg1.row_ptr, cfg1.col_idx, mode=1)
    xi = inlgen.vector_host(cfg1.n_global, mode=1)
    full, _ = run(ctx, cfg1.row_ptr, cfg1.col_idx, cfg1.n_global, vi, xi)
    b = inl.partition_rows(cfg1.n_rows, 3)
    parts = []
    for p in range(3):
        lo, hi = cfg1.row_ptr[b[p]], cfg1.row_ptr[b[p + 1]]
        rp = cfg1.row_ptr[b[p]:b[p + 1] + 1] - lo
        parts.append(run(ctx, rp, cfg1.col_idx[lo:hi], cfg1.n_global, vi[lo:hi], xi, row_begin=b[p])[0])
    assert np.array_equal(np.concatenate(parts), full)


def _adversarial():
    rng = np.random.default_rng(3)
    cases = {}
    cases["all_empty"] = np.zeros(1001, np.int64), np.zeros(0, np.int32), 1000
    cases["n1"] = np.array([0, 1], np.int64), np.array([0], np.int32), 1
    n = 2000
    deg = np.zeros(n, np.int64)
    deg[7] = 1_000_000  # one huge row (grid bin)
    deg[100:140] = rng.integers(0, 40, 40)
    rp = np.r_[0, np.cumsum(deg)]
    cases["huge_row"] = rp, rng.integers(0, n, int(rp[-1])).astype(np.int32), n
    degs = []
    for T in (8, 256, 2048, 4096, 1024, 32):  # lengths T and T+1 around every default threshold
        degs += [T, T + 1, T - 1]
    degs = np.array(degs + [1, 2, 3] * 5, np.int64)  # unaligned starts
    rng.shuffle(degs)
    rp = np.r_[0, np.cumsum(degs)]
    cases["thresholds"] = rp, rng.integers(0, 500, int(rp[-1])).astype(np.int32), 500
    d = np.full(3000, 0, np.int64)
    d[::3] = 1
    d[1::7] = 5
    rp = np.r_[0, np.cumsum(d)]
    cases["many_tiny_rows"] = rp, rng.integers(0, 3000, int(rp[-1])).astype(np.int32), 3000
    return cases


@pytest.mark.parametrize("name", ["all_empty", "n1", "huge_row", "thresholds", "many_tiny_rows"])
def test_adversarial_csrs(ctx, name):
    rp, ci, ng = _adversarial()[name]
    val = inlgen.values_host(rp, ci, mode=1)
    x = inlgen.vector_host(ng, mode=1)
    ref = oracle.spmv(rp, ci, val, x)
    for kw in (dict(), dict(t_thread=1, t_warp=32, t_block=256, grid_chunk=64)):
        if 255 * 15 * (np.diff(rp).max() if rp[-1] else 0) < 2 ** 24:
            y, _ = run(ctx, rp, ci, ng, val, x, inl.bins(**kw))
            assert np.array_equal(y.astype(np.float64), ref)
        valf = inlgen.values_host(rp, ci)
        xf = inlgen.vector_host(ng)
        y, _ = run(ctx, rp, ci, ng, valf, xf, inl.bins(**kw))
        assert rel_err(y, oracle.spmv(rp, ci, valf, xf)) <= RTOL


def test_misaligned_arrays_use_scalar_path(ctx, cfg1):
    val = inlgen.values_host(cfg1.row_ptr, cfg1.col_idx)
    x = inlgen.vector_host(cfg1.n_global)
    ci_d = torch.zeros(cfg1.nnz + 1, dtype=torch.int32, device="cuda")
    ci_d[1:] = dev(cfg1.col_idx)
    v_d = torch.zeros(cfg1.nnz + 3, dtype=torch.float32, device="cuda")
    v_d[3:] = dev(val)
    A = inl.Csr(dev(cfg1.row_ptr), ci_d[1:], cfg1.n_global)
    y = torch.empty(cfg1.n_rows, device="cuda")
    inl.spmv(ctx, A, v_d[3:], dev(x), y, inl.Plan(ctx, A))
    full, _ = run(ctx, cfg1.row_ptr, cfg1.col_idx, cfg1.n_global, val, x)
    assert np.array_equal(y.cpu().numpy(), full)


def test_plan_mismatch_rejected(ctx, cfg1):
    A = inl.Csr(dev(cfg1.row_ptr), dev(cfg1.col_idx), cfg1.n_global)
    B = inl.Csr(dev(cfg1.row_ptr), dev(cfg1.col_idx), cfg1.n_global)
    plan = inl.Plan(ctx, A)
    x = torch.zeros(cfg1.n_global, device="cuda")
    with pytest.raises(inl.InlError) as e:
        inl.spmv(ctx, B, torch.zeros(cfg1.nnz, device="cuda"), x, torch.zeros(cfg1.n_rows, device="cuda"), plan)
    assert e.value.code == 1


def test_gpu_generator_bit_identical_to_host():
    for scale, flags in ((12, 0), (12, inlgen.SYMMETRIC), (11, inlgen.TRANSPOSE), (14, 0)):
        h = inlgen.host_build(scale, 16, seed=7, flags=flags)
        d = inlgen.dev_build(scale, 16, seed=7, flags=flags)
        assert np.array_equal(d["row_ptr"].cpu().numpy(), h.row_ptr)
        assert np.array_equal(d["col_idx"].cpu().numpy(), h.col_idx)
        if flags & inlgen.TRANSPOSE:
            assert np.array_equal(d["out_degree"].cpu().numpy(), h.out_degree)
        w = inlgen.weights_dev(d["row_ptr"], d["col_idx"]).cpu().numpy().view(np.uint32)
        assert np.array_equal(w, inlgen.weights_host(h.row_ptr, h.col_idx))
        v = inlgen.values_dev(d["row_ptr"], d["col_idx"]).cpu().numpy()
        assert np.array_equal(v, inlgen.values_host(h.row_ptr, h.col_idx))
        x = inlgen.vector_dev(h.n_global).cpu().numpy()
        assert np.array_equal(x, inlgen.vector_host(h.n_global))
    part = inlgen.dev_build(12, 16, seed=7, flags=inlgen.SYMMETRIC, row_begin=1000, row_end=3000)
    hp = inlgen.host_build(12, 16, seed=7, flags=inlgen.SYMMETRIC, row_begin=1000, row_end=3000)
    assert np.array_equal(part["row_ptr"].cpu().numpy(), hp.row_ptr)
    assert np.array_equal(part["col_idx"].cpu().numpy(), hp.col_idx)


def test_cfg2_full_size_against_oracle(ctx):
    """BASELINE.json configs[1]: R-MAT scale 22, ef 16, the bench's launch configuration."""
    g = inlgen.dev_build(22, 16, seed=inlgen.SEED_GRAPH)
    rp, ci = g["row_ptr"], g["col_idx"]
    val = inlgen.values_dev(rp, ci)
    x = inlgen.vector_dev(g["n_global"])
    A = inl.Csr(rp, ci, g["n_global"])
    plan = inl.Plan(ctx, A)
    y = torch.empty(A.n_rows, device="cuda")
    inl.spmv(ctx, A, val, x, y, plan)
    torch.cuda.synchronize()
    ref = oracle.spmv(rp.cpu().numpy(), ci.cpu().numpy(), val.cpu().numpy(), x.cpu().numpy())
    assert rel_err(y.cpu().numpy(), ref) <= RTOL
    info = plan.info()
    assert info["rows_grid"] > 0 and info["n_grid_chunks"] > info["rows_grid"]
