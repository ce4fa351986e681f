"""GPU parity: tree descendants / heights (§II.C Fig. 3, §III.C)
through the C-ABI against the oracle, for the paper's flat template (thread per node, atomics up
the parent chain) and the level-synchronous pull — bit-exact (integers), and the flat kernel's
atomic count equals the sum of node depths (Fig. 7(c): d + 2d^2 + 3d^3 on regular depth-4 trees)."""
import numpy as np
import pytest
import torch

import inlgen
import oracle
from paper_conf_icpp_liwb15_b200 import inl

pytestmark = pytest.mark.gpu


def dev(a):
    return torch.from_numpy(np.ascontiguousarray(a)).cuda()


@pytest.fixture(scope="module")
def ctx():
    return inl.Ctx(0)


def run(ctx, t, method, heights, root=0, host=False):
    n = len(t.row_ptr) - 1
    if host:
        T = inl.Csr(t.row_ptr, t.col_idx, n)
        out = np.zeros(n, np.int64)
        par = t.parent
    else:
        T = inl.Csr(dev(t.row_ptr), dev(t.col_idx), n)
        out = torch.zeros(n, dtype=torch.int64, device="cuda")
        par = dev(t.parent) if t.parent is not None else None
    fn = inl.tree_heights if heights else inl.tree_descendants
    st = fn(ctx, T, par, out, root, method)
    return (out if host else out.cpu().numpy()), st


METHODS = [inl.TREE_FLAT, inl.TREE_LEVELS]


@pytest.mark.parametrize("method", METHODS)
@pytest.mark.parametrize("d,sparsity", [(3, 0), (32, 0), (64, 0), (128, 2), (512, 4), (1, 0)])
def test_generated_trees(ctx, method, d, sparsity):
    depth = 4 if d > 1 else 60  # a path of 60 nodes for d = 1
    t = inlgen.tree_build(depth, d, sparsity)
    ref_d = oracle.tree_descendants(t.row_ptr, t.col_idx, 0)
    ref_h = oracle.tree_heights(t.row_ptr, t.col_idx, 0)
    got_d, st = run(ctx, t, method, False)
    assert np.array_equal(got_d, ref_d)
    got_h, sth = run(ctx, t, method, True)
    assert np.array_equal(got_h, ref_h)
    assert st["levels"] == depth
    if method == inl.TREE_FLAT:
        assert st["atomics"] == int(ref_d.sum()) - t.n_global  # sum of depths
        if sparsity == 0 and d > 1:
            assert st["atomics"] == d + 2 * d * d + 3 * d ** 3
    else:
        assert st["atomics"] == 0 and st["launches"] == 1 + depth


class _T:  # a tree given by parent[] (not level ordered)
    def __init__(self, parent):
        from test_oracle_tree import children_csr
        self.parent = np.asarray(parent, np.int32)
        self.row_ptr, self.col_idx = children_csr(parent)
        self.n_global = len(parent)


@pytest.mark.parametrize("method", METHODS)
@pytest.mark.parametrize("seed", range(4))
def test_random_unordered_trees(ctx, method, seed):
    rng = np.random.default_rng(seed)
    n = 5000
    perm = rng.permutation(n)
    parent = np.full(n, -1, np.int64)
    for i in range(1, n):
        parent[perm[i]] = perm[int(rng.integers(max(0, i - 50), i))]  # deep-ish trees
    t = _T(parent)
    root = int(perm[0])
    got, _ = run(ctx, t, method, False, root)
    assert np.array_equal(got, oracle.tree_descendants(t.row_ptr, t.col_idx, root))
    got, _ = run(ctx, t, method, True, root)
    assert np.array_equal(got, oracle.tree_heights(t.row_ptr, t.col_idx, root))


def test_host_buffers_and_unreachable(ctx):
    t = _T([-1, 0, 0, -1, 3])
    for method in METHODS:
        got, _ = run(ctx, t, method, False, 0, host=True)
        assert got.tolist() == [3, 1, 1, 0, 0]
        got, _ = run(ctx, t, method, True, 3, host=True)
        assert got.tolist() == [0, 0, 0, 2, 1]
    with pytest.raises(RuntimeError):  # the flat template needs parent[]
        T = inl.Csr(dev(t.row_ptr), dev(t.col_idx), 5)
        inl.tree_descendants(ctx, T, None, torch.zeros(5, dtype=torch.int64, device="cuda"), 0, inl.TREE_FLAT)
