"""CPU-only checks of the C-ABI boundary: libinl.so loads, exports every entry point
declared in include/inl.h, and its host-only logic (row partition, status strings,
argument errors) behaves as documented.  No compute calls (no GPU here)."""
import ctypes as C
import os
import re
import subprocess

import numpy as np
import pytest

from conftest import ROOT, cuda_ok
from paper_conf_icpp_liwb15_b200 import inl


def _declared(header):
    txt = open(os.path.join(ROOT, "include", header)).read()
    txt = re.sub(r"/\*.*?\*/", "", txt, flags=re.S)
    return sorted(set(re.findall(r"\b((?:inl|inlgen)_[a-z0-9_]+)\s*\(", txt)))


def test_header_symbols_exported():
    names = _declared("inl.h")
    assert "inl_spmv" in names and "inl_sssp" in names and "inl_pagerank" in names and "inl_bfs" in names
    L = inl.lib()
    for n in names:
        assert hasattr(L, n), f"{n} declared in include/inl.h but not exported"
    out = subprocess.check_output(["nm", "-D", "--defined-only", inl.LIB_PATH], text=True)
    for n in names:
        assert re.search(rf"\bT {n}\b", out), n


def test_inlgen_symbols_exported():
    import inlgen
    for n in _declared("inlgen.h"):
        assert hasattr(inlgen.lib(), n), n


def test_library_is_sm100a_and_has_no_oracle_link():
    out = subprocess.check_output(["cuobjdump", "--list-elf", inl.LIB_PATH], text=True)
    assert "sm_100a" in out
    deps = subprocess.check_output(["ldd", inl.LIB_PATH], text=True)
    assert "liborc" not in deps
    strings = subprocess.check_output(["strings", inl.LIB_PATH], text=True)
    assert "orc_spmv" not in strings


def test_version_and_status_strings():
    assert "sm_100a" in inl.version()
    L = inl.lib()
    for code, name in inl.STATUS.items():
        assert L.inl_status_string(code).decode() == name


@pytest.mark.parametrize("n,p", [(0, 1), (1, 1), (10, 3), (4096, 8), (4095, 8), (7, 8), (1 << 22, 8)])
def test_partition_rows(n, p):
    b = inl.partition_rows(n, p)
    B = -(-n // p)
    assert b[0] == 0 and b[-1] == n and len(b) == p + 1
    assert all(b[i] <= b[i + 1] for i in range(p))
    assert all(b[i + 1] - b[i] == B for i in range(p) if b[i + 1] < n)
    assert b == [min(i * B, n) for i in range(p + 1)]


def test_partition_rows_rejects_bad_args():
    with pytest.raises(inl.InlError):
        inl.partition_rows(10, 0)
    with pytest.raises(inl.InlError):
        inl.partition_rows(-1, 2)


def test_null_ctx_is_invalid_argument():
    L = inl.lib()
    s = inl.CsrT(0, 0, 0, 0, None, None)
    assert L.inl_spmv(None, C.byref(s), None, None, None, None) == 1
    assert L.inl_bfs(None, C.byref(s), 0, None, None, None) == 1
    assert L.inl_ctx_create(None, 0, None) == 1


@pytest.mark.skipif(cuda_ok(), reason="checks the no-GPU error path")
def test_ctx_create_without_gpu_reports_cuda_error():
    h = C.c_void_p()
    assert inl.lib().inl_ctx_create(C.byref(h), 0, None) == 3  # INL_ERR_CUDA
    assert "cuda" in inl.lib().inl_last_error(None).decode().lower()


def test_loop_group_host_object():
    """The loopback communicator's host object needs no GPU: create / destroy / bad sizes."""
    L = inl.lib()
    for p in (1, 2, 8, 64):
        g = inl.LoopGroup(p)
        assert g.nranks == p
        g.close()
    h = C.c_void_p()
    assert L.inl_loop_create(0, C.byref(h)) == 1
    assert L.inl_loop_create(65, C.byref(h)) == 1
    assert L.inl_loop_destroy(None) == 0
    s = inl.CsrT(0, 0, 0, 0, None, None)
    assert L.inl_spmv_allgather(None, C.byref(s), None, None, None, None) == 1
    assert L.inl_comm_init_loopback(None, None, 0) == 1
