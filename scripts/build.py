"""Build every native artefact in-tree (no GPU needed; nvcc cross-compiles sm_100a).

  oracle/liborc.so                          plain C oracle (gcc, no fast-math, no FMA contraction)
  inlgen/libinlgen.so                       seeded input generator (host C++ + CUDA twin)
  paper_conf_icpp_liwb15_b200/libinl.so     the product: C-ABI + sm_100a kernels + NCCL

Usage: python scripts/build.py [--force] [--only oracle|inlgen|inl]
"""
from __future__ import annotations

import argparse
import glob
import os
import shutil
import subprocess
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
NVCC = os.environ.get("NVCC", shutil.which("nvcc") or "/usr/local/cuda/bin/nvcc")
ARCH = ["-gencode", "arch=compute_100a,code=sm_100a"]
NVCC_COMMON = ARCH + ["-O3", "-lineinfo", "-std=c++17", "-Xcompiler", "-fPIC",
                      "-Xcompiler", "-Wall", "--expt-relaxed-constexpr"]


def _nccl_dir() -> str:
    import importlib.util
    spec = importlib.util.find_spec("nvidia")
    cands = []
    if spec and spec.submodule_search_locations:
        for p in spec.submodule_search_locations:
            cands.append(os.path.join(p, "nccl"))
    for c in cands:
        if os.path.exists(os.path.join(c, "include", "nccl.h")):
            return c
    raise RuntimeError("nccl.h not found (expected the torch wheel's nvidia/nccl)")


def _stale(out: str, srcs: list[str]) -> bool:
    if not os.path.exists(out):
        return True
    t = os.path.getmtime(out)
    return any(os.path.getmtime(s) > t for s in srcs)


def _run(cmd: list[str]) -> None:
    print("+", " ".join(cmd), flush=True)
    subprocess.check_call(cmd, cwd=ROOT)


def build_oracle(force: bool = False) -> str:
    out = os.path.join(ROOT, "oracle", "liborc.so")
    srcs = [os.path.join(ROOT, "oracle", f) for f in ("orc.c", "orc.h")]
    if force or _stale(out, srcs):
        _run(["gcc", "-O2", "-std=c99", "-fPIC", "-shared", "-ffp-contract=off", "-fno-fast-math",
              "-Wall", "-o", out, srcs[0]])
    return out


def build_oracle_par(force: bool = False) -> str:
    """The OpenMP "CPU-parallel" context line (oracle/orc_par.c; bench cpu_baseline only)."""
    out = os.path.join(ROOT, "oracle", "liborc_par.so")
    src = os.path.join(ROOT, "oracle", "orc_par.c")
    if force or _stale(out, [src]):
        _run(["gcc", "-O2", "-std=c99", "-fPIC", "-shared", "-fopenmp", "-ffp-contract=off", "-fno-fast-math",
              "-Wall", "-o", out, src])
    return out


def build_inlgen(force: bool = False) -> str:
    out = os.path.join(ROOT, "inlgen", "libinlgen.so")
    d = os.path.join(ROOT, "inlgen")
    srcs = [os.path.join(d, f) for f in ("gen_host.cpp", "gen_dev.cu", "loader.cpp")]
    deps = srcs + glob.glob(os.path.join(d, "*.h")) + [os.path.join(ROOT, "include", "inlgen.h")]
    if force or _stale(out, deps):
        _run([NVCC] + NVCC_COMMON + ["-I", os.path.join(ROOT, "include"), "-shared", "-o", out] + srcs)
    return out


def build_inl(force: bool = False, defines: list[str] | None = None, out: str | None = None) -> str:
    """defines/out: an experiment variant (-D flags) written to another path (A/B runs
    select it with INL_LIB=<path>); the product build uses neither."""
    pkg = os.path.join(ROOT, "paper_conf_icpp_liwb15_b200")
    out = out or os.path.join(pkg, "libinl.so")
    csrc = os.path.join(pkg, "csrc")
    srcs = sorted(glob.glob(os.path.join(csrc, "*.cu")) + glob.glob(os.path.join(csrc, "*.cpp")))
    deps = srcs + glob.glob(os.path.join(csrc, "*.cuh")) + glob.glob(os.path.join(csrc, "*.h")) + \
        [os.path.join(ROOT, "include", "inl.h")]
    if not srcs:
        raise RuntimeError("no sources under " + csrc)
    if force or _stale(out, deps):
        nccl = _nccl_dir()
        os.makedirs(os.path.dirname(out), exist_ok=True)
        _run([NVCC] + NVCC_COMMON + ["-D" + d for d in (defines or [])] +
             ["-Xptxas", "-v" if os.environ.get("INL_PTXAS_V") else "-O3",
                                     "-I", os.path.join(nccl, "include"), "-I", os.path.join(ROOT, "include"),
                                     "-shared", "-o", out] + srcs +
             ["-L", os.path.join(nccl, "lib"), "-l:libnccl.so.2",
              "-Xlinker", "-rpath=" + os.path.join(nccl, "lib")])
    return out


def build_all(force: bool = False, only: str | None = None) -> list[str]:
    outs = []
    if only in (None, "oracle"):
        outs.append(build_oracle(force))
        outs.append(build_oracle_par(force))
    if only in (None, "inlgen"):
        outs.append(build_inlgen(force))
    if only in (None, "inl"):
        outs.append(build_inl(force))
    return outs


if __name__ == "__main__":
    ap = argparse.ArgumentParser()
    ap.add_argument("--force", action="store_true")
    ap.add_argument("--only", choices=["oracle", "inlgen", "inl"])
    ap.add_argument("--variant", nargs="+", metavar="NAME [DEFINE ...]",
                    help="build an experiment variant build/variants/libinl_NAME.so with -D DEFINEs")
    a = ap.parse_args()
    if a.variant:
        o = build_inl(True, a.variant[1:], os.path.join(ROOT, "build", "variants", f"libinl_{a.variant[0]}.so"))
        print("built", o)
        sys.exit(0)
    for o in build_all(a.force, a.only):
        print("built", o)
    sys.exit(0)
