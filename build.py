#!/usr/bin/env python3
"""Build every native artefact in-tree.

  paper_conf_sc_dastgeerlk12_b200/libpepp_spmv.so   CUDA C-ABI library (nvcc, sm_100a)
  gen/libpepp_gen.so                                input generator (gcc)
  oracle/liboracle.so                               CPU oracle (gcc, test infrastructure)

nvcc cross-compiles for sm_100a without a GPU, so this runs on the CPU box.
Usage: python build.py [--force] [--verbose]   (-Xptxas -v with --verbose)
"""
from __future__ import annotations

import argparse
import os
import shutil
import subprocess
import sys

ROOT = os.path.dirname(os.path.abspath(__file__))
PKG = os.path.join(ROOT, "paper_conf_sc_dastgeerlk12_b200")
CSRC = os.path.join(PKG, "csrc")
LIB = os.path.join(PKG, "libpepp_spmv.so")
SOURCES = ["plan.cu", "containers.cu", "host_util.cpp", "nccl_dl.cpp"]
HEADERS = ["kernels.cuh", "pepp_internal.h"]
ARCH = ["-gencode", "arch=compute_100a,code=sm_100a"]


def _nvcc() -> str:
    for c in (os.environ.get("NVCC"), "/usr/local/cuda/bin/nvcc", shutil.which("nvcc")):
        if c and os.path.exists(c):
            return c
    raise RuntimeError("nvcc not found")


def _stale(target: str, deps: list[str]) -> bool:
    if not os.path.exists(target):
        return True
    t = os.path.getmtime(target)
    return any(os.path.getmtime(d) > t for d in deps)


def build_cuda(force: bool = False, verbose: bool = False) -> str:
    deps = [os.path.join(CSRC, s) for s in SOURCES + HEADERS] + [os.path.join(ROOT, "include", "pepp_spmv.h"), __file__]
    if not force and not _stale(LIB, deps):
        return LIB
    nvcc = _nvcc()
    objdir = os.path.join(ROOT, "build", "obj")
    os.makedirs(objdir, exist_ok=True)
    common = ["-O3", "-std=c++17", "-lineinfo", *ARCH, "-I", os.path.join(ROOT, "include"), "-I", CSRC,
              "-Xcompiler", "-fPIC,-fvisibility=hidden,-Wall", "--expt-relaxed-constexpr"]
    if verbose:
        common += ["-Xptxas", "-v"]
    common += os.environ.get("PEPP_NVCC_EXTRA", "").split()   # experiments only (e.g. -DPEPP_PAT_U=4)
    objs = []
    for s in SOURCES:
        src = os.path.join(CSRC, s)
        obj = os.path.join(objdir, os.path.splitext(s)[0] + ".o")
        lang = [] if s.endswith(".cu") else ["-x", "cu"] if False else []
        subprocess.check_call([nvcc, *common, *lang, "-c", src, "-o", obj])
        objs.append(obj)
    tmp = LIB + ".tmp"
    subprocess.check_call([nvcc, *ARCH, "-shared", "-cudart=static", "-o", tmp, *objs, "-ldl", "-lpthread", "-lrt"])
    os.replace(tmp, LIB)
    return LIB


def build_all(force: bool = False, verbose: bool = False) -> None:
    sys.path.insert(0, ROOT)
    import gen
    import oracle
    gen.build(force)
    oracle.build(force)
    build_cuda(force, verbose)


if __name__ == "__main__":
    ap = argparse.ArgumentParser()
    ap.add_argument("--force", action="store_true")
    ap.add_argument("--verbose", action="store_true")
    a = ap.parse_args()
    build_all(a.force, a.verbose)
    print("built:", LIB)
