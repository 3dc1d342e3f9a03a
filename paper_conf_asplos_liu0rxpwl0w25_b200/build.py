"""Build libcomet.so in-tree (nvcc for sm_100a, g++ for host code).  Run: python -m
paper_conf_asplos_liu0rxpwl0w25_b200.build [--force]"""
from __future__ import annotations

import os
import subprocess
import sys
from concurrent.futures import ThreadPoolExecutor

PKG = os.path.dirname(os.path.abspath(__file__))
ROOT = os.path.dirname(PKG)
CSRC = os.path.join(PKG, "csrc")
BUILD = os.path.join(PKG, "build")
LIB = os.path.join(PKG, "lib", "libcomet.so")
NVCC = os.environ.get("NVCC", "/usr/local/cuda/bin/nvcc")
ARCH = ["-gencode", "arch=compute_100a,code=sm_100a"]
CU_SOURCES = ["quantize.cu", "kv4.cu", "gemm.cu", "gemm_n.cu", "gemm_v.cu", "api.cu"]
CPP_SOURCES = ["planner.cpp", "calibrate.cpp"]
HEADERS = ["internal.h", "sm100.cuh", "gemm_common.cuh", "fmpq.cuh"]


def _newer(src_paths, dst):
    if not os.path.exists(dst):
        return True
    t = os.path.getmtime(dst)
    return any(os.path.getmtime(s) > t for s in src_paths)


def _run(cmd):
    r = subprocess.run(cmd, capture_output=True, text=True)
    if r.returncode != 0:
        raise RuntimeError("build failed:\n" + " ".join(cmd) + "\n" + r.stdout + r.stderr)
    return r.stdout + r.stderr


def build(force: bool = False, verbose: bool = False) -> str:
    """COMET_DIAG=1 in the environment builds the diagnostic variant (timeline trace and
    stage-ablation hooks, tools/trace_gemm.py); normal builds compile them out.  Switching
    between the two needs force=True.  COMET_NVCC_DEFS="-DNAME=V ..." adds defines (kernel
    variant experiments only)."""
    os.makedirs(BUILD, exist_ok=True)
    os.makedirs(os.path.dirname(LIB), exist_ok=True)
    hdrs = [os.path.join(CSRC, h) for h in HEADERS] + [os.path.join(ROOT, "include", "comet.h")]
    jobs, objs = [], []
    for s in CU_SOURCES:
        src = os.path.join(CSRC, s)
        obj = os.path.join(BUILD, s + ".o")
        objs.append(obj)
        if force or _newer([src] + hdrs, obj):
            jobs.append([NVCC, *ARCH, "-O3", "-std=c++17", "-lineinfo", "-Xptxas", "-v",
                         f"-DCOMET_DIAG={1 if os.environ.get('COMET_DIAG') == '1' else 0}",
                         *os.environ.get("COMET_NVCC_DEFS", "").split(),
                         "-Xcompiler", "-fPIC", "-I", CSRC, "-I", os.path.join(ROOT, "include"),
                         "-c", src, "-o", obj])
    for s in CPP_SOURCES:
        src = os.path.join(CSRC, s)
        obj = os.path.join(BUILD, s + ".o")
        objs.append(obj)
        if force or _newer([src] + hdrs, obj):
            jobs.append(["g++", "-O2", "-std=c++17", "-fPIC", "-I", CSRC, "-I",
                         os.path.join(ROOT, "include"), "-I", "/usr/local/cuda/include", "-c", src,
                         "-o", obj])
    with ThreadPoolExecutor(max_workers=max(1, min(len(jobs), os.cpu_count() or 4))) as ex:
        outs = list(ex.map(_run, jobs))
    if verbose:
        for o in outs:
            sys.stdout.write(o)
    if force or jobs or _newer(objs, LIB):
        tmp = LIB + ".tmp"
        _run([NVCC, *ARCH, "-shared", "-cudart", "static", "-o", tmp, *objs])
        os.replace(tmp, LIB)
    return LIB


if __name__ == "__main__":
    print(build(force="--force" in sys.argv, verbose="-v" in sys.argv))
