#!/usr/bin/env python3
"""Build libwinrs.so (sm_100a) in-tree with nvcc, compiling translation units
in parallel.  Also regenerates the Winograd transform header when the
generator is newer.  Usage: python tools/build.py [--force] [-j N]"""
from __future__ import annotations

import argparse
import concurrent.futures as cf
import os
import subprocess
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
PKG = os.path.join(ROOT, "paper_conf_icpp_zhangc0zx0025_b200")
CSRC = os.path.join(PKG, "csrc")
OBJ = os.path.join(ROOT, "build", "obj")
LIB = os.path.join(PKG, "libwinrs.so")
GEN = os.path.join(ROOT, "tools", "gen_winograd.py")
GEN_OUT = os.path.join(CSRC, "winograd_generated.cuh")

NVCC = os.environ.get("NVCC", "/usr/local/cuda/bin/nvcc")
ARCH = ["-gencode", "arch=compute_100a,code=sm_100a"]
FLAGS = ["-O3", "-std=c++17", "-lineinfo", "--expt-relaxed-constexpr", "-Xcompiler", "-fPIC", "-Xcompiler", "-fvisibility=hidden",
         "-I", os.path.join(ROOT, "include")]

SOURCES = ["winrs_api.cpp", "planner.cpp", "registry.cpp", "reduce.cu", "allreduce.cu", "bfc_f16.cu", "bfc_tc2.cu", "bfc_tc2x.cu", "bfc_tc3.cu", "conv_map.cu",
           "bfc_f32_part0.cu", "bfc_f32_part1.cu", "bfc_f32_part2.cu", "bfc_f32_part3.cu",
           "bfc_f32_part4.cu", "bfc_f32_part5.cu"]


def _deps_mtime() -> float:
    m = 0.0
    for f in os.listdir(CSRC):
        if f.endswith((".h", ".cuh")):
            m = max(m, os.path.getmtime(os.path.join(CSRC, f)))
    m = max(m, os.path.getmtime(os.path.join(ROOT, "include", "winrs.h")))
    return m


def _compile(src: str, force: bool, hdr_m: float) -> str:
    s = os.path.join(CSRC, src)
    o = os.path.join(OBJ, src + ".o")
    if not force and os.path.exists(o) and os.path.getmtime(o) >= max(os.path.getmtime(s), hdr_m):
        return o
    cmd = [NVCC, *ARCH, *FLAGS, "-c", s, "-o", o]
    if src.endswith(".cpp"):
        cmd = [NVCC, *ARCH, *FLAGS, "-x", "cu", "-c", s, "-o", o]
    r = subprocess.run(cmd, capture_output=True, text=True)
    if r.returncode != 0:
        raise RuntimeError(f"nvcc failed for {src}:\n{r.stdout}\n{r.stderr}")
    return o


def build(force: bool = False, jobs: int = 0, trace: bool = False, extra=(), variant: str = "") -> str:
    global OBJ, LIB, FLAGS
    if variant:   # A/B build with extra -D knobs: libwinrs_<variant>.so (select with WINRS_LIB)
        OBJ = os.path.join(ROOT, "build", "obj_" + variant)
        LIB = os.path.join(PKG, "libwinrs_%s.so" % variant)
        FLAGS = FLAGS + ["-D" + e for e in extra]
    elif trace:   # debug build with the CTA-0 timeline (csrc/bfc_f16.cuh TRACE)
        OBJ = os.path.join(ROOT, "build", "obj_trace" + "".join(extra))
        LIB = os.path.join(PKG, "libwinrs_trace%s.so" % "".join(extra))
        FLAGS = FLAGS + ["-DWINRS_TRACE"] + ["-D" + e for e in extra]
    os.makedirs(OBJ, exist_ok=True)
    if not os.path.exists(GEN_OUT) or os.path.getmtime(GEN_OUT) < os.path.getmtime(GEN):
        subprocess.check_call([sys.executable, GEN])
    hdr_m = _deps_mtime()
    jobs = jobs or min(len(SOURCES), os.cpu_count() or 4)
    with cf.ThreadPoolExecutor(jobs) as ex:
        objs = list(ex.map(lambda s: _compile(s, force, hdr_m), SOURCES))
    if force or not os.path.exists(LIB) or os.path.getmtime(LIB) < max(os.path.getmtime(o) for o in objs):
        cmd = [NVCC, *ARCH, "-shared", "-cudart", "static", "-o", LIB, *objs, "-Xcompiler", "-fPIC"]
        r = subprocess.run(cmd, capture_output=True, text=True)
        if r.returncode != 0:
            raise RuntimeError(f"link failed:\n{r.stdout}\n{r.stderr}")
    return LIB


if __name__ == "__main__":
    ap = argparse.ArgumentParser()
    ap.add_argument("--force", action="store_true")
    ap.add_argument("-j", type=int, default=0)
    ap.add_argument("--trace", action="store_true")
    ap.add_argument("--define", action="append", default=[])
    ap.add_argument("--variant", default="")
    a = ap.parse_args()
    print(build(a.force, a.j, a.trace, tuple(a.define), a.variant))
