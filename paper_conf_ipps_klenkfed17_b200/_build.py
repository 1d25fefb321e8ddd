"""Builds the in-tree C-ABI library lib/libmm.so with nvcc for sm_100a."""
from __future__ import annotations

import glob
import os
import subprocess

PKG = os.path.dirname(os.path.abspath(__file__))
CSRC = os.path.join(PKG, "csrc")
LIBDIR = os.path.join(PKG, "lib")
LIB = os.path.join(LIBDIR, "libmm.so")
ROOT = os.path.dirname(PKG)
INCLUDE = os.path.join(ROOT, "include")

NVCC_FLAGS = [
    "-gencode", "arch=compute_100a,code=sm_100a",
    "-O3", "-lineinfo", "-std=c++17",
    "-Xcompiler", "-fPIC", "-shared",
]


def sources():
    return sorted(glob.glob(os.path.join(CSRC, "*.cu")))


def _inputs():
    return sources() + glob.glob(os.path.join(CSRC, "*.h")) + glob.glob(os.path.join(CSRC, "*.cuh")) + \
        [os.path.join(INCLUDE, "mm.h")]


def stale():
    if not os.path.exists(LIB):
        return True
    t = os.path.getmtime(LIB)
    return any(os.path.getmtime(f) > t for f in _inputs())


def build_library(force=False, verbose=False, variant=""):
    """Compile every csrc/*.cu into lib/libmm.so (sm_100a, -lineinfo).
    variant="timing" builds lib/libmm_timing.so with -DMM_PHASE_TIMING
    (per-phase clock64 accounting, a profiling aid only)."""
    lib = LIB if not variant else os.path.join(LIBDIR, "libmm_%s.so" % variant)
    if not force and not variant and not stale():
        return LIB
    os.makedirs(LIBDIR, exist_ok=True)
    nvcc = os.environ.get("NVCC", "nvcc")
    tmp = lib + ".tmp%d" % os.getpid()
    extra = ["-DMM_PHASE_TIMING"] if variant == "timing" else []
    if variant and variant != "timing":  # A/B builds: -D flags from MM_AB_DEFINES (profiling aid)
        extra = ["-D" + d for d in os.environ.get("MM_AB_DEFINES", "").split()]
        extra += os.environ.get("MM_AB_FLAGS", "").split()  # raw nvcc flags of an A/B build
    cmd = [nvcc, *NVCC_FLAGS, *extra, "-Xptxas", "-v", "-o", tmp, *sources()]
    res = subprocess.run(cmd, capture_output=True, text=True)
    with open(os.path.join(LIBDIR, "ptxas%s.log" % ("_" + variant if variant else "")), "w") as f:
        f.write(" ".join(cmd) + "\n" + res.stdout + res.stderr)
    if res.returncode != 0:
        raise RuntimeError("nvcc failed:\n" + res.stderr[-4000:])
    os.replace(tmp, lib)
    if verbose:
        print("built", lib)
    return lib
