"""Build libpt.so in-tree with nvcc for sm_100a (no JIT cache, no torch extension).

Each translation unit is compiled to an object in parallel (the tracking kernel's
instantiations are split by fibre count and precision into pt_track_f<F>_<f32|f16>.cu), then
linked."""
from __future__ import annotations

import os
import shutil
import subprocess
from concurrent.futures import ThreadPoolExecutor

PKG = os.path.dirname(os.path.abspath(__file__))
ROOT = os.path.dirname(PKG)
CSRC = os.path.join(PKG, "csrc")
INCLUDE = os.path.join(ROOT, "include")
LIB = os.environ.get("PT_LIB") or os.path.join(PKG, "libpt.so")  # PT_LIB: experiment builds
OBJDIR = os.path.join(PKG, "build")
SOURCES = ["pt_api.cu", "pt_kernels.cu", "pt_mcmc.cu", "pt_segmented.cu"] + \
    [f"pt_track_f{F}_{p}.cu" for F in (1, 2, 3) for p in ("f32", "f16")]
HEADERS = ["pt_device.cuh", "pt_internal.h", "pt_claim.cuh", "pt_track.cuh"]

ARCH = ["-gencode", "arch=compute_100a,code=sm_100a"]
NVCC_FLAGS = [
    *ARCH,
    "-O3", "-lineinfo", "-std=c++17",
    "-fmad=false",          # no FMA contraction anywhere in the library (R15)
    "-Xcompiler", "-fPIC",
    "-Xptxas", "-warn-spills", "-diag-suppress", "186",
]


def nvcc() -> str:
    for cand in (os.environ.get("NVCC"), shutil.which("nvcc"), "/usr/local/cuda/bin/nvcc"):
        if cand and os.path.exists(cand):
            return cand
    raise RuntimeError("nvcc not found: cannot build libpt.so")


def _inputs():
    files = [os.path.join(CSRC, s) for s in SOURCES + HEADERS]
    files.append(os.path.join(INCLUDE, "pt.h"))
    files.append(os.path.abspath(__file__))
    return files


def stale() -> bool:
    if not os.path.exists(LIB):
        return True
    t = os.path.getmtime(LIB)
    return any(os.path.getmtime(f) > t for f in _inputs())


def build(force: bool = False, verbose: bool = False) -> str:
    if not force and not stale():
        return LIB
    extra = os.environ.get("PT_NVCC_EXTRA", "").split()  # experiment builds: -D overrides
    tag = f"{os.getpid()}"
    os.makedirs(OBJDIR, exist_ok=True)
    objs = [os.path.join(OBJDIR, os.path.splitext(s)[0] + f".{tag}.o") for s in SOURCES]
    cmds = [[nvcc(), *NVCC_FLAGS, *extra, "-I", INCLUDE, "-c", "-o", o, os.path.join(CSRC, s)]
            for s, o in zip(SOURCES, objs)]
    if verbose:
        for c in cmds:
            print(" ".join(c))
    try:
        with ThreadPoolExecutor(max_workers=len(cmds)) as ex:
            for f in [ex.submit(subprocess.check_call, c) for c in cmds]:
                f.result()
        tmp = LIB + f".tmp{tag}"
        link = [nvcc(), *ARCH, "-shared", "-o", tmp, *objs]
        if verbose:
            print(" ".join(link))
        subprocess.check_call(link)
        os.replace(tmp, LIB)
    finally:
        for o in objs:
            if os.path.exists(o):
                os.remove(o)
    return LIB


if __name__ == "__main__":
    print(build(force=True, verbose=True))
