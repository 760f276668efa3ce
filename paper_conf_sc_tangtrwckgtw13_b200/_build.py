"""Build libbro.so in-tree with nvcc for sm_100a (no torch JIT, no cache dir).

The library is a plain C-ABI shared object (include/bro.h) linked against the
static CUDA runtime, so it loads next to PyTorch's own runtime and accepts
torch's cudaStream_t handles as-is.
"""
from __future__ import annotations

import os
import shutil
import subprocess
import sys

PKG = os.path.dirname(os.path.abspath(__file__))
ROOT = os.path.dirname(PKG)
CSRC = os.path.join(PKG, "csrc")
LIB = os.path.join(PKG, "libbro.so")
SOURCES = ["capi.cu", "kern_ell64.cu", "kern_ell32.cu", "kern_ell64_vi.cu", "kern_ell32_vi.cu", "kern_misc.cu",
           "encode.cpp"]
HEADERS = ["kernels.cuh", "kern_ell.cuh", "launch.hpp", "encode.hpp", os.path.join("..", "..", "include", "bro.h")]
OBJDIR = os.path.join(CSRC, "build")

ARCH = ["-gencode", "arch=compute_100a,code=sm_100a"]
CFLAGS = ["-O3", "-std=c++17", "-lineinfo", "-Xcompiler", "-fPIC,-pthread,-O3", "-Xptxas", "-v",
          "--expt-relaxed-constexpr"]
LFLAGS = ["-shared", "-cudart", "static", "-Xcompiler", "-pthread"]


def nvcc() -> str:
    for p in (os.environ.get("NVCC"), "/usr/local/cuda/bin/nvcc", shutil.which("nvcc")):
        if p and os.path.exists(p):
            return p
    raise RuntimeError("nvcc not found")


def _stale() -> bool:
    if not os.path.exists(LIB):
        return True
    t = os.path.getmtime(LIB)
    for f in SOURCES + HEADERS + ["../_build.py"]:
        if os.path.getmtime(os.path.join(CSRC, f)) > t:
            return True
    return False


def build(force: bool = False, verbose: bool = False) -> str:
    """Compile every translation unit for sm_100a in parallel (-lineinfo,
    ptxas -v into csrc/ptxas.log), then link libbro.so with the static CUDA
    runtime."""
    if not force and not _stale():
        return LIB
    os.makedirs(OBJDIR, exist_ok=True)
    procs = []
    for src in SOURCES:
        obj = os.path.join(OBJDIR, os.path.splitext(src)[0] + ".o")
        cmd = [nvcc(), *ARCH, *CFLAGS, "-I", os.path.join(ROOT, "include"), "-c", "-o", obj,
               os.path.join(CSRC, src)]
        procs.append((src, obj, subprocess.Popen(cmd, stdout=subprocess.PIPE, stderr=subprocess.PIPE,
                                                 text=True)))
    logs, objs, failed = [], [], []
    for src, obj, pr in procs:
        out, err = pr.communicate()
        logs.append(f"==== {src}\n{out}{err}")
        objs.append(obj)
        if pr.returncode != 0:
            failed.append(src)
            sys.stderr.write(out + err)
    if failed:
        raise RuntimeError(f"nvcc failed building {failed}")
    r = subprocess.run([nvcc(), *ARCH, *LFLAGS, "-o", LIB + ".tmp", *objs], capture_output=True, text=True)
    if r.returncode != 0:
        sys.stderr.write(r.stdout + r.stderr)
        raise RuntimeError("nvcc failed linking libbro.so")
    with open(os.path.join(CSRC, "ptxas.log"), "w") as f:
        f.write("\n".join(logs))
    if verbose:
        sys.stderr.write("\n".join(logs))
    os.replace(LIB + ".tmp", LIB)
    return LIB


if __name__ == "__main__":
    build(force="--force" in sys.argv, verbose=True)
    print(LIB)
