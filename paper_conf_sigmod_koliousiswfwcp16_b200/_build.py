"""In-tree build of the CUDA libraries (sm_100a), no torch JIT cache.

* ``libsaber.so``      -- the product: kernels.cu + runtime.cu behind include/saber.h
* ``saber_inputs/libsaber_gen.so`` -- the device twin of the input generator

nvcc cross-compiles for sm_100a without a GPU, so this runs on the CPU box.
"""
from __future__ import annotations

import os
import subprocess

PKG = os.path.dirname(os.path.abspath(__file__))
ROOT = os.path.dirname(PKG)
CSRC = os.path.join(PKG, "csrc")
LIB = os.path.join(PKG, "libsaber.so")
GEN_SRC = os.path.join(ROOT, "saber_inputs", "csrc", "gen.cu")
GEN_LIB = os.path.join(ROOT, "saber_inputs", "libsaber_gen.so")

NVCC = os.environ.get("NVCC", "/usr/local/cuda/bin/nvcc")
ARCH = ["-gencode", "arch=compute_100a,code=sm_100a"]
FLAGS = ["-O3", "-lineinfo", "-std=c++17", "-Xcompiler", "-fPIC", "-shared", "--expt-relaxed-constexpr",
         "-diag-suppress", "550"]


def _stale(out, srcs):
    if not os.path.exists(out):
        return True
    t = os.path.getmtime(out)
    return any(os.path.getmtime(s) > t for s in srcs)


def _sources():
    srcs = [os.path.join(CSRC, f) for f in sorted(os.listdir(CSRC))
            if f.endswith((".cu", ".cuh", ".h"))]
    srcs.append(os.path.join(ROOT, "include", "saber.h"))
    return srcs


def build(force: bool = False, verbose: bool = False) -> str:
    srcs = _sources()
    if force or _stale(LIB, srcs):
        cus = [f for f in sorted(os.listdir(CSRC)) if f.endswith(".cu")]
        objdir = os.path.join(CSRC, "..", "build")
        os.makedirs(objdir, exist_ok=True)
        objs, procs = [], []
        hdrs = [x for x in srcs if not x.endswith(".cu")]
        for f in cus:     # one nvcc per stale translation unit, in parallel
            o = os.path.join(objdir, f[:-3] + ".o")
            objs.append(o)
            if not force and not _stale(o, [os.path.join(CSRC, f), *hdrs]):
                continue
            cmd = [NVCC, *ARCH, *[x for x in FLAGS if x != "-shared"], "-c", "-I", os.path.join(ROOT, "include"),
                   os.path.join(CSRC, f), "-o", o]
            if verbose:
                print(" ".join(cmd))
            procs.append((f, subprocess.Popen(cmd)))
        for f, pr in procs:
            if pr.wait() != 0:
                raise RuntimeError(f"nvcc failed on {f}")
        subprocess.check_call([NVCC, *ARCH, "-shared", *objs, "-o", LIB + ".tmp"])
        os.replace(LIB + ".tmp", LIB)
    if force or _stale(GEN_LIB, [GEN_SRC]):
        cmd = [NVCC, *ARCH, *FLAGS, GEN_SRC, "-o", GEN_LIB + ".tmp"]
        subprocess.check_call(cmd)
        os.replace(GEN_LIB + ".tmp", GEN_LIB)
    return LIB


if __name__ == "__main__":
    build(force=True, verbose=True)
    print(LIB)
