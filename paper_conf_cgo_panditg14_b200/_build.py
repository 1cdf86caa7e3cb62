"""Build libfcl.so in-tree: nvcc for the sm_100a kernels, g++ for the host runtime.

The host work-group bodies are compiled with -ffp-contract=off (explicit fmaf only) so they
reproduce the GPU bodies' IEEE operation sequence bit for bit.  CUDA's runtime
is linked statically, so loading the library needs no CUDA installation (the C-ABI symbol
test runs on CPU-only machines); running it needs the NVIDIA driver.
"""
from __future__ import annotations

import os
import shutil
import subprocess
import sys

HERE = os.path.dirname(os.path.abspath(__file__))
CSRC = os.path.join(HERE, "csrc")
ROOT = os.path.dirname(HERE)
INCLUDE = os.path.join(ROOT, "include")
LIB = os.path.join(HERE, "libfcl.so")
BUILD = os.path.join(HERE, "build")

CUDA_HOME = os.environ.get("CUDA_HOME", "/usr/local/cuda")
NVCC = os.path.join(CUDA_HOME, "bin", "nvcc")
ARCH = ["-gencode", "arch=compute_100a,code=sm_100a"]

SOURCES = {
    "kernels.o": ("kernels.cu", "nvcc"),
    "host_bodies.o": ("host_bodies.cpp", "host_fp"),
    "runtime.o": ("runtime.cpp", "host"),
}


def _cmd(obj: str, src: str, kind: str):
    out = os.path.join(BUILD, obj)
    srcp = os.path.join(CSRC, src)
    if kind == "nvcc":
        return [NVCC, *ARCH, "-O3", "-lineinfo", "-std=c++17", "-Xcompiler", "-fPIC", "-Xptxas", "-v",
                "-I", INCLUDE, *os.environ.get("FCL_NVCC_EXTRA", "").split(), "-c", srcp, "-o", out]
    common = ["g++", "-std=c++17", "-fPIC", "-Wall", "-Wno-unused-function", "-I", INCLUDE,
              "-I", os.path.join(CUDA_HOME, "include"), "-c", srcp, "-o", out]
    if kind == "host_fp":
        # x86-64-v3 (AVX2 + FMA): present on every B200 host we run on; no fast-math, no contraction
        return common + ["-O3", "-march=x86-64-v3", "-ffp-contract=off", "-fno-fast-math"]
    return common + ["-O2", "-pthread"]


def _stale(outs, ins) -> bool:
    if not all(os.path.exists(o) for o in outs):
        return True
    t = min(os.path.getmtime(o) for o in outs)
    return any(os.path.getmtime(i) > t for i in ins)


def build(force: bool = False, verbose: bool = False) -> str:
    os.makedirs(BUILD, exist_ok=True)
    headers = [os.path.join(CSRC, "fcl_internal.h"), os.path.join(INCLUDE, "fcl.h")]
    objs = []
    for obj, (src, kind) in SOURCES.items():
        out = os.path.join(BUILD, obj)
        objs.append(out)
        if force or _stale([out], [os.path.join(CSRC, src), *headers, __file__]):
            cmd = _cmd(obj, src, kind)
            if verbose:
                print(" ".join(cmd), file=sys.stderr)
            r = subprocess.run(cmd, capture_output=True, text=True)
            if r.returncode != 0:
                raise RuntimeError(f"compile of {src} failed:\n{r.stdout}\n{r.stderr}")
            if kind == "nvcc":
                with open(os.path.join(BUILD, "ptxas.log"), "w") as f:
                    f.write(r.stderr)
    if force or _stale([LIB], objs):
        cmd = [NVCC, *ARCH, "-shared", "-Xcompiler", "-fPIC", "-cudart", "static", "-o", LIB, *objs,
               "-lpthread", "-ldl", "-lrt"]
        if verbose:
            print(" ".join(cmd), file=sys.stderr)
        r = subprocess.run(cmd, capture_output=True, text=True)
        if r.returncode != 0:
            raise RuntimeError(f"link failed:\n{r.stdout}\n{r.stderr}")
    return LIB


if __name__ == "__main__":
    print(build(force="--force" in sys.argv, verbose=True))
