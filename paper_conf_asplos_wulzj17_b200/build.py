"""Build libflep.so in-tree with nvcc for sm_100a (no JIT cache; the .so travels with the repo)."""
from __future__ import annotations

import os
import subprocess
import sys

HERE = os.path.dirname(os.path.abspath(__file__))
ROOT = os.path.dirname(HERE)
CSRC = os.path.join(HERE, "csrc")
LIB = os.path.join(HERE, "libflep.so")
SOURCES = ["kernels.cu", "gemm_tcgen05.cu", "gemm2_tcgen05.cu", "stencil_tma.cu", "runtime.cu"]
HEADERS = ["flep_device.cuh", "bodies.cuh", "gemm_tcgen05.cuh", "gemm2_tcgen05.cuh", "stencil_tma.cuh", "kernels.hpp",
           "policy.hpp"]

NVCC_FLAGS = [
    "-gencode", "arch=compute_100a,code=sm_100a",
    "-O3", "-lineinfo", "-std=c++17",
    "-Xcompiler", "-fPIC", "-Xcompiler", "-O2",
    "-shared",
]


def _nvcc():
    for c in (os.environ.get("NVCC"), "/usr/local/cuda/bin/nvcc", "nvcc"):
        if c and (os.path.isabs(c) and os.path.exists(c) or not os.path.isabs(c)):
            return c
    return "nvcc"


def sources():
    return [os.path.join(CSRC, s) for s in SOURCES if os.path.exists(os.path.join(CSRC, s))]


def needs_build() -> bool:
    if not os.path.exists(LIB):
        return True
    t = os.path.getmtime(LIB)
    deps = sources() + [os.path.join(CSRC, h) for h in HEADERS] + [os.path.join(ROOT, "include", "flep.h")]
    return any(os.path.exists(d) and os.path.getmtime(d) > t for d in deps)


def build(force: bool = False, verbose: bool = False) -> str:
    if os.environ.get("FLEP_LIB_PATH"):          # an experiment's prebuilt variant (flep.py loads it)
        return os.environ["FLEP_LIB_PATH"]
    if not force and not needs_build():
        return LIB
    extra = os.environ.get("FLEP_NVCC_EXTRA", "").split()     # experiment hook (e.g. -DFLEP_SPMV_U=4)
    cmd = [_nvcc()] + NVCC_FLAGS + extra + ["-o", LIB + ".tmp"] + sources() + ["-lpthread"]
    if verbose:
        print(" ".join(cmd), file=sys.stderr)
    r = subprocess.run(cmd, capture_output=True, text=True)
    if r.returncode != 0:
        raise RuntimeError("nvcc failed:\n" + r.stdout + r.stderr)
    os.replace(LIB + ".tmp", LIB)
    return LIB


def build_user_body(src: str, out: str, force: bool = False) -> str:
    """Compile a user-defined body (a .cu using include/flep_body.cuh and FLEP_DEFINE_BODY) into
    its own shared library with the flags and headers libflep.so was built with."""
    deps = [src, os.path.join(ROOT, "include", "flep_body.cuh"), os.path.join(ROOT, "include", "flep.h"),
            os.path.join(CSRC, "flep_device.cuh")]
    if not force and os.path.exists(out) and all(os.path.getmtime(d) <= os.path.getmtime(out) for d in deps):
        return out
    os.makedirs(os.path.dirname(os.path.abspath(out)), exist_ok=True)
    cmd = [_nvcc()] + NVCC_FLAGS + ["-I", os.path.join(ROOT, "include"), "-o", out + ".tmp", src]
    r = subprocess.run(cmd, capture_output=True, text=True)
    if r.returncode != 0:
        raise RuntimeError("nvcc failed for the user body:\n" + r.stdout + r.stderr)
    os.replace(out + ".tmp", out)
    return out


if __name__ == "__main__":
    print(build(force="--force" in sys.argv, verbose=True))
