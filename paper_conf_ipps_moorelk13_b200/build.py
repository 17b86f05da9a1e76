"""Build the sm_100a shared library libncc_b200.so in-tree (nvcc, no JIT cache).

The library is the product: every step of the hot path runs in its kernels, and the
Python binding (_native.py) only marshals arguments to its C ABI (include/ncc.h).
"""
from __future__ import annotations

import os
import subprocess
import sys

PKG = os.path.dirname(os.path.abspath(__file__))
ROOT = os.path.dirname(PKG)
CSRC = os.path.join(PKG, "csrc")
LIB = os.path.join(PKG, "libncc_b200.so")
SOURCES = [os.path.join(CSRC, "ncc_api.cu")]
KERNELS = os.path.join(CSRC, "ncc_kernels.cuh")
SRC_INC = os.path.join(CSRC, "ncc_kernels_src.inc")  # generated: the kernel source for NVRTC
# every source the library is compiled from: all of csrc/ (kernels, headers, includes) + the ABI header
DEPS = sorted(os.path.join(CSRC, f) for f in os.listdir(CSRC) if f.endswith((".cu", ".cuh", ".inc"))) + \
    [os.path.join(ROOT, "include", "ncc.h")]

NVCC_FLAGS = ["-gencode", "arch=compute_100a,code=sm_100a", "-O3", "-lineinfo", "-std=c++17",
              "--shared", "-Xcompiler", "-fPIC", "-Xptxas", "-v", "-ldl"]


def nvcc() -> str:
    for c in (os.environ.get("NVCC"), "/usr/local/cuda/bin/nvcc", "nvcc"):
        if c and (os.path.isabs(c) and os.path.exists(c) or not os.path.isabs(c)):
            return c
    return "nvcc"


def needs_build() -> bool:
    if not os.path.exists(LIB):
        return True
    t = os.path.getmtime(LIB)
    return any(os.path.getmtime(d) > t for d in DEPS)


def write_source_inc() -> None:
    """Embed ncc_kernels.cuh as a string: the run-time specialiser (NVRTC) compiles the very
    source the ahead-of-time instances come from."""
    src = open(KERNELS).read()
    assert ")NCC_SRC\"" not in src
    body = 'static const char kNccKernelSource[] = R"NCC_SRC(' + src + ')NCC_SRC";\n'
    if not os.path.exists(SRC_INC) or open(SRC_INC).read() != body:
        with open(SRC_INC, "w") as f:
            f.write(body)


def build(force: bool = False, verbose: bool = False) -> str:
    write_source_inc()
    if not force and not needs_build():
        return LIB
    tmp = LIB + f".tmp{os.getpid()}"
    cmd = [nvcc()] + NVCC_FLAGS + ["-o", tmp] + SOURCES
    r = subprocess.run(cmd, capture_output=True, text=True)
    if r.returncode != 0:
        sys.stderr.write(r.stdout + r.stderr)
        raise RuntimeError("nvcc failed building libncc_b200.so")
    if verbose:
        sys.stderr.write(r.stderr)
    os.replace(tmp, LIB)
    return LIB


if __name__ == "__main__":
    build(force="--force" in sys.argv, verbose=True)
    print(LIB)
