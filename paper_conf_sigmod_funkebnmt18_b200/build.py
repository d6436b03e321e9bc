"""Build libhq.so in-tree for sm_100a (nvcc cross-compiles without a GPU).

Every CUDA source of the engine is compiled with
``-gencode arch=compute_100a,code=sm_100a -lineinfo`` into one shared library
exporting the C ABI of ``include/hq.h``.
"""
from __future__ import annotations

import glob
import os
import subprocess
import sys

PKG = os.path.dirname(os.path.abspath(__file__))
ROOT = os.path.dirname(PKG)
CSRC = os.path.join(PKG, "csrc")
SO = os.path.join(PKG, "libhq.so")
NVCC = os.environ.get("NVCC", "/usr/local/cuda/bin/nvcc")
ARCH = ["-gencode", "arch=compute_100a,code=sm_100a"]


def sources():
    return sorted(glob.glob(os.path.join(CSRC, "*.cu")))


def headers():
    return sorted(glob.glob(os.path.join(CSRC, "*.h")) + glob.glob(os.path.join(CSRC, "*.cuh")) +
                  glob.glob(os.path.join(ROOT, "include", "*.h")))


def up_to_date() -> bool:
    if not os.path.exists(SO):
        return False
    t = os.path.getmtime(SO)
    return all(os.path.getmtime(f) <= t for f in sources() + headers())


def embed_prelude() -> None:
    """hq_jit_prelude.cuh -> hq_jit_prelude.inc (a raw string literal for NVRTC)."""
    src = os.path.join(CSRC, "hq_jit_prelude.cuh")
    dst = os.path.join(CSRC, "hq_jit_prelude.inc")
    text = 'R"HQJIT(' + open(src).read() + ')HQJIT"\n'
    if not os.path.exists(dst) or open(dst).read() != text:
        with open(dst, "w") as f:
            f.write(text)


def build(force: bool = False, verbose: bool = False) -> str:
    embed_prelude()
    if not force and up_to_date():
        return SO
    cudalib = os.path.join(os.path.dirname(os.path.dirname(NVCC)), "lib64")
    cmd = [NVCC, "-O3", "-std=c++17", *ARCH, "-lineinfo", "-Xcompiler", "-fPIC", "-shared",
           "-I" + os.path.join(ROOT, "include"), "-o", SO + ".tmp", *sources(),
           "-L" + cudalib, "-lnvrtc", "-Xlinker", "-rpath," + cudalib]
    if verbose:
        cmd.insert(1, "-Xptxas=-v")
    r = subprocess.run(cmd, capture_output=True, text=True)
    if r.returncode != 0:
        sys.stderr.write(r.stdout + r.stderr)
        raise RuntimeError("nvcc failed building libhq.so")
    if verbose:
        sys.stderr.write(r.stderr)
    os.replace(SO + ".tmp", SO)
    return SO


if __name__ == "__main__":
    build(force="--force" in sys.argv, verbose="-v" in sys.argv)
    print(SO)
