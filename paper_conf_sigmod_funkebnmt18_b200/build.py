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


def _compile(src: str, obj: str, verbose: bool) -> None:
    cmd = [NVCC, "-O3", "-std=c++17", *ARCH, "-lineinfo", "-Xcompiler", "-fPIC", "-c",
           "-I" + os.path.join(ROOT, "include"), "-o", obj + ".tmp", src]
    if verbose:
        cmd.insert(1, "-Xptxas=-v")
    r = subprocess.run(cmd, capture_output=True, text=True)
    if r.returncode != 0:
        sys.stderr.write(r.stdout + r.stderr)
        raise RuntimeError(f"nvcc failed compiling {os.path.basename(src)}")
    if verbose:
        sys.stderr.write(r.stderr)
    os.replace(obj + ".tmp", obj)


def build(force: bool = False, verbose: bool = False) -> str:
    """One object per CUDA source, compiled in parallel (a source is recompiled when it
    or any header is newer than its object), then linked into libhq.so."""
    from concurrent.futures import ThreadPoolExecutor
    embed_prelude()
    if not force and up_to_date():
        return SO
    objdir = os.path.join(ROOT, "build", "libhq")
    os.makedirs(objdir, exist_ok=True)
    hdr_t = max([os.path.getmtime(h) for h in headers()] + [0.0])
    jobs = []
    objs = []
    for src in sources():
        obj = os.path.join(objdir, os.path.basename(src)[:-3] + ".o")
        objs.append(obj)
        if force or not os.path.exists(obj) or os.path.getmtime(obj) < max(os.path.getmtime(src), hdr_t):
            jobs.append((src, obj))
    with ThreadPoolExecutor(max_workers=max(1, min(len(jobs), os.cpu_count() or 1))) as ex:
        for f in [ex.submit(_compile, s2, o, verbose) for s2, o in jobs]:
            f.result()
    cudalib = os.path.join(os.path.dirname(os.path.dirname(NVCC)), "lib64")
    cmd = [NVCC, *ARCH, "-shared", "-o", SO + ".tmp", *objs, "-L" + cudalib, "-lnvrtc", "-Xlinker", "-rpath," + cudalib]
    r = subprocess.run(cmd, capture_output=True, text=True)
    if r.returncode != 0:
        sys.stderr.write(r.stdout + r.stderr)
        raise RuntimeError("nvcc failed linking libhq.so")
    os.replace(SO + ".tmp", SO)
    return SO


if __name__ == "__main__":
    build(force="--force" in sys.argv, verbose="-v" in sys.argv)
    print(SO)
