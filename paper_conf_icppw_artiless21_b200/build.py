"""Build libturbobc.so in-tree with nvcc for sm_100a (no JIT cache; the .so travels with the repo)."""
from __future__ import annotations

import os
import shutil
import subprocess
import sys

PKG = os.path.dirname(os.path.abspath(__file__))
ROOT = os.path.dirname(PKG)
CSRC = os.path.join(PKG, "csrc")
LIB = os.path.join(PKG, "libturbobc.so")
LIB_DEBUG = os.path.join(PKG, "libturbobc_debug.so")  # -DTBC_DEBUG: device bounds checks
SOURCES = ["tbc_api.cu", "tbc_engine.cu", "tbc_batch.cu", "tbc_single.cu"]
HEADERS = ["tbc_internal.cuh", "tbc_device.cuh"]
ARCH = ["-gencode", "arch=compute_100a,code=sm_100a"]


def nvcc() -> str:
    for cand in (shutil.which("nvcc"), "/usr/local/cuda/bin/nvcc"):
        if cand and os.path.exists(cand):
            return cand
    raise RuntimeError("nvcc not found: cannot build libturbobc.so")


def _stale(lib=LIB) -> bool:
    if not os.path.exists(lib):
        return True
    t = os.path.getmtime(lib)
    deps = [os.path.join(CSRC, f) for f in SOURCES + HEADERS] + [os.path.join(ROOT, "include", "tbc.h")]
    return any(os.path.getmtime(p) > t for p in deps)


def build(force: bool = False, verbose: bool = False, debug: bool = False, variant: str = "") -> str:
    """variant: extra -D flags for tuning experiments (e.g. "-DTBC_BLOCK=1024 -DTBC_LANE_ITEMS=4"),
    built as libturbobc_<hash>.so next to the default library."""
    lib = LIB_DEBUG if debug else LIB
    vflags = variant.split()
    if vflags:
        import hashlib
        lib = os.path.join(PKG, "libturbobc_" + hashlib.sha1(variant.encode()).hexdigest()[:8] + ".so")
    if not force and not _stale(lib):
        return lib
    tmp = lib + f".tmp{os.getpid()}"
    cmd = [nvcc(), *ARCH, "-O3", "-lineinfo", "-std=c++17", "-shared", "-Xcompiler", "-fPIC",
           *(["-DTBC_DEBUG"] if debug else []), *vflags,
           "-Xptxas", "-v" if verbose else "-O3", f"-I{os.path.join(ROOT, 'include')}",
           "-o", tmp] + [os.path.join(CSRC, f) for f in SOURCES]
    res = subprocess.run(cmd, capture_output=True, text=True)
    if res.returncode != 0:
        sys.stderr.write(res.stdout + res.stderr)
        raise RuntimeError("nvcc failed building libturbobc.so")
    if verbose:
        sys.stderr.write(res.stderr)
    os.replace(tmp, lib)
    return lib


if __name__ == "__main__":
    print(build(force="--force" in sys.argv, verbose="-v" in sys.argv, debug="--debug" in sys.argv))
