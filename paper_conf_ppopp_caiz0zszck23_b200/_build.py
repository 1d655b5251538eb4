"""Builds libdsp.so in-tree with nvcc for sm_100a (no JIT cache, no torch extension)."""
from __future__ import annotations

import glob
import os
import subprocess

HERE = os.path.dirname(os.path.abspath(__file__))
ROOT = os.path.dirname(HERE)
LIB = os.path.join(HERE, "libdsp.so")
SOURCES = [os.path.join(HERE, "csrc", "dsp_runtime.cu")]
NVCC = os.environ.get("NVCC", "/usr/local/cuda/bin/nvcc")
NVCC_FLAGS = ["-O3", "-std=c++17", "-lineinfo", "-gencode", "arch=compute_100a,code=sm_100a",
              "-Xcompiler", "-fPIC,-O3", "-shared", "-I", os.path.join(ROOT, "include")]


def _inputs():
    return SOURCES + glob.glob(os.path.join(HERE, "csrc", "*.cuh")) + [os.path.join(ROOT, "include", "dsp.h")]


def stale() -> bool:
    if not os.path.exists(LIB):
        return True
    t = os.path.getmtime(LIB)
    return any(os.path.getmtime(p) > t for p in _inputs())


def build(force: bool = False, verbose: bool = False) -> str:
    if force or stale():
        tmp = LIB + f".tmp{os.getpid()}"
        extra = ["-DDSP_DEBUG_STAMPS"] if os.environ.get("DSP_DEBUG_STAMPS") else []
        cmd = [NVCC, *NVCC_FLAGS, *extra, *(["-Xptxas", "-v"] if verbose else []), "-o", tmp, *SOURCES]
        subprocess.check_call(cmd)
        os.replace(tmp, LIB)
    return LIB


def build_variant(name: str, defines) -> str:
    """Experiment build: libdsp_<name>.so with extra -D flags (selected at run time
    with DSP_LIB=<path>); never loaded by default."""
    out = os.path.join(HERE, f"libdsp_{name}.so")
    cmd = [NVCC, *NVCC_FLAGS, *[f"-D{d}" for d in defines], "-o", out, *SOURCES]
    subprocess.check_call(cmd)
    return out


if __name__ == "__main__":
    print(build(force=True, verbose=True))
