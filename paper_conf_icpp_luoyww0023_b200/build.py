"""Build libsplit_ga.so in-tree with nvcc for sm_100a (no JIT cache: the .so
travels with the repo snapshot to the GPU box)."""
from __future__ import annotations

import os
import subprocess
import sys

PKG = os.path.dirname(os.path.abspath(__file__))
ROOT = os.path.dirname(PKG)
CSRC = os.path.join(PKG, "csrc")
LIB_DIR = os.path.join(PKG, "lib")
LIB = os.path.join(LIB_DIR, "libsplit_ga.so")
SOURCES = [os.path.join(CSRC, f) for f in ("split_eval.cu", "split_ga.cu", "split_exact.cu", "split_qos.cu", "split_host.cpp")]
HEADERS = [os.path.join(CSRC, "split_internal.h"), os.path.join(CSRC, "split_device.cuh"),
           os.path.join(ROOT, "include", "split_ga.h")]
NVCC = os.environ.get("NVCC", "/usr/local/cuda/bin/nvcc")
ARCH = ["-gencode", "arch=compute_100a,code=sm_100a"]
FLAGS = [
    *ARCH, "-lineinfo", "-O3", "-std=c++17",
    "-fmad=false",                       # every FP64 op is one IEEE RN op (R5')
    "-Xcompiler", "-fPIC", "-Xcompiler", "-O2", "-Xcompiler", "-ffp-contract=off",
]
OBJ_DIR = os.path.join(LIB_DIR, "obj")


def _newest_dep() -> float:
    return max(os.path.getmtime(f) for f in HEADERS + [__file__])


def _obj(src: str) -> str:
    return os.path.join(OBJ_DIR, os.path.basename(src) + ".o")


def stale() -> bool:
    if not os.path.exists(LIB):
        return True
    t = os.path.getmtime(LIB)
    return any(os.path.getmtime(f) > t for f in SOURCES + HEADERS + [__file__])


def build(force: bool = False, verbose: bool = False) -> str:
    """Compile each translation unit to an object (in parallel, skipping
    up-to-date objects), then link the shared library with the static cudart."""
    if not force and not stale():
        return LIB
    os.makedirs(OBJ_DIR, exist_ok=True)
    extra = ["-DSPLIT_TRACE_BUILD"] if os.environ.get("SPLIT_TRACE_BUILD") else []
    if os.environ.get("SPLIT_GA_MIN_BLOCKS"):            # A/B builds of the GA kernel's occupancy
        extra.append(f"-DSPLIT_GA_MIN_BLOCKS={int(os.environ['SPLIT_GA_MIN_BLOCKS'])}")
    inc = ["-I", os.path.join(ROOT, "include"), "-I", CSRC]
    dep_t = _newest_dep()
    procs = []
    for src in SOURCES:
        obj = _obj(src)
        if not force and not extra and os.path.exists(obj) and os.path.getmtime(obj) > max(dep_t, os.path.getmtime(src)):
            continue
        tmp = obj + f".tmp{os.getpid()}"
        cmd = [NVCC, *FLAGS, *extra, *inc, "-c", src, "-o", tmp]
        if verbose:
            print(" ".join(cmd), file=sys.stderr)
        procs.append((subprocess.Popen(cmd), tmp, obj, cmd))
    failed = []
    for p, tmp, obj, cmd in procs:
        if p.wait() != 0:
            failed.append(cmd)
        else:
            os.replace(tmp, obj)
    if failed:
        raise subprocess.CalledProcessError(1, failed[0])
    tmp = LIB + f".tmp{os.getpid()}"
    cmd = [NVCC, *ARCH, "-shared", "-cudart", "static", *[_obj(s) for s in SOURCES], "-o", tmp, "-ldl"]
    if verbose:
        print(" ".join(cmd), file=sys.stderr)
    subprocess.check_call(cmd)
    os.replace(tmp, LIB)
    return LIB


if __name__ == "__main__":
    print(build(force="--force" in sys.argv, verbose=True))
