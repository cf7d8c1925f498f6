"""Build libtqr.so in-tree: nvcc for sm_100a only (no multi-arch, no JIT cache).

    python -m paper_conf_icpp_kimp13_b200.build [--force]

Objects are compiled in parallel into paper_conf_icpp_kimp13_b200/build/ and linked with the
static CUDA runtime into paper_conf_icpp_kimp13_b200/libtqr.so (git-ignored, travels with gpurun).
"""
from __future__ import annotations

import concurrent.futures as cf
import os
import subprocess
import sys

PKG = os.path.dirname(os.path.abspath(__file__))
ROOT = os.path.dirname(PKG)
CSRC = os.path.join(PKG, "csrc")
OBJ = os.path.join(PKG, "build")
LIB = os.path.join(PKG, "libtqr.so")
NVCC = os.environ.get("NVCC", "/usr/local/cuda/bin/nvcc")
ARCH = ["-gencode", "arch=compute_100a,code=sm_100a"]
COMMON = ["-O3", "-std=c++17", "-lineinfo", "-Xcompiler", "-fPIC", "-I" + os.path.join(ROOT, "include"),
          "-I" + CSRC]

SOURCES = [
    os.path.join(CSRC, "kernels", "qr_kernels.cu"),
    os.path.join(CSRC, "kernels", "qr_kernels_f32.cu"),
    os.path.join(CSRC, "kernels", "trsm.cu"),
    os.path.join(CSRC, "tqr_signal.cu"),
    os.path.join(CSRC, "tqr_api.cpp"),
    os.path.join(CSRC, "tqr_model.cpp"),
]


def _deps():
    out = []
    for d, _, fs in os.walk(CSRC):
        out += [os.path.join(d, f) for f in fs if f.endswith((".cu", ".cuh", ".h", ".hpp", ".cpp"))]
    out.append(os.path.join(ROOT, "include", "tqr.h"))
    return out


def _stale(target, deps):
    if not os.path.exists(target):
        return True
    t = os.path.getmtime(target)
    return any(os.path.getmtime(d) > t for d in deps)


def _compile(src, defines=(), tag=""):
    obj = os.path.join(OBJ, os.path.basename(src) + tag + ".o")
    cmd = [NVCC] + ARCH + COMMON + ["-D" + d for d in defines] + ["-c", src, "-o", obj]
    if src.endswith(".cpp"):
        cmd = [os.environ.get("CXX", "g++"), "-O3", "-std=c++17", "-g", "-fPIC", "-Wall",
               "-I" + os.path.join(ROOT, "include"), "-I" + CSRC, "-I/usr/local/cuda/include", "-c", src, "-o", obj]
    subprocess.check_call(cmd)
    return obj


def build(force: bool = False, verbose: bool = False) -> str:
    deps = _deps()
    if not force and not _stale(LIB, deps):
        return LIB
    os.makedirs(OBJ, exist_ok=True)
    with cf.ThreadPoolExecutor(max_workers=len(SOURCES)) as ex:
        objs = list(ex.map(_compile, SOURCES))
    tmp = LIB + ".%d.tmp" % os.getpid()
    subprocess.check_call([NVCC] + ARCH + ["-shared", "-cudart", "static", "-o", tmp] + objs + ["-ldl", "-lpthread"])
    os.replace(tmp, LIB)
    if verbose:
        print("built", LIB)
    return LIB


def build_variant(name: str, defines) -> str:
    """Probe-only variant library (e.g. phase-timing instrumentation), never loaded by the product."""
    os.makedirs(OBJ, exist_ok=True)
    with cf.ThreadPoolExecutor(max_workers=len(SOURCES)) as ex:
        objs = list(ex.map(lambda s: _compile(s, defines, "." + name), SOURCES))
    out = os.path.join(OBJ, "libtqr_%s.so" % name)
    subprocess.check_call([NVCC] + ARCH + ["-shared", "-cudart", "static", "-o", out] + objs + ["-ldl", "-lpthread"])
    return out


if __name__ == "__main__":
    build(force="--force" in sys.argv, verbose=True)
