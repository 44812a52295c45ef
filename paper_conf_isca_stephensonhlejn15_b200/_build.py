"""In-tree build of the native libraries (nvcc for sm_100a, gcc for the host generator).

  lib/libsassi.so           the product: C-ABI + CUDA kernels (csrc/*.cu)
  lib/libsassi_gen.so       device record generator (gen/gen_dev.cu)   — input generation only
  lib/libsassi_gen_host.so  host record generator (gen/gen_host.c)     — input generation only
Built .so files are git-ignored but travel to the GPU box with the gpurun snapshot.
"""
from __future__ import annotations

import glob
import os
import subprocess
import sys

PKG = os.path.dirname(os.path.abspath(__file__))
ROOT = os.path.dirname(PKG)
LIB = os.path.join(PKG, "lib")
CSRC = os.path.join(PKG, "csrc")
GEN = os.path.join(PKG, "gen")
INCLUDE = os.path.join(ROOT, "include")

NVCC = os.environ.get("NVCC", "/usr/local/cuda/bin/nvcc")
ARCH = ["-gencode", "arch=compute_100a,code=sm_100a"]
NVFLAGS = ARCH + ["-O3", "-lineinfo", "-std=c++17", "-Xcompiler", "-fPIC,-O2",
                  "--expt-relaxed-constexpr", "-Xptxas", "-warn-spills"]


def _stale(target: str, sources: list[str]) -> bool:
    if not os.path.exists(target):
        return True
    t = os.path.getmtime(target)
    return any(os.path.getmtime(s) > t for s in sources)


def _run(cmd: list[str], verbose: bool) -> None:
    if verbose:
        print(" ".join(cmd), file=sys.stderr)
    subprocess.check_call(cmd)


def build(force: bool = False, verbose: bool = False) -> dict:
    os.makedirs(LIB, exist_ok=True)
    out = {}
    # product library
    srcs = sorted(glob.glob(os.path.join(CSRC, "*.cu")) + glob.glob(os.path.join(CSRC, "*.cpp")))
    deps = srcs + glob.glob(os.path.join(CSRC, "*.cuh")) + glob.glob(os.path.join(CSRC, "*.h")) + \
        glob.glob(os.path.join(INCLUDE, "*.h"))
    tgt = os.path.join(LIB, "libsassi.so")
    if srcs and (force or _stale(tgt, deps)):
        from concurrent.futures import ThreadPoolExecutor
        objdir = os.path.join(ROOT, "build", "obj")
        os.makedirs(objdir, exist_ok=True)
        objs = [os.path.join(objdir, os.path.basename(s) + ".o") for s in srcs]
        with ThreadPoolExecutor(max_workers=min(8, len(srcs))) as ex:
            list(ex.map(lambda so: _run([NVCC] + NVFLAGS + ["-I", INCLUDE, "-I", CSRC, "-c", "-o",
                                                              so[1], so[0]], verbose),
                        zip(srcs, objs)))
        tmp = tgt + ".tmp%d" % os.getpid()
        _run([NVCC] + ARCH + ["-shared", "-o", tmp] + objs + ["-ldl", "-lpthread"], verbose)
        os.replace(tmp, tgt)
    out["libsassi"] = tgt
    # device generator
    tgt = os.path.join(LIB, "libsassi_gen.so")
    deps = [os.path.join(GEN, "gen_dev.cu"), os.path.join(GEN, "sassi_gen.h")]
    if force or _stale(tgt, deps):
        tmp = tgt + ".tmp%d" % os.getpid()
        _run([NVCC] + NVFLAGS + ["-shared", "-o", tmp, deps[0]], verbose)
        os.replace(tmp, tgt)
    out["libsassi_gen"] = tgt
    # host generator
    tgt = os.path.join(LIB, "libsassi_gen_host.so")
    deps = [os.path.join(GEN, "gen_host.c"), os.path.join(GEN, "sassi_gen.h")]
    if force or _stale(tgt, deps):
        tmp = tgt + ".tmp%d" % os.getpid()
        _run(["gcc", "-O2", "-std=c11", "-Wall", "-Wextra", "-shared", "-fPIC", "-o", tmp, deps[0]],
             verbose)
        os.replace(tmp, tgt)
    out["libsassi_gen_host"] = tgt
    return out


if __name__ == "__main__":
    print(build(force="--force" in sys.argv, verbose=True))
