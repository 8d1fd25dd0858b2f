"""In-tree build of the native libraries (sm_100a only).

libagnn.so    — the product: C-ABI (include/agnn.h) + hand-written CUDA kernels.
libagnngen.so — seeded input generators (host + device), shared test/bench infra.

Both are built with explicit ``nvcc -gencode arch=compute_100a,code=sm_100a``;
the .so files land next to their sources so they travel with gpurun snapshots.
"""
from __future__ import annotations

import glob
import os
import subprocess
import sys

PKG = os.path.dirname(os.path.abspath(__file__))
ROOT = os.path.dirname(PKG)
INCLUDE = os.path.join(ROOT, "include")
NVCC = os.environ.get("NVCC", "/usr/local/cuda/bin/nvcc")
ARCH = ["-gencode", "arch=compute_100a,code=sm_100a"]

GEN_DIR = os.path.join(PKG, "gen")
GEN_SO = os.path.join(GEN_DIR, "libagnngen.so")
CSRC = os.path.join(PKG, "csrc")
AGNN_SO = os.path.join(PKG, "libagnn.so")


def _nccl_dirs():
    try:
        import nvidia.nccl as nn  # the NCCL torch itself loads (2.28.x)
        base = os.path.dirname(nn.__file__) if nn.__file__ else list(nn.__path__)[0]
        inc, libd = os.path.join(base, "include"), os.path.join(base, "lib")
        if os.path.exists(os.path.join(inc, "nccl.h")):
            return inc, libd
    except Exception:
        pass
    return "/usr/include", "/usr/lib/x86_64-linux-gnu"


def _stale(target, sources):
    if not os.path.exists(target):
        return True
    t = os.path.getmtime(target)
    return any(os.path.getmtime(s) > t for s in sources)


def _run(cmd):
    print("[build]", " ".join(cmd), file=sys.stderr)
    subprocess.check_call(cmd)


def build_gen(force: bool = False) -> str:
    srcs = [os.path.join(GEN_DIR, "gen.cu"), os.path.join(GEN_DIR, "agnn_gen.h")]
    if force or _stale(GEN_SO, srcs):
        _run([NVCC, *ARCH, "-O3", "-std=c++17", "-lineinfo", "-shared", "-Xcompiler", "-fPIC,-fopenmp",
              "-o", GEN_SO, srcs[0], "-lgomp"])
    return GEN_SO


def agnn_sources():
    return sorted(glob.glob(os.path.join(CSRC, "*.cu")))


def agnn_deps():
    return agnn_sources() + sorted(glob.glob(os.path.join(CSRC, "*.cuh"))) + \
        sorted(glob.glob(os.path.join(INCLUDE, "*.h")))


def build_agnn(force: bool = False, verbose_ptxas: bool = False, out: str | None = None,
               defines=()) -> str:
    """Compile every csrc/*.cu to an object (in parallel) and link libagnn.so.
    out / defines: an extra build (e.g. -D experiment switches) at another path."""
    so = out or AGNN_SO
    if not (force or _stale(so, agnn_deps())):
        return so
    nccl_inc, nccl_lib = _nccl_dirs()
    objdir = os.path.join(ROOT, "build", "agnn" if not out else
                          "agnn_" + os.path.basename(out).replace(".so", ""))
    os.makedirs(objdir, exist_ok=True)
    headers = [d for d in agnn_deps() if not d.endswith(".cu")]
    flags = [*ARCH, "-O3", "-std=c++17", "-lineinfo", "-Xcompiler", "-fPIC",
             "--expt-relaxed-constexpr", "-I", INCLUDE, "-I", CSRC, "-I", nccl_inc]
    if verbose_ptxas:
        flags.append("-Xptxas=-v")
    flags += ["-D" + d for d in defines]
    jobs = []
    for src in agnn_sources():
        obj = os.path.join(objdir, os.path.basename(src)[:-3] + ".o")
        if force or _stale(obj, [src] + headers):
            jobs.append([NVCC, *flags, "-c", src, "-o", obj])
    from concurrent.futures import ThreadPoolExecutor
    with ThreadPoolExecutor(max_workers=max(1, min(8, os.cpu_count() or 1))) as ex:
        list(ex.map(_run, jobs))
    objs = [os.path.join(objdir, os.path.basename(s)[:-3] + ".o") for s in agnn_sources()]
    _run([NVCC, *ARCH, "-shared", "-o", so, *objs, "-L", nccl_lib, "-l:libnccl.so.2",
          "-Xlinker", "-rpath," + nccl_lib])
    return so


def build_all(force: bool = False):
    return build_gen(force), build_agnn(force)


if __name__ == "__main__":
    build_all(force="--force" in sys.argv)
