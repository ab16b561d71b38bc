"""Build libsq.so (product) and synth/libsqsynth.so (seeded inputs) with nvcc for sm_100a.

In-tree build (the .so files travel to the GPU box with the gpurun snapshot).
Objects are compiled in parallel and re-used when up to date.
"""
from __future__ import annotations

import concurrent.futures as cf
import glob
import os
import subprocess
import sys

PKG = os.path.dirname(os.path.abspath(__file__))
ROOT = os.path.dirname(PKG)
CSRC = os.path.join(PKG, "csrc")
INCLUDE = os.path.join(ROOT, "include")
# SQ_BUILD_TAG=<t> (experiments only): objects under build/obj_<t>, library libsq_<t>.so, loaded with
# SQ_LIB_PATH; the product build is the untagged libsq.so
_TAG = os.environ.get("SQ_BUILD_TAG", "")
OBJ = os.path.join(ROOT, "build", "obj" + (f"_{_TAG}" if _TAG else ""))
LIB = os.path.join(PKG, f"libsq_{_TAG}.so" if _TAG else "libsq.so")
SYNTH_SRC = os.path.join(ROOT, "synth", "synth.cu")
SYNTH_LIB = os.path.join(ROOT, "synth", "libsqsynth.so")

NVCC = os.environ.get("NVCC", "/usr/local/cuda/bin/nvcc")
ARCH = ["-gencode", "arch=compute_100a,code=sm_100a"]
FLAGS = ["-O3", "-lineinfo", "-std=c++17", "-Xcompiler", "-fPIC", "--expt-relaxed-constexpr",
         "-Xptxas", "-v,-warn-spills"]


# debug builds only (e.g. SQ_NVCC_EXTRA="-DSQ_TC_DEBUG=1" for the tcgen05 decode trace)
EXTRA = os.environ.get("SQ_NVCC_EXTRA", "").split()


def nccl_dir() -> str:
    import importlib.util
    spec = importlib.util.find_spec("nvidia")
    for base in (spec.submodule_search_locations or []) if spec else []:
        d = os.path.join(base, "nccl")
        if os.path.exists(os.path.join(d, "include", "nccl.h")):
            return d
    raise RuntimeError("pip NCCL (nvidia/nccl) not found; it ships with torch")


def _run(cmd: list[str]) -> str:
    r = subprocess.run(cmd, capture_output=True, text=True)
    if r.returncode != 0:
        sys.stderr.write(r.stdout + r.stderr)
        raise RuntimeError("build failed: " + " ".join(cmd))
    return r.stdout + r.stderr


def _newer(out: str, deps: list[str]) -> bool:
    return os.path.exists(out) and all(os.path.getmtime(out) >= os.path.getmtime(d) for d in deps)


def build(verbose: bool = False, force: bool = False) -> str:
    os.makedirs(OBJ, exist_ok=True)
    nccl = nccl_dir()
    inc = ["-I", INCLUDE, "-I", CSRC, "-I", os.path.join(nccl, "include")]
    headers = glob.glob(os.path.join(CSRC, "*.cuh")) + glob.glob(os.path.join(CSRC, "*.h")) + [os.path.join(INCLUDE, "sq.h")]
    srcs = sorted(glob.glob(os.path.join(CSRC, "*.cu")))
    objs = []
    jobs = []
    for s in srcs:
        o = os.path.join(OBJ, os.path.basename(s) + ".o")
        objs.append(o)
        if force or not _newer(o, [s, *headers, __file__]):
            jobs.append([NVCC, *ARCH, *FLAGS, *EXTRA, *inc, "-c", s, "-o", o])
    logs = []
    with cf.ThreadPoolExecutor(max_workers=os.cpu_count() or 4) as ex:
        for log in ex.map(_run, jobs):
            logs.append(log)
    if verbose:
        for l in logs:
            print(l)
    if force or jobs or not _newer(LIB, objs):
        nlib = os.path.join(nccl, "lib")
        _run([NVCC, *ARCH, "-shared", "-o", LIB, *objs, "-L", nlib, "-l:libnccl.so.2",
              "-Xlinker", f"-rpath={nlib}", "-lcuda" if False else "-lcudart_static", "-ldl", "-lrt", "-lpthread"])
    if force or not _newer(SYNTH_LIB, [SYNTH_SRC, __file__]):
        _run([NVCC, *ARCH, "-O3", "-std=c++17", "-Xcompiler", "-fPIC", "-shared", SYNTH_SRC, "-o", SYNTH_LIB])
    return LIB


if __name__ == "__main__":
    build(verbose="-v" in sys.argv, force="-f" in sys.argv)
    print(LIB)
