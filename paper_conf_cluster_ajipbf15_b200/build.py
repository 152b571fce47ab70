"""Build libmcl.so in-tree: every CUDA source compiled for sm_100a with nvcc.

    python -m paper_conf_cluster_ajipbf15_b200.build [--force]

Objects go to build/ (git-ignored); the shared library lands next to this file so it
travels with the repo snapshot to the GPU box.
"""
from __future__ import annotations

import concurrent.futures as cf
import os
import subprocess
import sys

PKG = os.path.dirname(os.path.abspath(__file__))
ROOT = os.path.dirname(PKG)
CSRC = os.path.join(PKG, "csrc")
BUILD = os.path.join(ROOT, "build", "mcl")
LIB = os.path.join(PKG, "libmcl.so")
NVCC = os.environ.get("NVCC", "/usr/local/cuda/bin/nvcc")
ARCH = ["-gencode", "arch=compute_100a,code=sm_100a"]
SOURCES = ["search_blocked.cu", "search_mixed.cu", "search_batch.cu", "search_flat.cu", "search_generic.cu", "search_small.cu",
           "search_bnb.cu", "resident.cu", "costs.cu", "reduce.cu", "score.cu", "probe.cu", "mcl.cpp"]
HEADERS = ["common.cuh", "kernels.h", "blocked_core.cuh", "peer.cuh"]


def _nccl_include() -> str:
    try:
        import nvidia.nccl  # noqa: F401  (the wheel torch uses)

        inc = os.path.join(os.path.dirname(nvidia.nccl.__file__), "include")
        if os.path.exists(os.path.join(inc, "nccl.h")):
            return inc
    except Exception:
        pass
    return "/usr/include"


def _flags() -> list[str]:
    return ARCH + [
        "-O3", "-lineinfo", "-std=c++17", "-Xcompiler", "-fPIC,-Wall",
        "-I", os.path.join(ROOT, "include"), "-I", CSRC, "-I", _nccl_include(),
    ]


def _stale(out: str, deps: list[str]) -> bool:
    if not os.path.exists(out):
        return True
    t = os.path.getmtime(out)
    return any(os.path.getmtime(d) > t for d in deps)


def build(force: bool = False, verbose: bool = False) -> str:
    os.makedirs(BUILD, exist_ok=True)
    common = [os.path.join(CSRC, h) for h in HEADERS] + [
        os.path.join(ROOT, "include", "mcl.h"), os.path.join(ROOT, "include", "mcl_ext.h"), __file__,
    ]
    jobs = []
    objs = []
    for src in SOURCES:
        path = os.path.join(CSRC, src)
        obj = os.path.join(BUILD, src + ".o")
        objs.append(obj)
        if force or _stale(obj, [path] + common):
            cmd = [NVCC] + _flags() + ["-c", path, "-o", obj]
            jobs.append(cmd)
    with cf.ThreadPoolExecutor(max_workers=len(jobs) or 1) as ex:
        futs = [ex.submit(subprocess.run, c, capture_output=True, text=True) for c in jobs]
        for cmd, f in zip(jobs, futs):
            r = f.result()
            if verbose or r.returncode:
                sys.stderr.write(" ".join(cmd) + "\n" + r.stdout + r.stderr)
            if r.returncode:
                raise RuntimeError(f"nvcc failed: {cmd[-3]}")
    if force or jobs or _stale(LIB, objs):
        cmd = [NVCC] + ARCH + ["-shared", "-o", LIB] + objs + ["-ldl", "-lpthread"]
        r = subprocess.run(cmd, capture_output=True, text=True)
        if r.returncode:
            raise RuntimeError("link failed:\n" + r.stdout + r.stderr)
    return LIB


if __name__ == "__main__":
    print(build(force="--force" in sys.argv, verbose="-v" in sys.argv))
