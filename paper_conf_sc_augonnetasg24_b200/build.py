"""Build libstf_cholesky.so in-tree for sm_100a (nvcc + g++, no torch extension
machinery).  Used by __graft_entry__.build() and by `python -m
paper_conf_sc_augonnetasg24_b200.build`.

The CUDA runtime is linked statically so the library does not depend on which
libcudart.so.12 happens to be loaded in the process (torch bundles its own).
"""
from __future__ import annotations

import concurrent.futures as cf
import os
import subprocess
import sys

HERE = os.path.dirname(os.path.abspath(__file__))
CSRC = os.path.join(HERE, "csrc")
ROOT = os.path.dirname(HERE)
BUILD = os.path.join(ROOT, "build", "obj")
LIB = os.path.join(HERE, "libstf_cholesky.so")
NVCC = os.environ.get("NVCC", "/usr/local/cuda/bin/nvcc")
ARCH = ["-gencode", "arch=compute_100a,code=sm_100a"]
COMMON = ["-O3", "-std=c++17", "-lineinfo", "-Xcompiler", "-fPIC", "-Xcompiler", "-Wall",
          "-I" + os.path.join(ROOT, "include"), "-I" + CSRC] + os.environ.get("STF_NVCC_DEFS", "").split()

SOURCES = [
    "kernels/gemm_dmma.cu",
    "kernels/panel.cu",
    "kernels/dataflow.cu",
    "kernels/trsm_panel.cu",
    "kernels/trsm_res.cu",
    "plan.cpp",
    "api.cpp",
    "exec.cpp",
    "mp.cpp",
    "harness.cpp",
    "mcast.cpp",
]


def _obj(src: str) -> str:
    return os.path.join(BUILD, src.replace("/", "_") + ".o")


def _deps_mtime() -> float:
    m = 0.0
    for dp, _, fs in os.walk(CSRC):
        for f in fs:
            m = max(m, os.path.getmtime(os.path.join(dp, f)))
    for h in ("stf_cholesky.h", "stf_harness.h"):
        m = max(m, os.path.getmtime(os.path.join(ROOT, "include", h)))
    return m


def _compile(src: str) -> str:
    out = _obj(src)
    cmd = [NVCC] + ARCH + COMMON + ["-c", os.path.join(CSRC, src), "-o", out]
    if src.endswith(".cu"):
        cmd += ["-Xptxas", "-v"]
    r = subprocess.run(cmd, capture_output=True, text=True)
    if r.returncode != 0:
        raise RuntimeError("nvcc failed for %s:\n%s\n%s" % (src, r.stdout, r.stderr))
    return r.stderr


def build(force: bool = False, verbose: bool = False) -> str:
    os.makedirs(BUILD, exist_ok=True)
    dep = _deps_mtime()
    if not force and os.path.exists(LIB) and os.path.getmtime(LIB) >= dep:
        return LIB
    with cf.ThreadPoolExecutor(max_workers=len(SOURCES)) as ex:
        logs = list(ex.map(_compile, SOURCES))
    if verbose:
        for s, lg in zip(SOURCES, logs):
            print("==", s)
            print(lg)
    cmd = [NVCC] + ARCH + ["-shared", "-cudart", "static", "-o", LIB] + [_obj(s) for s in SOURCES] + ["-lpthread"]
    r = subprocess.run(cmd, capture_output=True, text=True)
    if r.returncode != 0:
        raise RuntimeError("link failed:\n%s\n%s" % (r.stdout, r.stderr))
    return LIB


if __name__ == "__main__":
    print(build(force="--force" in sys.argv, verbose="-v" in sys.argv))
