"""Build libpcgcn.so (sm_100a CUDA kernels + host planner + C ABI) in-tree.

    python -m paper_conf_ipps_tianmyd20_b200.build

nvcc cross-compiles for sm_100a without a GPU.  The .so lands next to this
file so it travels with the repo snapshot to the GPU box.
"""
from __future__ import annotations

import os
import subprocess
import sys

HERE = os.path.dirname(os.path.abspath(__file__))
ROOT = os.path.dirname(HERE)
CSRC = os.path.join(HERE, "csrc")
OUT = os.path.join(HERE, "libpcgcn.so")
NVCC = os.environ.get("NVCC", "/usr/local/cuda/bin/nvcc")
ARCH = ["-gencode", "arch=compute_100a,code=sm_100a"]
CU_SOURCES = ["pcgcn_api.cu", "sparse.cu", "tc_engine.cu", "dense_simt.cu", "gemm.cu", "loss_opt.cu",
              "calibrate.cu", "probe.cu", "tc_pair.cu", "halo.cu"]
CXX_SOURCES = ["planner.cpp", "nccl_halo.cpp"]


def _run(cmd):
    print(" ".join(cmd), flush=True)
    subprocess.check_call(cmd)


def _stale(out, deps):
    if not os.path.exists(out):
        return True
    t = os.path.getmtime(out)
    return any(os.path.getmtime(d) > t for d in deps)


def build(verbose_ptxas: bool = False, force: bool = False) -> str:
    objdir = os.path.join(HERE, "build")
    os.makedirs(objdir, exist_ok=True)
    headers = [os.path.join(CSRC, f) for f in os.listdir(CSRC) if f.endswith((".h", ".cuh"))]
    headers.append(os.path.join(ROOT, "include", "pcgcn.h"))
    objs = []
    for src in CU_SOURCES:
        s = os.path.join(CSRC, src)
        o = os.path.join(objdir, src + ".o")
        objs.append(o)
        if force or _stale(o, [s] + headers):
            cmd = [NVCC, *ARCH, "-O3", "-lineinfo", "-std=c++17", "-Xcompiler", "-fPIC",
                   "-I" + os.path.join(ROOT, "include"), "-c", s, "-o", o]
            if verbose_ptxas:
                cmd.insert(1, "-Xptxas=-v")
            _run(cmd)
    for src in CXX_SOURCES:
        s = os.path.join(CSRC, src)
        o = os.path.join(objdir, src + ".o")
        objs.append(o)
        if force or _stale(o, [s] + headers):
            _run(["g++", "-O3", "-std=c++17", "-fPIC", "-pthread", "-I" + os.path.join(ROOT, "include"),
                  "-I/usr/local/cuda/include", "-c", s, "-o", o])
    if force or _stale(OUT, objs):
        _run([NVCC, *ARCH, "-shared", "-o", OUT, *objs, "-Xcompiler", "-pthread", "-lcuda" if False else "-ldl"])
    return OUT


def build_synth() -> str:
    src = os.path.join(ROOT, "synth", "csrc", "synth_gen.cpp")
    out = os.path.join(ROOT, "synth", "_synth_gen.so")
    if _stale(out, [src]):
        _run(["g++", "-O3", "-std=c++17", "-shared", "-fPIC", "-pthread", src, "-o", out])
    return out


if __name__ == "__main__":
    build(verbose_ptxas="-v" in sys.argv, force="-f" in sys.argv)
    build_synth()
