"""Build the in-tree C-ABI library ``libplgpu.so`` for sm_100a with nvcc.

Sources: csrc/executor.cu (persistent kernels), csrc/runtime.cu (host C-ABI),
csrc/solver.cpp (Fig. 1 / Fig. 2 solvers).  The .so lands next to this file so
it travels with the repo snapshot to the GPU box.
"""
from __future__ import annotations

import os
import subprocess
import sys

HERE = os.path.dirname(os.path.abspath(__file__))
CSRC = os.path.join(HERE, "csrc")
ROOT = os.path.dirname(HERE)
LIB = os.path.join(HERE, "libplgpu.so")
NVCC = os.environ.get("NVCC", "nvcc")
ARCH = ["-gencode", "arch=compute_100a,code=sm_100a"]
FLAGS = ["-O3", "-lineinfo", "-std=c++17", "-Xcompiler", "-fPIC,-O2", f"-I{ROOT}/include", f"-I{CSRC}"]
SOURCES = ["executor.cu", "runtime.cu", "solver.cpp"]
# measurement tool, not part of the product library (N3 co-runner experiment, tools/corunner.py)
CORUNNER_SRC = os.path.join(ROOT, "tools", "corunner", "corunner.cu")
CORUNNER_LIB = os.path.join(ROOT, "tools", "corunner", "libplcorunner.so")


def _stale() -> bool:
    if not os.path.exists(LIB):
        return True
    t = os.path.getmtime(LIB)
    deps = [os.path.join(CSRC, f) for f in os.listdir(CSRC)] + [os.path.join(ROOT, "include", "pl.h")]
    return any(os.path.getmtime(d) > t for d in deps)


def build(force: bool = False, verbose: bool = False) -> str:
    if not force and not _stale():
        return LIB
    objs = []
    bdir = os.path.join(HERE, "_build")
    os.makedirs(bdir, exist_ok=True)
    for src in SOURCES:
        obj = os.path.join(bdir, src + ".o")
        cmd = [NVCC, *ARCH, *FLAGS, "-c", os.path.join(CSRC, src), "-o", obj]
        if src.endswith(".cu"):
            cmd.insert(1, "-Xptxas=-v") if verbose else None
        r = subprocess.run(cmd, capture_output=True, text=True)
        if r.returncode != 0:
            raise RuntimeError(f"nvcc failed for {src}:\n{r.stderr}")
        if verbose and r.stderr:
            sys.stderr.write(r.stderr)
        objs.append(obj)
    tmp = LIB + ".tmp"
    cmd = [NVCC, *ARCH, "-shared", "-o", tmp, *objs, "-lcudart"]
    r = subprocess.run(cmd, capture_output=True, text=True)
    if r.returncode != 0:
        raise RuntimeError(f"link failed:\n{r.stderr}")
    os.replace(tmp, LIB)
    return LIB


def build_corunner() -> str:
    """The co-runner kernel of the N3 experiment as its own small library."""
    if os.path.exists(CORUNNER_LIB) and os.path.getmtime(CORUNNER_LIB) > os.path.getmtime(CORUNNER_SRC):
        return CORUNNER_LIB
    cmd = [NVCC, *ARCH, "-O3", "-Xcompiler", "-fPIC", "-shared", CORUNNER_SRC, "-o", CORUNNER_LIB]
    r = subprocess.run(cmd, capture_output=True, text=True)
    if r.returncode != 0:
        raise RuntimeError(f"nvcc failed for corunner.cu:\n{r.stderr}")
    return CORUNNER_LIB


if __name__ == "__main__":
    print(build(force="--force" in sys.argv, verbose="-v" in sys.argv))
