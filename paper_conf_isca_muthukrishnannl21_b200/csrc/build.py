"""Build libproact.so (sm_100a) in-tree with nvcc.

Sources: runtime.cu (host runtime + sync kernels) and workloads.cu (agent + producer kernels).
No relocatable device code: every device call stays inside its translation unit.
"""
from __future__ import annotations

import os
import subprocess
import sys

HERE = os.path.dirname(os.path.abspath(__file__))
PKG = os.path.dirname(HERE)
ROOT = os.path.dirname(PKG)
INC = os.path.join(ROOT, "include")
OUT = os.path.join(PKG, "libproact.so")
SOURCES = ["runtime.cu", "workloads.cu", "graph.cu", "mcast.cu"]
DEPS = SOURCES
HEADERS = sorted(f for f in os.listdir(INC) if f.endswith((".h", ".cuh")))   # every public header
NVCC = os.environ.get("NVCC", "/usr/local/cuda/bin/nvcc")
FLAGS = ["-gencode", "arch=compute_100a,code=sm_100a", "-O3", "-lineinfo", "-std=c++17",
         "-Xcompiler", "-fPIC,-O2", "-Xptxas", "-v", "--expt-relaxed-constexpr"]


def _stale() -> bool:
    if not os.path.exists(OUT):
        return True
    t = os.path.getmtime(OUT)
    srcs = [os.path.join(HERE, s) for s in DEPS] + [os.path.join(INC, h) for h in HEADERS]
    return any(os.path.getmtime(s) > t for s in srcs)


def build(force: bool = False, verbose: bool = False, defines=(), out: str | None = None) -> str:
    """Build libproact.so; `defines` (e.g. ["PROACT_JACOBI_RING=8"]) + `out` build a variant."""
    global OUT
    if out is not None:
        saved, OUT = OUT, out
        try:
            return build(True, verbose, defines)
        finally:
            OUT = saved
    if not force and not _stale():
        return OUT
    objs = []
    for s in SOURCES:
        obj = os.path.join(HERE, s.replace(".cu", f".{os.getpid()}.o"))   # parallel variant builds
        cmd = [NVCC, *FLAGS, *[f"-D{d}" for d in defines], "-I", INC, "-c", os.path.join(HERE, s), "-o", obj]
        r = subprocess.run(cmd, capture_output=True, text=True)
        if r.returncode != 0:
            sys.stderr.write(r.stdout + r.stderr)
            raise RuntimeError(f"nvcc failed on {s}")
        if verbose:
            sys.stderr.write(r.stderr)
        objs.append(obj)
    tmp = OUT + f".tmp{os.getpid()}"
    cmd = [NVCC, "-gencode", "arch=compute_100a,code=sm_100a", "-shared", "-o", tmp, *objs,
           "-lrt"]
    r = subprocess.run(cmd, capture_output=True, text=True)
    if r.returncode != 0:
        sys.stderr.write(r.stdout + r.stderr)
        raise RuntimeError("nvcc link failed")
    os.replace(tmp, OUT)
    for o in objs:
        os.remove(o)
    return OUT


if __name__ == "__main__":
    # python build.py [-f] [-v] [-o OUT.so] [-D NAME=VALUE ...]
    argv = sys.argv[1:]
    defs, out = [], None
    for i, a in enumerate(argv):
        if a == "-D":
            defs.append(argv[i + 1])
        if a == "-o":
            out = argv[i + 1]
    print(build(force="-f" in argv, verbose="-v" in argv, defines=defs, out=out))
