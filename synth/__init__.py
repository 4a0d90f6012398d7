"""Seeded synthetic input generators shared by the oracle and the CUDA path.

This module holds none of the method's arithmetic (see synth.c's header): it
only produces the inputs -- the Jacobi grid, the RMAT edge list (stand-in for
the Wikipedia / HV15R datasets of PAPER.md Sec. IV-C), SSSP edge
weights -- so that both sides consume byte-identical data.  The recipes are in
DESIGN.md Sec. "Input recipe".
"""
from __future__ import annotations

import ctypes
import os
import subprocess

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SRC = os.path.join(_HERE, "synth.c")
_LIB = os.path.join(_HERE, "libsynth.so")
_lib = None

# Seeds named in SURVEY.md Sec. 8(d) / DESIGN.md.
JACOBI_SEED = 0x1CA21
RMAT_SEED = 1
PERM_SEED = 2
WEIGHT_SEED = 3
MICRO_SEED = 0x5EED
BANDED_SEED = 0xBA4D


def build(force: bool = False) -> str:
    """Compile libsynth.so with gcc (OpenMP)."""
    if force or not os.path.exists(_LIB) or os.path.getmtime(_LIB) < os.path.getmtime(_SRC):
        tmp = _LIB + f".tmp{os.getpid()}"
        subprocess.check_call(["gcc", "-O2", "-std=c11", "-fopenmp", "-fPIC", "-shared",
                               "-o", tmp, _SRC])
        os.replace(tmp, _LIB)
    return _LIB


def lib():
    global _lib
    if _lib is None:
        build()
        L = ctypes.CDLL(_LIB)
        u64, i64, vp = ctypes.c_uint64, ctypes.c_int64, ctypes.c_void_p
        L.synth_splitmix64.restype = u64
        L.synth_splitmix64.argtypes = [u64]
        L.synth_jacobi_init.restype = None
        L.synth_jacobi_init.argtypes = [vp, i64, i64, i64, u64]
        L.synth_permutation.restype = None
        L.synth_permutation.argtypes = [vp, i64, u64]
        L.synth_rmat.restype = i64
        L.synth_rmat.argtypes = [vp, vp, ctypes.c_int, i64, u64, u64]
        L.synth_banded.restype = None
        L.synth_banded.argtypes = [vp, vp, i64, i64, u64]
        L.synth_weights.restype = None
        L.synth_weights.argtypes = [vp, i64, u64]
        _lib = L
    return _lib


def _ptr(a: np.ndarray) -> int:
    assert a.flags["C_CONTIGUOUS"]
    return a.ctypes.data


def splitmix64(x: int) -> int:
    return int(lib().synth_splitmix64(x & 0xFFFFFFFFFFFFFFFF))


def jacobi_init(N: int, seed: int = JACOBI_SEED, row0: int = 0, nrows: int | None = None,
                out: np.ndarray | None = None) -> np.ndarray:
    """Rows [row0, row0+nrows) of the N x N fp32 initial grid, values exact in [1, 2)."""
    if nrows is None:
        nrows = N - row0
    if out is None:
        out = np.empty((nrows, N), dtype=np.float32)
    assert out.dtype == np.float32 and out.size == nrows * N
    lib().synth_jacobi_init(_ptr(out), N, row0, nrows, seed)
    return out


def permutation(V: int, seed: int = PERM_SEED) -> np.ndarray:
    p = np.empty(V, dtype=np.uint32)
    lib().synth_permutation(_ptr(p), V, seed)
    return p


def rmat(scale: int, edge_factor: int = 16, seed: int = RMAT_SEED,
         perm_seed: int = PERM_SEED) -> tuple[np.ndarray, np.ndarray]:
    """RMAT edge list (src, dst) as uint32, self loops removed, duplicates kept."""
    E0 = (1 << scale) * edge_factor
    src = np.empty(E0, dtype=np.uint32)
    dst = np.empty(E0, dtype=np.uint32)
    k = lib().synth_rmat(_ptr(src), _ptr(dst), scale, edge_factor, seed, perm_seed)
    if k < 0:
        raise MemoryError("synth_rmat: allocation failed")
    return src[:k], dst[:k]


def weights(E: int, seed: int = WEIGHT_SEED) -> np.ndarray:
    w = np.empty(E, dtype=np.int32)
    if E:
        lib().synth_weights(_ptr(w), E, seed)
    return w


def banded(N: int, w: int, seed: int = BANDED_SEED) -> tuple[np.ndarray, np.ndarray]:
    """Banded system in DIA layout: a[(o+w), i] = A[i][i+o] (shape (2w+1, N)), and b (N)."""
    a = np.empty((2 * w + 1, N), dtype=np.float32)
    b = np.empty(N, dtype=np.float32)
    if N:
        lib().synth_banded(_ptr(a), _ptr(b), N, w, seed)
    return a, b
