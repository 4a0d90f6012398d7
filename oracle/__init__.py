"""CPU oracle for the PROACT hot path -- TEST INFRASTRUCTURE ONLY.

Only tests/, __graft_entry__.smoke() and bench.py's cpu_baseline / --impl
reference legs may import this package.  The product path
(paper_conf_isca_muthukrishnannl21_b200) never does, and shares no code with
it; see oracle.c's header for the passages each function follows.

Functions with no independent pin are listed here (none at present): every
function below is pinned by a test in tests/test_oracle_*.py against something
other than itself (published hash vectors, closed forms, a dense linear solve,
Dijkstra / dense min-plus brute force, invariants).
"""
from __future__ import annotations

import ctypes
import os
import subprocess

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SRC = os.path.join(_HERE, "oracle.c")
_LIB = os.path.join(_HERE, "liboracle.so")
_lib = None

DAMPING = 0.85          # reading R11: PageRank damping factor
INF = np.iinfo(np.int32).max


def build(force: bool = False) -> str:
    if force or not os.path.exists(_LIB) or os.path.getmtime(_LIB) < os.path.getmtime(_SRC):
        tmp = _LIB + f".tmp{os.getpid()}"
        subprocess.check_call(["gcc", "-O2", "-std=c11", "-fopenmp", "-fPIC", "-shared",
                               "-ffp-contract=off", "-o", tmp, _SRC, "-lpthread"])
        os.replace(tmp, _LIB)
    return _LIB


def lib():
    global _lib
    if _lib is None:
        build()
        L = ctypes.CDLL(_LIB)
        u32, i32, u64, i64, vp = (ctypes.c_uint32, ctypes.c_int, ctypes.c_uint64,
                                  ctypes.c_int64, ctypes.c_void_p)
        L.oracle_set_threads.restype = None
        L.oracle_set_threads.argtypes = [i32]
        L.oracle_get_threads.restype = i32
        L.oracle_get_threads.argtypes = []
        L.oracle_fmix32.restype = u32
        L.oracle_fmix32.argtypes = [u32]
        L.oracle_micro_word.restype = u32
        L.oracle_micro_word.argtypes = [u64, u32, u32, i32]
        L.oracle_micro_phase.restype = None
        L.oracle_micro_phase.argtypes = [vp, i64, u32, u32, i32]
        L.oracle_jacobi_step.restype = None
        L.oracle_jacobi_step.argtypes = [vp, vp, i64]
        L.oracle_jacobi.restype = i32
        L.oracle_jacobi.argtypes = [vp, i64, i32]
        L.oracle_pagerank.restype = i32
        L.oracle_pagerank.argtypes = [i64, i64, vp, vp, i32, ctypes.c_double, vp,
                                      ctypes.POINTER(ctypes.c_double)]
        L.oracle_sssp.restype = i32
        L.oracle_sssp.argtypes = [i64, i64, vp, vp, vp, i64, i32, vp, ctypes.POINTER(i32), vp,
                                  ctypes.POINTER(ctypes.c_double)]
        L.oracle_banded_jacobi.restype = i32
        L.oracle_banded_jacobi.argtypes = [vp, vp, vp, i64, i64, i32]
        L.oracle_proto_run.restype = i32
        L.oracle_proto_run.argtypes = [i32, i32, i32, i32, i64, i64, i64, i32, u32, i32, u64, vp, vp]
        _lib = L
    return _lib


def _p(a: np.ndarray) -> int:
    assert a.flags["C_CONTIGUOUS"]
    return a.ctypes.data


def set_threads(n: int) -> None:
    """OpenMP thread count for subsequent oracle calls (results do not depend on it)."""
    lib().oracle_set_threads(int(n))


def get_threads() -> int:
    return int(lib().oracle_get_threads())


# ---------------------------------------------------------------- microbenchmark (L259-L261)
def fmix32(h: int) -> int:
    return int(lib().oracle_fmix32(h & 0xFFFFFFFF))


def micro_word(k: int, phase: int, seed: int, K: int = 1) -> int:
    return int(lib().oracle_micro_word(k, phase & 0xFFFFFFFF, seed & 0xFFFFFFFF, K))


def micro_phase(W: int, phase: int, seed: int, K: int = 1) -> np.ndarray:
    out = np.empty(W, dtype=np.uint32)
    if W:
        lib().oracle_micro_phase(_p(out), W, phase & 0xFFFFFFFF, seed & 0xFFFFFFFF, K)
    return out


# ---------------------------------------------------------------- Jacobi (L271)
def jacobi_step(x: np.ndarray) -> np.ndarray:
    x = np.ascontiguousarray(x, dtype=np.float32)
    N = x.shape[0]
    out = np.empty_like(x)
    lib().oracle_jacobi_step(_p(x), _p(out), N)
    return out


def jacobi(x0: np.ndarray, iters: int) -> np.ndarray:
    x = np.array(x0, dtype=np.float32, copy=True, order="C")
    assert x.ndim == 2 and x.shape[0] == x.shape[1]
    if lib().oracle_jacobi(_p(x), x.shape[0], iters) != 0:
        raise MemoryError("oracle_jacobi")
    return x


def banded_jacobi(a: np.ndarray, b: np.ndarray, x0: np.ndarray, iters: int) -> np.ndarray:
    """Banded Jacobi (NEXT-2, L271): a is the DIA array (2w+1, N), b and x0 length N."""
    a = np.ascontiguousarray(a, dtype=np.float32)
    b = np.ascontiguousarray(b, dtype=np.float32)
    x = np.array(x0, dtype=np.float32, copy=True)
    w = (a.shape[0] - 1) // 2
    if lib().oracle_banded_jacobi(_p(a), _p(b), _p(x), x.size, w, iters) != 0:
        raise MemoryError("oracle_banded_jacobi")
    return x


# ---------------------------------------------------------------- PageRank (L265)
def pagerank(V: int, src: np.ndarray, dst: np.ndarray, iters: int,
             d: float = DAMPING, timing: dict | None = None) -> np.ndarray:
    """r^{iters}; timing (optional dict) receives "iter_seconds": the iterations alone."""
    src = np.ascontiguousarray(src, dtype=np.uint32)
    dst = np.ascontiguousarray(dst, dtype=np.uint32)
    r = np.empty(V, dtype=np.float32)
    t = ctypes.c_double(0.0)
    if lib().oracle_pagerank(V, src.size, _p(src), _p(dst), iters, d, _p(r), ctypes.byref(t)) != 0:
        raise MemoryError("oracle_pagerank")
    if timing is not None:
        timing["iter_seconds"] = t.value
    return r


# ---------------------------------------------------------------- SSSP (L267)
def sssp(V: int, src: np.ndarray, dst: np.ndarray, w: np.ndarray, s: int,
         max_rounds: int = 0, timing: dict | None = None) -> tuple[np.ndarray, int, np.ndarray]:
    """Synchronous Bellman-Ford; returns (d, rounds, changed_per_round); timing (optional dict)
    receives "iter_seconds": the rounds alone (the CSC build is input preparation)."""
    src = np.ascontiguousarray(src, dtype=np.uint32)
    dst = np.ascontiguousarray(dst, dtype=np.uint32)
    w = np.ascontiguousarray(w, dtype=np.int32)
    d = np.empty(V, dtype=np.int32)
    cap = max_rounds if max_rounds > 0 else max(V, 1)
    changed = np.zeros(cap + 1, dtype=np.int64)
    rounds = ctypes.c_int(0)
    t = ctypes.c_double(0.0)
    if lib().oracle_sssp(V, src.size, _p(src), _p(dst), _p(w), s, max_rounds, _p(d),
                         ctypes.byref(rounds), _p(changed), ctypes.byref(t)) != 0:
        raise MemoryError("oracle_sssp")
    if timing is not None:
        timing["iter_seconds"] = t.value
    return d, rounds.value, changed[:rounds.value]


# ---------------------------------------------------------------- O-proto (Sec. III-B/C)
PROTO_ERRORS = {
    -1: "I1 violated: a (chunk, dest) was not delivered exactly once in a phase",
    -2: "I2 violated: a readiness counter over-counted or was not reset",
    -3: "I3 violated: an arrival flag does not carry the last generation",
}


def proto_run(G: int, workload: str, size: int, chunk_words: int, tile_words: int,
              phases: int, P: int = 3, A: int = 2, seed: int = 0x5EED, K: int = 1,
              rng_seed: int = 1, init: np.ndarray | None = None) -> tuple[int, np.ndarray]:
    """Simulate G ranks running `phases` PROACT phases; returns (rc, replicas[G, words])."""
    wl = {"micro": 0, "jacobi": 1}[workload]
    W = size * size if wl == 1 else size
    out = np.empty((G, W), dtype=np.uint32)
    ip = None
    if init is not None:
        init = np.ascontiguousarray(init).view(np.uint32).reshape(-1)
        assert init.size == W
        ip = _p(init)
    rc = lib().oracle_proto_run(G, P, A, wl, size, chunk_words, tile_words, phases,
                                seed & 0xFFFFFFFF, K, rng_seed, ip, _p(out))
    return rc, out
