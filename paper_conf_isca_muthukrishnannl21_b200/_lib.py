"""ctypes binding of libproact.so (argument marshalling only).

Every step of the hot path runs in the library's CUDA kernels; this module only
declares the C signatures of include/proact.h and include/proact_workloads.h.
There is no fallback: if the shared library is missing or cannot be loaded the
import fails loudly (build it with __graft_entry__.build()).
"""
from __future__ import annotations

import ctypes
import os

_HERE = os.path.dirname(os.path.abspath(__file__))
# PROACT_LIB: an alternative build of the same library (tools/ variant sweeps only)
LIB_PATH = os.environ.get("PROACT_LIB") or os.path.join(_HERE, "libproact.so")

MAX_RANKS = 16
MAX_REGIONS = 8

OK = 0
ERR_INVALID, ERR_CUDA, ERR_NOPEER, ERR_STATE, ERR_TIMEOUT, ERR_PROTOCOL, ERR_NOMEM = range(-1, -8, -1)

MECH_FUSED, MECH_INLINE, MECH_BULK, MECH_LOCAL, MECH_ELIDE, MECH_DMA = range(6)
MECH_NAMES = {MECH_FUSED: "fused", MECH_INLINE: "inline", MECH_BULK: "bulk",
              MECH_LOCAL: "local", MECH_ELIDE: "elide", MECH_DMA: "dma"}
PUSH_VEC16, PUSH_BULK, PUSH_MULTICAST = 0, 1, 2
DISCOVER_QUEUE, DISCOVER_SCAN = 0, 1
AGENT_FUSED, AGENT_SEPARATE, AGENT_PRODUCER = 0, 1, 2
LAUNCH_TILE_PUSH = 1
SYNC_SIGNAL, SYNC_BARRIER = 0, 1
REGION_SPARSE = 1


class ProactError(RuntimeError):
    def __init__(self, code: int, what: str = ""):
        self.code = code
        name = _lib.proact_error_string(code).decode() if _lib is not None else str(code)
        super().__init__(f"{what}: {name} ({code})" if what else f"{name} ({code})")


class Config(ctypes.Structure):
    _fields_ = [("mech", ctypes.c_int32), ("push", ctypes.c_int32),
                ("agent_warps", ctypes.c_int32), ("block", ctypes.c_int32),
                ("piece_bytes", ctypes.c_uint32), ("watchdog_ms", ctypes.c_uint32),
                ("grid_cap", ctypes.c_int32), ("chunk_bytes", ctypes.c_uint32),
                ("discovery", ctypes.c_int32), ("agent_kernel", ctypes.c_int32)]

    def as_dict(self) -> dict:
        return {k: getattr(self, k) for k, _ in self._fields_}


class RegionInfo(ctypes.Structure):
    _fields_ = [("replica_base", ctypes.c_void_p), ("own_offset", ctypes.c_uint64),
                ("own_bytes", ctypes.c_uint64), ("total_bytes", ctypes.c_uint64),
                ("chunk_bytes", ctypes.c_uint64), ("n_own_chunks", ctypes.c_uint32),
                ("n_total_chunks", ctypes.c_uint32), ("first_chunk", ctypes.c_uint32),
                ("generation", ctypes.c_uint32), ("dest_mask", ctypes.c_uint64),
                ("rank_offset", ctypes.c_uint64 * (MAX_RANKS + 1))]


RUN_FN = ctypes.CFUNCTYPE(ctypes.c_double, ctypes.POINTER(Config), ctypes.c_void_p)

_lib = None


def _declare(L):
    i, u32, u64, sz, vp, cp = (ctypes.c_int, ctypes.c_uint32, ctypes.c_uint64, ctypes.c_size_t,
                               ctypes.c_void_p, ctypes.c_char_p)
    sigs = {
        "proact_init": (i, [i]),
        "proact_init_ex": (i, [i, i, cp]),
        "proact_finalize": (i, []),
        "proact_rank": (i, []),
        "proact_world": (i, []),
        "proact_ranks_on_device": (i, []),
        "proact_error_string": (cp, [i]),
        "proact_last_cuda_error": (i, []),
        "proact_set_config": (i, [ctypes.POINTER(Config)]),
        "proact_get_config": (i, [ctypes.POINTER(Config)]),
        "proact_register_region": (i, [vp, sz, sz, u64]),
        "proact_register_region_ex": (i, [vp, sz, sz, u64, u32]),
        "proact_region_set_chunk_dest": (i, [i, u32, u64]),
        "proact_region_info_get": (i, [i, ctypes.POINTER(RegionInfo)]),
        "proact_region_rechunk": (i, [i, sz]),
        "proact_region_debug_deliveries": (i, [i, ctypes.POINTER(u32), sz]),
        "proact_launch": (i, [ctypes.POINTER(i), i, vp, ctypes.c_uint, ctypes.c_uint,
                              ctypes.POINTER(vp), sz, vp]),
        "proact_phase_sync": (i, [vp, i]),
        "proact_launch_tallies": (i, []),
        "proact_launch_mode": (i, []),
        "proact_launch_ex": (i, [ctypes.POINTER(ctypes.c_int), i, vp, ctypes.c_uint, ctypes.c_uint,
                                 ctypes.POINTER(vp), sz, vp, ctypes.c_uint]),
        "proact_last_vote": (i, []),
        "proact_check": (i, []),
        "proact_host_barrier": (i, []),
        "proact_debug_agent_prof": (i, [ctypes.POINTER(ctypes.c_ulonglong)]),
        "proact_launch_count": (u64, []),
        "proact_plan_slices": (i, [i, ctypes.POINTER(u64), u64, ctypes.POINTER(u64), ctypes.POINTER(u32)]),
        "proact_rdv_allgather": (i, [cp, i, i, vp, sz, vp]),
        "proact_partition_bounds": (i, [vp, ctypes.c_uint, i, ctypes.c_uint, ctypes.POINTER(ctypes.c_uint)]),
        "proact_epoch": (u32, []),
        "proact_autotune": (i, [cp, cp, RUN_FN, vp, ctypes.POINTER(Config)]),
        # workloads
        "proact_jacobi_phase": (i, [i, i, ctypes.c_longlong, i, vp]),
        "proact_micro_phase": (i, [i, ctypes.c_uint, ctypes.c_uint, i, i, vp]),
        "proact_litmus_phase": (i, [i, i, ctypes.c_uint, ctypes.c_uint, vp, vp]),
        "proact_region_debug_state": (i, [i, vp, sz]),
        "proact_mcast_supported": (i, []),
        "proact_alloc_replica": (i, [sz, ctypes.POINTER(vp)]),
        "proact_free_replica": (i, [vp]),
        "proact_inject_double_commit": (i, [i, vp]),
        "proact_banded_phase": (i, [i, i, vp, vp, ctypes.c_longlong, ctypes.c_longlong, vp]),
        "proact_jacobi_solve_host": (i, [vp, vp, ctypes.c_longlong, i, sz, i, vp,
                                         ctypes.POINTER(ctypes.c_ulonglong),
                                         ctypes.POINTER(ctypes.c_ulonglong)]),
        "proact_jacobi_solve_host_pipelined": (i, [vp, vp, i, ctypes.c_longlong, i, sz, i, vp,
                                                   ctypes.POINTER(ctypes.c_ulonglong),
                                                   ctypes.POINTER(ctypes.c_ulonglong)]),
        "proact_graph_partition": (i, [vp, ctypes.c_ulonglong, ctypes.c_uint, i, ctypes.c_uint,
                                       ctypes.POINTER(ctypes.c_uint), vp]),
        "proact_graph_build": (i, [vp, vp, vp, ctypes.c_ulonglong, ctypes.c_uint, ctypes.c_uint,
                                   ctypes.c_uint, vp]),
        "proact_graph_build_ex": (i, [vp, vp, vp, ctypes.c_ulonglong, ctypes.c_uint, ctypes.c_uint,
                                      ctypes.c_uint, i, vp]),
        "proact_graph_hot": (i, [i, ctypes.POINTER(ctypes.c_uint), ctypes.POINTER(ctypes.c_ulonglong)]),
        "proact_graph_free": (i, [i]),
        "proact_graph_info": (i, [i, ctypes.POINTER(ctypes.c_ulonglong), ctypes.POINTER(ctypes.c_uint),
                                  ctypes.POINTER(ctypes.c_uint)]),
        "proact_pagerank_init": (i, [i, i, vp]),
        "proact_pagerank_phase": (i, [i, i, i, ctypes.c_double, vp]),
        "proact_pagerank_ranks": (i, [i, vp, vp]),
        "proact_sssp_phase": (i, [i, i, i, i, vp]),
        "proact_sssp_last_mode": (i, [i]),
    }
    missing = []
    for name, (res, args) in sigs.items():
        try:
            f = getattr(L, name)
        except AttributeError:
            if LIB_PATH.endswith("libproact.so") and "PROACT_LIB" not in os.environ:
                raise
            missing.append(name)   # an older variant build (tools/ sweeps): tolerate
            continue
        f.restype = res
        f.argtypes = args
    return sorted(set(sigs) - set(missing))


EXPORTED: list[str] = []


def load():
    """Load libproact.so (raises if it is missing: there is no CPU fallback)."""
    global _lib, EXPORTED
    if _lib is None:
        if not os.path.exists(LIB_PATH):
            raise ImportError(f"{LIB_PATH} is missing: run __graft_entry__.build() "
                              "(the CUDA path has no fallback)")
        L = ctypes.CDLL(LIB_PATH)
        EXPORTED = _declare(L)
        _lib = L
    return _lib


def check(rc: int, what: str = "") -> int:
    if rc < 0:
        raise ProactError(rc, what)
    return rc
