"""Thin Python face of include/proact.h (argument marshalling only).

PyTorch supplies device memory (tensors), streams and process groups; every
protocol step runs inside libproact.  Functions raise ProactError on a negative
status.  All calls act on the calling thread's rank context.
"""
from __future__ import annotations

import ctypes
import os
import uuid

import torch

from . import _lib
from ._lib import Config, ProactError, RegionInfo, check


def lib():
    return _lib.load()


def _stream_handle(stream) -> int:
    if stream is None:
        stream = torch.cuda.current_stream()
    return int(stream.cuda_stream) if hasattr(stream, "cuda_stream") else int(stream)


# ------------------------------------------------------------------ lifecycle
def init(world: int, rank: int | None = None, job: str | None = None) -> int:
    """COLLECTIVE: proact_init_ex.  rank defaults to $RANK / the current device; job to
    $PROACT_JOB, then $MASTER_ADDR:$MASTER_PORT."""
    L = lib()
    if torch.cuda.is_available():
        torch.cuda.init()
    if rank is None and job is None:
        return check(L.proact_init(world), "proact_init")
    if rank is None:
        rank = int(os.environ.get("RANK", torch.cuda.current_device()))
    if job is None:
        job = os.environ.get("PROACT_JOB") or (
            f"{os.environ.get('MASTER_ADDR', '')}:{os.environ['MASTER_PORT']}"
            if "MASTER_PORT" in os.environ else "default")
    return check(L.proact_init_ex(world, rank, job.encode()), "proact_init_ex")


def new_job_key() -> str:
    return "job" + uuid.uuid4().hex[:16]


def finalize() -> None:
    check(lib().proact_finalize(), "proact_finalize")


def rank() -> int:
    return lib().proact_rank()


def world() -> int:
    return lib().proact_world()


def ranks_on_device() -> int:
    return lib().proact_ranks_on_device()


def get_config() -> dict:
    c = Config()
    check(lib().proact_get_config(ctypes.byref(c)), "proact_get_config")
    return c.as_dict()


def set_config(**kw) -> dict:
    """Update fields of the rank's config (mech, push, agent_warps, block, piece_bytes,
    watchdog_ms, grid_cap, chunk_bytes)."""
    c = Config()
    check(lib().proact_get_config(ctypes.byref(c)), "proact_get_config")
    for k, v in kw.items():
        if not hasattr(c, k):
            raise KeyError(k)
        setattr(c, k, int(v))
    check(lib().proact_set_config(ctypes.byref(c)), "proact_set_config")
    return c.as_dict()


def reset_config() -> None:
    check(lib().proact_set_config(None), "proact_set_config")


# ------------------------------------------------------------------ NVLS multicast replicas
def mcast_supported() -> bool:
    return bool(lib().proact_mcast_supported())


class _CudaArray:
    """Minimal __cuda_array_interface__ exporter: a torch view of library-owned device memory."""

    def __init__(self, ptr: int, shape, typestr: str):
        self.__cuda_array_interface__ = {"shape": tuple(shape), "typestr": typestr, "data": (ptr, False),
                                         "version": 3, "strides": None}


def alloc_replica(shape, dtype=torch.float32) -> torch.Tensor:
    """COLLECTIVE proact_alloc_replica: a full-extent replica (bound to an NVLS multicast object
    when mcast_supported() on every rank) as a torch tensor view; release with free_replica."""
    n = 1
    for d in shape:
        n *= d
    nbytes = n * torch.empty(0, dtype=dtype).element_size()
    ptr = ctypes.c_void_p(0)
    check(lib().proact_alloc_replica(nbytes, ctypes.byref(ptr)), "proact_alloc_replica")
    typestr = {torch.float32: "<f4", torch.int32: "<i4", torch.uint8: "|u1"}[dtype]
    t = torch.as_tensor(_CudaArray(ptr.value, shape, typestr), device="cuda")
    assert t.data_ptr() == ptr.value
    return t


def free_replica(t: torch.Tensor) -> None:
    check(lib().proact_free_replica(ctypes.c_void_p(t.data_ptr())), "proact_free_replica")


# ------------------------------------------------------------------ regions
def register_region(replica: torch.Tensor, own_offset: int, own_bytes: int, chunk_bytes: int,
                    dest_mask: int | None = None, flags: int = 0) -> int:
    """COLLECTIVE.  `replica` is this rank's full-extent local replica (rank-ordered slices);
    [own_offset, own_offset+own_bytes) is my owned slice.  dest_mask None = all ranks."""
    assert replica.is_cuda and replica.is_contiguous()
    if dest_mask is None:
        dest_mask = (1 << world()) - 1
    ptr = replica.data_ptr() + own_offset
    rid = check(lib().proact_register_region_ex(ctypes.c_void_p(ptr), own_bytes, chunk_bytes,
                                                dest_mask, flags), "proact_register_region")
    info = region_info(rid)
    if info.replica_base != replica.data_ptr() or info.total_bytes != replica.numel() * replica.element_size():
        raise ProactError(_lib.ERR_INVALID, "replica layout != rank-ordered concatenation of slices")
    return rid


def region_info(rid: int) -> RegionInfo:
    info = RegionInfo()
    check(lib().proact_region_info_get(rid, ctypes.byref(info)), "proact_region_info_get")
    return info


def set_chunk_dest(rid: int, chunk: int, mask: int) -> None:
    check(lib().proact_region_set_chunk_dest(rid, chunk, mask), "proact_region_set_chunk_dest")


def rechunk(rid: int, chunk_bytes: int) -> None:
    check(lib().proact_region_rechunk(rid, chunk_bytes), "proact_region_rechunk")


def debug_deliveries(rid: int):
    import numpy as np
    info = region_info(rid)
    n = info.n_own_chunks * world()
    out = np.zeros(max(n, 1), dtype=np.uint32)
    check(lib().proact_region_debug_deliveries(
        rid, out.ctypes.data_as(ctypes.POINTER(ctypes.c_uint32)), out.size), "debug_deliveries")
    return out[:n].reshape(info.n_own_chunks, world())


def debug_state(rid: int) -> dict:
    """proact_region_debug_state as numpy arrays (post-mortem after a watchdog timeout)."""
    import numpy as np
    info = region_info(rid)
    n_own, n_total = info.n_own_chunks, info.n_total_chunks
    buf = np.zeros(3 * n_own + n_total + 8 + 32, dtype=np.uint32)
    check(lib().proact_region_debug_state(rid, ctypes.c_void_p(buf.ctypes.data), buf.size), "debug_state")
    o = 0
    out = {}
    for k, n in (("counter", n_own), ("expected", n_own), ("piecedone", n_own), ("arrive", n_total),
                 ("qctl", 8), ("done", 16), ("host", 16)):
        out[k] = buf[o:o + n].copy()
        o += n
    return out


# ------------------------------------------------------------------ phases
def phase_sync(stream=None, barrier: bool = False) -> None:
    check(lib().proact_phase_sync(ctypes.c_void_p(_stream_handle(stream)),
                                  _lib.SYNC_BARRIER if barrier else _lib.SYNC_SIGNAL),
          "proact_phase_sync")


def last_vote() -> int:
    return lib().proact_last_vote()


def host_barrier() -> None:
    check(lib().proact_host_barrier(), "proact_host_barrier")


def check_device() -> None:
    check(lib().proact_check(), "proact_check")


def launch_count() -> int:
    return int(lib().proact_launch_count())


def epoch() -> int:
    return int(lib().proact_epoch())


def autotune(key: str, run, space: str | None = None) -> dict:
    """COLLECTIVE brute-force profiler (proact_autotune).  run(cfg: dict) -> ms."""
    def _cb(cfgp, _user):
        try:
            return float(run(cfgp.contents.as_dict()))
        except Exception:   # a failing point is skipped, not fatal
            return -1.0
    cb = _lib.RUN_FN(_cb)
    out = Config()
    check(lib().proact_autotune(key.encode(), space.encode() if space else None, cb, None,
                                ctypes.byref(out)), "proact_autotune")
    return out.as_dict()
