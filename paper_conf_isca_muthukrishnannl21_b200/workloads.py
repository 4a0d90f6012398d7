"""Workload drivers over the C entry points of include/proact_workloads.h.

Host-side orchestration only (allocation through torch, region registration,
the phase loop); the arithmetic of every phase runs in libproact's kernels.
"""
from __future__ import annotations

import ctypes

import torch

from . import _lib
from . import runtime as rt
from ._lib import check


def _s(stream) -> ctypes.c_void_p:
    return ctypes.c_void_p(rt._stream_handle(stream))


def row_split(N: int, G: int, g: int) -> tuple[int, int]:
    """Rows of rank g: [g*N//G, (g+1)*N//G) (also proact_jacobi_solve_host's split)."""
    return (N * g) // G, (N * (g + 1)) // G


# ------------------------------------------------------------------ Jacobi (configs 1-2)
def jacobi_phase(r_in: int, r_out: int, N: int, rows_per_tile: int = 16, stream=None) -> None:
    check(rt.lib().proact_jacobi_phase(r_in, r_out, N, rows_per_tile, _s(stream)), "jacobi_phase")


class Jacobi:
    """Two replicated N x N fp32 grids (ping-pong), rows partitioned over the world.

    halo_only=True sets per-chunk destinations so that only chunks holding my first/last row
    go to the neighbours (reading R8); otherwise full replication (configs 1-2)."""

    def __init__(self, N: int, chunk_bytes: int, x0: torch.Tensor | None = None,
                 halo_only: bool = False, rows_per_tile: int = 16, device=None, mcast: bool = False):
        """mcast=True: the two replicas come from proact_alloc_replica (COLLECTIVE), bound to NVLS
        multicast objects when the system supports it (push=PUSH_MULTICAST then stores once for
        all peers); release them with free()."""
        G, g = rt.world(), rt.rank()
        self.N, self.G, self.g, self.rpt = N, G, g, rows_per_tile
        dev = device if device is not None else torch.device("cuda", torch.cuda.current_device())
        self.mcast = mcast
        if mcast:
            self.bufs = [rt.alloc_replica((N, N), torch.float32) for _ in range(2)]
        else:
            self.bufs = [torch.empty((N, N), dtype=torch.float32, device=dev) for _ in range(2)]
        if x0 is not None:
            self.bufs[0].copy_(x0)
            self.bufs[1].copy_(x0)
        # replicas must be initialised before registration: once the collective returns, peers
        # may push into them (credits only guard later generations)
        torch.cuda.synchronize()
        self.r0, self.r1 = row_split(N, G, g)
        rowb = N * 4
        self.rid = [rt.register_region(b, self.r0 * rowb, (self.r1 - self.r0) * rowb, chunk_bytes)
                    for b in self.bufs]
        if halo_only:
            self.set_halo_only()
        self.k = 0

    def set_halo_only(self) -> None:
        rowb = self.N * 4
        for rid in self.rid:
            info = rt.region_info(rid)
            cb = info.chunk_bytes
            n = info.n_own_chunks
            for c in range(n):
                lo, hi = c * cb, min((c + 1) * cb, info.own_bytes)
                m = 0
                if self.g > 0 and lo < rowb:                       # holds my first row
                    m |= 1 << (self.g - 1)
                if self.g < self.G - 1 and hi > info.own_bytes - rowb:  # holds my last row
                    m |= 1 << (self.g + 1)
                rt.set_chunk_dest(rid, c, m)

    def free(self) -> None:
        """COLLECTIVE when mcast: release library-allocated replicas (after the last phase)."""
        torch.cuda.synchronize()
        if self.mcast:
            for b in self.bufs:
                rt.free_replica(b)
        self.bufs = []

    def step(self, stream=None, barrier: bool = False) -> None:
        i = self.k & 1
        jacobi_phase(self.rid[i], self.rid[i ^ 1], self.N, self.rpt, stream)
        rt.phase_sync(stream, barrier=barrier)
        self.k += 1

    def step_allgather(self, stream=None, group=None) -> None:
        """BASELINE (north star: "a bulk ... NCCL-allgather version between kernels"): the
        uninstrumented phase kernel (config mech must be LOCAL), then an in-place NCCL all-gather
        of the rows into every replica, then the phase sync.  Equal row slices required."""
        import torch.distributed as dist
        i = self.k & 1
        if self.N % self.G:
            raise ValueError("all-gather baseline needs N divisible by the world size")
        jacobi_phase(self.rid[i], self.rid[i ^ 1], self.N, self.rpt, stream)
        out = self.bufs[i ^ 1].view(-1)
        mine = out[self.r0 * self.N:self.r1 * self.N]
        if self.G > 1:
            with torch.cuda.stream(stream) if stream is not None else _nullctx():
                dist.all_gather_into_tensor(out, mine, group=group)
        rt.phase_sync(stream, barrier=False)
        self.k += 1

    @property
    def current(self) -> torch.Tensor:
        return self.bufs[self.k & 1]


class _nullctx:
    def __enter__(self):
        return self

    def __exit__(self, *a):
        return False


def jacobi_solve_host(x0_host, out_host, N: int, iters: int, chunk_bytes: int,
                      rows_per_tile: int = 16, stream=None) -> tuple[int, int]:
    """proact_jacobi_solve_host on host buffers (torch CPU tensors, ideally pinned)."""
    assert x0_host.dtype == torch.float32 and out_host.dtype == torch.float32
    assert x0_host.is_contiguous() and out_host.is_contiguous()
    h2d, d2h = ctypes.c_ulonglong(0), ctypes.c_ulonglong(0)
    check(rt.lib().proact_jacobi_solve_host(ctypes.c_void_p(x0_host.data_ptr()),
                                            ctypes.c_void_p(out_host.data_ptr()), N, iters,
                                            chunk_bytes, rows_per_tile, _s(stream),
                                            ctypes.byref(h2d), ctypes.byref(d2h)), "jacobi_solve_host")
    return h2d.value, d2h.value


def jacobi_solve_host_pipelined(x0_host, outs_host, N: int, iters: int, chunk_bytes: int,
                                rows_per_tile: int = 16, stream=None) -> tuple[int, int]:
    """proact_jacobi_solve_host_pipelined: len(outs_host) solves of x0_host, pipelined; complete
    when `stream` is.  Returns the per-solve H2D / D2H byte counts."""
    assert x0_host.dtype == torch.float32 and x0_host.is_contiguous()
    for o in outs_host:
        assert o.dtype == torch.float32 and o.is_contiguous()
    ptrs = (ctypes.c_void_p * len(outs_host))(*[o.data_ptr() for o in outs_host])
    h2d, d2h = ctypes.c_ulonglong(0), ctypes.c_ulonglong(0)
    check(rt.lib().proact_jacobi_solve_host_pipelined(ctypes.c_void_p(x0_host.data_ptr()), ptrs, len(outs_host),
                                                      N, iters, chunk_bytes, rows_per_tile, _s(stream),
                                                      ctypes.byref(h2d), ctypes.byref(d2h)),
          "jacobi_solve_host_pipelined")
    return h2d.value, d2h.value


# ------------------------------------------------------------------ banded Jacobi (NEXT-2)
class Banded:
    """The paper's Jacobi (L271): A x = b with A banded (half-bandwidth w, DIA layout), x an
    N-float replicated vector, rows split like row_split()."""

    def __init__(self, a, b, chunk_bytes: int, x0=None, device=None):
        import numpy as np
        G, g = rt.world(), rt.rank()
        dev = device if device is not None else torch.device("cuda", torch.cuda.current_device())
        self.w = (a.shape[0] - 1) // 2
        self.N = a.shape[1]
        self.a = torch.from_numpy(np.ascontiguousarray(a)).to(dev)
        self.b = torch.from_numpy(np.ascontiguousarray(b)).to(dev)
        init = torch.zeros(self.N, dtype=torch.float32) if x0 is None else torch.from_numpy(np.asarray(x0))
        self.bufs = [init.to(dev).clone() for _ in range(2)]
        torch.cuda.synchronize()
        self.r0, self.r1 = row_split(self.N, G, g)
        # slices must be 16-byte multiples: round the split to 4 rows
        self.r0, self.r1 = (self.r0 // 4) * 4, (self.r1 // 4) * 4 if g < G - 1 else self.N
        self.rid = [rt.register_region(t, self.r0 * 4, (self.r1 - self.r0) * 4, chunk_bytes) for t in self.bufs]
        self.k = 0

    def step(self, stream=None, barrier: bool = False) -> None:
        i = self.k & 1
        check(rt.lib().proact_banded_phase(self.rid[i], self.rid[i ^ 1], ctypes.c_void_p(self.a.data_ptr()),
                                           ctypes.c_void_p(self.b.data_ptr()), self.N, self.w, _s(stream)),
              "banded_phase")
        rt.phase_sync(stream, barrier=barrier)
        self.k += 1

    @property
    def current(self) -> torch.Tensor:
        return self.bufs[self.k & 1]


# ------------------------------------------------------------------ microbenchmark (config 5)
def micro_phase(rid: int, phase: int, seed: int, K: int = 1, scattered: bool = False,
                stream=None) -> None:
    check(rt.lib().proact_micro_phase(rid, phase & 0xFFFFFFFF, seed & 0xFFFFFFFF, K,
                                      int(scattered), _s(stream)), "micro_phase")


def litmus_phase(r_in: int, r_out: int, phase: int, seed: int, bad: torch.Tensor, stream=None) -> None:
    """proact_litmus_phase: check every word of r_in's current generation against phase-1's tag
    (counting mismatches into the int32 CUDA tensor `bad`), then write phase `phase` of r_out."""
    assert bad.is_cuda and bad.dtype == torch.int32
    check(rt.lib().proact_litmus_phase(r_in, r_out, phase & 0xFFFFFFFF, seed & 0xFFFFFFFF,
                                       ctypes.c_void_p(bad.data_ptr()), _s(stream)), "litmus_phase")


def inject_double_commit(rid: int, stream=None) -> None:
    check(rt.lib().proact_inject_double_commit(rid, _s(stream)), "inject_double_commit")


class Micro:
    """A replicated region of `words` u32 words, all-gather shape (every rank produces W/G)."""

    def __init__(self, words: int, chunk_bytes: int, device=None, dest_mask: int | None = None):
        G, g = rt.world(), rt.rank()
        dev = device if device is not None else torch.device("cuda", torch.cuda.current_device())
        # slices are 4-word (16 B) aligned: rank g owns words [lo_g, lo_{g+1})
        bounds = [((words * p) // G) // 4 * 4 for p in range(G)] + [words]
        self.lo, self.hi = bounds[g], bounds[g + 1]
        self.buf = torch.zeros(words, dtype=torch.int32, device=dev)
        torch.cuda.synchronize()
        self.rid = rt.register_region(self.buf, self.lo * 4, (self.hi - self.lo) * 4, chunk_bytes,
                                      dest_mask)
        self.phase = 0

    def step(self, seed: int, K: int = 1, scattered: bool = False, stream=None,
             barrier: bool = False) -> None:
        micro_phase(self.rid, self.phase, seed, K, scattered, stream)
        rt.phase_sync(stream, barrier=barrier)
        self.phase += 1


# ------------------------------------------------------------------ graphs (configs 3-4)
def _u32_dev(a) -> torch.Tensor:
    """A host numpy uint32 / int32 array (or a CUDA tensor) as a contiguous CUDA int32 tensor."""
    if isinstance(a, torch.Tensor):
        t = a
    else:
        import numpy as np
        t = torch.from_numpy(np.ascontiguousarray(a).view(np.int32))
    return t.to(device="cuda", dtype=torch.int32).contiguous()


class _Graph:
    """Edge list -> this rank's destination partition + in-edge CSC (library-owned)."""

    def __init__(self, V: int, src, dst, w, chunk_bytes: int, stream=None, hot: int = -1):
        G, g = rt.world(), rt.rank()
        self.V = V
        s = _s(stream)
        d_src, d_dst = _u32_dev(src), _u32_dev(dst)
        d_w = _u32_dev(w) if w is not None else None
        E = d_src.numel()
        bounds = (ctypes.c_uint * (G + 1))()
        check(rt.lib().proact_graph_partition(ctypes.c_void_p(d_dst.data_ptr()), E, V, G, chunk_bytes // 4,
                                               bounds, s), "graph_partition")
        self.bounds = list(bounds)
        self.v0, self.v1 = self.bounds[g], self.bounds[g + 1]
        self.gid = check(rt.lib().proact_graph_build_ex(
            ctypes.c_void_p(d_src.data_ptr()), ctypes.c_void_p(d_dst.data_ptr()),
            ctypes.c_void_p(d_w.data_ptr() if d_w is not None else 0), E, V, self.v0, self.v1, hot, s),
            "graph_build")
        nh, eh = ctypes.c_uint(0), ctypes.c_ulonglong(0)
        check(rt.lib().proact_graph_hot(self.gid, ctypes.byref(nh), ctypes.byref(eh)), "graph_hot")
        self.nhot, self.e_hot = nh.value, eh.value
        e_own = ctypes.c_ulonglong(0)
        check(rt.lib().proact_graph_info(self.gid, ctypes.byref(e_own), None, None), "graph_info")
        self.e_own = e_own.value
        self.E = E
        del d_src, d_dst, d_w
        torch.cuda.synchronize()

    def free(self):
        rt.lib().proact_graph_free(self.gid)


class PageRank(_Graph):
    """Destination-partitioned PageRank over a replicated contrib = r/out vector (config 3)."""

    def __init__(self, V: int, src, dst, chunk_bytes: int, damping: float = 0.85, stream=None, hot: int = -1):
        """hot: size of the shared-memory hot-source table (-1 library default, 0 none)."""
        super().__init__(V, src, dst, None, chunk_bytes, stream, hot)
        self.d = damping
        self.bufs = [torch.zeros(V, dtype=torch.float32, device="cuda") for _ in range(2)]
        torch.cuda.synchronize()
        self.rid = [rt.register_region(b, self.v0 * 4, (self.v1 - self.v0) * 4, chunk_bytes) for b in self.bufs]
        check(rt.lib().proact_pagerank_init(self.gid, self.rid[0], _s(stream)), "pagerank_init")
        self.k = 0

    def step(self, stream=None, barrier: bool = False) -> None:
        i = self.k & 1
        check(rt.lib().proact_pagerank_phase(self.gid, self.rid[i], self.rid[i ^ 1], self.d, _s(stream)),
              "pagerank_phase")
        rt.phase_sync(stream, barrier=barrier)
        self.k += 1

    def ranks(self, stream=None) -> torch.Tensor:
        """My r' (nv floats), copied on `stream` after its phases; the current torch stream is made
        to wait for that copy, so the tensor can be used (e.g. .cpu()) on it directly."""
        out = torch.empty(self.v1 - self.v0, dtype=torch.float32, device="cuda")
        if stream is not None and stream != torch.cuda.current_stream():
            # `out` may reuse a block whose earlier users are still queued on the current stream
            stream.wait_stream(torch.cuda.current_stream())
        check(rt.lib().proact_pagerank_ranks(self.gid, ctypes.c_void_p(out.data_ptr()), _s(stream)),
              "pagerank_ranks")
        if stream is not None and stream != torch.cuda.current_stream():
            out.record_stream(stream)
            torch.cuda.current_stream().wait_stream(stream)
        return out


INF32 = 2**31 - 1


class SSSP(_Graph):
    """Synchronous Bellman-Ford over a replicated int32 distance vector, SPARSE regions (config 4)."""

    def __init__(self, V: int, src, dst, w, source: int, chunk_bytes: int, stream=None, hot: int = -1):
        """hot: size of the shared-memory hot-source table (-1 library default, 0 none)."""
        super().__init__(V, src, dst, w, chunk_bytes, stream, hot)
        self.source = source
        self.bufs = [torch.empty(V, dtype=torch.int32, device="cuda") for _ in range(2)]
        self._init_bufs()
        torch.cuda.synchronize()
        self.rid = [rt.register_region(b, self.v0 * 4, (self.v1 - self.v0) * 4, chunk_bytes,
                                       flags=_lib.REGION_SPARSE) for b in self.bufs]
        self.k = 0

    def _init_bufs(self):
        for b in self.bufs:
            b.fill_(INF32)
            b[self.source] = 0

    def reset(self) -> None:
        """Back to round 0 (d = INF except the source) on the same graph and regions.  Every rank
        calls it between runs, after a phase with a BARRIER sync (run() ends with one) and before
        any rank starts the next run (the caller's host barrier)."""
        torch.cuda.synchronize()
        self._init_bufs()
        torch.cuda.synchronize()
        self.k = 0

    def step(self, stream=None) -> bool:
        """One round with a BARRIER sync; returns True if any rank changed a distance."""
        i = self.k & 1
        check(rt.lib().proact_sssp_phase(self.gid, self.rid[i], self.rid[i ^ 1], int(self.k == 0), _s(stream)),
              "sssp_phase")
        rt.phase_sync(stream, barrier=True)
        self.k += 1
        if stream is None:
            torch.cuda.current_stream().synchronize()
        else:
            stream.synchronize()
        v = rt.last_vote()
        if v < 0:
            raise RuntimeError("vote not available")
        return bool(v)

    def run(self, max_rounds: int = 0, stream=None) -> int:
        """Rounds until (and including) the first round that changes nothing (reading R13)."""
        cap = max_rounds if max_rounds > 0 else self.V
        for r in range(cap):
            if not self.step(stream):
                return r + 1
        return cap

    @property
    def last_mode(self) -> int:
        """0 if the last round pulled over every in-edge, 1 if it pushed from the frontier (R24)."""
        return rt.lib().proact_sssp_last_mode(self.gid)

    @property
    def current(self) -> torch.Tensor:
        return self.bufs[self.k & 1]
