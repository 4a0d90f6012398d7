"""GPU parity: the CUDA Jacobi path (through the C ABI) vs the CPU oracle, bit-exact.

Reading R10: fixed association, fp32 round-to-nearest, no FMA on both
sides, so the replicas must equal the oracle bit for bit (the north star's 1e-5
relative bound is implied).  Multi-rank cases run G ranks as threads on one GPU
(loopback: peers are other buffers of the same device; every kernel, flag,
credit and push of the protocol runs unchanged).
"""
import os

import numpy as np
import pytest
import torch

import oracle
import synth
from paper_conf_isca_muthukrishnannl21_b200 import _lib, run_ranks
from paper_conf_isca_muthukrishnannl21_b200 import runtime as rt
from paper_conf_isca_muthukrishnannl21_b200 import workloads as wl

pytestmark = pytest.mark.gpu


def _run_jacobi(r, G, N, iters, chunk, mech, halo_only=False, rpt=16, check_deliv=False, **cfg):
    rt.set_config(mech=mech, watchdog_ms=20000, **cfg)
    x0 = torch.from_numpy(synth.jacobi_init(N)).cuda()
    J = wl.Jacobi(N, chunk, x0=x0, halo_only=halo_only, rows_per_tile=rpt)
    s = torch.cuda.Stream()
    deliv = []
    with torch.cuda.stream(s):
        for k in range(iters):
            J.step(s, barrier=(k == iters - 1))
            if check_deliv:
                s.synchronize()
                deliv.append(rt.debug_deliveries(J.rid[(k + 1) & 1]).copy())
                rt.host_barrier()
    s.synchronize()
    rt.check_device()
    return J.current.cpu().numpy(), (J.r0, J.r1), deliv


@pytest.mark.parametrize("mech", [_lib.MECH_FUSED, _lib.MECH_INLINE, _lib.MECH_BULK, _lib.MECH_DMA])
def test_config1_jacobi_1024_two_ranks_bit_exact(mech):
    """BASELINE.json config 1: 1024x1024 fp32, 2 row partitions, 10 iterations, full replica."""
    N, iters = 1024, 10
    want = oracle.jacobi(synth.jacobi_init(N), iters)
    outs = run_ranks(2, _run_jacobi, N, iters, 64 * 1024, mech)
    for g, (rep, _, _) in enumerate(outs):
        assert np.array_equal(rep.view(np.uint32), want.view(np.uint32)), f"rank {g} mech {mech}"


@pytest.mark.parametrize("G,N,chunk,rpt", [(1, 2048, 4096, 16), (3, 1000, 12288, 16),
                                           (4, 520, 4096, 7), (2, 4100, 1 << 20, 32)])
def test_jacobi_ragged_ranks_chunks_tiles(G, N, chunk, rpt):
    iters = 6
    want = oracle.jacobi(synth.jacobi_init(N), iters)
    outs = run_ranks(G, _run_jacobi, N, iters, chunk, _lib.MECH_FUSED, rpt=rpt)
    for g, (rep, _, _) in enumerate(outs):
        assert np.array_equal(rep.view(np.uint32), want.view(np.uint32)), f"rank {g}"


@pytest.mark.parametrize("cfg", [dict(push=1), dict(agent_kernel=1), dict(push=1, agent_kernel=1),
                                 dict(discovery=1, agent_warps=5), dict(agent_kernel=2)])
def test_config1_jacobi_agent_variants(cfg):
    N, iters = 1024, 10
    want = oracle.jacobi(synth.jacobi_init(N), iters)
    outs = run_ranks(2, _run_jacobi, N, iters, 64 * 1024, _lib.MECH_FUSED, **cfg)
    for g, (rep, _, _) in enumerate(outs):
        assert np.array_equal(rep.view(np.uint32), want.view(np.uint32)), (g, cfg)


@pytest.mark.parametrize("G,N,chunk,rpt", [(2, 2048, 4096, 16), (3, 1000, 12288, 16),
                                           (4, 520, 4096, 7), (2, 4100, 1 << 20, 32), (3, 2056, 4112, 5)])
def test_jacobi_tile_push_ragged(G, N, chunk, rpt):
    """PROACT_AGENT_PRODUCER (the producer CTA's transfer warp bulk-stores its row strips to every
    replica): ragged ranks, partial strips (N not a multiple of 1024), chunks that split a strip."""
    iters = 6
    want = oracle.jacobi(synth.jacobi_init(N), iters)
    outs = run_ranks(G, _run_jacobi, N, iters, chunk, _lib.MECH_FUSED, rpt=rpt, agent_kernel=_lib.AGENT_PRODUCER)
    for g, (rep, _, _) in enumerate(outs):
        assert np.array_equal(rep.view(np.uint32), want.view(np.uint32)), f"rank {g}"


def test_jacobi_tile_push_halo_only_and_elide():
    """Tile push with per-chunk destinations (halo-only) and under ELIDE at G = 1."""
    G, N, iters = 4, 512, 9
    want = oracle.jacobi(synth.jacobi_init(N), iters)
    outs = run_ranks(G, _run_jacobi, N, iters, 8192, _lib.MECH_FUSED, halo_only=True, agent_kernel=2)
    for g, (rep, (r0, r1), _) in enumerate(outs):
        lo, hi = max(r0 - 1, 0), min(r1 + 1, N)
        assert np.array_equal(rep[lo:hi].view(np.uint32), want[lo:hi].view(np.uint32)), g
    (rep, _, _), = run_ranks(1, _run_jacobi, 1536, 5, 65536, _lib.MECH_ELIDE, agent_kernel=2)
    assert np.array_equal(rep.view(np.uint32), oracle.jacobi(synth.jacobi_init(1536), 5).view(np.uint32))


def test_jacobi_mixed_mechanisms_across_phases():
    """Consumers wait according to the mechanism that produced the generation they read."""
    N, G = 768, 3
    seq = [_lib.MECH_FUSED, _lib.MECH_INLINE, _lib.MECH_DMA, _lib.MECH_BULK, _lib.MECH_FUSED, _lib.MECH_DMA,
           _lib.MECH_INLINE, _lib.MECH_FUSED]
    want = oracle.jacobi(synth.jacobi_init(N), len(seq))

    def body(r, G):
        J = wl.Jacobi(N, 8192, x0=torch.from_numpy(synth.jacobi_init(N)).cuda())
        s = torch.cuda.Stream()
        for k, m in enumerate(seq):
            rt.set_config(mech=m)
            J.step(s, barrier=(k == len(seq) - 1))
        s.synchronize()
        rt.check_device()
        return J.current.cpu().numpy()

    for g, rep in enumerate(run_ranks(G, body)):
        assert np.array_equal(rep.view(np.uint32), want.view(np.uint32)), g


@pytest.mark.parametrize("cfg", [dict(), dict(agent_kernel=_lib.AGENT_SEPARATE, push=_lib.PUSH_BULK),
                                 dict(agent_kernel=_lib.AGENT_SEPARATE, push=_lib.PUSH_VEC16,
                                      discovery=_lib.DISCOVER_SCAN, agent_warps=2),
                                 dict(agent_kernel=_lib.AGENT_FUSED, agent_warps=1),
                                 dict(agent_kernel=_lib.AGENT_FUSED, discovery=_lib.DISCOVER_SCAN, agent_warps=1)])
def test_jacobi_halo_only_owned_rows_and_halos(cfg):
    """Halo-only: chunks bound nowhere are published by their last committer and never reach
    the agent (queue sized / scan windows skipped from the per-chunk destinations), for every
    agent placement and discovery mode; ragged last chunk (N = 520 rows of 2080 B, 8 KiB chunks)."""
    for G, N, iters in ((4, 512, 9), (2, 520, 7)):
        want = oracle.jacobi(synth.jacobi_init(N), iters)
        outs = run_ranks(G, _run_jacobi, N, iters, 8192, _lib.MECH_FUSED, halo_only=True, **cfg)
        for g, (rep, (r0, r1), _) in enumerate(outs):
            lo, hi = max(r0 - 1, 0), min(r1 + 1, N)
            assert np.array_equal(rep[lo:hi].view(np.uint32), want[lo:hi].view(np.uint32)), (g, G, cfg)


def test_jacobi_halo_only_exactly_once():
    """Halo-only delivery counters: every chunk with a destination is delivered once per phase
    to each destination, chunks bound nowhere never."""
    os.environ["PROACT_DEBUG"] = "1"
    try:
        G, N, iters = 3, 768, 4
        outs = run_ranks(G, _run_jacobi, N, iters, 8192, _lib.MECH_FUSED, halo_only=True, check_deliv=True,
                         agent_kernel=_lib.AGENT_SEPARATE)
    finally:
        os.environ.pop("PROACT_DEBUG", None)
    rowb = N * 4
    for g, (_, (r0, r1), deliv) in enumerate(outs):
        own = (r1 - r0) * rowb
        nch = (own + 8191) // 8192
        assert len(deliv) == iters
        for k, d in enumerate(deliv):
            assert d.shape == (nch, G)
            for c in range(nch):
                lo, hi = c * 8192, min((c + 1) * 8192, own)
                for q in range(G):
                    bound = (q == g - 1 and lo < rowb) or (q == g + 1 and hi > own - rowb)
                    assert d[c, q] == (1 if bound else 0), (g, k, c, q, d[c, q])


@pytest.mark.parametrize("akern", [0, 2])
def test_jacobi_exactly_once_delivery(akern):
    os.environ["PROACT_DEBUG"] = "1"
    try:
        G, N, iters = 3, 768, 4
        outs = run_ranks(G, _run_jacobi, N, iters, 4096, _lib.MECH_FUSED, check_deliv=True, agent_kernel=akern)
    finally:
        del os.environ["PROACT_DEBUG"]
    for g, (_, _, deliv) in enumerate(outs):
        assert len(deliv) == iters
        for d in deliv:
            want = np.ones_like(d)
            want[:, g] = 0
            assert np.array_equal(d, want), f"rank {g}: {d}"


@pytest.mark.parametrize("mech", [_lib.MECH_FUSED, _lib.MECH_LOCAL, _lib.MECH_ELIDE])
def test_jacobi_single_gpu_mechanisms(mech):
    N, iters = 1536, 5
    want = oracle.jacobi(synth.jacobi_init(N), iters)
    (rep, _, _), = run_ranks(1, _run_jacobi, N, iters, 128 * 1024, mech)
    assert np.array_equal(rep.view(np.uint32), want.view(np.uint32))


def _window_oracle(N, iters, i, j):
    """Cell (i, j) after `iters` iterations from the (2*iters+3)^2 window of x0 around it:
    influence travels one cell per iteration, so the window's false boundary never reaches the
    centre (needs iters+1 <= i, j <= N-2-iters)."""
    h = iters + 1
    x0 = synth.jacobi_init(N, row0=i - h, nrows=2 * h + 1)[:, j - h:j + h + 1]
    return oracle.jacobi(np.ascontiguousarray(x0), iters)[h, h]


@pytest.mark.slow
def test_config2_full_size_sampled_single_gpu():
    """Config 2 size (16384^2, 100 iterations) in bench.py's N = 1 launch configuration.  At
    G = 1 there is nothing to replicate, so FUSED runs the uninstrumented kernel (reading R18):
    this checks the producer kernel alone, on sampled cells computed one by one by the oracle."""
    N, iters = 16384, 100
    (rep, _, _), = run_ranks(1, _run_jacobi, N, iters, 128 * 1024, _lib.MECH_FUSED, rpt=32)
    rng = np.random.default_rng(0)
    pts = [(int(a), int(b)) for a, b in rng.integers(iters + 1, N - iters - 2, size=(12, 2))]
    pts += [(iters + 1, iters + 1), (N - iters - 2, N - iters - 2), (8192, 1023), (8191, 1024),
            (8223, 2047), (8224, 2048)]   # tile-band and strip boundaries at rows_per_tile = 32
    for i, j in pts:
        assert rep[i, j] == _window_oracle(N, iters, i, j), (i, j)
    # boundary rows/cols are copied through (Dirichlet)
    x0 = synth.jacobi_init(N, row0=0, nrows=1)
    assert np.array_equal(rep[0], x0[0])


def _block_oracle(N, iters, i0, i1, j0, j1):
    """x^iters on rows [i0, i1) x cols [j0, j1), exactly: from a square window of x0 reaching
    iters + 1 cells beyond the block on every side that is not the grid's own boundary
    (influence travels one cell per iteration, so a false window edge never reaches the block)."""
    h = iters + 1
    S = min(N, max(i1 - i0, j1 - j0) + 2 * h)
    a = min(max(i0 - h, 0), N - S)
    b = min(max(j0 - h, 0), N - S)
    x0 = np.ascontiguousarray(synth.jacobi_init(N, row0=a, nrows=S)[:, b:b + S])
    return oracle.jacobi(x0, iters)[i0 - a:i1 - a, j0 - b:j1 - b]


def _run_jacobi_full(r, G, N, iters, chunk, cfg):
    """bench.py's N > 1 step on G loopback ranks; returns (my replica, rows, other ranks' rows
    of my replica are compared across ranks by the caller)."""
    rep, rows, _ = _run_jacobi(r, G, N, iters, chunk, _lib.MECH_FUSED, rpt=32, **cfg)
    return rep, rows


@pytest.mark.slow
@pytest.mark.parametrize("chunk,cfg", [
    (128 * 1024, dict(agent_kernel=_lib.AGENT_SEPARATE, push=_lib.PUSH_BULK, discovery=_lib.DISCOVER_QUEUE)),
    (1 << 20, dict(agent_kernel=_lib.AGENT_SEPARATE, push=_lib.PUSH_BULK, discovery=_lib.DISCOVER_QUEUE)),
    (1 << 20, dict(agent_kernel=_lib.AGENT_PRODUCER)),
    (128 * 1024, dict(agent_kernel=_lib.AGENT_SEPARATE, push=_lib.PUSH_VEC16, discovery=_lib.DISCOVER_SCAN)),
])
def test_config2_full_size_two_ranks(chunk, cfg):
    """Config 2 at full size (16384^2, 100 iterations) on G = 2 loopback ranks in the launch
    configuration bench.py times at N > 1 (FUSED: tallies, agent, pushes, flags, credits every
    phase).  Checked: every cell of the four rows around the rank boundary (the halo rows each
    rank waits on every phase) against exact block oracles, sampled cells elsewhere, and the two
    replicas equal bit for bit (every pushed byte arrived: replica bytes == producer bytes)."""
    N, iters, G = 16384, 100, 2
    outs = run_ranks(G, _run_jacobi_full, N, iters, chunk, cfg)
    (rep0, (r0a, r1a)), (rep1, (r0b, r1b)) = outs
    assert r1a == r0b == N // 2
    assert np.array_equal(rep0.view(np.uint32), rep1.view(np.uint32))
    b = N // 2
    for j0 in range(0, N, 1024):   # rows b-2 .. b+1, all columns, in 1024-column blocks
        want = _block_oracle(N, iters, b - 2, b + 2, j0, j0 + 1024)
        assert np.array_equal(rep0[b - 2:b + 2, j0:j0 + 1024].view(np.uint32), want.view(np.uint32)), j0
    rng = np.random.default_rng(1)
    for i, j in rng.integers(iters + 1, N - iters - 2, size=(8, 2)):
        assert rep0[i, j] == _window_oracle(N, iters, int(i), int(j)), (i, j)


@pytest.mark.slow
def test_config2_full_size_two_ranks_halo_only():
    """The halo-only variant (reading R8; per-chunk destinations = neighbours) at full size, in
    bench.py's halo leg configuration: the rows each rank reads are exact."""
    N, iters, G = 16384, 100, 2
    outs = run_ranks(G, _run_jacobi, N, iters, 1 << 20, _lib.MECH_FUSED, halo_only=True, rpt=32,
                     agent_kernel=_lib.AGENT_PRODUCER)
    b = N // 2
    for g, (rep, (r0, r1), _) in enumerate(outs):
        for j0 in range(0, N, 4096):
            want = _block_oracle(N, iters, b - 1, b + 1, j0, j0 + 4096)
            assert np.array_equal(rep[b - 1:b + 1, j0:j0 + 4096].view(np.uint32), want.view(np.uint32)), (g, j0)


def test_jacobi_allgather_baseline():
    """Jacobi.step_allgather (the north star's NCCL all-gather baseline: uninstrumented kernel +
    all_gather_into_tensor between phases) equals the oracle; NCCL needs one GPU per rank."""
    if torch.cuda.device_count() < 2:
        pytest.skip("NCCL all-gather needs 2 GPUs (one rank per GPU)")
    import socket
    import subprocess
    import sys
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    port = s.getsockname()[1]
    s.close()
    script = os.path.join(os.path.dirname(os.path.abspath(__file__)), "allgather_rank.py")
    cmd = [sys.executable, "-m", "torch.distributed.run", "--nnodes=1", "--nproc-per-node", "2",
           "--master-addr", "127.0.0.1", "--master-port", str(port), script]
    r = subprocess.run(cmd, capture_output=True, text=True, timeout=600)
    assert r.returncode == 0, r.stdout + r.stderr
    assert r.stdout.count("ALLGATHER_OK") == 2, r.stdout


def test_jacobi_e2e_host_buffers():
    N, iters = 512, 7
    x0 = synth.jacobi_init(N)
    want = oracle.jacobi(x0, iters)

    def body(r, G):
        xh = torch.from_numpy(x0).pin_memory()
        out = torch.zeros((N, N), dtype=torch.float32).pin_memory()
        s = torch.cuda.Stream()
        h2d, d2h = wl.jacobi_solve_host(xh, out, N, iters, 16384, stream=s)
        s.synchronize()
        r0, r1 = wl.row_split(N, G, r)
        return out.numpy()[r0:r1].copy(), (r0, r1), h2d, d2h

    outs = run_ranks(2, body)
    for rows, (r0, r1), h2d, d2h in outs:
        assert np.array_equal(rows, want[r0:r1])
        assert h2d == (min(r1 + 1, N) - max(r0 - 1, 0)) * N * 4 and d2h == (r1 - r0) * N * 4


@pytest.mark.parametrize("G,iters", [(1, 7), (2, 6), (2, 0), (3, 5)])
def test_jacobi_e2e_pipelined_host_buffers(G, iters):
    """proact_jacobi_solve_host_pipelined: every one of the nsolve outputs (two device buffer
    sets reused in turn, copies on library streams) equals the oracle, over two calls."""
    N = 512
    x0 = synth.jacobi_init(N)
    want = oracle.jacobi(x0, iters) if iters else x0

    def body(r, G_):
        xh = torch.from_numpy(x0).pin_memory()
        s = torch.cuda.Stream()
        got = []
        for nsolve in (5, 2):
            outs = [torch.full((N, N), -1.0, dtype=torch.float32).pin_memory() for _ in range(nsolve)]
            h2d, d2h = wl.jacobi_solve_host_pipelined(xh, outs, N, iters, 16384, stream=s)
            s.synchronize()
            r0, r1 = wl.row_split(N, G_, r)
            got.append(([o.numpy()[r0:r1].copy() for o in outs], (r0, r1), h2d, d2h))
        return got

    for per_rank in run_ranks(G, body):
        for rows_list, (r0, r1), h2d, d2h in per_rank:
            for rows in rows_list:
                assert np.array_equal(rows.view(np.uint32), want[r0:r1].view(np.uint32))
            assert h2d == (min(r1 + 1, N) - max(r0 - 1, 0)) * N * 4 and d2h == (r1 - r0) * N * 4


@pytest.mark.parametrize("G,N,chunk", [(1, 4, 4096), (2, 8, 4096), (2, 1024, 4112), (3, 36, 4096)])
def test_jacobi_degenerate_and_odd_chunks(G, N, chunk):
    """All-boundary grids (N = 4: every cell copied through), ranks owning a couple of rows,
    a chunk size that is not a multiple of the 4 KiB row segment (spans straddle chunks)."""
    iters = 3
    want = oracle.jacobi(synth.jacobi_init(N), iters)
    outs = run_ranks(G, _run_jacobi, N, iters, chunk, _lib.MECH_FUSED)
    for g, (rep, _, _) in enumerate(outs):
        assert np.array_equal(rep.view(np.uint32), want.view(np.uint32)), g
