"""GPU parity for the transfer microbenchmark (config 5 shape) and protocol invariants.

Replica bytes must equal the closed form (oracle.micro_phase) bit-exactly on
every rank after every phase; each (chunk, dest) delivered exactly once; a
watchdog turns a protocol stall into PROACT_ERR_TIMEOUT instead of a hang.
"""
import os

import numpy as np
import pytest
import torch

import oracle
from paper_conf_isca_muthukrishnannl21_b200 import _lib, run_ranks, ProactError
from paper_conf_isca_muthukrishnannl21_b200 import runtime as rt
from paper_conf_isca_muthukrishnannl21_b200 import workloads as wl

pytestmark = pytest.mark.gpu
SEED = 0x5EED


def _run_micro(r, G, words, chunk, mech, phases, K, scattered, piece=None, warps=None, push=0, akern=0):
    kw = dict(mech=mech, push=push, agent_kernel=akern)
    if piece:
        kw["piece_bytes"] = piece
    if warps:
        kw["agent_warps"] = warps
    rt.set_config(**kw)
    M = wl.Micro(words, chunk)
    s = torch.cuda.Stream()
    snaps = []
    for p in range(phases):
        M.step(SEED, K, scattered, stream=s, barrier=True)
        s.synchronize()
        snaps.append(M.buf.cpu().numpy().view(np.uint32).copy())
        rt.host_barrier()   # no peer may start phase p+1 (and overwrite) before every snapshot
    rt.check_device()
    return snaps


@pytest.mark.parametrize("G,words,chunk,mech,scattered,piece", [
    (2, 1 << 20, 4096, _lib.MECH_FUSED, False, None),
    (2, (1 << 20) + 4 * 37, 65536, _lib.MECH_FUSED, True, 16384),
    (4, 3_000_000, 1 << 20, _lib.MECH_FUSED, False, 65536),
    (3, 777_776, 12288, _lib.MECH_INLINE, True, None),
    (4, 1 << 21, 4 << 20, _lib.MECH_BULK, False, None),
    (3, 3 << 20, 1 << 20, _lib.MECH_DMA, False, None),
    (2, 1 << 20, 65536, _lib.MECH_DMA, True, None),
    (1, 1 << 20, 4096, _lib.MECH_FUSED, False, None),
])
def test_micro_replicas_equal_closed_form(G, words, chunk, mech, scattered, piece):
    phases, K = 3, 2
    outs = run_ranks(G, _run_micro, words, chunk, mech, phases, K, scattered, piece=piece)
    for p in range(phases):
        want = oracle.micro_phase(words, p, SEED, K)
        for g in range(G):
            assert np.array_equal(outs[g][p], want), (p, g)


@pytest.mark.parametrize("push,akern", [(0, 0), (1, 0), (0, 1), (1, 1), (1, 2)])
@pytest.mark.parametrize("G,words,chunk", [(2, (1 << 21) + 4 * 5, 1 << 20), (3, 1 << 20, 16384)])
def test_micro_push_modes_and_agent_kernels(G, words, chunk, push, akern):
    """TMA bulk pushes and the separate agent kernel give the same bytes as the SIMT/fused path."""
    phases = 3
    outs = run_ranks(G, _run_micro, words, chunk, _lib.MECH_FUSED, phases, 1, False, piece=65536, warps=4,
                     push=push, akern=akern)
    for p in range(phases):
        want = oracle.micro_phase(words, p, SEED, 1)
        for g in range(G):
            assert np.array_equal(outs[g][p], want), (p, g)


@pytest.mark.parametrize("G,words,chunk,scattered", [
    (2, 1 << 20, 4096, False), (2, (1 << 20) + 4 * 37, 65536, True), (4, 3_000_000, 1 << 20, False),
    (3, 777_776, 12288, True), (1, 1 << 20, 4096, False)])
def test_micro_tile_push_replicas(G, words, chunk, scattered):
    """PROACT_AGENT_PRODUCER: the producer CTAs' transfer warps bulk-store their own 4 KiB tiles
    to every replica; replicas equal the closed form; ragged slices and chunks that are not a
    multiple of the tile size (spans split at chunk boundaries)."""
    phases, K = 3, 3
    outs = run_ranks(G, _run_micro, words, chunk, _lib.MECH_FUSED, phases, K, scattered, akern=_lib.AGENT_PRODUCER)
    for p in range(phases):
        want = oracle.micro_phase(words, p, SEED, K)
        for g in range(G):
            assert np.array_equal(outs[g][p], want), (p, g)


@pytest.mark.parametrize("disc,akern", [(_lib.DISCOVER_QUEUE, 0), (_lib.DISCOVER_SCAN, 0),
                                        (_lib.DISCOVER_QUEUE, 2)])
def test_micro_exactly_once_and_counters(disc, akern):
    os.environ["PROACT_DEBUG"] = "1"

    def body(r, G):
        rt.set_config(mech=_lib.MECH_FUSED, piece_bytes=8192, agent_warps=3, discovery=disc, agent_kernel=akern)
        M = wl.Micro(1 << 20, 65536)
        s = torch.cuda.Stream()
        out = []
        for p in range(3):
            M.step(SEED, 1, False, stream=s, barrier=True)
            s.synchronize()
            out.append(rt.debug_deliveries(M.rid).copy())
            rt.host_barrier()
        return out

    try:
        outs = run_ranks(3, body)
    finally:
        del os.environ["PROACT_DEBUG"]
    for g, ds in enumerate(outs):
        for d in ds:
            want = np.ones_like(d)
            want[:, g] = 0
            assert np.array_equal(d, want)


def test_watchdog_turns_a_stall_into_timeout():
    """A consumer waiting for data that no producer will ever publish must time out, not hang
    (fault injection T5): rank 1 never launches phase 0, rank 0 waits for its credit."""

    def body(r, G):
        rt.set_config(mech=_lib.MECH_FUSED, watchdog_ms=300)
        M = wl.Micro(1 << 16, 4096)
        s = torch.cuda.Stream()
        if r == 0:
            wl.micro_phase(M.rid, 0, SEED, stream=s)
            try:
                rt.phase_sync(s, barrier=True)   # waits for rank 1's credit forever
                s.synchronize()
                rt.check_device()
            except ProactError as e:
                return e.code
            return 0
        s.synchronize()
        return None

    res = run_ranks(2, body)
    assert res[0] == _lib.ERR_TIMEOUT


def test_micro_ranks_with_empty_slices():
    """A region smaller than the world: some ranks own zero bytes (no chunks) but still take
    part in every collective and phase."""
    words, G = 8, 4   # slices of 0 / 4 / 0 / 4 words
    outs = run_ranks(G, _run_micro, words, 4096, _lib.MECH_FUSED, 2, 1, False)
    for p in range(2):
        want = oracle.micro_phase(words, p, SEED, 1)
        for g in range(G):
            assert np.array_equal(outs[g][p], want), (p, g)


@pytest.mark.slow
@pytest.mark.parametrize("chunk", [4 << 20, 64 << 10])
def test_config5_full_size_sampled(chunk):
    """Config 5 at its largest region (R = 4 GiB, 2^30 words), two loopback ranks, in bench
    launch configuration (default agent): every rank's replica equals the closed form on a random
    sample of 200k words plus every slice / chunk boundary word, after each of 2 phases."""
    W, G, K = 1 << 30, 2, 1
    rng = np.random.default_rng(5)
    samp = np.unique(np.concatenate([
        rng.integers(0, W, 200_000),
        np.array([0, 1, W // 2 - 1, W // 2, W // 2 + 1, W - 2, W - 1]),
        np.arange(0, W, chunk // 4)[:4096], np.arange(chunk // 4 - 1, W, chunk // 4)[:4096]])).astype(np.int64)

    def body(r, G_):
        rt.set_config(mech=_lib.MECH_FUSED)
        M = wl.Micro(W, chunk)
        s = torch.cuda.Stream()
        idx = torch.from_numpy(samp).cuda()
        got = []
        for p in range(2):
            M.step(SEED, K, False, stream=s, barrier=True)
            s.synchronize()
            got.append(M.buf.index_select(0, idx).cpu().numpy().view(np.uint32).copy())
            rt.host_barrier()
        rt.check_device()
        del M
        return got

    outs = run_ranks(G, body)
    for p in range(2):
        want = np.array([oracle.micro_word(int(k), p, SEED, K) for k in samp], dtype=np.uint32)
        for g in range(G):
            bad = np.nonzero(outs[g][p] != want)[0]
            assert bad.size == 0, (p, g, samp[bad[:5]])
