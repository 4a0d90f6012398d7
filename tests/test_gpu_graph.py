"""GPU parity for PageRank (config 3) and SSSP (config 4) vs the CPU oracle.

PageRank: elementwise relative error <= 1e-5 (north star fp32 tolerance) against the
fp64-accumulating oracle (reading R12); both sides round r to fp32 once per iteration.
SSSP: int32 distances bit-exact and the same number of rounds (reading R13).
Graphs: synthetic RMAT (stand-in for Wikipedia / HV15R).
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


def _pr_body(r, G, V, src, dst, iters, chunk, mech, hot=-1):
    rt.set_config(mech=mech)
    s = torch.cuda.Stream()
    P = wl.PageRank(V, src, dst, chunk, stream=s, hot=hot)
    for k in range(iters):
        P.step(s, barrier=(k == iters - 1))
    s.synchronize()
    rt.check_device()
    out = P.ranks(s).cpu().numpy()
    P.free()
    return P.v0, P.v1, out


# hot: -1 = library default (8192: nearly every source with out-edges fits the table at these
# sizes), 0 = no table (pagerank_kernel), 97 = a partial table (both read paths in one warp)
@pytest.mark.parametrize("G,scale,chunk,mech,hot", [(1, 12, 4096, _lib.MECH_FUSED, -1),
                                                    (1, 12, 4096, _lib.MECH_FUSED, 0),
                                                    (2, 13, 8192, _lib.MECH_FUSED, 97),
                                                    (2, 13, 8192, _lib.MECH_FUSED, -1),
                                                    (3, 12, 4096, _lib.MECH_FUSED, 0),
                                                    (2, 12, 16384, _lib.MECH_INLINE, 97),
                                                    (2, 12, 4096, _lib.MECH_BULK, -1),
                                                    (4, 14, 65536, _lib.MECH_FUSED, 1000)])
def test_pagerank_matches_oracle(G, scale, chunk, mech, hot):
    src, dst = synth.rmat(scale, 16)
    V, iters = 1 << scale, 20
    want = oracle.pagerank(V, src, dst, iters).astype(np.float64)
    outs = run_ranks(G, _pr_body, V, src, dst, iters, chunk, mech, hot)
    got = np.zeros(V)
    covered = 0
    for v0, v1, r in outs:
        got[v0:v1] = r
        covered += v1 - v0
    assert covered == V
    rel = np.abs(got - want) / want
    assert rel.max() <= 1e-5, rel.max()


def test_pagerank_hot_table_is_bit_identical():
    """The hot-source table changes where contributions are read, not the (exact fixed-point)
    sums: r' is bit-identical with no table, a partial table and the default table."""
    src, dst = synth.rmat(16, 16)
    V = 1 << 16
    hots = (0, 333, -1, 12000, 30000, 65536)   # 12000 / 30000 / 65536: DSMEM tables of 2 / 4 / 8 CTAs
    got = [run_ranks(1, _pr_body, V, src, dst, 5, 4096, _lib.MECH_FUSED, hot)[0][2] for hot in hots]
    for k in range(1, len(hots)):
        assert np.array_equal(got[0].view(np.uint32), got[k].view(np.uint32)), hots[k]


@pytest.mark.parametrize("G,hot", [(1, 12000), (2, 30000), (3, 65536)])
def test_cluster_hot_tables_match_oracle(G, hot):
    """Hot tables spread over thread-block clusters (DSMEM): PageRank within 1e-5 and SSSP
    bit-exact against the oracle, multi-rank included (separate agent next to cluster grids)."""
    src, dst = synth.rmat(16, 16)
    V = 1 << 16
    want = oracle.pagerank(V, src, dst, 10).astype(np.float64)
    got = np.zeros(V)
    for v0, v1, r in run_ranks(G, _pr_body, V, src, dst, 10, 16384, _lib.MECH_FUSED, hot):
        got[v0:v1] = r
    assert (np.abs(got - want) / want).max() <= 1e-5
    w = synth.weights(src.size)
    s0 = int(np.bincount(src, minlength=V).argmax())
    want_d, want_rounds, _ = oracle.sssp(V, src, dst, w, s0)
    for rounds, d, _, _ in run_ranks(G, _sssp_body, V, src, dst, w, s0, 16384, _lib.MECH_FUSED, hot):
        assert rounds == want_rounds and np.array_equal(d, want_d)


def _sssp_body(r, G, V, src, dst, w, s0, chunk, mech, hot=-1):
    rt.set_config(mech=mech)
    st = torch.cuda.Stream()
    S = wl.SSSP(V, src, dst, w, s0, chunk, stream=st, hot=hot)
    rounds = S.run(stream=st)
    rt.check_device()
    d = S.current.cpu().numpy().copy()
    S.free()
    return rounds, d, S.v0, S.v1


# hot as in test_pagerank_matches_oracle (0: sssp_kernel, else sssp_hot_kernel)
@pytest.mark.parametrize("G,scale,chunk,mech,hot", [(1, 12, 4096, _lib.MECH_FUSED, -1),
                                                    (1, 12, 4096, _lib.MECH_FUSED, 0),
                                                    (2, 13, 4096, _lib.MECH_FUSED, 97),
                                                    (2, 13, 4096, _lib.MECH_FUSED, 0),
                                                    (3, 12, 8192, _lib.MECH_FUSED, -1),
                                                    (2, 12, 4096, _lib.MECH_INLINE, 97),
                                                    (2, 12, 4096, _lib.MECH_BULK, -1),
                                                    (4, 14, 16384, _lib.MECH_FUSED, 1000)])
def test_sssp_matches_oracle(G, scale, chunk, mech, hot):
    src, dst = synth.rmat(scale, 16)
    V = 1 << scale
    w = synth.weights(src.size)
    s0 = int(np.bincount(src, minlength=V).argmax())
    want, want_rounds, _ = oracle.sssp(V, src, dst, w, s0)
    outs = run_ranks(G, _sssp_body, V, src, dst, w, s0, chunk, mech, hot)
    for rounds, d, v0, v1 in outs:
        assert rounds == want_rounds
        # owned slice always exact; full replica exact under FUSED/INLINE/BULK replication
        assert np.array_equal(d[v0:v1], want[v0:v1])
        assert np.array_equal(d, want)


def test_sssp_disconnected_and_tiny():
    # vertices unreachable from the source keep INF; a graph with no edges converges in 1 round
    V = 4096
    rng = np.random.default_rng(3)
    src = rng.integers(0, V // 2, 5000).astype(np.uint32)
    dst = rng.integers(0, V // 2, 5000).astype(np.uint32)
    keep = src != dst
    src, dst = src[keep], dst[keep]
    w = synth.weights(src.size, seed=5)
    want, want_rounds, _ = oracle.sssp(V, src, dst, w, 0)
    outs = run_ranks(2, _sssp_body, V, src, dst, w, 0, 4096, _lib.MECH_FUSED)
    for rounds, d, _, _ in outs:
        assert rounds == want_rounds and np.array_equal(d, want)
        assert np.all(d[V // 2:] == oracle.INF)


_RMAT24 = {}


def _rmat24():
    """RMAT-24 edge list + weights + source, generated once per test session."""
    if not _RMAT24:
        src, dst = synth.rmat(24, 16)
        V = 1 << 24
        _RMAT24.update(src=src, dst=dst, V=V, w=synth.weights(src.size),
                       s0=int(np.bincount(src, minlength=V).argmax()))
    return _RMAT24


def _pr_body_cfg(r, G, V, src, dst, iters, chunk, cfg):
    rt.set_config(**cfg)
    return _pr_body(r, G, V, src, dst, iters, chunk, _lib.MECH_FUSED)


def _sssp_body_cfg(r, G, V, src, dst, w, s0, chunk, cfg):
    rt.set_config(**cfg)
    return _sssp_body(r, G, V, src, dst, w, s0, chunk, _lib.MECH_FUSED)


# the graph benchmarks' launch configuration (tools/bench_workloads.py): FUSED with the separate
# agent, TMA pushes, queue discovery, 128 KiB chunks (RMAT-24: 256 chunks per rank at G = 2)
_GCFG = [(128 * 1024, dict(agent_kernel=_lib.AGENT_SEPARATE, push=_lib.PUSH_BULK, discovery=_lib.DISCOVER_QUEUE)),
         (1 << 20, dict(agent_kernel=_lib.AGENT_SEPARATE, push=_lib.PUSH_VEC16, discovery=_lib.DISCOVER_SCAN))]


@pytest.mark.slow
@pytest.mark.parametrize("G", [1, 2])
def test_config3_pagerank_full_size(G):
    """BASELINE.json config 3 at full size (RMAT-24, ef16, 20 iterations), every vertex.  G = 1
    runs the producer kernel alone (nothing to replicate, reading R18); G = 2 loopback runs the
    whole protocol in the benchmarks' launch configuration."""
    g = _rmat24()
    V, iters = g["V"], 20
    chunk, cfg = _GCFG[0]
    outs = run_ranks(G, _pr_body_cfg, V, g["src"], g["dst"], iters, chunk, cfg)
    want = oracle.pagerank(V, g["src"], g["dst"], iters).astype(np.float64)
    got = np.zeros(V)
    for v0, v1, r in outs:
        got[v0:v1] = r
    rel = np.abs(got - want) / want
    assert rel.max() <= 1e-5, rel.max()


@pytest.mark.slow
@pytest.mark.parametrize("G,k", [(1, 0), (2, 0), (2, 1)])
def test_config4_sssp_full_size(G, k):
    """BASELINE.json config 4 at full size (RMAT-24, int32, to convergence), bit-exact, every
    vertex of every rank's full replica and the round count.  At G = 2 each rank owns >= 32
    chunks of 1 MiB / 256 of 128 KiB, so the SPARSE push-iff-changed-now-or-last-round logic
    (reading R13) runs on many chunks per rank and round."""
    g = _rmat24()
    chunk, cfg = _GCFG[k]
    outs = run_ranks(G, _sssp_body_cfg, g["V"], g["src"], g["dst"], g["w"], g["s0"], chunk, cfg)
    want, want_rounds, _ = oracle.sssp(g["V"], g["src"], g["dst"], g["w"], g["s0"])
    for rounds, d, v0, v1 in outs:
        assert (v1 - v0) * 4 // chunk >= 32 or G == 1
        assert rounds == want_rounds
        assert np.array_equal(d, want)


def test_graph_without_edges():
    """E = 0: PageRank gives (1-d)/V everywhere, SSSP converges in one round."""
    V = 8192
    src = np.zeros(0, np.uint32)
    dst = np.zeros(0, np.uint32)
    outs = run_ranks(2, _pr_body, V, src, dst, 3, 4096, _lib.MECH_FUSED)
    want = oracle.pagerank(V, src, dst, 3).astype(np.float64)
    for v0, v1, r in outs:
        assert np.allclose(r, want[v0:v1], rtol=1e-6)
    outs = run_ranks(2, _sssp_body, V, src, dst, np.zeros(0, np.int32), 5, 4096, _lib.MECH_FUSED)
    d_want, rounds_want, _ = oracle.sssp(V, src, dst, np.zeros(0, np.int32), 5)
    for rounds, d, _, _ in outs:
        assert rounds == rounds_want and np.array_equal(d, d_want)


def _sssp_rerun_body(r, G, V, src, dst, w, s0, chunk):
    rt.set_config(mech=_lib.MECH_FUSED)
    st = torch.cuda.Stream()
    S = wl.SSSP(V, src, dst, w, s0, chunk, stream=st)
    out = []
    for _ in range(2):
        S.reset()
        rt.host_barrier()
        rounds = S.run(stream=st)
        out.append((rounds, S.current.cpu().numpy().copy()))
    rt.check_device()
    S.free()
    return out


def test_sssp_reset_reruns_identically():
    """SSSP.reset() restarts on the same graph and regions (the bench reuses one build)."""
    src, dst = synth.rmat(12, 16)
    V = 1 << 12
    w = synth.weights(src.size)
    s0 = int(np.bincount(src, minlength=V).argmax())
    want, want_rounds, _ = oracle.sssp(V, src, dst, w, s0)
    for runs in run_ranks(2, _sssp_rerun_body, V, src, dst, w, s0, 4096):
        for rounds, d in runs:
            assert rounds == want_rounds and np.array_equal(d, want)


def _sssp_modes_body(r, G, V, src, dst, w, s0, chunk, mech, hot, reruns=1):
    rt.set_config(mech=mech)
    st = torch.cuda.Stream()
    S = wl.SSSP(V, src, dst, w, s0, chunk, stream=st, hot=hot)
    out = []
    for _ in range(reruns):
        S.reset()
        rt.host_barrier()
        modes = []
        while True:
            more = S.step(st)
            modes.append(S.last_mode)
            if not more:
                break
        out.append((len(modes), modes, S.current.cpu().numpy().copy()))
    rt.check_device()
    S.free()
    return out


@pytest.mark.parametrize("push", ["1", "auto"])
@pytest.mark.parametrize("G,scale,chunk,mech,hot", [(1, 12, 4096, _lib.MECH_FUSED, -1),
                                                    (2, 13, 4096, _lib.MECH_FUSED, 0),
                                                    (3, 12, 8192, _lib.MECH_FUSED, 97),
                                                    (2, 12, 4096, _lib.MECH_INLINE, -1),
                                                    (2, 12, 4096, _lib.MECH_BULK, -1),
                                                    (2, 12, 4096, _lib.MECH_DMA, -1),
                                                    (4, 14, 16384, _lib.MECH_FUSED, 1000)])
def test_sssp_push_rounds_match_oracle(G, scale, chunk, mech, hot, push):
    """Push rounds (reading R24: only the sources whose distance changed in the previous round
    relax their edges into my vertices) give the oracle's distances and round count bit-exactly,
    always-push and auto (pull while the frontier is large), on every rank's full replica; a
    rerun after reset() (dprev then holds the previous run's last input) is identical."""
    src, dst = synth.rmat(scale, 16)
    V = 1 << scale
    w = synth.weights(src.size)
    s0 = int(np.bincount(src, minlength=V).argmax())
    want, want_rounds, _ = oracle.sssp(V, src, dst, w, s0)
    os.environ["PROACT_SSSP_PUSH"] = push if push != "auto" else "-1"
    try:
        outs = run_ranks(G, _sssp_modes_body, V, src, dst, w, s0, chunk, mech, hot, 2)
    finally:
        os.environ.pop("PROACT_SSSP_PUSH", None)
    for runs in outs:
        for rounds, modes, d in runs:
            assert rounds == want_rounds
            assert np.array_equal(d, want)
            assert modes[0] == 1                       # round 0: the frontier is the source
            if push == "1":
                assert all(m == 1 for m in modes)


def test_sssp_auto_switches_pull_and_push():
    """Auto mode on RMAT-14: the large middle rounds pull, the first and the late rounds push."""
    src, dst = synth.rmat(14, 16)
    V = 1 << 14
    w = synth.weights(src.size)
    s0 = int(np.bincount(src, minlength=V).argmax())
    want, want_rounds, _ = oracle.sssp(V, src, dst, w, s0)
    (runs,) = run_ranks(1, _sssp_modes_body, V, src, dst, w, s0, 4096, _lib.MECH_FUSED, -1)
    rounds, modes, d = runs[0]
    assert rounds == want_rounds and np.array_equal(d, want)
    assert 0 in modes and modes[0] == 1 and modes[-1] == 1, modes


def test_votes_are_epoch_tagged():
    """A vote cast in a SIGNAL phase must not leak into a later BARRIER phase that reuses its
    vote slot (epoch + 2): single-rank SIGNAL syncs enqueue nothing, so the slot is never
    cleared and the epoch tag decides (proact::vote)."""
    V = 4096
    src = np.zeros(64, np.uint32)                    # source 0 -> vertices 1..64: one hop
    dst = np.arange(1, 65, dtype=np.uint32)
    w = np.ones(64, np.int32)

    def body(r, G):
        rt.set_config(mech=_lib.MECH_FUSED)
        st = torch.cuda.Stream()
        S = wl.SSSP(V, src, dst, w, 0, 4096, stream=st)
        votes = []
        for barrier in (False, False, True):   # epochs e (vote), e+1 (none), e+2 (none, BARRIER)
            i = S.k & 1
            _lib.check(rt.lib().proact_sssp_phase(S.gid, S.rid[i], S.rid[i ^ 1], int(S.k == 0), wl._s(st)), "sssp")
            rt.phase_sync(st, barrier=barrier)
            S.k += 1
        st.synchronize()
        votes.append(rt.last_vote())
        S.reset()                                  # control: the voting phase itself with BARRIER
        _lib.check(rt.lib().proact_sssp_phase(S.gid, S.rid[0], S.rid[1], 1, wl._s(st)), "sssp")
        rt.phase_sync(st, barrier=True)
        S.k += 1
        st.synchronize()
        votes.append(rt.last_vote())
        rt.check_device()
        S.free()
        return votes

    (votes,) = run_ranks(1, body)
    assert votes == [0, 1]


def test_pagerank_ranks_is_stream_ordered():
    """PageRank.ranks(s) right after the phases (no host sync): the returned tensor must be
    readable on the current stream.  Before the fix .cpu() could run ahead of the copy on `s`
    and return recycled memory (seen as r ~ 3e-42 on the second run in one process)."""
    src, dst = synth.rmat(12, 16)
    V = 1 << 12
    want = oracle.pagerank(V, src, dst, 2).astype(np.float64)

    def body(r, G):
        rt.set_config(mech=_lib.MECH_FUSED)
        s = torch.cuda.Stream()
        P = wl.PageRank(V, src, dst, 4096, stream=s, hot=0)
        for k in range(2):
            P.step(s, barrier=(k == 1))
        out = (P.v0, P.v1, P.ranks(s).cpu().numpy())
        P.free()
        return out

    for _ in range(4):
        for v0, v1, r in run_ranks(2, body):
            assert np.max(np.abs(r - want[v0:v1]) / want[v0:v1]) <= 1e-5
