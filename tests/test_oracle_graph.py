"""Pins for the PageRank and SSSP oracles (Sec. IV-C).

PageRank (readings R11/R12): after many iterations the oracle must equal the
dense linear solve of (I - d M^T) r = (1-d)/V, M[u,v] = #(u->v)/out(u), which
shares nothing with the oracle's CSC gather; a regular graph gives the uniform
vector exactly; the mass identity sum r' = (1-d) + d * sum_{out(u)>0} r[u] holds.

SSSP (reading R13): final distances equal Dijkstra (heapq, written here);
d^k equals k rounds of dense min-plus brute force; the round count equals the
first k with d^k == d^{k+1}, plus one; invariants d[s]=0 and the triangle
inequality on every edge.
"""
import heapq

import numpy as np
import pytest

import oracle
import synth


def _rand_graph(rng, V, E):
    src = rng.integers(0, V, E).astype(np.uint32)
    dst = rng.integers(0, V, E).astype(np.uint32)
    keep = src != dst
    return src[keep], dst[keep]


@pytest.mark.parametrize("seed", [0, 1, 2])
def test_pagerank_matches_dense_solve(seed):
    rng = np.random.default_rng(seed)
    V = int(rng.integers(5, 64))
    src, dst = _rand_graph(rng, V, int(rng.integers(V, 6 * V)))
    d = oracle.DAMPING
    out = np.bincount(src, minlength=V).astype(np.float64)
    M = np.zeros((V, V))
    np.add.at(M, (src, dst), 1.0)
    M = np.divide(M, out[:, None], out=np.zeros_like(M), where=out[:, None] > 0)
    r_star = np.linalg.solve(np.eye(V) - d * M.T, np.full(V, (1 - d) / V))
    r = oracle.pagerank(V, src, dst, 200).astype(np.float64)
    assert np.max(np.abs(r - r_star) / r_star) < 1e-6


def test_pagerank_regular_graph_is_uniform_exactly():
    V, k = 64, 3
    src = np.repeat(np.arange(V, dtype=np.uint32), k)
    dst = ((src + np.tile(np.array([1, 5, 17], dtype=np.uint32), V)) % V).astype(np.uint32)
    r = oracle.pagerank(V, src, dst, 10)
    assert np.all(r == np.float32(1.0 / V))


def test_pagerank_mass_identity_and_dangling():
    rng = np.random.default_rng(7)
    V = 200
    src, dst = _rand_graph(rng, V, 900)
    keep = src >= 20           # vertices 0..19 dangling (no out-edges)
    src, dst = src[keep], dst[keep]
    out = np.bincount(src, minlength=V)
    d = oracle.DAMPING
    for k in (0, 1, 4):
        rk = oracle.pagerank(V, src, dst, k).astype(np.float64)
        rk1 = oracle.pagerank(V, src, dst, k + 1).astype(np.float64)
        want = (1 - d) + d * rk[out > 0].sum()
        assert abs(rk1.sum() - want) < 1e-6
    assert np.all(oracle.pagerank(V, src, dst, 5) >= np.float32((1 - d) / V) * (1 - 1e-7))


def test_pagerank_empty_graph():
    r = oracle.pagerank(10, np.zeros(0, np.uint32), np.zeros(0, np.uint32), 3)
    assert np.allclose(r, (1 - oracle.DAMPING) / 10, rtol=1e-7)


def _dijkstra(V, src, dst, w, s):
    adj = [[] for _ in range(V)]
    for a, b, c in zip(src.tolist(), dst.tolist(), w.tolist()):
        adj[a].append((b, c))
    dist = [None] * V
    pq = [(0, s)]
    while pq:
        dv, v = heapq.heappop(pq)
        if dist[v] is not None:
            continue
        dist[v] = dv
        for b, c in adj[v]:
            if dist[b] is None:
                heapq.heappush(pq, (dv + c, b))
    return np.array([oracle.INF if x is None else x for x in dist], dtype=np.int64)


@pytest.mark.parametrize("seed", [0, 1, 2, 3])
def test_sssp_final_matches_dijkstra(seed):
    rng = np.random.default_rng(seed)
    V = int(rng.integers(8, 300))
    src, dst = _rand_graph(rng, V, int(rng.integers(V, 5 * V)))
    w = synth.weights(src.size, seed=seed + 11)
    s = int(np.bincount(src, minlength=V).argmax())
    d, rounds, changed = oracle.sssp(V, src, dst, w, s)
    assert np.array_equal(d.astype(np.int64), _dijkstra(V, src, dst, w, s))
    assert changed[-1] == 0 and np.all(changed[:-1] > 0)


def test_sssp_rounds_match_dense_min_plus():
    rng = np.random.default_rng(5)
    V = 40
    src, dst = _rand_graph(rng, V, 90)
    w = synth.weights(src.size, seed=9)
    s = int(np.bincount(src, minlength=V).argmax())
    BIG = np.int64(1) << 40
    Wd = np.full((V, V), BIG, dtype=np.int64)
    np.minimum.at(Wd, (src, dst), w.astype(np.int64))
    dk = np.full(V, BIG, dtype=np.int64)
    dk[s] = 0
    hist = [dk]
    for _ in range(V + 1):
        nxt = np.minimum(hist[-1], np.min(hist[-1][:, None] + Wd, axis=0))
        hist.append(nxt)
    conv = next(k for k in range(V + 1) if np.array_equal(hist[k], hist[k + 1]))
    for k in range(1, conv + 2):
        dk_or, _, _ = oracle.sssp(V, src, dst, w, s, max_rounds=k)
        want = np.where(hist[k] >= BIG, oracle.INF, hist[k])
        assert np.array_equal(dk_or.astype(np.int64), want), k
    _, rounds, _ = oracle.sssp(V, src, dst, w, s)
    assert rounds == conv + 1


def test_sssp_invariants_on_rmat():
    src, dst = synth.rmat(10, 8)
    V = 1 << 10
    w = synth.weights(src.size)
    s = int(np.bincount(src, minlength=V).argmax())
    d, rounds, changed = oracle.sssp(V, src, dst, w, s)
    assert d[s] == 0
    fin = d[src] != oracle.INF
    assert np.all(d[dst[fin]].astype(np.int64) <= d[src[fin]].astype(np.int64) + w[fin])
    assert rounds == changed.size and changed[-1] == 0


def test_rmat_generator_shape():
    src, dst = synth.rmat(12, 16)
    V, E0 = 1 << 12, (1 << 12) * 16
    assert src.size == dst.size and 0.9 * E0 < src.size <= E0
    assert np.all(src != dst) and src.max() < V and dst.max() < V
    deg = np.bincount(src, minlength=V)
    assert deg.max() > 20 * deg.mean()            # heavy tail (RMAT a=.57)
    s2, d2 = synth.rmat(12, 16)
    assert np.array_equal(src, s2) and np.array_equal(dst, d2)
    p = synth.permutation(1000)
    assert np.array_equal(np.sort(p), np.arange(1000))


def test_splitmix64_reference_output():
    # first output of splitmix64 seeded with 0 (Vigna's reference implementation)
    assert synth.splitmix64(0) == 0xE220A8397B1DCDAF


def test_sssp_oracle_independent_of_thread_count():
    """The OpenMP pull (one vertex per iteration, a min over its in-edges) gives the same d and
    round count on 1 thread as on all of them (min over a fixed set is order independent)."""
    src, dst = synth.rmat(10, 8)
    V = 1 << 10
    w = synth.weights(src.size)
    s0 = int(np.bincount(src, minlength=V).argmax())
    n = oracle.get_threads()
    try:
        oracle.set_threads(1)
        d1, r1, c1 = oracle.sssp(V, src, dst, w, s0)
    finally:
        oracle.set_threads(n)
    dn, rn, cn = oracle.sssp(V, src, dst, w, s0)
    assert r1 == rn and np.array_equal(d1, dn) and np.array_equal(c1, cn)
