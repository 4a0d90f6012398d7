"""Pins for O-proto, the protocol simulator (Sec. III-B, III-C L137).

G simulated ranks (threads), producer CTAs storing only to the local copy and
bumping per-chunk counters, polling agents pushing ready chunks to every peer,
arrival flags and done credits, all under random yields.  It must reach exactly
the plain single-array result (the paper: PROACT only changes when bytes move,
L123) with invariants I1-I3 holding, for ragged ownerships and chunk sizes.
"""
import numpy as np
import pytest

import oracle
import synth


@pytest.mark.parametrize("G,W,chunk,tile", [(1, 1000, 64, 100), (2, 4096, 256, 256),
                                            (3, 5003, 97, 128), (4, 10000, 512, 1024)])
def test_proto_micro_all_gather(G, W, chunk, tile):
    phases = 3
    rc, reps = oracle.proto_run(G, "micro", W, chunk, tile, phases, K=2, rng_seed=G * 7 + 1)
    assert rc == 0, oracle.PROTO_ERRORS.get(rc, rc)
    want = oracle.micro_phase(W, phases - 1, 0x5EED, 2)
    for g in range(G):
        assert np.array_equal(reps[g], want)


@pytest.mark.parametrize("G,N,chunk,tile", [(1, 12, 16, 12), (2, 16, 16, 32),
                                            (3, 19, 7, 19), (4, 22, 11, 44)])
def test_proto_jacobi_matches_plain_jacobi(G, N, chunk, tile):
    phases = 5
    x0 = synth.jacobi_init(N)
    rc, reps = oracle.proto_run(G, "jacobi", N, chunk, tile, phases, P=3, A=2,
                                rng_seed=N, init=x0)
    assert rc == 0, oracle.PROTO_ERRORS.get(rc, rc)
    want = oracle.jacobi(x0, phases).view(np.uint32).reshape(-1)
    for g in range(G):
        assert np.array_equal(reps[g], want), g
