"""Pins for the microbenchmark oracle (Sec. IV-C, Sec. V-A).

The producer value is a chain of MurmurHash3 finalisers (reading R14).
fmix32 is pinned by MurmurHash3_x86_32's published vectors (tests/golden/): the
test supplies the MurmurHash3 body around oracle.fmix32, so a wrong shift, a
wrong multiplier or a dropped step in the oracle's finaliser fails them.
"""
import os

import numpy as np

import oracle

GOLDEN = os.path.join(os.path.dirname(__file__), "golden", "murmur3_x86_32.txt")
M32 = 0xFFFFFFFF


def _rotl(x, r):
    return ((x << r) | (x >> (32 - r))) & M32


def murmur3_x86_32(data: bytes, seed: int) -> int:
    """MurmurHash3_x86_32 body; finalisation delegated to oracle.fmix32."""
    c1, c2 = 0xCC9E2D51, 0x1B873593
    h = seed & M32
    n = len(data) // 4
    for i in range(n):
        k = int.from_bytes(data[4 * i:4 * i + 4], "little")
        k = (k * c1) & M32
        k = _rotl(k, 15)
        k = (k * c2) & M32
        h ^= k
        h = _rotl(h, 13)
        h = (h * 5 + 0xE6546B64) & M32
    tail = data[4 * n:]
    k = 0
    if len(tail) >= 3:
        k ^= tail[2] << 16
    if len(tail) >= 2:
        k ^= tail[1] << 8
    if len(tail) >= 1:
        k ^= tail[0]
        k = (k * c1) & M32
        k = _rotl(k, 15)
        k = (k * c2) & M32
        h ^= k
    h ^= len(data)
    return oracle.fmix32(h)


def _vectors():
    for line in open(GOLDEN):
        line = line.strip()
        if not line or line.startswith("#"):
            continue
        key, seed, want = line.split()
        data = b"" if key == "-" else bytes.fromhex(key)
        yield data, int(seed, 16), int(want, 16)


def test_fmix32_published_murmur3_vectors():
    n = 0
    for data, seed, want in _vectors():
        assert murmur3_x86_32(data, seed) == want, (data, hex(seed))
        n += 1
    assert n >= 15


def test_fmix32_is_a_bijection_on_a_window():
    # fmix32 is a composition of invertible steps; no collisions on 2^18 inputs
    xs = np.array([oracle.fmix32(i * 2654435761) for i in range(1 << 14)], dtype=np.uint64)
    assert np.unique(xs).size == xs.size
    assert oracle.fmix32(0) == 0          # every step maps 0 to 0


def test_micro_word_chain_and_phase_array():
    seed = 0x5EED
    for k in (0, 1, 4095, 4096, 123456789):
        for p in (0, 1, 7):
            v1 = oracle.micro_word(k, p, seed, 1)
            x = (k ^ ((p * 0x9E3779B9) & M32) ^ seed) & M32
            assert v1 == oracle.fmix32(x)
            v = v1
            for K in range(2, 5):
                v = oracle.fmix32(v)
                assert oracle.micro_word(k, p, seed, K) == v
    arr = oracle.micro_phase(5000, 3, seed, 2)
    assert arr.dtype == np.uint32 and arr.size == 5000
    for k in (0, 17, 4096, 4999):
        assert int(arr[k]) == oracle.micro_word(k, 3, seed, 2)
    # phases differ everywhere but a negligible number of words
    assert np.count_nonzero(oracle.micro_phase(5000, 4, seed, 2) == arr) < 5


def test_micro_empty():
    assert oracle.micro_phase(0, 0, 1).size == 0
