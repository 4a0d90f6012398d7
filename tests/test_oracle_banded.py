"""Pins for the banded-matrix Jacobi oracle (Sec. IV-C).

Reading R19: fp32, fixed summation order, no FMA, IEEE division.  Pins:
  * exact fixed point: with dyadic A and integer x*, b = A x* is exact in fp32 and x* must be
    reproduced bit-exactly every iteration (a dropped term, a wrong sign or a shifted index of
    any diagonal breaks it);
  * w = 0: x' = b / diag, closed form;
  * convergence to numpy's dense solve of A x = b for the diagonally dominant synthetic system.
"""
import numpy as np
import pytest

import oracle
import synth


def _dense(a):
    nd, N = a.shape
    w = (nd - 1) // 2
    A = np.zeros((N, N))
    for o in range(-w, w + 1):
        for i in range(N):
            if 0 <= i + o < N:
                A[i, i + o] = a[o + w, i]
    return A


@pytest.mark.parametrize("N,w", [(17, 1), (40, 3), (64, 7)])
def test_dyadic_fixed_point_bit_exact(N, w):
    rng = np.random.default_rng(N + w)
    a = np.zeros((2 * w + 1, N), dtype=np.float32)
    for o in range(-w, w + 1):
        for i in range(N):
            if o == 0:
                a[o + w, i] = 4.0
            elif 0 <= i + o < N:
                a[o + w, i] = -float(rng.integers(1, 4)) / 16.0
    x_star = rng.integers(-8, 9, N).astype(np.float32)
    b = (_dense(a) @ x_star.astype(np.float64)).astype(np.float32)   # exact: dyadic, small
    y = oracle.banded_jacobi(a, b, x_star, 5)
    assert np.array_equal(y, x_star)


def test_zero_bandwidth_closed_form():
    a, b = synth.banded(100, 0)
    x = oracle.banded_jacobi(a, b, np.zeros(100, np.float32), 3)
    assert np.array_equal(x, (b / a[0]).astype(np.float32))


def test_converges_to_dense_solve():
    N, w = 200, 5
    a, b = synth.banded(N, w)
    x = oracle.banded_jacobi(a, b, np.zeros(N, np.float32), 200).astype(np.float64)
    xs = np.linalg.solve(_dense(a), b.astype(np.float64))
    assert np.max(np.abs(x - xs) / np.abs(xs)) < 1e-5


def test_banded_generator_recipe():
    a, b = synth.banded(50, 4)
    assert a.shape == (9, 50) and np.all(a[4] == 2.0)
    assert np.all(a[0, :4] == 0) and np.all(a[8, -4:] == 0)        # outside the matrix
    assert np.all(np.abs(a[np.arange(9) != 4]).sum(axis=0) <= 1.0)   # dominance
    assert b.min() >= 1.0 and b.max() < 2.0
