"""Pins for the Jacobi oracle (Sec. IV-C, configs 1-2 of BASELINE.json).

Reading R9/R10: Laplace, Dirichlet boundary copied through,
x' = 0.25 * ((up + down) + (left + right)) in fp32.  Pins that do not re-type
the formula:
  * discrete harmonic functions (affine, bilinear) are fixed points, bit-exact
    with dyadic values -- a dropped term, a wrong sign or a wrong neighbour
    index breaks them;
  * the sine mode sin(p pi i/(N-1)) sin(q pi j/(N-1)) with zero boundary is an
    eigenvector with eigenvalue (cos(p pi/(N-1)) + cos(q pi/(N-1))) / 2;
  * transpose symmetry, maximum principle, boundary copy-through;
  * a non-symmetric mode (p != q) on a non-square-symmetric init catches a
    transposed operand together with the eigenvalue test.
"""
import numpy as np

import oracle
import synth


def test_affine_and_bilinear_fixed_points_bit_exact():
    N = 24
    i, j = np.meshgrid(np.arange(N), np.arange(N), indexing="ij")
    for f in (1.0 + i / 64.0 + j / 128.0,
              2.0 - i / 32.0 + 3 * j / 256.0,
              1.0 + (i * j) / 1024.0):
        x = f.astype(np.float32)
        y = oracle.jacobi(x, 7)
        assert np.array_equal(y.view(np.uint32), x.view(np.uint32))


def test_sine_mode_decays_by_closed_form_eigenvalue():
    N = 33
    for p, q in ((1, 1), (2, 3), (5, 1)):
        i, j = np.meshgrid(np.arange(N), np.arange(N), indexing="ij")
        x0 = np.sin(p * np.pi * i / (N - 1)) * np.sin(q * np.pi * j / (N - 1))
        x0[0, :] = x0[-1, :] = x0[:, 0] = x0[:, -1] = 0.0
        lam = (np.cos(p * np.pi / (N - 1)) + np.cos(q * np.pi / (N - 1))) / 2.0
        k = 9
        y = oracle.jacobi(x0.astype(np.float32), k).astype(np.float64)
        want = (lam ** k) * x0
        assert np.max(np.abs(y - want)) < 2e-6 * max(1.0, np.max(np.abs(want))) + 1e-6


def test_single_step_matches_eigen_relation_for_asymmetric_mode():
    N = 17
    i, j = np.meshgrid(np.arange(N), np.arange(N), indexing="ij")
    x0 = np.sin(3 * np.pi * i / (N - 1)) * np.sin(1 * np.pi * j / (N - 1))
    x0[0, :] = x0[-1, :] = x0[:, 0] = x0[:, -1] = 0.0
    lam = (np.cos(3 * np.pi / (N - 1)) + np.cos(np.pi / (N - 1))) / 2.0
    y = oracle.jacobi_step(x0.astype(np.float32)).astype(np.float64)
    assert np.max(np.abs(y - lam * x0)) < 1e-6


def test_symmetry_maximum_principle_boundary():
    N = 40
    x0 = synth.jacobi_init(N)
    sym = np.triu(x0) + np.triu(x0, 1).T          # transpose-symmetric init
    y = oracle.jacobi(sym, 12)
    assert np.array_equal(y, y.T)
    z = oracle.jacobi(x0, 12)
    assert z.min() >= x0.min() and z.max() <= x0.max()
    assert np.array_equal(z[0], x0[0]) and np.array_equal(z[-1], x0[-1])
    assert np.array_equal(z[:, 0], x0[:, 0]) and np.array_equal(z[:, -1], x0[:, -1])


def test_iters_compose_and_degenerate_sizes():
    x0 = synth.jacobi_init(20)
    a = oracle.jacobi(oracle.jacobi(x0, 3), 4)
    b = oracle.jacobi(x0, 7)
    assert np.array_equal(a, b)
    assert np.array_equal(oracle.jacobi(x0, 0), x0)
    for N in (1, 2):      # every cell is boundary: identity
        x = synth.jacobi_init(N)
        assert np.array_equal(oracle.jacobi(x, 5), x)


def test_jacobi_init_recipe():
    x = synth.jacobi_init(64)
    assert x.dtype == np.float32 and x.min() >= 1.0 and x.max() < 2.0
    m = (x.astype(np.float64) - 1.0) * (1 << 23)
    assert np.array_equal(m, np.round(m))      # exactly 23-bit dyadic values
    part = synth.jacobi_init(64, row0=10, nrows=5)
    assert np.array_equal(part, x[10:15])
