"""Pins of the radius-2 oracle (oracle/oracle.c oracle_st13_*; the general
stencil radius R of §V; readings X25/X26) against facts
fixed by the mathematics, not against the oracle itself.

* constant fixed point when alpha + 6 beta + 6 gamma = 1 (dyadic: bit-exact);
* impulse response: one sweep of a unit impulse is the 13-point star of
  weights (centre alpha, distance 1 beta, distance 2 gamma, nothing on the
  diagonals), two sweeps its self-convolution (exact with dyadic weights);
* polynomial exactness: with alpha = 1 - 7.5 nu, beta = 4 nu / 3,
  gamma = -nu / 12 the update is u + nu * L u with the 4th-order Laplacian L,
  exact on polynomials of degree <= 5; from u0 = x^4 + y^4 + z^4,
  u_T = u0 + 12 T nu (x^2 + y^2 + z^2) + 36 T (T - 1) nu^2 wherever the fixed
  shell has not reached (2 points per step).  A dropped or mis-weighted
  distance-2 term, or a distance-1 weight on the distance-2 points, breaks it
  (guards below);
* brute force: an independent per-point recursion on a small grid (same
  operation order, bit-exact);
* the shell (2 points thick, X26) never changes; x, y, z mirrors bit-exact;
  T-split.
CPU only.
"""
import functools
import itertools

import numpy as np
import pytest

import stgen

DYADIC = (7.0 / 16, 1.0 / 8, -1.0 / 32)          # 7/16 + 6/8 - 6/32 = 1
DISTINCT = (0.3, 0.11, -0.013)


def heat(nu):
    return (1.0 - 7.5 * nu, 4.0 * nu / 3.0, -nu / 12.0)


@pytest.mark.parametrize("dtype", [np.float32, np.float64])
def test_constant_fixed_point_dyadic(oracle_lib, dtype):
    a = np.full((9, 10, 12), 0.75, dtype=dtype)
    assert np.array_equal(oracle_lib.st13(a, *DYADIC, 5), a)


def _star(w):
    k = np.zeros((5, 5, 5))
    k[2, 2, 2] = w[0]
    for axis in range(3):
        for d in (-2, -1, 1, 2):
            idx = [2, 2, 2]
            idx[axis] += d
            k[tuple(idx)] = w[abs(d)]
    return k


@pytest.mark.parametrize("dtype", [np.float32, np.float64])
def test_impulse_one_sweep_is_star(oracle_lib, dtype):
    n = 11
    a = np.zeros((n, n, n), dtype=dtype)
    c = n // 2
    a[c, c, c] = 1
    out = oracle_lib.st13(a, *DISTINCT, 1)
    expect = np.zeros_like(out)
    expect[c - 2:c + 3, c - 2:c + 3, c - 2:c + 3] = _star([dtype(v) for v in DISTINCT]).astype(dtype)
    assert np.array_equal(out, expect)


def test_impulse_two_sweeps_self_convolution():
    import oracle
    n = 15
    a = np.zeros((n, n, n))
    c = n // 2
    a[c, c, c] = 1
    out = oracle.st13(a, *DYADIC, 2)
    k = _star(DYADIC)
    conv = np.zeros((9, 9, 9))           # full 3D convolution of the star with itself
    for i, j, l in itertools.product(range(5), repeat=3):
        if k[i, j, l]:
            conv[i:i + 5, j:j + 5, l:l + 5] += k[i, j, l] * k
    expect = np.zeros_like(out)
    expect[c - 4:c + 5, c - 4:c + 5, c - 4:c + 5] = conv
    assert np.array_equal(out, expect)


def _poly_exact(shape, T, nu):
    nz, ny, nx = shape
    z, y, x = np.meshgrid(np.arange(nz), np.arange(ny), np.arange(nx), indexing="ij")
    p4 = x.astype(float) ** 4 + y.astype(float) ** 4 + z.astype(float) ** 4
    p2 = x.astype(float) ** 2 + y.astype(float) ** 2 + z.astype(float) ** 2
    return p4, p4 + 12 * T * nu * p2 + 36 * T * (T - 1) * nu * nu


@pytest.mark.parametrize("T", [1, 2, 3])
def test_quartic_is_exact_for_the_4th_order_laplacian(oracle_lib, T):
    shape, nu = (20, 21, 22), 0.05
    p4, exact = _poly_exact(shape, T, nu)
    out = oracle_lib.st13(p4, *heat(nu), T)
    r = 2 + 2 * T                        # the fixed shell's influence: 2 points per step
    sl = tuple(slice(r, n - r) for n in shape)
    scale = np.max(np.abs(exact[sl]))
    assert np.max(np.abs(out[sl] - exact[sl])) <= 1e-13 * scale
    # guards: the plausible mistakes fail the same check
    for wrong in ((1 - 6 * nu, nu, 0.0),                    # 2nd-order Laplacian (no distance-2 term)
                  (1 - 7.5 * nu, 4 * nu / 3, nu / 12),      # sign of gamma
                  (1 - 7.5 * nu, -nu / 12, 4 * nu / 3)):    # distance-1 and distance-2 weights swapped
        bad = oracle_lib.st13(p4, *wrong, T)
        assert np.max(np.abs(bad[sl] - exact[sl])) > 1e-6 * scale


def test_brute_force_recursion(oracle_lib):
    # v(p, t) = (alpha v(p, t-1) + beta S1) + gamma S2, shell fixed: memoised
    # per-point recursion written independently of the loop oracle
    shape, T = (8, 9, 10), 3
    for dtype in (np.float32, np.float64):
        a = stgen.grid7(shape[2], shape[1], shape[0], 41, dtype)
        al, be, ga = (dtype(v) for v in DISTINCT)
        nz, ny, nx = shape

        @functools.lru_cache(maxsize=None)
        def v(z, y, x, t):
            if t == 0 or not (2 <= z < nz - 2 and 2 <= y < ny - 2 and 2 <= x < nx - 2):
                return a[z, y, x]
            s1 = (dtype(v(z, y, x - 1, t - 1) + v(z, y, x + 1, t - 1)) +
                  dtype(v(z, y - 1, x, t - 1) + v(z, y + 1, x, t - 1)))
            s1 = dtype(dtype(s1) + dtype(v(z - 1, y, x, t - 1) + v(z + 1, y, x, t - 1)))
            s2 = (dtype(v(z, y, x - 2, t - 1) + v(z, y, x + 2, t - 1)) +
                  dtype(v(z, y - 2, x, t - 1) + v(z, y + 2, x, t - 1)))
            s2 = dtype(dtype(s2) + dtype(v(z - 2, y, x, t - 1) + v(z + 2, y, x, t - 1)))
            return dtype(dtype(dtype(al * v(z, y, x, t - 1)) + dtype(be * s1)) + dtype(ga * s2))

        ref = np.array([[[v(z, y, x, T) for x in range(nx)] for y in range(ny)] for z in range(nz)], dtype=dtype)
        assert np.array_equal(oracle_lib.st13(a, *DISTINCT, T), ref)


@pytest.mark.parametrize("dtype", [np.float32, np.float64])
def test_shell_mirrors_split(oracle_lib, dtype):
    a = stgen.grid7(14, 13, 12, 43, dtype)
    out = oracle_lib.st13(a, *DISTINCT, 6)
    shell = np.ones(a.shape, bool)
    shell[2:-2, 2:-2, 2:-2] = False
    assert np.array_equal(out[shell], a[shell])
    for ax in range(3):
        m = np.flip(a, axis=ax).copy()
        assert np.array_equal(np.flip(oracle_lib.st13(m, *DISTINCT, 6), axis=ax), out)
    assert np.array_equal(oracle_lib.st13(oracle_lib.st13(a, *DISTINCT, 2), *DISTINCT, 4), out)
    assert np.array_equal(oracle_lib.st13(a, *DISTINCT, 0), a)
