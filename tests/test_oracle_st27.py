"""Pins of the 27-point oracle (oracle/oracle.c oracle_st27_*; SURVEY
§8(f) f1) against facts fixed by the paper and the mathematics, not against
itself.

* constant fixed point when alpha + 6 beta + 12 gamma + 8 delta = 1 (dyadic:
  bit-exact);
* impulse response: one sweep of a unit impulse reproduces the 3x3x3 weight
  cube (centre/face/edge/corner classes of P:119), two sweeps its
  self-convolution (exact with dyadic weights);
* Dirichlet eigenmode: sin modes are eigenvectors with the closed-form
  eigenvalue alpha + 2 beta S1 + 4 gamma S2 + 8 delta S3 (cx, cy, cz cosines;
  S1 = cx+cy+cz, S2 = cx cy + cy cz + cz cx, S3 = cx cy cz) — distinct weights
  make a neighbour put in the wrong class fail;
* brute force: an independent np.roll sum over the 26 offsets on a random grid
  (fp64, to rounding);
* x, y, z mirror symmetry bit-exact (reading X24 pairs every sum), T-split.
CPU only.
"""
import itertools
import math

import numpy as np
import pytest

import stgen

DYADIC = (0.5, 1.0 / 16, 1.0 / 128, 1.0 / 256)       # 1/2 + 6/16 + 12/128 + 8/256 = 1
DISTINCT = (0.3, 0.05, 0.02, 0.01)


def _weight(dx, dy, dz, w):
    return w[abs(dx) + abs(dy) + abs(dz)]


@pytest.mark.parametrize("dtype", [np.float32, np.float64])
def test_constant_fixed_point_dyadic(oracle_lib, dtype):
    a = np.full((9, 10, 12), 0.75, dtype=dtype)
    assert np.array_equal(oracle_lib.st27(a, *DYADIC, 5), a)


@pytest.mark.parametrize("dtype", [np.float32, np.float64])
def test_impulse_one_sweep_is_weight_cube(oracle_lib, dtype):
    n = 9
    a = np.zeros((n, n, n), dtype=dtype)
    c = n // 2
    a[c, c, c] = 1
    out = oracle_lib.st27(a, *DISTINCT, 1)
    expect = np.zeros_like(out)
    for dz, dy, dx in itertools.product((-1, 0, 1), repeat=3):
        expect[c + dz, c + dy, c + dx] = dtype(_weight(dx, dy, dz, DISTINCT))
    assert np.array_equal(out, expect)


def test_impulse_two_sweeps_self_convolution(oracle_lib):
    n = 11
    a = np.zeros((n, n, n))
    c = n // 2
    a[c, c, c] = 1
    out = oracle_lib.st27(a, *DYADIC, 2)
    k = np.zeros((3, 3, 3))
    for dz, dy, dx in itertools.product((-1, 0, 1), repeat=3):
        k[dz + 1, dy + 1, dx + 1] = _weight(dx, dy, dz, DYADIC)
    expect = np.zeros((5, 5, 5))
    for i, j in itertools.product(itertools.product(range(3), repeat=3), repeat=2):
        expect[i[0] + j[0], i[1] + j[1], i[2] + j[2]] += k[i] * k[j]
    assert np.array_equal(out[c - 2:c + 3, c - 2:c + 3, c - 2:c + 3], expect)
    rest = out.copy()
    rest[c - 2:c + 3, c - 2:c + 3, c - 2:c + 3] = 0
    assert not rest.any()


def _eigen(nx, ny, nz, k, l, m, w):
    x, y, z = np.arange(nx), np.arange(ny), np.arange(nz)
    phi = (np.sin(m * np.pi * z / (nz - 1))[:, None, None] * np.sin(l * np.pi * y / (ny - 1))[None, :, None]
           * np.sin(k * np.pi * x / (nx - 1))[None, None, :])
    phi[0] = phi[-1] = 0
    phi[:, 0] = phi[:, -1] = 0
    phi[:, :, 0] = phi[:, :, -1] = 0
    cx, cy, cz = (math.cos(k * math.pi / (nx - 1)), math.cos(l * math.pi / (ny - 1)),
                  math.cos(m * math.pi / (nz - 1)))
    a, b, g, d = w
    lam = a + 2 * b * (cx + cy + cz) + 4 * g * (cx * cy + cy * cz + cz * cx) + 8 * d * cx * cy * cz
    return phi, lam


@pytest.mark.parametrize("klm", [(1, 1, 1), (2, 1, 3), (3, 4, 2)])
def test_dirichlet_eigenmode_f64(oracle_lib, klm):
    nx, ny, nz, T = 12, 10, 9, 12
    phi, lam = _eigen(nx, ny, nz, *klm, DISTINCT)
    out = oracle_lib.st27(phi, *DISTINCT, T)
    expect = lam ** T * phi
    assert np.max(np.abs(out - expect)) <= 1e-12 * T * np.max(np.abs(expect))


def test_dirichlet_eigenmode_f32(oracle_lib):
    nx, ny, nz, T = 12, 10, 9, 8
    phi, lam = _eigen(nx, ny, nz, 1, 2, 1, DISTINCT)
    out = oracle_lib.st27(phi.astype(np.float32), *DISTINCT, T).astype(np.float64)
    expect = lam ** T * phi
    assert np.max(np.abs(out - expect)) <= 1e-6 * T * np.max(np.abs(expect))


def test_eigenmode_detects_swapped_classes(oracle_lib):
    # guard: exchanging the edge and corner weights changes lambda measurably
    phi, lam = _eigen(12, 10, 9, 1, 1, 1, DISTINCT)
    _, lam_wrong = _eigen(12, 10, 9, 1, 1, 1, (0.3, 0.05, 0.01, 0.02))
    out = oracle_lib.st27(phi, *DISTINCT, 1)
    assert abs(lam - lam_wrong) > 1e-3
    assert np.max(np.abs(out - lam_wrong * phi)) > 1e-4


def _brute(a, w, T):
    a = a.copy()
    inner = (slice(1, -1),) * 3
    for _ in range(T):
        b = a.copy()
        acc = np.zeros_like(a)
        for dz, dy, dx in itertools.product((-1, 0, 1), repeat=3):
            acc += _weight(dx, dy, dz, w) * np.roll(a, (-dz, -dy, -dx), axis=(0, 1, 2))
        b[inner] = acc[inner]
        a = b
    return a


def test_brute_force_random(oracle_lib):
    a = stgen.grid7(8, 9, 7, seed=11, dtype=np.float64)
    out = oracle_lib.st27(a, *DISTINCT, 3)
    assert np.max(np.abs(out - _brute(a, DISTINCT, 3))) <= 1e-14


@pytest.mark.parametrize("dtype", [np.float32, np.float64])
def test_mirrors_bit_exact_and_shell_fixed(oracle_lib, dtype):
    a = np.random.default_rng(5).random((10, 11, 12)).astype(dtype)
    out = oracle_lib.st27(a, *DISTINCT, 4)
    for ax in range(3):
        m = oracle_lib.st27(np.ascontiguousarray(np.flip(a, ax)), *DISTINCT, 4)
        assert np.array_equal(np.flip(m, ax), out)
    for sl in [np.s_[0], np.s_[-1], np.s_[:, 0], np.s_[:, -1], np.s_[:, :, 0], np.s_[:, :, -1]]:
        assert np.array_equal(out[sl], a[sl])
    assert np.array_equal(oracle_lib.st27(a, *DISTINCT, 0), a)


def test_t_split(oracle_lib):
    a = np.random.default_rng(6).random((9, 9, 10)).astype(np.float32)
    whole = oracle_lib.st27(a, *DISTINCT, 5)
    split = oracle_lib.st27(oracle_lib.st27(a, *DISTINCT, 2), *DISTINCT, 3)
    assert np.array_equal(whole, split)
