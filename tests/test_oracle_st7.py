"""Pins of the 7-point oracle (oracle/oracle.c) against
facts fixed by the paper and the mathematics, not against itself.

P1 constant fixed point, P3 Dirichlet eigenmode closed form, impulse response
golden values (tests/golden/st7_impulse.txt), P4 brute-force recursion,
P5 structural symmetries / T-split, linearity.  CPU only.
"""
import itertools
import math
import os

import numpy as np
import pytest

import stgen

GOLDEN = os.path.join(os.path.dirname(__file__), "golden")


@pytest.mark.parametrize("dtype", [np.float32, np.float64])
def test_constant_fixed_point_dyadic(oracle_lib, dtype):
    # alpha + 6 beta = 1 with dyadic alpha, beta, c: every op is exact (P1)
    a = np.full((9, 10, 12), 0.75, dtype=dtype)
    out = oracle_lib.st7(a, 0.25, 0.125, 5)
    assert np.array_equal(out, a)


@pytest.mark.parametrize("dtype,tol", [(np.float32, 4e-7), (np.float64, 1e-15)])
def test_constant_fixed_point_rounding(oracle_lib, dtype, tol):
    a = np.full((8, 9, 10), 0.3, dtype=dtype)
    out = oracle_lib.st7(a, 0.4, 0.1, 6)
    assert np.max(np.abs(out.astype(np.float64) - 0.3)) <= 6 * tol


def _eigenmode(nx, ny, nz, k, l, m):
    x = np.arange(nx)
    y = np.arange(ny)
    z = np.arange(nz)
    phx = np.sin(k * np.pi * x / (nx - 1))
    phy = np.sin(l * np.pi * y / (ny - 1))
    phz = np.sin(m * np.pi * z / (nz - 1))
    phi = phz[:, None, None] * phy[None, :, None] * phx[None, None, :]
    # shell exactly zero (sin(k*pi) is ~1e-16 in floating point)
    phi[0] = phi[-1] = 0
    phi[:, 0] = phi[:, -1] = 0
    phi[:, :, 0] = phi[:, :, -1] = 0
    lam = lambda a, b: a + 2 * b * (math.cos(k * math.pi / (nx - 1)) + math.cos(l * math.pi / (ny - 1))
                                     + math.cos(m * math.pi / (nz - 1)))
    return phi, lam


@pytest.mark.parametrize("klm", [(1, 1, 1), (2, 1, 3), (3, 4, 2)])
def test_dirichlet_eigenmode_f64(oracle_lib, klm):
    # P3: phi is an eigenvector of one sweep with eigenvalue lambda (closed form)
    nx, ny, nz, T = 12, 10, 9, 20
    alpha, beta = 0.4, 0.1
    phi, lam = _eigenmode(nx, ny, nz, *klm)
    out = oracle_lib.st7(phi, alpha, beta, T)
    expect = lam(alpha, beta) ** T * phi
    scale = np.max(np.abs(expect))
    assert np.max(np.abs(out - expect)) <= 1e-12 * T * max(scale, 1e-300) + 1e-300


def test_dirichlet_eigenmode_f32(oracle_lib):
    nx, ny, nz, T = 12, 10, 9, 10
    phi, lam = _eigenmode(nx, ny, nz, 1, 2, 1)
    out = oracle_lib.st7(phi.astype(np.float32), 0.4, 0.1, T).astype(np.float64)
    expect = lam(0.4, 0.1) ** T * phi
    assert np.max(np.abs(out - expect)) <= 1e-6 * T * np.max(np.abs(expect))


def test_wrong_lambda_would_fail(oracle_lib):
    # guard: the eigenmode pin is sensitive to a dropped neighbour term
    nx, ny, nz = 12, 10, 9
    phi, lam = _eigenmode(nx, ny, nz, 1, 1, 1)
    out = oracle_lib.st7(phi, 0.4, 0.1, 1)
    wrong = (0.4 + 2 * 0.1 * (math.cos(math.pi / (nx - 1)) + math.cos(math.pi / (ny - 1)))) * phi
    assert np.max(np.abs(out - wrong)) > 1e-3


def _golden_impulse():
    rows = []
    with open(os.path.join(GOLDEN, "st7_impulse.txt")) as fh:
        for line in fh:
            line = line.strip()
            if not line or line.startswith("#"):
                continue
            t, dx, dy, dz, v = line.split()
            rows.append((int(t), int(dx), int(dy), int(dz), float(v)))
    return rows


def test_impulse_response_golden(oracle_lib):
    n, c = 11, 5
    a = np.zeros((n, n, n), dtype=np.float64)
    a[c, c, c] = 1.0
    outs = {t: oracle_lib.st7(a, 0.4, 0.1, t) for t in (1, 2, 3)}
    for t, dx, dy, dz, v in _golden_impulse():
        got = outs[t][c + dz, c + dy, c + dx]
        assert abs(got - v) <= 1e-15, (t, dx, dy, dz, got, v)
    # total "mass" of the free-space response is (alpha + 6 beta)^T = 1
    for t in (1, 2, 3):
        assert abs(outs[t].sum() - 1.0) <= 1e-14


def _walks(k, p):
    """number of length-k walks on Z^3 from 0 to p (independent combinatorics)."""
    total = 0
    for a in range(k + 1):
        for b in range(k + 1 - a):
            c = k - a - b
            # a steps along x, b along y, c along z; each axis: n steps ending at d
            ways = math.factorial(k) // (math.factorial(a) * math.factorial(b) * math.factorial(c))
            for n_, d in ((a, p[0]), (b, p[1]), (c, p[2])):
                if (n_ + d) % 2 or abs(d) > n_:
                    ways = 0
                    break
                ways *= math.comb(n_, (n_ + d) // 2)
            total += ways
    return total


def test_impulse_response_closed_form(oracle_lib):
    # (alpha I + beta S)^T delta = sum_k C(T,k) alpha^(T-k) beta^k walks_k
    n, c, T = 13, 6, 4
    alpha, beta = 0.4, 0.1
    a = np.zeros((n, n, n))
    a[c, c, c] = 1.0
    out = oracle_lib.st7(a, alpha, beta, T)
    for p in itertools.product(range(-T, T + 1), repeat=3):
        v = sum(math.comb(T, k) * alpha ** (T - k) * beta ** k * _walks(k, p) for k in range(T + 1))
        assert abs(out[c + p[2], c + p[1], c + p[0]] - v) <= 1e-15


def _brute(a, alpha, beta, T, p, memo):
    """per-point recursion v(p,t) = alpha v(p,t-1) + beta * sum of neighbours,
    shell fixed, in the canonical order (X2) — an independent formulation."""
    key = (p, T)
    if key in memo:
        return memo[key]
    z, y, x = p
    nz, ny, nx = a.shape
    if T == 0 or x in (0, nx - 1) or y in (0, ny - 1) or z in (0, nz - 1):
        v = a[z, y, x]
    else:
        g = lambda q: _brute(a, alpha, beta, T - 1, q, memo)
        sx = g((z, y, x - 1)) + g((z, y, x + 1))
        sy = g((z, y - 1, x)) + g((z, y + 1, x))
        sz = g((z - 1, y, x)) + g((z + 1, y, x))
        s = (sx + sy) + sz
        v = alpha * g(p) + beta * s
    memo[key] = v
    return v


@pytest.mark.parametrize("dtype", [np.float32, np.float64])
def test_bruteforce_8cube(oracle_lib, dtype):
    a = stgen.grid7(8, 8, 8, 11, dtype)
    al, be = dtype(0.4), dtype(0.1)
    for T in (1, 2, 4):
        out = oracle_lib.st7(a, 0.4, 0.1, T)
        memo = {}
        ref = np.empty_like(a)
        for p in itertools.product(range(8), repeat=3):
            ref[p] = _brute(a, al, be, T, p, memo)
        assert np.array_equal(out, ref), T


@pytest.mark.parametrize("dtype", [np.float32, np.float64])
def test_structural(oracle_lib, dtype):
    a = stgen.grid7(16, 16, 14, 5, dtype)
    al, be, T = 0.4, 0.1, 6
    out = oracle_lib.st7(a, al, be, T)
    # T = 0 copies
    assert np.array_equal(oracle_lib.st7(a, al, be, 0), a)
    # shell unchanged (Dirichlet, X1)
    for sl in (np.s_[0], np.s_[-1], np.s_[:, 0], np.s_[:, -1], np.s_[:, :, 0], np.s_[:, :, -1]):
        assert np.array_equal(out[sl], a[sl])
    # interior changed
    assert not np.array_equal(out[1:-1, 1:-1, 1:-1], a[1:-1, 1:-1, 1:-1])
    # mirror symmetries are bit-exact with the canonical order (P5)
    for ax in (0, 1, 2):
        m = oracle_lib.st7(np.ascontiguousarray(np.flip(a, ax)), al, be, T)
        assert np.array_equal(np.flip(m, ax), out), ax
    # X<->Y transpose (nx == ny) is bit-exact
    tr = oracle_lib.st7(np.ascontiguousarray(a.transpose(0, 2, 1)), al, be, T)
    assert np.array_equal(tr.transpose(0, 2, 1), out)
    # T1 + T2 split equals one run of T
    mid = oracle_lib.st7(a, al, be, 2)
    assert np.array_equal(oracle_lib.st7(mid, al, be, T - 2), out)


def test_linearity_and_xz_transpose(oracle_lib):
    a = stgen.grid7(12, 12, 12, 7, np.float64)
    b = stgen.grid7(12, 12, 12, 8, np.float64)
    T = 5
    ra, rb = oracle_lib.st7(a, 0.4, 0.1, T), oracle_lib.st7(b, 0.4, 0.1, T)
    rab = oracle_lib.st7(a + 2 * b, 0.4, 0.1, T)
    assert np.max(np.abs(rab - (ra + 2 * rb))) <= 1e-13
    tz = oracle_lib.st7(np.ascontiguousarray(a.transpose(2, 1, 0)), 0.4, 0.1, T)
    assert np.max(np.abs(tz.transpose(2, 1, 0) - ra)) <= 1e-14


def test_maximum_principle(oracle_lib):
    # alpha, beta >= 0 and alpha + 6 beta = 1: a convex average, values stay in [min, max]
    a = stgen.grid7(20, 18, 16, 9, np.float32)
    out = oracle_lib.st7(a, 0.4, 0.1, 30)
    assert out.min() >= a.min() and out.max() <= a.max()
