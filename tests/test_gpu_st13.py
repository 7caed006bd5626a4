"""GPU parity of the 3.5D radius-2 13-point star (st13_run through the C ABI;
SURVEY §8(f) f4, general R of §V; readings X25/X26) against the CPU
oracle on the same seeded grids: FP32 max rel err <= 1e-5, FP64 <= 1e-12,
bit-exact in the oracle-order build, at every compiled depth, ragged and
degenerate shapes (5-point extents: one interior point per axis) and the
configs[1] size.
"""
import numpy as np
import pytest
import torch

import stgen
import paper_conf_sc_nguyensckd10_b200 as st

pytestmark = pytest.mark.gpu

TOL = {np.float32: 1e-5, np.float64: 1e-12}
NU = 0.05
W = (1.0 - 7.5 * NU, 4.0 * NU / 3.0, -NU / 12.0)     # 4th-order Laplacian heat step


def relerr(g, o):
    g = g.astype(np.float64)
    o = o.astype(np.float64)
    return float(np.max(np.abs(g - o) / np.maximum(np.abs(o), 1e-30)))


def run_gpu(a, T, dim_T, exact=False, w=W):
    nz, ny, nx = a.shape
    dt = torch.float32 if a.dtype == np.float32 else torch.float64
    with st.Plan(nx, ny, nz, dt, dim_T) as p:
        if exact:
            p.set_bitexact(True)
        x = torch.from_numpy(a).cuda()
        y = torch.empty_like(x)
        p.st13(x, y, *w, T)
        p.sync()
        return y.cpu().numpy()


SHAPES = [(64, 48, 24), (68, 52, 37), (16, 9, 7), (200, 70, 11), (64, 130, 9), (8, 5, 5)]


@pytest.mark.parametrize("dtype", [np.float32, np.float64])
@pytest.mark.parametrize("dim_T", [1, 2, 3, 4])
def test_ragged_all_depths(oracle_lib, dtype, dim_T):
    for k, (nx, ny, nz) in enumerate(SHAPES):
        if dtype == np.float64 and nx % 2:
            continue
        a = stgen.grid7(nx, ny, nz, 200 + k, dtype)
        T = dim_T * 2 + 1 + k % 3   # several sweeps incl. a remainder sweep
        ref = oracle_lib.st13(a, *W, T)
        got = run_gpu(a, T, dim_T, exact=True)
        assert np.array_equal(got, ref), (nx, ny, nz, T)
        got = run_gpu(a, T, dim_T)
        assert relerr(got, ref) <= TOL[dtype], (nx, ny, nz, T)


def test_dimT_invariance_and_weights(oracle_lib):
    # distinct weights (no heat relation) catch a distance-1 / distance-2 swap
    a = stgen.grid7(96, 80, 40, 7, np.float32)
    w = (0.3, 0.11, -0.013)
    ref = oracle_lib.st13(a, *w, 12)
    outs = [run_gpu(a, 12, d, exact=True, w=w) for d in (1, 2, 3, 4)]
    for o in outs:
        assert np.array_equal(o, ref)


def test_T0_and_host_buffers(oracle_lib):
    a = stgen.grid7(64, 40, 30, 3, np.float32)
    assert np.array_equal(run_gpu(a, 0, 2), a)
    out = np.empty_like(a)
    with st.Plan(64, 40, 30, torch.float32, 2) as p:
        p.set_bitexact(True)
        p.st13(a.copy(), out, *W, 5)                  # host buffers: staged, synchronous
    assert np.array_equal(out, oracle_lib.st13(a, *W, 5))


def test_errors():
    with st.Plan(64, 8, 4, torch.float32, 2) as p:   # nz = 4 < 5: no interior point
        x = torch.zeros(4, 8, 64, device="cuda")
        with pytest.raises(st.StError):
            p.st13(x, torch.empty_like(x), *W, 1)


@pytest.mark.parametrize("dtype,dim_T", [(np.float32, 2), (np.float32, 3), (np.float64, 2)])
def test_config2_size_256(oracle_lib, dtype, dim_T):
    # the configs[1] grid size, T = 20, every point compared
    n, T = 256, 20
    a = stgen.grid7(n, n, n, 2, dtype)
    ref = oracle_lib.st13(a, *W, T)
    assert relerr(run_gpu(a, T, dim_T), ref) <= TOL[dtype]
    assert np.array_equal(run_gpu(a, T, dim_T, exact=True), ref)
