"""GPU parity of the 3.5D 27-point sweep (st27_run through the C ABI; P:119,
SURVEY §8(f) f1) against the CPU oracle (oracle_st27_*) on the same seeded
grids: bit-exact in the -fmad=false-equivalent build (st_plan_set_bitexact,
reading X24 operation order), FP32 max rel err <= 1e-5 and FP64 <= 1e-12 with
FMA contraction (the 7-point gates of SURVEY §8(c), applied unchanged).
"""
import numpy as np
import pytest
import torch

import stgen
import paper_conf_sc_nguyensckd10_b200 as st

pytestmark = pytest.mark.gpu

TOL = {np.float32: 1e-5, np.float64: 1e-12}
W = (0.3, 0.05, 0.02, 0.01)          # distinct class weights (alpha + 6b + 12g + 8d = 0.92)
MAXD = {np.float32: 4, np.float64: 2}   # bit-exact build (st27.cu); the tolerance build reaches 4 for both


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
        p.st27(x, y, *w, T)
        p.sync()
        return y.cpu().numpy(), p.last_launches()


@pytest.mark.parametrize("dtype", [np.float32, np.float64])
def test_64cube(oracle_lib, dtype):
    a = stgen.grid7(64, 64, 64, 1, dtype)
    ref = oracle_lib.st27(a, *W, 4)
    got, launches = run_gpu(a, 4, 2)
    assert launches == 3                      # 4 = 2+1+1: odd sweep count
    assert relerr(got, ref) <= TOL[dtype]
    got, _ = run_gpu(a, 4, 2, exact=True)
    assert np.array_equal(got, ref)


# several X/Y tiles with a shifted last tile, a sub-warp width, Z chunks and ragged tails
SHAPES = [(68, 52, 37), (128, 96, 20), (16, 9, 5), (200, 70, 11), (36, 33, 64)]


@pytest.mark.parametrize("dtype", [np.float32, np.float64])
@pytest.mark.parametrize("dim_T", [1, 2, 3, 4])
def test_ragged_all_depths_bit_exact(oracle_lib, dtype, dim_T):
    for k, (nx, ny, nz) in enumerate(SHAPES):
        if dtype == np.float64 and nx % 2:
            continue
        a = stgen.grid7(nx, ny, nz, 200 + k, dtype)
        T = min(dim_T, MAXD[dtype]) * 2 + 1 + k
        ref = oracle_lib.st27(a, *W, T)
        got, _ = run_gpu(a, T, dim_T, exact=True)
        assert np.array_equal(got, ref), (nx, ny, nz, T)


@pytest.mark.parametrize("dtype", [np.float32, np.float64])
def test_ragged_tolerance(oracle_lib, dtype):
    for k, (nx, ny, nz) in enumerate(SHAPES):
        if dtype == np.float64 and nx % 2:
            continue
        a = stgen.grid7(nx, ny, nz, 300 + k, dtype)
        ref = oracle_lib.st27(a, *W, 9)
        got, _ = run_gpu(a, 9, MAXD[dtype])
        assert relerr(got, ref) <= TOL[dtype], (nx, ny, nz)


@pytest.mark.parametrize("dtype", [np.float32, np.float64])
@pytest.mark.parametrize("dim_T", [1, 2, 3, 4])
def test_ragged_all_depths_tolerance(oracle_lib, dtype, dim_T):
    # the tolerance build runs the 7-point-machinery kernel (st27t: lag-2 levels,
    # running partial sums) at every depth 1-4, FP64 included; ragged tiles, shifted
    # last tiles, multi-segment CTAs (36 x 33 x 64) and odd/even sweep counts
    for k, (nx, ny, nz) in enumerate(SHAPES):
        a = stgen.grid7(nx, ny, nz, 400 + k, dtype)
        T = dim_T * 2 + 1 + k
        ref = oracle_lib.st27(a, *W, T)
        got, _ = run_gpu(a, T, dim_T)
        assert relerr(got, ref) <= TOL[dtype], (nx, ny, nz, T)


@pytest.mark.parametrize("dtype", [np.float32, np.float64])
def test_degenerate_tolerance(oracle_lib, dtype):
    # single interior row / column / point, thin slabs, T = 0..5, every depth
    for k, (nx, ny, nz) in enumerate([(40, 3, 3), (4, 40, 3), (4, 3, 40), (4, 3, 3), (8, 8, 8), (64, 5, 4)]):
        a = stgen.grid7(nx, ny, nz, 500 + k, dtype)
        for T in (0, 1, 2, 5):
            for d in (1, 2, 4):
                got, _ = run_gpu(a, T, d)
                assert relerr(got, oracle_lib.st27(a, *W, T)) <= TOL[dtype], (nx, ny, nz, T, d)


def test_degenerate_and_host_pointers(oracle_lib):
    a = stgen.grid7(40, 3, 3, 7, np.float32)                 # one interior row
    for T in (0, 1, 2, 5):
        got, _ = run_gpu(a, T, 1, exact=True)
        assert np.array_equal(got, oracle_lib.st27(a, *W, T))
    b = stgen.grid7(48, 40, 12, 8, np.float32)
    out = np.empty_like(b)
    with st.Plan(48, 40, 12, torch.float32, 3) as p:
        p.set_bitexact(True)
        p.st27(b.copy(), out, *W, 7)                         # host buffers: staged, synchronous
    assert np.array_equal(out, oracle_lib.st27(b, *W, 7))


def test_dyadic_fixed_point_and_impulse():
    a = np.full((40, 40, 40), 0.75, dtype=np.float32)
    got, _ = run_gpu(a, 9, 4, w=(0.5, 1 / 16, 1 / 128, 1 / 256))
    assert np.array_equal(got, a)
    z = np.zeros((33, 35, 38), dtype=np.float64)
    z[16, 17, 18] = 1
    got, _ = run_gpu(z, 1, 2)
    cube = got[15:18, 16:19, 17:20]
    for dz in range(3):
        for dy in range(3):
            for dx in range(3):
                assert cube[dz, dy, dx] == W[abs(dz - 1) + abs(dy - 1) + abs(dx - 1)]
    assert np.count_nonzero(got) == 27


def test_256cube_f32(oracle_lib):
    # configs[1]-size grid, full compare (exact at the kernel's deepest depth, tolerance at the default)
    a = stgen.grid7(256, 256, 256, 2, np.float32)
    ref = oracle_lib.st27(a, *W, 12)
    got, _ = run_gpu(a, 12, 4, exact=True)
    assert np.array_equal(got, ref)
    for d in (1, 2, 3, 4):   # the tolerance kernel at every depth (12 = 3x4 = 4x3 = 6x2)
        got, _ = run_gpu(a, 12, d)
        assert relerr(got, ref) <= TOL[np.float32], d
