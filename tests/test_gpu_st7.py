"""GPU parity of the 3.5D 7-point sweep (st7_run through the C ABI) against
the CPU oracle on the same seeded grids (SURVEY §8(c) gates):
FP32 max rel err <= 1e-5, FP64 <= 1e-12, bit-exact in the -fmad=false /
oracle-order build (st_plan_set_bitexact).
"""
import numpy as np
import pytest
import torch

import stgen
import paper_conf_sc_nguyensckd10_b200 as st

pytestmark = pytest.mark.gpu

TOL = {np.float32: 1e-5, np.float64: 1e-12}


def relerr(g, o):
    g = g.astype(np.float64)
    o = o.astype(np.float64)
    return float(np.max(np.abs(g - o) / np.maximum(np.abs(o), 1e-30)))


def run_gpu(a, alpha, beta, T, dim_T, exact=False):
    nz, ny, nx = a.shape
    dt = torch.float32 if a.dtype == np.float32 else torch.float64
    with st.Plan(nx, ny, nz, dt, dim_T) as p:
        if exact:
            p.set_bitexact(True)
        x = torch.from_numpy(a).cuda()
        y = torch.empty_like(x)
        p.st7(x, y, alpha, beta, T)
        p.sync()
        return y.cpu().numpy(), p.info()


@pytest.mark.parametrize("dtype", [np.float32, np.float64])
def test_config1_64cube(oracle_lib, dtype):
    # BASELINE configs[0]: 64^3, T=4, dim_T=2, seed 1
    a = stgen.grid7(64, 64, 64, 1, dtype)
    ref = oracle_lib.st7(a, 0.4, 0.1, 4)
    got, _ = run_gpu(a, 0.4, 0.1, 4, 2)
    assert relerr(got, ref) <= TOL[dtype]
    got, _ = run_gpu(a, 0.4, 0.1, 4, 2, exact=True)
    assert np.array_equal(got, ref)


SHAPES = [(68, 52, 37), (128, 96, 20), (16, 9, 5), (200, 70, 11), (64, 130, 9)]


@pytest.mark.parametrize("dtype", [np.float32, np.float64])
@pytest.mark.parametrize("dim_T", [1, 2, 3, 4, 5, 6, 7, 8])
def test_ragged_all_depths(oracle_lib, dtype, dim_T):
    for k, (nx, ny, nz) in enumerate(SHAPES):
        if dtype == np.float64 and nx % 2:
            continue
        a = stgen.grid7(nx, ny, nz, 100 + k, dtype)
        T = dim_T * 2 + 1 + k  # several sweeps incl. a remainder sweep
        ref = oracle_lib.st7(a, 0.4, 0.1, T)
        got, _ = run_gpu(a, 0.4, 0.1, T, dim_T, exact=True)
        assert np.array_equal(got, ref), (nx, ny, nz, T)
        got, _ = run_gpu(a, 0.4, 0.1, T, dim_T)
        assert relerr(got, ref) <= TOL[dtype], (nx, ny, nz, T)


def test_dimT_invariance_bitexact():
    a = stgen.grid7(96, 80, 40, 7, np.float32)
    outs = [run_gpu(a, 0.4, 0.1, 12, d, exact=True)[0] for d in range(1, 9)]
    for o in outs[1:]:
        assert np.array_equal(o, outs[0])


def test_T0_T1_and_shell(oracle_lib):
    a = stgen.grid7(64, 40, 30, 3, np.float32)
    got, _ = run_gpu(a, 0.4, 0.1, 0, 4)
    assert np.array_equal(got, a)
    got, _ = run_gpu(a, 0.4, 0.1, 1, 4, exact=True)
    assert np.array_equal(got, oracle_lib.st7(a, 0.4, 0.1, 1))
    got, _ = run_gpu(a, 0.4, 0.1, 9, 4)
    for sl in (np.s_[0], np.s_[-1], np.s_[:, 0], np.s_[:, -1], np.s_[:, :, 0], np.s_[:, :, -1]):
        assert np.array_equal(got[sl], a[sl])


def test_host_pointer_path(oracle_lib):
    a = stgen.grid7(64, 48, 24, 5, np.float32)
    out = np.empty_like(a)
    h = st.st_plan_create(64, 48, 24, st.ST_F32, 3)
    try:
        st.st_plan_set_bitexact(h, True)
        st.st7_run(h, a.copy(), out, 0.4, 0.1, 7)
    finally:
        st.st_destroy(h)
    assert np.array_equal(out, oracle_lib.st7(a, 0.4, 0.1, 7))


def test_errors():
    with pytest.raises(st.StError):
        st.st_plan_create(2, 64, 64, st.ST_F32, 2)
    with pytest.raises(st.StError):
        st.st_plan_create(64, 64, 64, st.ST_F32, 9)
    with pytest.raises(st.StError):
        st.st_plan_create(66, 64, 64, st.ST_F32, 2)   # 264 B rows: not a 16 B multiple
    with st.Plan(64, 64, 64, torch.float32, 2) as p:
        x = torch.zeros(64, 64, 64, device="cuda")
        with pytest.raises(st.StError):
            p.st7(x, x, 0.4, 0.1, 3)                 # aliasing
        with pytest.raises(st.StError):
            p.st7(x, torch.empty_like(x), 0.4, 0.1, -1)
        with pytest.raises(ValueError):                 # mixed host/device (binding check)
            p.st7(x, np.empty((64, 64, 64), np.float32), 0.4, 0.1, 1)
        with pytest.raises(st.StError):                 # mixed host/device (C ABI check)
            st.st7_run(p.h, x, np.empty((64, 64, 64), np.float32), 0.4, 0.1, 1)
        with pytest.raises(ValueError):                 # short buffer
            p.st7(x, torch.empty(64, 64, 63, device="cuda"), 0.4, 0.1, 1)
        with pytest.raises(ValueError):                 # dtype does not match the plan
            p.st7(x.double(), torch.empty(64, 64, 64, dtype=torch.float64, device="cuda"), 0.4, 0.1, 1)


@pytest.mark.parametrize("dtype,dim_T", [(np.float32, 3), (np.float32, 4), (np.float64, 3)])
def test_config2_256_full_grid(oracle_lib, dtype, dim_T):
    # BASELINE configs[1] exactly as bench.py times it: 256^3, T = 100, seed 2
    n, T = 256, 100
    a = stgen.grid7(n, n, n, 2, dtype)
    ref = oracle_lib.st7(a, 0.4, 0.1, T)
    got, info = run_gpu(a, 0.4, 0.1, T, dim_T)
    assert relerr(got, ref) <= TOL[dtype]
    got, _ = run_gpu(a, 0.4, 0.1, T, dim_T, exact=True)
    assert np.array_equal(got, ref)


def test_config3_512_full_grid(oracle_lib):
    # configs[3] per-GPU size in the launch configuration bench.py's 512^3 extra times (dim_T 4)
    n, T = 512, 8
    a = stgen.grid7(n, n, n, 4, np.float32)
    ref = oracle_lib.st7(a, 0.4, 0.1, T)
    got, info = run_gpu(a, 0.4, 0.1, T, 4)
    assert info["dim_t_sweep"] == 4
    assert relerr(got, ref) <= TOL[np.float32]
    got, _ = run_gpu(a, 0.4, 0.1, T, 4, exact=True)
    assert np.array_equal(got, ref)


@pytest.mark.parametrize("dtype", [np.float32, np.float64])
@pytest.mark.parametrize("T", [0, 1, 4, 7])
def test_naive_variant_bitexact(oracle_lib, dtype, T):
    # the no-blocking ablation baseline (ST_VARIANT_NAIVE) computes in the oracle's order
    nx, ny, nz = (68, 52, 37) if dtype == np.float32 else (66, 40, 21)
    a = stgen.grid7(nx, ny, nz, 7, dtype)
    ref = oracle_lib.st7(a, 0.4, 0.1, T)
    dt = torch.float32 if dtype == np.float32 else torch.float64
    with st.Plan(nx, ny, nz, dt, 1) as p:
        p.set_variant(st.ST_VARIANT_NAIVE)
        x = torch.from_numpy(a).cuda()
        y = torch.empty_like(x)
        p.st7(x, y, 0.4, 0.1, T)
        p.sync()
        assert p.last_launches() == T
    assert np.array_equal(y.cpu().numpy(), ref)


@pytest.mark.parametrize("dtype", [np.float32, np.float64])
def test_autotune_picks_a_depth_and_stays_exact(oracle_lib, dtype):
    # st_plan_autotune: the eq. (3) seed from the measured Gamma, its neighbours timed,
    # the fastest timed depth kept, and it is a local minimum; results are depth-independent
    nx, ny, nz = 96, 72, 40
    dt = torch.float32 if dtype == np.float32 else torch.float64
    a = stgen.grid7(nx, ny, nz, 11, dtype)
    ref = oracle_lib.st7(a, 0.4, 0.1, 9)
    with st.Plan(nx, ny, nz, dt, 6) as p:
        x = torch.empty(nz, ny, nx, dtype=dt, device="cuda")
        y = torch.empty_like(x)
        d, eta, ms = p.autotune(x, y, 6)
        assert 1 <= d <= 6 and 1 <= eta
        assert 1 in ms and 6 in ms and d in ms            # the two Gamma probes and the choice
        assert ms[d] == min(ms.values())
        for nb in (d - 1, d + 1):                         # a local minimum of the timed depths
            assert not (1 <= nb <= 6) or nb in ms
        assert p.info()["dim_t_sweep"] == d
        rep = p.autotune_report(x, y, 6)
        assert rep["dim_T"] >= 1 and rep["Gamma_eff"] > 0 and rep["eta"] >= 1
        assert rep["gamma"] == pytest.approx(2 * np.dtype(dtype).itemsize / 7)
        assert all(s > 0 for s in rep["tile_side"])
        assert rep["tile_side"][0] < rep["tile_side"][1] < rep["tile_side"][2]
        p.set_bitexact(True)
        x.copy_(torch.from_numpy(a))
        p.st7(x, y, 0.4, 0.1, 9)
        p.sync()
    assert np.array_equal(y.cpu().numpy(), ref)


DEGENERATE = [(4, 3, 3), (4, 3, 17), (4, 200, 5), (300, 3, 3), (8, 5, 64), (1024, 4, 3)]


@pytest.mark.parametrize("shape", DEGENERATE)
@pytest.mark.parametrize("dim_T", [1, 2, 3, 5, 8])
def test_degenerate_shapes_bitexact(oracle_lib, shape, dim_T):
    # one interior point wide / one plane thick / single-row grids and deep sweeps on tiny grids
    nx, ny, nz = shape
    a = stgen.grid7(nx, ny, nz, 17, np.float32)
    T = 2 * dim_T + 1
    ref = oracle_lib.st7(a, 0.4, 0.1, T)
    got, _ = run_gpu(a, 0.4, 0.1, T, dim_T, exact=True)
    assert np.array_equal(got, ref)


@pytest.mark.parametrize("variant", [4256, 2256, 214512, 214256, 1256, 94256, 22256, 2512, 4384])
def test_kernel_variants_parity(oracle_lib, variant):
    # every compiled 7-point kernel variant (ST_OPT_ST7_VARIANT): rows per thread, threads
    # per CTA, CTAs per SM, the narrow FP32 layout (2 points per thread row) and the
    # ablation-ladder kernels -- bit-exact (ladder kernels: tolerance build only) and
    # within 1e-5 on ragged shapes at every depth the variant compiles
    ladder = variant in (1256, 94256)
    for k, (nx, ny, nz) in enumerate([(68, 52, 37), (200, 70, 11), (64, 130, 9)]):
        a = stgen.grid7(nx, ny, nz, 300 + k, np.float32)
        for D in (1, 2, 3, 4):
            T = 2 * D + 1
            ref = oracle_lib.st7(a, 0.4, 0.1, T)
            for exact in ((False,) if ladder else (True, False)):
                with st.Plan(nx, ny, nz, torch.float32, D) as p:
                    p.set_bitexact(exact)
                    p.set_option(st.ST_OPT_ST7_VARIANT, variant)
                    x = torch.from_numpy(a).cuda()
                    y = torch.empty_like(x)
                    p.st7(x, y, 0.4, 0.1, T)
                    p.sync()
                    got = y.cpu().numpy()
                if exact:
                    assert np.array_equal(got, ref), (variant, nx, ny, nz, D)
                else:
                    assert relerr(got, ref) <= TOL[np.float32], (variant, nx, ny, nz, D)
