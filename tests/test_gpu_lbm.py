"""GPU parity of lbm_d3q19_run (C ABI) against the CPU oracle on the same
seeded cavity lattices: FP32 max rel err <= 1e-4, FP64 <= 1e-12, bit-exact
in the oracle-order build."""
import numpy as np
import pytest
import torch

import stgen
import paper_conf_sc_nguyensckd10_b200 as st

pytestmark = pytest.mark.gpu
TOL = {np.float32: 1e-4, np.float64: 1e-12}


def relerr(g, o):
    g = g.astype(np.float64)
    o = o.astype(np.float64)
    return float(np.max(np.abs(g - o) / np.maximum(np.abs(o), 1e-30)))


def run_gpu(f0, flags, omega, T, dim_T=1, exact=False, lid=(0.05, 0.0, 0.0), batched=-1):
    _, nz, ny, nx = f0.shape
    dt = torch.float32 if f0.dtype == np.float32 else torch.float64
    with st.Plan(nx, ny, nz, dt, dim_T) as p:
        p.set_lid(*lid)
        p.set_option(st.ST_OPT_LBM_BATCHED, batched)
        if exact:
            p.set_bitexact(True)
        a = torch.from_numpy(f0).cuda()
        b = torch.empty_like(a)
        fl = torch.from_numpy(flags).cuda()
        p.lbm(a, b, omega, T, fl)
        p.sync()
        return b.cpu().numpy()


@pytest.mark.parametrize("dtype", [np.float32, np.float64])
@pytest.mark.parametrize("shape", [(32, 24, 20), (64, 40, 9), (16, 16, 16), (96, 50, 13)])
@pytest.mark.parametrize("dim_T", [1, 2, 3])
def test_cavity_random(oracle_lib, dtype, shape, dim_T):
    nx, ny, nz = shape
    flags = stgen.cavity_flags(nx, ny, nz)
    f0 = stgen.lbm_random(nx, ny, nz, 3, dtype)
    T = 7
    ref = oracle_lib.lbm(f0, flags, 1.6, T)
    got = run_gpu(f0, flags, 1.6, T, dim_T=dim_T, exact=True)
    assert np.array_equal(got, ref)
    got = run_gpu(f0, flags, 1.6, T, dim_T=dim_T)
    assert relerr(got, ref) <= TOL[dtype]


def test_obstacle_interior(oracle_lib):
    # an interior WALL block: neighbour-flag slow path away from the shell
    nx, ny, nz = 40, 30, 20
    flags = stgen.cavity_flags(nx, ny, nz)
    flags[8:12, 10:15, 12:20] = stgen.WALL
    flags[5, 20, 30] = stgen.LID
    f0 = stgen.lbm_random(nx, ny, nz, 9, np.float32)
    ref = oracle_lib.lbm(f0, flags, 1.2, 6)
    for d in (1, 2, 3):
        assert np.array_equal(run_gpu(f0, flags, 1.2, 6, dim_T=d, exact=True), ref), d


def test_dimT_invariance_lbm():
    nx, ny, nz = 64, 36, 24
    flags = stgen.cavity_flags(nx, ny, nz)
    f0 = stgen.lbm_random(nx, ny, nz, 5, np.float32)
    outs = [run_gpu(f0, flags, 1.6, 9, dim_T=d, exact=True) for d in (1, 2, 3)]
    assert np.array_equal(outs[0], outs[1]) and np.array_equal(outs[0], outs[2])


def test_T0_and_rest(oracle_lib):
    flags = stgen.cavity_flags(32, 16, 12)
    f0 = stgen.lbm_rest(32, 16, 12, np.float32)
    assert np.array_equal(run_gpu(f0, flags, 1.6, 0), f0)
    ref = oracle_lib.lbm(f0, flags, 1.6, 4, u_lid=(0, 0, 0))
    assert np.array_equal(run_gpu(f0, flags, 1.6, 4, lid=(0, 0, 0), exact=True), ref)
    assert relerr(run_gpu(f0, flags, 1.6, 4, lid=(0, 0, 0)), ref) <= TOL[np.float32]


def test_fluid_shell_rejected():
    flags = stgen.cavity_flags(32, 16, 12)
    flags[0, 5, 5] = stgen.FLUID
    f0 = stgen.lbm_rest(32, 16, 12, np.float32)
    with pytest.raises(st.StError) as ei:
        run_gpu(f0, flags, 1.6, 2)
    assert ei.value.code == st.ST_EUNSUPPORTED


def test_bad_omega():
    flags = stgen.cavity_flags(32, 16, 12)
    f0 = stgen.lbm_rest(32, 16, 12, np.float32)
    with pytest.raises(st.StError):
        run_gpu(f0, flags, 2.0, 2)


@pytest.mark.parametrize("dim_T", [1, 2])
def test_config2_lbm_256_full_lattice(oracle_lib, dim_T):
    # configs[2] size: 256^3 lid-driven cavity, random populations, every cell compared
    n, T = 256, 2
    flags = stgen.cavity_flags(n, n, n)
    f0 = stgen.lbm_random(n, n, n, 3, np.float32)
    ref = oracle_lib.lbm(f0, flags, 1.6, T)
    got = run_gpu(f0, flags, 1.6, T, dim_T=dim_T)
    assert relerr(got, ref) <= TOL[np.float32]
    got = run_gpu(f0, flags, 1.6, T, dim_T=dim_T, exact=True)
    assert np.array_equal(got, ref)


def test_flags_rewritten_in_place(oracle_lib):
    # the same flags buffer with new contents between two calls: the neighbour-flag
    # prepass of the multi-level path must see the new obstacle
    nx, ny, nz = 40, 30, 20
    flags = stgen.cavity_flags(nx, ny, nz)
    f0 = stgen.lbm_random(nx, ny, nz, 11, np.float32)
    flags2 = flags.copy()
    flags2[6:10, 8:14, 10:18] = stgen.WALL
    with st.Plan(nx, ny, nz, torch.float32, 2) as p:
        p.set_bitexact(True)
        fl = torch.from_numpy(flags).cuda()
        a = torch.from_numpy(f0).cuda()
        b = torch.empty_like(a)
        p.lbm(a, b, 1.3, 4, fl)
        p.sync()
        assert np.array_equal(b.cpu().numpy(), oracle_lib.lbm(f0, flags, 1.3, 4))
        fl.copy_(torch.from_numpy(flags2))
        a = torch.from_numpy(f0).cuda()
        p.lbm(a, b, 1.3, 4, fl)
        p.sync()
        assert np.array_equal(b.cpu().numpy(), oracle_lib.lbm(f0, flags2, 1.3, 4))


def _cavity_on_device(n, dtype):
    """configs[4]-size cavity from rest built on the device (a 1024^3 lattice does not fit host-side)."""
    fl = torch.zeros((n, n, n), dtype=torch.uint8, device="cuda")
    fl[:, 0, :] = stgen.WALL
    fl[:, :, 0] = stgen.WALL
    fl[:, :, n - 1] = stgen.WALL
    fl[0] = stgen.WALL
    fl[n - 1] = stgen.WALL
    fl[:, n - 1, :] = stgen.LID
    f = torch.empty((19, n, n, n), dtype=dtype, device="cuda")
    w = stgen.lbm_rest(1, 1, 1, np.float32 if dtype == torch.float32 else np.float64).reshape(19)
    for i in range(19):
        f[i].fill_(float(w[i]))
    torch.cuda.synchronize()   # the plan runs on its own stream
    return f, fl


def test_config4_lbm_1024_light_cone(oracle_lib):
    # configs[4] lattice (1024^3 FP32 cavity, the strong-scaling base) on one GPU, bit-exact
    # build.  After T steps from rest a cell depends only on its radius-T neighbourhood
    # (one lattice link per step), so windows at the lid centre, at lid corners, at a
    # bottom corner and at the centre must equal the same windows of the oracle run on a
    # small cavity with the same local geometry; every shifted window has its light cone
    # inside both lattices.  Fluid mass is conserved (P8b) over the whole lattice.
    n, T = 1024, 3
    torch.cuda.empty_cache()
    need = 2 * 19 * n ** 3 * 4 + 3 * n ** 3 + (4 << 30)
    if torch.cuda.mem_get_info()[0] < need:
        pytest.skip("1024^3 FP32 lattice pair does not fit this device")
    f, fl = _cavity_on_device(n, torch.float32)
    g = torch.empty_like(f)
    w = stgen.lbm_rest(1, 1, 1, np.float32).reshape(19).astype(np.float64)
    mass0 = float(w.sum()) * (n - 2) ** 3
    with st.Plan(n, n, n, torch.float32, 1) as p:
        p.set_lid(0.05, 0.0, 0.0)
        p.set_bitexact(True)
        p.lbm(f, g, 1.6, T, fl)
        p.sync()
    del f
    ns = 2 * T + 8
    ref = oracle_lib.lbm(stgen.lbm_rest(ns, ns, ns, np.float32), stgen.cavity_flags(ns, ns, ns), 1.6, T)
    h, c, cs = T + 3, n // 2, ns // 2
    windows = [   # (big z, y, x slices), (small z, y, x slices)
        ((slice(c - 2, c + 3), slice(n - h, n), slice(c - 2, c + 3)),
         (slice(cs - 2, cs + 3), slice(ns - h, ns), slice(cs - 2, cs + 3))),        # lid centre
        ((slice(0, h), slice(n - h, n), slice(0, h)), (slice(0, h), slice(ns - h, ns), slice(0, h))),   # lid corner
        ((slice(n - h, n), slice(n - h, n), slice(n - h, n)),
         (slice(ns - h, ns), slice(ns - h, ns), slice(ns - h, ns))),                 # far lid corner
        ((slice(0, h), slice(0, h), slice(0, h)), (slice(0, h), slice(0, h), slice(0, h))),   # bottom corner
        ((slice(c - 1, c + 2), slice(c - 1, c + 2), slice(c - 1, c + 2)),
         (slice(cs - 1, cs + 2), slice(cs - 1, cs + 2), slice(cs - 1, cs + 2))),     # centre
    ]
    for big, small in windows:
        got = g[(slice(None),) + big].cpu().numpy()
        assert np.array_equal(got, ref[(slice(None),) + small])
    mass = 0.0
    for i in range(19):
        for z0 in range(1, n - 1, 64):
            mass += float(g[i, z0:min(z0 + 64, n - 1), 1:n - 1, 1:n - 1].double().sum())
    assert abs(mass - mass0) <= 1e-6 * mass0


def test_config4_lbm_1024_random_windows(oracle_lib):
    # configs[4] lattice (1024^3 FP32 cavity) with RANDOM populations through the
    # automatic kernel choice (the TMA gather form with 128 x 2 tiles), bit-exact and
    # tolerance builds.  After T steps a cell depends only on its radius-T
    # neighbourhood, so windows are checked against the oracle run on a crop of the
    # same input: the crop keeps the real lattice faces and closes its cut faces
    # with WALL cells, and only cells farther than T + 1 from a cut face are
    # compared.  Windows: centre, lid centre, a bottom corner, the x = 0 wall, and a
    # seam of the 128-wide x tiles / 2-row y tiles.
    n, T, k = 1024, 5, 3   # T >= 4: the automatic choice is the gather form (T + 1 passes, odd: in-place collide)
    import gc
    gc.collect()
    torch.cuda.empty_cache()   # the previous 1024^3 test's lattices stay cached otherwise
    need = 2 * 19 * n ** 3 * 4 + 3 * n ** 3 + (4 << 30)
    if torch.cuda.mem_get_info()[0] < need:
        pytest.skip("1024^3 FP32 lattice pair does not fit this device")
    f, fl = _cavity_on_device(n, torch.float32)   # f is refilled with random populations below
    g = torch.empty_like(f)
    w = stgen.lbm_rest(1, 1, 1, np.float32).reshape(19)
    centres = [(512, 512, 512), (512, n - 1, 512), (0, 0, 0), (300, 700, 0), (77, 301, 128)]   # (z, y, x)
    m = k + T + 1
    crops = []
    for c in centres:
        lo = [max(0, v - m) for v in c]
        hi = [min(n, v + m + 1) for v in c]
        crops.append((lo, hi))

    def fill():
        gen = torch.Generator(device="cuda")
        gen.manual_seed(1234)
        for i in range(19):
            f[i].uniform_(-1.0, 1.0, generator=gen).mul_(0.1).add_(1.0).mul_(float(w[i]))
        torch.cuda.synchronize()

    for exact in (True, False):
        fill()
        inputs = [f[:, lo[0]:hi[0], lo[1]:hi[1], lo[2]:hi[2]].cpu().numpy() for lo, hi in crops]
        with st.Plan(n, n, n, torch.float32, 1) as p:
            p.set_lid(0.05, 0.0, 0.0)
            p.set_bitexact(exact)
            p.lbm(f, g, 1.6, T, fl)
            p.sync()
            assert p.info(True)["kernel"] == 400
        for (lo, hi), c, f0 in zip(crops, centres, inputs):
            flc = fl[lo[0]:hi[0], lo[1]:hi[1], lo[2]:hi[2]].cpu().numpy().copy()
            # cut faces (inside the lattice) become WALL
            if lo[0] > 0: flc[0] = stgen.WALL
            if hi[0] < n: flc[-1] = stgen.WALL
            if lo[1] > 0: flc[:, 0] = stgen.WALL
            if hi[1] < n: flc[:, -1] = stgen.WALL
            if lo[2] > 0: flc[:, :, 0] = stgen.WALL
            if hi[2] < n: flc[:, :, -1] = stgen.WALL
            ref = oracle_lib.lbm(f0, flc, 1.6, T)
            # compared: cells farther than T + 1 from every cut face
            sl = []
            for d in range(3):
                a = (T + 2) if lo[d] > 0 else 0
                b = (hi[d] - lo[d]) - ((T + 2) if hi[d] < n else 0)
                sl.append(slice(a, b))
            got = g[:, lo[0]:hi[0], lo[1]:hi[1], lo[2]:hi[2]].cpu().numpy()
            gw, rw = got[(slice(None),) + tuple(sl)], ref[(slice(None),) + tuple(sl)]
            assert gw.size > 0
            if exact:
                assert np.array_equal(gw, rw), c
            else:
                assert relerr(gw, rw) <= TOL[np.float32], c


@pytest.mark.parametrize("shape", [(4, 3, 3), (4, 3, 5), (8, 7, 3), (40, 3, 9)])
@pytest.mark.parametrize("dim_T", [1, 2])
def test_degenerate_lattices(oracle_lib, shape, dim_T):
    # two FLUID cells, one-cell-thick fluid layers (nx is a multiple of 4: TMA row pitch)
    nx, ny, nz = shape
    flags = stgen.cavity_flags(nx, ny, nz)
    f0 = stgen.lbm_random(nx, ny, nz, 5, np.float32)
    ref = oracle_lib.lbm(f0, flags, 1.6, 4)
    got = run_gpu(f0, flags, 1.6, 4, dim_T=dim_T, exact=True)
    assert np.array_equal(got, ref)


@pytest.mark.parametrize("batched", [0, 1])
@pytest.mark.parametrize("shape", [(32, 24, 20), (96, 50, 13)])
def test_push_kernels_random(oracle_lib, shape, batched):
    # both FP32 dim_T = 1 push kernels (per-direction flags / batched flags) on random
    # populations: the batched one serves every FP32 lattice above 2^24 cells (bench's
    # 1024^3 line), the per-direction one the smaller lattices
    nx, ny, nz = shape
    flags = stgen.cavity_flags(nx, ny, nz)
    flags[nz // 2, ny // 3: ny // 3 + 3, nx // 4: nx // 4 + 5] = stgen.WALL   # interior obstacle
    f0 = stgen.lbm_random(nx, ny, nz, 17, np.float32)
    ref = oracle_lib.lbm(f0, flags, 1.6, 5)
    assert np.array_equal(run_gpu(f0, flags, 1.6, 5, exact=True, batched=batched), ref)
    assert relerr(run_gpu(f0, flags, 1.6, 5, batched=batched), ref) <= TOL[np.float32]


def test_batched_kernel_above_2_24_cells(oracle_lib):
    # just above the 2^24-cell switch (260 x 256 x 256 = 17.0 M cells): the automatic
    # choice is the batched-flag kernel; random populations, whole lattice compared in
    # the bit-exact and the tolerance build
    nx, ny, nz, T = 260, 256, 256, 2
    assert nx * ny * nz > 1 << 24
    flags = stgen.cavity_flags(nx, ny, nz)
    f0 = stgen.lbm_random(nx, ny, nz, 23, np.float32)
    ref = oracle_lib.lbm(f0, flags, 1.6, T)
    assert np.array_equal(run_gpu(f0, flags, 1.6, T, exact=True), ref)
    assert relerr(run_gpu(f0, flags, 1.6, T), ref) <= TOL[np.float32]


@pytest.mark.parametrize("dtype", [np.float32, np.float64])
@pytest.mark.parametrize("T", [1, 2, 5])
def test_gather_form_kernels(oracle_lib, dtype, T):
    # ST_OPT_LBM_KERNEL 3: collide pass, T-1 pull (gather) passes, stream pass with
    # aligned stores -- the same operations per (cell, population) as the push step,
    # so bit-identical to the oracle, interior obstacle included
    nx, ny, nz = 96, 50, 13
    flags = stgen.cavity_flags(nx, ny, nz)
    flags[nz // 2, 5:8, 7:12] = stgen.WALL
    f0 = stgen.lbm_random(nx, ny, nz, 3, dtype)
    ref = oracle_lib.lbm(f0, flags, 1.6, T)
    for exact in (True, False):
        with st.Plan(nx, ny, nz, torch.float32 if dtype == np.float32 else torch.float64, 1) as p:
            p.set_bitexact(exact)
            p.set_option(st.ST_OPT_LBM_KERNEL, 3)
            a = torch.from_numpy(f0).cuda()
            b = torch.empty_like(a)
            p.lbm(a, b, 1.6, T, torch.from_numpy(flags).cuda())
            p.sync()
            got = b.cpu().numpy()
        if exact:
            assert np.array_equal(got, ref)
        else:
            assert relerr(got, ref) <= TOL[dtype]


@pytest.mark.parametrize("dtype", [np.float32, np.float64])
@pytest.mark.parametrize("shape", [(96, 50, 13), (64, 4, 5), (36, 9, 7), (128, 33, 10), (520, 5, 6)])
@pytest.mark.parametrize("T", [1, 2, 5])
def test_gather_form_tma_pulls(oracle_lib, dtype, shape, T):
    # ST_OPT_LBM_KERNEL 4: the gather form with the pull passes fed by TMA (shifted
    # 4D boxes per population, shared-memory ring): bit-identical to the oracle in the
    # exact build, within the gate otherwise; ragged tiles in x and y (36 x 9, 128 x 33),
    # a single tile row (64 x 4), the 128-wide FP32 tiles of rows >= 512 cells (520 x 5),
    # interior obstacle and LID cell, ring depths 1..5
    nx, ny, nz = shape
    flags = stgen.cavity_flags(nx, ny, nz)
    flags[nz // 2, 2:4, 3:6] = stgen.WALL
    flags[nz // 3, ny // 2, nx // 2] = stgen.LID
    f0 = stgen.lbm_random(nx, ny, nz, 29, dtype)
    ref = oracle_lib.lbm(f0, flags, 1.6, T)
    for exact, stages in ((True, 0), (False, 0), (True, 1), (True, 3), (False, 5)):
        with st.Plan(nx, ny, nz, torch.float32 if dtype == np.float32 else torch.float64, 1) as p:
            p.set_bitexact(exact)
            p.set_option(st.ST_OPT_LBM_KERNEL, 4)
            if stages and (dtype == np.float32 or stages <= 4):
                p.set_option(st.ST_OPT_LBM_STAGES, stages)
            a = torch.from_numpy(f0).cuda()
            b = torch.empty_like(a)
            p.lbm(a, b, 1.6, T, torch.from_numpy(flags).cuda())
            p.sync()
            got = b.cpu().numpy()
        if exact:
            assert np.array_equal(got, ref), (exact, stages)
        else:
            assert relerr(got, ref) <= TOL[dtype]


@pytest.mark.parametrize("dtype", [np.float32, np.float64])
def test_gather_form_tma_pulls_256(oracle_lib, dtype):
    # configs[2] size (256^3 cavity), random populations, T = 3, whole lattice
    nx = ny = nz = 256
    flags = stgen.cavity_flags(nx, ny, nz)
    f0 = stgen.lbm_random(nx, ny, nz, 31, dtype)
    ref = oracle_lib.lbm(f0, flags, 1.6, 3)
    for exact in (True, False):
        with st.Plan(nx, ny, nz, torch.float32 if dtype == np.float32 else torch.float64, 1) as p:
            p.set_bitexact(exact)
            p.set_option(st.ST_OPT_LBM_KERNEL, 4)
            a = torch.from_numpy(f0).cuda()
            b = torch.empty_like(a)
            p.lbm(a, b, 1.6, 3, torch.from_numpy(flags).cuda())
            p.sync()
            got = b.cpu().numpy()
        if exact:
            assert np.array_equal(got, ref)
        else:
            assert relerr(got, ref) <= TOL[dtype]


@pytest.mark.parametrize("dtype", [np.float32, np.float64])
def test_host_pointers(oracle_lib, dtype):
    # host (numpy) lattices and flags: staged through plan-owned device buffers, the call
    # synchronises; T = 5 takes the TMA gather form for FP32 and the push kernel for FP64
    nx, ny, nz = 64, 20, 11
    flags = stgen.cavity_flags(nx, ny, nz)
    flags[5, 8:10, 20:23] = stgen.WALL
    f0 = stgen.lbm_random(nx, ny, nz, 37, dtype)
    ref = oracle_lib.lbm(f0, flags, 1.6, 5)
    for exact in (True, False):
        with st.Plan(nx, ny, nz, torch.float32 if dtype == np.float32 else torch.float64, 1) as p:
            p.set_bitexact(exact)
            out = np.empty_like(f0)
            p.lbm(f0.copy(), out, 1.6, 5, flags.copy())
            assert p.info(True)["kernel"] == (400 if dtype == np.float32 else 100)
        if exact:
            assert np.array_equal(out, ref)
        else:
            assert relerr(out, ref) <= TOL[dtype]


@pytest.mark.parametrize("kernel", [1, 4])
@pytest.mark.parametrize("dtype", [np.float32, np.float64])
def test_porous_random_obstacles(oracle_lib, kernel, dtype):
    # a porous medium: ~12 % random WALL cells and ~3 % random LID cells inside the
    # cavity, so most FLUID cells take the bounce-back path in some direction (push
    # kernel and TMA gather form), bit-exact and within the gate
    nx, ny, nz = 64, 28, 19
    flags = stgen.cavity_flags(nx, ny, nz)
    rng = np.random.default_rng(7)
    u = rng.random((nz, ny, nx))
    inner = flags == 0
    flags[inner & (u < 0.12)] = stgen.WALL
    flags[inner & (u >= 0.12) & (u < 0.15)] = stgen.LID
    f0 = stgen.lbm_random(nx, ny, nz, 43, dtype)
    T = 6
    ref = oracle_lib.lbm(f0, flags, 1.6, T)
    for exact in (True, False):
        with st.Plan(nx, ny, nz, torch.float32 if dtype == np.float32 else torch.float64, 1) as p:
            p.set_bitexact(exact)
            p.set_option(st.ST_OPT_LBM_KERNEL, kernel)
            a = torch.from_numpy(f0).cuda()
            b = torch.empty_like(a)
            p.lbm(a, b, 1.6, T, torch.from_numpy(flags).cuda())
            p.sync()
            got = b.cpu().numpy()
        if exact:
            assert np.array_equal(got, ref), (kernel, exact)
        else:
            assert relerr(got, ref) <= TOL[dtype], (kernel, exact)
