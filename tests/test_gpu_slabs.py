"""Z-slab decomposition on one GPU (loopback transport, st_plan_set_loopback_slabs):
P virtual slabs with dim_T-deep ghost planes exchanged before every sweep
(the NCCL schedule with cudaMemcpyAsync as transport).  The result must be
bit-identical to the single-slab run (SURVEY §8(e) invariant) and, in the
bit-exact build, to the oracle."""
import numpy as np
import pytest
import torch

import stgen
import paper_conf_sc_nguyensckd10_b200 as st

pytestmark = pytest.mark.gpu


def st7_gpu(a, T, dim_T, slabs=1, exact=False):
    nz, ny, nx = a.shape
    with st.Plan(nx, ny, nz, torch.float32 if a.dtype == np.float32 else torch.float64, dim_T) as p:
        if exact:
            p.set_bitexact(True)
        if slabs > 1:
            st.st_plan_set_loopback_slabs(p.h, slabs)
        x = torch.from_numpy(a).cuda()
        y = torch.empty_like(x)
        p.st7(x, y, 0.4, 0.1, T)
        p.sync()
        return y.cpu().numpy()


@pytest.mark.parametrize("P", [2, 3, 4])
@pytest.mark.parametrize("dim_T", [1, 3, 4])
def test_st7_loopback_identical(oracle_lib, P, dim_T):
    a = stgen.grid7(64, 48, 41, 21, np.float32)
    T = 2 * dim_T + 3
    one = st7_gpu(a, T, dim_T)
    many = st7_gpu(a, T, dim_T, slabs=P)
    assert np.array_equal(one, many)
    ex = st7_gpu(a, T, dim_T, slabs=P, exact=True)
    assert np.array_equal(ex, oracle_lib.st7(a, 0.4, 0.1, T))


def lbm_gpu(f0, flags, T, dim_T, slabs=1, exact=False):
    _, nz, ny, nx = f0.shape
    with st.Plan(nx, ny, nz, torch.float32 if f0.dtype == np.float32 else torch.float64, dim_T) as p:
        if exact:
            p.set_bitexact(True)
        if slabs > 1:
            st.st_plan_set_loopback_slabs(p.h, slabs)
        a = torch.from_numpy(f0).cuda()
        b = torch.empty_like(a)
        p.lbm(a, b, 1.6, T, torch.from_numpy(flags).cuda())
        p.sync()
        return b.cpu().numpy()


@pytest.mark.parametrize("P", [2, 3])
@pytest.mark.parametrize("dim_T", [1, 2, 3])
def test_lbm_loopback_identical(oracle_lib, P, dim_T):
    nx, ny, nz = 40, 24, 23
    flags = stgen.cavity_flags(nx, ny, nz)
    flags[10:13, 8:12, 15:20] = stgen.WALL   # obstacle across a slab boundary
    f0 = stgen.lbm_random(nx, ny, nz, 31, np.float32)
    T = 7
    ref = oracle_lib.lbm(f0, flags, 1.6, T)
    got = lbm_gpu(f0, flags, T, dim_T, slabs=P, exact=True)
    assert np.array_equal(got, ref)
    assert np.array_equal(lbm_gpu(f0, flags, T, dim_T, slabs=P), lbm_gpu(f0, flags, T, max(dim_T, 2), slabs=1)) \
        or dim_T == 1


def test_slab_too_thin():
    with st.Plan(64, 64, 16, torch.float32, 4) as p:
        with pytest.raises(st.StError):
            st.st_plan_set_loopback_slabs(p.h, 8)   # 2-plane slabs < dim_T


@pytest.mark.parametrize("kind", ["st7", "lbm"])
@pytest.mark.parametrize("overlap", [1, 0])
def test_nccl_one_rank_communicator(oracle_lib, kind, overlap):
    # the NCCL transport path on one GPU: st_plan_set_dist with an id and one rank builds a
    # communicator (ncclCommInitRankConfig, maxCTAs) and runs the distributed schedule --
    # slab buffers with dim_T ghost planes per side, boundary sweeps, the grouped
    # send/recv (no peers) on the side stream, the interior sweep, the wait, the async
    # error poll -- and must still equal the oracle bit for bit
    dim_T, T = 3, 8
    uid = st.st_nccl_unique_id()
    if kind == "st7":
        nx, ny, nz = 64, 40, 30
        a = stgen.grid7(nx, ny, nz, 33, np.float32)
        with st.Plan(nx, ny, nz, torch.float32, dim_T) as p:
            p.set_bitexact(True)
            p.set_option(st.ST_OPT_OVERLAP, overlap)
            p.set_dist(uid, 0, 1)
            g = st.st_plan_ghost_planes(p.h)
            assert st.st_plan_local_slab(p.h) == (0, nz)
            buf = np.zeros((nz + 2 * g, ny, nx), np.float32)
            buf[g:g + nz] = a
            x = torch.from_numpy(buf).cuda()
            y = torch.zeros_like(x)
            p.st7(x, y, 0.4, 0.1, T)
            p.sync()
            got = y.cpu().numpy()[g:g + nz]
        assert np.array_equal(got, oracle_lib.st7(a, 0.4, 0.1, T))
    else:
        nx, ny, nz = 32, 24, 20
        flags = stgen.cavity_flags(nx, ny, nz)
        f0 = stgen.lbm_random(nx, ny, nz, 34, np.float32)
        with st.Plan(nx, ny, nz, torch.float32, 1) as p:
            p.set_bitexact(True)
            p.set_option(st.ST_OPT_OVERLAP, overlap)
            p.set_dist(uid, 0, 1)
            g = st.st_plan_ghost_planes(p.h)
            buf = np.zeros((19, nz + 2 * g, ny, nx), np.float32)
            buf[:, g:g + nz] = f0
            fl = np.full((nz + 2 * g, ny, nx), stgen.WALL, np.uint8)
            fl[g:g + nz] = flags
            x = torch.from_numpy(buf).cuda()
            y = torch.zeros_like(x)
            p.lbm(x, y, 1.6, T, torch.from_numpy(fl).cuda())
            p.sync()
            got = y.cpu().numpy()[:, g:g + nz]
        assert np.array_equal(got, oracle_lib.lbm(f0, flags, 1.6, T))


@pytest.mark.parametrize("P", [2, 3, 4])
@pytest.mark.parametrize("T", [4, 7])
def test_lbm_loopback_tma_gather(oracle_lib, P, T):
    # FP32 dim_T = 1 runs of T >= 4 take the TMA gather form on Z slabs too: T + 1
    # passes as depth-1 sweeps of the slab schedule (one ghost plane exchanged per
    # face before each pull / stream pass, boundary planes first, interior overlapped);
    # bit-identical to the oracle in the exact build, within the gate otherwise
    nx, ny, nz = 64, 20, 26
    flags = stgen.cavity_flags(nx, ny, nz)
    flags[12:15, 5:9, 20:30] = stgen.WALL    # obstacle across a slab boundary
    flags[7, 10, 40] = stgen.LID
    f0 = stgen.lbm_random(nx, ny, nz, 41, np.float32)
    ref = oracle_lib.lbm(f0, flags, 1.6, T)
    for exact in (True, False):
        with st.Plan(nx, ny, nz, torch.float32, 1) as p:
            p.set_bitexact(exact)
            st.st_plan_set_loopback_slabs(p.h, P)
            a = torch.from_numpy(f0).cuda()
            b = torch.empty_like(a)
            p.lbm(a, b, 1.6, T, torch.from_numpy(flags).cuda())
            p.sync()
            assert p.info(True)["kernel"] == 400
            got = b.cpu().numpy()
        if exact:
            assert np.array_equal(got, ref), (P, T)
        else:
            g = got.astype(np.float64)
            assert float(np.max(np.abs(g - ref) / np.maximum(np.abs(ref), 1e-30))) <= 1e-4
