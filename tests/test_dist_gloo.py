"""Multi-process (world_size 2, gloo, CPU) check of the Z-slab decomposition
host logic of §8(e): slab ranges from the library (st_slab_range, host-only),
dim_T-deep ghost planes exchanged with the neighbour rank before every
sweep, each rank advancing only its slab.  The compute here is the CPU oracle
on the slab buffer (its fixed buffer edges are exactly the ghost-zone
argument of P:216: after d steps only planes >= d away from the buffer edge
are valid), so the test checks the decomposition and exchange schedule the
NCCL transport uses, independently of the GPU."""
import os
import socket

import numpy as np
import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp

import stgen


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _sweep_depths(T, D):
    S = -(-T // D)
    q, rem = divmod(T, S)
    return [q + (1 if s < rem else 0) for s in range(S)]


def _worker(rank, world, port, kind, q):
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        import oracle
        import paper_conf_sc_nguyensckd10_b200 as st
        nx, ny, nz, D, T = 20, 18, 27, 3, 8
        z0, nzl = st.st_slab_range(nz, world, rank)
        g = D
        lo, hi = max(0, z0 - g), min(nz, z0 + nzl + g)     # buffer planes (clipped at the lattice)
        own = slice(z0 - lo, z0 - lo + nzl)
        if kind == "st7":
            full = stgen.grid7(nx, ny, nz, 41, np.float64)
            buf = full[lo:hi].copy()
            comp = lambda b: b[None]                           # noqa: E731
        else:
            flags_full = stgen.cavity_flags(nx, ny, nz)
            full = stgen.lbm_random(nx, ny, nz, 42, np.float64)
            buf = full[:, lo:hi].copy()
            fl = flags_full[lo:hi].copy()
            comp = lambda b: b                                 # noqa: E731
        for d in _sweep_depths(T, D):
            # ghost exchange: my d planes next to each face <-> neighbour's
            c = comp(buf)
            reqs = []
            if rank > 0:
                send_lo = torch.from_numpy(np.ascontiguousarray(c[:, z0 - lo:z0 - lo + d]))
                recv_lo = torch.empty_like(send_lo)
                reqs += [dist.isend(send_lo, rank - 1), dist.irecv(recv_lo, rank - 1)]
            if rank < world - 1:
                e = z0 - lo + nzl
                send_hi = torch.from_numpy(np.ascontiguousarray(c[:, e - d:e]))
                recv_hi = torch.empty_like(send_hi)
                reqs += [dist.isend(send_hi, rank + 1), dist.irecv(recv_hi, rank + 1)]
            for r in reqs:
                r.wait()
            if rank > 0:
                c[:, z0 - lo - d:z0 - lo] = recv_lo.numpy()
            if rank < world - 1:
                e = z0 - lo + nzl
                c[:, e:e + d] = recv_hi.numpy()
            # d steps on the slab buffer; only owned planes are kept valid
            if kind == "st7":
                buf = oracle.st7(buf, 0.4, 0.1, d)
            else:
                buf = oracle.lbm(buf, fl, 1.6, d)
        owned = buf[own] if kind == "st7" else buf[:, own]
        parts = [None] * world
        dist.all_gather_object(parts, (z0, owned))
        if rank == 0:
            if kind == "st7":
                ref = oracle.st7(full, 0.4, 0.1, T)
                got = np.concatenate([p[1] for p in sorted(parts, key=lambda t: t[0])], axis=0)
            else:
                ref = oracle.lbm(full, flags_full, 1.6, T)
                got = np.concatenate([p[1] for p in sorted(parts, key=lambda t: t[0])], axis=1)
            q.put(bool(np.array_equal(got, ref)))
    finally:
        dist.destroy_process_group()


@pytest.mark.parametrize("kind", ["st7", "lbm"])
def test_zslab_world2_gloo(kind):
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(r, 2, port, kind, q)) for r in range(2)]
    for p in procs:
        p.start()
    for p in procs:
        p.join(timeout=300)
    assert all(p.exitcode == 0 for p in procs)
    assert q.get(timeout=5) is True


def test_slab_ranges():
    import paper_conf_sc_nguyensckd10_b200 as st
    for nz, P in ((512, 8), (1024, 8), (27, 2), (100, 7)):
        ranges = [st.st_slab_range(nz, P, r) for r in range(P)]
        assert ranges[0][0] == 0
        assert sum(n for _, n in ranges) == nz
        assert all(ranges[i][0] + ranges[i][1] == ranges[i + 1][0] for i in range(P - 1))
        assert max(n for _, n in ranges) - min(n for _, n in ranges) <= 1
        assert [n for _, n in ranges] == sorted([n for _, n in ranges], reverse=True)
