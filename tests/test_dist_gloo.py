"""Multi-process (world_size 2 and 3, gloo, CPU) check of the Z-slab
decomposition of §8(e) as the library runs it: every rank executes the step
list the library itself builds for st7_run / lbm_d3q19_run
(st_slab_schedule, host-only: ghosts of the input, boundary planes first,
the exchange of the next sweep's ghosts overlapped with the interior sweep,
waits, the final copy), with gloo send/recv as the transport and the CPU
oracle as the per-step compute on the slab buffer (its fixed buffer edges are
the ghost-zone argument of P:216: after d steps only planes >= d away from an
artificial buffer edge are valid).  The gathered result must equal the
single-domain oracle bit for bit, so a wrong plane range, ghost depth,
buffer parity or wait in the library's schedule fails it."""
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
        nzb = nzl + 2 * g
        steps = st.st_slab_schedule(nz, world, rank, D, T, overlap=True)
        # buffer plane L <-> global z0 - g + L; planes outside the grid stay zero (never valid)
        lo, hi = max(0, z0 - g), min(nz, z0 + nzl + g)
        Lmin, Lmax = lo - (z0 - g), hi - (z0 - g)
        if kind == "st7":
            full = stgen.grid7(nx, ny, nz, 41, np.float64)
            bufs = [np.zeros((1, nzb, ny, nx)), np.zeros((1, nzb, ny, nx))]
            bufs[0][0, Lmin:Lmax] = full[lo:hi]
        else:
            flags_full = stgen.cavity_flags(nx, ny, nz)
            full = stgen.lbm_random(nx, ny, nz, 42, np.float64)
            bufs = [np.zeros((19, nzb, ny, nx)), np.zeros((19, nzb, ny, nx))]
            bufs[0][:, Lmin:Lmax] = full[:, lo:hi]
            fl = flags_full[lo:hi].copy()

        def compute(src, depth):   # the oracle on the part of the buffer inside the grid
            if kind == "st7":
                return oracle.st7(np.ascontiguousarray(src[0, Lmin:Lmax]), 0.4, 0.1, depth)[None]
            return oracle.lbm(np.ascontiguousarray(src[:, Lmin:Lmax]), fl, 1.6, depth)

        pending = []

        def start_exchange(b, d):
            c = bufs[b]
            ops = []
            if rank > 0:
                send = torch.from_numpy(np.ascontiguousarray(c[:, g:g + d]))
                recv = torch.empty_like(send)
                ops.append((dist.isend(send, rank - 1), dist.irecv(recv, rank - 1), b, g - d, g, recv))
            if rank < world - 1:
                e = g + nzl
                send = torch.from_numpy(np.ascontiguousarray(c[:, e - d:e]))
                recv = torch.empty_like(send)
                ops.append((dist.isend(send, rank + 1), dist.irecv(recv, rank + 1), b, e, e + d, recv))
            return ops

        def finish(ops):
            for s_, r_, b, z_a, z_b, recv in ops:
                s_.wait()
                r_.wait()
                bufs[b][:, z_a:z_b] = recv.numpy()

        result = None
        for stp in steps:
            if stp["kind"] == st.ST_STEP_EXCHANGE:
                ops = start_exchange(stp["src"], stp["depth"])
                if stp["async"]:
                    pending = ops       # completes at the next WAIT
                else:
                    finish(ops)
            elif stp["kind"] == st.ST_STEP_SWEEP:
                out = compute(bufs[stp["src"]], stp["depth"])
                za, zb = stp["z_begin"], stp["z_end"]
                assert g <= za <= zb <= g + nzl
                bufs[1 - stp["src"]][:, za:zb] = out[:, za - Lmin:zb - Lmin]
                result = 1 - stp["src"]
            elif stp["kind"] == st.ST_STEP_WAIT:
                finish(pending)
                pending = []
            elif stp["kind"] == st.ST_STEP_COPY:
                result = 0
        assert not pending
        owned = bufs[result][:, g:g + nzl]
        parts = [None] * world
        dist.all_gather_object(parts, (z0, owned))
        if rank == 0:
            got = np.concatenate([p[1] for p in sorted(parts, key=lambda t: t[0])], axis=1)
            if kind == "st7":
                ok = np.array_equal(got[0], oracle.st7(full, 0.4, 0.1, T))
            else:
                ok = np.array_equal(got, oracle.lbm(full, flags_full, 1.6, T))
            q.put(bool(ok))
    finally:
        dist.destroy_process_group()


@pytest.mark.parametrize("kind,world", [("st7", 2), ("lbm", 2), ("st7", 3)])
def test_zslab_schedule_gloo(kind, world):
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(r, world, port, kind, q)) for r in range(world)]
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


def test_schedule_structure():
    # host-only properties of the library's schedule: every owned plane is written by
    # exactly one SWEEP step per sweep, the ghost depth of an exchange equals the depth
    # of the sweep that reads it, async exchanges are closed by a WAIT before the next sweep
    import paper_conf_sc_nguyensckd10_b200 as st
    for nz, P, D, T, ov in ((512, 8, 4, 100, True), (27, 2, 3, 8, False), (100, 7, 2, 9, True), (64, 4, 1, 6, True)):
        for r in range(P):
            z0, nzl = st.st_slab_range(nz, P, r)
            steps = st.st_slab_schedule(nz, P, r, D, T, ov)
            cover, open_async, ghost = {}, False, {}
            for s in steps:
                if s["kind"] == st.ST_STEP_EXCHANGE:
                    ghost[s["src"]] = s["depth"]
                    open_async = bool(s["async"])
                elif s["kind"] == st.ST_STEP_SWEEP:
                    assert 1 <= s["depth"] <= D
                    if s["sweep"] not in cover:    # the ghosts this sweep reads are as deep as the sweep
                        assert ghost.get(s["src"]) == s["depth"] or P == 1
                    cover.setdefault(s["sweep"], []).extend(range(s["z_begin"], s["z_end"]))
                elif s["kind"] == st.ST_STEP_WAIT:
                    assert open_async
                    open_async = False
            assert not open_async
            for k, planes in cover.items():
                assert sorted(planes) == list(range(D, D + nzl)), (nz, P, r, k)
            depths = [s["depth"] for s in steps if s["kind"] == st.ST_STEP_SWEEP and s["z_begin"] == D]
            assert sum(depths) == T
