#!/usr/bin/env python
"""bench.py — throughput of the 3.5D-blocked sweeps on B200 (BASELINE.json metric).

Headline (N=1): BASELINE configs[1], 7-point stencil FP32 256^3, T=100, with
dim_T chosen by measurement (one pass of every dim_T in 1..8, the fastest is
timed).  One step = one st7_run call (T=100 Jacobi steps, all §8(a) rows of
the 7-point path: planner, prolog, TMA plane loads, on-chip levels, final
store, sweep driver).  value = interior updates per second over all ranks
(Mupdates/s; X3: an update is one interior point advanced one time step).

Extra lines inside the same JSON object: FP64 256^3, FP32 512^3 (configs[3]
per-GPU size), the 27-point stencil FP32/FP64 256^3 at every depth (SURVEY
f1), the ablation ladder and the D3Q19 cavity 256^3 / 1024^3 (configs[2],
configs[4] lattice, MLUPS).

Timing: W warm-up steps, then K steps each bracketed by CUDA events on the
plan's stream; L2 (126 MB) is flushed by writing a 512 MiB buffer between
timed steps (outside the timed region); max over ranks.  e2e repeats the
headline through the C ABI with HOST (pinned) buffers, copies inside the
timed region.  `--impl reference` times the CPU oracle on the host cores.
"""
from __future__ import annotations

import argparse
import json
import os
import sys
import threading
import time

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

import numpy as np  # noqa: E402

PEAKS_PATH = os.path.join(ROOT, "MEASURED_PEAKS.json")
TRAFFIC_PATH = os.path.join(ROOT, "profiles", "traffic.json")
SM_COUNT = 148
FP32_LANES, FP64_LANES = 128, 64
ST7_OPS = 7            # FP instructions per 7-point update: 5 add, 1 mul, 1 fma (8 flops)
ST27_OPS = 13          # FP lane instructions per 27-point update of the tolerance kernel st27t (FMA = 1)
ST13_OPS = 13          # FP lane-ops per radius-2 update (X25 with FMA): 9 add, 1 mul, 3 fma
# measured FP32 throughput of the 7-point instruction mix (4 FADD2, FMUL2, 2 FFMA2 with a
# scalar coefficient, distinct register pairs): tools/microbench.cu "mix7 scalar", 512
# threads x 2 CTAs per SM, profiles/r02/microbench.txt -- above the 128-lane nominal
MIX7_LANE_OPS_PER_CLK_SM = 167.7
LBM_BYTES = {4: 153, 8: 305}   # (19*2*E + 1) per LBM update at dim_T = 1 (X12)


def parse():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=10)
    ap.add_argument("--warmup", type=int, default=3)
    ap.add_argument("--impl", default="ours", choices=["ours", "reference"])
    ap.add_argument("--n", type=int, default=256)
    ap.add_argument("--T", type=int, default=100)
    ap.add_argument("--dim-t", type=int, default=0, help="0 = choose by measurement")
    ap.add_argument("--no-extras", action="store_true")
    return ap.parse_args()


def peaks():
    try:
        with open(PEAKS_PATH) as fh:
            d = json.load(fh)
        return float(d["hbm_gbs"]), float(d.get("sm_max_mhz", 1965.0)), "measured"
    except Exception:
        return 6650.0, 1965.0, "fallback"


class ClockSampler:
    """nvidia-smi style clock / throttle sampling during the timed region (pynvml)."""

    def __init__(self, dev: int):
        self.dev = dev
        self.samples = []
        self.reasons = set()
        self.max_mhz = None
        self._stop = threading.Event()
        self._t = None

    def __enter__(self):
        try:
            import pynvml
            pynvml.nvmlInit()
            h = pynvml.nvmlDeviceGetHandleByIndex(self.dev)
            self.max_mhz = pynvml.nvmlDeviceGetMaxClockInfo(h, pynvml.NVML_CLOCK_SM)
            names = {
                "hw_slowdown": getattr(pynvml, "nvmlClocksThrottleReasonHwSlowdown", 0x8),
                "hw_thermal_slowdown": getattr(pynvml, "nvmlClocksThrottleReasonHwThermalSlowdown", 0x40),
                "sw_thermal_slowdown": getattr(pynvml, "nvmlClocksThrottleReasonSwThermalSlowdown", 0x20),
                "sw_power_cap": getattr(pynvml, "nvmlClocksThrottleReasonSwPowerCap", 0x4),
            }

            def run():
                while not self._stop.is_set():
                    try:
                        self.samples.append(pynvml.nvmlDeviceGetClockInfo(h, pynvml.NVML_CLOCK_SM))
                        r = pynvml.nvmlDeviceGetCurrentClocksThrottleReasons(h)
                        for k, bit in names.items():
                            if r & bit:
                                self.reasons.add(k)
                    except Exception:
                        pass
                    time.sleep(0.05)

            self._t = threading.Thread(target=run, daemon=True)
            self._t.start()
        except Exception:
            self._t = None
        return self

    def __exit__(self, *a):
        self._stop.set()
        if self._t:
            self._t.join()

    def summary(self):
        s = sorted(self.samples)
        return {"sm_mhz": s[len(s) // 2] if s else None, "sm_max_mhz": self.max_mhz,
                "reasons": sorted(self.reasons), "samples": len(s)}


def n_sweeps(T, D):
    """sweeps of a T-step run at depth D: ceil(T/D), made odd (the library's sweep_depths)"""
    S = (T + D - 1) // D
    if S % 2 == 0 and S < T:
        S += 1
    return S


def load_traffic(key):
    """dram__bytes_read.sum + dram__bytes_write.sum per launch of that kernel (ncu, profiles/)"""
    try:
        with open(TRAFFIC_PATH) as fh:
            v = json.load(fh).get(key)
        return v.get("per_launch_bytes") if isinstance(v, dict) else v
    except Exception:
        return None


# ----------------------------------------------------------------------------
# reference arm: the CPU oracle as it stands, on the host cores
# ----------------------------------------------------------------------------
def run_reference(args, rank, world):
    if rank != 0:
        return
    import oracle
    import stgen
    n = args.n
    a = stgen.grid7(n, n, n, 2, np.float32)
    # one step = the configs[1] run (T sweeps) when the host finishes the whole
    # --steps/--warmup run in ~2.5 min at that size; else a bounded sample of Ts sweeps
    t0 = time.perf_counter()
    oracle.st7(a, 0.4, 0.1, 4)
    per_sweep = (time.perf_counter() - t0) / 4
    Ts = int(max(1, min(args.T, 150.0 / (args.steps + args.warmup) / max(per_sweep, 1e-6))))
    for _ in range(args.warmup):
        oracle.st7(a, 0.4, 0.1, Ts)
    t0 = time.perf_counter()
    for _ in range(args.steps):
        oracle.st7(a, 0.4, 0.1, Ts)
    dt = time.perf_counter() - t0
    upd = (n - 2) ** 3 * Ts * args.steps
    v = upd / dt / 1e6
    cores = oracle.num_threads()
    line = {
        "impl": "reference", "metric": "Mupdates/s (7-pt)", "value": round(v, 2), "unit": "Mupdates/s",
        "n_gpus": args.gpus, "steps": args.steps, "warmup": args.warmup,
        "ms_per_step": round(dt / args.steps * 1e3, 3), "higher_is_better": True, "scaling": "weak",
        "vs_baseline": None, "dtype": "f32", "data": "synthetic (splitmix64 U[0,1), seed 2)",
        "config": {"workload": f"7-point FP32 {n}^3 (configs[1]); each step {Ts} of the T={args.T} sweeps",
                   "grid": [n, n, n], "T_sample": Ts},
        "cpu_baseline": {"value": round(v, 2), "unit": "Mupdates/s", "cores": cores, "kind": "oracle",
                         "sample": f"{n}^3 FP32, {Ts} Jacobi sweeps per step, {args.steps} steps"},
        "e2e": {"value": round(v, 2), "unit": "Mupdates/s", "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0},
    }
    print(json.dumps(line), flush=True)


def cpu_baseline_7pt(n, T):
    """the oracle timed on a bounded sample (~12 s) of the headline workload: whole
    configs[1] runs (T sweeps of the n^3 grid), as many as fit."""
    import oracle
    import stgen
    a = stgen.grid7(n, n, n, 2, np.float32)
    t0 = time.perf_counter()
    oracle.st7(a, 0.4, 0.1, T)
    t1 = time.perf_counter() - t0
    reps = int(max(1, min(200, round(12.0 / max(t1, 1e-3)))))
    t0 = time.perf_counter()
    for _ in range(reps):
        oracle.st7(a, 0.4, 0.1, T)
    dt = time.perf_counter() - t0
    return {"value": round((n - 2) ** 3 * T * reps / dt / 1e6, 2), "unit": "Mupdates/s",
            "cores": oracle.num_threads(), "kind": "oracle",
            "sample": f"7-point FP32 {n}^3, {reps} runs of T={T} ({dt:.1f} s), OpenMP over z"}


# ----------------------------------------------------------------------------
# our arm
# ----------------------------------------------------------------------------
def main():
    args = parse()
    world = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    if args.impl == "reference":
        run_reference(args, rank, world)
        return

    import torch
    import torch.distributed as dist
    import stgen
    import paper_conf_sc_nguyensckd10_b200 as st

    torch.cuda.set_device(local)
    if world > 1:
        dist.init_process_group("nccl", device_id=torch.device("cuda", local))

    def barrier():
        if world > 1:
            dist.barrier()

    def max_over_ranks(x):
        if world == 1:
            return x
        t = torch.tensor([x], dtype=torch.float64, device="cuda")
        dist.all_reduce(t, op=dist.ReduceOp.MAX)
        return float(t.item())

    hbm_gbs, sm_max, peak_src = peaks()
    stream = torch.cuda.Stream()
    flush = torch.empty(512 * 2 ** 20 // 4, dtype=torch.float32, device="cuda")

    def l2_flush():
        flush.fill_(1.0)

    def time_steps(run, steps, warmup):
        """returns (total device ms, per-step ms list); events on `stream`."""
        for _ in range(warmup):
            run()
        torch.cuda.synchronize()
        tot = 0.0
        per = []
        for _ in range(steps):
            l2_flush()
            torch.cuda.synchronize()
            barrier()
            e0 = torch.cuda.Event(enable_timing=True)
            e1 = torch.cuda.Event(enable_timing=True)
            e0.record(stream)
            run()
            e1.record(stream)
            e1.synchronize()
            ms = e0.elapsed_time(e1)
            per.append(ms)
            tot += ms
        torch.cuda.synchronize()
        return tot, per

    # ------------------------------------------------------------------ 7-point
    def choose_dim_t(n, T, dtype, choose=range(1, 9)):
        """dim_T by measurement: one timed pass of every dim_T on a local n^3 grid."""
        tdt = torch.float32 if dtype == np.float32 else torch.float64
        x = torch.from_numpy(stgen.grid7(n, n, n, 2, dtype)).cuda()
        y = torch.empty_like(x)
        sweep = {}
        for d in choose:
            with st.Plan(n, n, n, tdt, d) as p:
                p.set_stream(stream)
                p.st7(x, y, 0.4, 0.1, T)
                torch.cuda.synchronize()
                tms, _ = time_steps(lambda: p.st7(x, y, 0.4, 0.1, T), 2, 0)
                sweep[d] = round((n - 2) ** 3 * T / (tms / 2 / 1e3) / 1e6, 1)
        best = max(sweep, key=sweep.get)
        if world > 1:   # every rank runs rank 0's choice
            obj = [best]
            dist.broadcast_object_list(obj, src=0)
            best = obj[0]
        return best, sweep

    uid = None
    if world > 1:
        obj = [st.st_nccl_unique_id() if rank == 0 else None]
        dist.broadcast_object_list(obj, src=0)
        uid = obj[0]

    def st7_case(n, T, dtype, D, steps=args.steps, warmup=args.warmup):
        """weak scaling: each rank owns an n^3 Z-slab of an n x n x (n*world) grid."""
        tdt = torch.float32 if dtype == np.float32 else torch.float64
        nzg = n * world
        p = st.Plan(n, n, nzg, tdt, D)
        p.set_stream(stream)
        if world > 1:
            p.set_dist(uid, rank, world)
            z0, nzl = st.st_plan_local_slab(p.h)
            g = st.st_plan_ghost_planes(p.h)
        else:
            z0, nzl, g = 0, nzg, 0
        nzb = nzl + 2 * g
        host = np.zeros((nzb, n, n), dtype=dtype)
        zlo, zhi = max(0, z0 - g), min(nzg, z0 + nzl + g)
        host[zlo - (z0 - g):zhi - (z0 - g)] = stgen.grid7(n, n, nzg, 2, dtype, z0=zlo, nzl=zhi - zlo)
        a0 = torch.from_numpy(host).cuda()
        x = a0.clone()
        y = torch.empty_like(a0)
        tms, per = time_steps(lambda: p.st7(x, y, 0.4, 0.1, T), steps, warmup)
        launches = p.last_launches()
        info = p.info()
        ms = max_over_ranks(tms / steps)
        upd = (n - 2) ** 2 * (nzg - 2) * T          # interior updates of the whole job
        return p, ms, upd, launches, info, host

    with ClockSampler(local) as clk:
        n, T = args.n, args.T
        if args.dim_t:
            D, sweep = args.dim_t, {}
        else:
            D, sweep = choose_dim_t(n, T, np.float32)
        p7, ms, upd, launches, info, host0 = st7_case(n, T, np.float32, D)
        value = upd / (ms / 1e3) / 1e6
        per_launch_ms = ms / launches
        d_eff = info["dim_t_sweep"]
        upd_rank = upd / world
        # roofline of the dominant kernel (st7_35d, the only kernel of the step): both roofs,
        # the binding one first.  Algorithmic bytes: every sweep reads and writes the grid
        # once (2 E n^3 per sweep); the sweep count (incl. the remainder sweeps that
        # make it odd) comes from the run itself (launches per step).
        ops_peak = SM_COUNT * FP32_LANES * sm_max * 1e6 / 1e12          # T FP32 lane-ops/s (nominal lanes)
        ops_peak_mix = SM_COUNT * MIX7_LANE_OPS_PER_CLK_SM * sm_max * 1e6 / 1e12
        achieved_ops = ST7_OPS * upd_rank / (ms / 1e3) / 1e12
        sweeps = n_sweeps(T, d_eff)
        bytes_step = 2 * 4 * n * n * n * sweeps                  # per rank (its n^3 slab)
        bytes_per_upd = bytes_step / upd_rank
        achieved_gbs = bytes_step / (ms / 1e3) / 1e9
        hbm_roof_upd = hbm_gbs * 1e9 / bytes_per_upd
        alu_roof_upd = ops_peak * 1e12 / ST7_OPS
        traffic = load_traffic(f"st7_f32_{n}_D{D}")
        r_alu = {"bound": "alu", "achieved": round(achieved_ops, 3), "peak": round(ops_peak, 2),
                 "unit": "Top/s (FP32 lane-ops; 7 per update)",
                 "frac": round(achieved_ops / ops_peak, 4), "traffic": traffic,
                 "frac_of_measured_mix": round(achieved_ops / ops_peak_mix, 4),
                 "peak_source": f"148 SM x 128 FP32 lanes x {sm_max:.0f} MHz (clocks.max.sm); "
                                f"frac_of_measured_mix uses the microbenchmarked 7-point mix, "
                                f"{MIX7_LANE_OPS_PER_CLK_SM} lane-ops/clk/SM"}
        r_hbm = {"bound": "hbm", "achieved": round(achieved_gbs, 1), "peak": hbm_gbs, "unit": "GB/s",
                 "frac": round(achieved_gbs / hbm_gbs, 4), "traffic": traffic,
                 "bytes_per_update": round(bytes_per_upd, 4),
                 "peak_source": f"MEASURED_PEAKS.json hbm_gbs ({peak_src}); algorithmic 2E n^3 per sweep, "
                                f"{sweeps} sweeps per step"}
        roof, alt = (r_hbm, r_alu) if hbm_roof_upd < alu_roof_upd else (r_alu, r_hbm)
        roof = dict(roof, frac_hbm=r_hbm["frac"], frac_fp=r_alu["frac"])

    # ------------------------------------------------------------------ e2e (host buffers)
    a_host = torch.from_numpy(host0).pin_memory()
    o_host = torch.empty_like(a_host).pin_memory()
    hin, hout = a_host.numpy(), o_host.numpy()
    for _ in range(max(1, args.warmup)):
        st.st7_run(p7.h, hin, hout, 0.4, 0.1, T)
    e2e_t = 0.0
    for _ in range(args.steps):
        barrier()
        t0 = time.perf_counter()
        st.st7_run(p7.h, hin, hout, 0.4, 0.1, T)
        e2e_t += time.perf_counter() - t0
    e2e_ms = max_over_ranks(e2e_t / args.steps * 1e3)
    grid_bytes = host0.nbytes

    extras = {}
    if not args.no_extras and world == 1:
        # FP64 256^3 (configs[1] FP64)
        D64, sw64 = choose_dim_t(n, T, np.float64)
        _, ms64, upd64, l64, inf64, _ = st7_case(n, T, np.float64, D64, steps=3, warmup=1)
        extras["st7_f64_256"] = {"value": round(upd64 / (ms64 / 1e3) / 1e6, 1), "unit": "Mupdates/s",
                                 "dim_T": D64, "dim_T_sweep": sw64, "ms_per_step": round(ms64, 3),
                                 "frac_alu": round(ST7_OPS * upd64 / (ms64 / 1e3) /
                                                   (SM_COUNT * FP64_LANES * sm_max * 1e6), 4)}
        # FP32 512^3 (configs[3] per-GPU size)
        D5, sw5 = choose_dim_t(512, T, np.float32)
        _, ms5, upd5, l5, inf5, _ = st7_case(512, T, np.float32, D5, steps=3, warmup=1)
        extras["st7_f32_512"] = {"value": round(upd5 / (ms5 / 1e3) / 1e6, 1), "unit": "Mupdates/s",
                                 "dim_T": D5, "dim_T_sweep": sw5, "ms_per_step": round(ms5, 3),
                                 "frac_alu": round(ST7_OPS * upd5 / (ms5 / 1e3) / (ops_peak * 1e12), 4),
                                 "info": inf5}
        # 27-point stencil on the configs[1] grid, T = 100, every depth
        for dtn, dt_np, tdt, dmax, lanes in (("f32", np.float32, torch.float32, 4, 128),
                                             ("f64", np.float64, torch.float64, 4, FP64_LANES)):
            x27 = torch.from_numpy(stgen.grid7(n, n, n, 2, dt_np)).cuda()
            y27 = torch.empty_like(x27)
            sw27, l27 = {}, 0
            for d in range(1, dmax + 1):
                with st.Plan(n, n, n, tdt, d) as p27:
                    p27.set_stream(stream)
                    t27, _ = time_steps(lambda: p27.st27(x27, y27, 0.3, 0.05, 0.02, 0.01, T), 2, 1)
                    sw27[d] = round((n - 2) ** 3 * T / (t27 / 2 / 1e3) / 1e6, 1)
                    l27 = max(l27, p27.last_launches())
            d27 = max(sw27, key=sw27.get)
            v27 = sw27[d27] * 1e6
            E27 = 4 if dtn == "f32" else 8
            extras[f"st27_{dtn}_256"] = {
                "value": sw27[d27], "unit": "Mupdates/s", "dim_T": d27, "dim_T_sweep": sw27,
                "roofline_hbm": {"achieved": round(2 * E27 / d27 * v27 / 1e9, 1), "peak": hbm_gbs, "unit": "GB/s",
                                 "frac": round(2 * E27 / d27 * v27 / 1e9 / hbm_gbs, 4)},
                "frac_alu": round(ST27_OPS * v27 / (SM_COUNT * lanes * sm_max * 1e6), 4),
                "note": f"{ST27_OPS} FP lane instructions per update in the tolerance kernel (st27t: "
                        "4 in-plane adds, 2 adds + 1 mul + 6 FMA for the running partial and the completion); "
                        "the paper's definition counts 30 flops (4 mul + 26 add, P:119)"}
            del x27, y27
        # radius-2 13-point star on the configs[1] grid, T = 100, every depth
        for dtn, dt_np, tdt, dmax, lanes in (("f32", np.float32, torch.float32, 4, 128),
                                             ("f64", np.float64, torch.float64, 3, FP64_LANES)):
            x13 = torch.from_numpy(stgen.grid7(n, n, n, 2, dt_np)).cuda()
            y13 = torch.empty_like(x13)
            sw13 = {}
            w13 = (1 - 7.5 * 0.05, 4 * 0.05 / 3, -0.05 / 12)
            for d in range(1, dmax + 1):
                with st.Plan(n, n, n, tdt, d) as p13:
                    p13.set_stream(stream)
                    t13, _ = time_steps(lambda: p13.st13(x13, y13, *w13, T), 2, 1)
                    sw13[d] = round((n - 4) ** 3 * T / (t13 / 2 / 1e3) / 1e6, 1)
            d13 = max(sw13, key=sw13.get)
            v13 = sw13[d13] * 1e6
            E13 = 4 if dtn == "f32" else 8
            b13 = 2 * E13 * n ** 3 * n_sweeps(T, d13) / ((n - 4) ** 3 * T)
            extras[f"st13_{dtn}_256"] = {
                "value": sw13[d13], "unit": "Mupdates/s", "dim_T": d13, "dim_T_sweep": sw13,
                "roofline_hbm": {"achieved": round(b13 * v13 / 1e9, 1), "peak": hbm_gbs, "unit": "GB/s",
                                 "frac": round(b13 * v13 / 1e9 / hbm_gbs, 4)},
                "frac_alu": round(ST13_OPS * v13 / (SM_COUNT * lanes * sm_max * 1e6), 4),
                "note": f"radius 2, interior (n-4)^3 points; {ST13_OPS} FP lane-ops per update (X25 with FMA)"}
            del x13, y13
        # ablation ladder (Fig. 5(b)), FP32 256^3, T = 100:
        # no blocking -> 2.5D spatial (dim_T = 1) -> 4D (3D blocks of 64 planes + temporal,
        # P:349) -> 3.5D with one row of points per thread -> + several rows per thread
        # (multi-update) -> + two-phase rounds (ILP, the production kernel)
        xa = torch.from_numpy(stgen.grid7(n, n, n, 2, np.float32)).cuda()
        ya = torch.empty_like(xa)

        def bar(D_, variant=0, zchunk=0, naive=False):
            with st.Plan(n, n, n, torch.float32, D_) as pb:
                pb.set_stream(stream)
                if naive:
                    pb.set_variant(st.ST_VARIANT_NAIVE)
                pb.set_option(st.ST_OPT_ST7_VARIANT, variant)
                pb.set_option(st.ST_OPT_ZCHUNK, zchunk)
                tb, _ = time_steps(lambda: pb.st7(xa, ya, 0.4, 0.1, T), 2, 1)
                return round((n - 2) ** 3 * T / (tb / 2 / 1e3) / 1e6, 1)

        def best_of(fn, depths=(2, 3, 4)):
            r = {d: fn(d) for d in depths}
            b = max(r, key=r.get)
            return {"value": r[b], "dim_T": b, "dim_T_sweep": r}

        ladder = {
            "naive_no_blocking": {"value": bar(1, naive=True)},
            "2.5D_spatial_dim_T_1": {"value": sweep.get(1) or bar(1)},
            "4D_3D_blocks_64_planes": best_of(lambda d: bar(d, zchunk=64)),
            "3.5D_one_row_per_thread": best_of(lambda d: bar(d, variant=1256)),
            "3.5D_multi_update_level_by_level": best_of(lambda d: bar(d, variant=94256)),
            "3.5D_multi_update_two_phase": {"value": round(value, 1), "dim_T": D},
        }
        with st.Plan(n, n, n, torch.float32, 8) as pa:   # the library's model-seeded depth search (f3)
            pa.set_stream(stream)
            rep = pa.autotune_report(xa, ya, 24)
        del xa, ya
        gamma = 8.0 / ST7_OPS                                    # B per FP instruction
        Gamma = hbm_gbs * 1e9 / (ops_peak * 1e12)                # measured HBM / nominal FP32 lane rate
        mdl = st.st_blocking_model(227 * 1024, 4, 1, gamma, Gamma, 0, 0)
        extras["ablation_f32_256"] = {
            "unit": "Mupdates/s", "bars": ladder,
            "note": "each bar's kernel is captured by tools/ladder_ncu.sh (profiles/r02/ladder/)"}
        extras["model_f3"] = {
            "gamma_B_per_op": round(gamma, 4), "Gamma_nominal_B_per_op": round(Gamma, 4), "eta_nominal": mdl["eta"],
            "autotune": {k: (round(v, 6) if isinstance(v, float) else v) for k, v in rep.items()},
            "predicted_dim_T": rep["eta"], "measured_best_dim_T": D, "autotune_choice": rep["dim_T"],
            "tile_side_eq4": {"cta_smem": rep["tile_side"][0], "sm_smem_rf": rep["tile_side"][1],
                              "cluster8_dsmem": rep["tile_side"][2]},
            "tile_used": [info["tile_x"], info["tile_y"]],
            "note": "eta = ceil(gamma/Gamma_eff) with Gamma_eff = measured depth-1 bytes/s over the deepest "
                    "sweep's FP lane-ops/s; the nominal-peak eta assumes an FP-pipe-bound kernel"}
        # LBM D3Q19 cavity 256^3 (configs[2])
        for dtn, dt_np, tdt in (("f32", np.float32, torch.float32), ("f64", np.float64, torch.float64)):
            nl, Tl = 256, 100
            flags = torch.from_numpy(stgen.cavity_flags(nl, nl, nl)).cuda()
            f0 = torch.from_numpy(stgen.lbm_rest(nl, nl, nl, dt_np)).cuda()
            fa, fb = f0.clone(), torch.empty_like(f0)
            with st.Plan(nl, nl, nl, tdt, 1) as pl:
                pl.set_stream(stream)
                pl.set_lid(0.05, 0.0, 0.0)
                tl, _ = time_steps(lambda: pl.lbm(fa, fb, 1.6, Tl, flags), 2, 1)
                msl = max_over_ranks(tl / 2)
                cells = (nl - 2) ** 3
                mlups = cells * Tl * world / (msl / 1e3) / 1e6
                E = 4 if dtn == "f32" else 8
                gbs = LBM_BYTES[E] * cells * Tl / (msl / 1e3) / 1e9
                extras[f"lbm_{dtn}_256"] = {"value": round(mlups, 1), "unit": "MLUPS", "dim_T": 1,
                                            "ms_per_step": round(msl, 3),
                                            "roofline": {"bound": "hbm", "achieved": round(gbs, 1),
                                                         "peak": hbm_gbs, "unit": "GB/s",
                                                         "frac": round(gbs / hbm_gbs, 4),
                                                         "traffic": load_traffic(f"lbm_{dtn}_256_D1"),
                                                         "algorithmic_bytes_per_pass": LBM_BYTES[E] * nl ** 3},
                                            "launches": pl.last_launches(),
                                            "kernel": pl.info(True)["kernel"]}
            del fa, fb, f0, flags
        # configs[4] lattice on one GPU (1024^3 FP32 cavity from rest: the strong-scaling base,
        # 163 GB for the two lattices), built on the device
        torch.cuda.empty_cache()
        nb = 1024
        if torch.cuda.mem_get_info()[0] >= 2 * 19 * nb ** 3 * 4 + 3 * nb ** 3 + (4 << 30):
            flb = torch.zeros((nb, nb, nb), dtype=torch.uint8, device="cuda")
            flb[:, 0, :] = 1
            flb[:, :, 0] = 1
            flb[:, :, nb - 1] = 1
            flb[0] = 1
            flb[nb - 1] = 1
            flb[:, nb - 1, :] = 2
            fa = torch.empty((19, nb, nb, nb), dtype=torch.float32, device="cuda")
            wv = stgen.lbm_rest(1, 1, 1, np.float32).reshape(19)
            for i in range(19):
                fa[i].fill_(float(wv[i]))
            fb = torch.empty_like(fa)
            Tb = 10
            with st.Plan(nb, nb, nb, torch.float32, 1) as pl:
                pl.set_stream(stream)
                pl.set_lid(0.05, 0.0, 0.0)
                tl, _ = time_steps(lambda: pl.lbm(fa, fb, 1.6, Tb, flb), 2, 1)
                msl = tl / 2
                cells = (nb - 2) ** 3
                gbs = LBM_BYTES[4] * cells * Tb / (msl / 1e3) / 1e9
                extras["lbm_f32_1024"] = {"value": round(cells * Tb / (msl / 1e3) / 1e6, 1), "unit": "MLUPS",
                                          "dim_T": 1, "T": Tb, "ms_per_step": round(msl, 3),
                                          "kernel": pl.info(True)["kernel"],
                                          "note": "configs[4] lattice on one GPU (strong-scaling base)",
                                          "roofline": {"bound": "hbm", "achieved": round(gbs, 1), "peak": hbm_gbs,
                                                       "unit": "GB/s", "frac": round(gbs / hbm_gbs, 4),
                                                       "traffic": load_traffic("lbm_f32_1024_D1"),
                                                       "algorithmic_bytes_per_pass": LBM_BYTES[4] * nb ** 3}}
            del fa, fb, flb
            torch.cuda.empty_cache()
    cpu = cpu_baseline_7pt(n, T) if (rank == 0 and world == 1) else None

    if rank == 0:
        line = {
            "metric": "Mupdates/s (7-pt)", "value": round(value, 1), "unit": "Mupdates/s",
            "n_gpus": world, "steps": args.steps, "warmup": args.warmup,
            "ms_per_step": round(ms, 4), "higher_is_better": True, "scaling": "weak",
            "vs_baseline": None, "dtype": "f32",
            "data": "synthetic (splitmix64 U[0,1) grid, seed 2; alpha=0.4 beta=0.1)",
            "config": {"workload": (f"7-point stencil FP32 {n}^3, T={T} (BASELINE configs[1]); "
                                    f"dim_T chosen by measurement") if world == 1 else
                                   (f"7-point stencil FP32 {n}x{n}x{n * world} (n^3 per GPU, configs[3] weak "
                                    f"scaling), T={T}, Z-slabs with dim_T-deep NCCL ghost exchange"),
                       "grid": [n, n, n * world], "T": T, "dim_T": D, "dim_T_sweep_Mupd": sweep,
                       "parallelism": f"zslab{world}" if world > 1 else "single",
                       "l2": "flushed between timed steps (512 MiB write)",
                       "plan": info},
            "roofline": roof, "roofline_alt": alt,
            "e2e": {"value": round(upd / (e2e_ms / 1e3) / 1e6, 1), "unit": "Mupdates/s",
                    "h2d_bytes_per_step": grid_bytes, "d2h_bytes_per_step": grid_bytes,
                    "ms_per_step": round(e2e_ms, 3)},
            "gpu_launches": launches * args.steps,
            "kernel_ms_per_launch": round(per_launch_ms, 5),
            "clocks": clk.summary(),
            "cpu_baseline": cpu,
            "extras": extras,
        }
        print(json.dumps(line), flush=True)
    if world > 1:
        dist.destroy_process_group()


if __name__ == "__main__":
    main()
