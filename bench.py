#!/usr/bin/env python
"""bench.py -- grid-point RK-stage updates/sec (fp64) of the CRoCCo v2.0 hot path
on 1..8 B200 (BASELINE.json metric), one process per GPU.

Workload (BASELINE.json configs[4], the north_star's 512^3 target): weak
scaling, 512^3 interior points per GPU of a sinusoidally perturbed periodic
curvilinear grid holding a Taylor-Green vortex + 1% smooth noise, viscous
(mu = 1/1600, Pr = 0.71), fixed dt.  N GPUs hold a (512a)x(512b)x(512c)
global grid, one block per rank, ghost exchange over NCCL.  A step is one
full RK3 time step = 3 x (FillPatch + BC_Fill + WENOx/y/z + Viscous + Update)
(Algorithm 2); value = interior points x 3 x steps / time.

  python bench.py [--gpus N --steps K --warmup W]        # CUDA path (default)
  python bench.py --impl reference ...                   # CPU oracle arm (rank 0)
torchrun launches one rank per GPU for N > 1.
"""
from __future__ import annotations

import argparse
import json
import math
import os
import statistics
import subprocess
import sys
import tempfile
import time

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

METRIC = "grid-point RK-stage updates/sec (fp64) at 1/2/4/8 B200; % HBM roofline"
UNIT = "point-stages/s"
N_BLOCK = 512
# FP64 operations of one characteristic-WENO interface flux:
# hand count of the v1 formulation (FMA = 2, div/sqrt = 1), frozen as the unit of work;
# ncu executed DADD+DMUL+2*DFMA on v1 = 1951 per interface (profiles/r01_ncu.md).
FLUX_FLOPS_PER_IFACE = float(os.environ.get("CROCCO_FLUX_FLOPS", "1924"))
# B200 FP64 (non-tensor) peak: 148 SMs x 64 FMA/clk x 2 flop x 1.965 GHz
FP64_PEAK_TFLOPS = 148 * 64 * 2 * 1.965e9 / 1e12
# compulsory HBM bytes per point-stage of a fused stage: 240 (200 at stage 0)
HBM_BYTES_PER_PT_STAGE = (200 + 240 + 240) / 3.0


WORKLOADS = {
    "weak": f"weak: {N_BLOCK}^3/GPU periodic curvilinear TGV+noise, viscous (BASELINE.json configs[4])",
    "ramp": "ramp: Mach-6 compression ramp 1024x512x256 in 2x2x2 blocks, walls, Sutherland (configs[3])",
    "tgv": "tgv: Taylor-Green vortex 256^3 on the wavy grid, viscous (configs[2])",
    "vortex": "vortex: isentropic vortex on the wavy periodic 64^3 grid, inviscid (configs[1])",
    "sod": "sod: Sod shock tube 200x4x4, inviscid (configs[0])",
    "dmr": "dmr: double Mach reflection 2048x512x128 in 2x2x1 blocks, slip wall + moving shock BCs "
           "(the paper's case, PAPER.md:183-185; SURVEY NEXT-2)",
    "dmr_amr": "dmr_amr: the paper's DMR on a three-level hierarchy (PAPER.md:185, 195): base 1024x256x64 "
               "(2x2x1 blocks) + level-1 patch 1280x128x128 along the wall + level-2 patch 1280x128x256 "
               "around the reflection, ratio 2, slip wall / moving-shock SPLIT faces on every level",
    "amr": "amr: two-level hierarchy (SURVEY NEXT-4): TGV 256^3 coarse level on the wavy grid + a "
           "256^3-node fine level (ratio 2) over its central 128^3 region, C/F faces all round, viscous",
}


def weak_grid(n):
    return {1: (1, 1, 1), 2: (2, 1, 1), 4: (2, 2, 1), 8: (2, 2, 2)}.get(n) or _factor3(n)


def _factor3(n):
    f = [1, 1, 1]
    k = 0
    m = n
    p = 2
    while m > 1:
        while m % p == 0:
            f[k % 3] *= p
            k += 1
            m //= p
        p += 1
    return tuple(f)


def measured_peaks():
    try:
        with open(os.path.join(ROOT, "MEASURED_PEAKS.json")) as f:
            return json.load(f)
    except Exception:
        return {}


# ------------------------------------------------------------------ clocks
class ClockSampler:
    """nvidia-smi clocks + throttle reasons sampled during the timed region."""

    def __init__(self, gpu_index):
        self.f = tempfile.NamedTemporaryFile("w+", suffix=".csv", delete=False)
        q = ("clocks.sm,clocks.max.sm,power.draw,clocks_event_reasons.hw_slowdown,"
             "clocks_event_reasons.hw_thermal_slowdown,clocks_event_reasons.sw_thermal_slowdown,"
             "clocks_event_reasons.sw_power_cap")
        try:
            self.p = subprocess.Popen(["nvidia-smi", "-i", str(gpu_index), f"--query-gpu={q}",
                                       "--format=csv,noheader,nounits", "-lms", "200"],
                                      stdout=self.f, stderr=subprocess.DEVNULL)
        except Exception:
            self.p = None

    def stop(self):
        if self.p is None:
            return None
        self.p.terminate()
        try:
            self.p.wait(timeout=5)
        except Exception:
            self.p.kill()
        self.f.flush()
        rows = []
        with open(self.f.name) as fh:
            for line in fh:
                parts = [x.strip() for x in line.split(",")]
                if len(parts) < 7:
                    continue
                try:
                    rows.append((float(parts[0]), float(parts[1]), parts[3:7]))
                except ValueError:
                    pass
        os.unlink(self.f.name)
        if not rows:
            return None
        names = ["hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown", "sw_power_cap"]
        reasons = sorted({names[i] for _, _, r in rows for i, v in enumerate(r) if v.lower() == "active"})
        return {"sm_mhz": statistics.median(r[0] for r in rows), "sm_max_mhz": max(r[1] for r in rows),
                "reasons": reasons, "samples": len(rows)}


# ------------------------------------------------------------------ oracle (CPU baseline)
def oracle_rate(max_seconds=12.0, n=64, max_steps=100, steps=None, warmup=0):
    """Time the CPU oracle (as it stands) on a bounded sample of the workload:
    an n^3 periodic wavy-grid TGV+noise box, whole RK3 steps, all host cores."""
    import numpy as np

    import oracle
    import synth
    oracle.build()
    cores = os.cpu_count() or 1
    oracle.set_threads(cores)
    nn = (n, n, n)
    grid = synth.Wavy3D(L=(2 * math.pi,) * 3, N=nn, x0=(-math.pi,) * 3, k=2.0, A=0.15)
    xyz = grid.coords(nn, (0, 0, 0), oracle.GC)
    met = oracle.metrics(nn, ((0, 0),) * 3, xyz)
    U = synth.pad_state(synth.tgv(xyz, noise=0.01, seed=5))
    ph = oracle.phys(gamma=1.4, R=1.0, Pr=0.71, mu_ref=1 / 1600, terms=3)
    bc = ((0, 0),) * 3
    for _ in range(warmup):
        oracle.advance(nn, bc, ph, 2e-3, 1, U, met)
    done = 0
    t0 = time.perf_counter()
    per_step = []
    while True:
        ts = time.perf_counter()
        oracle.advance(nn, bc, ph, 2e-3, 1, U, met)
        per_step.append(time.perf_counter() - ts)
        done += 1
        el = time.perf_counter() - t0
        if steps is not None:
            if done >= steps:
                break
        elif el >= max_seconds or done >= max_steps:
            break
    el = time.perf_counter() - t0
    pts = n ** 3 * 3 * done
    return {"value": pts / el, "unit": UNIT, "cores": oracle.get_threads(), "kind": "oracle",
            "sample": f"{done} RK3 step(s) (3 stages each) of a {n}^3 periodic wavy-grid TGV+noise box "
                      f"(same discretisation and per-point work as the {N_BLOCK}^3 workload), "
                      f"{el:.2f} s wall", "seconds": el, "steps": done, "per_step_s": per_step}


def oracle_suite(max_total=60.0):
    """BASELINE.md sec. 4's CPU baseline: the oracle (as it stands) on the paper-shaped configs at
    1 host core and at all host cores -- Sod 200x4x4 for 100 RK3 steps (wall seconds), the
    isentropic vortex on the 64^3 wavy grid (100 steps on all cores, a bounded number on one
    core), and one RK3 step (3 stages) of a 128^3 TGV box; each as point-stages/s."""
    import oracle
    import synth
    oracle.build()
    cores = os.cpu_count() or 1
    out = []
    t_start = time.perf_counter()

    def run(name, n, bc, grid, U0, ph, dt, steps, threads, note):
        oracle.set_threads(threads)
        xyz = grid.coords(n, (0, 0, 0), oracle.GC)
        met = oracle.metrics(n, bc, xyz)
        U = synth.pad_state(U0(xyz))
        t0 = time.perf_counter()
        oracle.advance(n, bc, ph, dt, steps, U, met)
        el = time.perf_counter() - t0
        pts = n[0] * n[1] * n[2] * 3 * steps
        out.append({"config": name, "cores": oracle.get_threads(), "steps": steps, "seconds": round(el, 4),
                    "value": pts / el, "unit": UNIT, "note": note})

    sod = synth.case("sod")
    vtx = synth.case("vortex")
    tgv = synth.case("tgv", scale=2)  # 128^3
    ph_inv = oracle.phys(gamma=1.4, R=1.0, terms=1)
    ph_tgv = oracle.phys(**tgv.phys)
    for threads in (1, cores):
        run("sod 200x4x4 (configs[0])", sod.n_global, sod.bc, sod.grid, synth.sod, ph_inv, sod.dt, 100, threads,
            "100 RK3 steps, wall seconds")
        vsteps = 100 if threads == cores else 4
        run("vortex 64^3 wavy (configs[1])", vtx.n_global, vtx.bc, vtx.grid, synth.vortex, ph_inv, vtx.dt, vsteps,
            threads, "100 RK3 steps" if vsteps == 100 else f"bounded sample: {vsteps} RK3 steps on one core")
        run("tgv 128^3 wavy, viscous (configs[2] at half resolution)", tgv.n_global, tgv.bc, tgv.grid,
            synth.tgv, ph_tgv, tgv.dt, 1, threads, "3 RK stages (one RK3 step)")
        if time.perf_counter() - t_start > max_total:
            break
    oracle.set_threads(cores)
    return out


# ------------------------------------------------------------------ reference arm
def run_reference(args, rank, world):
    if rank != 0:
        return 0
    r = oracle_rate(steps=args.steps, warmup=args.warmup, n=args.ref_n)
    ms = 1e3 * r["seconds"] / r["steps"]
    out = {"impl": "reference", "metric": METRIC, "value": r["value"], "unit": UNIT,
           "n_gpus": args.gpus, "steps": args.steps, "warmup": args.warmup, "ms_per_step": ms,
           "higher_is_better": True, "scaling": "weak", "vs_baseline": None, "dtype": "f64",
           "data": "synthetic",
           "config": {"workload": f"weak: {N_BLOCK}^3/GPU periodic curvilinear TGV+noise, viscous; "
                                  f"reference arm times a bounded {args.ref_n}^3 sample per step",
                      "sample_points": args.ref_n ** 3},
           "cpu_baseline": {k: r[k] for k in ("value", "unit", "cores", "kind", "sample")},
           "e2e": {"value": r["value"], "unit": UNIT, "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0}}
    print(json.dumps(out), flush=True)
    return 0


# ------------------------------------------------------------------ CUDA arm
def run_crocco(args, rank, world, local_rank):
    import numpy as np
    import torch
    import torch.distributed as dist

    import synth
    from paper_conf_ipps_davissngmb23_b200 import crocco as cc
    from paper_conf_ipps_davissngmb23_b200.solver import Solver

    torch.cuda.set_device(local_rank)
    dev = torch.device("cuda", local_rank)
    uid = None
    if world > 1:
        t = torch.zeros(128, dtype=torch.uint8, device=dev)
        if rank == 0:
            t.copy_(torch.frombuffer(bytearray(cc.crocco_nccl_unique_id()), dtype=torch.uint8))
        dist.broadcast(t, 0)
        uid = bytes(t.cpu().numpy().tobytes())
    if args.config == "weak":
        # weak scaling: 512^3 per GPU, one block per rank (BASELINE.json configs[4])
        a, b, c = weak_grid(world)
        nb = (a, b, c)
        n = (N_BLOCK * a, N_BLOCK * b, N_BLOCK * c)
        grid = synth.Wavy3D(L=(2 * math.pi * a, 2 * math.pi * b, 2 * math.pi * c), N=n,
                            x0=(-math.pi,) * 3, k=2.0, A=0.15)
        phys = dict(gamma=1.4, R=1.0, Pr=0.71, mu_ref=1.0 / 1600.0, terms=3)
        dt, bc, state = 2e-4, ((0, 0),) * 3, "tgv_noise"
        block_rank = list(range(world))
        case = synth.Case("weak", n, nb, bc, grid, state, phys, dt)
    else:
        # fixed global problem (strong scaling for N > 1): configs[0..3]
        case = synth.case(args.config)
        n, nb, bc, grid, phys, dt = case.n_global, case.n_blocks, case.bc, case.grid, case.phys, case.dt
        nbt = nb[0] * nb[1] * nb[2]
        block_rank = [bb * world // nbt for bb in range(nbt)]
    dirichlet, split = None, None
    if args.config == "dmr":
        bc, dirichlet, split = synth.dmr_bc(1.0 / n[1])
    S = Solver(n, nb, bc, cc.make_phys(**phys), rank=rank, nranks=world, dirichlet=dirichlet,
               block_rank=block_rank, device=dev, nccl_unique_id=uid, split=split)
    for bl in range(S.nloc):
        L = S.layouts[bl]
        origin, bn = tuple(L.origin), tuple(L.n)
        if case.state in ("tgv", "tgv_noise"):
            # generated on the device (torch ops on the synth formulas) -- input setup only
            if isinstance(grid, synth.Wavy3D):
                xyz = grid.coords(bn, origin, cc.GHOST_COORDS, device=dev)
            else:
                xyz = torch.from_numpy(grid.coords(bn, origin, cc.GHOST_COORDS)).to(dev)
            U0 = synth.tgv(xyz, noise=0.01 if case.state == "tgv_noise" else 0.0, seed=5)
        else:
            xyz, U0 = synth.block_inputs(case, origin, bn)
        S.set_coords_block(bl, xyz)
        S.set_state_block(bl, U0)
        del xyz, U0
    pts_local = sum(L.n[0] * L.n[1] * L.n[2] for L in S.layouts)
    pts_total = n[0] * n[1] * n[2]
    bn = tuple(S.layouts[0].n)
    torch.cuda.synchronize()
    stream = S.stream

    for _ in range(args.warmup):
        S.step(dt)
    torch.cuda.synchronize()

    # ---------------- timed region (device-resident inputs)
    state_bytes = sum(u.numel() for u in S.U) * 8
    flush = state_bytes < 4 * 126e6  # small configs: flush L2 between timed steps
    # kernel-class CUDA events inside the timed region for the large (non-graph) workloads;
    # small launch-bound configs run CUDA-graph steps and get their breakdown afterwards
    cc.crocco_set_timing(S.ctx, not flush)
    cc.crocco_kernel_times(S.ctx)          # reset accumulators
    cc.crocco_launch_count(S.ctx, reset=True)
    clk = ClockSampler(local_rank) if not args.no_clocks else None
    scratch = torch.empty(int(256e6) // 8, dtype=torch.float64, device=dev) if flush else None
    evs = [(torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True))
           for _ in range(args.steps if flush else 1)]
    if world > 1:
        dist.barrier()
    torch.cuda.synchronize()
    if flush:
        for e0, e1 in evs:
            scratch.fill_(1.0)               # 256 MB write evicts L2 (outside the timed events)
            e0.record(stream)
            S.step(dt)
            e1.record(stream)
    else:
        e0, e1 = evs[0]
        e0.record(stream)
        for _ in range(args.steps):
            S.step(dt)
        e1.record(stream)
    torch.cuda.synchronize()
    if world > 1:
        dist.barrier()
    ms_local = sum(a_.elapsed_time(b_) for a_, b_ in evs)
    clocks = clk.stop() if clk else None
    launches = cc.crocco_launch_count(S.ctx)
    if flush:  # breakdown pass (eager launches with events) after the graph-timed region
        cc.crocco_set_timing(S.ctx, True)
        cc.crocco_kernel_times(S.ctx)
        for _ in range(args.steps):
            S.step(dt)
        torch.cuda.synchronize()
    ktimes = cc.crocco_kernel_times(S.ctx)
    cc.crocco_set_timing(S.ctx, False)
    t = torch.tensor([ms_local], dtype=torch.float64, device=dev)
    if world > 1:
        dist.all_reduce(t, op=dist.ReduceOp.MAX)
    ms = float(t.item())
    value = pts_total * 3 * args.steps / (ms / 1e3)
    # state sanity (finite, positive density) -- not part of the timed region
    finite = S.check_state() == 0   # crocco_check_state: no non-finite value, rho, p > 0

    # ---------------- end-to-end through the public API with host buffers
    e2e = None
    if args.e2e_steps > 0:
        # each step is an independent job: its input state (the interior points: the step's fill
        # makes the ghosts) is uploaded from pinned host memory and its result downloaded;
        # Solver.steps_from_host overlaps job n's download and job n+1's upload with compute on two
        # copy streams (the host link is full duplex)
        G_ = cc.GHOST
        ints = [S.view(u, b, 5)[:, G_:-G_, G_:-G_, G_:-G_] for b, u in enumerate(S.U)]
        h_in = [[torch.empty(v.shape, dtype=torch.float64, pin_memory=True) for v in ints] for _ in range(2)]
        h_out = [[torch.empty(v.shape, dtype=torch.float64, pin_memory=True) for v in ints] for _ in range(2)]
        for hs in h_in:
            for h, v in zip(hs, ints):
                h.copy_(v)
        del ints
        S.steps_from_host([h_in[0]], [h_out[0]], dt, interior=True)   # untimed: graphs for both pairs
        S.steps_from_host([h_in[1]], [h_out[1]], dt, interior=True)
        torch.cuda.synchronize()
        if world > 1:
            dist.barrier()
        f0 = torch.cuda.Event(enable_timing=True)
        f1 = torch.cuda.Event(enable_timing=True)
        f0.record(stream)
        S.steps_from_host([h_in[n % 2] for n in range(args.e2e_steps)],
                          [h_out[n % 2] for n in range(args.e2e_steps)], dt, interior=True)
        f1.record(stream)
        torch.cuda.synchronize()
        te = torch.tensor([f0.elapsed_time(f1)], dtype=torch.float64, device=dev)
        if world > 1:
            dist.all_reduce(te, op=dist.ReduceOp.MAX)
        nbytes = sum(h.numel() for h in h_in[0]) * 8
        if world > 1:
            tb = torch.tensor([nbytes], dtype=torch.float64, device=dev)
            dist.all_reduce(tb)
            nbytes = int(tb.item())
        e2e = {"value": pts_total * 3 * args.e2e_steps / (float(te.item()) / 1e3), "unit": UNIT,
               "h2d_bytes_per_step": nbytes, "d2h_bytes_per_step": nbytes,
               "steps": args.e2e_steps,
               "note": "independent jobs: per step H2D of the input state (interior points) from pinned host "
                       "memory, RK3 step, D2H of the result (interior points); copies on two streams overlap "
                       "neighbouring jobs' compute"}

    # ---------------- end-to-end solver loop (Algorithm 1): state uploaded
    # once, every step ComputeDt (device reduction, dt read back: the step's result) + RK3 step,
    # final state downloaded
    e2e_loop = None
    if args.e2e_steps > 0:
        hosts = [torch.empty(u.numel(), dtype=torch.float64, pin_memory=True) for u in S.U]
        for h, u in zip(hosts, S.U):
            h.copy_(u)
        torch.cuda.synchronize()
        if world > 1:
            dist.barrier()
        g0 = torch.cuda.Event(enable_timing=True)
        g1 = torch.cuda.Event(enable_timing=True)
        g0.record(stream)
        for h, u in zip(hosts, S.U):
            u.copy_(h, non_blocking=True)
        for _ in range(args.e2e_steps):
            dtn = S.compute_dt(0.4)
            S.step(min(dtn, dt))
        for h, u in zip(hosts, S.U):
            h.copy_(u, non_blocking=True)
        g1.record(stream)
        torch.cuda.synchronize()
        tl = torch.tensor([g0.elapsed_time(g1)], dtype=torch.float64, device=dev)
        if world > 1:
            dist.all_reduce(tl, op=dist.ReduceOp.MAX)
        e2e_loop = {"value": pts_total * 3 * args.e2e_steps / (float(tl.item()) / 1e3), "unit": UNIT,
                    "steps": args.e2e_steps, "h2d_bytes_total": sum(h.numel() for h in hosts) * 8,
                    "d2h_bytes_per_step": 8,
                    "note": "Alg. 1 loop: ComputeDt (dt read back each step) + RK3 step; state uploaded "
                            "once before and downloaded once after the steps"}

    # ---------------- roofline of the dominant kernel (CUDA events on the launching stream)
    flux_cls = {"sweep_xi": 0, "sweep_eta": 1, "sweep_zeta_update": 2}
    dom = max(ktimes.items(), key=lambda kv: kv[1][1])
    name, (nl, kms) = dom
    avg_ms = kms / max(nl, 1)
    roof = None
    if name in flux_cls:
        d = flux_cls[name]
        ifaces = (bn[d] + 1) * (bn[0] * bn[1] * bn[2]) // bn[d]  # per launch (one block)
        ach = FLUX_FLOPS_PER_IFACE * ifaces / (avg_ms / 1e3) / 1e12
        roof = {"bound": "alu", "kernel": f"k_sweep_s<{d}> ({name})", "achieved": ach,
                "peak": FP64_PEAK_TFLOPS, "unit": "TFLOP/s", "frac": ach / FP64_PEAK_TFLOPS,
                "peak_source": "derived: 148 SM x 64 FP64 FMA/clk x 2 x 1.965 GHz (DESIGN.md sec. 6)",
                "flops_per_unit": FLUX_FLOPS_PER_IFACE, "unit_of_work": "interface flux",
                "units_per_launch": ifaces, "avg_launch_ms": avg_ms,
                "traffic": _profiled_traffic(f"k_sweep_s<{d},"),
                "fp64_pipe_active_pct": _profiled_traffic(f"k_sweep_s<{d},", "fp64_pipe_pct"),
                "achieved_occupancy_pct": _profiled_traffic(f"k_sweep_s<{d},", "achieved_occupancy_pct"),
                "traffic_source": "profiles/ncu_summary.json (ncu --set full, dram__bytes_read+write per launch; "
                                  "sm__pipe_fp64_cycles_active and achieved occupancy of the same capture)"}
    peaks = measured_peaks()
    hbm = peaks.get("hbm_gbs", 6650.0)
    stage_gbs = value / world * HBM_BYTES_PER_PT_STAGE / 1e9
    ktot = sum(v[1] for v in ktimes.values())
    breakdown = {k: {"launches": v[0], "ms": v[1], "share_of_kernel_time": v[1] / max(ktot, 1e-9)}
                 for k, v in ktimes.items() if v[0]}
    out = {"metric": METRIC, "value": value, "unit": UNIT, "n_gpus": world, "steps": args.steps,
           "warmup": args.warmup, "ms_per_step": ms / args.steps, "higher_is_better": True,
           "scaling": "weak" if args.config == "weak" else "strong", "vs_baseline": None, "dtype": "f64",
           "data": "synthetic (seeded, " + WORKLOADS[args.config].split(":")[0] + " recipe of DESIGN.md sec. 4)",
           "config": {"workload": WORKLOADS[args.config] + "; step = 1 RK3 step (3 stages)",
                      "n_global": list(n), "n_blocks": list(nb), "points_per_gpu": pts_local,
                      "dt": dt,
                      "l2": ("L2 flushed (256 MB write) between timed steps" if flush else
                             f"inputs larger than L2 ({state_bytes / 1e9:.1f} GB state vs 126 MB L2)"),
                      "parallelism": f"spatial blocks {nb[0]}x{nb[1]}x{nb[2]} over {world} GPU(s), "
                                     "NCCL halo exchange"},
           "roofline": roof,
           "hbm": {"algorithmic_gbs_per_gpu": stage_gbs, "peak_gbs": hbm,
                   "frac": stage_gbs / hbm, "bytes_per_point_stage": HBM_BYTES_PER_PT_STAGE,
                   "note": "whole-stage compulsory traffic; the path is FP64-pipe bound"},
           "kernel_breakdown": breakdown,
           "gpu_launches": launches, "clocks": clocks, "e2e": e2e, "e2e_solver_loop": e2e_loop,
           "state_finite": finite}
    if rank == 0 and world == 1 and not args.no_cpu_baseline:
        r = oracle_rate()
        out["cpu_baseline"] = {k: r[k] for k in ("value", "unit", "cores", "kind", "sample")}
        # 1 core and all cores on Sod / vortex / TGV (same run, same host)
        out["cpu_baseline"]["suite"] = oracle_suite()
    S.close()
    if rank == 0:
        print(json.dumps(out), flush=True)
    return 0


def run_amr(args):
    """--config amr (one GPU): Algorithm 2 with two levels -- per stage the coarse level, the fine
    level with its C/F ghosts interpolated from the coarse stage input (k_cf_interp), AverageDown
    (k_average_down) at the third stage.  value = (coarse + fine interior points) x 3 x steps / time."""
    import torch

    import synth
    from paper_conf_ipps_davissngmb23_b200 import crocco as cc
    from paper_conf_ipps_davissngmb23_b200.solver import AmrSolver, Solver

    dev = torch.device("cuda", 0)
    torch.cuda.set_device(dev)
    nc, c0, nf = (256, 256, 256), (64, 64, 64), (256, 256, 256)
    grid = synth.Wavy3D(L=(2 * math.pi,) * 3, N=nc, x0=(-math.pi,) * 3, k=2.0, A=0.15)
    fgrid = synth.Refined(grid, c0)
    phys = cc.make_phys(gamma=1.4, R=1.0, Pr=0.71, mu_ref=1.0 / 1600.0, terms=3)
    CF = cc.BC_COARSE_FINE
    C = Solver(nc, (1, 1, 1), ((0, 0),) * 3, phys, device=dev)
    F = Solver(nf, (1, 1, 1), ((CF, CF),) * 3, phys, device=dev)
    for S, g, n in ((C, grid, nc), (F, fgrid, nf)):
        xyz = torch.from_numpy(g.coords(n, (0, 0, 0), cc.GHOST_COORDS)).to(dev)
        S.set_coords_block(0, xyz)
        S.set_state_block(0, synth.tgv(xyz, noise=0.01, seed=5))
        del xyz
    A = AmrSolver(C, F, c0)
    dt = 2e-4
    for _ in range(args.warmup):
        A.step(dt)
    torch.cuda.synchronize()
    for S in (C, F):
        cc.crocco_set_timing(S.ctx, True)
        cc.crocco_kernel_times(S.ctx)
        cc.crocco_launch_count(S.ctx, reset=True)
    clk = ClockSampler(0) if not args.no_clocks else None
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    torch.cuda.synchronize()
    e0.record(C.stream)
    A.step(dt, args.steps)
    e1.record(C.stream)
    torch.cuda.synchronize()
    ms = e0.elapsed_time(e1)
    clocks = clk.stop() if clk else None
    launches = cc.crocco_launch_count(C.ctx) + cc.crocco_launch_count(F.ctx)
    kt = {}
    for lv, S in (("coarse", C), ("fine", F)):
        for k, (nl, kms) in cc.crocco_kernel_times(S.ctx).items():
            if nl:
                kt[f"{lv}:{k}"] = {"launches": nl, "ms": kms}
    ktot = sum(v["ms"] for v in kt.values())
    for v in kt.values():
        v["share_of_kernel_time"] = v["ms"] / max(ktot, 1e-9)
    pts = nc[0] * nc[1] * nc[2] + nf[0] * nf[1] * nf[2]
    value = pts * 3 * args.steps / (ms / 1e3)
    amr_ms = sum(v["ms"] for k, v in kt.items() if k.endswith(":amr"))
    finite = all(S.check_state() == 0 for S in (C, F))
    # C/F interpolation and AverageDown: HBM gathers; algorithmic bytes = 5 comps x 8 B written per
    # C/F ghost point (+ the coarse corners read once, 1/8 of that) and 27+1 fine/coarse values per
    # covered coarse point -- reported as a share of the step, not as a roofline (they are < 1 %)
    out = {"metric": METRIC, "value": value, "unit": UNIT, "n_gpus": 1, "steps": args.steps,
           "warmup": args.warmup, "ms_per_step": ms / args.steps, "higher_is_better": True,
           "scaling": "strong", "vs_baseline": None, "dtype": "f64",
           "data": "synthetic (seeded TGV + 1 % noise on both levels, DESIGN.md sec. 4)",
           "config": {"workload": WORKLOADS["amr"] + "; step = 1 RK3 step (3 stages x 2 levels + AverageDown)",
                      "n_coarse": list(nc), "n_fine": list(nf), "c0": list(c0), "points": pts, "dt": dt,
                      "l2": "inputs larger than L2 (1.5 GB state per level)", "parallelism": "1 GPU"},
           "amr_kernels_share": amr_ms / max(ktot, 1e-9), "kernel_breakdown": kt,
           "gpu_launches": launches, "clocks": clocks, "state_finite": finite, "impl": "crocco"}
    C.close()
    F.close()
    print(json.dumps(out), flush=True)
    return 0


def run_dmr_amr(args):
    """--config dmr_amr (one GPU): Algorithm 2 over three levels (AmrHierarchy): per stage the base
    DMR grid, the level-1 and level-2 patches (C/F ghosts from the parent's stage input, DMR
    boundary data on the wall faces), AverageDown of each level after its third-stage update.
    value = (all levels' interior points) x 3 x steps / time."""
    import torch

    import synth
    from paper_conf_ipps_davissngmb23_b200 import crocco as cc
    from paper_conf_ipps_davissngmb23_b200.solver import AmrHierarchy, Solver

    dev = torch.device("cuda", 0)
    torch.cuda.set_device(dev)
    c = synth.case("dmr", scale=2)
    n0 = c.n_global
    h = 1.0 / n0[1]
    bc0, dv0, sp0 = synth.dmr_bc(h)
    specs = [(n0, c.grid, bc0, dv0, sp0, c.n_blocks, None)]
    for c0, nf, nb in (((128, 0, 0), (1280, 128, 128), (2, 1, 1)), ((320, 0, 0), (1280, 128, 256), (2, 1, 2))):
        n_up, g_up, bc_up, dv_up, sp_up = specs[-1][:5]
        bcf, dvf, spf = synth.refine_bc(n_up, bc_up, dv_up, sp_up, c0, nf)
        specs.append((nf, synth.Refined(g_up, c0), bcf, dvf, spf, nb, c0))
    phys = cc.make_phys(**c.phys)
    S = []
    for n, g, bc, dv, sp, nb, _ in specs:
        X = Solver(n, nb, bc, phys, dirichlet=dv, split=sp, device=dev)
        for bl in range(X.nloc):
            L = X.layouts[bl]
            xyz = g.coords(tuple(L.n), tuple(L.origin), cc.GHOST_COORDS)
            X.set_coords_block(bl, xyz)
            X.set_state_block(bl, synth.dmr_state(xyz))
        S.append(X)
    H = AmrHierarchy(S[0], [[(S[1], 0, specs[1][6])], [(S[2], 0, specs[2][6])]])
    dt = 0.2 * (h / 4) / 13.0
    for _ in range(args.warmup):
        H.step(dt)
    torch.cuda.synchronize()
    for X in S:
        cc.crocco_set_timing(X.ctx, True)
        cc.crocco_kernel_times(X.ctx)
        cc.crocco_launch_count(X.ctx, reset=True)
    clk = ClockSampler(0) if not args.no_clocks else None
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    torch.cuda.synchronize()
    e0.record(S[0].stream)
    H.step(dt, args.steps)
    e1.record(S[0].stream)
    torch.cuda.synchronize()
    ms = e0.elapsed_time(e1)
    clocks = clk.stop() if clk else None
    launches = sum(cc.crocco_launch_count(X.ctx) for X in S)
    kt = {}
    for lv, X in enumerate(S):
        for k, (nl, kms) in cc.crocco_kernel_times(X.ctx).items():
            if nl:
                kt[f"level{lv}:{k}"] = {"launches": nl, "ms": kms}
    ktot = sum(v["ms"] for v in kt.values())
    for v in kt.values():
        v["share_of_kernel_time"] = v["ms"] / max(ktot, 1e-9)
    pts = [n[0] * n[1] * n[2] for n, *_ in specs]
    value = sum(pts) * 3 * args.steps / (ms / 1e3)
    finite = all(X.check_state() == 0 for X in S)
    out = {"metric": METRIC, "value": value, "unit": UNIT, "n_gpus": 1, "steps": args.steps,
           "warmup": args.warmup, "ms_per_step": ms / args.steps, "higher_is_better": True,
           "scaling": "strong", "vs_baseline": None, "dtype": "f64",
           "data": "synthetic (Woodward-Colella DMR initial state on every level, DESIGN.md sec. 4)",
           "config": {"workload": WORKLOADS["dmr_amr"] + "; step = 1 RK3 step (3 stages x 3 levels + AverageDown)",
                      "levels": [{"n": list(n), "c0": list(c0) if c0 else None, "blocks": list(nb), "points": p}
                                 for (n, _, _, _, _, nb, c0), p in zip(specs, pts)],
                      "points": sum(pts), "dt": dt,
                      "l2": "inputs larger than L2", "parallelism": "1 GPU"},
           "amr_kernels_share": sum(v["ms"] for k, v in kt.items() if k.endswith(":amr")) / max(ktot, 1e-9),
           "kernel_breakdown": kt, "gpu_launches": launches, "clocks": clocks, "state_finite": finite,
           "impl": "crocco"}
    for X in S:
        X.close()
    print(json.dumps(out), flush=True)
    return 0


def run_size_sweep(args):
    """The paper's Fig. 3 analogue (sec. VI-A): time per RK3 step spent in the
    WENOx and Viscous work over a range of problem sizes, on the GPU (this library: the xi sweep
    class and the viscous kernel class, CUDA events per launch) and on the host CPU (the oracle as
    it stands, at 1 core and all cores: its RHS with only the xi inviscid flux, and with only the
    viscous terms).  The GPU viscous class holds the point fluxes and the xi / zeta divergences
    (the eta divergence rides in the eta sweep); the oracle's viscous RHS holds all three.
    Weak-recipe boxes (periodic wavy grid, TGV + noise), one block, one GPU."""
    import torch

    import synth
    from paper_conf_ipps_davissngmb23_b200 import crocco as cc
    from paper_conf_ipps_davissngmb23_b200.solver import Solver

    phys = dict(gamma=1.4, R=1.0, Pr=0.71, mu_ref=1.0 / 1600.0, terms=3)
    dt = 2e-4
    gpu = []
    for N in (32, 64, 96, 128, 192, 256, 384, 512):
        n = (N, N, N)
        grid = synth.Wavy3D(L=(2 * math.pi,) * 3, N=n, x0=(-math.pi,) * 3, k=2.0, A=0.15)
        S = Solver(n, (1, 1, 1), ((0, 0),) * 3, cc.make_phys(**phys))
        dev = S.device
        xyz = torch.from_numpy(grid.coords(n, (0, 0, 0), cc.GHOST_COORDS)).to(dev)
        S.set_coords_block(0, xyz)
        S.set_state_block(0, synth.tgv(xyz, noise=0.01, seed=5))
        del xyz
        for _ in range(max(args.warmup, 1)):
            S.step(dt, graph=False)
        reps = max(2, min(50, int(2e8 // N ** 3)))
        cc.crocco_set_timing(S.ctx, True)
        cc.crocco_kernel_times(S.ctx)
        torch.cuda.synchronize()
        for _ in range(reps):
            S.step(dt, graph=False)
        kt = cc.crocco_kernel_times(S.ctx)
        S.close()
        row = {"n": N, "points": N ** 3, "rk3_steps": reps}
        for cls, key in (("sweep_xi", "wenox_ms_per_step"), ("viscous", "viscous_ms_per_step")):
            row[key] = kt[cls][1] / reps
        row["all_kernels_ms_per_step"] = sum(v[1] for v in kt.values()) / reps
        gpu.append(row)
    cpu = []
    if not args.no_cpu_baseline:
        import oracle
        oracle.build()
        cores = os.cpu_count() or 1
        t_start = time.perf_counter()
        for threads in (1, cores):
            oracle.set_threads(threads)
            for N in (16, 24, 32, 48, 64):
                n = (N, N, N)
                grid = synth.Wavy3D(L=(2 * math.pi,) * 3, N=n, x0=(-math.pi,) * 3, k=2.0, A=0.15)
                xyz = grid.coords(n, (0, 0, 0), oracle.GC)
                met = oracle.metrics(n, ((0, 0),) * 3, xyz)
                U = synth.pad_state(synth.tgv(xyz, noise=0.01, seed=5))
                oracle.fill(n, ((0, 0),) * 3, U)
                row = {"n": N, "points": N ** 3, "cores": oracle.get_threads()}
                for key, kw in (("wenox_ms_per_step", dict(terms=1, dir_mask=1)), ("viscous_ms_per_step", dict(terms=2))):
                    ph = oracle.phys(**dict(phys, **kw))
                    t0 = time.perf_counter()
                    k = 0
                    while True:
                        oracle.rhs(n, ph, U, met)
                        k += 1
                        if time.perf_counter() - t0 > 0.5 or k >= 20:
                            break
                    row[key] = 3e3 * (time.perf_counter() - t0) / k   # 3 RHS evaluations per RK3 step
                cpu.append(row)
                if time.perf_counter() - t_start > 120:
                    break
        oracle.set_threads(cores)
    out = {"metric": "WENOx / Viscous time per RK3 step vs problem size (PAPER.md Fig. 3 analogue)",
           "unit": "ms per RK3 step", "dtype": "f64", "data": "synthetic",
           "config": {"workload": "size sweep: weak-recipe boxes N^3 (periodic wavy grid, TGV + noise, viscous), "
                                  "one block, one GPU; CPU = the oracle at 1 core and all cores"},
           "gpu": gpu, "cpu": cpu}
    print(json.dumps(out), flush=True)
    return 0


def _profiled_traffic(kname, key="dram_bytes_per_launch"):
    """A per-launch ncu figure (default: dram bytes) of the dominant kernel from the committed
    ncu summary (profiles/ncu_summary.json), if any."""
    p = os.path.join(ROOT, "profiles", "ncu_summary.json")
    try:
        with open(p) as f:
            ks = json.load(f).get("kernels", {})
        for k, v in ks.items():  # kname: full kernel name or a prefix of it
            if k.startswith(kname) and key in v:
                return v[key]
        return None
    except Exception:
        return None


def relaunch(ngpus):
    """`python bench.py --gpus N` without torchrun: check that N GPUs are visible, then run
    the same command line as N ranks (one process per GPU) under torch.distributed.run on
    127.0.0.1, with NCCL's INIT lines on stderr.  Fails loudly (exit 2) with fewer GPUs:
    N ranks on one device is not a multi-GPU run (NCCL refuses it anyway)."""
    import socket

    import torch
    have = torch.cuda.device_count()
    if have < ngpus:
        print(f"bench.py: --gpus {ngpus} needs {ngpus} visible CUDA devices, found {have}", file=sys.stderr)
        return 2
    with socket.socket() as so:
        so.bind(("127.0.0.1", 0))
        port = so.getsockname()[1]
    env = dict(os.environ)
    env.setdefault("NCCL_DEBUG", "INFO")
    env.setdefault("NCCL_DEBUG_SUBSYS", "INIT")
    cmd = [sys.executable, "-m", "torch.distributed.run", "--nnodes=1", f"--nproc-per-node={ngpus}",
           "--master-addr=127.0.0.1", f"--master-port={port}", os.path.abspath(__file__), *sys.argv[1:]]
    print("bench.py: relaunching as " + " ".join(cmd), file=sys.stderr, flush=True)
    return subprocess.call(cmd, env=env)


def main():
    ap = argparse.ArgumentParser(description=__doc__, formatter_class=argparse.RawDescriptionHelpFormatter)
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=5)
    ap.add_argument("--warmup", type=int, default=3)
    ap.add_argument("--impl", choices=["crocco", "reference"], default="crocco")
    ap.add_argument("--config", choices=["weak", "ramp", "tgv", "vortex", "sod", "dmr", "amr", "dmr_amr",
                                         "size_sweep"],
                    default="weak",
                    help="weak (default, the north_star 512^3/GPU workload) or a fixed BASELINE config")
    ap.add_argument("--e2e-steps", type=int, default=48,
                    help="independent jobs streamed through host memory for e2e (pipeline fill + drain amortised)")
    ap.add_argument("--no-cpu-baseline", action="store_true")
    ap.add_argument("--no-clocks", action="store_true")
    ap.add_argument("--ref-n", type=int, default=64)
    args = ap.parse_args()
    launched = "WORLD_SIZE" in os.environ
    rank = int(os.environ.get("RANK", "0"))
    world = int(os.environ.get("WORLD_SIZE", "1"))
    local_rank = int(os.environ.get("LOCAL_RANK", "0"))
    if args.gpus < 1:
        raise SystemExit("--gpus must be >= 1")
    if args.impl == "reference":
        # the CPU oracle arm: rank 0 alone runs (under torchrun the other ranks exit 0)
        return run_reference(args, rank, world)
    if not launched and args.gpus > 1:
        return relaunch(args.gpus)
    if world != args.gpus:
        raise SystemExit(f"bench.py: --gpus {args.gpus} but WORLD_SIZE={world}: one rank per GPU required")
    if args.config == "size_sweep":
        if world > 1:
            raise SystemExit("--config size_sweep runs on one GPU")
        return run_size_sweep(args)
    if args.config in ("amr", "dmr_amr"):
        if world > 1:
            raise SystemExit(f"--config {args.config} runs on one GPU")
        return run_amr(args) if args.config == "amr" else run_dmr_amr(args)
    if world > 1:
        import torch
        import torch.distributed as dist
        os.environ.setdefault("NCCL_DEBUG", "INFO")        # INIT lines (transport, NVLS) on stderr
        os.environ.setdefault("NCCL_DEBUG_SUBSYS", "INIT")
        if torch.cuda.device_count() < world:
            raise SystemExit(f"bench.py: {world} ranks but {torch.cuda.device_count()} visible GPUs")
        torch.cuda.set_device(local_rank)
        dist.init_process_group("nccl", device_id=torch.device("cuda", local_rank))
    try:
        return run_crocco(args, rank, world, local_rank)
    finally:
        if world > 1:
            import torch.distributed as dist
            dist.destroy_process_group()


if __name__ == "__main__":
    sys.exit(main())
