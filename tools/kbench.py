"""Kernel-variant micro-benchmark: per-kernel-class CUDA-event times of RK stages on
the bench workload (CROCCO_LIB selects a variant .so).  Not a bench.py number."""
import json, math, os, sys, time
sys.path.insert(0, os.getcwd())
import torch
import synth
from paper_conf_ipps_davissngmb23_b200 import crocco as cc
from paper_conf_ipps_davissngmb23_b200.solver import Solver
N = int(os.environ.get("KB_N", "512"))
NB = tuple(int(x) for x in os.environ.get("KB_BLOCKS", "1,1,1").split(","))   # N^3 per block
n = (N * NB[0], N * NB[1], N * NB[2])
grid = synth.Wavy3D(L=(2 * math.pi * NB[0], 2 * math.pi * NB[1], 2 * math.pi * NB[2]), N=n, x0=(-math.pi,) * 3,
                    k=2.0, A=0.15)
S = Solver(n, NB, ((0, 0),) * 3, cc.make_phys(gamma=1.4, R=1.0, Pr=0.71, mu_ref=1 / 1600, terms=int(os.environ.get("KB_TERMS", "3")),
                                                  weno_limiter=int(os.environ.get("KB_LIM", "0")), weno_alpha_rl=5.0, weno_alpha_al=1e-4,
                                                  visc_form=int(os.environ.get("KB_VISC_FORM", "0"))))
cc.crocco_set_overlap(S.ctx, int(os.environ.get("KB_OVERLAP", "1")))
if int(os.environ.get("KB_LOOPBACK", "0")):   # same-rank copies through NCCL (multi-rank exchange code)
    cc.crocco_set_nccl_loopback(S.ctx, True)
for b in range(S.nloc):
    L = S.layouts[b]
    xyz = torch.from_numpy(grid.coords(tuple(L.n), tuple(L.origin), 10)).cuda()
    S.set_coords_block(b, xyz); S.set_state_block(b, synth.tgv(xyz, noise=0.01, seed=5)); del xyz
for s in range(3): S.stage(s, 2e-4)
torch.cuda.synchronize()
REPS = int(os.environ.get("KB_REPS", "3"))
best = None
best_k = {}
for rep in range(REPS):
    cc.crocco_set_timing(S.ctx, True); cc.crocco_kernel_times(S.ctx)
    e0 = torch.cuda.Event(enable_timing=True); e1 = torch.cuda.Event(enable_timing=True)
    e0.record()
    for it in range(2):
        for s in range(3): S.stage(s, 2e-4)
    e1.record(); torch.cuda.synchronize()
    kt = cc.crocco_kernel_times(S.ctx)
    tot = e0.elapsed_time(e1) / 6
    best = tot if best is None else min(best, tot)
    for k, v in kt.items():
        if v[0]:
            best_k[k] = min(best_k.get(k, 1e30), v[1] / v[0])
tot = best
out = {"lib": os.path.basename(cc.LIB_PATH), "overlap": os.environ.get("KB_OVERLAP", "1"), "loopback": os.environ.get("KB_LOOPBACK", "0"), "weno_limiter": os.environ.get("KB_LIM", "0"), "visc_form": os.environ.get("KB_VISC_FORM", "0"), "blocks": NB, "ms_per_stage": tot, "pts_stage_per_s": n[0] * n[1] * n[2] / tot * 1e3,
       "kernels_ms": {k: round(v, 3) for k, v in best_k.items()}}
out["finite"] = all(bool(torch.isfinite(S.view(S.U[b], b, 5)[:, 4:-4, 4:-4, 4:-4]).all().item()) for b in range(S.nloc))
print(json.dumps(out), flush=True)
