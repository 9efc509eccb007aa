"""Long run of the bench workload (512^3 periodic curvilinear TGV + noise, viscous) through the product
path: the discrete conservation of sum_i U_i / J_i (periodic, strong-conservation form: PAPER.md:48,
DESIGN reading 4) after many RK3 steps, the kinetic-energy decay of the TGV, the state check, and the
step rate.  Tool, not a test (no oracle involved)."""
import json, math, os, sys, time
sys.path.insert(0, os.getcwd())
import torch
import synth
from paper_conf_ipps_davissngmb23_b200 import crocco as cc
from paper_conf_ipps_davissngmb23_b200.solver import Solver

N = int(os.environ.get("LR_N", "512"))
STEPS = int(os.environ.get("LR_STEPS", "1000"))
n = (N, N, N)
grid = synth.Wavy3D(L=(2 * math.pi,) * 3, N=n, x0=(-math.pi,) * 3, k=2.0, A=0.15)
S = Solver(n, (1, 1, 1), ((0, 0),) * 3, cc.make_phys(gamma=1.4, R=1.0, Pr=0.71, mu_ref=1 / 1600, terms=3))
xyz = torch.from_numpy(grid.coords(n, (0, 0, 0), cc.GHOST_COORDS)).cuda()
S.set_coords([xyz]); S.set_state([synth.tgv(xyz, noise=0.01, seed=5)]); del xyz
G = cc.GHOST
iJ = 1.0 / S.view(S.met[0], 0, 1)[0, G:-G, G:-G, G:-G]  # metric comp 0 = J (crocco.h layout)


def totals():
    U = S.view(S.U[0], 0, 5)[:, G:-G, G:-G, G:-G]
    tot = [(U[c] * iJ).sum().item() for c in range(5)]
    mag = [(U[c].abs() * iJ).sum().item() for c in range(5)]
    ke = (0.5 * (U[1] ** 2 + U[2] ** 2 + U[3] ** 2) / U[0] * iJ).sum().item()
    return tot, mag, ke


dt = 2e-4
t0, m0, ke0 = totals()
torch.cuda.synchronize()
w0 = time.perf_counter()
kes = [ke0]
for k in range(STEPS // 100):
    S.step(dt, 100)
    kes.append(totals()[2])
torch.cuda.synchronize()
wall = time.perf_counter() - w0
t1, m1, ke1 = totals()
out = {"n": N, "steps": STEPS, "dt": dt, "t_end": STEPS * dt,
       "rel_drift_sum_U_over_J": [abs(a - b) / m for a, b, m in zip(t1, t0, m0)],
       "ke_every_100_steps": kes, "ke_monotone_decreasing": all(b <= a for a, b in zip(kes, kes[1:])),
       "bad_points": S.check_state(), "wall_s": wall, "pts_stage_per_s_wall": N ** 3 * 3 * STEPS / wall}
print(json.dumps(out), flush=True)
