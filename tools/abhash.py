"""Bitwise A/B check of two libcrocco builds (CROCCO_LIB): hash of the state after one RK3
step of the weak recipe at AB_N^3 (blocks AB_NB) with viscous terms.  Tool, not a test."""
import hashlib, json, math, os, sys
sys.path.insert(0, os.getcwd())
import numpy as np, torch
import synth
from paper_conf_ipps_davissngmb23_b200 import crocco as cc
from paper_conf_ipps_davissngmb23_b200.solver import Solver
N = int(os.environ.get("AB_N", "128"))
nb = tuple(int(x) for x in os.environ.get("AB_NB", "2,1,1").split(","))
n = (N, N, N)
grid = synth.Wavy3D(L=(2 * math.pi,) * 3, N=n, x0=(-math.pi,) * 3, k=2.0, A=0.15)
S = Solver(n, nb, ((0, 0),) * 3, cc.make_phys(gamma=1.4, R=1.0, Pr=0.71, mu_law=1, mu_ref=1 / 1600, T_ref=1.0, S=0.4))
cc.crocco_set_overlap(S.ctx, int(os.environ.get("AB_OVERLAP", "0")))
bn = tuple(n[d] // nb[d] for d in range(3))
xyz, U0 = [], []
for bz in range(nb[2]):
    for by in range(nb[1]):
        for bx in range(nb[0]):
            o = (bx * bn[0], by * bn[1], bz * bn[2])
            x = grid.coords(bn, o, 10)
            xyz.append(x)
            U0.append(synth.tgv(x, noise=0.01, seed=5))
S.set_coords(xyz); S.set_state(U0)
S.step(2e-4, 2)
S.sync()
h = hashlib.sha256()
for a in S.get(S.U):
    h.update(np.ascontiguousarray(a[:, 4:-4, 4:-4, 4:-4]).tobytes())
print(json.dumps({"lib": os.path.basename(cc.LIB_PATH), "N": N, "nb": nb, "hash": h.hexdigest()[:16]}))
