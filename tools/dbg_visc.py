import sys, os
sys.path.insert(0, os.getcwd()); sys.path.insert(0, os.path.join(os.getcwd(), "tests"))
import numpy as np, synth, oracle
from _harness import Problem
n = (24, 20, 16)
g = synth.Wavy3D(L=(10.0,) * 3, N=n)
pb = Problem(n, g, ((0, 0),) * 3, synth.random_state(n, seed=2, amp=0.2), dict(terms=int(sys.argv[1]), mu_ref=0.02))
S = pb.solver()
S.fill()
r = S.rhs()
S.sync()
print("ok")
