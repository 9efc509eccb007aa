import sys, os
sys.path.insert(0, os.getcwd()); sys.path.insert(0, os.path.join(os.getcwd(), 'tests'))
import numpy as np, oracle, synth
from _harness import Problem, inner, rel_linf
c = synth.case("sod")
xyz = c.grid.coords(c.n_global, (0, 0, 0), oracle.GC)
pb = Problem(c.n_global, c.grid, c.bc, synth.sod(xyz), c.phys)
_, met, U = pb.oracle_inputs()
n = c.n_global
S = pb.solver()
V = np.zeros_like(U); dU = np.zeros_like(U)
ph = pb.oracle_phys()
a, o = U, V
for step in range(3):
    for s in range(3):
        oracle.rk_stage(n, c.bc, ph, s, c.dt, a, o, dU, met)
        a, o = o, a
        S.stage(s, c.dt); S.sync()
        g = pb.gather(S, S.get(S.U))
        gd = pb.gather(S, S.get(S.dU))
        e = np.abs(g - inner(a)); ed = np.abs(gd - inner(dU))
        idx = np.unravel_index(np.argmax(e), e.shape)
        print(step, s, "U err", e.max(), "at", idx, "dU err", ed.max(), np.unravel_index(np.argmax(ed), ed.shape), flush=True)
# also GPU full-padded U vs oracle after fill
