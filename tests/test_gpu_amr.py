"""GPU parity of the two-level AMR path (readings 24-26)
through the C ABI against the oracle (oracle section 9) on the same seeded inputs:
  FillPatchTwoLevels (C/F ghosts)   bitwise (dyadic weights, same corner order)
  AverageDown                       bitwise (same 27-term order, exact products)
  two-level RK3 steps               <= 1e-9 relative L_inf per component
for single- and multi-block coarse and fine levels, plus the ABI's refusals.
"""
import numpy as np
import pytest

import oracle
import synth
from _harness import block_slices, rel_linf, state_scale

pytestmark = pytest.mark.gpu

G = 4
CF = oracle.COARSE_FINE
PER = ((0, 0),) * 3


@pytest.fixture(autouse=True)
def _need_gpu():
    torch = pytest.importorskip("torch")
    if not torch.cuda.is_available():
        pytest.fail("GPU test run without a CUDA device")


def _blocks_of(a_glob_padded, n, nb):
    """Per-block padded views (ghost 4) cut out of a global padded array."""
    bn, blocks = block_slices(n, nb)
    out = []
    for o, _ in blocks:
        out.append(a_glob_padded[:, o[2]:o[2] + bn[2] + 2 * G, o[1]:o[1] + bn[1] + 2 * G,
                                 o[0]:o[0] + bn[0] + 2 * G])
    return bn, blocks, out


class Hier:
    """One two-level problem, built identically for the oracle (global single boxes) and the GPU
    (any block decomposition of either level)."""

    def __init__(self, nc, c0, nf, bcf, grid, phys_kw, seed=3, state="random", bcc=PER):
        self.nc, self.c0, self.nf, self.bcf, self.grid, self.bcc = nc, c0, nf, bcf, grid, bcc
        self.phys_kw = phys_kw
        self.fgrid = synth.Refined(grid, c0)
        if callable(state):
            self.Uc0 = state(grid.coords(nc, (0, 0, 0), oracle.GC))
            self.Uf0 = state(self.fgrid.coords(nf, (0, 0, 0), oracle.GC))
        elif state == "random":
            self.Uc0 = synth.random_state(nc, seed=seed, amp=0.2)
            self.Uf0 = synth.random_state(nf, seed=seed + 1, amp=0.2)
        else:
            self.Uc0 = synth.vortex(grid.coords(nc, (0, 0, 0), oracle.GC))
            self.Uf0 = synth.vortex(self.fgrid.coords(nf, (0, 0, 0), oracle.GC))

    def oracle(self):
        xc = self.grid.coords(self.nc, (0, 0, 0), oracle.GC)
        xf = self.fgrid.coords(self.nf, (0, 0, 0), oracle.GC)
        metc = oracle.metrics(self.nc, self.bcc, xc)
        metf = oracle.metrics(self.nf, self.bcf, xf)
        Uc = synth.pad_state(self.Uc0)
        Uf = synth.pad_state(self.Uf0)
        oracle.fill(self.nc, self.bcc, Uc)
        return metc, Uc, metf, Uf

    def gpu(self, nbc, nbf):
        from paper_conf_ipps_davissngmb23_b200 import crocco as cc
        from paper_conf_ipps_davissngmb23_b200.solver import AmrSolver, Solver
        kw = dict(self.phys_kw)
        C = Solver(self.nc, nbc, self.bcc, cc.make_phys(**kw))
        F = Solver(self.nf, nbf, self.bcf, cc.make_phys(**kw))
        for S, n, nb, g, U0 in ((C, self.nc, nbc, self.grid, self.Uc0), (F, self.nf, nbf, self.fgrid, self.Uf0)):
            bn, blocks = block_slices(n, nb)
            S.set_coords([g.coords(bn, o, oracle.GC) for o, _ in blocks])
            S.set_state([np.ascontiguousarray(U0[(slice(None),) + sl]) for _, sl in blocks])
            S.blocks = blocks
        C.fill()
        return C, F, AmrSolver(C, F, self.c0)


def _check_padded(S, bufs, ref_glob, n, nb, exact=True, tol=0.0, floor=0.0):
    bn, blocks, refs = _blocks_of(ref_glob, n, nb)
    got = S.get(bufs)
    for g, r in zip(got, refs):
        if exact:
            assert np.array_equal(g, r)
        else:
            assert rel_linf(g[:, G:-G, G:-G, G:-G], r[:, G:-G, G:-G, G:-G], floor) <= tol


@pytest.mark.parametrize("nbc,nbf,nf", [((1, 1, 1), (1, 1, 1), (20, 16, 12)), ((2, 2, 2), (2, 2, 1), (20, 16, 12)),
                                        ((3, 1, 2), (1, 2, 3), (20, 16, 12)), ((2, 2, 1), (1, 1, 1), (17, 13, 11))])
def test_fill_patch_two_levels_bitwise(nbc, nbf, nf):
    nc, c0 = (24, 20, 16), (3, 4, 2)
    h = Hier(nc, c0, nf, ((CF, CF),) * 3, synth.Wavy3D(L=(10.0,) * 3, N=nc), dict(terms=3, mu_ref=0.02))
    metc, Uc, metf, Uf = h.oracle()
    oracle.fill_two_levels(nf, h.bcf, Uf, nc, c0, Uc)
    C, F, A = h.gpu(nbc, nbf)
    A.fill_fine()
    _check_padded(F, F.U, Uf, nf, nbf)                    # interior, inter-block and C/F ghosts
    C.close()
    F.close()


def test_fill_patch_two_levels_mixed_faces_bitwise():
    """Fine level spanning the periodic zeta direction (PERIODIC) and touching the xi-lo domain
    boundary (EXTRAP there), C/F elsewhere."""
    nc, c0 = (20, 16, 8), (0, 3, 0)
    nf = (24, 16, 16)
    bcf = ((1, CF), (CF, CF), (0, 0))
    h = Hier(nc, c0, nf, bcf, synth.Wavy3D(L=(10.0,) * 3, N=nc), dict(terms=3, mu_ref=0.02))
    metc, Uc, metf, Uf = h.oracle()
    oracle.fill_two_levels(nf, bcf, Uf, nc, c0, Uc)
    C, F, A = h.gpu((2, 2, 2), (2, 2, 2))
    A.fill_fine()
    _check_padded(F, F.U, Uf, nf, (2, 2, 2))
    C.close()
    F.close()


@pytest.mark.parametrize("bcf,nf,c0,nbf", [(((CF, CF),) * 3, (18, 14, 12), (2, 3, 1), (2, 1, 2)),
                                           (((CF, CF), (CF, CF), (0, 0)), (18, 14, 16), (2, 3, 0), (2, 1, 2)),
                                           (((CF, CF),) * 3, (17, 13, 12), (3, 2, 1), (1, 1, 3))])
def test_average_down_bitwise(bcf, nf, c0, nbf):
    nc = (16, 12, 8)
    h = Hier(nc, c0, nf, bcf, synth.Wavy3D(L=(10.0,) * 3, N=nc), dict(terms=3, mu_ref=0.02))
    metc, Uc, metf, Uf = h.oracle()
    oracle.average_down(nf, bcf, Uf, nc, c0, Uc)
    C, F, A = h.gpu((2, 2, 1), nbf)
    A.average_down()
    bn, blocks, refs = _blocks_of(Uc, nc, (2, 2, 1))
    for g, r in zip(C.get(C.U), refs):
        assert np.array_equal(g[:, G:-G, G:-G, G:-G], r[:, G:-G, G:-G, G:-G])
    C.close()
    F.close()


@pytest.mark.parametrize("nbc,nbf,state", [((1, 1, 1), (1, 1, 1), "vortex"), ((2, 2, 1), (2, 1, 2), "random")])
def test_two_level_rk3_parity(nbc, nbf, state):
    nc, c0, nf = (24, 24, 16), (5, 6, 3), (24, 20, 16)
    bcf = ((CF, CF),) * 3
    h = Hier(nc, c0, nf, bcf, synth.Wavy3D(L=(10.0,) * 3, N=nc), dict(terms=3, mu_ref=0.01),
             state=state)
    metc, Uc, metf, Uf = h.oracle()
    dt, nsteps = 0.01, 10
    oracle.amr_advance(nc, PER, nf, bcf, c0, oracle.phys(terms=3, mu_ref=0.01), dt, nsteps, Uc, metc, Uf, metf)
    C, F, A = h.gpu(nbc, nbf)
    A.step(dt, nsteps)
    A.sync()
    for S, n, nb, ref in ((C, nc, nbc, Uc), (F, nf, nbf, Uf)):
        bn, blocks, refs = _blocks_of(ref, n, nb)
        for g, r in zip(S.get(S.U), refs):
            ri = r[:, G:-G, G:-G, G:-G]
            assert rel_linf(g[:, G:-G, G:-G, G:-G], ri, state_scale(ri)) <= 1e-9
    C.close()
    F.close()


def test_two_level_ramp_wall_parity():
    """Compression-ramp flow (walls, Sutherland, Mach 6) with a fine level on the no-slip wall:
    eta-lo WALL on both levels, zeta spanned periodically, xi and eta-hi C/F; multi-block levels."""
    E, W = 1, 3
    nc = (64, 32, 16)
    grid = synth.Ramp(N=nc)
    bcc = ((E, E), (W, E), (0, 0))
    c0, nf = (16, 0, 0), (40, 32, 32)
    bcf = ((CF, CF), (W, CF), (0, 0))
    phys = dict(gamma=1.4, R=1.0, Pr=0.72, mu_law=1, mu_ref=1e-3, T_ref=1.0, S=0.3, terms=3)
    h = Hier(nc, c0, nf, bcf, grid, phys, state=lambda x: synth.ramp_state(x, grid), bcc=bcc)
    metc, Uc, metf, Uf = h.oracle()
    dt, nsteps = 2e-4, 5
    oracle.amr_advance(nc, bcc, nf, bcf, c0, oracle.phys(**phys), dt, nsteps, Uc, metc, Uf, metf)
    C, F, A = h.gpu((2, 2, 1), (2, 2, 2))
    A.step(dt, nsteps)
    A.sync()
    for S, n, nb, ref in ((C, nc, (2, 2, 1), Uc), (F, nf, (2, 2, 2), Uf)):
        bn, blocks, refs = _blocks_of(ref, n, nb)
        for g, r in zip(S.get(S.U), refs):
            ri = r[:, G:-G, G:-G, G:-G]
            assert rel_linf(g[:, G:-G, G:-G, G:-G], ri, state_scale(ri)) <= 1e-9
    C.close()
    F.close()


@pytest.mark.slow
def test_full_size_amr_bench_config_bitwise():
    """bench.py --config amr at full size and in its launch configuration: 256^3 coarse TGV level,
    256^3-node fine level at c0 = (64, 64, 64), C/F faces all round.  Every fine ghost after
    FillPatchTwoLevels and every coarse interior point after AverageDown equal the oracle's."""
    import math
    nc, c0, nf = (256, 256, 256), (64, 64, 64), (256, 256, 256)
    grid = synth.Wavy3D(L=(2 * math.pi,) * 3, N=nc, x0=(-math.pi,) * 3, k=2.0, A=0.15)
    phys = dict(gamma=1.4, R=1.0, Pr=0.71, mu_ref=1.0 / 1600.0, terms=3)
    tgv = lambda x: synth.tgv(x, noise=0.01, seed=5)
    h = Hier(nc, c0, nf, ((CF, CF),) * 3, grid, phys, state=tgv)
    C, F, A = h.gpu((1, 1, 1), (1, 1, 1))
    Uc = synth.pad_state(h.Uc0)
    oracle.fill(nc, PER, Uc)
    Uf = synth.pad_state(h.Uf0)
    oracle.fill_two_levels(nf, h.bcf, Uf, nc, c0, Uc)
    A.fill_fine()
    assert np.array_equal(F.get(F.U)[0], Uf)
    oracle.average_down(nf, h.bcf, Uf, nc, c0, Uc)
    A.average_down()
    assert np.array_equal(C.get(C.U)[0][:, G:-G, G:-G, G:-G], Uc[:, G:-G, G:-G, G:-G])
    C.close()
    F.close()


def test_two_disjoint_fine_patches_parity():
    """Same-level multi-patch (NEXT-4): two disjoint fine patches on one coarse level, each its
    own ctx.  Reference: the pinned oracle functions composed in Algorithm 2's order (per stage
    the coarse stage, then every patch's FillPatchTwoLevels + RHS + update, AverageDown of every
    patch at the third stage)."""
    from paper_conf_ipps_davissngmb23_b200 import crocco as cc
    from paper_conf_ipps_davissngmb23_b200.solver import AmrSolver, Solver
    nc = (32, 24, 16)
    grid = synth.Wavy3D(L=(10.0,) * 3, N=nc)
    phys = dict(terms=3, mu_ref=0.01)
    ph = oracle.phys(**phys)
    patches = [((2, 3, 2), (16, 16, 12), (1, 1, 1)), ((18, 6, 3), (20, 24, 16), (2, 2, 1))]
    bcf = ((CF, CF),) * 3
    st = lambda x: synth.vortex(x)
    xc = grid.coords(nc, (0, 0, 0), oracle.GC)
    metc = oracle.metrics(nc, PER, xc)
    Uc = synth.pad_state(st(xc))
    P = []
    for c0, nf, _ in patches:
        xf = synth.Refined(grid, c0).coords(nf, (0, 0, 0), oracle.GC)
        P.append([c0, nf, oracle.metrics(nf, bcf, xf), synth.pad_state(st(xf))])
    dt, nsteps = 0.01, 4
    # oracle reference (composition of pinned functions, Alg. 2 order)
    Vc, dUc = Uc.copy(), np.zeros_like(Uc)
    ref = [[U.copy(), U.copy(), np.zeros_like(U)] for _, _, _, U in P]   # a, o, dU
    ac, oc = Uc.copy(), Vc
    for _ in range(nsteps):
        for s in range(3):
            oracle.rk_stage(nc, PER, ph, s, dt, ac, oc, dUc, metc)
            for (c0, nf, metf, _), R in zip(P, ref):
                oracle.fill_two_levels(nf, bcf, R[0], nc, c0, ac)
                r = oracle.rhs(nf, ph, R[0], metf)
                oracle.rk_update(nf, s, dt, R[0], R[1], R[2], r)
                if s == 2:
                    oracle.average_down(nf, bcf, R[1], nc, c0, oc)
                R[0], R[1] = R[1], R[0]
            ac, oc = oc, ac
    # GPU
    C = Solver(nc, (2, 2, 1), PER, cc.make_phys(**phys))
    bn, blocks = block_slices(nc, (2, 2, 1))
    C.set_coords([grid.coords(bn, o, oracle.GC) for o, _ in blocks])
    C.set_state([np.ascontiguousarray(st(xc)[(slice(None),) + sl]) for _, sl in blocks])
    Fs = []
    for (c0, nf, nb), (_, _, _, U0) in zip(patches, P):
        F = Solver(nf, nb, bcf, cc.make_phys(**phys))
        bnf, bl = block_slices(nf, nb)
        F.set_coords([synth.Refined(grid, c0).coords(bnf, o, oracle.GC) for o, _ in bl])
        Ui = U0[:, G:-G, G:-G, G:-G]
        F.set_state([np.ascontiguousarray(Ui[(slice(None),) + sl]) for _, sl in bl])
        Fs.append(F)
    A = AmrSolver(C, Fs, [p[0] for p in patches])
    A.step(dt, nsteps)
    A.sync()
    for S, n, nb, r in [(C, nc, (2, 2, 1), ac)] + [(F, p[1], p[2], R[0]) for F, p, R in zip(Fs, patches, ref)]:
        _, _, refs = _blocks_of(r, n, nb)
        for g, rr in zip(S.get(S.U), refs):
            ri = rr[:, G:-G, G:-G, G:-G]
            assert rel_linf(g[:, G:-G, G:-G, G:-G], ri, state_scale(ri)) <= 1e-9
    with pytest.raises(ValueError):               # patches with overlapping interiors
        AmrSolver(C, Fs, [(2, 3, 2), (9, 6, 3)])
    C.close()
    for F in Fs:
        F.close()


def test_three_level_hierarchy_parity():
    """Three levels (the paper's DMR runs three-level AMR): level 2 is a patch of
    level 1, which is a patch of level 0.  Reference: the pinned oracle functions composed in
    Algorithm 2's literal order (reading 29): per stage, level by level, FillPatch + RHS + update,
    and at the third stage AverageDown of level n onto n-1 right after level n's update."""
    from paper_conf_ipps_davissngmb23_b200 import crocco as cc
    from paper_conf_ipps_davissngmb23_b200.solver import AmrHierarchy, Solver
    n0 = (24, 24, 16)
    g0 = synth.Wavy3D(L=(10.0,) * 3, N=n0)
    c01, n1 = (4, 5, 2), (28, 24, 20)           # level 1 in level-0 index space
    c12, n2 = (6, 4, 5), (24, 24, 16)           # level 2 in level-1 index space
    g1 = synth.Refined(g0, c01)
    g2 = synth.Refined(g1, c12)
    bcf = ((CF, CF),) * 3
    phys = dict(terms=3, mu_ref=0.01)
    ph = oracle.phys(**phys)
    st = lambda x: synth.vortex(x)
    lv = []
    for n, g, bc in ((n0, g0, PER), (n1, g1, bcf), (n2, g2, bcf)):
        x = g.coords(n, (0, 0, 0), oracle.GC)
        lv.append([n, g, bc, oracle.metrics(n, bc, x), synth.pad_state(st(x))])
    oracle.fill(n0, PER, lv[0][4])
    dt, nsteps = 0.005, 3
    A = [L[4].copy() for L in lv]
    O = [L[4].copy() for L in lv]
    D = [np.zeros_like(L[4]) for L in lv]
    c0s = [None, c01, c12]
    for _ in range(nsteps):
        for s in range(3):
            for k in range(3):
                n, _, bc, met, _ = lv[k]
                if k == 0:
                    oracle.rk_stage(n, PER, ph, s, dt, A[0], O[0], D[0], met)
                else:
                    oracle.fill_two_levels(n, bc, A[k], lv[k - 1][0], c0s[k], A[k - 1])
                    r = oracle.rhs(n, ph, A[k], met)
                    oracle.rk_update(n, s, dt, A[k], O[k], D[k], r)
                    if s == 2:
                        oracle.average_down(n, bc, O[k], lv[k - 1][0], c0s[k], O[k - 1])
            for k in range(3):
                A[k], O[k] = O[k], A[k]
    # GPU (multi-block levels)
    nbs = [(2, 2, 1), (2, 1, 2), (1, 2, 1)]
    S = []
    for (n, g, bc, _, U0), nb in zip(lv, nbs):
        X = Solver(n, nb, bc, cc.make_phys(**phys))
        bn, bl = block_slices(n, nb)
        X.set_coords([g.coords(bn, o, oracle.GC) for o, _ in bl])
        Ui = U0[:, G:-G, G:-G, G:-G]
        X.set_state([np.ascontiguousarray(Ui[(slice(None),) + sl]) for _, sl in bl])
        S.append(X)
    H = AmrHierarchy(S[0], [[(S[1], 0, c01)], [(S[2], 0, c12)]])
    H.step(dt, nsteps)
    H.sync()
    for X, (n, *_), nb, ref in zip(S, lv, nbs, A):
        _, _, refs = _blocks_of(ref, n, nb)
        for gg, rr in zip(X.get(X.U), refs):
            ri = rr[:, G:-G, G:-G, G:-G]
            assert rel_linf(gg[:, G:-G, G:-G, G:-G], ri, state_scale(ri)) <= 1e-9
    for X in S:
        X.close()


def _dmr_hierarchy(scale, patches):
    """The paper's DMR with a three-level hierarchy: base grid of
    synth.case("dmr", scale), then patches (c0, nf, nblocks) of levels 1, 2 (each inside the
    previous one) with their boundary data from synth.refine_bc."""
    c = synth.case("dmr", scale=scale)
    n0 = c.n_global
    h = 1.0 / n0[1]
    bc0, dv0, sp0 = synth.dmr_bc(h)
    levels = [dict(n=n0, grid=c.grid, bc=bc0, dir=dv0, split=sp0, nb=c.n_blocks, c0=None)]
    for c0, nf, nb in patches:
        up = levels[-1]
        bcf, dvf, spf = synth.refine_bc(up["n"], up["bc"], up["dir"], up["split"], c0, nf)
        levels.append(dict(n=nf, grid=synth.Refined(up["grid"], c0), bc=bcf, dir=dvf, split=spf, nb=nb, c0=c0))
    return c, levels


@pytest.mark.parametrize("patches", [
    [((2, 0, 0), (128, 24, 16), (2, 1, 2)), ((4, 0, 0), (64, 16, 32), (1, 1, 2))],       # on the wall
    [((6, 16, 0), (96, 31, 16), (2, 1, 1)), ((20, 14, 0), (80, 33, 32), (1, 1, 2))],     # under the moving top
])
def test_three_level_dmr_parity(patches):
    """DMR with three levels on the GPU (SLIPWALL and the static / moving SPLIT faces of the bottom /
    top boundary on the fine patches that touch them, C/F faces elsewhere) against the oracle
    functions composed in Alg. 2's order."""
    from paper_conf_ipps_davissngmb23_b200 import crocco as cc
    from paper_conf_ipps_davissngmb23_b200.solver import AmrHierarchy, Solver
    c, L = _dmr_hierarchy(16, patches)
    ph = oracle.phys(**c.phys)
    h2 = 1.0 / c.n_global[1] / 4
    dt, nsteps = 0.2 * h2 / 13.0, 4
    for lv in L:
        x = lv["grid"].coords(lv["n"], (0, 0, 0), oracle.GC)
        lv["met"] = oracle.metrics(lv["n"], lv["bc"], x)
        lv["U0"] = synth.dmr_state(x)
        lv["sp"] = oracle.splits(lv["split"])
    A = [synth.pad_state(lv["U0"]) for lv in L]
    O = [a.copy() for a in A]
    D = [np.zeros_like(a) for a in A]
    t = 0.0
    for _ in range(nsteps):
        for s in range(3):
            ts = t + (0.0, 1.0 / 3.0, 3.0 / 4.0)[s] * dt
            for k, lv in enumerate(L):
                if k == 0:
                    oracle.rk_stage(lv["n"], lv["bc"], ph, s, dt, A[0], O[0], D[0], lv["met"],
                                    dirichlet=lv["dir"], split=lv["sp"], t=t)
                else:
                    oracle.fill_two_levels(lv["n"], lv["bc"], A[k], L[k - 1]["n"], lv["c0"], A[k - 1],
                                           dirichlet=lv["dir"], met=lv["met"], split=lv["sp"], t=ts)
                    r = oracle.rhs(lv["n"], ph, A[k], lv["met"])
                    oracle.rk_update(lv["n"], s, dt, A[k], O[k], D[k], r)
                    if s == 2:
                        oracle.average_down(lv["n"], lv["bc"], O[k], L[k - 1]["n"], lv["c0"], O[k - 1])
            for k in range(len(L)):
                A[k], O[k] = O[k], A[k]
        t = t + dt
    S = []
    for lv in L:
        X = Solver(lv["n"], lv["nb"], lv["bc"], cc.make_phys(**c.phys), dirichlet=lv["dir"], split=lv["split"])
        bn, bl = block_slices(lv["n"], lv["nb"])
        X.set_coords([lv["grid"].coords(bn, o, oracle.GC) for o, _ in bl])
        X.set_state([np.ascontiguousarray(lv["U0"][(slice(None),) + sl]) for _, sl in bl])
        S.append(X)
    H = AmrHierarchy(S[0], [[(S[1], 0, L[1]["c0"])], [(S[2], 0, L[2]["c0"])]])
    # ComputeDt over the hierarchy = min over levels (the finest level binds: spacing h/4)
    dts = [oracle.compute_dt(lv["n"], ph, synth.pad_state(lv["U0"]), lv["met"], 0.5) for lv in L]
    assert abs(H.compute_dt(0.5) - min(dts)) <= 1e-13 * min(dts)
    assert min(dts) == dts[2]
    H.step(dt, nsteps)
    H.sync()
    for X, lv, ref in zip(S, L, A):
        _, _, refs = _blocks_of(ref, lv["n"], lv["nb"])
        for gg, rr in zip(X.get(X.U), refs):
            ri = rr[:, G:-G, G:-G, G:-G]
            assert rel_linf(gg[:, G:-G, G:-G, G:-G], ri, state_scale(ri)) <= 1e-9
        assert X.check_state() == 0
    for X in S:
        X.close()


def test_two_level_overlapped_stage_equals_serial_bitwise():
    """The fine level's C/F interpolation also runs inside the overlapped stage (fill on the
    comm stream beside the ghost-free viscous tiles): forcing the overlap on gives the serial
    result bit for bit."""
    from paper_conf_ipps_davissngmb23_b200 import crocco as cc
    nc, c0, nf = (48, 24, 80), (4, 5, 2), (72, 20, 136)   # fine level has ghost-free viscous tiles
    outs = []
    for ov in (0, 1):
        h = Hier(nc, c0, nf, ((CF, CF),) * 3, synth.Wavy3D(L=(10.0,) * 3, N=nc), dict(terms=3, mu_ref=0.01),
                 state="vortex")
        C, F, A = h.gpu((1, 1, 1), (1, 1, 1))
        cc.crocco_set_overlap(F.ctx, ov)
        cc.crocco_set_overlap(C.ctx, ov)
        A.step(0.005, 2)
        A.sync()
        assert cc.crocco_overlap_count(F.ctx) == (6 if ov else 0)
        outs.append([C.get(C.U)[0], F.get(F.U)[0]])
        C.close()
        F.close()
    assert np.array_equal(outs[0][0], outs[1][0]) and np.array_equal(outs[0][1], outs[1][1])


@pytest.mark.parametrize("nbc,nbf,c0,nf,bcf", [
    ((1, 1, 1), (1, 1, 1), (5, 6, 3), (24, 20, 16), ((CF, CF),) * 3),
    ((2, 2, 1), (2, 1, 2), (5, 6, 3), (24, 20, 16), ((CF, CF),) * 3),
    ((2, 1, 2), (2, 2, 1), (0, 4, 3), (48, 20, 16), ((0, 0), (CF, CF), (CF, CF)))])
def test_inter_level_boxes_through_nccl_loopback_bitwise(nbc, nbf, c0, nf, bcf):
    """Multi-rank AMR on one GPU (each level decomposed on its own; include/
    crocco.h crocco_amr_plan): with the NCCL loopback on the fine ctx every inter-level box --
    the coarse corners of the C/F interpolation into the coarse-block mirrors, the averaged
    coarse nodes back from the mirrors -- goes pack -> ncclSend/ncclRecv -> unpack, the code a
    fine block on another rank than its coarse footprint runs.  3 RK3 steps are bitwise those of
    the in-place path, which the oracle pins (test_two_level_rk3_parity)."""
    from paper_conf_ipps_davissngmb23_b200 import crocco as cc
    nc = (24, 24, 16)
    outs = []
    for lb in (0, 1):
        h = Hier(nc, c0, nf, bcf, synth.Wavy3D(L=(10.0,) * 3, N=nc), dict(terms=3, mu_ref=0.01), state="random")
        C, F, A = h.gpu(nbc, nbf)
        if lb:
            cc.crocco_set_nccl_loopback(F.ctx, 1)
        s0 = cc.crocco_scratch_bytes(F.ctx)
        A.step(0.01, 3)
        A.sync()
        if lb:   # the coarse-block mirrors and the AMR staging were allocated by the exchange
            assert cc.crocco_scratch_bytes(F.ctx) > s0
        outs.append([C.get(C.U), F.get(F.U)])
        C.close()
        F.close()
    for a, b in zip(outs[0], outs[1]):
        for x, y in zip(a, b):
            assert np.array_equal(x, y)


def test_amr_abi_refusals():
    from paper_conf_ipps_davissngmb23_b200 import crocco as cc
    from paper_conf_ipps_davissngmb23_b200.solver import AmrSolver, Solver
    nc = (16, 16, 16)
    grid = synth.Wavy3D(L=(10.0,) * 3, N=nc)
    C = Solver(nc, (1, 1, 1), PER)
    F = Solver((12, 12, 12), (1, 1, 1), ((CF, CF),) * 3)
    for S, g, n in ((C, grid, nc), (F, synth.Refined(grid, (2, 2, 2)), (12, 12, 12))):
        S.set_coords([g.coords(n, (0, 0, 0), oracle.GC)])
        S.set_state([synth.random_state(n, seed=1)])
    with pytest.raises(cc.CroccoError):          # C/F faces without a coarse level
        F.stage(0, 0.01)
    with pytest.raises(cc.CroccoError):          # RK3 graph step on a fine level
        F.step(0.01)
    with pytest.raises(cc.CroccoError):          # fine level leaves the coarse domain
        AmrSolver(C, F, (10, 2, 2))
    with pytest.raises(cc.CroccoError):          # periodic fine level must span the domain
        F2 = Solver((16, 16, 16), (1, 1, 1), PER)
        try:
            AmrSolver(C, F2, (0, 0, 0))
        finally:
            F2.close()
    A = AmrSolver(C, F, (2, 2, 2))
    C.fill()
    A.step(0.01, 1)
    A.sync()
    C.close()
    F.close()


def _gpu_level(nc, grid, nbc, specs, state, phys):
    from paper_conf_ipps_davissngmb23_b200 import crocco as cc
    from paper_conf_ipps_davissngmb23_b200.solver import AmrSolver, Solver
    bcf = ((CF, CF),) * 3
    xc = grid.coords(nc, (0, 0, 0), oracle.GC)
    C = Solver(nc, nbc, PER, cc.make_phys(**phys))
    bn, blocks = block_slices(nc, nbc)
    C.set_coords([grid.coords(bn, o, oracle.GC) for o, _ in blocks])
    C.set_state([np.ascontiguousarray(state(xc)[(slice(None),) + sl]) for _, sl in blocks])
    Fs = []
    for c0, nf, nb in specs:
        F = Solver(nf, nb, bcf, cc.make_phys(**phys))
        bnf, bl = block_slices(nf, nb)
        xf = synth.Refined(grid, c0).coords(nf, (0, 0, 0), oracle.GC)
        F.set_coords([synth.Refined(grid, c0).coords(bnf, o, oracle.GC) for o, _ in bl])
        U0 = state(xf)
        F.set_state([np.ascontiguousarray(U0[(slice(None),) + sl]) for _, sl in bl])
        Fs.append(F)
    return C, Fs, AmrSolver(C, Fs, [s[0] for s in specs])


@pytest.mark.parametrize("axis", [0, 1])
def test_abutting_patches_parity_and_union(axis):
    """NEXT-4 completion (reading 31): two abutting fine patches of one level,
    siblings exchanging their ghosts (crocco_amr_rk_stage_level / crocco_average_down_level),
    multi-block on both levels.  (a) parity <= 1e-9 with the oracle functions composed in
    Algorithm 2's order (tests/test_oracle_amr.py advance_level) after 3 RK3 steps; (b) bitwise
    equal to the GPU run of the single patch covering their union."""
    from test_oracle_amr import advance_level, _level_setup
    nc = (24, 20, 16)
    grid = synth.Wavy3D(L=(10.0,) * 3, N=nc)
    phys = dict(terms=3, mu_ref=0.01)
    c0, nu = (3, 4, 2), [24, 16, 12]
    half = [nu[d] // 2 if d == axis else nu[d] for d in range(3)]
    c0b = tuple(c0[d] + (half[d] // 2 if d == axis else 0) for d in range(3))
    st = lambda x: synth.vortex(x)
    specs = [(c0, tuple(half), (2, 1, 1) if axis == 1 else (1, 2, 1)), (c0b, tuple(half), (1, 1, 2))]
    dt, nsteps = 0.01, 3
    metc, Uc, P = _level_setup(nc, grid, [(s[0], s[1]) for s in specs], st)
    advance_level(nc, metc, Uc, P, oracle.phys(**phys), dt, nsteps)
    C, Fs, A = _gpu_level(nc, grid, (2, 1, 1), specs, st, phys)
    assert A.sibs == [[1], [0]]
    A.step(dt, nsteps)
    A.sync()
    _, _, refs = _blocks_of(Uc, nc, (2, 1, 1))
    for g, rr in zip(C.get(C.U), refs):
        ri = rr[:, G:-G, G:-G, G:-G]
        assert rel_linf(g[:, G:-G, G:-G, G:-G], ri, state_scale(ri)) <= 1e-9
    got_parts = []
    for F, (c0p, nf, nb), p in zip(Fs, specs, P):
        _, _, refs = _blocks_of(p["U"], nf, nb)
        gl = F.get(F.U)
        for g, rr in zip(gl, refs):
            ri = rr[:, G:-G, G:-G, G:-G]
            assert rel_linf(g[:, G:-G, G:-G, G:-G], ri, state_scale(ri)) <= 1e-9
        glob = np.zeros((5, nf[2], nf[1], nf[0]))
        bnf, bl = block_slices(nf, nb)
        for (o, sl), g in zip(bl, gl):
            glob[(slice(None),) + sl] = g[:, G:-G, G:-G, G:-G]
        got_parts.append(glob)
    coarse_two = [g.copy() for g in C.get(C.U)]
    for S in [C] + Fs:
        S.close()
    # the union patch on the GPU
    Cu, Fu, Au = _gpu_level(nc, grid, (2, 1, 1), [(c0, tuple(nu), (1, 1, 1))], st, phys)
    Au.step(dt, nsteps)
    Au.sync()
    union = Fu[0].get(Fu[0].U)[0][:, G:-G, G:-G, G:-G]
    assert np.array_equal(np.concatenate(got_parts, axis=3 - axis), union)
    for a, b in zip(coarse_two, Cu.get(Cu.U)):
        assert np.array_equal(a, b)
    for S in [Cu] + Fu:
        S.close()


@pytest.mark.parametrize("axis", [0, 1])
def test_sibling_boxes_through_nccl_loopback_bitwise(axis):
    """Sibling patches on different ranks (include/crocco.h crocco_amr_link_sibling, kind-2 boxes
    of crocco_amr_sibling_plan) on one GPU: with the NCCL loopback on both patch ctx every
    sibling ghost box and every inter-level box goes pack -> ncclSend/ncclRecv -> unpack into the
    mirrors; 3 RK3 steps of two abutting multi-block patches are bitwise those of the in-place
    run, which test_abutting_patches_parity_and_union pins to the oracle and to the union patch."""
    from paper_conf_ipps_davissngmb23_b200 import crocco as cc
    nc = (24, 20, 16)
    grid = synth.Wavy3D(L=(10.0,) * 3, N=nc)
    phys = dict(terms=3, mu_ref=0.01)
    c0, nu = (3, 4, 2), [24, 16, 12]
    half = [nu[d] // 2 if d == axis else nu[d] for d in range(3)]
    c0b = tuple(c0[d] + (half[d] // 2 if d == axis else 0) for d in range(3))
    specs = [(c0, tuple(half), (2, 1, 1) if axis == 1 else (1, 2, 1)), (c0b, tuple(half), (1, 1, 2))]
    outs = []
    for lb in (0, 1):
        C, Fs, A = _gpu_level(nc, grid, (2, 1, 1), specs, lambda x: synth.vortex(x), phys)
        assert A.sibs == [[1], [0]]
        if lb:
            for F in Fs:
                cc.crocco_set_nccl_loopback(F.ctx, 1)
        s0 = [cc.crocco_scratch_bytes(F.ctx) for F in Fs]
        A.step(0.01, 3)
        A.sync()
        if lb:
            assert all(cc.crocco_scratch_bytes(F.ctx) > s for F, s in zip(Fs, s0))
        outs.append([C.get(C.U)] + [F.get(F.U) for F in Fs])
        for S in [C] + Fs:
            S.close()
    for a, b in zip(outs[0], outs[1]):
        for x, y in zip(a, b):
            assert np.array_equal(x, y)


def test_three_level_hierarchy_through_nccl_loopback_bitwise():
    """Every inter-level box of a three-level hierarchy (level 1 is the fine level of level 0 and
    the coarse level of level 2) through ncclSend/ncclRecv to self: 2 RK3 steps bitwise equal to
    the in-place run (which test_three_level_hierarchy_parity pins to the oracle)."""
    from paper_conf_ipps_davissngmb23_b200 import crocco as cc
    from paper_conf_ipps_davissngmb23_b200.solver import AmrHierarchy, Solver
    n0 = (24, 24, 16)
    g0 = synth.Wavy3D(L=(10.0,) * 3, N=n0)
    c01, n1 = (4, 5, 2), (28, 24, 20)
    c12, n2 = (6, 4, 5), (24, 24, 16)
    g1 = synth.Refined(g0, c01)
    g2 = synth.Refined(g1, c12)
    bcf = ((CF, CF),) * 3
    phys = dict(terms=3, mu_ref=0.01)
    outs = []
    for lb in (0, 1):
        S = []
        for n, g, bc, nb in ((n0, g0, PER, (2, 2, 1)), (n1, g1, bcf, (2, 1, 2)), (n2, g2, bcf, (1, 2, 1))):
            X = Solver(n, nb, bc, cc.make_phys(**phys))
            bn, bl = block_slices(n, nb)
            X.set_coords([g.coords(bn, o, oracle.GC) for o, _ in bl])
            x = g.coords(n, (0, 0, 0), oracle.GC)
            U0 = synth.vortex(x)
            X.set_state([np.ascontiguousarray(U0[(slice(None),) + sl]) for _, sl in bl])
            S.append(X)
        H = AmrHierarchy(S[0], [[(S[1], 0, c01)], [(S[2], 0, c12)]])
        if lb:
            cc.crocco_set_nccl_loopback(S[1].ctx, 1)
            cc.crocco_set_nccl_loopback(S[2].ctx, 1)
        H.step(0.005, 2)
        H.sync()
        outs.append([X.get(X.U) for X in S])
        for X in S:
            X.close()
    for a, b in zip(outs[0], outs[1]):
        for x, y in zip(a, b):
            assert np.array_equal(x, y)
