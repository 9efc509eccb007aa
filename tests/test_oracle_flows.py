"""Flow-level pins of the oracle RHS and time stepping against closed forms
and invariants (SURVEY 8(c) 'What pins each part').  CPU only; sized to run
in well under a minute each with the oracle's OpenMP threads.
"""
import math
import os

import numpy as np
import pytest

import oracle
import synth

GOLD = os.path.join(os.path.dirname(__file__), "golden")
G = 4
PER = ((0, 0),) * 3


def _inner(a):
    return a[:, G:-G, G:-G, G:-G]


def _setup(grid, n, bc, Ui):
    xyz = grid.coords(n, (0, 0, 0), oracle.GC)
    met = oracle.metrics(n, bc, xyz)
    U = synth.pad_state(Ui(xyz) if callable(Ui) else Ui)
    oracle.fill(n, bc, U)
    return xyz, met, U


def _flux_scale(U, met):
    """max_i J |m| max|F| -- the floor used where the exact RHS is ~0 (reading 17)."""
    J = _inner(met)[0]
    m = np.sqrt((_inner(met)[1:] ** 2).reshape(3, 3, *J.shape).sum(1)).max(0)
    Ui = _inner(U)
    rho = Ui[0]
    vel = Ui[1:4] / rho
    p = 0.4 * (Ui[4] - 0.5 * rho * (vel ** 2).sum(0))
    F = np.abs(Ui[1:4] * np.abs(vel).max(0)).max(0) + p + np.abs(Ui[4] + p) * np.abs(vel).max(0)
    return float((J * m * F).max())


# ------------------------------------------------------------------ free stream (reading 6)

@pytest.mark.parametrize("terms", [1, 3])
def test_free_stream_preserved_on_wavy_grid(terms):
    n = (20, 18, 16)
    grid = synth.Wavy3D(L=(10.0, 10.0, 10.0), N=n)
    xyz, met, U = _setup(grid, n, PER, synth.free_stream)
    ph = oracle.phys(terms=terms, mu_ref=0.05)
    r = oracle.rhs(n, ph, U, met)
    assert np.abs(_inner(r)).max() < 1e-13 * _flux_scale(U, met)


# ------------------------------------------------------------------ conservation (periodic)

@pytest.mark.parametrize("lim", [{}, dict(weno_limiter=3, weno_alpha_rl=5.0, weno_alpha_al=1e-3)])
def test_periodic_conservation_of_sum_U_over_J(lim):
    n = (16, 14, 12)
    grid = synth.Wavy3D(L=(10.0,) * 3, N=n)
    Ui = synth.random_state(n, seed=7, amp=0.2)
    xyz, met, U = _setup(grid, n, PER, Ui)
    ph = oracle.phys(terms=3, mu_law=1, mu_ref=0.02, S=0.5, **lim)
    r = _inner(oracle.rhs(n, ph, U, met))
    J = _inner(met)[0]
    tot = (r / J).reshape(5, -1).sum(1)
    mag = np.abs(r / J).reshape(5, -1).sum(1)
    assert np.all(np.abs(tot) < 1e-13 * mag), tot / mag


# ------------------------------------------------------------------ symmetries

def _smooth_random_state(n, seed):
    rng = np.random.default_rng(seed)
    i, j, k = np.meshgrid(*[np.arange(m) * 2 * np.pi / m for m in n], indexing="ij")
    f = lambda: sum(rng.uniform(-1, 1) * np.sin(a * i + b * j + c * k + rng.uniform(0, 6))
                    for a, b, c in rng.integers(0, 3, (3, 3)))
    rho = 1 + 0.2 * f()
    u, v, w = 0.3 * f(), 0.3 * f(), 0.3 * f()
    p = 0.8 + 0.2 * f()
    cons = synth.prim_to_cons(rho, u, v, w, p)
    return np.ascontiguousarray(cons.transpose(0, 3, 2, 1))  # (c, k, j, i)


def test_rhs_cyclic_axis_permutation():
    m = 12
    n = (m, m, m)
    grid = synth.Cartesian(h=(0.1,) * 3)
    Ui = _smooth_random_state(n, 3)
    # add a sharp feature so WENO weights are nonlinear
    Ui[0, :, :, 5:] *= 1.5
    Ui[4, :, :, 5:] *= 1.5
    ph = oracle.phys(terms=3, mu_ref=0.01)
    _, met, U = _setup(grid, n, PER, Ui)
    r = _inner(oracle.rhs(n, ph, U, met))
    # permutation: new(i,j,k) = old(j,k,i) i.e. new axis x = old y, new y = old z, new z = old x
    # array axes (k, j, i): new[k, j, i] = old[i, k, j]
    Up = Ui.transpose(0, 3, 1, 2).copy()
    Up[1:4] = Up[[2, 3, 1]]
    _, met2, U2 = _setup(grid, n, PER, np.ascontiguousarray(Up))
    r2 = _inner(oracle.rhs(n, ph, U2, met2))
    rp = r.transpose(0, 3, 1, 2).copy()
    rp[1:4] = rp[[2, 3, 1]]
    assert np.abs(r2 - rp).max() < 1e-12 * np.abs(r).max()


def test_rhs_mirror_symmetry():
    m = 12
    n = (m, 10, 8)
    grid = synth.Cartesian(h=(0.1,) * 3)
    Ui = _smooth_random_state(n, 4)
    Ui[0, :, :, 6:] *= 2.0
    ph = oracle.phys(terms=3, mu_ref=0.01)
    _, met, U = _setup(grid, n, PER, Ui)
    r = _inner(oracle.rhs(n, ph, U, met))
    # reflect i -> m-1-i (periodic), negate rho*u
    Um = Ui[:, :, :, ::-1].copy()
    Um[1] *= -1
    _, met2, U2 = _setup(grid, n, PER, np.ascontiguousarray(Um))
    r2 = _inner(oracle.rhs(n, ph, U2, met2))
    rm = r[:, :, :, ::-1].copy()
    rm[1] *= -1
    assert np.abs(r2 - rm).max() < 1e-12 * np.abs(r).max()


# ------------------------------------------------------------------ viscous closed form (reading 12)

@pytest.mark.parametrize("mcount", [1, 3])
def test_viscous_shear_wave_exact_discrete(mcount):
    N = 24
    n = (N, 5, 4)
    h = 1.0 / N
    grid = synth.Cartesian(h=(h,) * 3)
    a, mu = 0.1, 0.05
    xyz = grid.coords(n, (0, 0, 0), oracle.GC)
    Ui = synth.shear_wave(xyz, a=a, m=mcount, Lx=1.0)
    _, met, U = _setup(grid, n, PER, Ui)
    ph = oracle.phys(terms=2, mu_ref=mu)
    r = _inner(oracle.rhs(n, ph, U, met))
    k = 2 * np.pi * mcount
    kt = (8 * np.sin(k * h) - np.sin(2 * k * h)) / (6 * h)
    kt2 = (8 * np.sin(2 * k * h) - np.sin(4 * k * h)) / (6 * h)
    x = synth._interior_xyz(xyz)[0]
    exp_v = -mu * a * kt ** 2 * np.sin(k * x)
    exp_E = 0.5 * mu * a * a * kt * kt2 * np.cos(2 * k * x)
    sc = mu * a * k * k
    assert np.abs(r[2] - exp_v).max() < 1e-12 * sc
    assert np.abs(r[4] - exp_E).max() < 1e-12 * sc
    assert np.abs(r[[0, 1, 3]]).max() < 1e-12 * sc


def test_tgv_initial_kinetic_energy_dissipation():
    # DeBonis TGV, L = 1, V0 = 1: -dEk/dt = mu <|grad u|^2>/rho0 = 3 mu / 4 at t=0
    # (viscous terms only; the inviscid part conserves KE up to WENO dissipation)
    N = 32
    n = (N,) * 3
    h = 2 * np.pi / N
    grid = synth.Cartesian(h=(h,) * 3, x0=(-np.pi,) * 3)
    mu = 1 / 1600
    _, met, U = _setup(grid, n, PER, lambda xyz: synth.tgv(xyz))
    ph = oracle.phys(terms=2, mu_ref=mu, Pr=0.71)
    r = _inner(oracle.rhs(n, ph, U, met))
    Ui = _inner(U)
    vel = Ui[1:4] / Ui[0]
    dEk = ((vel * r[1:4]).sum(0) - 0.5 * (vel ** 2).sum(0) * r[0]).mean()
    rho0 = Ui[0].mean()
    assert abs(-dEk / (3 * mu / 4 * rho0) - 1.0) < 0.02


# ------------------------------------------------------------------ Sod vs exact Riemann (Toro)

def _exact_riemann(WL, WR, gamma=1.4):
    """Toro (2009) ch. 4 exact Riemann solver: returns (p*, u*, sampler)."""
    rL, uL, pL = WL
    rR, uR, pR = WR
    cL, cR = math.sqrt(gamma * pL / rL), math.sqrt(gamma * pR / rR)

    def f(p, r, pk, ck):
        if p > pk:
            A = 2 / ((gamma + 1) * r)
            B = (gamma - 1) / (gamma + 1) * pk
            return (p - pk) * math.sqrt(A / (p + B))
        return 2 * ck / (gamma - 1) * ((p / pk) ** ((gamma - 1) / (2 * gamma)) - 1)

    from scipy.optimize import brentq
    F = lambda p: f(p, rL, pL, cL) + f(p, rR, pR, cR) + uR - uL
    ps = brentq(F, 1e-8, 10 * max(pL, pR), xtol=1e-14)
    us = 0.5 * (uL + uR) + 0.5 * (f(ps, rR, pR, cR) - f(ps, rL, pL, cL))
    g1 = (gamma - 1) / (gamma + 1)
    rsL = rL * (ps / pL) ** (1 / gamma)                                   # rarefaction
    rsR = rR * ((ps / pR) + g1) / (g1 * (ps / pR) + 1)                    # shock
    SR = uR + cR * math.sqrt((gamma + 1) / (2 * gamma) * ps / pR + (gamma - 1) / (2 * gamma))
    csL = cL * (ps / pL) ** ((gamma - 1) / (2 * gamma))

    def rho_at(s):
        if s < uL - cL:
            return rL
        if s < us - csL:
            c = 2 / (gamma + 1) * (cL + (gamma - 1) / 2 * (uL - s))
            return rL * (c / cL) ** (2 / (gamma - 1))
        if s < us:
            return rsL
        if s < SR:
            return rsR
        return rR

    return ps, us, rsL, rsR, SR, rho_at


def test_exact_riemann_solver_matches_toro_table():
    gold = {}
    with open(os.path.join(GOLD, "sod_toro_test1.txt")) as fh:
        for line in fh:
            if line.strip() and not line.startswith("#"):
                k, v = line.split()
                gold[k] = float(v)
    ps, us, rsL, rsR, _, _ = _exact_riemann((1.0, 0.0, 1.0), (0.125, 0.0, 0.1))
    assert abs(ps - gold["p_star"]) < 1e-5
    assert abs(us - gold["u_star"]) < 1e-5
    assert abs(rsL - gold["rho_star_L"]) < 1e-5
    assert abs(rsR - gold["rho_star_R"]) < 1e-5


@pytest.mark.parametrize("lim", [{}, dict(weno_limiter=1, weno_alpha_rl=5.0)])
def test_sod_shock_tube_vs_exact(lim):
    c = synth.case("sod")
    n = c.n_global
    xyz = c.grid.coords(n, (0, 0, 0), oracle.GC)
    met = oracle.metrics(n, c.bc, xyz)
    U = synth.pad_state(synth.sod(xyz))
    ph = oracle.phys(terms=1, **lim)
    oracle.advance(n, c.bc, ph, c.dt, c.steps, U, met)
    rho = _inner(U)[0]
    x = synth._interior_xyz(xyz)[0][0, 0]
    *_, SR, rho_at = _exact_riemann((1.0, 0.0, 1.0), (0.125, 0.0, 0.1))
    t = c.dt * c.steps
    exact = np.array([rho_at((xi - 0.5) / t) for xi in x])
    l1 = np.abs(rho[0, 0] - exact).mean()
    assert l1 < 6e-3, l1
    # j,k independence (1-D problem) to round-off
    assert np.abs(rho - rho[0:1, 0:1]).max() < 1e-12
    # shock position: where rho crosses (rho*_R + rho_R)/2, within 2 cells of 0.5 + SR t
    half = 0.5 * (0.26557 + 0.125)
    ishock = np.where((rho[0, 0][:-1] > half) & (rho[0, 0][1:] <= half))[0][-1]
    assert abs(x[ishock] - (0.5 + SR * t)) < 2.0 / 200
    Ui = _inner(U)
    p = 0.4 * (Ui[4] - 0.5 * Ui[1] ** 2 / Ui[0])
    assert np.isfinite(Ui).all() and p.min() > 0 and Ui[0].min() > 0


# ------------------------------------------------------------------ isentropic vortex (closed form)

@pytest.mark.slow
def test_isentropic_vortex_translation_converges():
    errs = []
    t_end = 0.5
    for N in (32, 64):
        n = (N, N, 4)
        grid = synth.Wavy2D(L=(10.0, 10.0, 1.0), N=(N, N, 4))
        xyz = grid.coords(n, (0, 0, 0), oracle.GC)
        met = oracle.metrics(n, PER, xyz)
        U = synth.pad_state(synth.vortex(xyz))
        steps = int(round(t_end / (0.25 * 10.0 / N / 2.6)))
        dt = t_end / steps
        oracle.advance(n, PER, oracle.phys(terms=1), dt, steps, U, met)
        exact = synth.vortex(xyz, t=t_end)
        errs.append(np.abs(_inner(U)[0] - exact[0]).max())
    assert errs[0] < 2e-2
    assert errs[1] < errs[0] / 4.0, errs     # observed order >= 2
