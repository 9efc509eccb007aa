"""Pins of the oracle's building blocks against what mathematics fixes
(closed forms, textbook routines, library routines, invariants) -- never
against a retyped copy of the oracle's own formula.  CPU only.

Citations: PAPER.md line numbers (/root/reference); readings = DESIGN.md sec. 3.
"""
import math
import os

import numpy as np
import pytest

import oracle
import synth

GOLD = os.path.join(os.path.dirname(__file__), "golden")


def _gold_weights():
    vals = []
    with open(os.path.join(GOLD, "weno_symbo_weights.txt")) as f:
        for line in f:
            line = line.strip()
            if line and not line.startswith("#"):
                vals.append(float(line))
    return np.array(vals)


# ------------------------------------------------------------------ WENO-SYMBO (reading 8)

# Textbook 3-point reconstructions of the value at x_{i+1/2} from cell averages
# (Shu 1998, "Essentially non-oscillatory and WENO schemes ...", Table 2.1, k = 3,
# rows r = 2, 1, 0), plus the downwind stencil {i+1,i+2,i+3} (the r = -1 row).
SHU_STENCILS = [
    (0, [1 / 3, -7 / 6, 11 / 6]),
    (1, [-1 / 6, 5 / 6, 1 / 3]),
    (2, [1 / 3, 5 / 6, -1 / 6]),
    (3, [11 / 6, -7 / 6, 1 / 3]),
]


def test_weno_linear_stencil_is_weighted_textbook_stencils():
    C = _gold_weights()
    expect = np.zeros(6)
    for k, (start, coef) in enumerate(SHU_STENCILS):
        expect[start:start + 3] += C[k] * np.array(coef)
    expect /= C.sum()
    got = np.array([oracle.weno_symbo(np.eye(6)[l], linear=True) for l in range(6)])
    np.testing.assert_allclose(got, expect, rtol=0, atol=1e-15)
    # 6-point linear SYMBO stencil (verified there independently)
    np.testing.assert_allclose(got, [0.03154918197, -0.18176783894, 0.66634545493,
                                     0.60941218254, -0.14853528393, 0.02299630344], atol=2e-11)


def test_weights_sum_to_one():
    assert abs(_gold_weights().sum() - 1.0) < 2e-12


def _cell_avgs(poly, centers):
    """Exact cell averages over [c-1/2, c+1/2] of a numpy polynomial."""
    P = np.polynomial.Polynomial(poly).integ()
    return np.array([P(c + 0.5) - P(c - 0.5) for c in centers])


@pytest.mark.parametrize("linear", [True, False])
def test_weno_exact_for_quadratics(linear):
    rng = np.random.default_rng(1)
    for _ in range(50):
        coef = rng.normal(size=3)
        v = _cell_avgs(coef, np.arange(-2, 4))
        exact = np.polynomial.Polynomial(coef)(0.5)
        assert abs(oracle.weno_symbo(v, linear=linear) - exact) < 1e-12 * (1 + abs(exact))


def test_weno_linear_is_third_order_not_fourth():
    v = _cell_avgs([0, 0, 0, 1.0], np.arange(-2, 4))   # x^3
    assert abs(oracle.weno_symbo(v, linear=True) - 0.125) > 1e-3


def test_weno_constant():
    for c in [0.0, 1.0, -3.7, 1e5]:
        assert abs(oracle.weno_symbo([c] * 6) - c) <= 1e-15 * max(1, abs(c))


def test_weno_nonoscillatory_at_step():
    # jump between v_1 and v_2: the smooth upwind stencils 0,1 must dominate
    # (beta_3 <- max(beta) keeps the downwind stencil off, reading 8)
    assert abs(oracle.weno_symbo([0, 0, 0, 0, 1, 1])) < 1e-10
    # jump between v_0 and v_1: stencils 0 (all 0) must dominate -> ~0
    assert abs(oracle.weno_symbo([0, 0, 0, 1, 1, 1])) < 1e-9
    # jump between v_{-1} and v_0: stencils 1..3 smooth (all 1) -> ~1
    assert abs(oracle.weno_symbo([0, 0, 1, 1, 1, 1]) - 1.0) < 1e-9


def test_weno_scale_invariance_in_smooth_limit():
    # equal smoothness indicators -> omega = C / sum(C) (reading 8)
    v = np.array([0.1, 0.2, 0.3, 0.4, 0.5, 0.6])
    assert abs(oracle.weno_symbo(v) - oracle.weno_symbo(v, linear=True)) < 1e-14


# ------------------------------------------------------------------ eigenvectors (reading 9)

def _flux_n(U, n, gamma):
    """Euler flux projected on n, from Eq. 1 restated; complex-safe."""
    rho, m, E = U[0], U[1:4], U[4]
    vel = m / rho
    p = (gamma - 1) * (E - 0.5 * rho * np.dot(vel, vel))
    th = np.dot(n, vel)
    return np.concatenate([[rho * th], m * th + n * p, [(E + p) * th]])


def _jacobian_complex_step(U, n, gamma):
    h = 1e-30
    A = np.zeros((5, 5))
    for j in range(5):
        Uc = U.astype(complex)
        Uc[j] += 1j * h
        A[:, j] = np.imag(_flux_n(Uc, n, gamma)) / h
    return A


def test_eigvecs_inverse_and_diagonalise():
    rng = np.random.default_rng(2)
    gamma = 1.4
    for _ in range(200):
        n = rng.normal(size=3)
        n /= np.linalg.norm(n)
        rho = rng.uniform(0.1, 5)
        vel = rng.normal(size=3) * 2
        p = rng.uniform(0.1, 5)
        c = math.sqrt(gamma * p / rho)
        T, Ti = oracle.eigvecs(n, rho, *vel, c, gamma)
        assert np.abs(Ti @ T - np.eye(5)).max() < 1e-12
        U = np.array([rho, *(rho * vel), p / (gamma - 1) + 0.5 * rho * vel @ vel])
        A = _jacobian_complex_step(U, n, gamma)
        th = n @ vel
        lam = np.array([th, th, th, th + c, th - c])
        scale = np.abs(A).max() * np.abs(T).max()
        assert np.abs(A @ T - T * lam).max() < 1e-12 * scale


def _cons(rho, vel, p, gamma=1.4):
    return np.array([rho, *(rho * np.asarray(vel)), p / (gamma - 1) + 0.5 * rho * np.dot(vel, vel)])


def test_roe_state_satisfies_roe_property():
    """Roe (1981): the flux Jacobian at the Roe-averaged state maps the jump of the states
    onto the jump of the fluxes, A(U~)(U_R - U_L) = F_n(U_R) - F_n(U_L), for any normal n.
    A comes from a complex-step derivative of Eq. 1's flux (not from the oracle), and also
    as T Lambda T^-1 from the (separately pinned) eigenvectors.  Inverted Roe weights or an
    arithmetic mean fail it (next test, so the pin has teeth).  rho~ does not enter A;
    it is pinned by its definition rho~^2 = rho_L rho_R (reading 9)."""
    rng = np.random.default_rng(21)
    gamma = 1.4
    worst = worst_eig = 0.0
    for _ in range(200):
        n = rng.normal(size=3)
        n /= np.linalg.norm(n)
        UL = _cons(rng.uniform(0.1, 5), rng.normal(size=3) * 2, rng.uniform(0.1, 5), gamma)
        UR = _cons(rng.uniform(0.1, 5), rng.normal(size=3) * 2, rng.uniform(0.1, 5), gamma)
        rt, ut, vt, wt, ct = oracle.roe_state(UL, UR, gamma)
        assert abs(rt * rt - UL[0] * UR[0]) < 1e-13 * UL[0] * UR[0]
        vel = np.array([ut, vt, wt])
        Ut = _cons(rt, vel, rt * ct * ct / gamma, gamma)
        A = _jacobian_complex_step(Ut, n, gamma)
        jump = _flux_n(UR, n, gamma) - _flux_n(UL, n, gamma)
        scale = np.abs(jump).max() + np.abs(A).max() * np.abs(UR - UL).max()
        worst = max(worst, np.abs(A @ (UR - UL) - jump).max() / scale)
        T, Ti = oracle.eigvecs(n, rt, ut, vt, wt, ct, gamma)
        th = n @ vel
        lam = np.array([th, th, th, th + ct, th - ct])
        worst_eig = max(worst_eig, np.abs(T @ (lam * (Ti @ (UR - UL))) - jump).max() / scale)
    assert worst < 1e-13, worst
    assert worst_eig < 1e-12, worst_eig


def test_roe_wrong_averages_violate_property_typically():
    """Teeth of the pin above: on a generic pair the arithmetic mean / inverted weights miss
    Roe's property by many orders of magnitude more than rounding."""
    gamma = 1.4
    n = np.array([0.6, 0.0, 0.8])
    UL = _cons(1.0, [0.3, -0.2, 0.5], 1.0, gamma)
    UR = _cons(3.0, [-0.4, 0.6, 0.1], 2.5, gamma)
    jump = _flux_n(UR, n, gamma) - _flux_n(UL, n, gamma)
    r = math.sqrt(UR[0] / UL[0])
    vL, vR = UL[1:4] / UL[0], UR[1:4] / UR[0]
    pL = (gamma - 1) * (UL[4] - 0.5 * UL[0] * vL @ vL)
    pR = (gamma - 1) * (UR[4] - 0.5 * UR[0] * vR @ vR)
    HL, HR = (UL[4] + pL) / UL[0], (UR[4] + pR) / UR[0]
    for wl, wr in ((0.5, 0.5), (r / (1 + r), 1 / (1 + r))):
        v2 = wl * vL + wr * vR
        c2 = (gamma - 1) * (wl * HL + wr * HR - 0.5 * v2 @ v2)
        A2 = _jacobian_complex_step(_cons(1.7, v2, 1.7 * c2 / gamma, gamma), n, gamma)
        assert np.abs(A2 @ (UR - UL) - jump).max() > 1e-3 * np.abs(jump).max()
    rt, ut, vt, wt, ct = oracle.roe_state(UL, UR, gamma)
    A = _jacobian_complex_step(_cons(rt, [ut, vt, wt], rt * ct * ct / gamma, gamma), n, gamma)
    assert np.abs(A @ (UR - UL) - jump).max() < 1e-13 * np.abs(jump).max()


def _linear_weno_coeffs():
    C = _gold_weights()
    c = np.zeros(6)
    for k, (start, coef) in enumerate(SHU_STENCILS):
        c[start:start + 3] += C[k] * np.array(coef)
    return c / C.sum()


def _flux_linear_mode(U6, m, points, gamma=1.4):
    """Interface flux of readings 8-11 in linear-weight mode, composed from independently
    pinned pieces (Roe state, eigenvectors, linear SYMBO stencil from the golden weights,
    Eq. 1's flux), with the LLF speed lambda_s = max over the stencil points `points`."""
    c = _linear_weno_coeffs()
    mag = np.linalg.norm(m)
    n = m / mag
    rt, ut, vt, wt, ct = oracle.roe_state(U6[2], U6[3], gamma)
    T, Ti = oracle.eigvecs(n, rt, ut, vt, wt, ct, gamma)
    g = np.array([Ti @ _flux_n(U6[l], n, gamma) for l in range(6)]).T   # (s, l)
    w = np.array([Ti @ U6[l] for l in range(6)]).T
    eig = np.zeros((5, 6))
    for l in range(6):
        vel = U6[l, 1:4] / U6[l, 0]
        p = (gamma - 1) * (U6[l, 4] - 0.5 * U6[l, 0] * vel @ vel)
        th, cl = n @ vel, math.sqrt(gamma * p / U6[l, 0])
        eig[:, l] = np.abs([th, th, th, th + cl, th - cl])
    lam = eig[:, points].max(1)
    gp = 0.5 * (g + lam[:, None] * w)
    gm = 0.5 * (g - lam[:, None] * w)
    gh = gp @ c + gm @ c[::-1]          # W(g+) + W(mirror of g-)
    return mag * (T @ gh)


def test_llf_speed_is_max_over_all_six_stencil_points():
    """Reading 10: lambda_s = max over the 6 stencil points i-2..i+3.  A stencil whose fastest
    point is l = 0 (i-2) only: the oracle's linear-mode flux equals the composition with the
    6-point maximum and differs clearly from the (i, i+1) maximum."""
    gamma = 1.4
    ph = _ph(terms=1, weno_linear=1)
    rng = np.random.default_rng(22)
    for trial in range(20):
        U6 = np.array([_cons(rng.uniform(0.8, 1.2), rng.normal(size=3) * 0.1, rng.uniform(0.8, 1.2), gamma)
                       for _ in range(6)])
        m = rng.normal(size=3) + np.array([2.0, 0, 0])
        n = m / np.linalg.norm(m)
        fast = 3.0 + trial * 0.1
        U6[0] = _cons(1.0, fast * n, 1.0, gamma)   # |theta + c| largest at l = 0 only
        F = oracle.interface_flux(ph, U6, np.tile(m, (6, 1)))
        F6 = _flux_linear_mode(U6, m, [0, 1, 2, 3, 4, 5], gamma)
        F2 = _flux_linear_mode(U6, m, [2, 3], gamma)
        F5 = _flux_linear_mode(U6, m, [1, 2, 3, 4, 5], gamma)
        sc = np.abs(F6).max()
        assert np.abs(F - F6).max() < 1e-12 * sc, (trial, F, F6)
        assert np.abs(F - F2).max() > 1e-3 * sc
        assert np.abs(F - F5).max() > 1e-3 * sc


# ------------------------------------------------------------------ interface flux (readings 8-11)

def _ph(**kw):
    return oracle.phys(**kw)


def test_flux_constant_state_is_exact():
    rng = np.random.default_rng(3)
    ph = _ph(terms=1)
    for _ in range(20):
        rho, p = rng.uniform(0.2, 3, 2)
        vel = rng.normal(size=3)
        U = np.array([rho, *(rho * vel), p / 0.4 + 0.5 * rho * vel @ vel])
        m = rng.normal(size=3)
        F = oracle.interface_flux(ph, np.tile(U, 6), np.tile(m, 6))
        expect = np.linalg.norm(m) * _flux_n(U, m / np.linalg.norm(m), 1.4)
        assert np.abs(F - expect).max() < 1e-13 * np.abs(expect).max()


def _random_stencil(rng, gamma=1.4):
    rho = rng.uniform(0.3, 2, 6)
    vel = rng.normal(size=(6, 3))
    p = rng.uniform(0.3, 2, 6)
    E = p / (gamma - 1) + 0.5 * rho * (vel ** 2).sum(1)
    return np.column_stack([rho, rho[:, None] * vel, E])


def test_flux_cyclic_axis_permutation():
    # Pulliam-Chaussee vectors are cyclic in (x,y,z): permuting the axes of the
    # momenta and of the metric permutes the momentum flux (reading 9).
    rng = np.random.default_rng(4)
    ph = _ph(terms=1)
    for _ in range(30):
        U = _random_stencil(rng)
        m = rng.normal(size=(6, 3)) + np.array([1.0, 0, 0])
        F = oracle.interface_flux(ph, U, m)
        perm = [2, 0, 1]  # new x = old z, new y = old x, new z = old y
        Up = U.copy()
        Up[:, 1:4] = U[:, 1:4][:, perm]
        Fp = oracle.interface_flux(ph, Up, m[:, perm])
        expect = F.copy()
        expect[1:4] = F[1:4][perm]
        assert np.abs(Fp - expect).max() < 1e-12 * np.abs(F).max()


def test_flux_mirror_symmetry():
    # reflect x -> -x: reverse the stencil, negate rho*u and the metric's x part;
    # the interface flux of mass/energy/transverse momentum changes sign and
    # the normal momentum flux is unchanged.
    rng = np.random.default_rng(5)
    ph = _ph(terms=1)
    for _ in range(30):
        U = _random_stencil(rng)
        m = np.tile([1.0, 0.0, 0.0], (6, 1)) * rng.uniform(0.5, 2, (6, 1))
        F = oracle.interface_flux(ph, U, m)
        Ur = U[::-1].copy()
        Ur[:, 1] *= -1
        Fr = oracle.interface_flux(ph, Ur, m[::-1])
        expect = F * np.array([-1, 1, -1, -1, -1])
        assert np.abs(Fr - expect).max() < 1e-12 * np.abs(F).max()


def test_flux_divergence_third_order_smooth():
    # smooth 1-D data, Cartesian metric: (F^_{i+1/2} - F^_{i-1/2})/h -> dF/dx(x_i)
    # with the 3rd order of the linear SYMBO stencil, so the
    # observed order is >= 2.5 (ideal 3).  dF/dx by complex step.
    ph = _ph(terms=1)
    gamma = 1.4

    def state(x):
        rho = 1 + 0.2 * np.sin(x)
        u = 0.5 + 0.1 * np.cos(x)
        p = 1 + 0.1 * np.sin(2 * x)
        return np.stack([rho, rho * u, 0 * u, 0 * u, p / (gamma - 1) + 0.5 * rho * u * u], -1)

    def err(h, x0=0.3):
        m = np.tile([1.0, 0, 0], (6, 1))
        Fp = oracle.interface_flux(ph, state(x0 + h * np.arange(-2, 4)), m)
        Fm = oracle.interface_flux(ph, state(x0 + h * np.arange(-3, 3)), m)
        hc = 1e-30
        dF = np.imag(_flux_n(state(np.array(x0 + 1j * hc)), np.array([1.0, 0, 0]), gamma)) / hc
        return np.abs((Fp - Fm) / h - dF).max()

    # asymptotic range (the LLF max switches argmax at coarse h)
    e1, e2 = err(0.025), err(0.0125)
    assert e2 < e1 / 5.6, (e1, e2)     # observed order >= 2.5


# ------------------------------------------------------------------ metrics (readings 5-6)

def _metrics_of(grid, n, bc=((0, 0),) * 3):
    xyz = grid.coords(n, (0, 0, 0), oracle.GC)
    return xyz, oracle.metrics(n, bc, xyz)


class _Affine:
    def __init__(self, A, b):
        self.A, self.b = np.array(A), np.array(b)

    def coords(self, n, origin=(0, 0, 0), g=10):
        I, J, K = synth._index_grids(n, origin, g)
        X = synth._stack3(I, J, K)
        return np.einsum("ad,d...->a...", self.A, X) + self.b[:, None, None, None]


def test_metrics_affine_exact():
    A = [[0.9, 0.2, -0.1], [0.15, 1.1, 0.05], [-0.2, 0.1, 0.8]]
    n = (8, 7, 6)
    bc = ((1, 1),) * 3
    _, met = _metrics_of(_Affine(A, [1.0, -2.0, 0.5]), n, bc)
    M = np.array(A)
    cof = np.linalg.det(M) * np.linalg.inv(M).T       # cof[a, d] = m^d_a
    Jinv = np.linalg.det(M)
    assert np.abs(met[0] - 1 / Jinv).max() < 1e-13
    for d in range(3):
        for a in range(3):
            assert np.abs(met[1 + 3 * d + a] - cof[a, d]).max() < 1e-13


def test_metrics_sixth_order_vs_analytic():
    # wavy map: analytic d xi/d x via numpy.linalg.inv of the analytic Jacobian
    def analytic(grid, n):
        I, J, K = np.broadcast_arrays(*synth._index_grids(n, (0, 0, 0), 4))
        h = grid.L[0] / grid.N[0]
        xi, et, ze = I * h, J * h, K * h
        k, A = grid.k, grid.A
        s, c = np.sin, np.cos
        M = np.empty(xi.shape + (3, 3))   # M[..., a, d] = d x_a / d xi_d (per index)
        M[..., 0, 0] = h
        M[..., 0, 1] = h * A * k * c(k * et) * s(k * ze)
        M[..., 0, 2] = h * A * k * s(k * et) * c(k * ze)
        M[..., 1, 0] = h * A * k * s(k * ze) * c(k * xi)
        M[..., 1, 1] = h
        M[..., 1, 2] = h * A * k * c(k * ze) * s(k * xi)
        M[..., 2, 0] = h * A * k * c(k * xi) * s(k * et)
        M[..., 2, 1] = h * A * k * s(k * xi) * c(k * et)
        M[..., 2, 2] = h
        det = np.linalg.det(M)
        inv = np.linalg.inv(M)                 # inv[..., d, a] = d xi_d / d x_a
        return 1 / det, inv * det[..., None, None]

    errs = []
    for N in (24, 48):
        g = synth.Wavy3D(L=(10.0,) * 3, N=(N,) * 3)
        _, met = _metrics_of(g, (N, N, N), ((1, 1),) * 3)
        J, m = analytic(g, (N, N, N))
        e = np.abs(met[0] - J).max() / np.abs(J).max()
        for d in range(3):
            for a in range(3):
                e = max(e, np.abs(met[1 + 3 * d + a] - m[..., d, a]).max() / np.abs(m).max())
        errs.append(e)
    assert errs[1] < errs[0] / 40.0, errs      # 6th order: ideal ratio 64


def _d6(f, axis):
    r = lambda s: np.roll(f, -s, axis=axis)
    return (45 * (r(1) - r(-1)) - 9 * (r(2) - r(-2)) + (r(3) - r(-3))) / 60


def test_metrics_geometric_conservation_law():
    # sum_d D6_d m^d_a = 0 (Thomas-Lombard form, reading 6) to round-off
    N = 24
    g = synth.Wavy3D(L=(10.0,) * 3, N=(N,) * 3)
    _, met = _metrics_of(g, (N, N, N))
    axes = {0: 2, 1: 1, 2: 0}  # array axis of computational direction d
    for a in range(3):
        s = sum(_d6(met[1 + 3 * d + a], axes[d]) for d in range(3))
        inner = s[3 + 4:-3 - 4, 3 + 4:-3 - 4, 3 + 4:-3 - 4]  # avoid roll wrap
        assert np.abs(inner).max() < 1e-14 * 10 + 1e-13 * np.abs(met[1:]).max()


def test_metrics_periodic_ghost_copy():
    N = 12
    g = synth.Wavy3D(L=(10.0,) * 3, N=(N,) * 3)
    _, met = _metrics_of(g, (N, N, N))
    G = 4
    inner = met[:, G:-G, G:-G, G:-G]
    wrapped = np.pad(inner, ((0, 0), (G, G), (G, G), (G, G)), mode="wrap")
    assert np.array_equal(wrapped, met)


# ------------------------------------------------------------------ fill (reading 15)

def _rand_padded(n, nc, seed):
    a = oracle.padded(n, nc)
    G = 4
    a[:, G:-G, G:-G, G:-G] = np.random.default_rng(seed).uniform(0.5, 1.5, (nc, n[2], n[1], n[0]))
    return a


def test_fill_periodic_is_numpy_wrap():
    n = (6, 5, 4)
    a = _rand_padded(n, 5, 0)
    oracle.fill(n, ((0, 0),) * 3, a)
    assert np.array_equal(a, np.pad(a[:, 4:-4, 4:-4, 4:-4], ((0, 0),) + ((4, 4),) * 3, mode="wrap"))


def test_fill_extrap_is_numpy_edge():
    n = (6, 5, 4)
    a = _rand_padded(n, 5, 1)
    oracle.fill(n, ((1, 1),) * 3, a)
    assert np.array_equal(a, np.pad(a[:, 4:-4, 4:-4, 4:-4], ((0, 0),) + ((4, 4),) * 3, mode="edge"))


def test_fill_wall_is_numpy_symmetric_with_momentum_flip():
    n = (6, 5, 4)
    a = _rand_padded(n, 5, 2)
    oracle.fill(n, ((1, 1), (3, 3), (0, 0)), a)
    inner = a[:, 4:-4, 4:-4, 4:-4]
    # eta walls: mirror about j = -1/2 and j = n-1/2 with the momentum negated
    ref = np.pad(inner, ((0, 0), (0, 0), (4, 4), (0, 0)), mode="symmetric")
    sgn = np.ones((5, 1, 1, 1))
    sgn[1:4] = -1
    ghost = ref.copy()
    ghost[:, :, :4] *= sgn
    ghost[:, :, -4:] *= sgn
    # xi: edge, zeta: wrap -- order xi, eta, zeta as in reading 16
    ghost = np.pad(ghost, ((0, 0), (0, 0), (0, 0), (4, 4)), mode="edge")
    ghost = np.pad(ghost, ((0, 0), (4, 4), (0, 0), (0, 0)), mode="wrap")
    # xi phase ran before eta: xi ghosts at eta-ghost rows are then eta-mirrors of xi-edge values
    inner_x = np.pad(inner, ((0, 0), (0, 0), (0, 0), (4, 4)), mode="edge")
    ref2 = np.pad(inner_x, ((0, 0), (0, 0), (4, 4), (0, 0)), mode="symmetric")
    ref2[:, :, :4] *= sgn
    ref2[:, :, -4:] *= sgn
    ref2 = np.pad(ref2, ((0, 0), (4, 4), (0, 0), (0, 0)), mode="wrap")
    assert np.array_equal(a, ref2)


def test_fill_dirichlet_and_metric_kind():
    n = (5, 5, 5)
    a = _rand_padded(n, 5, 3)
    dv = np.arange(30, dtype=float).reshape(3, 2, 5)
    oracle.fill(n, ((2, 2), (0, 0), (0, 0)), a, dirichlet=dv)
    assert np.all(a[:, 4:-4, 4:-4, :4] == dv[0, 0][:, None, None, None])
    assert np.all(a[:, 4:-4, 4:-4, -4:] == dv[0, 1][:, None, None, None])
    m = _rand_padded(n, 10, 4)
    before = m.copy()
    oracle.fill(n, ((1, 2), (3, 1), (1, 1)), m, kind=oracle.FIELD_METRIC)
    assert np.array_equal(m, before)  # physical faces keep their computed ghost metrics


# ------------------------------------------------------------------ RK3 (PAPER.md:50 ref [10]; reading 13)

def test_williamson_rk3_amplification():
    n = (3, 3, 3)
    for z in [-0.5, 0.3 + 0.0, -1.2, 0.05]:
        U = oracle.padded(n, 5)
        U[:, 4:-4, 4:-4, 4:-4] = 1.0
        V = U.copy()
        dU = np.full_like(U, np.nan)
        dt = 0.1
        lam = z / dt
        a, o = U, V
        for s in range(3):
            r = lam * a
            oracle.rk_update(n, s, dt, a, o, dU, np.ascontiguousarray(r))
            a, o = o, a
        got = a[0, 5, 5, 5]
        assert abs(got - (1 + z + z * z / 2 + z ** 3 / 6)) < 1e-15 * 4
        assert np.isfinite(dU[:, 4:-4, 4:-4, 4:-4]).all()  # stage 0 never reads dU


def test_williamson_stage_times_second_order_conditions():
    # linear, time-dependent rhs f(t): one step must integrate polynomials of
    # degree <= 2 in t exactly (3rd-order method); stage times c = (0, 1/3, 3/4)
    n = (1, 1, 1)
    for deg in range(3):
        U = oracle.padded(n, 5)
        V = U.copy()
        dU = U.copy()
        dt = 0.7
        cst = [0.0, 1 / 3, 3 / 4]
        a, o = U, V
        for s in range(3):
            r = np.full_like(U, (cst[s] * dt) ** deg)
            oracle.rk_update(n, s, dt, a, o, dU, r)
            a, o = o, a
        assert abs(a[0, 4, 4, 4] - dt ** (deg + 1) / (deg + 1)) < 1e-15


# ------------------------------------------------------------------ ComputeDt (Eq. 3; NEXT-1)

def test_compute_dt_cartesian_closed_form():
    # uniform state on a Cartesian grid: dt = CFL / sum_d (|u_d| + c)/h_d  (Eq. 3 per direction)
    n = (6, 5, 4)
    h = (0.1, 0.2, 0.05)
    grid = synth.Cartesian(h=h)
    xyz = grid.coords(n, (0, 0, 0), 10)
    met = oracle.metrics(n, ((0, 0),) * 3, xyz)
    vel = (0.3, -0.7, 0.2)
    U = synth.pad_state(synth.free_stream(xyz, rho=1.3, vel=vel, p=0.9))
    c = math.sqrt(1.4 * 0.9 / 1.3)
    expect = 0.8 / sum((abs(vel[d]) + c) / h[d] for d in range(3))
    got = oracle.compute_dt(n, oracle.phys(), U, met, 0.8)
    assert abs(got - expect) < 1e-13 * expect


def test_compute_dt_affine_grid_via_matrix_inverse():
    # affine grid x = A xi: d xi_d/d x_a = inv(A)[d, a]; the spectral radius of
    # the contravariant flux Jacobian of direction d is |grad xi_d . u| + c |grad xi_d|
    A = np.array([[0.9, 0.2, -0.1], [0.15, 1.1, 0.05], [-0.2, 0.1, 0.8]])
    n = (5, 5, 5)
    xyz = _Affine(A, [0.0, 0.0, 0.0]).coords(n, (0, 0, 0), 10)
    met = oracle.metrics(n, ((1, 1),) * 3, xyz)
    rng = np.random.default_rng(11)
    Ui = synth.random_state(n, seed=12)
    U = synth.pad_state(Ui)
    gradxi = np.linalg.inv(A)                      # rows: grad xi_d
    rho = Ui[0]
    vel = Ui[1:4] / rho
    p = 0.4 * (Ui[4] - 0.5 * rho * (vel ** 2).sum(0))
    c = np.sqrt(1.4 * p / rho)
    lam = sum(np.abs(np.einsum("a,a...->...", gradxi[d], vel)) + c * np.linalg.norm(gradxi[d])
              for d in range(3))
    expect = 0.5 / lam.max()
    got = oracle.compute_dt(n, oracle.phys(), U, met, 0.5)
    assert abs(got - expect) < 1e-13 * expect


# ------------------------------------------------------------------ SYMOO weights (NEXT-3, reading 22)

def test_symoo_linear_stencil_is_sixth_order_central():
    # C = (1, 9, 9, 1)/20 turns the 4 candidate stencils into the 6th-order central
    # interface reconstruction (1, -8, 37, 37, -8, 1)/60
    got = np.array([oracle.weno_symbo(np.eye(6)[l], linear=True, weights=1) for l in range(6)])
    np.testing.assert_allclose(got, np.array([1, -8, 37, 37, -8, 1]) / 60.0, rtol=0, atol=1e-15)


def test_symoo_exact_for_quintic_cell_averages_in_linear_mode():
    rng = np.random.default_rng(8)
    for _ in range(20):
        coef = rng.normal(size=6)
        v = _cell_avgs(coef, np.arange(-2, 4))
        exact = np.polynomial.Polynomial(coef)(0.5)
        assert abs(oracle.weno_symbo(v, linear=True, weights=1) - exact) < 1e-12 * (1 + abs(exact))


def test_symoo_nonlinear_still_nonoscillatory():
    assert abs(oracle.weno_symbo([0, 0, 0, 0, 1, 1], weights=1)) < 1e-9


# ------------------------------------------------------------------ WENO limiters (reading 23, NEXT-3)

# v_i = i^3 at i = -2..3.  Jiang-Shu indicators by hand (App. A.3 definitions):
#   beta_0 = 13/12 (-6)^2 + 1/4 (-4)^2 = 43,  beta_1 = 0 + 1/4 (-2)^2 = 1,
#   beta_2 = 13/12 6^2 + 1/4 4^2 = 43,        beta_3 = 13/12 12^2 + 1/4 (-22)^2 = 277
# so max/min = 277 and max = 277 (the downwind beta_3 is already the largest).
CUBIC = [-8.0, -1.0, 0.0, 1.0, 8.0, 27.0]


def test_limiter_thresholds_on_hand_computed_indicators():
    lin = oracle.weno_symbo(CUBIC, linear=True)
    non = oracle.weno_symbo(CUBIC)
    assert abs(lin - non) > 1e-2                       # the two branches are distinguishable
    lim = lambda **kw: oracle.weno_limited(CUBIC, **kw)
    assert lim(limiter=1, alpha_rl=278.0) == lin       # 277 < 278 * 1: relative fires
    assert lim(limiter=1, alpha_rl=276.0) == non
    assert lim(limiter=2, alpha_al=278.0) == lin       # 277 < 278: absolute fires
    assert lim(limiter=2, alpha_al=276.0) == non
    assert lim(limiter=3, alpha_rl=276.0, alpha_al=278.0) == lin   # either limiter suffices
    assert lim(limiter=3, alpha_rl=278.0, alpha_al=276.0) == lin
    assert lim(limiter=3, alpha_rl=276.0, alpha_al=276.0) == non
    assert lim(limiter=0, alpha_rl=1e300, alpha_al=1e300) == non   # flags off


def test_limiter_limits_reduce_to_linear_and_plain_weno():
    rng = np.random.default_rng(23)
    for _ in range(200):
        v = rng.normal(size=6) * 10.0 ** rng.uniform(-3, 3)
        # thresholds that always / never fire (beta >= 0, so max < 0 * min is never true)
        assert oracle.weno_limited(v, limiter=1, alpha_rl=1e300) == oracle.weno_symbo(v, linear=True)
        assert oracle.weno_limited(v, limiter=3, alpha_rl=0.0, alpha_al=0.0) == oracle.weno_symbo(v)


def test_limiter_keeps_step_nonoscillatory_and_smooth_data_linear():
    # at a jump the indicators differ by orders of magnitude -> nonlinear weights stay;
    # on a gentle sine they are within a factor ~1.5 -> relative limiter (5) goes linear
    step = [0.0, 0.0, 0.0, 1.0, 1.0, 1.0]
    assert oracle.weno_limited(step, limiter=1, alpha_rl=5.0) == oracle.weno_symbo(step)
    x = np.arange(-2, 4) * 0.05
    s = np.sin(x + 0.3)
    assert oracle.weno_limited(s, limiter=1, alpha_rl=5.0) == oracle.weno_symbo(s, linear=True)
