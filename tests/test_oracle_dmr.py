"""Pins of the double-Mach-reflection workload
and of the two boundary kinds it needs (SLIPWALL, SPLIT; readings 19-20).
CPU only."""
import math

import numpy as np
import pytest

import oracle
import synth

G = 4


def _prim(q, gamma=1.4):
    rho, u, v, w, p = q
    return rho, np.array([u, v, w]), p


def test_dmr_states_satisfy_rankine_hugoniot():
    # Mach-10 shock moving at speed 10 (c_pre = 1) along its normal n = (cos30, -sin30)
    rho1, u1, p1 = _prim(synth.DMR_PRE)
    rho2, u2, p2 = _prim(synth.DMR_POST)
    g = 1.4
    assert abs(math.sqrt(g * p1 / rho1) - 1.0) < 1e-15
    n = np.array([math.cos(math.pi / 6), -math.sin(math.pi / 6), 0.0])
    Us = 10.0
    w1, w2 = u1 @ n - Us, u2 @ n - Us
    assert np.abs(np.cross(u2, n)).max() < 1e-14               # post-shock velocity normal to the shock
    assert abs(rho1 * w1 - rho2 * w2) < 1e-12                   # mass
    assert abs((p1 + rho1 * w1 ** 2) - (p2 + rho2 * w2 ** 2)) < 1e-11   # momentum
    h1, h2 = g * p1 / ((g - 1) * rho1), g * p2 / ((g - 1) * rho2)
    assert abs((h1 + 0.5 * w1 ** 2) - (h2 + 0.5 * w2 ** 2)) < 1e-12    # energy
    # the shock line x = 1/6 + y/sqrt(3) is perpendicular to n
    assert abs(np.array([1 / math.sqrt(3), 1.0, 0.0]) @ n) < 1e-15


class _Rot:
    """Affine grid rotated by `ang` in the x-y plane (unit spacing)."""

    def __init__(self, ang):
        c, s = math.cos(ang), math.sin(ang)
        self.A = np.array([[c, -s, 0.0], [s, c, 0.0], [0.0, 0.0, 1.0]])

    def coords(self, n, origin=(0, 0, 0), g=10):
        I, J, K = np.broadcast_arrays(*synth._index_grids(n, origin, g))
        X = np.stack([I, J, K])
        return np.einsum("ad,d...->a...", self.A, X)


def test_slipwall_reflects_normal_momentum_on_rotated_grid():
    n = (6, 5, 4)
    grid = _Rot(0.4)
    xyz = grid.coords(n)
    met = oracle.metrics(n, ((1, 1), (1, 1), (0, 0)), xyz)
    U = synth.pad_state(synth.random_state(n, seed=3))
    bc = ((1, 1), (oracle.SLIPWALL, oracle.SLIPWALL), (0, 0))
    oracle.fill(n, bc, U, met=met)
    eta_n = np.linalg.inv(grid.A)[1]          # grad eta, the face normal direction
    eta_n /= np.linalg.norm(eta_n)
    for gg in range(1, G + 1):
        for side in (0, 1):
            jd = G - gg if side == 0 else G + n[1] - 1 + gg   # array index of the ghost row
            js = G + gg - 1 if side == 0 else G + n[1] - gg    # its mirror
            gh, src = U[:, G:-G, jd, G:-G], U[:, G:-G, js, G:-G]
            assert np.array_equal(gh[0], src[0]) and np.array_equal(gh[4], src[4])
            mg = np.einsum("a,a...->...", eta_n, gh[1:4])
            ms = np.einsum("a,a...->...", eta_n, src[1:4])
            assert np.abs(mg + ms).max() < 1e-14
            tg = gh[1:4] - eta_n[:, None, None] * mg
            ts = src[1:4] - eta_n[:, None, None] * ms
            assert np.abs(tg - ts).max() < 1e-14


def test_split_boundary_left_right_and_time():
    n = (20, 6, 4)
    h = 0.05
    xyz = synth.Cartesian(h=(h, h, h)).coords(n)
    met = oracle.metrics(n, ((1, 1), (1, 1), (0, 0)), xyz)
    U = synth.pad_state(synth.random_state(n, seed=5))
    left = np.arange(1.0, 6.0)
    right = np.arange(11.0, 16.0)
    sp = oracle.splits({(1, 1): dict(axis=0, i0=4.2, di_dt=10.0, left=left, right_kind=oracle.DIRICHLET,
                                     right=right),
                        (1, 0): dict(axis=0, i0=7.0, di_dt=0.0, left=left, right_kind=oracle.SLIPWALL)})
    bc = ((1, 1), (oracle.SPLIT, oracle.SPLIT), (0, 0))
    t = 0.31                                   # top split at 4.2 + 3.1 = 7.3: columns i <= 6 left
    oracle.fill(n, bc, U, met=met, split=sp, t=t)
    top = U[:, G:-G, G + n[1]:, :]             # eta-hi ghost rows, all i incl. xi ghosts
    i = np.arange(-G, n[0] + G)
    is_left = i + 0.5 < 4.2 + 10.0 * t
    assert np.all(top[:, :, :, is_left] == left[:, None, None, None])
    assert np.all(top[:, :, :, ~is_left] == right[:, None, None, None])
    bot = U[:, G:-G, :G, :]
    is_left = i + 0.5 < 7.0
    assert np.all(bot[:, :, :, is_left] == left[:, None, None, None])
    # right part: slip wall mirror (Cartesian: rho v flips, others copy)
    mir = U[:, G:-G, G:2 * G, :][:, :, ::-1, :]
    assert np.array_equal(bot[[0, 1, 3, 4]][..., ~is_left], mir[[0, 1, 3, 4]][..., ~is_left])
    assert np.array_equal(bot[2][..., ~is_left], -mir[2][..., ~is_left])


@pytest.mark.slow
def test_dmr_incident_shock_moves_at_the_exact_speed():
    c = synth.case("dmr", scale=16)            # 128 x 32 x 8
    n = c.n_global
    h = 1.0 / n[1]
    xyz = c.grid.coords(n, (0, 0, 0), oracle.GC)
    met = oracle.metrics(n, c.bc, xyz)
    U = synth.pad_state(synth.dmr_state(xyz))
    bc, dv, spec = synth.dmr_bc(h)
    steps = 30
    oracle.advance(n, bc, oracle.phys(terms=1), c.dt, steps, U, met, dirichlet=dv,
                   split=oracle.splits(spec))
    t = steps * c.dt
    Ui = U[:, G:-G, G:-G, G:-G]
    assert np.isfinite(Ui).all() and Ui[0].min() > 0
    rho = Ui[0, 0]                              # k = 0 plane, (j, i)
    x = (np.arange(n[0]) + 0.5) * h
    half = 0.5 * (synth.DMR_PRE[0] + synth.DMR_POST[0])
    for j in (22, 26, 30):                      # upper rows, away from the Mach stem
        y = (j + 0.5) * h
        cross = np.where((rho[j][:-1] > half) & (rho[j][1:] <= half))[0]
        xs = x[cross[-1]] + h / 2
        assert abs(xs - synth.dmr_shock_x(y, t)) < 2.5 * h, (j, xs, synth.dmr_shock_x(y, t))
