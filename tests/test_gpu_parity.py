"""GPU parity: the CUDA path (through the C ABI) against the CPU oracle on the
same seeded inputs.  Tolerances (north_star, DESIGN.md sec. 3 reading 17):
  metrics      <= 1e-13 relative (same D6 formula, FMA contraction only)
  fill         bitwise
  RHS          <= 1e-11 relative L_inf per component (floor: flux scale)
  100 RK steps <= 1e-9  relative L_inf per component
  decomposition (n blocks vs 1 block on the GPU) bitwise
"""
import math

import numpy as np
import pytest

import oracle
import synth
from _harness import Problem, block_slices, flux_scale, inner, rel_linf, state_scale

pytestmark = pytest.mark.gpu

PER = ((0, 0),) * 3
P, E, D, W = 0, 1, 2, 3


def _torch_cuda():
    torch = pytest.importorskip("torch")
    if not torch.cuda.is_available():
        pytest.fail("GPU test run without a CUDA device")
    return torch


@pytest.fixture(autouse=True)
def _need_gpu():
    _torch_cuda()


def wavy_random(n, seed=0, phys=None, amp=0.2):
    g = synth.Wavy3D(L=(10.0,) * 3, N=n)
    return Problem(n, g, PER, synth.random_state(n, seed=seed, amp=amp),
                   phys or dict(terms=3, mu_ref=0.02))


# ------------------------------------------------------------------ library identity

def test_native_library_loaded():
    from paper_conf_ipps_davissngmb23_b200 import crocco as cc
    L = cc.lib()
    assert L._name.endswith("libcrocco.so")
    assert "sm_100a" in cc.crocco_version()


# ------------------------------------------------------------------ metrics

@pytest.mark.parametrize("nb", [(1, 1, 1), (2, 3, 1)])
def test_metrics_parity(nb):
    n = (26, 21, 13)
    pb = wavy_random(n, 1)
    xyz, met, U = pb.oracle_inputs()
    S = pb.solver(nb)
    got = [S.view(m, b, 10).cpu().numpy() for b, m in enumerate(S.met)]
    ref = inner(met)
    glob = pb.gather(S, got)
    assert rel_linf(glob[1:], ref[1:]) < 1e-13
    assert rel_linf(glob[:1], ref[:1]) < 1e-13
    # ghost metrics: periodic copies from the owners -> equal the wrapped global values
    bn, blocks = block_slices(n, nb)
    Gw = np.pad(ref, ((0, 0),) + ((4, 4),) * 3, mode="wrap")
    for (o, _), a in zip(blocks, got):
        sl = (slice(None), slice(o[2], o[2] + bn[2] + 8), slice(o[1], o[1] + bn[1] + 8),
              slice(o[0], o[0] + bn[0] + 8))
        assert rel_linf(a, Gw[sl]) < 1e-13
    S.close()


# ------------------------------------------------------------------ fill

@pytest.mark.parametrize("bc,nb", [
    (PER, (1, 1, 1)),
    (PER, (2, 2, 2)),
    (((E, E), (W, E), (P, P)), (2, 2, 2)),
    (((D, W), (E, D), (W, W)), (1, 2, 3)),
])
def test_fill_bitwise(bc, nb):
    n = (16, 12, 18)
    rng = np.random.default_rng(3)
    dv = rng.uniform(0.5, 2.0, (3, 2, 5))
    pb = Problem(n, synth.Cartesian(h=(0.1,) * 3), bc, synth.random_state(n, seed=4),
                 dict(terms=3), dirichlet=dv)
    _, _, Uref = pb.oracle_inputs()
    S = pb.solver(nb)
    S.fill()
    bn, blocks = block_slices(n, nb)
    for b, (o, _) in enumerate(blocks):
        got = S.view(S.U[b], b, 5).cpu().numpy()
        ref = Uref[:, o[2]:o[2] + bn[2] + 8, o[1]:o[1] + bn[1] + 8, o[0]:o[0] + bn[0] + 8]
        assert np.array_equal(got, ref), f"block {b}"
    S.close()


# ------------------------------------------------------------------ RHS

def _rhs_parity(pb, nb=(1, 1, 1)):
    xyz, met, U = pb.oracle_inputs()
    ref = inner(oracle.rhs(pb.n, pb.oracle_phys(), U, met))
    S = pb.solver(nb)
    S.fill()
    r = S.rhs()
    got = pb.gather(S, S.get(r))
    S.close()
    return rel_linf(got, ref, flux_scale(U, met)), got, ref


@pytest.mark.parametrize("terms,mask,weights", [(1, 1, 0), (1, 2, 0), (1, 4, 0), (1, 7, 0), (2, 7, 0),
                                                (3, 7, 0), (3, 7, 1)])
def test_rhs_parity_terms(terms, mask, weights):
    n = (37, 29, 23)   # ragged w.r.t. every thread-block tile
    pb = wavy_random(n, 2, dict(terms=terms, dir_mask=mask, mu_ref=0.02, weno_weights=weights))
    err, _, _ = _rhs_parity(pb)
    assert err < 1e-11, err


@pytest.mark.parametrize("lim,arl,aal", [(1, 5.0, 0.0), (2, 0.0, 2e-3), (3, 3.0, 1e-4)])
def test_rhs_parity_weno_limiters(lim, arl, aal):
    """Reading 23 limiters (NEXT-3): random wavy state (both branches taken) and the smooth
    vortex (relative limiter mostly linear), against the oracle."""
    n = (37, 29, 23)
    kw = dict(terms=3, mu_ref=0.02, weno_limiter=lim, weno_alpha_rl=arl, weno_alpha_al=aal)
    err, _, _ = _rhs_parity(wavy_random(n, 41, kw))
    assert err < 1e-11, err
    c = synth.case("vortex", scale=2)
    _, U = synth.block_inputs(c, (0, 0, 0), c.n_global)
    pb = Problem(c.n_global, c.grid, c.bc, U, dict(c.phys, weno_limiter=lim, weno_alpha_rl=arl,
                                                     weno_alpha_al=aal))
    err, _, _ = _rhs_parity(pb)
    assert err < 1e-11, err


def test_weno_limiter_changes_the_result():
    """The limited GPU RHS differs from the plain one (the switch is live) and matches the
    oracle's limited RHS, not its plain one."""
    n = (24, 20, 16)
    base = dict(terms=1)
    _, plain, ref_plain = _rhs_parity(wavy_random(n, 43, base))
    err, lim, ref_lim = _rhs_parity(wavy_random(n, 43, dict(base, weno_limiter=1, weno_alpha_rl=5.0)))
    assert err < 1e-11, err
    assert np.abs(lim - plain).max() > 1e3 * np.abs(lim - ref_lim).max()


def test_rhs_parity_sutherland_multiblock():
    n = (40, 24, 16)
    pb = wavy_random(n, 5, dict(terms=3, mu_law=1, mu_ref=0.03, T_ref=1.0, S=0.4, Pr=0.71))
    err, _, _ = _rhs_parity(pb, (2, 2, 2))
    assert err < 1e-11, err


def test_rhs_parity_sod():
    c = synth.case("sod")
    xyz = c.grid.coords(c.n_global, (0, 0, 0), oracle.GC)
    pb = Problem(c.n_global, c.grid, c.bc, synth.sod(xyz), c.phys)
    err, _, _ = _rhs_parity(pb)
    assert err < 1e-11, err


def test_rhs_parity_ramp_downscaled_walls():
    c = synth.case("ramp", scale=16)          # 64 x 32 x 16, 2x2x2 blocks
    xyz = c.grid.coords(c.n_global, (0, 0, 0), oracle.GC)
    pb = Problem(c.n_global, c.grid, c.bc, synth.ramp_state(xyz, c.grid), c.phys)
    err, _, _ = _rhs_parity(pb, c.n_blocks)
    assert err < 1e-11, err


def test_rhs_parity_vortex_and_tgv():
    for name, scale in (("vortex", 2), ("tgv", 8)):
        c = synth.case(name, scale=scale)
        xyz = c.grid.coords(c.n_global, (0, 0, 0), oracle.GC)
        _, U = synth.block_inputs(c, (0, 0, 0), c.n_global)
        pb = Problem(c.n_global, c.grid, c.bc, U, c.phys)
        err, _, _ = _rhs_parity(pb)
        assert err < 1e-11, (name, err)


def test_rhs_minimum_block_size_and_edge_bcs():
    n = (4, 8, 4)       # blocks of exactly 4 points (= ghost width)
    dv = np.tile(synth.prim_to_cons(1.1, 0.2, -0.1, 0.05, 0.9).reshape(1, 1, 5), (3, 2, 1))
    pb = Problem(n, synth.Cartesian(h=(0.2, 0.1, 0.3)), ((D, W), (P, P), (E, W)),
                 synth.random_state(n, seed=9), dict(terms=3, mu_ref=0.05), dirichlet=dv)
    err, _, _ = _rhs_parity(pb, (1, 2, 1))
    assert err < 1e-11, err


def test_gpu_free_stream_and_conservation():
    n = (24, 20, 16)
    g = synth.Wavy3D(L=(10.0,) * 3, N=n)
    xyz = g.coords(n, (0, 0, 0), oracle.GC)
    pb = Problem(n, g, PER, synth.free_stream(xyz), dict(terms=3, mu_ref=0.05))
    _, met, U = pb.oracle_inputs()
    S = pb.solver((2, 1, 2))
    S.fill()
    got = pb.gather(S, S.get(S.rhs()))
    assert np.abs(got).max() < 1e-13 * flux_scale(U, met)
    S.close()
    pb = wavy_random(n, 11)
    _, met, U = pb.oracle_inputs()
    S = pb.solver()
    S.fill()
    r = pb.gather(S, S.get(S.rhs()))
    J = inner(met)[0]
    tot = (r / J).reshape(5, -1).sum(1)
    mag = np.abs(r / J).reshape(5, -1).sum(1)
    assert np.all(np.abs(tot) < 1e-13 * mag)
    S.close()


# ------------------------------------------------------------------ decomposition invariance

def test_decomposition_invariance_bitwise():
    n = (32, 24, 16)
    pb = wavy_random(n, 13, dict(terms=3, mu_law=1, mu_ref=0.02, S=0.3))
    outs = []
    for nb in [(1, 1, 1), (2, 2, 2), (4, 1, 2)]:
        S = pb.solver(nb)
        S.fill()
        r1 = pb.gather(S, S.get(S.rhs()))
        S.step(1e-3, 2)
        u = pb.gather(S, S.get(S.U))
        outs.append((r1, u))
        S.close()
    for r1, u in outs[1:]:
        assert np.array_equal(r1, outs[0][0])
        assert np.array_equal(u, outs[0][1])


# ------------------------------------------------------------------ RK

def test_rk_update_parity():
    n = (20, 10, 6)
    pb = wavy_random(n, 17)
    S = pb.solver()
    rng = np.random.default_rng(1)
    torch = _torch_cuda()
    arrs = [rng.normal(size=(5, n[2] + 8, n[1] + 8, n[0] + 8)) for _ in range(3)]
    Uin, dU, rhs = [a.copy() for a in arrs]
    bufs = [S._alloc(S.layouts[0], 5) for _ in range(4)]
    for t, a in zip(bufs[:3], (Uin, dU, rhs)):
        S.view(t, 0, 5).copy_(torch.from_numpy(a))
    from paper_conf_ipps_davissngmb23_b200 import crocco as cc
    for stage in range(3):
        Uo = np.zeros_like(Uin)
        dUo = dU.copy()
        oracle.rk_update(n, stage, 0.013, Uin, Uo, dUo, rhs)
        cc.crocco_rk_update(S.ctx, stage, 0.013, [bufs[0].data_ptr()], [bufs[3].data_ptr()],
                            [bufs[1].data_ptr()], [bufs[2].data_ptr()])
        S.sync()
        gU = S.view(bufs[3], 0, 5).cpu().numpy()
        gd = S.view(bufs[1], 0, 5).cpu().numpy()
        assert rel_linf(inner(gU), inner(Uo)) < 1e-15
        assert rel_linf(inner(gd), inner(dUo)) < 1e-15
        dU = dUo
        S.view(bufs[1], 0, 5).copy_(torch.from_numpy(dU))
    S.close()


@pytest.mark.parametrize("name", ["sod", "vortex"])
def test_rk3_100_steps_parity(name):
    if name == "sod":
        c = synth.case("sod")
        xyz = c.grid.coords(c.n_global, (0, 0, 0), oracle.GC)
        U0 = synth.sod(xyz)
        n, dt = c.n_global, c.dt
    else:
        n = (24, 24, 24)
        c = synth.case("vortex")
        c.grid = synth.Wavy3D(L=(10.0,) * 3, N=n)
        xyz = c.grid.coords(n, (0, 0, 0), oracle.GC)
        U0 = synth.vortex(xyz)
        dt = 0.01
    pb = Problem(n, c.grid, c.bc, U0, c.phys)
    _, met, U = pb.oracle_inputs()
    oracle.advance(n, c.bc, pb.oracle_phys(), dt, 100, U, met)
    S = pb.solver()
    S.step(dt, 100)
    S.sync()
    got = pb.gather(S, S.get(S.U))
    S.close()
    assert rel_linf(got, inner(U), state_scale(inner(U))) < 1e-9


@pytest.mark.parametrize("name", ["weak64", "ramp_down"])
def test_rk3_100_steps_viscous_parity(name):
    """The north_star's "<= 1e-9 after 100 RK steps" on the default VISCOUS path (reading 12,
    PAPER.md:50): the weak recipe (wavy periodic TGV + 1 % noise, Re 1600) at
    64^3 in 2 x 2 x 1 blocks, and the Mach-6 ramp at 64 x 32 x 16 in 2 x 2 x 2 blocks (no-slip
    wall, extrapolation faces, Sutherland viscosity).  100 RK3 steps through crocco_rk3_step
    (CUDA graph) against oracle.advance on the same seeded inputs; floor of reading 30."""
    if name == "weak64":
        c = synth.case("weak", scale=8)
        nb = (2, 2, 1)
        xyz = c.grid.coords(c.n_global, (0, 0, 0), oracle.GC)
        U0 = synth.tgv(xyz, noise=0.01, seed=5)
    else:
        c = synth.case("ramp", scale=16)
        nb = (2, 2, 2)
        xyz = c.grid.coords(c.n_global, (0, 0, 0), oracle.GC)
        U0 = synth.ramp_state(xyz, c.grid)
    n = c.n_global
    pb = Problem(n, c.grid, c.bc, U0, c.phys)
    _, met, U = pb.oracle_inputs()
    oracle.advance(n, c.bc, pb.oracle_phys(), c.dt, 100, U, met)
    S = pb.solver(nb)
    S.step(c.dt, 100)
    S.sync()
    got = pb.gather(S, S.get(S.U))
    S.close()
    ref = inner(U)
    assert np.isfinite(ref).all()
    err = rel_linf(got, ref, state_scale(ref))
    assert err < 1e-9, (name, err)


# ------------------------------------------------------------------ full size, sampled

def _block_points(bn, rng, k_random):
    """Sampled interior points of a block: random ones plus corners, edges and faces."""
    pts = [tuple(int(rng.integers(0, m)) for m in bn) for _ in range(k_random)]
    hi = [m - 1 for m in bn]
    pts += [(0, 0, 0), tuple(hi), (0, hi[1], 3 % bn[2]), (hi[0], 0, hi[2]), (1, 2, hi[2] - 1),
            (hi[0] - 1, 5 % bn[1], 0), (bn[0] // 2, 0, hi[2]), (hi[0], bn[1] // 2, 0)]
    return pts


@pytest.mark.slow
@pytest.mark.parametrize("name", ["weak", "ramp", "tgv", "dmr", "weak_max"])
def test_full_size_config_sampled(name):
    """BASELINE.json full sizes in bench.py's launch configuration (crocco_rk_stage):
    weak = 512^3 periodic wavy TGV (configs[4]); ramp = 1024 x 512 x 256 Mach-6
    ramp in 2 x 2 x 2 blocks with walls (configs[3]); weak_max = the weak recipe at 768^3
    in one block, the maximum-size case (element offsets past 2^31 in every state and
    metric array; corners and faces of the block are among the sampled points).  Stages 0 and 1; sampled
    points recomputed by the oracle one by one from the GPU's filled 9^3
    neighbourhood of U (plus the stage-1 dU) and the ORACLE's metrics of that
    neighbourhood, computed from the generator's coordinates around the point
    (a 1-point block with non-periodic faces, so every window value is computed,
    none copied); the GPU's metric arrays are compared with those windows at the
    full size (1.4e9 elements at 512^3: 64-bit offsets)."""
    _torch_cuda()
    c = synth.case(name)
    n = c.n_global
    from paper_conf_ipps_davissngmb23_b200 import crocco as cc
    from paper_conf_ipps_davissngmb23_b200.solver import Solver
    bc, dirichlet, split = c.bc, None, None
    if name == "dmr":  # the paper's case (NEXT-2): slip wall + moving-shock SPLIT faces
        bc, dirichlet, split = synth.dmr_bc(1.0 / n[1])
    S = Solver(n, c.n_blocks, bc, cc.make_phys(**c.phys), dirichlet=dirichlet, split=split)
    bn, blocks = block_slices(n, c.n_blocks)
    # weak, weak_max (one block each): coordinates and state generated on the device (the same
    # generator formulas through torch; numpy takes minutes at 768^3); the oracle's metric
    # windows below then come from the same device path, so both sides see identical coordinates
    dev = "cuda" if name in ("weak", "weak_max") else None
    if dev:
        import torch
        x = c.grid.coords(bn, blocks[0][0], oracle.GC, device=dev).cpu()  # host copy: InitGridMetrics
        torch.cuda.empty_cache()                                             # needs 35 GB of scratch
        S.set_coords_block(0, x)
        del x
        Uv = S.view(S.U[0], 0, 5)
        for k0 in range(0, bn[2], 64):  # the state in k slabs (pointwise in the coordinates)
            ks = min(64, bn[2] - k0)
            xs = c.grid.coords((bn[0], bn[1], ks), (0, 0, k0), oracle.GC, device=dev)
            Uv[:, 4 + k0:4 + k0 + ks, 4:-4, 4:-4].copy_(synth.tgv(xs, noise=0.01, seed=5))
        del xs, Uv
    else:
        xyz = []
        U0 = []
        for o, _ in blocks:
            x, u = synth.block_inputs(c, o, bn)
            xyz.append(x)
            U0.append(u)
        S.set_coords(xyz)
        S.set_state(U0)
        del xyz, U0
    rng = np.random.default_rng(0)
    per_block = max(8, 64 // len(blocks))
    pts = [(b, p) for b in range(len(blocks)) for p in _block_points(bn, rng, per_block)]
    ph = oracle.phys(**c.phys)
    EXT = ((E, E),) * 3
    Mo = {}
    worst_m = 0.0
    for b, p in pts:
        o = blocks[b][0]
        gp = (o[0] + p[0], o[1] + p[1], o[2] + p[2])
        xw = c.grid.coords((1, 1, 1), gp, oracle.GC, device=dev).cpu().numpy() if dev else \
            c.grid.coords((1, 1, 1), gp, oracle.GC)
        Mo[(b, p)] = oracle.metrics((1, 1, 1), EXT, xw)
        sl = (slice(None), slice(p[2], p[2] + 9), slice(p[1], p[1] + 9), slice(p[0], p[0] + 9))
        Mg = S.view(S.met[b], b, 10)[sl].cpu().numpy()
        ref = Mo[(b, p)]
        # centre point: computed on both sides from the same coordinates (<= 1e-13, SURVEY 8(c)
        # metrics pin); window: ghost metrics across periodic / inter-block faces are copies of
        # the owner's (reading 6), equal to the computed value up to coordinate rounding
        # floor: the largest metric of the window (components that vanish analytically, e.g.
        # m^zeta_x on the ramp, are compared on the scale of the metric tensor)
        fl = np.abs(ref[1:]).max()
        worst_m = max(worst_m, rel_linf(Mg[:1, 4, 4, 4][:, None], ref[:1, 4, 4, 4][:, None]),
                      rel_linf(Mg[1:, 4, 4, 4][:, None], ref[1:, 4, 4, 4][:, None], fl))
        assert rel_linf(Mg[:1].reshape(1, -1), ref[:1].reshape(1, -1)) < 1e-11, (name, b, p)
        assert rel_linf(Mg[1:].reshape(9, -1), ref[1:].reshape(9, -1), fl) < 1e-11, (name, b, p)
    assert worst_m < 1e-13, (name, worst_m)
    for stage in (0, 1):
        Uin_bufs, dU_bufs = list(S.U), list(S.dU)
        dU_before = {(b, p): S.view(dU_bufs[b], b, 5)[:, p[2] + 4, p[1] + 4, p[0] + 4].cpu().numpy()
                     for b, p in pts}
        S.stage(stage, c.dt)
        S.sync()
        worst = 0.0
        for b, p in pts:
            Uin = S.view(Uin_bufs[b], b, 5)
            Uout = S.view(S.U[b], b, 5)
            dUv = S.view(dU_bufs[b], b, 5)
            sl = (slice(None), slice(p[2], p[2] + 9), slice(p[1], p[1] + 9), slice(p[0], p[0] + 9))
            Uw = np.ascontiguousarray(Uin[sl].cpu().numpy())
            Mw = Mo[(b, p)]
            r = oracle.rhs((1, 1, 1), ph, Uw, Mw)
            Uo = np.zeros_like(Uw)
            dUo = np.zeros_like(Uw)
            dUo[:, 4, 4, 4] = dU_before[(b, p)]
            oracle.rk_update((1, 1, 1), stage, c.dt, Uw, Uo, dUo, r)
            gU = Uout[:, p[2] + 4, p[1] + 4, p[0] + 4].cpu().numpy()
            gd = dUv[:, p[2] + 4, p[1] + 4, p[0] + 4].cpu().numpy()
            scale = flux_scale(Uw, Mw) * c.dt
            worst = max(worst, float(np.abs(gd - dUo[:, 4, 4, 4]).max() / max(np.abs(dUo[:, 4, 4, 4]).max(), scale)))
            worst = max(worst, float(np.abs(gU - Uo[:, 4, 4, 4]).max() / np.abs(Uo[:, 4, 4, 4]).max()))
        assert worst < 1e-11, (name, stage, worst)
    S.close()


# ------------------------------------------------------------------ DMR (NEXT-2): SLIPWALL / SPLIT faces

def _dmr_problem(scale=16):
    c = synth.case("dmr", scale=scale)
    h = 1.0 / c.n_global[1]
    bc, dv, spec = synth.dmr_bc(h)
    xyz = c.grid.coords(c.n_global, (0, 0, 0), oracle.GC)
    return c, Problem(c.n_global, c.grid, bc, synth.dmr_state(xyz), c.phys, dirichlet=dv, split=spec)


@pytest.mark.parametrize("nb", [(1, 1, 1), (2, 2, 1)])
def test_fill_slipwall_split_parity(nb):
    c, pb = _dmr_problem()
    # random state so every ghost value is distinguishable; move the top split with t
    pb.U0 = synth.random_state(pb.n, seed=31)
    t = 0.0123
    xyz, met, Uref = pb.oracle_inputs()
    oracle.fill(pb.n, pb.bc, Uref, dirichlet=pb.dirichlet, split=pb.oracle_split(), t=t, met=met)
    S = pb.solver(nb)
    S.set_time(t)
    S.fill()
    bn, blocks = block_slices(pb.n, nb)
    for b, (o, _) in enumerate(blocks):
        got = S.view(S.U[b], b, 5).cpu().numpy()
        ref = Uref[:, o[2]:o[2] + bn[2] + 8, o[1]:o[1] + bn[1] + 8, o[0]:o[0] + bn[0] + 8]
        # copies and constants are exact; slip-wall reflections round differently (FMA)
        assert np.abs(got - ref).max() <= 1e-14 * np.abs(ref).max(), b
    S.close()


def test_dmr_rk3_parity_and_decomposition():
    c, pb = _dmr_problem()
    n = pb.n
    _, met, U = pb.oracle_inputs()
    steps = 40
    oracle.advance(n, pb.bc, pb.oracle_phys(), c.dt, steps, U, met, dirichlet=pb.dirichlet,
                   split=pb.oracle_split())
    outs = []
    for nb in [(1, 1, 1), (2, 2, 1)]:
        S = pb.solver(nb)
        S.step(c.dt, steps)
        S.sync()
        assert abs(S.time - steps * c.dt) < 1e-15
        outs.append(pb.gather(S, S.get(S.U)))
        S.close()
    assert np.array_equal(outs[0], outs[1])
    assert rel_linf(outs[0], inner(U), state_scale(inner(U))) < 1e-9


# ------------------------------------------------------------------ CUDA-graph RK3 steps

def test_rk3_step_graph_equals_eager_bitwise():
    n = (40, 16, 12)
    pb = wavy_random(n, 29, dict(terms=3, mu_ref=0.02))
    outs = []
    for graph in (False, True):
        S = pb.solver((2, 1, 1))
        for _ in range(5):                       # 5 steps: both cached buffer orders replayed
            S.step(1e-3, graph=graph)
        S.sync()
        outs.append(pb.gather(S, S.get(S.U)))
        from paper_conf_ipps_davissngmb23_b200 import crocco as cc
        nl = cc.crocco_launch_count(S.ctx)
        S.close()
        assert nl > 0
    assert np.array_equal(outs[0], outs[1])


@pytest.mark.parametrize("nb,n", [((1, 1, 1), (72, 40, 140)), ((2, 1, 2), (144, 36, 280))])
def test_overlapped_stage_equals_serial_bitwise(nb, n):
    """crocco_rk_stage with the ghost fill on the comm stream beside the ghost-free viscous
    tiles equals the serial stage bit for bit.  Blocks >= 60 wide in x (a
    ghost-free 32-column tile advancing by 28) and >= 132 deep in z (an interior slab), and
    crocco_overlap_count proves the overlapped path ran (eager and graph-captured steps)."""
    from paper_conf_ipps_davissngmb23_b200 import crocco as cc
    pb = wavy_random(n, 37, dict(terms=3, mu_law=1, mu_ref=0.02, S=0.3))
    outs = []
    for ov in (False, True):
        S = pb.solver(nb)
        cc.crocco_set_overlap(S.ctx, ov)
        S.step(1e-3, 2, graph=False)
        S.step(1e-3, 1, graph=True)
        S.step(1e-3, 1, graph=True)           # replay
        S.sync()
        outs.append(pb.gather(S, S.get(S.U)))
        assert cc.crocco_overlap_count(S.ctx) == (12 if ov else 0)
        S.close()
    assert np.array_equal(outs[0], outs[1])


@pytest.mark.parametrize("change", ["limiter", "visc_form", "gamma"])
def test_graph_dropped_on_set_phys(change):
    """crocco_set_phys drops the cached RK3 step graphs (they bake in Phys and the kernel
    variants): graph step -> set_phys -> graph step equals the same sequence taken eagerly,
    bit for bit, and differs from keeping the old physics."""
    from paper_conf_ipps_davissngmb23_b200 import crocco as cc
    n = (32, 24, 20)
    base = dict(terms=3, mu_ref=0.02)
    new = dict(base)
    if change == "limiter":
        new.update(weno_limiter=1, weno_alpha_rl=5.0)
    elif change == "visc_form":
        new.update(visc_form=1)
    else:
        new.update(gamma=1.3)
    pb = wavy_random(n, 47, base)
    outs = []
    for graph, switch in ((True, True), (False, True), (True, False)):
        S = pb.solver((2, 1, 1))
        S.step(1e-3, 2, graph=graph)
        if switch:
            S.set_phys(cc.make_phys(**new))
        S.step(1e-3, 2, graph=graph)
        S.sync()
        outs.append(pb.gather(S, S.get(S.U)))
        S.close()
    assert np.array_equal(outs[0], outs[1])
    assert not np.array_equal(outs[0], outs[2])


def test_compute_dt_reports_non_finite_state():
    """A NaN / negative-pressure point is not dropped by the CFL maximum: ComputeDt
    fails instead of returning a dt from the healthy points."""
    from paper_conf_ipps_davissngmb23_b200 import crocco as cc
    n = (16, 12, 8)
    pb = wavy_random(n, 48)
    S = pb.solver()
    dt = cc.crocco_compute_dt(S.ctx, S._ptrs(S.U), S._ptrs(S.met), 0.5)
    assert dt > 0
    v = S.view(S.U[0], 0, 5)
    v[4, 6, 7, 8] = -1.0                     # negative energy -> negative pressure -> NaN c
    with pytest.raises(cc.CroccoError, match="non-finite"):
        cc.crocco_compute_dt(S.ctx, S._ptrs(S.U), S._ptrs(S.met), 0.5)
    S.close()


@pytest.mark.parametrize("interior", [False, True])
def test_steps_from_host_equals_resident_steps_bitwise(interior):
    """Solver.steps_from_host (bench e2e: independent jobs through pinned host memory, copies
    overlapped with compute on two streams) gives each job exactly the resident RK3 step;
    interior=True moves only the interior points (the step's fill makes every ghost it reads)."""
    import torch
    n = (32, 16, 12)
    pb = wavy_random(n, 31, dict(terms=3, mu_ref=0.02))
    S = pb.solver((2, 1, 1))
    jobs = []
    for j in range(5):                           # 5 distinct inputs: state after j resident steps
        if interior:
            jobs.append([S.view(u, b, 5)[:, 4:-4, 4:-4, 4:-4].contiguous().cpu().pin_memory()
                         for b, u in enumerate(S.U)])
        else:
            jobs.append([u.detach().cpu().pin_memory() for u in S.U])
        S.step(1e-3)
    S.sync()
    ref = []
    for j in range(5):                           # resident reference: one step from each input
        for b, (u, h) in enumerate(zip(S.U, jobs[j])):
            if interior:
                S.view(u, b, 5)[:, 4:-4, 4:-4, 4:-4].copy_(h)
            else:
                u.copy_(h)
        S.step(1e-3)
        S.sync()
        ref.append([u.detach().cpu().clone() for u in S.U])
    outs = [[torch.empty_like(h).pin_memory() for h in jobs[0]] for _ in range(5)]
    # stale ghosts in the device buffers (interior mode must not depend on them)
    if interior:
        for buf in S.U + S.V:
            buf.fill_(float("nan"))
    S.steps_from_host(jobs, outs, 1e-3, interior=interior)
    torch.cuda.synchronize()
    for j in range(5):
        for b in range(S.nloc):
            v = outs[j][b] if interior else S.view(outs[j][b], b, 5)[:, 4:-4, 4:-4, 4:-4]
            r = S.view(ref[j][b], b, 5)[:, 4:-4, 4:-4, 4:-4]
            assert torch.equal(v, r), (j, b)
    S.close()


# ------------------------------------------------------------------ ComputeDt (NEXT-1)

@pytest.mark.parametrize("nb", [(1, 1, 1), (2, 3, 2)])
def test_compute_dt_parity(nb):
    n = (36, 30, 20)
    pb = wavy_random(n, 23)
    _, met, U = pb.oracle_inputs()
    ref = oracle.compute_dt(n, pb.oracle_phys(), U, met, 0.7)
    S = pb.solver(nb)
    got = S.compute_dt(0.7)
    S.close()
    assert abs(got - ref) <= 1e-13 * ref, (got, ref)


def test_compute_dt_sod_closed_form():
    # Sod initial state on the Cartesian 1/200 grid: max over the two states of
    # sum_d (|u_d| + c)/h = 3 c_L / h (u = 0), c_L = sqrt(1.4)
    c = synth.case("sod")
    xyz = c.grid.coords(c.n_global, (0, 0, 0), oracle.GC)
    pb = Problem(c.n_global, c.grid, c.bc, synth.sod(xyz), c.phys)
    S = pb.solver()
    got = S.compute_dt(0.9)
    S.close()
    expect = 0.9 / (3 * math.sqrt(1.4) * 200)
    assert abs(got - expect) < 1e-12 * expect


# ------------------------------------------------------------------ state check

def test_check_state_counts_bad_points():
    n = (20, 16, 12)
    pb = wavy_random(n, 9)
    S = pb.solver((2, 1, 1))
    assert S.check_state() == 0
    v = S.view(S.U[0], 0, 5)
    v[0, 4 + 3, 4 + 2, 4 + 1] = float("nan")          # non-finite
    v[0, 4 + 5, 4 + 6, 4 + 7] = -1.0                  # rho <= 0
    v[4, 4 + 1, 4 + 1, 4 + 1] = 0.0                   # E = 0 -> p < 0
    v[1, 0, 0, 0] = float("inf")                      # a ghost point: not counted
    assert S.check_state() == 3
    S.close()


def test_degenerate_no_terms_is_exactly_stationary():
    """terms = 0 (no inviscid, no viscous flux): the RHS is exactly zero and an RK stage
    returns U_in bit for bit (dU = 0) -- the degenerate case of the method."""
    n = (19, 13, 11)
    pb = wavy_random(n, 4, phys=dict(terms=0))
    S = pb.solver((1, 1, 1))
    S.fill()
    r = S.get(S.rhs())[0][:, 4:-4, 4:-4, 4:-4]
    assert np.all(r == 0.0)
    U0 = S.get(S.U)[0][:, 4:-4, 4:-4, 4:-4]
    S.stage(0, 1e-2)
    S.sync()
    assert np.array_equal(S.get(S.U)[0][:, 4:-4, 4:-4, 4:-4], U0)
    S.close()


# ------------------------------------------------------------------ NCCL halo path on one GPU

@pytest.mark.parametrize("bc,nb,ov", [(PER, (2, 2, 2), 0), (((E, E), (W, E), (P, P)), (2, 1, 2), 0),
                                      (PER, (2, 1, 1), 1)])
def test_nccl_loopback_equals_local_and_oracle(bc, nb, ov):
    """The multi-rank exchange code (pack -> ncclSend/ncclRecv -> unpack, PAPER.md:129-131
    FillBoundary) and ComputeDt's ncclAllReduce run on hardware through a 1-rank
    communicator (crocco_set_nccl_loopback): the fill is bitwise the local fill and the oracle's,
    RK3 steps (also with the overlapped stage) are bitwise the local steps, dt is identical."""
    from paper_conf_ipps_davissngmb23_b200 import crocco as cc
    n = (144, 24, 280) if ov else (24, 20, 16)
    g = synth.Wavy3D(L=(10.0,) * 3, N=n) if bc == PER else synth.Cartesian(h=(0.1, 0.07, 0.05))
    pb = Problem(n, g, bc, synth.random_state(n, seed=51, amp=0.2), dict(terms=3, mu_ref=0.02))
    _, met, Uref = pb.oracle_inputs()
    outs, dts = [], []
    for loop in (False, True):
        S = pb.solver(nb)
        if loop:
            cc.crocco_set_nccl_loopback(S.ctx, True)
            S.fill(S.met, cc.FIELD_METRIC)       # metric ghosts through NCCL too
        cc.crocco_set_overlap(S.ctx, ov)
        S.fill()
        S.sync()
        got = S.get(S.U)
        bn, blocks = block_slices(n, nb)
        for b, (o, _) in enumerate(blocks):
            ref = Uref[:, o[2]:o[2] + bn[2] + 8, o[1]:o[1] + bn[1] + 8, o[0]:o[0] + bn[0] + 8]
            assert np.array_equal(got[b], ref), (loop, b)
        dts.append(cc.crocco_compute_dt(S.ctx, S._ptrs(S.U), S._ptrs(S.met), 0.5))
        S.step(2e-3, 2)
        S.sync()
        if ov:
            assert cc.crocco_overlap_count(S.ctx) == 6
        outs.append(pb.gather(S, S.get(S.U)))
        S.close()
    assert np.array_equal(outs[0], outs[1])
    assert dts[0] == dts[1]


@pytest.mark.slow
def test_overlap_has_interior_slabs_at_bench_depth():
    """with the run-time slab depth of 256 planes (chosen when the block is large) no
    viscous tile was ghost-free and the overlapped stage silently ran serially.  With overlap the
    depth is capped so an interior slab exists: a 512 x 512 x 264 block (slab 256 without the cap)
    runs every stage overlapped, bitwise equal to the serial stage."""
    from paper_conf_ipps_davissngmb23_b200 import crocco as cc
    n = (512, 512, 264)
    g = synth.Wavy3D(L=(2 * math.pi,) * 3, N=n, x0=(-math.pi,) * 3, k=2.0, A=0.15)
    import torch
    outs = []
    for ov in (0, 1):
        from paper_conf_ipps_davissngmb23_b200.solver import Solver
        S = Solver(n, (1, 1, 1), PER, cc.make_phys(gamma=1.4, R=1.0, Pr=0.71, mu_ref=1 / 1600))
        xyz = torch.from_numpy(g.coords(n, (0, 0, 0), oracle.GC)).cuda()
        S.set_coords([xyz])
        S.set_state([synth.tgv(xyz, noise=0.01, seed=5)])
        del xyz
        cc.crocco_set_overlap(S.ctx, ov)
        S.step(2e-4, 1)
        S.sync()
        assert cc.crocco_overlap_count(S.ctx) == (3 if ov else 0)
        outs.append(S.view(S.U[0], 0, 5)[:, 4:-4, 4:-4, 4:-4].cpu().numpy())
        S.close()
        torch.cuda.empty_cache()
    assert np.array_equal(outs[0], outs[1])
