"""GPU parity of the 27-component metric set and the expanded viscous form (
SURVEY 8(f) NEXT-3; readings 27-28) through the C ABI against the oracle:
  second metrics              <= 1e-12 relative (same D6 formula, FMA contraction only)
  RHS (visc_form = 1)         <= 1e-11 relative L_inf per component (floor: flux scale)
  RK3 steps                   <= 1e-9
  decomposition (n blocks)    bitwise
"""
import numpy as np
import pytest

import oracle
import synth
from _harness import Problem, block_slices, flux_scale, inner, rel_linf, state_scale

pytestmark = pytest.mark.gpu

PER = ((0, 0),) * 3


@pytest.fixture(autouse=True)
def _need_gpu():
    torch = pytest.importorskip("torch")
    if not torch.cuda.is_available():
        pytest.fail("GPU test run without a CUDA device")


def _problem(n, seed=2, **kw):
    phys = dict(terms=3, mu_law=1, mu_ref=0.03, T_ref=1.0, S=0.4, visc_form=1)
    phys.update(kw)
    g = synth.Wavy3D(L=(10.0,) * 3, N=n)
    return Problem(n, g, PER, synth.random_state(n, seed=seed, amp=0.2), phys)


@pytest.mark.parametrize("nb", [(1, 1, 1), (2, 1, 3)])
def test_second_metrics_parity(nb):
    n = (22, 17, 15)
    pb = _problem(n)
    xyz, met, U = pb.oracle_inputs()
    ref = inner(oracle.metrics2(n, met))
    S = pb.solver(nb)
    got = np.zeros_like(ref)
    for b, (o, sl) in enumerate(S.blocks):
        got[(slice(None),) + sl] = S.metrics2(b).cpu().numpy()
    assert rel_linf(got, ref) < 1e-12
    S.close()


@pytest.mark.parametrize("terms,nb", [(2, (1, 1, 1)), (3, (1, 1, 1)), (3, (2, 2, 1)), (2, (1, 3, 2))])
def test_rhs_parity_expanded_viscous(terms, nb):
    n = (24, 18, 14)
    pb = _problem(n, terms=terms)
    xyz, met, U = pb.oracle_inputs()
    ref = inner(oracle.rhs(n, pb.oracle_phys(), U, met))
    S = pb.solver(nb)
    S.fill()
    got = pb.gather(S, S.get(S.rhs()))
    assert rel_linf(got, ref, flux_scale(U, met)) < 1e-11
    S.close()


def test_rhs_expanded_constant_mu_and_decomposition_bitwise():
    n = (24, 16, 16)
    pb = _problem(n, mu_law=0, mu_ref=0.02)
    xyz, met, U = pb.oracle_inputs()
    ref = inner(oracle.rhs(n, pb.oracle_phys(), U, met))
    outs = []
    for nb in [(1, 1, 1), (2, 2, 2)]:
        S = pb.solver(nb)
        S.fill()
        outs.append(pb.gather(S, S.get(S.rhs())))
        S.close()
    assert np.array_equal(outs[0], outs[1])
    assert rel_linf(outs[0], ref, flux_scale(U, met)) < 1e-11


def test_rk3_parity_expanded_viscous():
    n = (20, 20, 16)
    g = synth.Wavy3D(L=(10.0,) * 3, N=n)
    xyz = g.coords(n, (0, 0, 0), oracle.GC)
    pb = Problem(n, g, PER, synth.vortex(xyz), dict(terms=3, mu_ref=0.01, visc_form=1))
    _, met, U = pb.oracle_inputs()
    dt, steps = 0.01, 10
    oracle.advance(n, PER, pb.oracle_phys(), dt, steps, U, met)
    S = pb.solver((2, 1, 1))
    S.step(dt, steps)
    S.sync()
    got = pb.gather(S, S.get(S.U))
    assert rel_linf(got, inner(U), state_scale(inner(U))) < 1e-9
    S.close()


def test_expanded_form_needs_second_metrics():
    from paper_conf_ipps_davissngmb23_b200 import crocco as cc
    from paper_conf_ipps_davissngmb23_b200.solver import Solver
    n = (16, 16, 16)
    g = synth.Wavy3D(L=(10.0,) * 3, N=n)
    S = Solver(n, (1, 1, 1), PER, cc.make_phys(terms=3, mu_ref=0.01))   # conservative form
    S.set_coords([g.coords(n, (0, 0, 0), oracle.GC)])
    S.set_state([synth.random_state(n, seed=4)])
    with pytest.raises(cc.CroccoError):
        cc.crocco_copy_metrics2(S.ctx, 0, S.U[0].data_ptr())
    # switching to visc_form = 1 through set_phys computes them (Solver), the raw ABI would refuse
    S.set_phys(cc.make_phys(terms=3, mu_ref=0.01, visc_form=1))
    S.stage(0, 1e-3)
    S.sync()
    S.close()
