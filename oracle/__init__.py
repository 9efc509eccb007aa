"""ctypes wrapper of the CPU fp64 oracle (oracle/crocco_oracle.c).

TEST INFRASTRUCTURE ONLY: imported by tests/, __graft_entry__.smoke() and the
cpu_baseline / ``--impl reference`` legs of bench.py -- never by the product
package.  No code is shared with paper_conf_ipps_davissngmb23_b200/; the
arithmetic lives in crocco_oracle.c, this file only marshals numpy arrays.

Arrays are numpy float64, C-contiguous, shape (ncomp, P2, P1, P0) with
Pd = n[d] + 2*g (g = 4 for state/metrics/rhs, 10 for coordinates): index
[c, k+g, j+g, i+g] is point (i, j, k).
"""
from __future__ import annotations

import ctypes as C
import os
import subprocess

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SRC = os.path.join(_HERE, "crocco_oracle.c")
_LIB = os.path.join(_HERE, "liboracle.so")

G = 4
GC = 10
PERIODIC, EXTRAP, DIRICHLET, WALL, SLIPWALL, SPLIT, COARSE_FINE = 0, 1, 2, 3, 4, 5, 6
INVISCID, VISCOUS = 1, 2
FIELD_STATE, FIELD_METRIC = 0, 1
MU_CONST, MU_SUTHERLAND = 0, 1


def build(force: bool = False) -> str:
    """Compile the oracle with gcc (-O2, no FMA contraction, OpenMP)."""
    if force or not os.path.exists(_LIB) or os.path.getmtime(_LIB) < os.path.getmtime(_SRC):
        cmd = ["gcc", "-O2", "-ffp-contract=off", "-fno-fast-math", "-fopenmp", "-fPIC",
               "-shared", "-std=c11", "-o", _LIB + ".tmp", _SRC, "-lm"]
        subprocess.check_call(cmd)
        os.replace(_LIB + ".tmp", _LIB)
    return _LIB


class Phys(C.Structure):
    _fields_ = [("gamma", C.c_double), ("R", C.c_double), ("Pr", C.c_double),
                ("mu_law", C.c_int32), ("mu_ref", C.c_double), ("T_ref", C.c_double),
                ("S", C.c_double), ("weno_eps", C.c_double), ("terms", C.c_int32),
                ("dir_mask", C.c_int32), ("weno_linear", C.c_int32), ("weno_weights", C.c_int32),
                ("weno_limiter", C.c_int32), ("weno_alpha_rl", C.c_double), ("weno_alpha_al", C.c_double),
                ("visc_form", C.c_int32)]


class Split(C.Structure):
    """Moving split of boundary data along a tangential axis (SPLIT faces, DMR)."""
    _fields_ = [("axis", C.c_int32), ("i0", C.c_double), ("di_dt", C.c_double),
                ("left", C.c_double * 5), ("right_kind", C.c_int32), ("right", C.c_double * 5)]


def splits(spec=None):
    """spec: {(d, side): dict(axis, i0, di_dt, left, right_kind, right)} -> Split[6]."""
    arr = (Split * 6)()
    for (d, side), v in (spec or {}).items():
        s = arr[2 * d + side]
        s.axis, s.i0, s.di_dt, s.right_kind = int(v["axis"]), float(v["i0"]), float(v["di_dt"]), int(v["right_kind"])
        for c in range(5):
            s.left[c] = float(v["left"][c])
            s.right[c] = float(v.get("right", [0.0] * 5)[c])
    return arr


def phys(gamma=1.4, R=1.0, Pr=0.72, mu_law=MU_CONST, mu_ref=0.0, T_ref=1.0, S=0.0,
         weno_eps=1e-6, terms=INVISCID | VISCOUS, dir_mask=7, weno_linear=0, weno_weights=0,
         weno_limiter=0, weno_alpha_rl=0.0, weno_alpha_al=0.0, visc_form=0) -> Phys:
    return Phys(gamma, R, Pr, mu_law, mu_ref, T_ref, S, weno_eps, terms, dir_mask, weno_linear, weno_weights,
                weno_limiter, weno_alpha_rl, weno_alpha_al, visc_form)


_lib = None


def lib():
    global _lib
    if _lib is None:
        L = C.CDLL(build())
        dp = C.POINTER(C.c_double)
        i64p = C.POINTER(C.c_int64)
        i32p = C.POINTER(C.c_int32)
        L.oracle_fill.argtypes = [i64p, i32p, dp, dp, C.c_int32, C.c_int32]
        L.oracle_metrics.argtypes = [i64p, i32p, dp, dp]
        L.oracle_weno_symbo.argtypes = [dp, C.c_double, C.c_int]
        L.oracle_weno_symbo.restype = C.c_double
        L.oracle_weno.argtypes = [dp, C.c_double, C.c_int, C.c_int]
        L.oracle_weno.restype = C.c_double
        L.oracle_weno_lim.argtypes = [dp, C.c_double, C.c_int, C.c_int, C.c_int, C.c_double, C.c_double]
        L.oracle_weno_lim.restype = C.c_double
        L.oracle_eigvecs.argtypes = [dp, C.c_double, C.c_double, C.c_double, C.c_double,
                                     C.c_double, C.c_double, dp, dp]
        L.oracle_interface_flux.argtypes = [C.POINTER(Phys), dp, dp, dp]
        L.oracle_roe_state.argtypes = [dp, dp, C.c_double, dp]
        L.oracle_rhs.argtypes = [i64p, C.POINTER(Phys), dp, dp, dp]
        L.oracle_rk_update.argtypes = [i64p, C.c_int32, C.c_double, dp, dp, dp, dp]
        L.oracle_rk_stage.argtypes = [i64p, i32p, dp, C.POINTER(Phys), C.c_int32, C.c_double,
                                      dp, dp, dp, dp]
        L.oracle_advance.argtypes = [i64p, i32p, dp, C.POINTER(Phys), C.c_double, C.c_int32,
                                     dp, dp]
        sp = C.POINTER(Split)
        L.oracle_fill_ex.argtypes = [i64p, i32p, dp, sp, C.c_double, dp, dp, C.c_int32, C.c_int32]
        L.oracle_rk_stage_ex.argtypes = [i64p, i32p, dp, sp, C.c_double, C.POINTER(Phys), C.c_int32,
                                         C.c_double, dp, dp, dp, dp]
        L.oracle_advance_ex.argtypes = [i64p, i32p, dp, sp, C.c_double, C.POINTER(Phys), C.c_double,
                                        C.c_int32, dp, dp]
        L.oracle_compute_dt.argtypes = [i64p, C.POINTER(Phys), dp, dp, C.c_double]
        L.oracle_compute_dt.restype = C.c_double
        L.oracle_fill_two_levels.argtypes = [i64p, i32p, dp, dp, dp, i64p, i64p, dp]
        L.oracle_fill_two_levels_ex.argtypes = [i64p, i32p, dp, C.POINTER(Split), C.c_double, dp, dp, i64p,
                                                i64p, dp]
        L.oracle_average_down.argtypes = [i64p, i32p, dp, dp, i64p, i64p, dp]
        dpp = C.POINTER(dp)
        L.oracle_fill_two_levels_sib.argtypes = [i64p, i32p, dp, dp, dp, i64p, i64p, dp, C.c_int32, i64p, i64p, dpp]
        L.oracle_average_down_sib.argtypes = [i64p, i32p, dp, dp, i64p, i64p, dp, C.c_int32, i64p, i64p, dpp]
        L.oracle_amr_advance.argtypes = [i64p, i32p, dp, i64p, i32p, dp, i64p, C.POINTER(Phys),
                                         C.c_double, C.c_int32, dp, dp, dp, dp]
        L.oracle_metrics2.argtypes = [i64p, dp, dp]
        L.oracle_rhs_ex.argtypes = [i64p, C.POINTER(Phys), dp, dp, dp, dp]
        L.oracle_set_threads.argtypes = [C.c_int]
        L.oracle_get_threads.restype = C.c_int
        _lib = L
    return _lib


def _dp(a: np.ndarray):
    assert a.dtype == np.float64 and a.flags.c_contiguous
    return a.ctypes.data_as(C.POINTER(C.c_double))


def _n(n):
    return (C.c_int64 * 3)(*[int(x) for x in n])


def _bc(bc):
    flat = [int(x) for pair in bc for x in pair]
    return (C.c_int32 * 6)(*flat)


def _dir(dirichlet):
    arr = np.zeros(30) if dirichlet is None else np.ascontiguousarray(dirichlet, dtype=np.float64).reshape(30)
    return arr


def padded(n, ncomp, g=G):
    return np.zeros((ncomp, n[2] + 2 * g, n[1] + 2 * g, n[0] + 2 * g))


def set_threads(k: int):
    lib().oracle_set_threads(int(k))


def get_threads() -> int:
    return int(lib().oracle_get_threads())


def fill(n, bc, f, kind=FIELD_STATE, dirichlet=None, split=None, t=0.0, met=None):
    """FillPatch + BC_Fill in place; split/t/met for SPLIT and SLIPWALL faces."""
    d = _dir(dirichlet)
    sp = split if split is not None else splits()
    mp = _dp(met) if met is not None else None
    lib().oracle_fill_ex(_n(n), _bc(bc), _dp(d), sp, float(t), mp, _dp(f), f.shape[0], kind)
    return f


def metrics(n, bc, xyz):
    """10-component metrics (J, m^d_a) on the padded box from coordinates."""
    met = padded(n, 10)
    lib().oracle_metrics(_n(n), _bc(bc), _dp(np.ascontiguousarray(xyz)), _dp(met))
    return met


def weno_symbo(v, eps=1e-6, linear=False, weights=0) -> float:
    """W(v_{-2..3}) at the +1/2 interface; weights 0 = SYMBO, 1 = SYMOO."""
    a = np.ascontiguousarray(v, dtype=np.float64)
    return float(lib().oracle_weno(_dp(a), eps, int(linear), int(weights)))


def weno_limited(v, eps=1e-6, limiter=0, alpha_rl=0.0, alpha_al=0.0, weights=0, linear=False) -> float:
    """W with the relative (bit 0) / absolute (bit 1) limiters of reading 23."""
    a = np.ascontiguousarray(v, dtype=np.float64)
    return float(lib().oracle_weno_lim(_dp(a), eps, int(linear), int(weights), int(limiter),
                                        float(alpha_rl), float(alpha_al)))


def eigvecs(nrm, rho, u, v, w, c, gamma=1.4):
    T = np.zeros(25)
    Ti = np.zeros(25)
    a = np.ascontiguousarray(nrm, dtype=np.float64)
    lib().oracle_eigvecs(_dp(a), rho, u, v, w, c, gamma, _dp(T), _dp(Ti))
    return T.reshape(5, 5), Ti.reshape(5, 5)


def roe_state(UL, UR, gamma=1.4):
    """Roe average (rho~, u~, v~, w~, c~) of the conserved states at points i, i+1 (reading 9)."""
    a = np.ascontiguousarray(UL, dtype=np.float64)
    b = np.ascontiguousarray(UR, dtype=np.float64)
    out = np.zeros(5)
    lib().oracle_roe_state(_dp(a), _dp(b), float(gamma), _dp(out))
    return out


def interface_flux(ph: Phys, Ul, ml):
    Ua = np.ascontiguousarray(Ul, dtype=np.float64).reshape(30)
    ma = np.ascontiguousarray(ml, dtype=np.float64).reshape(18)
    F = np.zeros(5)
    lib().oracle_interface_flux(C.byref(ph), _dp(Ua), _dp(ma), _dp(F))
    return F


def rhs(n, ph: Phys, U, met):
    """rhs = J(-sum delta F_inv + sum D4 F_v) on interior points (ghosts of U must be filled)."""
    out = padded(n, 5)
    lib().oracle_rhs(_n(n), C.byref(ph), _dp(U), _dp(met), _dp(out))
    return out


def metrics2(n, met):
    """18 second metrics xi_{a,jk} (j <= k; component 6a + pair) on interior points from the
    10-component metrics (PAPER.md:139's 27-component set = these + the 9 first metrics)."""
    out = padded(n, 18)
    lib().oracle_metrics2(_n(n), _dp(met), _dp(out))
    return out


def rk_update(n, stage, dt, Uin, Uout, dU, r):
    lib().oracle_rk_update(_n(n), stage, dt, _dp(Uin), _dp(Uout), _dp(dU), _dp(r))


def rk_stage(n, bc, ph, stage, dt, Uin, Uout, dU, met, dirichlet=None, split=None, t=0.0):
    """One RK stage (fill at t + c_s dt, RHS, update); t = start of the step."""
    d = _dir(dirichlet)
    sp = split if split is not None else splits()
    lib().oracle_rk_stage_ex(_n(n), _bc(bc), _dp(d), sp, float(t), C.byref(ph), stage, dt, _dp(Uin),
                             _dp(Uout), _dp(dU), _dp(met))


def advance(n, bc, ph, dt, nsteps, U, met, dirichlet=None, split=None, t0=0.0):
    """nsteps RK3 steps in place on U (padded) from time t0, ghosts filled on return."""
    d = _dir(dirichlet)
    sp = split if split is not None else splits()
    lib().oracle_advance_ex(_n(n), _bc(bc), _dp(d), sp, float(t0), C.byref(ph), dt, nsteps, _dp(U), _dp(met))
    return U


def compute_dt(n, ph: Phys, U, met, cfl):
    """ComputeDt: CFL / max_i sum_d J(|m^d.u| + c|m^d|) (Eq. 3, 95, 131)."""
    return float(lib().oracle_compute_dt(_n(n), C.byref(ph), _dp(U), _dp(met), float(cfl)))


# ---- two-level AMR (oracle section 9, readings 24-26) ----
def fill_two_levels(nf, bcf, Uf, nc, c0, Uc, dirichlet=None, met=None, split=None, t=0.0):
    """FillPatchTwoLevels in place on the fine state Uf: the three-phase fill with COARSE_FINE
    faces interpolated (trilinear, ratio 2, node-centred) from the coarse state Uc (ghosts filled);
    the fine level's own physical faces (SPLIT data at time t, SLIPWALL with met) as in fill()."""
    d = _dir(dirichlet)
    mp = _dp(met) if met is not None else None
    sp = split if split is not None else splits()
    lib().oracle_fill_two_levels_ex(_n(nf), _bc(bcf), _dp(d), sp, float(t), mp, _dp(Uf), _n(nc), _n(c0),
                                    _dp(Uc))
    return Uf


def average_down(nf, bcf, Uf, nc, c0, Uc, dirichlet=None):
    """AverageDown in place on Uc (covered coarse nodes = trapezoid average of the fine data over
    the coarse cell); refills the same-level ghosts of Uf first."""
    d = _dir(dirichlet)
    lib().oracle_average_down(_n(nf), _bc(bcf), _dp(d), _dp(Uf), _n(nc), _n(c0), _dp(Uc))
    return Uc


def _sibs(sibs):
    """[(offset (3), n (3), padded state)] -> ctypes arrays (offset = fine index of the sibling's
    node 0 in this patch's fine index space, 2 (c0_sibling - c0))."""
    k = len(sibs)
    so = (C.c_int64 * (3 * max(k, 1)))(*[int(x) for o, _, _ in sibs for x in o])
    sn = (C.c_int64 * (3 * max(k, 1)))(*[int(x) for _, n, _ in sibs for x in n])
    su = (C.POINTER(C.c_double) * max(k, 1))(*[_dp(U) for _, _, U in sibs])
    return k, so, sn, su


def fill_two_levels_sib(nf, bcf, Uf, nc, c0, Uc, sibs, dirichlet=None, met=None):
    """FillPatchTwoLevels with same-level siblings (reading 31): C/F ghosts inside a sibling's
    interior take the sibling's value, the others are interpolated from the coarse level."""
    k, so, sn, su = _sibs(sibs)
    mp = _dp(met) if met is not None else None
    lib().oracle_fill_two_levels_sib(_n(nf), _bc(bcf), _dp(_dir(dirichlet)), mp, _dp(Uf), _n(nc), _n(c0),
                                     _dp(Uc), k, so, sn, su)
    return Uf


def average_down_sib(nf, bcf, Uf, nc, c0, Uc, sibs, dirichlet=None):
    """AverageDown with same-level siblings (reading 31): nodes whose central fine node this patch
    owns and whose 27 fine nodes lie in the level's patch interiors."""
    k, so, sn, su = _sibs(sibs)
    lib().oracle_average_down_sib(_n(nf), _bc(bcf), _dp(_dir(dirichlet)), _dp(Uf), _n(nc), _n(c0), _dp(Uc),
                                  k, so, sn, su)
    return Uc


def amr_advance(nc, bcc, nf, bcf, c0, ph, dt, nsteps, Uc, metc, Uf, metf, dirc=None, dirf=None):
    """nsteps two-level RK3 steps (Alg. 2 with levels 0, 1 and AverageDown), in place on Uc, Uf."""
    lib().oracle_amr_advance(_n(nc), _bc(bcc), _dp(_dir(dirc)), _n(nf), _bc(bcf), _dp(_dir(dirf)),
                             _n(c0), C.byref(ph), float(dt), int(nsteps), _dp(Uc), _dp(metc),
                             _dp(Uf), _dp(metf))
    return Uc, Uf
