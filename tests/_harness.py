"""Shared test harness: builds the same seeded inputs for the oracle (global
grid, one block) and for the CUDA path (any block decomposition), and the
parity metric of DESIGN.md sec. 3 reading 17.  Test infrastructure only.
"""
from __future__ import annotations

import numpy as np

import oracle
import synth

G = 4


def inner(a, g=G):
    return a[:, g:-g, g:-g, g:-g]


def block_slices(n_global, n_blocks):
    """Global interior slices (k, j, i) of every block in gid order."""
    bn = [n_global[d] // n_blocks[d] for d in range(3)]
    out = []
    for bz in range(n_blocks[2]):
        for by in range(n_blocks[1]):
            for bx in range(n_blocks[0]):
                o = (bx * bn[0], by * bn[1], bz * bn[2])
                out.append((o, (slice(o[2], o[2] + bn[2]), slice(o[1], o[1] + bn[1]),
                                slice(o[0], o[0] + bn[0]))))
    return bn, out


def flux_scale(U, met, gamma=1.4):
    """max_i J |m| max|F| over interior points (floor of the parity metric, reading 17)."""
    J = inner(met)[0]
    m = np.sqrt((inner(met)[1:] ** 2).reshape(3, 3, *J.shape).sum(1)).max(0)
    Ui = inner(U)
    rho = Ui[0]
    vel = Ui[1:4] / rho
    p = (gamma - 1) * (Ui[4] - 0.5 * rho * (vel ** 2).sum(0))
    sp = np.abs(vel).max(0)
    F = np.abs(Ui[1:4]).max(0) * sp + np.abs(p) + np.abs(Ui[4] + p) * sp + np.abs(rho) * sp
    return float((J * m * F).max())


def state_scale(Ui, gamma=1.4):
    """max_i rho_i (|u_i| + c_i): the momentum scale used as the parity floor for
    state comparisons where a component is identically ~0 (e.g. transverse
    momentum of the 1-D Sod problem)."""
    rho = Ui[0]
    vel = Ui[1:4] / rho
    p = (gamma - 1) * (Ui[4] - 0.5 * rho * (vel ** 2).sum(0))
    c = np.sqrt(np.abs(gamma * p / rho))
    return float((rho * (np.sqrt((vel ** 2).sum(0)) + c)).max())


def rel_linf(got, ref, floor=0.0):
    """Per component max|got-ref| / max(max|ref|, floor); returns the max over components."""
    got = np.asarray(got)
    ref = np.asarray(ref)
    worst = 0.0
    for c in range(ref.shape[0]):
        den = max(np.abs(ref[c]).max(), floor, 1e-300)
        worst = max(worst, float(np.abs(got[c] - ref[c]).max() / den))
    return worst


class Problem:
    """A global problem: grid object, BCs, initial interior state (global)."""

    def __init__(self, n, grid, bc, U_interior, phys_kw=None, dirichlet=None, split=None):
        self.n = tuple(n)
        self.grid = grid
        self.bc = bc
        self.U0 = U_interior
        self.phys_kw = dict(phys_kw or {})
        self.dirichlet = dirichlet
        self.split = split  # {(d, side): spec} for SPLIT faces

    # ---------------- oracle side (global single block)
    def oracle_inputs(self):
        xyz = self.grid.coords(self.n, (0, 0, 0), oracle.GC)
        met = oracle.metrics(self.n, self.bc, xyz)
        U = synth.pad_state(self.U0)
        oracle.fill(self.n, self.bc, U, dirichlet=self.dirichlet, split=self.oracle_split(), met=met)
        return xyz, met, U

    def oracle_split(self):
        return oracle.splits(self.split) if self.split else None

    def oracle_phys(self):
        return oracle.phys(**self.phys_kw)

    # ---------------- GPU side
    def solver(self, n_blocks=(1, 1, 1), stream=None):
        from paper_conf_ipps_davissngmb23_b200 import crocco as cc
        from paper_conf_ipps_davissngmb23_b200.solver import Solver
        kw = dict(self.phys_kw)
        kw.pop("weno_linear", None)  # oracle-only test flag
        S = Solver(self.n, n_blocks, self.bc, cc.make_phys(**kw), dirichlet=self.dirichlet,
                   split=self.split, stream=stream)
        bn, blocks = block_slices(self.n, n_blocks)
        xyz = [self.grid.coords(bn, o, oracle.GC) for o, _ in blocks]
        S.set_coords(xyz)
        S.set_state([np.ascontiguousarray(self.U0[(slice(None),) + sl]) for _, sl in blocks])
        S.blocks = blocks
        return S

    def gather(self, S, arrays):
        """Stitch per-block interiors back into a global interior array."""
        out = np.zeros((arrays[0].shape[0],) + tuple(self.n[::-1]))
        for (o, sl), a in zip(S.blocks, arrays):
            out[(slice(None),) + sl] = inner(a)
        return out
