"""Convenience driver over the C ABI: allocates caller-owned device arrays with
torch per crocco_block_layout, uploads/downloads numpy padded arrays, and runs
RK3 steps (Algorithm 1/2 of the paper, without Regrid and
with a fixed dt).  Plumbing only -- every numerical step is a libcrocco kernel.
"""
from __future__ import annotations

import numpy as np
import torch

from . import crocco as cc

G = cc.GHOST
GC = cc.GHOST_COORDS


class Solver:
    def __init__(self, n_global, n_blocks=(1, 1, 1), bc=((0, 0),) * 3, phys=None, dirichlet=None,
                 rank=0, nranks=1, block_rank=None, device=None, stream=None, nccl_unique_id=None,
                 split=None):
        if not torch.cuda.is_available():
            raise RuntimeError("libcrocco needs a CUDA device (no CPU fallback)")
        if device is None:
            device = torch.device("cuda", torch.cuda.current_device())
        self.device = torch.device(device)
        if self.device.index is None:
            self.device = torch.device("cuda", torch.cuda.current_device())
        torch.cuda.set_device(self.device)
        self.stream = stream if stream is not None else torch.cuda.current_stream(self.device)
        self.phys = phys if phys is not None else cc.make_phys()
        self.desc = cc.make_desc(n_global, n_blocks, bc, dirichlet, rank, nranks, block_rank,
                                 self.stream.cuda_stream, nccl_unique_id, split)
        self.ctx = cc.crocco_init_grid(self.desc, self.phys)
        self.nloc = cc.crocco_num_local_blocks(self.ctx)
        self.layouts = [cc.crocco_get_block_layout(self.ctx, b) for b in range(self.nloc)]
        self.U = [self._alloc(L, 5) for L in self.layouts]
        self.V = [self._alloc(L, 5) for L in self.layouts]
        self.dU = [self._alloc(L, 5) for L in self.layouts]
        self.met = [self._alloc(L, 10) for L in self.layouts]
        self.rhs_buf = None

    # ------------------------------------------------------------ memory
    def _alloc(self, L, ncomp):
        return torch.zeros(ncomp * L.comp_stride, dtype=torch.float64, device=self.device)

    def view(self, buf, b, ncomp, coords=False):
        """(ncomp, P2, P1, P0) strided view of a block array (index [c, k+g, j+g, i+g])."""
        L = self.layouts[b]
        if coords:
            g, off, py, pz, cs = GC, L.coffset, L.cpitch_y, L.cpitch_z, L.ccomp_stride
        else:
            g, off, py, pz, cs = G, L.offset, L.pitch_y, L.pitch_z, L.comp_stride
        n = L.n
        return torch.as_strided(buf, (ncomp, n[2] + 2 * g, n[1] + 2 * g, n[0] + 2 * g),
                                (cs, pz, py, 1), off - g - g * py - g * pz)

    @staticmethod
    def _ptrs(bufs):
        return [t.data_ptr() for t in bufs]

    # ------------------------------------------------------------ setup
    def set_coords(self, xyz_blocks):
        """xyz_blocks[b]: (3, P2, P1, P0) numpy/torch on the coordinate band (g = 10); runs InitGridMetrics."""
        for b in range(self.nloc):
            self._stage_coords(b, xyz_blocks[b])
        self._init_metrics()

    def set_coords_block(self, b, xyz):
        """Stage one block's coordinates; InitGridMetrics runs once all blocks are staged."""
        self._stage_coords(b, xyz)
        if all(t is not None for t in self._coords):
            self._init_metrics()

    def _stage_coords(self, b, xyz):
        if not hasattr(self, "_coords") or self._coords is None:
            self._coords = [None] * self.nloc
        L = self.layouts[b]
        t = torch.zeros(3 * L.ccomp_stride, dtype=torch.float64, device=self.device)
        src = xyz if isinstance(xyz, torch.Tensor) else torch.from_numpy(np.ascontiguousarray(xyz))
        self.view(t, b, 3, coords=True).copy_(src)
        self._coords[b] = t

    def _init_metrics(self):
        cc.crocco_init_metrics(self.ctx, self._ptrs(self._coords), self._ptrs(self.met))
        if self.phys.visc_form == 1:     # expanded viscous form: the 18 second metrics
            cc.crocco_init_metrics2(self.ctx, self._ptrs(self.met))
        self.sync()
        self._coords = None

    def set_phys(self, phys):
        """Replace the gas / scheme constants (crocco_set_phys drops the cached step graphs);
        switching to the expanded viscous form computes the second metrics."""
        cc.crocco_set_phys(self.ctx, phys)
        self.phys = phys
        if phys.visc_form == 1:
            cc.crocco_init_metrics2(self.ctx, self._ptrs(self.met))

    def metrics2(self, b):
        """(18, n2, n1, n0) second metrics of local block b (expanded viscous form; tests)."""
        L = self.layouts[b]
        out = torch.empty((18, L.n[2], L.n[1], L.n[0]), dtype=torch.float64, device=self.device)
        cc.crocco_copy_metrics2(self.ctx, b, out.data_ptr())
        self.sync()
        return out

    def set_state(self, U_blocks, interior=True):
        """U_blocks[b]: numpy/torch conserved state, interior (5, n2, n1, n0) or padded."""
        for b in range(self.nloc):
            self.set_state_block(b, U_blocks[b], interior)

    def set_state_block(self, b, U, interior=True):
        v = self.view(self.U[b], b, 5)
        src = U if isinstance(U, torch.Tensor) else torch.from_numpy(np.ascontiguousarray(U))
        if interior:
            v[:, G:-G, G:-G, G:-G].copy_(src)
        else:
            v.copy_(src)

    def get(self, bufs, ncomp=5):
        return [self.view(bufs[b], b, ncomp).cpu().numpy() for b in range(self.nloc)]

    # ------------------------------------------------------------ hot path
    def fill(self, bufs=None, kind=cc.FIELD_STATE):
        cc.crocco_fill_boundary(self.ctx, self._ptrs(bufs if bufs is not None else self.U), kind,
                                self._ptrs(self.met) if kind == cc.FIELD_STATE else None)

    def set_time(self, t):
        cc.crocco_set_time(self.ctx, t)

    @property
    def time(self):
        return cc.crocco_get_time(self.ctx)

    def rhs(self):
        if self.rhs_buf is None:
            self.rhs_buf = [self._alloc(L, 5) for L in self.layouts]
        cc.crocco_rhs(self.ctx, self._ptrs(self.U), self._ptrs(self.met), self._ptrs(self.rhs_buf))
        return self.rhs_buf

    def stage(self, s, dt):
        cc.crocco_rk_stage(self.ctx, s, dt, self._ptrs(self.U), self._ptrs(self.V),
                           self._ptrs(self.dU), self._ptrs(self.met))
        self.U, self.V = self.V, self.U

    def step(self, dt, nsteps=1, graph=True):
        """nsteps full RK3 steps (crocco_rk3_step; one CUDA-graph launch per step)."""
        for _ in range(nsteps):
            cc.crocco_rk3_step(self.ctx, dt, self._ptrs(self.U), self._ptrs(self.V),
                               self._ptrs(self.dU), self._ptrs(self.met), graph)
            self.U, self.V = self.V, self.U

    def steps_from_host(self, h_in, h_out, dt, interior=False):
        """Independent RK3 steps streamed through pinned host memory: job n's padded state is
        uploaded from h_in[n] (list over local blocks of flat pinned float64 tensors sized like
        the state arrays), advanced one RK3 step and downloaded into h_out[n].  Uploads and
        downloads run on their own copy streams, so job n's download and job n+1's upload
        overlap the compute of the neighbouring jobs (two device state pairs alternate).
        interior=True: the host tensors hold only the interior points, (5, n2, n1, n0) per
        block (the ghosts are the step's own fill), 9 % fewer bytes over the host link at 512^3;
        the copies go through contiguous device staging (torch).
        Plumbing only: the step itself is crocco_rk3_step."""
        def dev_view(buf, b):
            v = self.view(buf, b, 5)
            return v[:, G:-G, G:-G, G:-G] if interior else buf

        def host_view(h, b):
            n = self.layouts[b].n
            return h.view(5, n[2], n[1], n[0]) if interior else h
        if not hasattr(self, "_pairs"):
            self._pairs = [(self.U, self.V), ([self._alloc(L, 5) for L in self.layouts],
                                              [self._alloc(L, 5) for L in self.layouts])]
            self._h2d = torch.cuda.Stream(self.device)
            self._d2h = torch.cuda.Stream(self.device)
        comp = self.stream
        e0 = torch.cuda.Event()
        e0.record(comp)                                        # earlier work on the buffers
        self._h2d.wait_event(e0)
        self._d2h.wait_event(e0)
        ev_c, ev_d = {}, {}
        for n in range(len(h_in)):
            X, Y = self._pairs[n % 2]
            with torch.cuda.stream(self._h2d):
                if n - 2 in ev_c:
                    self._h2d.wait_event(ev_c[n - 2])          # X clobbered by job n-2's stages
                for b, (h, x) in enumerate(zip(h_in[n], X)):
                    dev_view(x, b).copy_(host_view(h, b), non_blocking=True)
                eh = torch.cuda.Event()
                eh.record(self._h2d)
            comp.wait_event(eh)
            if n - 2 in ev_d:
                comp.wait_event(ev_d[n - 2])                   # Y still being downloaded
            cc.crocco_rk3_step(self.ctx, dt, self._ptrs(X), self._ptrs(Y), self._ptrs(self.dU),
                               self._ptrs(self.met), True)
            ev_c[n] = torch.cuda.Event()
            ev_c[n].record(comp)
            with torch.cuda.stream(self._d2h):
                self._d2h.wait_event(ev_c[n])
                for b, (h, y) in enumerate(zip(h_out[n], Y)):
                    host_view(h, b).copy_(dev_view(y, b), non_blocking=True)
                ev_d[n] = torch.cuda.Event()
                ev_d[n].record(self._d2h)
        comp.wait_stream(self._d2h)

    def check_state(self):
        """Number of interior points with a non-finite value, rho <= 0 or p <= 0 (crocco_check_state)."""
        return cc.crocco_check_state(self.ctx, self._ptrs(self.U))

    def compute_dt(self, cfl):
        """ComputeDt (Alg. 1 l.9): CFL time step of the current state (synchronises)."""
        return cc.crocco_compute_dt(self.ctx, self._ptrs(self.U), self._ptrs(self.met), cfl)

    def set_phys(self, phys):
        switch = phys.visc_form == 1 and self.phys.visc_form != 1
        self.phys = phys
        cc.crocco_set_phys(self.ctx, phys)
        if switch:
            cc.crocco_init_metrics2(self.ctx, self._ptrs(self.met))

    def sync(self):
        cc.crocco_sync(self.ctx)

    def close(self):
        if self.ctx is not None:
            cc.crocco_finalize(self.ctx)
            self.ctx = None

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass


class AmrSolver:
    """Two-level hierarchy (DESIGN readings 24-26): a coarse Solver and one or
    more fine patches (Solvers whose faces inside the coarse domain are BC_COARSE_FINE), patch p's
    fine node 0 at coarse node c0[p] (ratio 2, node-centred).  step() follows Algorithm 2
    (PAPER.md:102-119): per stage the coarse level, then every patch of the fine level with its
    C/F ghosts interpolated from the coarse stage input, then AverageDown at the third stage.
    Patches of the same level must have disjoint interiors; patches whose 4-point ghost band
    reaches into another patch's interior (abutting or nearby patches) are linked as siblings
    (crocco_amr_link_sibling, reading 31): their C/F ghosts inside a sibling take the sibling's
    stage input, and AverageDown covers the nodes whose cell lies in the union of the level's
    patches.  Plumbing only -- the C ABI does every step."""

    def __init__(self, coarse: Solver, fine, c0):
        fines = list(fine) if isinstance(fine, (list, tuple)) else [fine]
        c0s = [tuple(int(x) for x in c) for c in c0] if isinstance(fine, (list, tuple)) else \
            [tuple(int(x) for x in c0)]
        if len(fines) != len(c0s):
            raise ValueError("one c0 per fine patch")
        self.coarse = coarse
        self.patches = list(zip(fines, c0s))
        self.fine, self.c0 = self.patches[0]
        pairs = self._sibling_pairs()
        for F, c in self.patches:
            cc.crocco_amr_link(F.ctx, coarse.ctx, c)
        self.sibs = [[] for _ in self.patches]   # per patch, sibling indices in link order
        for a, b in pairs:
            cc.crocco_amr_link_sibling(self.patches[a][0].ctx, self.patches[b][0].ctx)
            self.sibs[a].append(b)
            self.sibs[b].append(a)

    def _box(self, F, c, grow):
        """Fine-level index box [lo, hi) of a patch in the common fine index space (2x coarse);
        a direction a PERIODIC patch spans is the whole axis (None)."""
        out = []
        for d in range(3):
            if F.desc.bc[d][0] == cc.BC_PERIODIC:
                out.append(None)
            else:
                out.append((2 * c[d] - grow, 2 * c[d] + F.desc.n_global[d] + grow))
        return out

    def _sibling_pairs(self):
        """Pairs of patches whose ghost bands reach into each other's interior (siblings);
        overlapping interiors are refused."""
        G4 = cc.GHOST

        def meets(A, B):
            return all(x is None or y is None or (x[0] < y[1] and y[0] < x[1]) for x, y in zip(A, B))

        pairs = []
        for a in range(len(self.patches)):
            for b in range(a + 1, len(self.patches)):
                if meets(self._box(*self.patches[a], 0), self._box(*self.patches[b], 0)):
                    raise ValueError(f"fine patches {a} and {b} overlap")
                if meets(self._box(*self.patches[a], G4), self._box(*self.patches[b], 0)) or \
                        meets(self._box(*self.patches[b], G4), self._box(*self.patches[a], 0)):
                    pairs.append((a, b))
        return pairs

    def _sib_ptrs(self, i, states):
        return [states[j] for j in self.sibs[i]]

    def fill_fine(self):
        """FillPatchTwoLevels of every patch's current state from the current coarse state
        (and its siblings' current states)."""
        cur = [F._ptrs(F.U) for F, _ in self.patches]
        for i, (F, _) in enumerate(self.patches):
            cc.crocco_fill_patch_level(F.ctx, F._ptrs(F.U), F._ptrs(F.met), self.coarse._ptrs(self.coarse.U),
                                       self._sib_ptrs(i, cur))

    def average_down(self):
        cur = [F._ptrs(F.U) for F, _ in self.patches]
        for i, (F, _) in enumerate(self.patches):
            cc.crocco_average_down_level(F.ctx, F._ptrs(F.U), self.coarse._ptrs(self.coarse.U),
                                         self._sib_ptrs(i, cur))

    def stage(self, s, dt):
        C = self.coarse
        Uc_in = C.U
        C.stage(s, dt)                                   # fills Uc_in's ghosts, writes C.V; swaps
        ins = [F._ptrs(F.U) for F, _ in self.patches]    # every patch's stage input
        for i, (F, _) in enumerate(self.patches):
            cc.crocco_amr_rk_stage_level(F.ctx, s, dt, F._ptrs(F.U), F._ptrs(F.V), F._ptrs(F.dU),
                                         F._ptrs(F.met), C._ptrs(Uc_in), self._sib_ptrs(i, ins))
        for F, _ in self.patches:
            F.U, F.V = F.V, F.U
        if s == 2:
            self.average_down()

    def step(self, dt, nsteps=1):
        for _ in range(nsteps):
            for s in range(3):
                self.stage(s, dt)
            self.coarse.set_time(self.coarse.time + dt)
            for F, _ in self.patches:
                F.set_time(F.time + dt)

    def sync(self):
        self.coarse.sync()
        for F, _ in self.patches:
            F.sync()


class AmrHierarchy:
    """Multi-level hierarchy (the paper's DMR runs "three-level curvilinear AMR", PAPER.md:195;
    SURVEY NEXT-4; DESIGN readings 24-26, 29).  levels[0] is the base Solver; levels[k] (k >= 1)
    is a list of (Solver, parent, c0): a patch of level k whose fine node 0 sits at node c0 of
    patch `parent` of level k-1 (ratio 2 between consecutive levels; the base level has the
    single "patch" 0).  A level-k patch is an ordinary fine ctx whose coarse level is its
    parent -- crocco_amr_link composes, since the parent's ghosts (its own C/F faces included)
    are filled by the parent's stage before the child interpolates from them.
    stage() follows Algorithm 2 literally: for each level n = 0..nlevels in
    ascending order, FillPatch + RHS + Update of every patch of level n, and at the third stage
    AverageDown of level n onto level n-1 right after level n's update (reading 29)."""

    def __init__(self, base: Solver, levels):
        self.levels = [[(base, None, None)]] + [list(lv) for lv in levels]
        self.sibs = [[[]]]
        for k in range(1, len(self.levels)):
            for S, parent, c0 in self.levels[k]:
                P = self.levels[k - 1][parent][0]
                cc.crocco_amr_link(S.ctx, P.ctx, tuple(int(x) for x in c0))
            # patches of one level under the same parent whose ghost bands meet: siblings (reading 31)
            lv = self.levels[k]
            sib = [[] for _ in lv]
            for parent in sorted({p for _, p, _ in lv}):
                idx = [i for i, (_, p, _) in enumerate(lv) if p == parent]
                tmp = AmrSolver.__new__(AmrSolver)
                tmp.patches = [(lv[i][0], tuple(int(x) for x in lv[i][2])) for i in idx]
                for a, b in tmp._sibling_pairs():
                    cc.crocco_amr_link_sibling(lv[idx[a]][0].ctx, lv[idx[b]][0].ctx)
                    sib[idx[a]].append(idx[b])
                    sib[idx[b]].append(idx[a])
            self.sibs.append(sib)

    def stage(self, s, dt):
        prev_in = None
        for k, lv in enumerate(self.levels):
            cur_in = [S._ptrs(S.U) for S, _, _ in lv]     # every patch's stage input
            for i, (S, parent, _) in enumerate(lv):
                if k == 0:
                    S.stage(s, dt)                       # fills U_in's ghosts, writes S.V; swaps
                else:
                    cc.crocco_amr_rk_stage_level(S.ctx, s, dt, S._ptrs(S.U), S._ptrs(S.V), S._ptrs(S.dU),
                                                 S._ptrs(S.met), prev_in[parent],
                                                 [cur_in[j] for j in self.sibs[k][i]])
            if k >= 1:
                for S, _, _ in lv:
                    S.U, S.V = S.V, S.U
            if s == 2 and k >= 1:                        # AverageDown of level k onto level k-1
                cur = [S._ptrs(S.U) for S, _, _ in lv]
                for i, (S, parent, _) in enumerate(lv):
                    P = self.levels[k - 1][parent][0]
                    cc.crocco_average_down_level(S.ctx, S._ptrs(S.U), P._ptrs(P.U),
                                                 [cur[j] for j in self.sibs[k][i]])
            prev_in = cur_in

    def step(self, dt, nsteps=1):
        for _ in range(nsteps):
            for s in range(3):
                self.stage(s, dt)
            for lv in self.levels:
                for S, _, _ in lv:
                    S.set_time(S.time + dt)

    def compute_dt(self, cfl):
        """ComputeDt over the whole hierarchy (Alg. 1 l.9; every patch iterates with the same dt,
        PAPER.md:131): the minimum of every patch's crocco_compute_dt."""
        return min(S.compute_dt(cfl) for lv in self.levels for S, _, _ in lv)

    def sync(self):
        for lv in self.levels:
            for S, _, _ in lv:
                S.sync()
