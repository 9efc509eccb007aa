"""Pins of the oracle's two-level AMR functions (oracle section 9;
DESIGN.md readings 24-26) against what the paper and the mathematics fix:

- FillPatchTwoLevels (trilinear, ratio 2, node-centred): reproduces every
  multilinear field exactly (with dyadic data the fp result is exact), interpolates x^2 at a
  halfway point to x^2 + 1/4 (linear, not higher order), copies coincident nodes, leaves the
  fine interior untouched;
- AverageDown ("average of the covering fine cells"): exact for linear fields,
  x^2 -> x^2 + 1/8 per direction (trapezoid rule over the coarse cell), the covered set, and the
  periodic conservation identity sum_c = sum_f / 8;
- the two-level RK3 advance: free-stream preservation across the coarse/fine interface on a
  wavy grid; with a fine level covering the whole periodic domain it reduces exactly to the
  single-level advance of the fine grid (and the coarse level to its full-weighting average);
  an isentropic vortex is resolved more accurately on the fine patch than on the coarse grid.
CPU only.
"""
import numpy as np
import pytest

import oracle
import synth

G = 4
CF = oracle.COARSE_FINE
PER = ((0, 0),) * 3


def _pad_index(n, origin, scale=1.0):
    """Index arrays over the padded box (ghost 4) at positions origin + scale * local."""
    ax = [origin[d] + scale * np.arange(-G, n[d] + G, dtype=np.float64) for d in range(3)]
    return ax[0][None, None, :], ax[1][None, :, None], ax[2][:, None, None]


def _multilinear(X, Y, Z, coef):
    a, b, c, d, e, f, g, h = coef
    return a + b * X + c * Y + d * Z + e * X * Y + f * Y * Z + g * X * Z + h * X * Y * Z


def _coarse_field(nc, fn):
    X, Y, Z = _pad_index(nc, (0, 0, 0))
    U = np.zeros((5, nc[2] + 2 * G, nc[1] + 2 * G, nc[0] + 2 * G))
    for q in range(5):
        U[q] = np.broadcast_to(fn(q, X, Y, Z), U[q].shape)
    return U


def _ghost_mask(nf):
    m = np.ones((nf[2] + 2 * G, nf[1] + 2 * G, nf[0] + 2 * G), bool)
    m[G:-G, G:-G, G:-G] = False
    return m


COEF = [(3, 1, -2, 1, 1, -1, 2, 1), (1, 0, 0, 0, 0, 0, 0, 0), (-2, 2, 1, 3, 0, 1, -1, 0),
        (5, -1, 1, 1, 2, 0, 0, -1), (0, 0, 0, 1, 1, 1, 1, 1)]


@pytest.mark.parametrize("c0", [(3, 2, 4), (2, 3, 2)])
def test_interp_reproduces_multilinear_fields(c0):
    nc = (14, 12, 13)
    nf = (10, 12, 8)
    Uc = _coarse_field(nc, lambda q, X, Y, Z: _multilinear(X, Y, Z, COEF[q]))
    Uf = np.full((5, nf[2] + 2 * G, nf[1] + 2 * G, nf[0] + 2 * G), 7.25)
    oracle.fill_two_levels(nf, ((CF, CF),) * 3, Uf, nc, c0, Uc)
    Xf, Yf, Zf = _pad_index(nf, c0, 0.5)
    m = _ghost_mask(nf)
    for q in range(5):
        exact = np.broadcast_to(_multilinear(Xf, Yf, Zf, COEF[q]), m.shape)
        assert np.array_equal(Uf[q][m], exact[m]), q           # every ghost, edges and corners
        assert np.all(Uf[q][~m] == 7.25)                          # interior untouched


def test_interp_is_linear_halfway():
    """x^2 at a fine node halfway between two coarse nodes -> x^2 + 1/4 (coarse index units);
    coincident nodes are copies.  A cubic or WENO interpolant would give x^2 exactly."""
    nc = (16, 10, 10)
    c0 = (4, 3, 3)
    nf = (8, 8, 6)
    Uc = _coarse_field(nc, lambda q, X, Y, Z: X * X + 0 * Y * Z + q)
    Uf = np.zeros((5, nf[2] + 2 * G, nf[1] + 2 * G, nf[0] + 2 * G))
    oracle.fill_two_levels(nf, ((CF, CF), (0, 0), (0, 0)), Uf, nc, c0, Uc)
    # xi ghosts at interior j, k (periodic eta/zeta phases copy them further)
    for gi, f in [(0, -4), (1, -3), (2, -2), (3, -1)]:
        X = c0[0] + 0.5 * f
        want = X * X + (0.25 if f % 2 else 0.0)
        assert np.all(Uf[2, G:-G, G:-G, gi] == want + 2)


@pytest.mark.parametrize("c0", [(2, 3, 1), (3, 2, 2)])
def test_average_down_linear_exact_and_covered_set(c0):
    nc = (12, 12, 10)
    nf = (12, 10, 11)
    bcf = ((CF, CF),) * 3
    Xf, Yf, Zf = _pad_index(nf, c0, 0.5)
    Uf = np.zeros((5, nf[2] + 2 * G, nf[1] + 2 * G, nf[0] + 2 * G))
    for q in range(5):
        Uf[q] = np.broadcast_to(1.0 + 2 * Xf - Yf + 3 * Zf + q * Xf * Xf * 0, Uf[q].shape)
    Uf[3] = np.broadcast_to(Xf * Xf + Yf * Yf + Zf * Zf, Uf[3].shape)
    Uc = np.full((5, nc[2] + 2 * G, nc[1] + 2 * G, nc[0] + 2 * G), -99.0)
    oracle.average_down(nf, bcf, Uf, nc, c0, Uc)
    X, Y, Z = _pad_index(nc, (0, 0, 0))
    cov = np.zeros(Uc.shape[1:], bool)
    rng = [range(c0[d] + 1, c0[d] + (nf[d] - 2) // 2 + 1) for d in range(3)]
    for k in rng[2]:
        for j in rng[1]:
            for i in rng[0]:
                cov[k + G, j + G, i + G] = True
    assert cov.sum() == np.prod([len(r) for r in rng]) > 0
    lin = np.broadcast_to(1.0 + 2 * X - Y + 3 * Z, cov.shape)
    assert np.array_equal(Uc[0][cov], lin[cov])
    quad = np.broadcast_to(X * X + Y * Y + Z * Z + 3.0 / 8.0, cov.shape)   # trapezoid: +1/8 per direction
    assert np.array_equal(Uc[3][cov], quad[cov])
    assert np.all(Uc[:, ~cov] == -99.0)


def test_average_down_periodic_conservation():
    nc = (8, 6, 10)
    nf = tuple(2 * x for x in nc)
    rng = np.random.default_rng(11)
    Uf = synth.pad_state(rng.uniform(0.5, 1.5, (5, nf[2], nf[1], nf[0])))
    Uc = np.zeros((5, nc[2] + 2 * G, nc[1] + 2 * G, nc[0] + 2 * G))
    oracle.average_down(nf, PER, Uf, nc, (0, 0, 0), Uc)
    ci = Uc[:, G:-G, G:-G, G:-G]
    fi = Uf[:, G:-G, G:-G, G:-G]
    assert np.all(ci != 0.0)                                      # every coarse node covered
    np.testing.assert_allclose(ci.sum(axis=(1, 2, 3)), fi.sum(axis=(1, 2, 3)) / 8.0, rtol=1e-13)
    # the coarse node coincident with fine node (2, 4, 6): explicit 27-point average
    i, j, k = 1, 2, 3
    w = np.array([0.25, 0.5, 0.25])
    blk = Uf[:, G + 2 * k - 1:G + 2 * k + 2, G + 2 * j - 1:G + 2 * j + 2, G + 2 * i - 1:G + 2 * i + 2]
    want = np.einsum("qcba,c,b,a->q", blk, w, w, w)
    np.testing.assert_allclose(Uc[:, G + k, G + j, G + i], want, rtol=1e-15)


def _two_level(grid_c, nc, bcc, c0, nf, bcf, state_fn, ph):
    xc = grid_c.coords(nc, (0, 0, 0), oracle.GC)
    metc = oracle.metrics(nc, bcc, xc)
    Uc = synth.pad_state(state_fn(xc))
    gf = synth.Refined(grid_c, c0)
    xf = gf.coords(nf, (0, 0, 0), oracle.GC)
    metf = oracle.metrics(nf, bcf, xf)
    Uf = synth.pad_state(state_fn(xf))
    return xc, metc, Uc, xf, metf, Uf


def test_two_level_free_stream_preserved():
    nc = (16, 16, 16)
    grid = synth.Wavy3D(L=(10.0,) * 3, N=nc)
    c0 = (4, 5, 3)
    nf = (14, 12, 16)
    bcf = ((CF, CF),) * 3
    ph = oracle.phys(terms=3, mu_ref=0.01)
    xc, metc, Uc, xf, metf, Uf = _two_level(grid, nc, PER, c0, nf, bcf, synth.free_stream, ph)
    U0 = synth.free_stream(xc)[:, 0, 0, 0]
    oracle.amr_advance(nc, PER, nf, bcf, c0, ph, 0.02, 2, Uc, metc, Uf, metf)
    for U in (Uc, Uf):
        dev = np.abs(U[:, G:-G, G:-G, G:-G] - U0[:, None, None, None]).max(axis=(1, 2, 3))
        assert np.all(dev <= 1e-12 * np.abs(U0).max()), dev


def test_two_level_full_cover_reduces_to_single_level():
    """Fine level = the whole periodic domain: no C/F faces, so its evolution is the
    single-level advance of the fine grid bit for bit, and the coarse level ends as the
    full-weighting average of the fine state."""
    nc = (8, 8, 6)
    nf = tuple(2 * x for x in nc)
    grid = synth.Wavy3D(L=(10.0,) * 3, N=nc)
    ph = oracle.phys(terms=3, mu_ref=0.02)
    st = lambda x: synth.vortex(x)
    xc, metc, Uc, xf, metf, Uf = _two_level(grid, nc, PER, (0, 0, 0), nf, PER, st, ph)
    Uf1 = Uf.copy()
    oracle.amr_advance(nc, PER, nf, PER, (0, 0, 0), ph, 0.01, 2, Uc, metc, Uf, metf)
    oracle.advance(nf, PER, ph, 0.01, 2, Uf1, metf)
    assert np.array_equal(Uf[:, G:-G, G:-G, G:-G], Uf1[:, G:-G, G:-G, G:-G])
    Uc2 = np.zeros_like(Uc)
    oracle.average_down(nf, PER, Uf1, nc, (0, 0, 0), Uc2)
    assert np.array_equal(Uc[:, G:-G, G:-G, G:-G], Uc2[:, G:-G, G:-G, G:-G])


def test_two_level_vortex_more_accurate_on_fine_patch():
    """Shu vortex (quasi-2D wavy grid, periodic) advected to t = 1 with a fine patch around its
    path: the fine-level error against the translated closed form is well below the error of
    the same coarse grid run without refinement, at the same (coincident) points."""
    nc = (32, 32, 4)
    grid = synth.Wavy2D(N=nc)
    c0 = (8, 8, 0)
    nf = (34, 34, 8)
    bcf = ((CF, CF), (CF, CF), (0, 0))
    ph = oracle.phys(terms=1)
    dt, nsteps = 0.025, 40
    st = lambda x: synth.vortex(x)
    xc, metc, Uc, xf, metf, Uf = _two_level(grid, nc, PER, c0, nf, bcf, st, ph)
    Uc1 = Uc.copy()
    oracle.amr_advance(nc, PER, nf, bcf, c0, ph, dt, nsteps, Uc, metc, Uf, metf)
    oracle.fill(nc, PER, Uc1)
    oracle.advance(nc, PER, ph, dt, nsteps, Uc1, metc)
    t = dt * nsteps
    fi = range(2, nf[0] - 2, 2)                       # even fine interior nodes away from the C/F faces
    fj = range(2, nf[1] - 2, 2)
    ci = slice(c0[0] + fi[0] // 2, c0[0] + fi[-1] // 2 + 1)   # the coincident coarse nodes
    cj = slice(c0[1] + fj[0] // 2, c0[1] + fj[-1] // 2 + 1)
    fsl = (0, slice(None, None, 2), slice(fj[0], fj[-1] + 1, 2), slice(fi[0], fi[-1] + 1, 2))
    csl = (0, slice(None), cj, ci)
    exf = synth.vortex(xf, t=t)
    exc = synth.vortex(xc, t=t)
    err_fine = np.abs(Uf[:, G:-G, G:-G, G:-G][fsl] - exf[fsl]).max()
    err_coarse = np.abs(Uc1[:, G:-G, G:-G, G:-G][csl] - exc[csl]).max()
    err_comp = np.abs(Uc[:, G:-G, G:-G, G:-G][csl] - exc[csl]).max()
    assert exf[fsl].shape == exc[csl].shape
    assert err_fine < 0.5 * err_coarse, (err_fine, err_coarse)
    assert err_comp < err_coarse, (err_comp, err_coarse)


def test_refined_dmr_split_faces_follow_the_physical_rule():
    """DMR boundary data on a fine patch at the bottom wall (synth.refine_bc, reading 20 + 24): the
    fine bottom ghosts take the post-shock state exactly where the ghost's physical x < 1/6 (the
    coarse rule re-expressed in the fine index space), slip-wall reflections elsewhere; the top
    face inside the domain is C/F."""
    n = (96, 32, 4)
    h = 1.0 / n[1]
    bc, dv, spec = synth.dmr_bc(h)
    grid = synth.Cartesian(h=(h,) * 3)
    c0, nf = (2, 0, 0), (40, 20, 8)
    bcf, dirf, splf = synth.refine_bc(n, bc, dv, spec, c0, nf)
    assert bcf == ((CF, CF), (synth.SPL, CF), (0, 0))
    xf = synth.Refined(grid, c0).coords(nf, (0, 0, 0), oracle.GC)
    metf = oracle.metrics(nf, bcf, xf)
    Uf = synth.pad_state(synth.random_state(nf, seed=12))
    Uc = synth.pad_state(synth.random_state(n, seed=13))
    oracle.fill(n, bc, Uc, dirichlet=dv, split=oracle.splits(spec), met=oracle.metrics(n, bc, grid.coords(n, (0, 0, 0), oracle.GC)))
    oracle.fill_two_levels(nf, bcf, Uf, n, c0, Uc, dirichlet=dirf, met=metf, split=oracle.splits(splf), t=0.0)
    post = np.array(synth.prim_to_cons(*[np.float64(a) for a in synth.DMR_POST]))
    x = (c0[0] + 0.5 * np.arange(-G, nf[0] + G) + 0.5) * h      # physical x of the fine columns
    for g in range(1, G + 1):                                      # bottom ghost rows j = -g
        row = Uf[:, G:-G, G - g, :]                                # (5, k, i)
        is_post = np.all(np.isclose(row, post[:, None, None], rtol=0, atol=0), axis=(0, 1))
        assert np.array_equal(is_post[G:-G], x[G:-G] < 1.0 / 6.0)
        mirror = Uf[:, G:-G, G + g - 1, :]
        slip = ~(x < 1.0 / 6.0)
        assert np.array_equal(row[0][:, slip], mirror[0][:, slip])                 # rho mirrored
        assert np.array_equal(row[2][:, slip], -mirror[2][:, slip])                # v reflected


# ------------------------------------------------------------------ same-level siblings (reading 31)

def advance_level(nc, metc, Uc, patches, ph, dt, nsteps):
    """Algorithm 2 on a periodic coarse level + one fine level of patches,
    composed from the oracle functions: per stage the coarse stage, every patch's FillPatch (C/F
    ghosts inside a sibling patch copied from the sibling's stage input -- FillBoundary,
    PAPER.md:129 -- the others interpolated), RHS, update; AverageDown of every patch at the third
    stage.  patches: list of dicts c0, nf, metf, U (padded, updated in place).  Test helper; the
    arithmetic is the oracle's."""
    bcf = ((CF, CF),) * 3
    ac, oc, dUc = Uc, Uc.copy(), np.zeros_like(Uc)
    st = [dict(a=p["U"], o=p["U"].copy(), dU=np.zeros_like(p["U"])) for p in patches]

    def sibs(i, key):
        p = patches[i]
        return [(tuple(2 * (q["c0"][d] - p["c0"][d]) for d in range(3)), q["nf"], st[j][key])
                for j, q in enumerate(patches) if j != i]

    for _ in range(nsteps):
        for s in range(3):
            oracle.rk_stage(nc, PER, ph, s, dt, ac, oc, dUc, metc)
            for i, p in enumerate(patches):
                oracle.fill_two_levels_sib(p["nf"], bcf, st[i]["a"], nc, p["c0"], ac, sibs(i, "a"))
            for i, p in enumerate(patches):
                r = oracle.rhs(p["nf"], ph, st[i]["a"], p["metf"])
                oracle.rk_update(p["nf"], s, dt, st[i]["a"], st[i]["o"], st[i]["dU"], r)
            if s == 2:
                for i, p in enumerate(patches):
                    oracle.average_down_sib(p["nf"], bcf, st[i]["o"], nc, p["c0"], oc, sibs(i, "o"))
            for x in st:
                x["a"], x["o"] = x["o"], x["a"]
            ac, oc = oc, ac
    for p, x in zip(patches, st):
        p["U"][...] = x["a"]
    Uc[...] = ac
    return Uc


def _level_setup(nc, grid, specs, state):
    bcf = ((CF, CF),) * 3
    xc = grid.coords(nc, (0, 0, 0), oracle.GC)
    metc = oracle.metrics(nc, PER, xc)
    Uc = synth.pad_state(state(xc))
    P = []
    for c0, nf in specs:
        xf = synth.Refined(grid, c0).coords(nf, (0, 0, 0), oracle.GC)
        P.append(dict(c0=c0, nf=nf, metf=oracle.metrics(nf, bcf, xf), U=synth.pad_state(state(xf))))
    return metc, Uc, P


@pytest.mark.parametrize("axis", [0, 1, 2])
def test_abutting_patches_equal_their_union_bitwise(axis):
    """Reading 31: two abutting fine patches (each other's siblings) advance exactly like the one
    patch covering their union -- fine states on the union and the coarse state bit for bit, over
    3 RK3 steps of a viscous vortex flow -- because a C/F ghost inside the sibling takes the
    sibling's value (the union's interior value), every other C/F ghost is interpolated at the
    same position, and AverageDown covers exactly the union's covered set."""
    nc = (16, 16, 16)
    grid = synth.Wavy3D(L=(10.0,) * 3, N=nc)
    ph = oracle.phys(terms=3, mu_ref=0.01)
    c0, nu = (3, 4, 2), [16, 16, 12]   # halves even: a patch starts at an even fine index
    half = [nu[d] // 2 if d == axis else nu[d] for d in range(3)]
    c0b = tuple(c0[d] + (half[d] // 2 if d == axis else 0) for d in range(3))
    metc, Uu, Pu = _level_setup(nc, grid, [(c0, tuple(nu))], lambda x: synth.vortex(x))
    metc2, Us, Ps = _level_setup(nc, grid, [(c0, tuple(half)), (c0b, tuple(half))], lambda x: synth.vortex(x))
    assert np.array_equal(metc, metc2)
    # the two halves' fine metrics are the union's (same coordinates)
    sl = [slice(G, -G)] * 3
    su = list(sl)
    su[2 - axis] = slice(G, G + half[axis])
    assert np.array_equal(Pu[0]["metf"][(slice(None),) + tuple(su)], Ps[0]["metf"][:, G:-G, G:-G, G:-G])
    advance_level(nc, metc, Uu, Pu, ph, 0.01, 3)
    advance_level(nc, metc, Us, Ps, ph, 0.01, 3)
    assert np.array_equal(Uu, Us)
    union = Pu[0]["U"][:, G:-G, G:-G, G:-G]
    parts = [P["U"][:, G:-G, G:-G, G:-G] for P in Ps]
    assert np.array_equal(np.concatenate(parts, axis=3 - axis), union)


def test_sibling_ghosts_are_copies_and_covered_set():
    """The C/F ghosts of patch A that lie in sibling B's interior equal B's values exactly (the
    others keep the trilinear value), and AverageDown with the sibling covers the coarse nodes
    whose 27 fine nodes lie in A or B, each written by the patch owning the central node."""
    nc = (14, 12, 13)
    c0a, nfa, c0b, nfb = (2, 2, 2), (10, 12, 8), (7, 3, 2), (8, 10, 8)   # B abuts A's hi-x face
    bcf = ((CF, CF),) * 3
    Uc = _coarse_field(nc, lambda q, X, Y, Z: (q + 1) * (1 + 0.1 * X - 0.2 * Y + 0.05 * Z * X))
    rng = np.random.default_rng(31)
    Ua = rng.uniform(1, 2, (5, nfa[2] + 2 * G, nfa[1] + 2 * G, nfa[0] + 2 * G))
    Ub = rng.uniform(1, 2, (5, nfb[2] + 2 * G, nfb[1] + 2 * G, nfb[0] + 2 * G))
    Ua0 = Ua.copy()
    oracle.fill_two_levels_sib(nfa, bcf, Ua, nc, c0a, Uc, [((10, 2, 0), nfb, Ub)])
    ref = oracle.fill_two_levels(nfa, bcf, Ua0.copy(), nc, c0a, Uc)
    assert np.array_equal(Ua[:, G:-G, G:-G, G:-G], Ua0[:, G:-G, G:-G, G:-G])
    n_copied = 0
    for k in range(-G, nfa[2] + G):
        for j in range(-G, nfa[1] + G):
            for i in range(-G, nfa[0] + G):
                if 0 <= i < nfa[0] and 0 <= j < nfa[1] and 0 <= k < nfa[2]:
                    continue
                ib, jb, kb = i - 10, j - 2, k
                got = Ua[:, k + G, j + G, i + G]
                if 0 <= ib < nfb[0] and 0 <= jb < nfb[1] and 0 <= kb < nfb[2]:
                    assert np.array_equal(got, Ub[:, kb + G, jb + G, ib + G])
                    n_copied += 1
                else:
                    assert np.array_equal(got, ref[:, k + G, j + G, i + G])
    assert n_copied == G * nfb[1] * nfa[2] - G * 0  # the hi-x ghost slab over B's j-range
    # AverageDown: mark coarse nodes
    Ca = np.full_like(Uc, -7.0)
    Cb = Ca.copy()
    oracle.average_down_sib(nfa, bcf, Ua.copy(), nc, c0a, Ca, [((10, 2, 0), nfb, Ub)])
    oracle.average_down_sib(nfb, bcf, Ub.copy(), nc, c0b, Cb, [((-10, -2, 0), nfa, Ua)])
    for K in range(nc[2]):
        for J in range(nc[1]):
            for I in range(nc[0]):
                fa = (2 * (I - c0a[0]), 2 * (J - c0a[1]), 2 * (K - c0a[2]))
                fb = (2 * (I - c0b[0]), 2 * (J - c0b[1]), 2 * (K - c0b[2]))
                ina = lambda f: all(0 <= f[d] < nfa[d] for d in range(3))
                inb = lambda f: all(0 <= f[d] < nfb[d] for d in range(3))
                allin = all(ina((fa[0] + a, fa[1] + b, fa[2] + c)) or inb((fb[0] + a, fb[1] + b, fb[2] + c))
                            for a in (-1, 0, 1) for b in (-1, 0, 1) for c in (-1, 0, 1))
                wa = Ca[0, K + G, J + G, I + G] != -7.0
                wb = Cb[0, K + G, J + G, I + G] != -7.0
                assert wa == (allin and ina(fa)) and wb == (allin and inb(fb)), (I, J, K)
    assert (Ca[0] != -7.0).sum() + (Cb[0] != -7.0).sum() > 0
