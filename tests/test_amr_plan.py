"""Host logic of the inter-level AMR exchange (crocco_amr_plan, include/crocco.h; PAPER.md:125-131:
each level is decomposed over the ranks on its own, so FillPatch and AverageDown move boxes
between the ranks of the two levels).  No GPU: the plan is pure host code of libcrocco.

Checked by brute force against the definitions the kernels use (readings 25, 26):
  - kind 0 (FillPatch): every corner k_cf_interp reads for every C/F ghost point of every fine
    block -- I = floor((2 c0 + f)/2) and I + 1 per direction, in the block that owns the
    clamped I -- lies in a box the plan routes from that coarse block to that fine block;
  - kind 1 (AverageDown): the boxes partition the covered set exactly (each covered node once),
    and each node's central fine node 2 (I - c0) lies in the box's fine block;
  - NCCL matching: what rank r lists as sent to rank s equals, in order, what s lists as
    received from r; local boxes appear once on their rank.
"""
import itertools

import numpy as np
import pytest

from paper_conf_ipps_davissngmb23_b200 import crocco as cc

G = 4
CF, PER, EXT, WALL = cc.BC_COARSE_FINE, cc.BC_PERIODIC, cc.BC_EXTRAP, cc.BC_WALL


def _plans(nf, nbf, bcf, nc, nbc, bcc, c0, nranks, seed):
    rng = np.random.default_rng(seed)
    rf = rng.integers(0, nranks, int(np.prod(nbf))).tolist()
    rc = rng.integers(0, nranks, int(np.prod(nbc))).tolist()
    out = []
    for r in range(nranks):
        fd = cc.make_desc(nf, nbf, bcf, rank=r, nranks=nranks, block_rank=rf)
        cd = cc.make_desc(nc, nbc, bcc, rank=r, nranks=nranks, block_rank=rc)
        out.append(cc.crocco_amr_plan(fd, cd, c0))
    return rf, rc, out


def _t(m):
    return (m.kind, m.coarse_block, m.fine_block, m.src_rank, m.dst_rank, tuple(m.lo), tuple(m.ext))


def _blocks(n, nb):
    bn = [n[d] // nb[d] for d in range(3)]
    for bz, by, bx in itertools.product(range(nb[2]), range(nb[1]), range(nb[0])):
        yield bx + nb[0] * (by + nb[1] * bz), (bx, by, bz), [(bx, by, bz)[d] * bn[d] for d in range(3)], bn


CASES = [
    # fine level strictly inside, C/F on all faces; both levels multi-block
    dict(nf=(20, 16, 12), nbf=(2, 2, 1), bcf=((CF, CF),) * 3, nc=(24, 24, 16), nbc=(2, 2, 2),
         bcc=((PER, PER),) * 3, c0=(5, 6, 3)),
    # fine level touching the domain: physical faces on the boundary, C/F elsewhere
    dict(nf=(24, 17, 12), nbf=(3, 1, 2), bcf=((EXT, CF), (CF, WALL), (CF, CF)), nc=(24, 16, 16),
         nbc=(3, 2, 1), bcc=((EXT, EXT), (WALL, WALL), (PER, PER)), c0=(0, 7, 2)),
    # periodic fine level spanning the periodic coarse domain in x (the AMR TGV bench shape)
    dict(nf=(32, 12, 12), nbf=(2, 1, 2), bcf=((PER, PER), (CF, CF), (CF, CF)), nc=(16, 16, 16),
         nbc=(2, 2, 2), bcc=((PER, PER),) * 3, c0=(0, 4, 3)),
]


def _covered(case):
    """Coarse nodes averaged down (reading 26), per direction [lo, hi]."""
    rng = []
    for d in range(3):
        nf, c0 = case["nf"][d], case["c0"][d]
        rng.append((0, nf // 2 - 1) if case["bcf"][d][0] == PER else (c0 + 1, c0 + (nf - 2) // 2))
    return rng


@pytest.mark.parametrize("case", CASES, ids=["interior", "boundary", "periodic"])
@pytest.mark.parametrize("nranks,seed", [(1, 0), (2, 1), (3, 2)])
def test_plan_matches_between_ranks(case, nranks, seed):
    _, _, plans = _plans(case["nf"], case["nbf"], case["bcf"], case["nc"], case["nbc"], case["bcc"], case["c0"],
                         nranks, seed)
    for r, p in enumerate(plans):
        assert all(m.src_rank == r or m.dst_rank == r for m in p)
        kinds = [m.kind for m in p]
        assert kinds == sorted(kinds)                      # kind 0 first
    for r, s in itertools.product(range(nranks), repeat=2):
        if r == s:
            continue
        for k in (0, 1):
            sent = [_t(m) for m in plans[r] if m.kind == k and m.src_rank == r and m.dst_rank == s]
            recv = [_t(m) for m in plans[s] if m.kind == k and m.src_rank == r and m.dst_rank == s]
            assert sent == recv


@pytest.mark.parametrize("case", CASES, ids=["interior", "boundary", "periodic"])
def test_fillpatch_boxes_cover_every_interpolation_corner(case):
    nranks = 3
    rf, rc, plans = _plans(case["nf"], case["nbf"], case["bcf"], case["nc"], case["nbc"], case["bcc"], case["c0"],
                           nranks, 7)
    allm = {_t(m) for p in plans for m in p if m.kind == 0}
    nc, nbc, c0 = case["nc"], case["nbc"], case["c0"]
    bnc = [nc[d] // nbc[d] for d in range(3)]
    for m in allm:                                          # boxes stay inside the padded block
        assert all(-G <= m[5][d] and m[5][d] + m[6][d] <= bnc[d] + G for d in range(3))
        assert m[3] == rc[m[1]] and m[4] == rf[m[2]]
    boxes = {}
    for m in allm:
        boxes.setdefault((m[1], m[2]), []).append((m[5], m[6]))
    checked = 0
    for gid, bidx, org, bn in _blocks(case["nf"], case["nbf"]):
        for D, side in itertools.product(range(3), range(2)):
            if case["bcf"][D][side] != CF or bidx[D] != (0 if side == 0 else case["nbf"][D] - 1):
                continue
            rngs = []
            for e in range(3):
                if e == D:
                    lo, ext = (-G if side == 0 else bn[e]), G
                elif e < D:
                    lo, ext = -G, bn[e] + 2 * G
                else:
                    lo, ext = 0, bn[e]
                rngs.append(range(lo, lo + ext))
            for f in itertools.product(*rngs):
                own, loc = [], []
                for d in range(3):
                    I = (2 * c0[d] + org[d] + f[d]) // 2       # floor
                    Ic = min(max(I, 0), nc[d] - 1)
                    bx = Ic // bnc[d]
                    own.append(bx)
                    loc.append(I - bx * bnc[d])
                cg = own[0] + nbc[0] * (own[1] + nbc[1] * own[2])
                ok = any(all(lo[d] <= loc[d] and loc[d] + 1 < lo[d] + ext[d] for d in range(3))
                         for lo, ext in boxes.get((cg, gid), []))
                assert ok, (gid, f, cg, loc)
                checked += 1
    assert checked > 0


@pytest.mark.parametrize("case", CASES, ids=["interior", "boundary", "periodic"])
def test_averagedown_boxes_partition_the_covered_set(case):
    nranks = 2
    rf, rc, plans = _plans(case["nf"], case["nbf"], case["bcf"], case["nc"], case["nbc"], case["bcc"], case["c0"],
                           nranks, 11)
    allm = {_t(m) for p in plans for m in p if m.kind == 1}
    nc, nbc, c0 = case["nc"], case["nbc"], case["c0"]
    bnc = [nc[d] // nbc[d] for d in range(3)]
    bnf = [case["nf"][d] // case["nbf"][d] for d in range(3)]
    hits = np.zeros(nc[::-1], dtype=np.int64)
    for kind, cg, fg, src, dst, lo, ext in allm:
        assert src == rf[fg] and dst == rc[cg]
        cb = (cg % nbc[0], (cg // nbc[0]) % nbc[1], cg // (nbc[0] * nbc[1]))
        fb = (fg % case["nbf"][0], (fg // case["nbf"][0]) % case["nbf"][1], fg // (case["nbf"][0] * case["nbf"][1]))
        I0 = [cb[d] * bnc[d] + lo[d] for d in range(3)]
        assert all(0 <= lo[d] and lo[d] + ext[d] <= bnc[d] for d in range(3))
        for d in range(3):                                  # central fine nodes in the fine block
            f_lo, f_hi = 2 * (I0[d] - c0[d]), 2 * (I0[d] + ext[d] - 1 - c0[d])
            assert fb[d] * bnf[d] <= f_lo and f_hi < (fb[d] + 1) * bnf[d]
        hits[I0[2]:I0[2] + ext[2], I0[1]:I0[1] + ext[1], I0[0]:I0[0] + ext[0]] += 1
    want = np.zeros_like(hits)
    (x0, x1), (y0, y1), (z0, z1) = _covered(case)
    want[z0:z1 + 1, y0:y1 + 1, x0:x1 + 1] = 1
    assert np.array_equal(hits, want)


def test_plan_refuses_what_link_refuses():
    fd = cc.make_desc((20, 16, 12), (1, 1, 1), ((CF, CF),) * 3)
    cd = cc.make_desc((10, 10, 8), (1, 1, 1), ((PER, PER),) * 3)
    with pytest.raises(RuntimeError):
        cc.crocco_amr_plan(fd, cd, (2, 2, 2))               # fine level outside the coarse domain
    fd2 = cc.make_desc((20, 16, 12), (1, 1, 1), ((CF, CF),) * 3, rank=0, nranks=2, block_rank=[1])
    cd2 = cc.make_desc((24, 24, 16), (1, 1, 1), ((PER, PER),) * 3, rank=1, nranks=2, block_rank=[0])
    with pytest.raises(RuntimeError):
        cc.crocco_amr_plan(fd2, cd2, (1, 1, 1))             # different ranks of one process


SIB = [  # two patches of one level in the common fine index space 2 c0 + f (reading 31)
    dict(nf=(16, 16, 12), nbf=(2, 1, 1), c0=(3, 4, 2), ng=(16, 16, 12), nbg=(1, 2, 2), c0g=(11, 4, 2)),   # abut in x
    dict(nf=(16, 12, 12), nbf=(1, 2, 1), c0=(3, 4, 2), ng=(12, 16, 8), nbg=(2, 1, 2), c0g=(5, 11, 3)),    # gap of 2 in y
]


@pytest.mark.parametrize("sc", SIB, ids=["abutting", "nearby"])
@pytest.mark.parametrize("nranks", [1, 2, 3])
def test_sibling_boxes_cover_the_ghost_points_inside_the_sibling(sc, nranks):
    """Kind-2 boxes (crocco_amr_sibling_plan): a C/F ghost point of a patch block lying in a sibling
    block's interior is in exactly the box routed from that sibling block to that patch block;
    boxes hold no other point; sends and receives of every rank pair match in order."""
    bcf = ((CF, CF),) * 3
    rng = np.random.default_rng(nranks)
    rf = rng.integers(0, nranks, int(np.prod(sc["nbf"]))).tolist()
    rg = rng.integers(0, nranks, int(np.prod(sc["nbg"]))).tolist()
    plans = []
    for r in range(nranks):
        fd = cc.make_desc(sc["nf"], sc["nbf"], bcf, rank=r, nranks=nranks, block_rank=rf)
        gd = cc.make_desc(sc["ng"], sc["nbg"], bcf, rank=r, nranks=nranks, block_rank=rg)
        plans.append(cc.crocco_amr_sibling_plan(fd, sc["c0"], gd, sc["c0g"], 1))
    for r, s in itertools.product(range(nranks), repeat=2):
        if r != s:
            assert [_t(m) for m in plans[r] if m.src_rank == r and m.dst_rank == s] == \
                   [_t(m) for m in plans[s] if m.src_rank == r and m.dst_rank == s]
    allm = {_t(m) + (m.sibling,) for p in plans for m in p}
    assert allm and all(m[0] == 2 and m[7] == 1 for m in allm)
    # sibling blocks in the common index space
    gbl = {gid: [2 * sc["c0g"][d] + org[d] for d in range(3)] for gid, _, org, _ in _blocks(sc["ng"], sc["nbg"])}
    bng = [sc["ng"][d] // sc["nbg"][d] for d in range(3)]
    want = set()
    for gid, bidx, org, bn in _blocks(sc["nf"], sc["nbf"]):
        for D, side in itertools.product(range(3), range(2)):
            if bidx[D] != (0 if side == 0 else sc["nbf"][D] - 1):
                continue
            rngs = []
            for e in range(3):
                if e == D:
                    lo, ext = (-G if side == 0 else bn[e]), G
                elif e < D:
                    lo, ext = -G, bn[e] + 2 * G
                else:
                    lo, ext = 0, bn[e]
                rngs.append(range(lo, lo + ext))
            for f in itertools.product(*rngs):
                p = [2 * sc["c0"][d] + org[d] + f[d] for d in range(3)]
                for sg, o in gbl.items():
                    if all(o[d] <= p[d] < o[d] + bng[d] for d in range(3)):
                        want.add((sg, gid, tuple(p[d] - o[d] for d in range(3))))
    got = set()
    for kind, sg, fg, src, dst, lo, ext, _ in allm:
        assert src == rg[sg] and dst == rf[fg]
        for q in itertools.product(*[range(lo[d], lo[d] + ext[d]) for d in range(3)]):
            got.add((sg, fg, q))
    assert got == want and want
