"""CPU tests of the C ABI: the library loads, exports every symbol the header
declares, validates arguments synchronously (CROCCO_ERR_ARG, no CUDA call),
and its host-side ghost-exchange plan is correct (every ghost point written
exactly once per phase, sources inside the source block's filled region,
identical canonical order on every rank).  No kernels are launched here.
"""
import os
import re
import subprocess

import numpy as np
import pytest

from paper_conf_ipps_davissngmb23_b200 import build as B
from paper_conf_ipps_davissngmb23_b200 import crocco as cc

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


@pytest.fixture(scope="module", autouse=True)
def built():
    B.build()


def header_symbols():
    txt = open(os.path.join(ROOT, "include", "crocco.h")).read()
    return sorted(set(re.findall(r"^\s*(?:crocco_status|const char \*)\s*(crocco_\w+)\s*\(", txt, re.M)))


def test_exports_every_header_symbol():
    syms = header_symbols()
    assert len(syms) >= 18
    out = subprocess.check_output(["nm", "-D", "--defined-only", B.LIB]).decode()
    exported = set(re.findall(r"\bT (crocco_\w+)", out))
    missing = [s for s in syms if s not in exported]
    assert not missing, missing
    assert sorted(cc.EXPORTED) == syms          # the binding wraps exactly the ABI
    L = cc.lib()
    for s in syms:
        assert hasattr(L, s)


def test_sm100a_code_in_library():
    out = subprocess.check_output(["/usr/local/cuda/bin/cuobjdump", "--list-elf", B.LIB]).decode()
    assert "sm_100a" in out


def test_version():
    assert "sm_100a" in cc.crocco_version()


@pytest.mark.parametrize("kw,frag", [
    (dict(n_global=(10, 8, 8), n_blocks=(3, 1, 1)), "divisible"),
    (dict(n_global=(6, 8, 8), n_blocks=(2, 1, 1)), "ghost width"),
    (dict(n_global=(8, 8, 8), bc=((0, 1), (0, 0), (0, 0))), "PERIODIC must be paired"),
    (dict(n_global=(8, 8, 8), nranks=2, rank=0), "block_rank"),
    (dict(n_global=(8, 8, 8), block_rank=[3], nranks=2), "out of range"),
    (dict(n_global=(0, 8, 8)), "bad n_global"),                                   # empty domain
    (dict(n_global=(70000, 8, 8)), "65535"),                                      # beyond the grid limits
    (dict(n_global=(8, 8, 8), bc=((7, 7), (0, 0), (0, 0))), "bad bc kind"),
])
def test_invalid_desc_is_err_arg(kw, frag):
    d = cc.make_desc(**kw)
    with pytest.raises(cc.CroccoError) as ei:
        cc.crocco_init_grid(d, cc.make_phys())
    assert ei.value.status == cc.CROCCO_ERR_ARG
    assert frag in str(ei.value)


@pytest.mark.parametrize("kw,frag", [
    (dict(gamma=1.0), "gas constants"),
    (dict(weno_limiter=4), "weno_limiter"),
    (dict(weno_limiter=1, weno_alpha_rl=-1.0), "thresholds"),
    (dict(weno_weights=2), "weno_weights"),
    (dict(visc_form=2), "visc_form"),
])
def test_invalid_phys_is_err_arg(kw, frag):
    d = cc.make_desc((8, 8, 8))
    with pytest.raises(cc.CroccoError) as ei:
        cc.crocco_init_grid(d, cc.make_phys(**kw))
    assert ei.value.status == cc.CROCCO_ERR_ARG
    assert frag in str(ei.value)


def _plan_all(n, nb, bc, nranks=1, block_rank=None):
    out = {}
    for r in range(nranks):
        d = cc.make_desc(n, nb, bc, rank=r, nranks=nranks, block_rank=block_rank)
        out[r] = [cc.crocco_exchange_plan(d, ph) for ph in range(3)]
    return out


@pytest.mark.parametrize("nb,bc", [
    ((1, 1, 1), ((0, 0),) * 3),
    ((2, 3, 2), ((0, 0), (1, 3), (2, 1))),
    ((4, 1, 1), ((3, 1), (0, 0), (0, 0))),
])
def test_plan_covers_every_ghost_point_once(nb, bc):
    n = tuple(8 * b for b in nb)
    plans = _plan_all(n, nb, bc)[0]
    bn = [n[d] // nb[d] for d in range(3)]
    nbt = nb[0] * nb[1] * nb[2]
    G = 4
    written = np.zeros((nbt, bn[2] + 8, bn[1] + 8, bn[0] + 8), dtype=int)
    for ph in range(3):
        for m in plans[ph]:
            lo, ext = list(m.dst_lo), list(m.ext)
            written[m.dst_block, lo[2] + G:lo[2] + G + ext[2], lo[1] + G:lo[1] + G + ext[1],
                    lo[0] + G:lo[0] + G + ext[0]] += 1
            if m.kind == 0:
                # source box is interior along the phase axis, and inside the region
                # already valid after the earlier phases along the others
                s = list(m.src_lo)
                assert 0 <= s[ph] and s[ph] + ext[ph] <= bn[ph]
                for e in range(3):
                    if e < ph:
                        assert s[e] >= -G and s[e] + ext[e] <= bn[e] + G
                    elif e > ph:
                        assert s[e] >= 0 and s[e] + ext[e] <= bn[e]
    interior = np.zeros_like(written[0])
    interior[G:-G, G:-G, G:-G] = 1
    for b in range(nbt):
        # each ghost point exactly once, interior never
        assert np.all(written[b] + interior == 1)


def test_plan_is_identical_across_ranks_for_shared_messages():
    n, nb = (16, 16, 8), (2, 2, 1)
    br = [0, 1, 1, 0]
    plans = _plan_all(n, nb, ((0, 0),) * 3, nranks=2, block_rank=br)
    for ph in range(3):
        key = lambda m: (m.dst_block, m.side, m.src_block)
        remote = [[key(m) for m in plans[r][ph] if m.kind == 0 and m.src_rank != m.dst_rank]
                  for r in range(2)]
        # rank 0 and 1 see the same remote messages in the same order
        assert remote[0] == remote[1]
        for r in range(2):
            for m in plans[r][ph]:
                assert m.dst_rank == br[m.dst_block]
                if m.kind == 0:
                    assert m.src_rank == br[m.src_block]
                    assert r in (m.src_rank, m.dst_rank)


def test_plan_marks_coarse_fine_faces_physical():
    """A fine AMR level (CROCCO_BC_COARSE_FINE faces, NEXT-4) gets no copy message across a C/F
    face: those ghosts belong to the two-level fill (host plan, no GPU needed)."""
    CF = cc.BC_COARSE_FINE
    d = cc.make_desc((16, 8, 8), (2, 1, 1), ((CF, CF), (CF, CF), (0, 0)))
    xi = cc.crocco_exchange_plan(d, 0)
    outer = [m for m in xi if (m.dst_block == 0 and m.side == 0) or (m.dst_block == 1 and m.side == 1)]
    inner = [m for m in xi if m not in outer]
    assert len(outer) == 2 and all(m.kind == 1 and m.src_block == -1 and m.bc_kind == CF for m in outer)
    assert len(inner) == 2 and all(m.kind == 0 for m in inner)      # same-level copy between blocks
    for m in cc.crocco_exchange_plan(d, 1):                         # eta: both faces C/F, no copies
        assert m.kind == 1 and m.src_block == -1


def test_amr_patch_sibling_detection_host_logic():
    """AmrSolver links same-level patches whose ghost band reaches another patch as siblings
    (reading 31) and refuses overlapping interiors (host logic)."""
    from types import SimpleNamespace as NS
    from paper_conf_ipps_davissngmb23_b200.solver import AmrSolver
    CF = cc.BC_COARSE_FINE

    def patch(n):
        return NS(desc=NS(bc=((CF, CF), (CF, CF), (0, 0)), n_global=n))
    A = AmrSolver.__new__(AmrSolver)
    A.patches = [(patch((16, 16, 8)), (2, 2, 0)), (patch((16, 16, 8)), (14, 2, 0))]
    assert A._sibling_pairs() == []                          # x: [4,20)+-4 vs [28,44): apart
    A.patches[1] = (patch((16, 16, 8)), (11, 2, 0))          # [22,38) within 4 of [4,20)
    assert A._sibling_pairs() == [(0, 1)]
    A.patches[1] = (patch((16, 16, 8)), (10, 2, 0))          # [20,36): abutting
    assert A._sibling_pairs() == [(0, 1)]
    A.patches[1] = (patch((16, 16, 8)), (9, 2, 0))           # [18,34): interiors overlap
    with pytest.raises(ValueError):
        A._sibling_pairs()
