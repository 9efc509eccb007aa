"""Thin ctypes binding of libcrocco.so (include/crocco.h), same names as the C ABI.

Argument marshalling only: every numerical step runs in the CUDA kernels of
csrc/.  PyTorch is used for device memory (torch.empty on the GPU), streams
and torch.distributed plumbing.  There is no CPU fallback: if the shared
library is missing or fails to load, :func:`lib` raises.
"""
from __future__ import annotations

import ctypes as C
import os

HERE = os.path.dirname(os.path.abspath(__file__))
LIB_PATH = os.environ.get("CROCCO_LIB") or os.path.join(HERE, "libcrocco.so")  # env: variant builds (tools/)

CROCCO_OK, CROCCO_ERR_ARG, CROCCO_ERR_CUDA, CROCCO_ERR_NCCL, CROCCO_ERR_NOMEM, CROCCO_ERR_STATE = range(6)
BC_PERIODIC, BC_EXTRAP, BC_DIRICHLET, BC_WALL, BC_SLIPWALL, BC_SPLIT, BC_COARSE_FINE = 0, 1, 2, 3, 4, 5, 6
TERM_INVISCID, TERM_VISCOUS = 1, 2
MU_CONST, MU_SUTHERLAND = 0, 1
FIELD_STATE, FIELD_METRIC = 0, 1
GHOST, GHOST_COORDS = 4, 10


class CroccoError(RuntimeError):
    def __init__(self, status, msg):
        super().__init__(f"crocco status {status}: {msg}")
        self.status = status


class Split(C.Structure):
    _fields_ = [("axis", C.c_int32), ("i0", C.c_double), ("di_dt", C.c_double),
                ("left", C.c_double * 5), ("right_kind", C.c_int32), ("right", C.c_double * 5)]


class GridDesc(C.Structure):
    _fields_ = [("n_global", C.c_int64 * 3), ("n_blocks", C.c_int32 * 3),
                ("bc", (C.c_int32 * 2) * 3), ("dirichlet", ((C.c_double * 5) * 2) * 3),
                ("rank", C.c_int32), ("nranks", C.c_int32),
                ("block_rank", C.POINTER(C.c_int32)), ("stream", C.c_void_p),
                ("nccl_unique_id", C.c_void_p), ("split", (Split * 2) * 3)]


class PhysC(C.Structure):
    _fields_ = [("gamma", C.c_double), ("R", C.c_double), ("Pr", C.c_double),
                ("mu_law", C.c_int32), ("mu_ref", C.c_double), ("T_ref", C.c_double),
                ("S", C.c_double), ("weno_eps", C.c_double), ("terms", C.c_int32),
                ("dir_mask", C.c_int32), ("weno_weights", C.c_int32), ("weno_limiter", C.c_int32),
                ("weno_alpha_rl", C.c_double), ("weno_alpha_al", C.c_double), ("visc_form", C.c_int32)]


class BlockLayout(C.Structure):
    _fields_ = [("n", C.c_int32 * 3), ("origin", C.c_int64 * 3), ("ghost", C.c_int32),
                ("ghost_coords", C.c_int32), ("offset", C.c_int64), ("pitch_y", C.c_int64),
                ("pitch_z", C.c_int64), ("comp_stride", C.c_int64), ("coffset", C.c_int64),
                ("cpitch_y", C.c_int64), ("cpitch_z", C.c_int64), ("ccomp_stride", C.c_int64),
                ("global_id", C.c_int32)]


class Msg(C.Structure):
    _fields_ = [("phase", C.c_int32), ("dst_block", C.c_int32), ("side", C.c_int32),
                ("kind", C.c_int32), ("bc_kind", C.c_int32), ("src_block", C.c_int32),
                ("src_rank", C.c_int32), ("dst_rank", C.c_int32), ("dst_lo", C.c_int64 * 3),
                ("src_lo", C.c_int64 * 3), ("ext", C.c_int64 * 3)]


class AmrMsg(C.Structure):
    _fields_ = [("kind", C.c_int32), ("coarse_block", C.c_int32), ("fine_block", C.c_int32),
                ("sibling", C.c_int32), ("src_rank", C.c_int32), ("dst_rank", C.c_int32), ("lo", C.c_int64 * 3),
                ("ext", C.c_int64 * 3)]


_lib = None

DPP = C.POINTER(C.c_void_p)  # double *const * (array of device pointers)

_SIGS = {
    "crocco_init_grid": [C.POINTER(GridDesc), C.POINTER(PhysC), C.POINTER(C.c_void_p)],
    "crocco_num_local_blocks": [C.c_void_p, C.POINTER(C.c_int32)],
    "crocco_get_block_layout": [C.c_void_p, C.c_int32, C.POINTER(BlockLayout)],
    "crocco_set_phys": [C.c_void_p, C.POINTER(PhysC)],
    "crocco_scratch_bytes": [C.c_void_p, C.POINTER(C.c_int64)],
    "crocco_init_metrics": [C.c_void_p, DPP, DPP],
    "crocco_fill_boundary": [C.c_void_p, DPP, C.c_int32, DPP],
    "crocco_set_time": [C.c_void_p, C.c_double],
    "crocco_get_time": [C.c_void_p, C.POINTER(C.c_double)],
    "crocco_rhs": [C.c_void_p, DPP, DPP, DPP],
    "crocco_rk_stage": [C.c_void_p, C.c_int32, C.c_double, DPP, DPP, DPP, DPP],
    "crocco_rk_update": [C.c_void_p, C.c_int32, C.c_double, DPP, DPP, DPP, DPP],
    "crocco_sync": [C.c_void_p],
    "crocco_finalize": [C.c_void_p],
    "crocco_launch_count": [C.c_void_p, C.POINTER(C.c_int64), C.c_int32],
    "crocco_set_timing": [C.c_void_p, C.c_int32],
    "crocco_set_overlap": [C.c_void_p, C.c_int32],
    "crocco_overlap_count": [C.c_void_p, C.POINTER(C.c_int64), C.c_int32],
    "crocco_set_nccl_loopback": [C.c_void_p, C.c_int32],
    "crocco_kernel_times": [C.c_void_p, C.c_int32, C.POINTER(C.c_int64), C.POINTER(C.c_double),
                            C.POINTER(C.c_int32)],
    "crocco_exchange_plan": [C.POINTER(GridDesc), C.c_int32, C.POINTER(Msg), C.c_int32,
                             C.POINTER(C.c_int32)],
    "crocco_amr_plan": [C.POINTER(GridDesc), C.POINTER(GridDesc), C.POINTER(C.c_int64), C.POINTER(AmrMsg),
                        C.c_int32, C.POINTER(C.c_int32)],
    "crocco_amr_sibling_plan": [C.POINTER(GridDesc), C.POINTER(C.c_int64), C.POINTER(GridDesc),
                                C.POINTER(C.c_int64), C.c_int32, C.POINTER(AmrMsg), C.c_int32,
                                C.POINTER(C.c_int32)],
    "crocco_nccl_unique_id": [C.c_void_p, C.c_int32],
    "crocco_compute_dt": [C.c_void_p, DPP, DPP, C.c_double, C.POINTER(C.c_double)],
    "crocco_rk3_step": [C.c_void_p, C.c_double, DPP, DPP, DPP, DPP, C.c_int32],
    "crocco_amr_link": [C.c_void_p, C.c_void_p, C.POINTER(C.c_int64)],
    "crocco_init_metrics2": [C.c_void_p, DPP],
    "crocco_check_state": [C.c_void_p, DPP, C.POINTER(C.c_int64)],
    "crocco_copy_metrics2": [C.c_void_p, C.c_int32, C.c_void_p],
    "crocco_fill_patch_two_levels": [C.c_void_p, DPP, DPP, DPP],
    "crocco_amr_rk_stage": [C.c_void_p, C.c_int32, C.c_double, DPP, DPP, DPP, DPP, DPP],
    "crocco_average_down": [C.c_void_p, DPP, DPP],
    "crocco_amr_link_sibling": [C.c_void_p, C.c_void_p],
    "crocco_fill_patch_level": [C.c_void_p, DPP, DPP, DPP, C.POINTER(DPP)],
    "crocco_amr_rk_stage_level": [C.c_void_p, C.c_int32, C.c_double, DPP, DPP, DPP, DPP, DPP, C.POINTER(DPP)],
    "crocco_average_down_level": [C.c_void_p, DPP, DPP, C.POINTER(DPP)],
}
_STR = {"crocco_last_error": [C.c_void_p], "crocco_version": [],
        "crocco_kernel_class_name": [C.c_int32]}

EXPORTED = sorted(list(_SIGS) + list(_STR))


def lib() -> C.CDLL:
    """Load libcrocco.so (fails loudly if it is missing -- no fallback)."""
    global _lib
    if _lib is None:
        if not os.path.exists(LIB_PATH):
            raise ImportError(f"{LIB_PATH} missing: run `python -m paper_conf_ipps_davissngmb23_b200.build`")
        L = C.CDLL(LIB_PATH)
        for name, args in _SIGS.items():
            f = getattr(L, name)
            f.argtypes = args
            f.restype = C.c_int
        for name, args in _STR.items():
            f = getattr(L, name)
            f.argtypes = args
            f.restype = C.c_char_p
        _lib = L
    return _lib


def _check(st, ctx=None):
    if st != CROCCO_OK:
        msg = lib().crocco_last_error(ctx)
        raise CroccoError(st, msg.decode() if msg else "")


def _ptrs(ptrs):
    arr = (C.c_void_p * len(ptrs))(*[int(p) for p in ptrs])
    return C.cast(arr, DPP), arr


# ---------------------------------------------------------------- C-ABI mirrors

def crocco_version() -> str:
    return lib().crocco_version().decode()


def crocco_kernel_class_name(k: int) -> str:
    return lib().crocco_kernel_class_name(k).decode()


def make_desc(n_global, n_blocks=(1, 1, 1), bc=((0, 0),) * 3, dirichlet=None, rank=0, nranks=1,
              block_rank=None, stream=0, nccl_unique_id=None, split=None):
    """split: {(d, side): dict(axis, i0, di_dt, left, right_kind, right)} for SPLIT faces."""
    d = GridDesc()
    for a in range(3):
        d.n_global[a] = int(n_global[a])
        d.n_blocks[a] = int(n_blocks[a])
        for s in range(2):
            d.bc[a][s] = int(bc[a][s])
            for c in range(5):
                d.dirichlet[a][s][c] = 0.0 if dirichlet is None else float(dirichlet[a][s][c])
    d.rank, d.nranks = int(rank), int(nranks)
    keep = []
    if block_rank is not None:
        arr = (C.c_int32 * len(block_rank))(*[int(x) for x in block_rank])
        d.block_rank = C.cast(arr, C.POINTER(C.c_int32))
        keep.append(arr)
    d.stream = C.c_void_p(int(stream))
    if nccl_unique_id is not None:
        buf = C.create_string_buffer(bytes(nccl_unique_id), 128)
        d.nccl_unique_id = C.cast(buf, C.c_void_p)
        keep.append(buf)
    for (a, sd), v in (split or {}).items():
        sp = d.split[a][sd]
        sp.axis, sp.i0, sp.di_dt = int(v["axis"]), float(v["i0"]), float(v["di_dt"])
        sp.right_kind = int(v["right_kind"])
        for c in range(5):
            sp.left[c] = float(v["left"][c])
            sp.right[c] = float(v.get("right", [0.0] * 5)[c])
    d._keep = keep
    return d


def make_phys(gamma=1.4, R=1.0, Pr=0.72, mu_law=MU_CONST, mu_ref=0.0, T_ref=1.0, S=0.0,
              weno_eps=1e-6, terms=TERM_INVISCID | TERM_VISCOUS, dir_mask=7, weno_weights=0,
              weno_limiter=0, weno_alpha_rl=0.0, weno_alpha_al=0.0, visc_form=0):
    return PhysC(gamma, R, Pr, mu_law, mu_ref, T_ref, S, weno_eps, terms, dir_mask, weno_weights,
                 weno_limiter, weno_alpha_rl, weno_alpha_al, visc_form)


def crocco_init_grid(desc: GridDesc, phys: PhysC):
    ctx = C.c_void_p()
    _check(lib().crocco_init_grid(C.byref(desc), C.byref(phys), C.byref(ctx)))
    return ctx


def crocco_num_local_blocks(ctx) -> int:
    n = C.c_int32()
    _check(lib().crocco_num_local_blocks(ctx, C.byref(n)), ctx)
    return n.value


def crocco_get_block_layout(ctx, b: int) -> BlockLayout:
    L = BlockLayout()
    _check(lib().crocco_get_block_layout(ctx, b, C.byref(L)), ctx)
    return L


def crocco_set_phys(ctx, phys: PhysC):
    _check(lib().crocco_set_phys(ctx, C.byref(phys)), ctx)


def crocco_scratch_bytes(ctx) -> int:
    v = C.c_int64()
    _check(lib().crocco_scratch_bytes(ctx, C.byref(v)), ctx)
    return v.value


def crocco_init_metrics(ctx, xyz_ptrs, met_ptrs):
    a, ka = _ptrs(xyz_ptrs)
    b, kb = _ptrs(met_ptrs)
    _check(lib().crocco_init_metrics(ctx, a, b), ctx)


def crocco_fill_boundary(ctx, field_ptrs, kind=FIELD_STATE, met_ptrs=None):
    a, ka = _ptrs(field_ptrs)
    if met_ptrs is None:
        _check(lib().crocco_fill_boundary(ctx, a, kind, None), ctx)
    else:
        b, kb = _ptrs(met_ptrs)
        _check(lib().crocco_fill_boundary(ctx, a, kind, b), ctx)


def crocco_set_time(ctx, t):
    _check(lib().crocco_set_time(ctx, float(t)), ctx)


def crocco_get_time(ctx) -> float:
    v = C.c_double()
    _check(lib().crocco_get_time(ctx, C.byref(v)), ctx)
    return v.value


def crocco_rhs(ctx, U_ptrs, met_ptrs, rhs_ptrs):
    a, ka = _ptrs(U_ptrs)
    b, kb = _ptrs(met_ptrs)
    c, kc = _ptrs(rhs_ptrs)
    _check(lib().crocco_rhs(ctx, a, b, c), ctx)


def crocco_rk_stage(ctx, stage, dt, Uin_ptrs, Uout_ptrs, dU_ptrs, met_ptrs):
    a, ka = _ptrs(Uin_ptrs)
    b, kb = _ptrs(Uout_ptrs)
    c, kc = _ptrs(dU_ptrs)
    d, kd = _ptrs(met_ptrs)
    _check(lib().crocco_rk_stage(ctx, stage, dt, a, b, c, d), ctx)


def crocco_rk_update(ctx, stage, dt, Uin_ptrs, Uout_ptrs, dU_ptrs, rhs_ptrs):
    a, ka = _ptrs(Uin_ptrs)
    b, kb = _ptrs(Uout_ptrs)
    c, kc = _ptrs(dU_ptrs)
    d, kd = _ptrs(rhs_ptrs)
    _check(lib().crocco_rk_update(ctx, stage, dt, a, b, c, d), ctx)


def crocco_sync(ctx):
    _check(lib().crocco_sync(ctx), ctx)


def crocco_finalize(ctx):
    _check(lib().crocco_finalize(ctx))


def crocco_launch_count(ctx, reset=False) -> int:
    v = C.c_int64()
    _check(lib().crocco_launch_count(ctx, C.byref(v), int(reset)), ctx)
    return v.value


def crocco_set_nccl_loopback(ctx, enable=True):
    """Single-rank debug: same-rank ghost copies through ncclSend/ncclRecv to self, ComputeDt
    through ncclAllReduce on a 1-rank communicator (bitwise equal to the local path)."""
    _check(lib().crocco_set_nccl_loopback(ctx, int(enable)), ctx)


def crocco_overlap_count(ctx, reset=False) -> int:
    v = C.c_int64()
    _check(lib().crocco_overlap_count(ctx, C.byref(v), int(reset)), ctx)
    return v.value


def crocco_set_overlap(ctx, enable=True):
    """1 / True on, 0 / False off, -1 auto (on when nranks > 1)."""
    _check(lib().crocco_set_overlap(ctx, int(enable)), ctx)


def crocco_set_timing(ctx, enable=True):
    _check(lib().crocco_set_timing(ctx, int(enable)), ctx)


def crocco_kernel_times(ctx):
    n = 32
    launches = (C.c_int64 * n)()
    ms = (C.c_double * n)()
    nc = C.c_int32()
    _check(lib().crocco_kernel_times(ctx, n, launches, ms, C.byref(nc)), ctx)
    return {crocco_kernel_class_name(k): (launches[k], ms[k]) for k in range(nc.value)}


def crocco_exchange_plan(desc: GridDesc, phase: int):
    n = C.c_int32()
    _check(lib().crocco_exchange_plan(C.byref(desc), phase, None, 0, C.byref(n)))
    arr = (Msg * max(n.value, 1))()
    _check(lib().crocco_exchange_plan(C.byref(desc), phase, arr, n.value, C.byref(n)))
    return [arr[i] for i in range(n.value)]


def crocco_amr_plan(fine: GridDesc, coarse: GridDesc, c0):
    """Inter-level boxes of a two-level pair for rank fine.rank (host only, no GPU)."""
    c = (C.c_int64 * 3)(*[int(x) for x in c0])
    n = C.c_int32()
    _check(lib().crocco_amr_plan(C.byref(fine), C.byref(coarse), c, None, 0, C.byref(n)))
    arr = (AmrMsg * max(n.value, 1))()
    _check(lib().crocco_amr_plan(C.byref(fine), C.byref(coarse), c, arr, n.value, C.byref(n)))
    return [arr[i] for i in range(n.value)]


def crocco_amr_sibling_plan(fine: GridDesc, c0, sib: GridDesc, c0s, sibling=0):
    """Kind-2 (sibling ghost) boxes of patch `fine` from sibling patch `sib` (host only)."""
    a = (C.c_int64 * 3)(*[int(x) for x in c0])
    b = (C.c_int64 * 3)(*[int(x) for x in c0s])
    n = C.c_int32()
    _check(lib().crocco_amr_sibling_plan(C.byref(fine), a, C.byref(sib), b, sibling, None, 0, C.byref(n)))
    arr = (AmrMsg * max(n.value, 1))()
    _check(lib().crocco_amr_sibling_plan(C.byref(fine), a, C.byref(sib), b, sibling, arr, n.value, C.byref(n)))
    return [arr[i] for i in range(n.value)]


def crocco_nccl_unique_id() -> bytes:
    buf = C.create_string_buffer(128)
    _check(lib().crocco_nccl_unique_id(C.cast(buf, C.c_void_p), 128))
    return buf.raw


def crocco_compute_dt(ctx, U_ptrs, met_ptrs, cfl) -> float:
    a, ka = _ptrs(U_ptrs)
    b, kb = _ptrs(met_ptrs)
    dt = C.c_double()
    _check(lib().crocco_compute_dt(ctx, a, b, float(cfl), C.byref(dt)), ctx)
    return dt.value


def crocco_rk3_step(ctx, dt, U_ptrs, V_ptrs, dU_ptrs, met_ptrs, use_graph=True):
    a, ka = _ptrs(U_ptrs)
    b, kb = _ptrs(V_ptrs)
    c, kc = _ptrs(dU_ptrs)
    d, kd = _ptrs(met_ptrs)
    _check(lib().crocco_rk3_step(ctx, float(dt), a, b, c, d, int(use_graph)), ctx)


# ---- two-level AMR (include/crocco.h) ----
def crocco_amr_link(fine, coarse, c0):
    arr = (C.c_int64 * 3)(*[int(x) for x in c0])
    _check(lib().crocco_amr_link(fine, coarse, arr), fine)


def crocco_fill_patch_two_levels(fine, Uf_ptrs, metf_ptrs, Uc_ptrs):
    a, ka = _ptrs(Uf_ptrs)
    b, kb = _ptrs(metf_ptrs) if metf_ptrs is not None else (None, None)
    c, kc = _ptrs(Uc_ptrs)
    _check(lib().crocco_fill_patch_two_levels(fine, a, b, c), fine)


def crocco_amr_rk_stage(fine, stage, dt, Uin_ptrs, Uout_ptrs, dU_ptrs, met_ptrs, Uc_in_ptrs):
    a, ka = _ptrs(Uin_ptrs)
    b, kb = _ptrs(Uout_ptrs)
    c, kc = _ptrs(dU_ptrs)
    d, kd = _ptrs(met_ptrs)
    e, ke = _ptrs(Uc_in_ptrs)
    _check(lib().crocco_amr_rk_stage(fine, stage, dt, a, b, c, d, e), fine)


def crocco_average_down(fine, Uf_ptrs, Uc_ptrs):
    a, ka = _ptrs(Uf_ptrs)
    b, kb = _ptrs(Uc_ptrs)
    _check(lib().crocco_average_down(fine, a, b), fine)


def crocco_amr_link_sibling(fine, sibling):
    _check(lib().crocco_amr_link_sibling(fine, sibling), fine)


def _sib_table(sib_ptr_lists):
    """[[block pointers of sibling 0], ...] -> (double **)[] plus the arrays keeping it alive."""
    keep = [_ptrs(pl) for pl in sib_ptr_lists]
    tab = (DPP * max(len(keep), 1))(*[k[0] for k in keep])
    return tab, keep


def crocco_fill_patch_level(fine, Uf_ptrs, metf_ptrs, Uc_ptrs, sib_ptr_lists):
    a, ka = _ptrs(Uf_ptrs)
    b, kb = _ptrs(metf_ptrs) if metf_ptrs is not None else (None, None)
    c, kc = _ptrs(Uc_ptrs)
    t, kt = _sib_table(sib_ptr_lists)
    _check(lib().crocco_fill_patch_level(fine, a, b, c, t), fine)


def crocco_amr_rk_stage_level(fine, stage, dt, Uin_ptrs, Uout_ptrs, dU_ptrs, met_ptrs, Uc_in_ptrs, sib_in_lists):
    a, ka = _ptrs(Uin_ptrs)
    b, kb = _ptrs(Uout_ptrs)
    c, kc = _ptrs(dU_ptrs)
    d, kd = _ptrs(met_ptrs)
    e, ke = _ptrs(Uc_in_ptrs)
    t, kt = _sib_table(sib_in_lists)
    _check(lib().crocco_amr_rk_stage_level(fine, stage, dt, a, b, c, d, e, t), fine)


def crocco_average_down_level(fine, Uf_ptrs, Uc_ptrs, sib_ptr_lists):
    a, ka = _ptrs(Uf_ptrs)
    b, kb = _ptrs(Uc_ptrs)
    t, kt = _sib_table(sib_ptr_lists)
    _check(lib().crocco_average_down_level(fine, a, b, t), fine)


# ---- 27-component metrics / expanded viscous form (readings 27-28) ----
def crocco_init_metrics2(ctx, met_ptrs):
    a, ka = _ptrs(met_ptrs)
    _check(lib().crocco_init_metrics2(ctx, a), ctx)


def crocco_copy_metrics2(ctx, b, dst_ptr):
    _check(lib().crocco_copy_metrics2(ctx, int(b), C.c_void_p(int(dst_ptr))), ctx)


def crocco_check_state(ctx, U_ptrs) -> int:
    """Interior points with a non-finite component, rho <= 0 or p <= 0 (synchronises)."""
    a, ka = _ptrs(U_ptrs)
    n = C.c_int64()
    _check(lib().crocco_check_state(ctx, a, C.byref(n)), ctx)
    return int(n.value)
