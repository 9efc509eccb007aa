/*
 * crocco.h -- C ABI of libcrocco.so, the B200 (sm_100a) implementation of the
 * data-parallel hot path of CRoCCo v2.0 (Davis et al., IPDPS 2023).
 *
 * Citations "PAPER.md:N" are lines of the paper text;
 * "reading N" refers to the readings table in DESIGN.md section 3, which fixes
 * everything the paper leaves unstated (scheme constants, eigenvectors, BCs ...).
 *
 * Call order follows Algorithm 1/2:
 *   crocco_init_grid      (InitGrid, Alg. 1 l.1)
 *   crocco_init_metrics   (InitGridMetrics, Alg. 1 l.2; coordinates held in memory)
 *   per RK stage: crocco_rk_stage = FillPatch + BC_Fill + WENOx/y/z + Viscous + Update
 *                 (Alg. 2 l.3-9), or the unfused crocco_fill_boundary / crocco_rhs /
 *                 crocco_rk_update used by the tests.
 *
 * Conventions
 *  - Every entry point returns crocco_status; CROCCO_OK == 0.  No C++ exception
 *    crosses the ABI.  Text for the last error: crocco_last_error(ctx) (or
 *    crocco_last_error(NULL) for failures before a ctx exists).
 *  - All field arrays are fp64, structure-of-arrays, CALLER-OWNED DEVICE memory,
 *    one pointer per LOCAL block (array of crocco_num_local_blocks pointers).
 *    Layout of every state/metric/rhs array of local block b: see
 *    crocco_block_layout; point (i,j,k) (interior 0 <= i < n[0] ..., ghosts down to
 *    -ghost) of component c is element
 *        c*comp_stride + offset + i + j*pitch_y + k*pitch_z.
 *    Coordinates use the same formula with coffset/cpitch_y/cpitch_z/ccomp_stride
 *    and ghost width ghost_coords (=10).  Allocate ncomp*comp_stride doubles
 *    (5 for U/dU/rhs, 10 for metrics, 3*ccomp_stride for xyz).  The library
 *    never frees or retains caller pointers beyond a call.
 *  - The library owns: the ctx, its device scratch (interface-flux buffers,
 *    primitive and viscous-flux buffers, halo staging; sized at init_grid and
 *    reported by crocco_scratch_bytes), the internal comm stream/events, and
 *    the NCCL communicator when nranks > 1.  All freed by crocco_finalize.
 *  - Execution: every call is asynchronous on desc.stream (a cudaStream_t);
 *    asynchronous device faults surface at crocco_sync.  After any CUDA/NCCL
 *    error the ctx is poisoned and later calls return CROCCO_ERR_STATE.
 *  - Collectives: init_grid, init_metrics, fill_boundary, rhs (does not
 *    communicate, but keep order) and rk_stage must be called by all ranks in
 *    the same order when nranks > 1.
 *  - Threading: not thread-safe; one ctx per process/GPU.
 */
#ifndef CROCCO_H
#define CROCCO_H

#include <stddef.h>
#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

typedef enum {
    CROCCO_OK = 0,
    CROCCO_ERR_ARG = 1,   /* invalid argument / shape (synchronous, nothing launched) */
    CROCCO_ERR_CUDA = 2,  /* CUDA launch/runtime failure */
    CROCCO_ERR_NCCL = 3,  /* NCCL failure */
    CROCCO_ERR_NOMEM = 4, /* device scratch allocation failed */
    CROCCO_ERR_STATE = 5  /* ctx poisoned by an earlier CUDA/NCCL error */
} crocco_status;

typedef struct crocco_ctx_s *crocco_ctx;

/* Boundary kinds per face (PAPER.md:83 BC_Fill; reading 15). */
enum {
    CROCCO_BC_PERIODIC = 0,  /* copy from the periodic partner; lo/hi must both be PERIODIC */
    CROCCO_BC_EXTRAP = 1,    /* zeroth-order extrapolation: ghost = nearest interior layer */
    CROCCO_BC_DIRICHLET = 2, /* ghost = constant conserved state dirichlet[d][side][0..4] */
    CROCCO_BC_WALL = 3,      /* no-slip adiabatic wall, mirror about the face at index -1/2 (n-1/2):
                                (rho, -rho u, -rho v, -rho w, E) of the mirrored interior point */
    CROCCO_BC_SLIPWALL = 4,  /* inviscid reflecting wall (DMR; reading 19): mirror, the
                                momentum reflected about the plane normal to n = m^d/|m^d| of the
                                mirrored point (needs the metrics in the fill) */
    CROCCO_BC_SPLIT = 5,     /* boundary data switching at a moving index (DMR bottom/top, reading 20):
                                see crocco_split; the right part may be DIRICHLET or SLIPWALL */
    CROCCO_BC_COARSE_FINE = 6 /* face of a fine AMR level inside the coarse domain (SURVEY NEXT-4,
                                readings 24-25): its ghosts are interpolated from the coarse level by
                                crocco_fill_patch_two_levels / crocco_amr_rk_stage; crocco_fill_boundary
                                leaves them untouched, crocco_rk_stage / rk3_step refuse the ctx */
};
enum { CROCCO_TERM_INVISCID = 1, CROCCO_TERM_VISCOUS = 2 }; /* bitmask (Alg. 2 l.5-7 / l.8) */
enum { CROCCO_MU_CONST = 0, CROCCO_MU_SUTHERLAND = 1 };
enum { CROCCO_FIELD_STATE = 0, CROCCO_FIELD_METRIC = 1 };
enum { CROCCO_GHOST = 4, CROCCO_GHOST_COORDS = 10 }; /* reading 7 */

/* SPLIT face data: ghost point with global index g along `axis` (a tangential axis
   of the face) takes the DIRICHLET state `left` if g + 1/2 < s(t) = i0 + di_dt * t,
   else `right_kind` (CROCCO_BC_DIRICHLET with state `right`, or CROCCO_BC_SLIPWALL). */
typedef struct {
    int32_t axis;
    double i0, di_dt;
    double left[5];
    int32_t right_kind;
    double right[5];
} crocco_split;

typedef struct {
    int64_t n_global[3];        /* interior points N_xi, N_eta, N_zeta of the whole domain */
    int32_t n_blocks[3];        /* equal boxes per direction; n_global[d] % n_blocks[d] == 0,
                                   block interior >= 4 points per direction */
    int32_t bc[3][2];           /* per direction d, side lo(0)/hi(1): CROCCO_BC_* */
    double dirichlet[3][2][5];  /* conserved ghost state for DIRICHLET faces */
    int32_t rank, nranks;       /* this process / world size */
    const int32_t *block_rank;  /* owner rank of global block b = bx + nbx*(by + nby*bz);
                                   NULL = all blocks on rank 0 (requires nranks == 1) */
    void *stream;               /* cudaStream_t the library enqueues on (NULL = legacy default) */
    const void *nccl_unique_id; /* 128-byte ncclUniqueId broadcast by the caller (torch.distributed);
                                   ignored when nranks == 1 */
    crocco_split split[3][2];   /* data of CROCCO_BC_SPLIT faces (ignored elsewhere) */
} crocco_grid_desc;

typedef struct {
    double gamma, R, Pr;   /* calorically perfect gas p = rho R T, c_v = R/(gamma-1), c_p = gamma c_v */
    int32_t mu_law;        /* CROCCO_MU_CONST: mu = mu_ref;
                              CROCCO_MU_SUTHERLAND: mu = mu_ref (T/T_ref)^{3/2} (T_ref+S)/(T+S) */
    double mu_ref, T_ref, S;
    double weno_eps;       /* WENO-SYMBO epsilon in alpha_k = C_k/(eps+beta_k)^2 (reading 8), 1e-6 */
    int32_t terms;         /* CROCCO_TERM_* bitmask */
    int32_t dir_mask;      /* inviscid directions evaluated, bit d = direction d (tests; 7 = all) */
    int32_t weno_weights;  /* optimal weights: 0 = SYMBO (bandwidth-optimised, Martin et al. 2006),
                              1 = SYMOO (1/20, 9/20, 9/20, 1/20: 6th-order central linear stencil);
                              reading 22, SURVEY NEXT-3 */
    int32_t weno_limiter;  /* WENO limiters (reading 23), bitmask, 0 = off: after
                              beta_3 <- max(beta), use the linear weights omega = C when
                              bit 0: max beta < weno_alpha_rl * min beta (relative limiter),
                              bit 1: max beta < weno_alpha_al (absolute limiter; beta of the
                              reconstructed characteristic flux (g +- lambda w)/2) */
    double weno_alpha_rl, weno_alpha_al;  /* thresholds, >= 0 */
    int32_t visc_form;     /* viscous discretisation: 0 = conservative point-flux form (reading 12,
                              default); 1 = expanded (non-conservative) form with the paper's
                              27-component metrics (readings 27-28):
                              needs crocco_init_metrics2 after crocco_init_metrics */
} crocco_phys;

typedef struct {
    int32_t n[3];          /* interior points of this block */
    int64_t origin[3];     /* global index of its interior point (0,0,0) */
    int32_t ghost;         /* 4 */
    int32_t ghost_coords;  /* 10 */
    int64_t offset;        /* element offset of interior point (0,0,0) inside one component */
    int64_t pitch_y, pitch_z, comp_stride;     /* elements; state / metric / rhs arrays */
    int64_t coffset, cpitch_y, cpitch_z, ccomp_stride; /* elements; coordinate arrays */
    int32_t global_id;     /* global block id b */
} crocco_block_layout;

/* One exchange message of the ghost fill (host-side plan, exposed for tests). */
typedef struct {
    int32_t phase;          /* direction d of the fill phase (0, 1, 2) */
    int32_t dst_block;      /* global id of the block whose ghosts are written */
    int32_t side;           /* 0 = lo face, 1 = hi face of dst_block */
    int32_t kind;           /* 0 = copy from src_block, 1 = physical BC (bc value in bc_kind) */
    int32_t bc_kind;        /* CROCCO_BC_* of the face */
    int32_t src_block;      /* global id of the source block (copy), -1 for physical */
    int32_t src_rank, dst_rank;
    int64_t dst_lo[3];      /* box of ghost points written, block-local indices, [lo, lo+ext) */
    int64_t src_lo[3];      /* box of source points read, src-block-local indices */
    int64_t ext[3];
} crocco_msg;

/* ---- setup --------------------------------------------------------------- */

/* Validate the decomposition, build neighbour tables and the exchange plan,
   allocate device scratch for the local blocks on the current CUDA device,
   create the NCCL communicator if nranks > 1.  Collective. */
crocco_status crocco_init_grid(const crocco_grid_desc *desc, const crocco_phys *phys,
                               crocco_ctx *out);
crocco_status crocco_num_local_blocks(crocco_ctx ctx, int32_t *n_local);
crocco_status crocco_get_block_layout(crocco_ctx ctx, int32_t local_block,
                                      crocco_block_layout *out);
/* Replace the gas / scheme constants (validated like crocco_init_grid).  Drops every cached
   RK3 step graph (crocco_rk3_step): a graph bakes in the kernel arguments and variants. */
crocco_status crocco_set_phys(crocco_ctx ctx, const crocco_phys *phys);
crocco_status crocco_scratch_bytes(crocco_ctx ctx, int64_t *bytes);

/* InitGridMetrics (readings 5-6): from the coordinates
   xyz (3 comps, interior +-10 filled by the caller) compute
   metrics (10 comps: 0 = J = 1/det(d x/d xi), 1+3d+a = m^d_a = (d xi_d/d x_a)/J,
   Thomas-Lombard form with the 6th-order central operator D6) on the whole
   padded box (interior +-4), then copy the periodic / inter-block ghost metrics
   from their owners (crocco_fill_boundary(METRIC)).  Collective. */
crocco_status crocco_init_metrics(crocco_ctx ctx, double *const *xyz, double *const *metrics);
/* The 18 second metrics of the paper's 27-component set (reading 27):
   xi_{a,jk} = d2 xi_a / dx_j dx_k = sum_b xi_{b,k} D6_b(xi_{a,j}), xi_{a,j} = J m^a_j, j <= k,
   component 6a + pair index of (00, 01, 02, 11, 12, 22), on interior points, computed from
   `metrics` (filled by crocco_init_metrics) into LIBRARY-OWNED device memory (18 fp64 per
   interior point; reported by crocco_scratch_bytes) used by the expanded viscous form
   (visc_form = 1).  Call again after changing the metrics.  Drops the cached RK3 step
   graphs.  Not collective. */
crocco_status crocco_init_metrics2(crocco_ctx ctx, double *const *metrics);
/* Copy local block b's second metrics to dst (device memory, 18 x n0 n1 n2 fp64, component
   q at q * n0 n1 n2 + i + n0 (j + n1 k)); tests.  CROCCO_ERR_STATE if not initialised. */
crocco_status crocco_copy_metrics2(crocco_ctx ctx, int32_t local_block, double *dst);

/* FillPatch + BC_Fill: in place on 4 ghost layers,
   phases xi -> eta (spanning xi ghosts) -> zeta (spanning xi, eta ghosts).
   kind STATE: 5 comps, copies + physical BCs at the ctx time (crocco_set_time).
   kind METRIC: 10 comps, periodic / inter-block copies only.  metrics: required
   for STATE fills when a face is SLIPWALL or SPLIT, else may be NULL.  Collective. */
crocco_status crocco_fill_boundary(crocco_ctx ctx, double *const *field, int32_t kind,
                                   double *const *metrics);
/* Simulation time t_n of the start of the current step (time-dependent SPLIT faces).
   crocco_rk_stage evaluates the boundary data of stage s at t_n + c_s dt,
   c = (0, 1/3, 3/4); crocco_rk3_step advances it by dt (t <- t + dt). */
crocco_status crocco_set_time(crocco_ctx ctx, double t);
crocco_status crocco_get_time(crocco_ctx ctx, double *t);

/* RHS: rhs = J ( -sum_d delta_d F^_inv^d + sum_d D4_d F^_v^d )
   on interior points (ghosts of rhs untouched).  U must have its ghosts filled;
   metrics from crocco_init_metrics.  rhs may not alias U. */
crocco_status crocco_rhs(crocco_ctx ctx, double *const *U, double *const *metrics,
                         double *const *rhs);

/* One Williamson low-storage RK3 stage (reading 13):
   fill(U_in) (in place on U_in's ghosts) + RHS + dU <- A_s dU + dt rhs,
   U_out = U_in + B_s dU on interior points; A = (0, -5/9, -153/128),
   B = (1/3, 15/16, 8/15).  dU is not read at stage 0.  U_out != U_in.
   Collective.  With viscous terms the ghost fill (local copies, physical BCs and
   the NCCL send/recv of remote faces) runs on an internal comm stream while the
   viscous tiles that read no ghost point run on `stream`; the rest of the stage
   waits for the fill (SURVEY 8(e) overlap; see crocco_set_overlap). */
crocco_status crocco_rk_stage(crocco_ctx ctx, int32_t stage, double dt, double *const *U_in,
                              double *const *U_out, double *const *dU,
                              double *const *metrics);

/* One full RK3 time step (Alg. 2 l.1: stages 1..3) = crocco_rk_stage(0: U -> V),
   (1: V -> U), (2: U -> V): the new state is in V, U was used for the middle stage.
   use_graph != 0: the three stages (fills, sweeps, update: ~20 kernels) are captured
   once per (U, V, dU, metrics, dt) into a CUDA graph and replayed with one launch
   (at most 4 graphs cached per ctx; eager launches when kernel timing is on,
   nranks > 1 or a SPLIT face moves in time).  Advances the ctx time by dt.  Collective. */
crocco_status crocco_rk3_step(crocco_ctx ctx, double dt, double *const *U, double *const *V,
                              double *const *dU, double *const *metrics, int32_t use_graph);

/* The Update step alone (tests): dU <- A_s dU + dt rhs ; U_out = U_in + B_s dU. */
crocco_status crocco_rk_update(crocco_ctx ctx, int32_t stage, double dt, double *const *U_in,
                               double *const *U_out, double *const *dU, double *const *rhs);

/* ComputeDt (Eq. 3, 95 Alg. 1 l.9, 131 ReduceRealMin):
   *dt = cfl / max_i sum_d J_i (|m^d_i . u_i| + c_i |m^d_i|) over the interior points of
   all blocks of all ranks (global reduction with ncclAllReduce(max) when nranks > 1).
   U: conserved state (ghosts not read); metrics from crocco_init_metrics; dt: HOST
   pointer.  Synchronises the stream.  Collective.  A non-finite local radius (NaN
   component, negative pressure) is not dropped by the maximum: CROCCO_ERR_ARG with
   "non-finite spectral radius". */
crocco_status crocco_compute_dt(crocco_ctx ctx, double *const *U, double *const *metrics,
                                double cfl, double *dt);

/* ---- two-level block-structured AMR (PAPER.md:56, 75, 83, 102-119,
   129, 141, 258; readings 24-26) --------------------------------------------
   A fine level is its own ctx (crocco_init_grid over the fine region, any equal-block
   decomposition) whose faces inside the coarse domain are CROCCO_BC_COARSE_FINE.  Refinement
   ratio 2, node-centred: fine node f (fine-level global index) lies at coarse index c0 + f/2.
   All levels take the same dt; per RK stage the coarse level runs first (Alg. 2 l.2 level loop
   inside the stage loop), then the fine level with its C/F ghosts interpolated from the coarse
   stage INPUT, then at stage 2 (the third) AverageDown.  Both ctx must enqueue on the same
   stream (or the caller orders them).
   The levels may be decomposed independently over the ranks (each level is
   distributed and load-balanced on its own).  Inter-level data then moves as NCCL p2p boxes on
   the fine ctx's communicator (plan: crocco_amr_plan, fixed at link time):
     - FillPatch: every coarse box a fine block's C/F ghosts interpolate from (the 8-corner
       stencils of its ghost boxes, coarse ghosts included) goes from the coarse block's rank to
       the fine block's rank, into a mirror of that coarse block; the interpolation reads the
       mirror (bitwise the values it would read from the coarse block itself);
     - AverageDown: the covered coarse nodes whose central fine node lies in a fine block are
       averaged on the fine block's rank (into a mirror of the coarse block) and sent to the
       coarse block's rank, which writes them into U_coarse.
   Boxes whose coarse and fine blocks share a rank are read / written in place (or through
   ncclSend/ncclRecv to self under crocco_set_nccl_loopback on the FINE ctx).  So the two-level
   calls are collective over the fine ctx's communicator: every rank calls them, also a rank
   that owns no fine block (it may still own coarse blocks that others read).
   Several patches of one level: see the sibling calls below. */

/* Declare `fine` a refinement of `coarse` with fine node 0 at coarse node c0[3].  Checks:
   per direction either the fine level is PERIODIC and spans the periodic coarse domain
   (N_f = 2 N_c, c0 = 0), or 0 <= c0 and 2 c0 + N_f - 1 <= 2 (N_c - 1) with physical (non-C/F)
   faces only on the domain boundary; <= 512 blocks per level; local coarse blocks + coarse
   mirrors of this rank <= 64; both ctx on the same ranks; a communicator on the fine ctx when
   the plan has inter-rank boxes.  CROCCO_ERR_ARG otherwise.  Allocates the coarse-block
   mirrors and the staging buffers of the plan (crocco_scratch_bytes counts them).  The ctx keep
   no reference beyond the pair (finalize the fine level first or relink). */
crocco_status crocco_amr_link(crocco_ctx fine, crocco_ctx coarse, const int64_t c0[3]);
/* FillPatch of the fine level (FillPatchTwoLevels + BC_Fill; reading 25):
   the 3-phase fill of U_fine in place, COARSE_FINE ghosts = trilinear interpolation from the
   coarse state U_coarse (one device pointer per coarse local block; its ghosts must be filled,
   e.g. by the coarse level's own fill of this stage).  metrics_fine as crocco_fill_boundary.
   Collective over the fine level. */
crocco_status crocco_fill_patch_two_levels(crocco_ctx fine, double *const *U_fine,
                                           double *const *metrics_fine, double *const *U_coarse);
/* crocco_rk_stage of the fine level with its C/F ghosts interpolated from U_coarse_in, the
   coarse level's input state of the same stage (ghosts filled). */
crocco_status crocco_amr_rk_stage(crocco_ctx fine, int32_t stage, double dt, double *const *U_in,
                                  double *const *U_out, double *const *dU, double *const *metrics,
                                  double *const *U_coarse_in);
/* AverageDown (Alg. 2 l.10-12; reading 26): refills the same-level ghosts of U_fine
   (periodic / inter-block copies only), then every covered coarse node of U_coarse (interior
   points only) becomes the full-weighting (trapezoid) average of the fine data over its cell. */
crocco_status crocco_average_down(crocco_ctx fine, double *const *U_fine, double *const *U_coarse);

/* ---- same-level sibling patches (NEXT-4 completion; a level is a union of
   patches, FillPatchSingleLevel -> FillBoundary exchanges their ghosts; reading 31) ---
   Declare two fine patches of the same level (both crocco_amr_link'ed to the same coarse ctx,
   interiors disjoint, even fine offset 2 (c0_g - c0_f), the same ranks) siblings of each other;
   symmetric, idempotent; <= 8 siblings / 16 sibling blocks (all ranks) per patch; CROCCO_ERR_ARG
   otherwise.  Sibling blocks on other ranks (or all of them under the loopback) reach the patch
   as kind-2 boxes of its plan (crocco_amr_sibling_plan) through NCCL p2p into sibling-block
   mirrors, so the _level calls are collective over the patch's communicator.
   With siblings, the _level calls below replace the two-level calls; `sib` holds, for each
   sibling in link order, the pointer array of its local blocks (caller-owned, device):
   - C/F ghosts lying inside a sibling's interior take the sibling's value (the stage INPUT of
     the sibling for crocco_amr_rk_stage_level), all others are interpolated as before;
   - AverageDown averages the coarse nodes whose central fine node lies in this patch and whose
     27 fine nodes lie in the interiors of this patch or its siblings (`sib` = the siblings'
     updated states), so each covered node of the level is written by exactly one patch.
   Two abutting patches then advance exactly like the one patch covering their union (oracle
   pin tests/test_oracle_amr.py; GPU parity tests/test_gpu_amr.py). */
crocco_status crocco_amr_link_sibling(crocco_ctx fine, crocco_ctx sibling);
crocco_status crocco_fill_patch_level(crocco_ctx fine, double *const *U_fine, double *const *metrics_fine,
                                      double *const *U_coarse, double *const *const *sib);
crocco_status crocco_amr_rk_stage_level(crocco_ctx fine, int32_t stage, double dt, double *const *U_in,
                                        double *const *U_out, double *const *dU, double *const *metrics,
                                        double *const *U_coarse_in, double *const *const *sib_in);
crocco_status crocco_average_down_level(crocco_ctx fine, double *const *U_fine, double *const *U_coarse,
                                        double *const *const *sib);

/* State check (SURVEY sec. 5 failure detection; test / bench utility): *n_bad = number of
   interior points of all local blocks with a non-finite component, rho <= 0 or p <= 0
   (p from the ctx's gamma).  n_bad: HOST pointer.  Synchronises the stream.  Not collective. */
crocco_status crocco_check_state(crocco_ctx ctx, double *const *U, int64_t *n_bad);

/* Block until all work of the ctx finished; surfaces asynchronous errors. */
crocco_status crocco_sync(crocco_ctx ctx);
const char *crocco_last_error(crocco_ctx ctx);
crocco_status crocco_finalize(crocco_ctx ctx);

/* Overlap of the ghost exchange with interior compute inside crocco_rk_stage /
   crocco_rk3_step: 1 on, 0 off, -1 auto (default: on when nranks > 1, i.e. when
   the fill has NCCL faces; a purely local fill is too short to hide and the split
   viscous launch costs more than it saves -- measured on one B200).  Results are
   bitwise identical either way: the fill writes only ghost points, the overlapped
   tiles read only interior points.  CROCCO_ERR_ARG for other values.  Changing it
   drops the cached RK3 step graphs (the stage structure differs).  With overlap the
   viscous slab depth is capped so that an interior slab exists ((n2 - 4)/vk >= 2). */
crocco_status crocco_set_overlap(crocco_ctx ctx, int32_t enable);

/* ---- instrumentation (bench / tests) ---------------------------------------- */

/* Number of kernels this ctx launched since init (or the last reset). */
crocco_status crocco_launch_count(crocco_ctx ctx, int64_t *count, int32_t reset);
/* Debug / hardware check of the NCCL halo path on ONE GPU (nranks == 1 only): with enable != 0
   the library creates a 1-rank NCCL communicator and routes every same-rank inter-block and
   periodic ghost copy of crocco_fill_boundary / crocco_rk_stage through the multi-rank code path
   -- pack kernel -> ncclGroupStart; ncclSend + ncclRecv to itself; ncclGroupEnd -> unpack kernel
   -- and crocco_compute_dt through ncclAllReduce(max) on that communicator; on a fine AMR level
   also every inter-level box of crocco_amr_plan (coarse mirrors filled / averaged values
   returned through ncclSend + ncclRecv to itself).  Results are bitwise those of the local copies.  Steps launch eagerly (no graphs) while a communicator exists.
   enable = 0 destroys the communicator.  CROCCO_ERR_ARG when nranks > 1. */
crocco_status crocco_set_nccl_loopback(crocco_ctx ctx, int32_t enable);
/* Number of RK stages that ran overlapped (fill on the comm stream beside the ghost-free
   viscous tiles) since init (or the last reset); graph replays count their captured stages.
   Lets tests assert that the overlap path really ran. */
crocco_status crocco_overlap_count(crocco_ctx ctx, int64_t *count, int32_t reset);
/* Kernel-class timing with CUDA events recorded on the launching stream.
   When enabled, every launch of class k is bracketed by events; crocco_kernel_times
   returns, per class, the number of launches and the summed milliseconds
   (synchronises).  Classes: see crocco_kernel_class_name. */
crocco_status crocco_set_timing(crocco_ctx ctx, int32_t enable);
crocco_status crocco_kernel_times(crocco_ctx ctx, int32_t max_classes, int64_t *launches,
                                  double *ms, int32_t *n_classes);
const char *crocco_kernel_class_name(int32_t cls);

/* ---- host-only helpers (no CUDA needed; used by the CPU tests) -------------- */

/* The ghost-exchange plan of desc for phase d and rank desc->rank: every
   message whose dst block or src block lives on this rank, in the canonical
   order both sides use for NCCL send/recv matching.  Writes up to cap entries,
   *n_out = total count. */
crocco_status crocco_exchange_plan(const crocco_grid_desc *desc, int32_t phase, crocco_msg *out,
                                   int32_t cap, int32_t *n_out);
/* One inter-level box of a two-level AMR pair (crocco_amr_link; ratio 2, node-centred). */
typedef struct {
    int32_t kind;          /* 0 = FillPatch: coarse values to the fine block's rank (its C/F ghosts
                              interpolate from them); 1 = AverageDown: averaged coarse values from
                              the fine block's rank to the coarse block's rank; 2 = sibling ghosts:
                              interior values of a same-level sibling block to the fine block's
                              rank (its C/F ghosts inside the sibling copy them) */
    int32_t coarse_block;  /* global id of the coarse block (the box is in its local indices) */
    int32_t fine_block;    /* global id of the fine block the box serves */
    int32_t sibling;       /* kind 2: index of the sibling patch in link order; -1 otherwise */
    int32_t src_rank, dst_rank;
    int64_t lo[3];         /* coarse-block-local box [lo, lo+ext); kind 0 may reach into the
                              coarse ghosts, kind 1 lies in the interior; kind 2: box of the
                              sibling block (coarse_block = its global id in the sibling patch) */
    int64_t ext[3];
} crocco_amr_msg;
/* The inter-level plan of fine level `fine` linked at coarse node c0 to `coarse`, for rank
   fine->rank: every box it sends or receives (src_rank or dst_rank = rank; both for boxes
   local to the rank), kind 0 first, each kind in the canonical order both sides use for NCCL
   matching (fine block id, then phase / side of the C/F ghost box, then coarse block id).
   Kind 0: for each C/F ghost box of a fine block, per coarse block, the coarse nodes I and I+1
   per direction of the corners its trilinear stencils read, I = floor((2 c0 + f)/2), with the
   owner block of I chosen by clamping I into the domain (k_cf_interp).  Kind 1: per fine block
   and coarse block, the covered nodes (reading 26) whose central fine node 2 (I - c0) lies in
   the fine block.  Writes up to cap entries, *n_out = total count; CROCCO_ERR_ARG for
   descriptors crocco_amr_link would refuse.  Without sibling semantics: a patch with siblings
   gets the kind-1 boxes of the sibling rule and its kind-2 boxes from crocco_amr_link_sibling. */
crocco_status crocco_amr_plan(const crocco_grid_desc *fine, const crocco_grid_desc *coarse, const int64_t c0[3],
                              crocco_amr_msg *out, int32_t cap, int32_t *n_out);
/* Kind-2 boxes (sibling index `sibling`) of fine patch `fine` at coarse node c0 with its sibling
   patch `sib` at coarse node c0s, for rank fine->rank: per fine block (id order), per C/F ghost
   box (phase, side), per sibling block (id order), the part of the ghost box inside the sibling
   block's interior, in the sibling block's local indices.  crocco_amr_link_sibling adds these to
   both patches' plans (and then computes the kind-1 boxes over the nodes whose central fine node
   is the patch's, which k_average_down filters by the 27-node rule).  Host only. */
crocco_status crocco_amr_sibling_plan(const crocco_grid_desc *fine, const int64_t c0[3], const crocco_grid_desc *sib,
                                      const int64_t c0s[3], int32_t sibling, crocco_amr_msg *out, int32_t cap,
                                      int32_t *n_out);
/* Generate an ncclUniqueId (128 bytes written to out, size >= 128) on the rank
   that bootstraps the communicator; the caller broadcasts it (torch.distributed)
   and passes it as desc.nccl_unique_id on every rank. */
crocco_status crocco_nccl_unique_id(void *out, int32_t size);
/* Library version string. */
const char *crocco_version(void);

#ifdef __cplusplus
}
#endif
#endif /* CROCCO_H */
