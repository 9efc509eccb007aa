// crocco.cu -- host side of libcrocco.so: the C ABI of include/crocco.h.
//
// Block decomposition, ghost-exchange plan, scratch management, launch
// orchestration of the sm_100a kernels (sweep/pointwise/fill/metrics .cuh), NCCL halo exchange.
// Algorithm 1/2 of the paper is the call order; every
// numerical step runs in the CUDA kernels, never on the host.
#include <cuda_runtime.h>
#include <nccl.h>
#include <nvtx3/nvToolsExt.h>

#include <algorithm>
#include <cmath>
#include <cstdarg>
#include <cstdio>
#include <cstring>
#include <functional>
#include <string>
#include <vector>

#include "../../include/crocco.h"
#include "amr.cuh"
#include "fill.cuh"
#include "metrics.cuh"
#include "pointwise.cuh"
#include "sweep.cuh"
#include "viscexp.cuh"

using namespace crocco;

namespace {

thread_local std::string g_err;  // error text before a ctx exists

struct BlockGeom {
    int gid;
    int bidx[3];
    int n[3];
    int64_t origin[3];
    int rank;
};

struct LocalBlock {
    BlockGeom g;
    Lay L;       // state/metric layout
    Lay C;       // coordinate layout
    VLay V;      // viscous-flux box
    double *racc = nullptr;  // RHS accumulator R (5 comps, compact interior)
    int64_t rcs = 0;
    double *fv = nullptr;    // viscous point flux F^_v^eta (4 comps, interior +-2 box)
    double *met2 = nullptr;  // expanded viscous form: 18 second metrics (compact interior, rcs)
};

enum { K_RESERVED = 0, K_FLUX_X, K_FLUX_Y, K_FLUX_Z, K_VISC, K_UPDATE, K_FILL, K_METRICS, K_CFL, K_AMR,
       K_NCLASS };
const char *k_names[K_NCLASS] = {"unused", "sweep_xi", "sweep_eta", "sweep_zeta_update", "viscous",
                                 "update", "fill", "metrics", "compute_dt", "amr"};
// internal fill kind: 5-component state, periodic / inter-block copies only (AverageDown)
enum { FILL_STATE_COPIES = 100 };

// NVTX range of a host-side region (tracing): visible in nsys / ncu --nvtx
struct NvtxRange {
    explicit NvtxRange(const char *name) { nvtxRangePushA(name); }
    ~NvtxRange() { nvtxRangePop(); }
};

struct TimedLaunch {
    int cls;
    cudaEvent_t e0, e1;
};

}  // namespace

struct crocco_ctx_s {
    crocco_grid_desc desc;
    std::vector<int32_t> block_rank;
    crocco_phys phys_in;
    Phys ph;
    cudaStream_t stream = nullptr;
    std::vector<BlockGeom> all;
    std::vector<LocalBlock> loc;
    std::vector<int> gid_to_local;
    int nb[3];
    int bn[3];  // block interior size
    std::string err;
    bool poisoned = false;
    int64_t launches = 0;
    int64_t scratch = 0;
    // exchange plan per phase
    std::vector<crocco_msg> plan[3];
    // NCCL
    ncclComm_t comm = nullptr;
    bool loopback = false;  // debug: same-rank copies through ncclSend/ncclRecv to self (crocco_set_nccl_loopback)
    double *send_stage = nullptr, *recv_stage = nullptr;
    unsigned long long *dmax = nullptr;  // ComputeDt reduction cell
    // CUDA graphs of full RK3 steps, keyed by (buffers, dt)
    struct StepGraph {
        std::vector<const void *> key;
        double dt;
        cudaGraphExec_t exec;
        int64_t nodes;
        int64_t ov_stages;  // overlapped stages inside the captured step
    };
    std::vector<StepGraph> graphs;
    cudaStream_t cap_stream = nullptr;
    // overlapped stage: ghost fill / exchange on comm_stream beside the interior viscous tiles
    int overlap = -1;  // -1 auto (on when the fill has remote faces, nranks > 1), 0 off, 1 on
    int64_t overlapped_stages = 0;  // stages that ran the fill beside the ghost-free tiles
    cudaStream_t comm_stream = nullptr;
    cudaEvent_t ev_fork = nullptr, ev_join = nullptr;
    double time = 0.0;  // start of the current step (time-dependent SPLIT faces)
    // two-level AMR (NEXT-4): this ctx as the fine level of `amr_coarse`
    bool has_cf = false;                 // some face is CROCCO_BC_COARSE_FINE
    crocco_ctx amr_coarse = nullptr;     // set by crocco_amr_link
    int64_t amr_c0[3] = {0, 0, 0};       // coarse index of fine node 0
    double *const *amr_Uc = nullptr;     // coarse state of the current two-level call only
    std::vector<crocco_ctx> sibs;        // same-level sibling patches (crocco_amr_link_sibling)
    double *const *const *amr_sibU = nullptr;  // their states for the current call only
    // inter-level boxes touching this rank (crocco_amr_plan), the coarse-block mirrors they fill
    // (allocated on first use) and their NCCL staging
    std::vector<crocco_amr_msg> amr_plan;
    std::vector<int> amr_mirror_gid;
    std::vector<double *> amr_mirror;
    std::vector<int> amr_cf_gids;        // coarse blocks read from mirrors by the current fill
    std::vector<int> amr_smirror_key;    // sibling-block mirrors: key sibling * AMR_MAX_BLOCKS + gid
    std::vector<double *> amr_smirror;
    double *amr_send = nullptr, *amr_recv = nullptr;
    int64_t amr_stage_elems = 0;
    int64_t stage_elems = 0;
    // timing
    bool timing = false;
    std::vector<TimedLaunch> pending;
    std::vector<cudaEvent_t> pool;
    int64_t t_launch[K_NCLASS] = {0};
    double t_ms[K_NCLASS] = {0};
};

// ---------------------------------------------------------------------------
// error helpers
// ---------------------------------------------------------------------------
static crocco_status fail(crocco_ctx c, crocco_status st, const char *fmt, ...) {
    char buf[512];
    va_list ap;
    va_start(ap, fmt);
    vsnprintf(buf, sizeof buf, fmt, ap);
    va_end(ap);
    if (c) {
        c->err = buf;
        if (st == CROCCO_ERR_CUDA || st == CROCCO_ERR_NCCL) c->poisoned = true;
    } else {
        g_err = buf;
    }
    return st;
}
#define CK(ctx, call)                                                                          \
    do {                                                                                       \
        cudaError_t e_ = (call);                                                               \
        if (e_ != cudaSuccess)                                                                 \
            return fail(ctx, CROCCO_ERR_CUDA, "%s:%d %s: %s", __FILE__, __LINE__, #call,       \
                        cudaGetErrorString(e_));                                               \
    } while (0)
#define NK(ctx, call)                                                                          \
    do {                                                                                       \
        ncclResult_t r_ = (call);                                                              \
        if (r_ != ncclSuccess)                                                                 \
            return fail(ctx, CROCCO_ERR_NCCL, "%s:%d %s: %s", __FILE__, __LINE__, #call,       \
                        ncclGetErrorString(r_));                                               \
    } while (0)
#define LIVE(ctx)                                                                              \
    do {                                                                                       \
        if (!(ctx)) return fail(nullptr, CROCCO_ERR_ARG, "null ctx");                           \
        if ((ctx)->poisoned) return CROCCO_ERR_STATE;                                          \
    } while (0)

// launch bookkeeping: count + optional event timing on the launching stream
static void pre_launch(crocco_ctx c, int cls, TimedLaunch *tl) {
    c->launches++;
    if (!c->timing) return;
    auto get = [&]() {
        cudaEvent_t e;
        if (!c->pool.empty()) {
            e = c->pool.back();
            c->pool.pop_back();
        } else {
            cudaEventCreate(&e);
        }
        return e;
    };
    tl->cls = cls;
    tl->e0 = get();
    tl->e1 = get();
    cudaEventRecord(tl->e0, c->stream);
}
static crocco_status post_launch(crocco_ctx c, TimedLaunch *tl) {
    cudaError_t e = cudaGetLastError();
    if (e != cudaSuccess) return fail(c, CROCCO_ERR_CUDA, "kernel launch: %s", cudaGetErrorString(e));
    if (c->timing) {
        cudaEventRecord(tl->e1, c->stream);
        c->pending.push_back(*tl);
    }
    return CROCCO_OK;
}
#define LAUNCH(ctx, cls, ...)                                                                  \
    do {                                                                                       \
        TimedLaunch tl_;                                                                       \
        pre_launch(ctx, cls, &tl_);                                                            \
        __VA_ARGS__;                                                                           \
        crocco_status s_ = post_launch(ctx, &tl_);                                             \
        if (s_ != CROCCO_OK) return s_;                                                        \
    } while (0)

static inline int64_t rup(int64_t x, int64_t m) { return (x + m - 1) / m * m; }
static inline unsigned cdiv(int64_t a, int64_t b) { return (unsigned)((a + b - 1) / b); }

// padded layout: rows aligned to 128 B with interior i=0 on a 128-B boundary
static Lay make_layout(const int n[3], int g) {
    Lay L;
    L.n0 = n[0];
    L.n1 = n[1];
    L.n2 = n[2];
    const int64_t lead = 16;  // interior starts at element 16 of each row
    L.py = rup(lead + n[0] + g + 8, 16);  // +8: whole 8-column tiles of the sweeps stay in the row
    L.pz = L.py * (n[1] + 2 * g);
    L.off = lead + L.py * g + L.pz * g;
    L.cs = L.pz * (n[2] + 2 * g);
    return L;
}

// ---------------------------------------------------------------------------
// decomposition + exchange plan (host only)
// ---------------------------------------------------------------------------
static crocco_status validate(const crocco_grid_desc *d, int nb[3], int bn[3]) {
    if (!d) return fail(nullptr, CROCCO_ERR_ARG, "null desc");
    for (int a = 0; a < 3; a++) {
        if (d->n_blocks[a] < 1 || d->n_global[a] < 1)
            return fail(nullptr, CROCCO_ERR_ARG, "bad n_global/n_blocks in direction %d", a);
        if (d->n_global[a] % d->n_blocks[a])
            return fail(nullptr, CROCCO_ERR_ARG, "n_global[%d]=%lld not divisible by n_blocks=%d", a,
                        (long long)d->n_global[a], d->n_blocks[a]);
        nb[a] = d->n_blocks[a];
        int64_t b = d->n_global[a] / nb[a];
        if (b < G) return fail(nullptr, CROCCO_ERR_ARG, "block interior %lld < ghost width 4 in direction %d",
                               (long long)b, a);
        if (b > 65535) return fail(nullptr, CROCCO_ERR_ARG, "block interior > 65535 points in direction %d", a);
        bn[a] = (int)b;
        for (int s = 0; s < 2; s++)
            if (d->bc[a][s] < 0 || d->bc[a][s] > CROCCO_BC_COARSE_FINE)
                return fail(nullptr, CROCCO_ERR_ARG, "bad bc kind %d", d->bc[a][s]);
        for (int s = 0; s < 2; s++)
            if (d->bc[a][s] == CROCCO_BC_SPLIT) {
                const crocco_split &sp = d->split[a][s];
                if (sp.axis < 0 || sp.axis > 2 || sp.axis == a)
                    return fail(nullptr, CROCCO_ERR_ARG, "SPLIT face %d/%d: axis must be tangential", a, s);
                if (sp.right_kind != CROCCO_BC_DIRICHLET && sp.right_kind != CROCCO_BC_SLIPWALL)
                    return fail(nullptr, CROCCO_ERR_ARG, "SPLIT face %d/%d: right_kind must be DIRICHLET or SLIPWALL", a, s);
            }
        if ((d->bc[a][0] == CROCCO_BC_PERIODIC) != (d->bc[a][1] == CROCCO_BC_PERIODIC))
            return fail(nullptr, CROCCO_ERR_ARG, "PERIODIC must be paired in direction %d", a);
    }
    if (d->nranks < 1 || d->rank < 0 || d->rank >= d->nranks)
        return fail(nullptr, CROCCO_ERR_ARG, "bad rank/nranks");
    const int nbt = nb[0] * nb[1] * nb[2];
    if (!d->block_rank && d->nranks != 1)
        return fail(nullptr, CROCCO_ERR_ARG, "block_rank required when nranks > 1");
    if (d->block_rank)
        for (int b = 0; b < nbt; b++)
            if (d->block_rank[b] < 0 || d->block_rank[b] >= d->nranks)
                return fail(nullptr, CROCCO_ERR_ARG, "block_rank[%d] out of range", b);
    return CROCCO_OK;
}

static void build_blocks(const crocco_grid_desc *d, const int nb[3], const int bn[3],
                         std::vector<BlockGeom> &all) {
    all.clear();
    for (int bz = 0; bz < nb[2]; bz++)
        for (int by = 0; by < nb[1]; by++)
            for (int bx = 0; bx < nb[0]; bx++) {
                BlockGeom g;
                g.gid = bx + nb[0] * (by + nb[1] * bz);
                g.bidx[0] = bx;
                g.bidx[1] = by;
                g.bidx[2] = bz;
                for (int a = 0; a < 3; a++) {
                    g.n[a] = bn[a];
                    g.origin[a] = (int64_t)g.bidx[a] * bn[a];
                }
                g.rank = d->block_rank ? d->block_rank[g.gid] : 0;
                all.push_back(g);
            }
}

// every message of phase `phase` touching rank `me` (me < 0: all), canonical order
static void build_plan(const crocco_grid_desc *d, const int nb[3], const int bn[3],
                       const std::vector<BlockGeom> &all, int phase, int me,
                       std::vector<crocco_msg> &out) {
    out.clear();
    const int D = phase;
    for (const BlockGeom &b : all) {
        for (int side = 0; side < 2; side++) {
            crocco_msg m;
            memset(&m, 0, sizeof m);
            m.phase = D;
            m.dst_block = b.gid;
            m.side = side;
            m.bc_kind = d->bc[D][side];
            m.dst_rank = b.rank;
            // ghost box
            for (int e = 0; e < 3; e++) {
                if (e == D) {
                    m.dst_lo[e] = side == 0 ? -G : bn[e];
                    m.ext[e] = G;
                } else if (e < D) {
                    m.dst_lo[e] = -G;
                    m.ext[e] = bn[e] + 2 * G;
                } else {
                    m.dst_lo[e] = 0;
                    m.ext[e] = bn[e];
                }
                m.src_lo[e] = m.dst_lo[e];
            }
            int nbi = b.bidx[D] + (side == 0 ? -1 : 1);
            bool physical = false;
            if (nbi < 0 || nbi >= nb[D]) {
                if (d->bc[D][side] == CROCCO_BC_PERIODIC)
                    nbi = (nbi + nb[D]) % nb[D];
                else
                    physical = true;
            }
            if (physical) {
                m.kind = 1;
                m.src_block = -1;
                m.src_rank = b.rank;
            } else {
                int idx[3] = {b.bidx[0], b.bidx[1], b.bidx[2]};
                idx[D] = nbi;
                const int sg = idx[0] + nb[0] * (idx[1] + nb[1] * idx[2]);
                m.kind = 0;
                m.src_block = sg;
                m.src_rank = all[sg].rank;
                m.src_lo[D] = side == 0 ? bn[D] - G : 0;
            }
            if (me < 0 || m.dst_rank == me || (m.kind == 0 && m.src_rank == me)) out.push_back(m);
        }
    }
}

constexpr int SEG_MIN = 32;        // shortest march segment of a sweep line (small blocks split lines)
constexpr int SEG_WARPS = 16384;   // lines are split until at least this many warps march
template <int D, bool V>
static constexpr size_t sweep_smem_bytes() {
    return (size_t)(sweep_threads(D) / 32) * RingGeom<D, V>::PER_WARP * sizeof(double);
}
template <int D, bool V, int MODE>
static cudaError_t sweep_attr1() {
    cudaError_t e = cudaFuncSetAttribute(k_sweep_s<D, V, false, MODE>, cudaFuncAttributeMaxDynamicSharedMemorySize,
                                         (int)sweep_smem_bytes<D, V>());
    if (e == cudaSuccess)
        e = cudaFuncSetAttribute(k_sweep_s<D, V, true, MODE, 2>, cudaFuncAttributeMaxDynamicSharedMemorySize,
                                 (int)sweep_smem_bytes<D, V>());
    if (e == cudaSuccess)  // no inviscid term in this direction (dir_mask / terms): the limiter is moot
        e = cudaFuncSetAttribute(k_sweep_s<D, V, false, MODE, 0>, cudaFuncAttributeMaxDynamicSharedMemorySize,
                                 (int)sweep_smem_bytes<D, V>());
    return e;
}
static cudaError_t sweep_attrs() {
    // the variants rhs_block launches: only the eta sweep carries a viscous interface term; modes:
    // xi 0 (write R) or 4 (add to the viscous divergence), eta 1 (add), zeta 2 (rhs) or 3 (RK update)
    cudaError_t e = sweep_attr1<0, false, 0>();
    if (e == cudaSuccess) e = sweep_attr1<0, false, 4>();
    if (e == cudaSuccess) e = sweep_attr1<1, false, 1>();
    if (e == cudaSuccess) e = sweep_attr1<1, true, 1>();
    if (e == cudaSuccess) e = sweep_attr1<2, false, 2>();
    if (e == cudaSuccess) e = sweep_attr1<2, false, 3>();
    if (e == cudaSuccess)
        e = cudaFuncSetAttribute(k_visc_tiled<0>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)VISC_SMEM);
    if (e == cudaSuccess)
        e = cudaFuncSetAttribute(k_visc_tiled<1>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)VISC_SMEM);
    if (e == cudaSuccess)
        e = cudaFuncSetAttribute(k_visc_exp_tiled, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)VISC_EXP_SMEM);
    return e;
}

// one launch of the viscous kernel over `nt` tiles (sel / vk as k_visc_tiled)
static crocco_status launch_visc(crocco_ctx c, const LocalBlock &b, const double *U, const double *M,
                                 const Phys &ph, int64_t nt, int sel, int vk) {
    if (ph.mu_law == 1)
        LAUNCH(c, K_VISC, k_visc_tiled<1><<<(unsigned)nt, VTX * VTY, VISC_SMEM, c->stream>>>(
                              U, M, b.fv, b.L, b.V, ph, b.racc, b.rcs, sel, vk));
    else
        LAUNCH(c, K_VISC, k_visc_tiled<0><<<(unsigned)nt, VTX * VTY, VISC_SMEM, c->stream>>>(
                              U, M, b.fv, b.L, b.V, ph, b.racc, b.rcs, sel, vk));
    return CROCCO_OK;
}

// ---------------------------------------------------------------------------
// ABI
// ---------------------------------------------------------------------------
extern "C" {

crocco_status crocco_nccl_unique_id(void *out, int32_t size) {
    if (!out || size < (int32_t)sizeof(ncclUniqueId))
        return fail(nullptr, CROCCO_ERR_ARG, "need a %zu-byte buffer", sizeof(ncclUniqueId));
    ncclUniqueId id;
    ncclResult_t r = ncclGetUniqueId(&id);
    if (r != ncclSuccess) return fail(nullptr, CROCCO_ERR_NCCL, "ncclGetUniqueId: %s", ncclGetErrorString(r));
    memcpy(out, &id, sizeof id);
    return CROCCO_OK;
}

const char *crocco_version(void) { return "crocco-b200 0.1 (sm_100a, fp64)"; }

const char *crocco_last_error(crocco_ctx c) { return c ? c->err.c_str() : g_err.c_str(); }

const char *crocco_kernel_class_name(int32_t cls) {
    return (cls >= 0 && cls < K_NCLASS) ? k_names[cls] : "";
}

crocco_status crocco_exchange_plan(const crocco_grid_desc *desc, int32_t phase, crocco_msg *out,
                                   int32_t cap, int32_t *n_out) {
    int nb[3], bn[3];
    crocco_status st = validate(desc, nb, bn);
    if (st) return st;
    if (phase < 0 || phase > 2) return fail(nullptr, CROCCO_ERR_ARG, "phase out of range");
    std::vector<BlockGeom> all;
    build_blocks(desc, nb, bn, all);
    std::vector<crocco_msg> plan;
    build_plan(desc, nb, bn, all, phase, desc->rank, plan);
    if (n_out) *n_out = (int32_t)plan.size();
    for (int i = 0; i < (int)plan.size() && i < cap; i++) out[i] = plan[i];
    return CROCCO_OK;
}

static Phys to_phys(const crocco_phys *p) {
    Phys ph;
    ph.gamma = p->gamma;
    ph.gm1 = p->gamma - 1.0;
    ph.igm1 = 1.0 / (p->gamma - 1.0);
    ph.R = p->R;
    ph.Pr = p->Pr;
    ph.cp_over_Pr = p->gamma * p->R / ((p->gamma - 1.0) * p->Pr);
    ph.mu_law = p->mu_law;
    ph.mu_ref = p->mu_ref;
    ph.T_ref = p->T_ref;
    ph.iT_ref = p->T_ref > 0 ? 1.0 / p->T_ref : 0.0;
    ph.S = p->S;
    ph.eps = p->weno_eps;
    ph.terms = p->terms;
    ph.dir_mask = p->dir_mask;
    static const double SYMBO[4] = {0.094647545896, 0.428074212384, 0.408289331408, 0.068988910311};
    static const double SYMOO[4] = {1.0 / 20.0, 9.0 / 20.0, 9.0 / 20.0, 1.0 / 20.0};
    for (int k = 0; k < 4; k++) ph.wC[k] = p->weno_weights == 1 ? SYMOO[k] : SYMBO[k];
    ph.lim = p->weno_limiter;
    ph.arl = p->weno_alpha_rl;
    // b_k of the kernels = (12/13) beta_k of the reconstructed values, which carry a factor 2
    // (LLF 1/2 folded, flux.cuh): b = (48/13) beta of (g +- lambda w)/2
    ph.aal_b = p->weno_alpha_al * (4.0 * WENO_BSCALE);
    ph.visc_form = p->visc_form;
    // only the ratios C_k / C_0 enter W (weno.cuh); alpha_0 then needs no multiply
    const double c0 = ph.wC[0];
    for (int k = 0; k < 4; k++) ph.wC[k] = k == 0 ? 1.0 : ph.wC[k] / c0;
    return ph;
}

static crocco_status check_phys(const crocco_phys *p) {
    if (!p) return fail(nullptr, CROCCO_ERR_ARG, "null phys");
    if (!(p->gamma > 1.0) || !(p->R > 0) || !(p->Pr > 0) || !(p->weno_eps > 0))
        return fail(nullptr, CROCCO_ERR_ARG, "bad gas constants (need gamma>1, R>0, Pr>0, eps>0)");
    if (p->mu_law != 0 && p->mu_law != 1) return fail(nullptr, CROCCO_ERR_ARG, "bad mu_law");
    if (p->mu_law == 1 && !(p->T_ref > 0)) return fail(nullptr, CROCCO_ERR_ARG, "bad T_ref");
    if (p->terms & ~3) return fail(nullptr, CROCCO_ERR_ARG, "bad terms mask");
    if (p->weno_weights != 0 && p->weno_weights != 1) return fail(nullptr, CROCCO_ERR_ARG, "bad weno_weights");
    if (p->weno_limiter & ~3) return fail(nullptr, CROCCO_ERR_ARG, "bad weno_limiter mask");
    if (!(p->weno_alpha_rl >= 0) || !(p->weno_alpha_al >= 0))
        return fail(nullptr, CROCCO_ERR_ARG, "WENO limiter thresholds must be >= 0");
    if (p->visc_form != 0 && p->visc_form != 1) return fail(nullptr, CROCCO_ERR_ARG, "bad visc_form");
    return CROCCO_OK;
}

// cached RK3 step graphs bake in the kernel arguments (Phys), the kernel variants (limiter,
// viscous form) and the scratch pointers of the capture: any change of those drops them
static void drop_graphs(crocco_ctx c) {
    for (auto &g : c->graphs) cudaGraphExecDestroy(g.exec);
    c->graphs.clear();
}

crocco_status crocco_set_phys(crocco_ctx c, const crocco_phys *p) {
    LIVE(c);
    crocco_status st = check_phys(p);
    if (st) return fail(c, st, "%s", g_err.c_str());
    c->phys_in = *p;
    c->ph = to_phys(p);
    drop_graphs(c);
    return CROCCO_OK;
}

static void free_ctx(crocco_ctx c) {
    for (auto &b : c->loc) {
        cudaFree(b.racc);
        cudaFree(b.fv);
        cudaFree(b.met2);
    }
    cudaFree(c->send_stage);
    cudaFree(c->dmax);
    cudaFree(c->recv_stage);
    for (double *m : c->amr_mirror) cudaFree(m);
    for (double *m : c->amr_smirror) cudaFree(m);
    cudaFree(c->amr_send);
    cudaFree(c->amr_recv);
    for (auto &t : c->pending) {
        cudaEventDestroy(t.e0);
        cudaEventDestroy(t.e1);
    }
    for (auto e : c->pool) cudaEventDestroy(e);
    drop_graphs(c);
    if (c->cap_stream) cudaStreamDestroy(c->cap_stream);
    if (c->comm_stream) cudaStreamDestroy(c->comm_stream);
    if (c->ev_fork) cudaEventDestroy(c->ev_fork);
    if (c->ev_join) cudaEventDestroy(c->ev_join);
    if (c->comm) ncclCommDestroy(c->comm);
    delete c;
}

crocco_status crocco_init_grid(const crocco_grid_desc *desc, const crocco_phys *phys,
                               crocco_ctx *out) {
    if (!out) return fail(nullptr, CROCCO_ERR_ARG, "null out");
    *out = nullptr;
    int nb[3], bn[3];
    crocco_status st = validate(desc, nb, bn);
    if (st) return st;
    st = check_phys(phys);
    if (st) return st;
    crocco_ctx c = new crocco_ctx_s();
    c->desc = *desc;
    const int nbt = nb[0] * nb[1] * nb[2];
    if (desc->block_rank) c->block_rank.assign(desc->block_rank, desc->block_rank + nbt);
    else c->block_rank.assign(nbt, 0);
    c->desc.block_rank = c->block_rank.data();
    c->phys_in = *phys;
    c->ph = to_phys(phys);
    for (int d = 0; d < 3; d++)
        for (int sd = 0; sd < 2; sd++) c->has_cf = c->has_cf || desc->bc[d][sd] == CROCCO_BC_COARSE_FINE;
    c->stream = (cudaStream_t)desc->stream;
    for (int a = 0; a < 3; a++) {
        c->nb[a] = nb[a];
        c->bn[a] = bn[a];
    }
    build_blocks(&c->desc, nb, bn, c->all);
    c->gid_to_local.assign(nbt, -1);
    for (const BlockGeom &g : c->all) {
        if (g.rank != desc->rank) continue;
        LocalBlock lb;
        lb.g = g;
        lb.L = make_layout(g.n, G);
        lb.C = make_layout(g.n, GC);
        lb.V.b0 = g.n[0] + 4;
        lb.V.b1 = g.n[1] + 4;
        lb.V.b2 = g.n[2] + 4;
        lb.V.py = rup(lb.V.b0 + 8, 16);
        lb.V.pz = lb.V.py * lb.V.b1;
        lb.V.cs = rup(lb.V.pz * lb.V.b2, 32);
        c->gid_to_local[g.gid] = (int)c->loc.size();
        c->loc.push_back(lb);
    }
    for (int d = 0; d < 3; d++) build_plan(&c->desc, nb, bn, c->all, d, desc->rank, c->plan[d]);

    // device scratch
    auto alloc = [&](double **p, int64_t elems) -> bool {
        if (cudaMalloc((void **)p, (size_t)elems * sizeof(double)) != cudaSuccess) return false;
        // defined padding: whole-tile copies of the sweeps read (and discard) row padding
        if (cudaMemset(*p, 0, (size_t)elems * sizeof(double)) != cudaSuccess) return false;
        c->scratch += elems * (int64_t)sizeof(double);
        return true;
    };
    for (auto &b : c->loc) {
        // R accumulator; of the viscous point fluxes only F^_v^eta goes to HBM (k_visc_tiled
        // differences the xi and zeta ones on chip)
        b.rcs = rup((int64_t)b.g.n[0] * b.g.n[1] * b.g.n[2], 32);
        bool ok = alloc(&b.racc, 5 * b.rcs);
        ok = ok && alloc(&b.fv, 4 * b.V.cs);
        if (!ok) {
            cudaGetLastError();
            free_ctx(c);
            return fail(nullptr, CROCCO_ERR_NOMEM, "device scratch allocation failed");
        }
    }
    {
        cudaError_t e = sweep_attrs();
        if (e != cudaSuccess) {
            free_ctx(c);
            return fail(nullptr, CROCCO_ERR_CUDA, "cudaFuncSetAttribute: %s", cudaGetErrorString(e));
        }
    }
    // NCCL communicator + staging for remote halo messages
    if (desc->nranks > 1) {
        int64_t maxe = 0;
        for (int d = 0; d < 3; d++) {
            int64_t s = 0, r = 0;
            for (auto &m : c->plan[d])
                if (m.kind == 0 && m.src_rank != m.dst_rank) {
                    const int64_t v = m.ext[0] * m.ext[1] * m.ext[2] * 10;
                    if (m.src_rank == desc->rank) s += v;
                    if (m.dst_rank == desc->rank) r += v;
                }
            maxe = std::max(maxe, std::max(s, r));
        }
        c->stage_elems = maxe;
        if (maxe > 0) {
            if (!alloc(&c->send_stage, maxe) || !alloc(&c->recv_stage, maxe)) {
                cudaGetLastError();
                free_ctx(c);
                return fail(nullptr, CROCCO_ERR_NOMEM, "halo staging allocation failed");
            }
        }
        if (!desc->nccl_unique_id) {
            free_ctx(c);
            return fail(nullptr, CROCCO_ERR_ARG, "nccl_unique_id required when nranks > 1");
        }
        ncclUniqueId id;
        memcpy(&id, desc->nccl_unique_id, sizeof id);
        ncclResult_t r = ncclCommInitRank(&c->comm, desc->nranks, id, desc->rank);
        if (r != ncclSuccess) {
            c->comm = nullptr;
            free_ctx(c);
            return fail(nullptr, CROCCO_ERR_NCCL, "ncclCommInitRank: %s", ncclGetErrorString(r));
        }
    }
    *out = c;
    return CROCCO_OK;
}

crocco_status crocco_num_local_blocks(crocco_ctx c, int32_t *n) {
    LIVE(c);
    if (!n) return fail(c, CROCCO_ERR_ARG, "null out");
    *n = (int32_t)c->loc.size();
    return CROCCO_OK;
}

crocco_status crocco_scratch_bytes(crocco_ctx c, int64_t *bytes) {
    LIVE(c);
    if (!bytes) return fail(c, CROCCO_ERR_ARG, "null out");
    *bytes = c->scratch;
    return CROCCO_OK;
}

crocco_status crocco_get_block_layout(crocco_ctx c, int32_t lb, crocco_block_layout *o) {
    LIVE(c);
    if (!o || lb < 0 || lb >= (int)c->loc.size()) return fail(c, CROCCO_ERR_ARG, "bad local block");
    const LocalBlock &b = c->loc[lb];
    memset(o, 0, sizeof *o);
    for (int a = 0; a < 3; a++) {
        o->n[a] = b.g.n[a];
        o->origin[a] = b.g.origin[a];
    }
    o->ghost = G;
    o->ghost_coords = GC;
    o->offset = b.L.off;
    o->pitch_y = b.L.py;
    o->pitch_z = b.L.pz;
    o->comp_stride = b.L.cs;
    o->coffset = b.C.off;
    o->cpitch_y = b.C.py;
    o->cpitch_z = b.C.pz;
    o->ccomp_stride = b.C.cs;
    o->global_id = b.g.gid;
    return CROCCO_OK;
}

// ---------------------------------------------------------------------------
// ghost fill
// ---------------------------------------------------------------------------
static crocco_status flush_ops(crocco_ctx c, BoxOps &ops) {
    if (ops.nops == 0) return CROCCO_OK;
    int64_t mx = 0;
    for (int i = 0; i < ops.nops; i++)
        mx = std::max(mx, (int64_t)ops.op[i].ext[0] * ops.op[i].ext[1] * ops.op[i].ext[2]);
    dim3 grid(std::min<int64_t>(cdiv(mx, 256), 4096), ops.nops);
    LAUNCH(c, K_FILL, k_boxops<<<grid, 256, 0, c->stream>>>(ops));
    ops.nops = 0;
    return CROCCO_OK;
}
static crocco_status push_op(crocco_ctx c, BoxOps &ops, const BoxOp &o) {
    ops.op[ops.nops++] = o;
    if (ops.nops == MAX_OPS) return flush_ops(c, ops);
    return CROCCO_OK;
}

static void op_strides(const Lay &L, int64_t st[3]) {
    st[0] = 1;
    st[1] = L.py;
    st[2] = L.pz;
}

static crocco_status flush_cf(crocco_ctx c, CFOps &cf, const LevelTab &ct, const SibTab &sb) {
    if (cf.nops == 0) return CROCCO_OK;
    int64_t mx = 0;
    for (int i = 0; i < cf.nops; i++)
        mx = std::max(mx, (int64_t)cf.op[i].ext[0] * cf.op[i].ext[1] * cf.op[i].ext[2]);
    dim3 grid(std::min<int64_t>(cdiv(mx, 256), 4096), cf.nops);
    LAUNCH(c, K_AMR, k_cf_interp<<<grid, 256, 0, c->stream>>>(cf, ct, sb));
    cf.nops = 0;
    return CROCCO_OK;
}

// table of one level's local blocks for the AMR kernels
static void level_tab(const crocco_ctx_s *lv, double *const *ptr, LevelTab &t) {
    memset(&t, 0, sizeof t);
    for (size_t b = 0; b < lv->loc.size(); b++) t.p[b] = ptr[b];
    for (int g = 0; g < AMR_MAX_BLOCKS; g++)
        t.g2l[g] = g < (int)lv->gid_to_local.size() ? (int16_t)lv->gid_to_local[g] : (int16_t)-1;
    t.L = make_layout(lv->bn, G);  // equal blocks (also when this rank owns none of the level)
    for (int d = 0; d < 3; d++) {
        t.bn[d] = lv->bn[d];
        t.nb[d] = lv->nb[d];
        t.N[d] = lv->desc.n_global[d];
    }
}

static crocco_status amr_fill_exchange(crocco_ctx f);  // two-level AMR section below
static crocco_status amr_sib_exchange(crocco_ctx f);
static double *amr_mirror(crocco_ctx f, int gid);
static double *amr_sib_mirror_if(crocco_ctx f, int s, int gid);
// the blocks of f's same-level siblings in f's fine index space, with the states of this call
// (every block of every sibling, on any rank: the geometry decides which ghost points copy and
// which coarse nodes are covered; the data of a block on another rank -- or of every block under
// the loopback -- is read from its mirror, filled by the kind-2 boxes of amr_sib_exchange)
static void sib_tab(crocco_ctx f, SibTab &t) {
    memset(&t, 0, sizeof t);
    if (!f->amr_sibU) return;
    for (size_t s = 0; s < f->sibs.size(); s++) {
        const crocco_ctx_s *g = f->sibs[s];
        for (size_t b = 0; b < g->all.size() && t.n < SIB_MAX_BLOCKS; b++) {
            const BlockGeom &bg = g->all[b];
            for (int d = 0; d < 3; d++) {
                t.lo[t.n][d] = 2 * (g->amr_c0[d] - f->amr_c0[d]) + bg.origin[d];
                t.hi[t.n][d] = t.lo[t.n][d] + bg.n[d];
            }
            const int l = g->gid_to_local[bg.gid];
            t.p[t.n] = (l >= 0 && !f->loopback) ? f->amr_sibU[s][l] : amr_sib_mirror_if(f, (int)s, bg.gid);
            t.L[t.n] = make_layout(bg.n, G);
            t.n++;
        }
    }
}

static crocco_status fill_phase(crocco_ctx c, double *const *f, int kind, int D,
                                double *const *met, double t) {
    const bool copies_only = kind == FILL_STATE_COPIES;
    if (copies_only) kind = CROCCO_FIELD_STATE;
    const int ncomp = kind == CROCCO_FIELD_STATE ? 5 : 10;
    BoxOps ops;
    ops.nops = 0;
    CFOps cf;
    cf.nops = 0;
    LevelTab ct;
    memset(&ct, 0, sizeof ct);
    const bool interp = kind == CROCCO_FIELD_STATE && !copies_only && c->amr_Uc && c->amr_coarse;
    // C/F faces: interpolation (+ sibling copies), or -- copies-only fills of AverageDown with
    // siblings -- the sibling copies alone
    const bool cfface = interp || (copies_only && c->amr_sibU && !c->sibs.empty());
    SibTab sb;
    sib_tab(c, sb);
    cf.interp = interp ? 1 : 0;
    if (cfface) {
        cf.Lf = c->loc.empty() ? Lay{} : c->loc[0].L;
        for (int e = 0; e < 3; e++) cf.c0[e] = c->amr_c0[e];
    }
    if (interp) {
        level_tab(c->amr_coarse, c->amr_Uc, ct);
        // coarse blocks whose boxes came through NCCL (other rank / loopback): read the mirrors
        int slot = (int)c->amr_coarse->loc.size();
        for (int gid : c->amr_cf_gids) {
            ct.p[slot] = amr_mirror(c, gid);
            ct.g2l[gid] = (int16_t)slot++;
        }
        cf.Lf = c->loc.empty() ? Lay{} : c->loc[0].L;
        for (int e = 0; e < 3; e++) cf.c0[e] = c->amr_c0[e];
    }
    std::vector<const crocco_msg *> remote;
    for (const crocco_msg &m : c->plan[D]) {
        if (m.kind == 0 && (m.src_rank != m.dst_rank || c->loopback)) {
            remote.push_back(&m);
            continue;
        }
        if (m.dst_rank != c->desc.rank) continue;
        const int dl = c->gid_to_local[m.dst_block];
        const LocalBlock &db = c->loc[dl];
        BoxOp o;
        memset(&o, 0, sizeof o);
        o.dst = f[dl];
        op_strides(db.L, o.dst_);
        o.dcs = db.L.cs;
        o.dbase = at(db.L, (int)m.dst_lo[0], (int)m.dst_lo[1], (int)m.dst_lo[2]);
        for (int e = 0; e < 3; e++) o.ext[e] = (int)m.ext[e];
        o.ncomp = ncomp;
        if (m.kind == 0) {  // periodic / inter-block copy, same rank
            const int sl = c->gid_to_local[m.src_block];
            const LocalBlock &sb = c->loc[sl];
            o.src = f[sl];
            op_strides(sb.L, o.sst);
            o.scs = sb.L.cs;
            o.sbase = at(sb.L, (int)m.src_lo[0], (int)m.src_lo[1], (int)m.src_lo[2]);
            o.mode = BOX_COPY;
        } else {
            const int bc = m.bc_kind;
            if (kind == CROCCO_FIELD_METRIC || (copies_only && !(bc == CROCCO_BC_COARSE_FINE && cfface)))
                continue;  // physical faces keep computed metrics; copies-only fills skip BCs
            if (bc == CROCCO_BC_COARSE_FINE) {  // FillPatchTwoLevels (reading 25); untouched without a coarse level
                if (!cfface) continue;
                CFOp q;
                q.dst = f[dl];
                q.dbase = o.dbase;
                for (int e = 0; e < 3; e++) {
                    q.ext[e] = o.ext[e];
                    q.fo[e] = db.g.origin[e] + m.dst_lo[e];
                }
                cf.op[cf.nops++] = q;
                if (cf.nops == CF_MAX_OPS) {
                    crocco_status s2 = flush_cf(c, cf, ct, sb);
                    if (s2) return s2;
                }
                continue;
            }
            const int n = db.g.n[D];
            int64_t st[3];
            op_strides(db.L, st);
            o.src = f[dl];
            o.scs = db.L.cs;
            for (int e = 0; e < 3; e++) o.sst[e] = st[e];
            int lo[3] = {(int)m.dst_lo[0], (int)m.dst_lo[1], (int)m.dst_lo[2]};
            if (bc == CROCCO_BC_EXTRAP) {
                lo[D] = m.side == 0 ? 0 : n - 1;
                o.sst[D] = 0;
                o.mode = BOX_COPY;
            } else if (bc == CROCCO_BC_DIRICHLET) {
                o.mode = BOX_CONST;
                for (int q = 0; q < 5; q++) o.val[q] = c->desc.dirichlet[D][m.side][q];
            } else {
                // WALL / SLIPWALL / SPLIT: dst index (lo + t) <- src index mirrored about the face
                lo[D] = m.side == 0 ? G - 1 : n - 1;
                o.sst[D] = -st[D];
                o.mode = bc == CROCCO_BC_WALL ? BOX_WALL : (bc == CROCCO_BC_SLIPWALL ? BOX_SLIP : BOX_SPLIT);
                if (bc != CROCCO_BC_WALL) {
                    if (!met || !met[dl])
                        return fail(c, CROCCO_ERR_ARG, "SLIPWALL/SPLIT faces need the metrics in the fill");
                    o.met = met[dl] + (int64_t)(1 + 3 * D) * db.L.cs;
                    o.mcs = db.L.cs;
                }
                if (bc == CROCCO_BC_SPLIT) {
                    const crocco_split &sp = c->desc.split[D][m.side];
                    o.axis = sp.axis;
                    o.g0 = db.g.origin[sp.axis] + m.dst_lo[sp.axis];
                    o.s = sp.i0 + sp.di_dt * t;
                    for (int q = 0; q < 5; q++) o.val[q] = sp.left[q];
                    o.right_mode = sp.right_kind == CROCCO_BC_SLIPWALL ? BOX_SLIP : BOX_CONST;
                    for (int q = 0; q < 5; q++) o.rval[q] = sp.right[q];
                }
            }
            o.sbase = at(db.L, lo[0], lo[1], lo[2]);
        }
        crocco_status st = push_op(c, ops, o);
        if (st) return st;
    }
    crocco_status st = flush_ops(c, ops);
    if (st) return st;
    if (cfface && (st = flush_cf(c, cf, ct, sb))) return st;
    if (remote.empty()) return CROCCO_OK;
    if (!c->comm) return fail(c, CROCCO_ERR_STATE, "remote halo without communicator");
    // pack sends (a loopback message is both sent and received by this rank)
    int64_t soff = 0, roff = 0;
    std::vector<int64_t> offs(remote.size()), roffs(remote.size());
    for (size_t r = 0; r < remote.size(); r++) {
        const crocco_msg &m = *remote[r];
        const int64_t vol = m.ext[0] * m.ext[1] * m.ext[2];
        if (m.dst_rank == c->desc.rank) {
            roffs[r] = roff;
            roff += vol * ncomp;
        }
        if (m.src_rank == c->desc.rank) {
            const int sl = c->gid_to_local[m.src_block];
            const LocalBlock &sb = c->loc[sl];
            BoxOp o;
            memset(&o, 0, sizeof o);
            o.src = f[sl];
            op_strides(sb.L, o.sst);
            o.scs = sb.L.cs;
            o.sbase = at(sb.L, (int)m.src_lo[0], (int)m.src_lo[1], (int)m.src_lo[2]);
            o.dst = c->send_stage + soff;
            o.dst_[0] = 1;
            o.dst_[1] = m.ext[0];
            o.dst_[2] = m.ext[0] * m.ext[1];
            o.dcs = vol;
            o.dbase = 0;
            for (int e = 0; e < 3; e++) o.ext[e] = (int)m.ext[e];
            o.ncomp = ncomp;
            offs[r] = soff;
            soff += vol * ncomp;
            st = push_op(c, ops, o);
            if (st) return st;
        }
    }
    st = flush_ops(c, ops);
    if (st) return st;
    NvtxRange nv("crocco:nccl_halo");
    NK(c, ncclGroupStart());
    for (size_t r = 0; r < remote.size(); r++) {
        const crocco_msg &m = *remote[r];
        const size_t cnt = (size_t)(m.ext[0] * m.ext[1] * m.ext[2] * ncomp);
        if (m.src_rank == c->desc.rank)
            NK(c, ncclSend(c->send_stage + offs[r], cnt, ncclDouble, m.dst_rank, c->comm, c->stream));
        if (m.dst_rank == c->desc.rank)
            NK(c, ncclRecv(c->recv_stage + roffs[r], cnt, ncclDouble, m.src_rank, c->comm, c->stream));
    }
    NK(c, ncclGroupEnd());
    // unpack receives
    for (size_t r = 0; r < remote.size(); r++) {
        const crocco_msg &m = *remote[r];
        if (m.dst_rank != c->desc.rank) continue;
        const int dl = c->gid_to_local[m.dst_block];
        const LocalBlock &db = c->loc[dl];
        const int64_t vol = m.ext[0] * m.ext[1] * m.ext[2];
        BoxOp o;
        memset(&o, 0, sizeof o);
        o.src = c->recv_stage + roffs[r];
        o.sst[0] = 1;
        o.sst[1] = m.ext[0];
        o.sst[2] = m.ext[0] * m.ext[1];
        o.scs = vol;
        o.sbase = 0;
        o.dst = f[dl];
        op_strides(db.L, o.dst_);
        o.dcs = db.L.cs;
        o.dbase = at(db.L, (int)m.dst_lo[0], (int)m.dst_lo[1], (int)m.dst_lo[2]);
        for (int e = 0; e < 3; e++) o.ext[e] = (int)m.ext[e];
        o.ncomp = ncomp;
        st = push_op(c, ops, o);
        if (st) return st;
    }
    return flush_ops(c, ops);
}

static crocco_status check_ptrs(crocco_ctx c, double *const *p, const char *what) {
    if (!p) return fail(c, CROCCO_ERR_ARG, "null %s pointer array", what);
    for (size_t b = 0; b < c->loc.size(); b++)
        if (!p[b]) return fail(c, CROCCO_ERR_ARG, "null %s pointer for local block %zu", what, b);
    return CROCCO_OK;
}

// single-pass gather fill (fill.cuh k_fill_gather): state fills whose faces are all PERIODIC,
// EXTRAP, WALL or DIRICHLET with every block on this rank (bitwise equal to the 3 phases)
static bool gather_fill_ok(const crocco_ctx_s *c, int32_t kind) {
    if (kind != CROCCO_FIELD_STATE || c->loopback) return false;
    if (c->loc.size() != c->all.size() || c->loc.size() > AMR_MAX_LOCAL || c->all.size() > AMR_MAX_BLOCKS)
        return false;
    for (int d = 0; d < 3; d++)
        for (int sd = 0; sd < 2; sd++) {
            const int k = c->desc.bc[d][sd];
            if (k != CROCCO_BC_PERIODIC && k != CROCCO_BC_EXTRAP && k != CROCCO_BC_WALL && k != CROCCO_BC_DIRICHLET)
                return false;
        }
    return true;
}

static crocco_status fill_gather(crocco_ctx c, double *const *f) {
    GatherArgs ga;
    memset(&ga, 0, sizeof ga);
    level_tab(c, f, ga.t);
    for (size_t b = 0; b < c->loc.size(); b++)
        for (int d = 0; d < 3; d++) ga.org[b][d] = c->loc[b].g.origin[d];
    for (int d = 0; d < 3; d++)
        for (int sd = 0; sd < 2; sd++) {
            ga.bc[d][sd] = c->desc.bc[d][sd];
            for (int q = 0; q < 5; q++) ga.dir[d][sd][q] = c->desc.dirichlet[d][sd][q];
        }
    const int64_t n0 = c->bn[0], n1 = c->bn[1], n2 = c->bn[2];
    const int64_t shell = (int64_t)2 * G * (n0 + 2 * G) * (n1 + 2 * G) + (int64_t)2 * G * n2 * (n0 + 2 * G) +
                          (int64_t)2 * G * n2 * n1;
    dim3 grid(std::min<int64_t>(cdiv(shell, 256), 4096), (unsigned)c->loc.size());
    LAUNCH(c, K_FILL, k_fill_gather<<<grid, 256, 0, c->stream>>>(ga));
    return CROCCO_OK;
}

static crocco_status fill_all(crocco_ctx c, double *const *f, int32_t kind, double *const *met, double t) {
    NvtxRange nv(c->amr_Uc ? "crocco:fill_two_levels" : "crocco:fill");
    if (kind != CROCCO_FIELD_STATE && kind != CROCCO_FIELD_METRIC && kind != FILL_STATE_COPIES)
        return fail(c, CROCCO_ERR_ARG, "bad field kind");
    crocco_status st = check_ptrs(c, f, "field");
    if (st) return st;
    // FillPatchTwoLevels: the inter-level boxes first (collective over the fine level)
    if (kind == CROCCO_FIELD_STATE && c->amr_Uc && c->amr_coarse && (st = amr_fill_exchange(c))) return st;
    if (((kind == CROCCO_FIELD_STATE && c->amr_Uc) || kind == FILL_STATE_COPIES) && c->amr_sibU && !c->sibs.empty() &&
        (st = amr_sib_exchange(c)))
        return st;
    if (gather_fill_ok(c, kind)) return fill_gather(c, f);
    for (int d = 0; d < 3; d++) {
        st = fill_phase(c, f, kind, d, met, t);
        if (st) return st;
    }
    return CROCCO_OK;
}

crocco_status crocco_fill_boundary(crocco_ctx c, double *const *f, int32_t kind, double *const *met) {
    LIVE(c);
    if (kind != CROCCO_FIELD_STATE && kind != CROCCO_FIELD_METRIC) return fail(c, CROCCO_ERR_ARG, "bad field kind");
    return fill_all(c, f, kind, met, c->time);
}

crocco_status crocco_set_time(crocco_ctx c, double t) {
    LIVE(c);
    c->time = t;
    return CROCCO_OK;
}

crocco_status crocco_get_time(crocco_ctx c, double *t) {
    LIVE(c);
    if (!t) return fail(c, CROCCO_ERR_ARG, "null out");
    *t = c->time;
    return CROCCO_OK;
}

// ---------------------------------------------------------------------------
// metrics
// ---------------------------------------------------------------------------
crocco_status crocco_init_metrics(crocco_ctx c, double *const *xyz, double *const *met) {
    LIVE(c);
    crocco_status st = check_ptrs(c, xyz, "xyz");
    if (st) return st;
    st = check_ptrs(c, met, "metrics");
    if (st) return st;
    for (size_t b = 0; b < c->loc.size(); b++) {
        const LocalBlock &lb = c->loc[b];
        double *dx = nullptr;
        CK(c, cudaMallocAsync((void **)&dx, (size_t)(9 * lb.C.cs) * sizeof(double), c->stream));
        const int W = G + 3;
        const int64_t nd = (int64_t)(lb.g.n[0] + 2 * W) * (lb.g.n[1] + 2 * W) * (lb.g.n[2] + 2 * W);
        LAUNCH(c, K_METRICS, k_coord_deriv<<<cdiv(nd, 256), 256, 0, c->stream>>>(xyz[b], dx, lb.C));
        const int64_t nm = (int64_t)(lb.g.n[0] + 2 * G) * (lb.g.n[1] + 2 * G) * (lb.g.n[2] + 2 * G);
        LAUNCH(c, K_METRICS, k_metric<<<cdiv(nm, 128), 128, 0, c->stream>>>(xyz[b], dx, met[b], lb.C, lb.L));
        CK(c, cudaFreeAsync(dx, c->stream));
    }
    return fill_all(c, met, CROCCO_FIELD_METRIC, nullptr, 0.0);
}

crocco_status crocco_init_metrics2(crocco_ctx c, double *const *met) {
    LIVE(c);
    crocco_status st = check_ptrs(c, met, "metrics");
    if (st) return st;
    drop_graphs(c);  // new scratch pointers / kernel variant of the expanded viscous form
    for (auto &b : c->loc) {
        if (!b.met2) {
            if (cudaMalloc((void **)&b.met2, (size_t)(18 * b.rcs) * sizeof(double)) != cudaSuccess) {
                cudaGetLastError();
                return fail(c, CROCCO_ERR_NOMEM, "second-metric allocation failed");
            }
            c->scratch += 18 * b.rcs * (int64_t)sizeof(double);
        }
    }
    for (size_t bi = 0; bi < c->loc.size(); bi++) {
        const LocalBlock &b = c->loc[bi];
        const int64_t ni = (int64_t)b.g.n[0] * b.g.n[1] * b.g.n[2];
        LAUNCH(c, K_METRICS, k_metric2<<<cdiv(ni, 128), 128, 0, c->stream>>>(met[bi], b.met2, b.L, b.rcs));
    }
    return CROCCO_OK;
}

crocco_status crocco_copy_metrics2(crocco_ctx c, int32_t lb, double *dst) {
    LIVE(c);
    if (lb < 0 || lb >= (int)c->loc.size() || !dst) return fail(c, CROCCO_ERR_ARG, "bad local block / dst");
    const LocalBlock &b = c->loc[lb];
    if (!b.met2) return fail(c, CROCCO_ERR_STATE, "second metrics not initialised");
    const int64_t ni = (int64_t)b.g.n[0] * b.g.n[1] * b.g.n[2];
    for (int q = 0; q < 18; q++)
        CK(c, cudaMemcpyAsync(dst + q * ni, b.met2 + q * b.rcs, (size_t)ni * sizeof(double),
                              cudaMemcpyDeviceToDevice, c->stream));
    return CROCCO_OK;
}

// ---------------------------------------------------------------------------
// RHS / RK
// ---------------------------------------------------------------------------
static const double RK_A[3] = {0.0, -5.0 / 9.0, -153.0 / 128.0};
static const double RK_C[3] = {0.0, 1.0 / 3.0, 3.0 / 4.0};  // stage times (reading 13)
static const double RK_B[3] = {1.0 / 3.0, 15.0 / 16.0, 8.0 / 15.0};

// One RHS evaluation of a block (Alg. 2 l.5-9): primitives, viscous point
// fluxes, then the xi / eta / zeta sweeps; the zeta sweep finishes every point
// (mode 2: rhs = J R, mode 3: Williamson update).
// ghost-free interior tiles of the viscous kernel (k_visc_tiled sel 1) of one block;
// returns false if the block has none or the configuration has no such split
static bool visc_overlap_possible(crocco_ctx c) {
    const bool viscous = (c->ph.terms & CROCCO_TERM_VISCOUS) != 0 && c->ph.visc_form == 0;
    if (!viscous) return false;
    for (const auto &b : c->loc) {
        const VTiles t = visc_interior_tiles(b.L, visc_slab(b.L, b.V, true));
        if (t.x1 > t.x0 && t.y1 > t.y0 && t.z1 > t.z0) return true;
    }
    return false;
}
static crocco_status visc_interior(crocco_ctx c, const LocalBlock &b, const double *U, const double *M) {
    const int vk = visc_slab(b.L, b.V, true);
    const VTiles t = visc_interior_tiles(b.L, vk);
    const int64_t nt = (int64_t)(t.x1 - t.x0) * (t.y1 - t.y0) * (t.z1 - t.z0);
    if (nt == 0) return CROCCO_OK;
    return launch_visc(c, b, U, M, c->ph, nt, 1, vk);
}



static crocco_status rhs_block(crocco_ctx c, const LocalBlock &b, const double *U, const double *M,
                               int final_mode, double *rhs, const double *Uin, double *Uout,
                               double *dU, int stage, double dt, int visc_sel = 0) {
    const Phys &ph = c->ph;
    const bool inviscid = (ph.terms & CROCCO_TERM_INVISCID) != 0;
    const bool vexp = (ph.terms & CROCCO_TERM_VISCOUS) != 0 && ph.visc_form == 1;  // readings 27-28
    const bool viscous = (ph.terms & CROCCO_TERM_VISCOUS) != 0 && !vexp;
    if (vexp) {  // expanded viscous form: V / J -> R comps 1..4, the xi sweep adds (mode 4)
        if (!b.met2)
            return fail(c, CROCCO_ERR_STATE, "visc_form = 1 needs crocco_init_metrics2");
        const unsigned nt = (unsigned)(((b.g.n[0] + XTX - 1) / XTX) * ((b.g.n[1] + XTY - 1) / XTY) *
                                       ((b.g.n[2] + XVK - 1) / XVK));
        LAUNCH(c, K_VISC, k_visc_exp_tiled<<<nt, XTX * XTY, VISC_EXP_SMEM, c->stream>>>(U, M, b.met2, b.racc,
                                                                                       b.rcs, b.L, ph));
    } else if (viscous && visc_sel != 1) {
        // k_visc_tiled: R comps 1..4 = D4_xi + D4_zeta of the point fluxes, F^_v^eta -> HBM
        // (sel 1, the ghost-free tiles, was launched by visc_interior() beside the fill)
        const int vk = visc_slab(b.L, b.V, visc_sel != 0);
        int64_t nt = (int64_t)visc_tiles_x(b.L) * ((b.V.b1 + VTY - 1) / VTY) * ((b.g.n[2] + vk - 1) / vk);
        if (visc_sel == 2) {
            const VTiles t = visc_interior_tiles(b.L, vk);
            nt -= (int64_t)(t.x1 - t.x0) * (t.y1 - t.y0) * (t.z1 - t.z0);
        }
        if (nt > 0) {
            crocco_status st = launch_visc(c, b, U, M, ph, nt, visc_sel, vk);
            if (st) return st;
        }
    }
    for (int d = 0; d < 3; d++) {
        SweepArgs a;
        memset(&a, 0, sizeof a);
        a.in.U = U;
        a.in.M = M;
        a.in.FV = b.fv;  // F^_v^eta: only the eta sweep has a viscous interface term
        a.in.cs = b.L.cs;
        a.in.vcs = b.V.cs;
        a.V = b.V;
        a.R = b.racc;
        a.rcs = b.rcs;
        a.inv = inviscid && (ph.dir_mask >> d & 1);
        a.visc = viscous && d == 1;
        // R: the viscous kernel wrote comps 1..4 (xi sweep adds, mode 4), else the xi sweep writes
        a.mode = d == 0 ? ((ph.terms & CROCCO_TERM_VISCOUS) ? 4 : 0) : (d == 1 ? 1 : final_mode);
        a.rhs = rhs;
        a.Uin = Uin;
        if (final_mode == 3 && Uin != U) return fail(c, CROCCO_ERR_ARG, "RK stage: U_in must be the swept state");
        a.Uout = Uout;
        a.dU = dU;
        a.stage = stage;
        a.A = RK_A[stage];
        a.B = RK_B[stage];
        a.dt = dt;
        // warp tiles: xi 4 lines x 8 interfaces, eta/zeta 8 i x 4 interfaces; lines are
        // marched whole unless that leaves too few warps for 148 SMs
        const int64_t nd = b.g.n[d];
        const int64_t lines = d == 0 ? ((int64_t)b.g.n[1] * b.g.n[2] + 3) / 4
                                     : (int64_t)((b.g.n[0] + 7) / 8) * (d == 1 ? b.g.n[2] : b.g.n[1]);
        int64_t seg = nd;
        // fewer lines than SMs (e.g. Sod's 4 xi lines): segments down to 8 points (measured 8.6e7 -> 1.1e8
        // point-stages/s on Sod); otherwise >= 32 (shorter segments measured slower on the 64^3 vortex)
        const int64_t segmin = lines < 148 ? 8 : SEG_MIN;
        while (lines * ((nd + seg - 1) / seg) < SEG_WARPS && seg > segmin) seg = (seg + 1) / 2;
        a.seg = (int)seg;
        const int64_t warps = lines * ((nd + seg - 1) / seg);
        const unsigned grid = cdiv(warps * 32, sweep_threads(d));
#define SWEEP_LAUNCH(DD, VV, MM)                                                                          \
    do {                                                                                                  \
        if (!a.inv)                                                                                       \
            k_sweep_s<DD, VV, false, MM, 0><<<grid, sweep_threads(DD), sweep_smem_bytes<DD, VV>(), c->stream>>>(a, b.L, ph); \
        else if (ph.lim)                                                                                  \
            k_sweep_s<DD, VV, true, MM, 2><<<grid, sweep_threads(DD), sweep_smem_bytes<DD, VV>(), c->stream>>>(a, b.L, ph);  \
        else                                                                                              \
            k_sweep_s<DD, VV, false, MM><<<grid, sweep_threads(DD), sweep_smem_bytes<DD, VV>(), c->stream>>>(a, b.L, ph); \
    } while (0)
        if (d == 0) LAUNCH(c, K_FLUX_X, if (a.mode == 4) SWEEP_LAUNCH(0, false, 4); else SWEEP_LAUNCH(0, false, 0));
        else if (d == 1) LAUNCH(c, K_FLUX_Y, if (a.visc) SWEEP_LAUNCH(1, true, 1); else SWEEP_LAUNCH(1, false, 1));
        else LAUNCH(c, K_FLUX_Z, if (a.mode == 3) SWEEP_LAUNCH(2, false, 3); else SWEEP_LAUNCH(2, false, 2));
#undef SWEEP_LAUNCH
    }
    return CROCCO_OK;
}

crocco_status crocco_rhs(crocco_ctx c, double *const *U, double *const *M, double *const *rhs) {
    LIVE(c);
    NvtxRange nv("crocco:rhs");
    crocco_status st;
    if ((st = check_ptrs(c, U, "U")) || (st = check_ptrs(c, M, "metrics")) ||
        (st = check_ptrs(c, rhs, "rhs")))
        return st;
    for (size_t bi = 0; bi < c->loc.size(); bi++)
        if (rhs[bi] == U[bi]) return fail(c, CROCCO_ERR_ARG, "rhs aliases U");
    for (size_t bi = 0; bi < c->loc.size(); bi++) {
        if ((st = rhs_block(c, c->loc[bi], U[bi], M[bi], 2, rhs[bi], nullptr, nullptr, nullptr, 0, 0.0)))
            return st;
    }
    return CROCCO_OK;
}

crocco_status crocco_rk_stage(crocco_ctx c, int32_t stage, double dt, double *const *Uin,
                              double *const *Uout, double *const *dU, double *const *M) {
    LIVE(c);
    NvtxRange nv("crocco:rk_stage");
    crocco_status st;
    if (stage < 0 || stage > 2) return fail(c, CROCCO_ERR_ARG, "stage must be 0..2");
    if ((st = check_ptrs(c, Uin, "U_in")) || (st = check_ptrs(c, Uout, "U_out")) ||
        (st = check_ptrs(c, dU, "dU")) || (st = check_ptrs(c, M, "metrics")))
        return st;
    for (size_t bi = 0; bi < c->loc.size(); bi++)
        if (Uin[bi] == Uout[bi] || dU[bi] == Uin[bi] || dU[bi] == Uout[bi])
            return fail(c, CROCCO_ERR_ARG, "U_in, U_out and dU must be distinct");
    if (c->has_cf && !c->amr_Uc)
        return fail(c, CROCCO_ERR_ARG, "COARSE_FINE faces need the coarse level: use crocco_amr_rk_stage");
    const double ts = c->time + RK_C[stage] * dt;
    const bool ov = c->overlap < 0 ? c->desc.nranks > 1 : c->overlap != 0;
    if (!(ov && visc_overlap_possible(c))) {
        if ((st = fill_all(c, Uin, CROCCO_FIELD_STATE, M, ts))) return st;
        for (size_t bi = 0; bi < c->loc.size(); bi++) {
            if ((st = rhs_block(c, c->loc[bi], Uin[bi], M[bi], 3, nullptr, Uin[bi], Uout[bi], dU[bi], stage,
                                dt)))
                return st;
        }
        return CROCCO_OK;
    }
    // Overlapped stage: the ghost fill -- local copies, BCs and the NCCL
    // exchange -- runs on the comm stream while the viscous tiles that read no ghost point
    // run on the compute stream; the remaining tiles and the sweeps follow the fill.
    // Disjoint memory: the fill writes only ghost points of U_in, the interior tiles read
    // only interior points; the result is bitwise that of the serial stage.
    if (!c->comm_stream) CK(c, cudaStreamCreateWithFlags(&c->comm_stream, cudaStreamNonBlocking));
    if (!c->ev_fork) CK(c, cudaEventCreateWithFlags(&c->ev_fork, cudaEventDisableTiming));
    if (!c->ev_join) CK(c, cudaEventCreateWithFlags(&c->ev_join, cudaEventDisableTiming));
    CK(c, cudaEventRecord(c->ev_fork, c->stream));
    CK(c, cudaStreamWaitEvent(c->comm_stream, c->ev_fork, 0));
    {
        cudaStream_t comp = c->stream;
        c->stream = c->comm_stream;
        st = fill_all(c, Uin, CROCCO_FIELD_STATE, M, ts);
        c->stream = comp;
        if (st) return st;
    }
    CK(c, cudaEventRecord(c->ev_join, c->comm_stream));
    c->overlapped_stages++;
    for (size_t bi = 0; bi < c->loc.size(); bi++)
        if ((st = visc_interior(c, c->loc[bi], Uin[bi], M[bi]))) return st;
    CK(c, cudaStreamWaitEvent(c->stream, c->ev_join, 0));
    for (size_t bi = 0; bi < c->loc.size(); bi++) {
        if ((st = rhs_block(c, c->loc[bi], Uin[bi], M[bi], 3, nullptr, Uin[bi], Uout[bi], dU[bi], stage, dt,
                            2)))
            return st;
    }
    return CROCCO_OK;
}

static crocco_status rk3_eager(crocco_ctx c, double dt, double *const *U, double *const *V,
                               double *const *dU, double *const *M) {
    crocco_status st;
    if ((st = crocco_rk_stage(c, 0, dt, U, V, dU, M))) return st;
    if ((st = crocco_rk_stage(c, 1, dt, V, U, dU, M))) return st;
    return crocco_rk_stage(c, 2, dt, U, V, dU, M);
}

crocco_status crocco_rk3_step(crocco_ctx c, double dt, double *const *U, double *const *V,
                              double *const *dU, double *const *M, int32_t use_graph) {
    LIVE(c);
    crocco_status st;
    if ((st = check_ptrs(c, U, "U")) || (st = check_ptrs(c, V, "V")) || (st = check_ptrs(c, dU, "dU")) ||
        (st = check_ptrs(c, M, "metrics")))
        return st;
    if (c->has_cf)
        return fail(c, CROCCO_ERR_ARG, "COARSE_FINE faces: step the hierarchy with crocco_amr_rk_stage");
    bool moving = false;
    for (int d = 0; d < 3; d++)
        for (int sd = 0; sd < 2; sd++)
            moving = moving || (c->desc.bc[d][sd] == CROCCO_BC_SPLIT && c->desc.split[d][sd].di_dt != 0.0);
    if (!use_graph || c->timing || c->desc.nranks > 1 || c->comm || moving) {
        st = rk3_eager(c, dt, U, V, dU, M);
        if (st == CROCCO_OK) c->time = c->time + dt;
        return st;
    }
    std::vector<const void *> key;
    for (size_t b = 0; b < c->loc.size(); b++) {
        key.push_back(U[b]);
        key.push_back(V[b]);
        key.push_back(dU[b]);
        key.push_back(M[b]);
    }
    crocco_ctx_s::StepGraph *g = nullptr;
    for (auto &x : c->graphs)
        if (x.key == key && x.dt == dt) g = &x;
    if (!g) {
        if (!c->cap_stream) CK(c, cudaStreamCreateWithFlags(&c->cap_stream, cudaStreamNonBlocking));
        // capture on a private stream ordered after the caller's stream, then restore
        cudaEvent_t ev;
        CK(c, cudaEventCreateWithFlags(&ev, cudaEventDisableTiming));
        CK(c, cudaEventRecord(ev, c->stream));
        CK(c, cudaStreamWaitEvent(c->cap_stream, ev, 0));
        cudaStream_t orig = c->stream;
        const int64_t l0 = c->launches, o0 = c->overlapped_stages;
        c->stream = c->cap_stream;
        CK(c, cudaStreamBeginCapture(c->cap_stream, cudaStreamCaptureModeThreadLocal));
        st = rk3_eager(c, dt, U, V, dU, M);
        cudaGraph_t graph;
        cudaError_t e = cudaStreamEndCapture(c->cap_stream, &graph);
        c->stream = orig;
        cudaEventDestroy(ev);
        if (st) return st;
        if (e != cudaSuccess) return fail(c, CROCCO_ERR_CUDA, "graph capture: %s", cudaGetErrorString(e));
        cudaGraphExec_t exec;
        e = cudaGraphInstantiate(&exec, graph, 0);
        cudaGraphDestroy(graph);
        if (e != cudaSuccess) return fail(c, CROCCO_ERR_CUDA, "graph instantiate: %s", cudaGetErrorString(e));
        if (c->graphs.size() >= 4) {
            cudaGraphExecDestroy(c->graphs.front().exec);
            c->graphs.erase(c->graphs.begin());
        }
        c->graphs.push_back({key, dt, exec, c->launches - l0, c->overlapped_stages - o0});
        c->launches = l0;  // captured, not launched
        c->overlapped_stages = o0;
        g = &c->graphs.back();
    }
    CK(c, cudaGraphLaunch(g->exec, c->stream));
    c->launches += g->nodes;
    c->overlapped_stages += g->ov_stages;
    c->time = c->time + dt;
    return CROCCO_OK;
}

crocco_status crocco_rk_update(crocco_ctx c, int32_t stage, double dt, double *const *Uin,
                               double *const *Uout, double *const *dU, double *const *rhs) {
    LIVE(c);
    crocco_status st;
    if (stage < 0 || stage > 2) return fail(c, CROCCO_ERR_ARG, "stage must be 0..2");
    if ((st = check_ptrs(c, Uin, "U_in")) || (st = check_ptrs(c, Uout, "U_out")) ||
        (st = check_ptrs(c, dU, "dU")) || (st = check_ptrs(c, rhs, "rhs")))
        return st;
    for (size_t bi = 0; bi < c->loc.size(); bi++) {
        const LocalBlock &b = c->loc[bi];
        dim3 grd(cdiv(b.g.n[0], 128), b.g.n[1], b.g.n[2]);
        LAUNCH(c, K_UPDATE, k_update<<<grd, 128, 0, c->stream>>>(Uin[bi], Uout[bi], dU[bi], rhs[bi], b.L,
                                                                  stage, RK_A[stage], RK_B[stage], dt));
    }
    return CROCCO_OK;
}

crocco_status crocco_compute_dt(crocco_ctx c, double *const *U, double *const *M, double cfl,
                                double *dt) {
    LIVE(c);
    crocco_status st;
    if ((st = check_ptrs(c, U, "U")) || (st = check_ptrs(c, M, "metrics"))) return st;
    if (!dt || !(cfl > 0)) return fail(c, CROCCO_ERR_ARG, "need cfl > 0 and a dt pointer");
    if (!c->dmax) CK(c, cudaMalloc((void **)&c->dmax, sizeof(unsigned long long)));
    CK(c, cudaMemsetAsync(c->dmax, 0, sizeof(unsigned long long), c->stream));
    for (size_t bi = 0; bi < c->loc.size(); bi++) {
        const LocalBlock &b = c->loc[bi];
        const int64_t tot = (int64_t)b.g.n[0] * b.g.n[1] * b.g.n[2];
        const unsigned grid = (unsigned)std::min<int64_t>(cdiv(tot, 256), 148 * 8);
        LAUNCH(c, K_CFL, k_cfl<<<grid, 256, 0, c->stream>>>(U[bi], M[bi], b.L, c->ph, c->dmax));
    }
    if (c->comm)  // global max over ranks (the bit pattern is the double itself)
        NK(c, ncclAllReduce(c->dmax, c->dmax, 1, ncclFloat64, ncclMax, c->comm, c->stream));
    unsigned long long h = 0;
    CK(c, cudaMemcpyAsync(&h, c->dmax, sizeof h, cudaMemcpyDeviceToHost, c->stream));
    CK(c, cudaStreamSynchronize(c->stream));
    double lam;
    memcpy(&lam, &h, sizeof lam);
    if (!(lam > 0)) return fail(c, CROCCO_ERR_ARG, "non-positive spectral radius (state not set?)");
    if (!(lam < INFINITY))
        return fail(c, CROCCO_ERR_ARG, "non-finite spectral radius: NaN or negative pressure in the state");
    *dt = cfl / lam;
    return CROCCO_OK;
}

// ---------------------------------------------------------------------------
// two-level AMR (readings 24-26)
// ---------------------------------------------------------------------------
static int64_t floor_half_h(int64_t h) { return h >= 0 ? h / 2 : -((-h + 1) / 2); }

// coarse nodes I in [lo, hi] along d of the covered set (reading 26); empty when lo > hi
static void covered_range_of(const crocco_grid_desc *fd, const int64_t c0[3], int d, int64_t &lo, int64_t &hi) {
    const int64_t nf = fd->n_global[d];
    if (fd->bc[d][0] == CROCCO_BC_PERIODIC) {
        lo = 0;
        hi = nf / 2 - 1;
    } else {
        lo = c0[d] + 1;
        hi = c0[d] + (nf - 2) / 2;
    }
}

// geometry of a two-level pair (crocco_amr_link's checks; reading 24)
static crocco_status amr_geom_check(crocco_ctx ec, const crocco_grid_desc *fd, const crocco_grid_desc *cd,
                                    const int fnb[3], const int cnb[3], const int64_t c0[3]) {
    if (fd->nranks != cd->nranks || fd->rank != cd->rank)
        return fail(ec, CROCCO_ERR_ARG, "fine and coarse levels must share the process group");
    if ((int64_t)fnb[0] * fnb[1] * fnb[2] > AMR_MAX_BLOCKS || (int64_t)cnb[0] * cnb[1] * cnb[2] > AMR_MAX_BLOCKS)
        return fail(ec, CROCCO_ERR_ARG, "two-level AMR: at most %d blocks per level", AMR_MAX_BLOCKS);
    for (int d = 0; d < 3; d++) {
        const int64_t nf = fd->n_global[d], nc = cd->n_global[d];
        const int *bf = fd->bc[d], *bcc = cd->bc[d];
        if (bf[0] == CROCCO_BC_PERIODIC) {
            if (bcc[0] != CROCCO_BC_PERIODIC || nf != 2 * nc || c0[d] != 0)
                return fail(ec, CROCCO_ERR_ARG,
                            "direction %d: a PERIODIC fine level must span the periodic coarse domain "
                            "(N_f = 2 N_c, c0 = 0)", d);
            continue;
        }
        if (c0[d] < 0 || 2 * c0[d] + nf - 1 > 2 * (nc - 1))
            return fail(ec, CROCCO_ERR_ARG, "direction %d: fine level outside the coarse domain", d);
        if (bf[0] != CROCCO_BC_COARSE_FINE && c0[d] != 0)
            return fail(ec, CROCCO_ERR_ARG, "direction %d: a physical lo face must lie on the domain boundary", d);
        if (bf[1] != CROCCO_BC_COARSE_FINE && 2 * c0[d] + nf - 1 != 2 * (nc - 1))
            return fail(ec, CROCCO_ERR_ARG, "direction %d: a physical hi face must lie on the domain boundary", d);
        if (nf < 3) return fail(ec, CROCCO_ERR_ARG, "direction %d: fine level needs >= 3 points", d);
    }
    return CROCCO_OK;
}

static bool cf_ghost_box(const crocco_grid_desc *fd, const int fnb[3], const int fbn[3], const BlockGeom &fb, int D,
                         int side, int64_t lo[3], int64_t ext[3]);
// The inter-level plan (crocco_amr_plan, include/crocco.h): every box of the pair touching rank
// `me` (me < 0: all), kind 0 then kind 1, canonical order.
static void build_amr_plan(const crocco_grid_desc *fd, const int fnb[3], const int fbn[3],
                           const std::vector<BlockGeom> &fall, const crocco_grid_desc *cd, const int cnb[3],
                           const int cbn[3], const std::vector<BlockGeom> &call, const int64_t c0[3], int me,
                           bool sib_mode, std::vector<crocco_amr_msg> &out) {
    out.clear();
    auto keep = [&](const crocco_amr_msg &m) {
        if (me < 0 || m.src_rank == me || m.dst_rank == me) out.push_back(m);
    };
    // kind 0: per C/F ghost box of a fine block, the coarse corners of its trilinear stencils
    for (const BlockGeom &fb : fall)
        for (int D = 0; D < 3; D++)
            for (int side = 0; side < 2; side++) {
                int64_t lo[3], ext[3];  // the ghost box of phase D (build_plan)
                if (!cf_ghost_box(fd, fnb, fbn, fb, D, side, lo, ext)) continue;
                int64_t Ilo[3], Ihi[3];
                for (int e = 0; e < 3; e++) {
                    Ilo[e] = floor_half_h(2 * c0[e] + fb.origin[e] + lo[e]);
                    Ihi[e] = floor_half_h(2 * c0[e] + fb.origin[e] + lo[e] + ext[e] - 1);
                }
                for (const BlockGeom &cb : call) {
                    crocco_amr_msg m;
                    memset(&m, 0, sizeof m);
                    bool empty = false;
                    for (int e = 0; e < 3; e++) {
                        // nodes I whose clamped owner block is cb (k_cf_interp), corners I and I+1
                        const int64_t o = cb.origin[e];
                        const int64_t own_lo = cb.bidx[e] == 0 ? INT64_MIN / 4 : o;
                        const int64_t own_hi = cb.bidx[e] == cnb[e] - 1 ? INT64_MAX / 4 : o + cbn[e] - 1;
                        const int64_t a = std::max(Ilo[e], own_lo), b2 = std::min(Ihi[e], own_hi);
                        if (a > b2) {
                            empty = true;
                            break;
                        }
                        m.lo[e] = a - o;
                        m.ext[e] = b2 + 1 - a + 1;
                    }
                    if (empty) continue;
                    m.kind = 0;
                    m.coarse_block = cb.gid;
                    m.fine_block = fb.gid;
                    m.sibling = -1;
                    m.src_rank = cb.rank;
                    m.dst_rank = fb.rank;
                    keep(m);
                }
            }
    // kind 1: covered nodes whose central fine node lies in the fine block, per coarse block
    for (const BlockGeom &fb : fall)
        for (const BlockGeom &cb : call) {
            crocco_amr_msg m;
            memset(&m, 0, sizeof m);
            bool empty = false;
            for (int e = 0; e < 3 && !empty; e++) {
                int64_t lo, hi;
                covered_range_of(fd, c0, e, lo, hi);
                if (sib_mode && fd->bc[e][0] != CROCCO_BC_PERIODIC) {  // central fine node ours;
                    lo = c0[e];                                         // k_average_down checks
                    hi = c0[e] + (fd->n_global[e] - 1) / 2;             // the 27 nodes
                }
                // 2 (I - c0) in [origin, origin + n - 1]
                lo = std::max(lo, c0[e] + (fb.origin[e] + 1) / 2);
                hi = std::min(hi, c0[e] + (fb.origin[e] + fbn[e] - 1) / 2);
                lo = std::max<int64_t>(lo, cb.origin[e]);
                hi = std::min<int64_t>(hi, cb.origin[e] + cbn[e] - 1);
                empty = lo > hi;
                m.lo[e] = lo - cb.origin[e];
                m.ext[e] = hi - lo + 1;
            }
            if (empty) continue;
            m.kind = 1;
            m.coarse_block = cb.gid;
            m.fine_block = fb.gid;
            m.sibling = -1;
            m.src_rank = fb.rank;
            m.dst_rank = cb.rank;
            keep(m);
        }
}

// C/F ghost box (phase D, side) of block fb, [lo, lo+ext) in fine-block-local indices; false when
// the face is not a C/F domain face
static bool cf_ghost_box(const crocco_grid_desc *fd, const int fnb[3], const int fbn[3], const BlockGeom &fb, int D,
                         int side, int64_t lo[3], int64_t ext[3]) {
    if (fd->bc[D][side] != CROCCO_BC_COARSE_FINE || fb.bidx[D] != (side == 0 ? 0 : fnb[D] - 1)) return false;
    for (int e = 0; e < 3; e++) {
        if (e == D) {
            lo[e] = side == 0 ? -G : fbn[e];
            ext[e] = G;
        } else if (e < D) {
            lo[e] = -G;
            ext[e] = fbn[e] + 2 * G;
        } else {
            lo[e] = 0;
            ext[e] = fbn[e];
        }
    }
    return true;
}

// kind 2 (crocco_amr_sibling_plan): the parts of the C/F ghost boxes of f's blocks inside the
// interiors of sibling g's blocks, in the common fine index space 2 c0 + f
static void build_sib_plan(const crocco_grid_desc *fd, const int fnb[3], const int fbn[3],
                           const std::vector<BlockGeom> &fall, const int64_t c0f[3], const int gbn[3],
                           const std::vector<BlockGeom> &gall, const int64_t c0g[3], int sidx, int me,
                           std::vector<crocco_amr_msg> &out) {
    for (const BlockGeom &fb : fall)
        for (int D = 0; D < 3; D++)
            for (int side = 0; side < 2; side++) {
                int64_t lo[3], ext[3];
                if (!cf_ghost_box(fd, fnb, fbn, fb, D, side, lo, ext)) continue;
                for (const BlockGeom &gb : gall) {
                    crocco_amr_msg m;
                    memset(&m, 0, sizeof m);
                    bool empty = false;
                    for (int e = 0; e < 3 && !empty; e++) {
                        const int64_t a0 = 2 * c0f[e] + fb.origin[e] + lo[e], a1 = a0 + ext[e];
                        const int64_t b0 = 2 * c0g[e] + gb.origin[e], b1 = b0 + gbn[e];
                        const int64_t x0 = std::max(a0, b0), x1 = std::min(a1, b1);
                        empty = x0 >= x1;
                        m.lo[e] = x0 - b0;
                        m.ext[e] = x1 - x0;
                    }
                    if (empty) continue;
                    m.kind = 2;
                    m.coarse_block = gb.gid;
                    m.fine_block = fb.gid;
                    m.sibling = sidx;
                    m.src_rank = gb.rank;
                    m.dst_rank = fb.rank;
                    if (me < 0 || m.src_rank == me || m.dst_rank == me) out.push_back(m);
                }
            }
}

crocco_status crocco_amr_sibling_plan(const crocco_grid_desc *fine, const int64_t c0[3], const crocco_grid_desc *sib,
                                      const int64_t c0s[3], int32_t sibling, crocco_amr_msg *out, int32_t cap,
                                      int32_t *n_out) {
    int fnb[3], fbn[3], gnb[3], gbn[3];
    crocco_status st = validate(fine, fnb, fbn);
    if (!st) st = validate(sib, gnb, gbn);
    if (st) return st;
    if (!c0 || !c0s) return fail(nullptr, CROCCO_ERR_ARG, "null c0");
    if (fine->nranks != sib->nranks || fine->rank != sib->rank)
        return fail(nullptr, CROCCO_ERR_ARG, "sibling patches must share the process group");
    std::vector<BlockGeom> fall, gall;
    build_blocks(fine, fnb, fbn, fall);
    build_blocks(sib, gnb, gbn, gall);
    std::vector<crocco_amr_msg> plan;
    build_sib_plan(fine, fnb, fbn, fall, c0, gbn, gall, c0s, sibling, fine->rank, plan);
    if (n_out) *n_out = (int32_t)plan.size();
    for (int i = 0; i < (int)plan.size() && i < cap; i++) out[i] = plan[i];
    return CROCCO_OK;
}

crocco_status crocco_amr_plan(const crocco_grid_desc *fine, const crocco_grid_desc *coarse, const int64_t c0[3],
                              crocco_amr_msg *out, int32_t cap, int32_t *n_out) {
    int fnb[3], fbn[3], cnb[3], cbn[3];
    crocco_status st = validate(fine, fnb, fbn);
    if (!st) st = validate(coarse, cnb, cbn);
    if (st) return st;
    if (!c0) return fail(nullptr, CROCCO_ERR_ARG, "null c0");
    if ((st = amr_geom_check(nullptr, fine, coarse, fnb, cnb, c0))) return st;
    std::vector<BlockGeom> fall, call;
    build_blocks(fine, fnb, fbn, fall);
    build_blocks(coarse, cnb, cbn, call);
    std::vector<crocco_amr_msg> plan;
    build_amr_plan(fine, fnb, fbn, fall, coarse, cnb, cbn, call, c0, fine->rank, false, plan);
    if (n_out) *n_out = (int32_t)plan.size();
    for (int i = 0; i < (int)plan.size() && i < cap; i++) out[i] = plan[i];
    return CROCCO_OK;
}

static void amr_release(crocco_ctx f) {
    for (double *m : f->amr_mirror) cudaFree(m);
    f->amr_mirror.clear();
    f->amr_mirror_gid.clear();
    cudaFree(f->amr_send);
    cudaFree(f->amr_recv);
    f->amr_send = f->amr_recv = nullptr;
    f->amr_stage_elems = 0;
    f->amr_plan.clear();
}

crocco_status crocco_amr_link(crocco_ctx f, crocco_ctx c, const int64_t c0[3]) {
    LIVE(f);
    LIVE(c);
    if (!c0 || f == c) return fail(f, CROCCO_ERR_ARG, "need distinct fine / coarse ctx and c0");
    crocco_status st = amr_geom_check(f, &f->desc, &c->desc, f->nb, c->nb, c0);
    if (st) return st;
    if (f->loc.size() > (size_t)AMR_MAX_LOCAL)
        return fail(f, CROCCO_ERR_ARG, "two-level AMR: at most %d local fine blocks", AMR_MAX_LOCAL);
    std::vector<crocco_amr_msg> plan;
    build_amr_plan(&f->desc, f->nb, f->bn, f->all, &c->desc, c->nb, c->bn, c->all, c0, f->desc.rank, false, plan);
    // slots of the coarse-level table: the local coarse blocks plus the mirrors this rank may use
    std::vector<int> mg;
    for (const crocco_amr_msg &m : plan)
        if ((m.kind == 0 && m.dst_rank == f->desc.rank) || (m.kind == 1 && m.src_rank == f->desc.rank))
            if (std::find(mg.begin(), mg.end(), m.coarse_block) == mg.end()) mg.push_back(m.coarse_block);
    if (c->loc.size() + mg.size() > (size_t)AMR_MAX_LOCAL)
        return fail(f, CROCCO_ERR_ARG, "two-level AMR: %zu local coarse blocks + %zu mirrors > %d", c->loc.size(),
                    mg.size(), AMR_MAX_LOCAL);
    for (const crocco_amr_msg &m : plan)
        if (m.src_rank != m.dst_rank && !f->comm)
            return fail(f, CROCCO_ERR_ARG, "inter-rank AMR boxes need the fine level's communicator");
    amr_release(f);
    f->amr_plan = std::move(plan);
    for (int d = 0; d < 3; d++) f->amr_c0[d] = c0[d];
    f->amr_coarse = c;
    return CROCCO_OK;
}

// a box of the plan goes through ncclSend / ncclRecv (other rank, or loopback)
static bool amr_routed(const crocco_ctx_s *f, const crocco_amr_msg &m) {
    return m.src_rank != m.dst_rank || f->loopback;
}

// mirror of coarse block gid (coarse block layout, 5 comps), allocated zeroed on first use
static double *amr_mirror(crocco_ctx f, int gid) {
    for (size_t i = 0; i < f->amr_mirror_gid.size(); i++)
        if (f->amr_mirror_gid[i] == gid) return f->amr_mirror[i];
    const crocco_ctx_s *c = f->amr_coarse;
    const Lay L = make_layout(c->bn, G);
    double *p = nullptr;
    if (cudaMalloc((void **)&p, (size_t)(5 * L.cs) * sizeof(double)) != cudaSuccess ||
        cudaMemset(p, 0, (size_t)(5 * L.cs) * sizeof(double)) != cudaSuccess) {
        cudaGetLastError();
        cudaFree(p);
        return nullptr;
    }
    f->scratch += 5 * L.cs * (int64_t)sizeof(double);
    f->amr_mirror_gid.push_back(gid);
    f->amr_mirror.push_back(p);
    return p;
}

// box [lo, lo+ext) of a 5-component array in layout L <-> a contiguous staging slice
static BoxOp amr_box_op(double *arr, const Lay &L, const crocco_amr_msg &m, double *stage, bool pack) {
    BoxOp o;
    memset(&o, 0, sizeof o);
    const int64_t vol = m.ext[0] * m.ext[1] * m.ext[2];
    int64_t st[3];
    op_strides(L, st);
    const int64_t base = at(L, (int)m.lo[0], (int)m.lo[1], (int)m.lo[2]);
    const int64_t cst[3] = {1, m.ext[0], m.ext[0] * m.ext[1]};
    if (pack) {
        o.src = arr;
        for (int e = 0; e < 3; e++) o.sst[e] = st[e];
        o.scs = L.cs;
        o.sbase = base;
        o.dst = stage;
        for (int e = 0; e < 3; e++) o.dst_[e] = cst[e];
        o.dcs = vol;
        o.dbase = 0;
    } else {
        o.src = stage;
        for (int e = 0; e < 3; e++) o.sst[e] = cst[e];
        o.scs = vol;
        o.sbase = 0;
        o.dst = arr;
        for (int e = 0; e < 3; e++) o.dst_[e] = st[e];
        o.dcs = L.cs;
        o.dbase = base;
    }
    for (int e = 0; e < 3; e++) o.ext[e] = (int)m.ext[e];
    o.ncomp = 5;
    o.mode = BOX_COPY;
    return o;
}

// The routed boxes of one kind: pack (src arrays) -> grouped ncclSend / ncclRecv -> unpack (dst
// arrays).  src_arr / dst_arr give the array of a box on the sending / receiving side.
typedef std::function<double *(const crocco_amr_msg &)> AmrArr;
typedef std::vector<std::pair<const crocco_amr_msg *, int64_t>> AmrRecv;
// recv_out non-null: the received boxes are not unpacked; (box, offset in amr_recv) are returned
static crocco_status amr_exchange(crocco_ctx f, int kind, const AmrArr &src_arr, const AmrArr &dst_arr,
                                  AmrRecv *recv_out = nullptr) {
    const int me = f->desc.rank;
    std::vector<const crocco_amr_msg *> r;
    int64_t ns = 0, nr = 0;
    for (const crocco_amr_msg &m : f->amr_plan)
        if (m.kind == kind && amr_routed(f, m)) {
            r.push_back(&m);
            const int64_t v = 5 * m.ext[0] * m.ext[1] * m.ext[2];
            if (m.src_rank == me) ns += v;
            if (m.dst_rank == me) nr += v;
        }
    if (r.empty()) return CROCCO_OK;
    if (!f->comm) return fail(f, CROCCO_ERR_STATE, "inter-level boxes without communicator");
    const int64_t need = std::max(ns, nr);
    if (need > f->amr_stage_elems) {
        cudaStreamSynchronize(f->stream);  // the old staging may still be read
        cudaFree(f->amr_send);
        cudaFree(f->amr_recv);
        f->amr_send = f->amr_recv = nullptr;
        if (cudaMalloc((void **)&f->amr_send, (size_t)need * sizeof(double)) != cudaSuccess ||
            cudaMalloc((void **)&f->amr_recv, (size_t)need * sizeof(double)) != cudaSuccess) {
            cudaGetLastError();
            f->amr_stage_elems = 0;
            return fail(f, CROCCO_ERR_NOMEM, "AMR staging allocation failed");
        }
        f->scratch += 2 * (need - f->amr_stage_elems) * (int64_t)sizeof(double);
        f->amr_stage_elems = need;
    }
    const Lay Lc = make_layout(f->amr_coarse->bn, G);
    auto lay = [&](const crocco_amr_msg &m) { return m.kind == 2 ? make_layout(f->sibs[m.sibling]->bn, G) : Lc; };
    BoxOps ops;
    ops.nops = 0;
    crocco_status st;
    std::vector<int64_t> so(r.size()), ro(r.size());
    int64_t s = 0, q = 0;
    for (size_t i = 0; i < r.size(); i++) {
        const int64_t v = 5 * r[i]->ext[0] * r[i]->ext[1] * r[i]->ext[2];
        if (r[i]->dst_rank == me) {
            ro[i] = q;
            q += v;
        }
        if (r[i]->src_rank != me) continue;
        so[i] = s;
        double *a = src_arr(*r[i]);
        if (!a) return fail(f, CROCCO_ERR_NOMEM, "AMR mirror allocation failed");
        if ((st = push_op(f, ops, amr_box_op(a, lay(*r[i]), *r[i], f->amr_send + s, true)))) return st;
        s += v;
    }
    if ((st = flush_ops(f, ops))) return st;
    {
        NvtxRange nv("crocco:nccl_amr");
        NK(f, ncclGroupStart());
        for (size_t i = 0; i < r.size(); i++) {
            const size_t cnt = (size_t)(5 * r[i]->ext[0] * r[i]->ext[1] * r[i]->ext[2]);
            if (r[i]->src_rank == me)
                NK(f, ncclSend(f->amr_send + so[i], cnt, ncclDouble, r[i]->dst_rank, f->comm, f->stream));
            if (r[i]->dst_rank == me)
                NK(f, ncclRecv(f->amr_recv + ro[i], cnt, ncclDouble, r[i]->src_rank, f->comm, f->stream));
        }
        NK(f, ncclGroupEnd());
    }
    for (size_t i = 0; i < r.size(); i++) {
        if (r[i]->dst_rank != me) continue;
        if (recv_out) {
            recv_out->push_back({r[i], ro[i]});
            continue;
        }
        double *a = dst_arr(*r[i]);
        if (!a) return fail(f, CROCCO_ERR_NOMEM, "AMR mirror allocation failed");
        if ((st = push_op(f, ops, amr_box_op(a, lay(*r[i]), *r[i], f->amr_recv + ro[i], false)))) return st;
    }
    return flush_ops(f, ops);
}

// FillPatch, inter-level part: the coarse boxes the C/F interpolation of this rank's fine blocks
// reads from other ranks (or through the loopback) land in the coarse-block mirrors;
// fill_phase then maps those coarse blocks to their mirrors (amr_cf_gids).
static crocco_status amr_fill_exchange(crocco_ctx f) {
    f->amr_cf_gids.clear();
    const crocco_ctx_s *c = f->amr_coarse;
    for (const crocco_amr_msg &m : f->amr_plan)
        if (m.kind == 0 && m.dst_rank == f->desc.rank && amr_routed(f, m) &&
            std::find(f->amr_cf_gids.begin(), f->amr_cf_gids.end(), m.coarse_block) == f->amr_cf_gids.end())
            f->amr_cf_gids.push_back(m.coarse_block);
    double *const *Uc = f->amr_Uc;
    return amr_exchange(
        f, 0, [&](const crocco_amr_msg &m) { return Uc[c->gid_to_local[m.coarse_block]]; },
        [&](const crocco_amr_msg &m) { return amr_mirror(f, m.coarse_block); });
}

// mirror of block gid of sibling s (the sibling's block layout), allocated zeroed on first use;
// amr_sib_mirror_if: the existing one or null (a block no routed box of this rank lands in)
static double *amr_sib_mirror(crocco_ctx f, int s, int gid) {
    const int key = s * AMR_MAX_BLOCKS + gid;
    for (size_t i = 0; i < f->amr_smirror_key.size(); i++)
        if (f->amr_smirror_key[i] == key) return f->amr_smirror[i];
    const Lay L = make_layout(f->sibs[s]->bn, G);
    double *p = nullptr;
    if (cudaMalloc((void **)&p, (size_t)(5 * L.cs) * sizeof(double)) != cudaSuccess ||
        cudaMemset(p, 0, (size_t)(5 * L.cs) * sizeof(double)) != cudaSuccess) {
        cudaGetLastError();
        cudaFree(p);
        return nullptr;
    }
    f->scratch += 5 * L.cs * (int64_t)sizeof(double);
    f->amr_smirror_key.push_back(key);
    f->amr_smirror.push_back(p);
    return p;
}
static double *amr_sib_mirror_if(crocco_ctx f, int s, int gid) {
    const int key = s * AMR_MAX_BLOCKS + gid;
    for (size_t i = 0; i < f->amr_smirror_key.size(); i++)
        if (f->amr_smirror_key[i] == key) return f->amr_smirror[i];
    return nullptr;
}

// same-level part of the C/F fill with siblings: the sibling interior boxes this rank's ghost
// bands copy from other ranks (or through the loopback) land in the sibling-block mirrors
static crocco_status amr_sib_exchange(crocco_ctx f) {
    double *const *const *sU = f->amr_sibU;
    return amr_exchange(
        f, 2,
        [&](const crocco_amr_msg &m) { return sU[m.sibling][f->sibs[m.sibling]->gid_to_local[m.coarse_block]]; },
        [&](const crocco_amr_msg &m) { return amr_sib_mirror(f, m.sibling, m.coarse_block); });
}

static crocco_status amr_ready(crocco_ctx f, double *const *Uc) {
    if (!f->amr_coarse) return fail(f, CROCCO_ERR_ARG, "fine level not linked (crocco_amr_link)");
    if (f->amr_coarse->poisoned) return CROCCO_ERR_STATE;
    if (!f->sibs.empty() && !f->amr_sibU)
        return fail(f, CROCCO_ERR_ARG, "patch has siblings: use the _level calls with their states");
    if (!Uc) return fail(f, CROCCO_ERR_ARG, "null coarse pointer array");
    for (size_t b = 0; b < f->amr_coarse->loc.size(); b++)
        if (!Uc[b]) return fail(f, CROCCO_ERR_ARG, "null coarse pointer for local block %zu", b);
    return CROCCO_OK;
}

crocco_status crocco_fill_patch_two_levels(crocco_ctx f, double *const *Uf, double *const *Mf,
                                           double *const *Uc) {
    LIVE(f);
    crocco_status st = amr_ready(f, Uc);
    if (st) return st;
    f->amr_Uc = Uc;
    st = fill_all(f, Uf, CROCCO_FIELD_STATE, Mf, f->time);
    f->amr_Uc = nullptr;
    return st;
}

crocco_status crocco_amr_rk_stage(crocco_ctx f, int32_t stage, double dt, double *const *Uin,
                                  double *const *Uout, double *const *dU, double *const *M,
                                  double *const *Uc_in) {
    LIVE(f);
    crocco_status st = amr_ready(f, Uc_in);
    if (st) return st;
    f->amr_Uc = Uc_in;
    st = crocco_rk_stage(f, stage, dt, Uin, Uout, dU, M);
    f->amr_Uc = nullptr;
    return st;
}

crocco_status crocco_average_down(crocco_ctx f, double *const *Uf, double *const *Uc) {
    LIVE(f);
    NvtxRange nv("crocco:average_down");
    crocco_status st = amr_ready(f, Uc);
    if (st) return st;
    if ((st = check_ptrs(f, Uf, "U_fine"))) return st;
    // same-level ghosts of the fine state (copies only; C/F and physical ghosts are not read)
    if ((st = fill_all(f, Uf, FILL_STATE_COPIES, nullptr, f->time))) return st;
    const crocco_ctx_s *c = f->amr_coarse;
    LevelTab ft;
    level_tab(f, Uf, ft);
    SibTab sb;
    sib_tab(f, sb);
    ADOps ops;
    memset(&ops, 0, sizeof ops);
    ops.Lc = make_layout(c->bn, G);
    for (int d = 0; d < 3; d++) {
        ops.c0[d] = f->amr_c0[d];
        ops.Nf[d] = f->desc.n_global[d];
        ops.per[d] = f->desc.bc[d][0] == CROCCO_BC_PERIODIC;
    }
    int64_t mx = 0;
    auto flush = [&]() -> crocco_status {
        if (ops.nops == 0) return CROCCO_OK;
        dim3 grid(std::min<int64_t>(cdiv(mx, 256), 4096), ops.nops);
        LAUNCH(f, K_AMR, k_average_down<<<grid, 256, 0, f->stream>>>(ops, ft, sb));
        ops.nops = 0;
        mx = 0;
        return CROCCO_OK;
    };
    auto push = [&](double *dst, const Lay &Lb, const int64_t org[3], const int64_t lo[3], const int64_t hi[3],
                    const double *buf) -> crocco_status {
        ADOp &o = ops.op[ops.nops++];
        o.dst = dst;
        o.buf = buf;
        o.dbase = at(Lb, (int)(lo[0] - org[0]), (int)(lo[1] - org[1]), (int)(lo[2] - org[2]));
        for (int d = 0; d < 3; d++) {
            o.ext[d] = (int)(hi[d] - lo[d] + 1);
            o.Io[d] = lo[d];
        }
        mx = std::max<int64_t>(mx, (int64_t)o.ext[0] * o.ext[1] * o.ext[2]);
        return ops.nops == CF_MAX_OPS ? flush() : CROCCO_OK;
    };
    // the plan's kind-1 boxes computed on this rank: in place when the coarse block is ours,
    // else (or under the loopback) into its mirror, then sent to the coarse block's rank; with
    // siblings the boxes hold the nodes whose central fine node is ours and k_average_down keeps
    // those whose 27 fine nodes lie in the level's patch interiors (reading 31)
    for (const crocco_amr_msg &m : f->amr_plan) {
        if (m.kind != 1 || m.src_rank != f->desc.rank) continue;
        const BlockGeom &cb = c->all[m.coarse_block];
        double *dst = amr_routed(f, m) ? amr_mirror(f, m.coarse_block) : Uc[c->gid_to_local[m.coarse_block]];
        if (!dst) return fail(f, CROCCO_ERR_NOMEM, "AMR mirror allocation failed");
        int64_t lo[3], hi[3];
        for (int d = 0; d < 3; d++) {
            lo[d] = cb.origin[d] + m.lo[d];
            hi[d] = lo[d] + m.ext[d] - 1;
        }
        if ((st = push(dst, ops.Lc, cb.origin, lo, hi, nullptr))) return st;
    }
    if ((st = flush())) return st;
    // the boxes averaged on other ranks: their covered nodes (the same 27-node rule, evaluated
    // here) take the received values -- the others of a sibling-mode box were not averaged
    AmrRecv got;
    if ((st = amr_exchange(
             f, 1, [&](const crocco_amr_msg &m) { return amr_mirror(f, m.coarse_block); },
             [&](const crocco_amr_msg &) { return (double *)nullptr; }, &got)))
        return st;
    for (auto &g : got) {
        const crocco_amr_msg &m = *g.first;
        const BlockGeom &cb = c->all[m.coarse_block];
        int64_t lo[3], hi[3];
        for (int d = 0; d < 3; d++) {
            lo[d] = cb.origin[d] + m.lo[d];
            hi[d] = lo[d] + m.ext[d] - 1;
        }
        if ((st = push(Uc[c->gid_to_local[m.coarse_block]], ops.Lc, cb.origin, lo, hi, f->amr_recv + g.second)))
            return st;
    }
    return flush();
}

// f's plan with its siblings: kind-1 boxes over the nodes whose central fine node is f's, plus the
// kind-2 boxes of every sibling in link order
static crocco_status amr_rebuild_plan(crocco_ctx f) {
    const crocco_ctx_s *c = f->amr_coarse;
    std::vector<crocco_amr_msg> plan;
    build_amr_plan(&f->desc, f->nb, f->bn, f->all, &c->desc, c->nb, c->bn, c->all, f->amr_c0, f->desc.rank,
                   !f->sibs.empty(), plan);
    for (size_t i = 0; i < f->sibs.size(); i++) {
        const crocco_ctx_s *g = f->sibs[i];
        build_sib_plan(&f->desc, f->nb, f->bn, f->all, f->amr_c0, g->bn, g->all, g->amr_c0, (int)i, f->desc.rank,
                       plan);
    }
    for (const crocco_amr_msg &m : plan)
        if (m.src_rank != m.dst_rank && !f->comm)
            return fail(f, CROCCO_ERR_ARG, "inter-rank AMR boxes need the patch's communicator");
    f->amr_plan = std::move(plan);
    return CROCCO_OK;
}

crocco_status crocco_amr_link_sibling(crocco_ctx f, crocco_ctx g) {
    LIVE(f);
    LIVE(g);
    if (f == g) return fail(f, CROCCO_ERR_ARG, "a patch is not its own sibling");
    if (!f->amr_coarse || f->amr_coarse != g->amr_coarse)
        return fail(f, CROCCO_ERR_ARG, "siblings must be linked (crocco_amr_link) to the same coarse level");
    if (f->desc.nranks != g->desc.nranks || f->desc.rank != g->desc.rank)
        return fail(f, CROCCO_ERR_ARG, "sibling patches must share the process group");
    for (auto s : f->sibs)
        if (s == g) return CROCCO_OK;
    if (f->sibs.size() >= 8 || g->sibs.size() >= 8) return fail(f, CROCCO_ERR_ARG, "at most 8 siblings per patch");
    int nb = 0;
    for (auto s : f->sibs) nb += (int)s->all.size();
    int ng = 0;
    for (auto s : g->sibs) ng += (int)s->all.size();
    if (nb + (int)g->all.size() > SIB_MAX_BLOCKS || ng + (int)f->all.size() > SIB_MAX_BLOCKS)
        return fail(f, CROCCO_ERR_ARG, "at most %d sibling blocks per patch", SIB_MAX_BLOCKS);
    // interiors disjoint (in the common fine index space 2 c0 + f); a periodic direction spans all
    bool overlap = true;
    for (int d = 0; d < 3; d++) {
        if (f->desc.bc[d][0] == CROCCO_BC_PERIODIC || g->desc.bc[d][0] == CROCCO_BC_PERIODIC) continue;
        const int64_t a0 = 2 * f->amr_c0[d], a1 = a0 + f->desc.n_global[d];
        const int64_t b0 = 2 * g->amr_c0[d], b1 = b0 + g->desc.n_global[d];
        overlap = overlap && a0 < b1 && b0 < a1;
        if (((b0 - a0) & 1) != 0) return fail(f, CROCCO_ERR_ARG, "sibling offset must be even in direction %d", d);
    }
    if (overlap) return fail(f, CROCCO_ERR_ARG, "sibling patches overlap");
    f->sibs.push_back(g);
    g->sibs.push_back(f);
    crocco_status st = amr_rebuild_plan(f);
    if (!st) st = amr_rebuild_plan(g);
    if (st) {
        f->sibs.pop_back();
        g->sibs.pop_back();
        amr_rebuild_plan(f);
        amr_rebuild_plan(g);
    }
    return st;
}

static crocco_status sib_ready(crocco_ctx f, double *const *const *sibU) {
    if (f->sibs.empty()) return CROCCO_OK;
    if (!sibU) return fail(f, CROCCO_ERR_ARG, "null sibling pointer table");
    for (size_t s = 0; s < f->sibs.size(); s++) {
        if (!sibU[s]) return fail(f, CROCCO_ERR_ARG, "null sibling %zu pointer array", s);
        for (size_t b = 0; b < f->sibs[s]->loc.size(); b++)
            if (!sibU[s][b]) return fail(f, CROCCO_ERR_ARG, "null sibling %zu block %zu pointer", s, b);
    }
    return CROCCO_OK;
}

crocco_status crocco_fill_patch_level(crocco_ctx f, double *const *Uf, double *const *Mf, double *const *Uc,
                                      double *const *const *sibU) {
    LIVE(f);
    crocco_status st = sib_ready(f, sibU);
    if (st) return st;
    f->amr_sibU = sibU;
    st = crocco_fill_patch_two_levels(f, Uf, Mf, Uc);
    f->amr_sibU = nullptr;
    return st;
}

crocco_status crocco_amr_rk_stage_level(crocco_ctx f, int32_t stage, double dt, double *const *Uin,
                                        double *const *Uout, double *const *dU, double *const *M,
                                        double *const *Uc_in, double *const *const *sib_in) {
    LIVE(f);
    crocco_status st = sib_ready(f, sib_in);
    if (st) return st;
    f->amr_sibU = sib_in;
    st = crocco_amr_rk_stage(f, stage, dt, Uin, Uout, dU, M, Uc_in);
    f->amr_sibU = nullptr;
    return st;
}

crocco_status crocco_average_down_level(crocco_ctx f, double *const *Uf, double *const *Uc,
                                        double *const *const *sibU) {
    LIVE(f);
    crocco_status st = sib_ready(f, sibU);
    if (st) return st;
    f->amr_sibU = sibU;
    st = crocco_average_down(f, Uf, Uc);
    f->amr_sibU = nullptr;
    return st;
}

crocco_status crocco_check_state(crocco_ctx c, double *const *U, int64_t *n_bad) {
    LIVE(c);
    crocco_status st = check_ptrs(c, U, "U");
    if (st) return st;
    if (!n_bad) return fail(c, CROCCO_ERR_ARG, "null n_bad");
    if (!c->dmax) CK(c, cudaMalloc((void **)&c->dmax, sizeof(unsigned long long)));
    CK(c, cudaMemsetAsync(c->dmax, 0, sizeof(unsigned long long), c->stream));
    for (size_t bi = 0; bi < c->loc.size(); bi++) {
        const LocalBlock &b = c->loc[bi];
        const int64_t tot = (int64_t)b.g.n[0] * b.g.n[1] * b.g.n[2];
        const unsigned grid = (unsigned)std::min<int64_t>(cdiv(tot, 256), 148 * 8);
        LAUNCH(c, K_CFL, k_check_state<<<grid, 256, 0, c->stream>>>(U[bi], b.L, c->ph, c->dmax));
    }
    unsigned long long h = 0;
    CK(c, cudaMemcpyAsync(&h, c->dmax, sizeof h, cudaMemcpyDeviceToHost, c->stream));
    CK(c, cudaStreamSynchronize(c->stream));
    *n_bad = (int64_t)h;
    return CROCCO_OK;
}

crocco_status crocco_sync(crocco_ctx c) {
    LIVE(c);
    CK(c, cudaStreamSynchronize(c->stream));
    CK(c, cudaGetLastError());
    return CROCCO_OK;
}

crocco_status crocco_finalize(crocco_ctx c) {
    if (!c) return CROCCO_OK;
    cudaStreamSynchronize(c->stream);
    free_ctx(c);
    return CROCCO_OK;
}

crocco_status crocco_launch_count(crocco_ctx c, int64_t *count, int32_t reset) {
    if (!c) return fail(nullptr, CROCCO_ERR_ARG, "null ctx");
    if (count) *count = c->launches;
    if (reset) c->launches = 0;
    return CROCCO_OK;
}

crocco_status crocco_set_overlap(crocco_ctx c, int32_t enable) {
    LIVE(c);
    if (enable < -1 || enable > 1) return fail(c, CROCCO_ERR_ARG, "overlap must be -1, 0 or 1");
    if (enable != c->overlap) drop_graphs(c);  // the captured stage structure changes
    c->overlap = enable;
    return CROCCO_OK;
}

crocco_status crocco_set_nccl_loopback(crocco_ctx c, int32_t enable) {
    LIVE(c);
    if (c->desc.nranks != 1) return fail(c, CROCCO_ERR_ARG, "NCCL loopback is a single-rank debug mode");
    drop_graphs(c);
    if (!enable) {
        c->loopback = false;
        if (c->comm) ncclCommDestroy(c->comm);
        c->comm = nullptr;
        return CROCCO_OK;
    }
    // staging for every same-rank copy of a phase, sent and received by this rank
    int64_t maxe = 0;
    for (int d = 0; d < 3; d++) {
        int64_t v = 0;
        for (auto &m : c->plan[d])
            if (m.kind == 0) v += m.ext[0] * m.ext[1] * m.ext[2] * 10;
        maxe = std::max(maxe, v);
    }
    if (maxe > c->stage_elems) {
        cudaFree(c->send_stage);
        cudaFree(c->recv_stage);
        c->send_stage = c->recv_stage = nullptr;
        if (cudaMalloc((void **)&c->send_stage, (size_t)maxe * sizeof(double)) != cudaSuccess ||
            cudaMalloc((void **)&c->recv_stage, (size_t)maxe * sizeof(double)) != cudaSuccess) {
            cudaGetLastError();
            c->stage_elems = 0;
            return fail(c, CROCCO_ERR_NOMEM, "loopback staging allocation failed");
        }
        c->scratch += 2 * (maxe - c->stage_elems) * (int64_t)sizeof(double);
        c->stage_elems = maxe;
    }
    if (!c->comm) {
        ncclUniqueId id;
        NK(c, ncclGetUniqueId(&id));
        NK(c, ncclCommInitRank(&c->comm, 1, id, 0));
    }
    c->loopback = true;
    return CROCCO_OK;
}

crocco_status crocco_overlap_count(crocco_ctx c, int64_t *count, int32_t reset) {
    if (!c) return fail(nullptr, CROCCO_ERR_ARG, "null ctx");
    if (count) *count = c->overlapped_stages;
    if (reset) c->overlapped_stages = 0;
    return CROCCO_OK;
}

crocco_status crocco_set_timing(crocco_ctx c, int32_t enable) {
    LIVE(c);
    c->timing = enable != 0;
    return CROCCO_OK;
}

crocco_status crocco_kernel_times(crocco_ctx c, int32_t maxc, int64_t *launches, double *ms,
                                  int32_t *ncls) {
    LIVE(c);
    for (auto &t : c->pending) {
        CK(c, cudaEventSynchronize(t.e1));
        float f = 0.f;
        CK(c, cudaEventElapsedTime(&f, t.e0, t.e1));
        c->t_launch[t.cls]++;
        c->t_ms[t.cls] += f;
        c->pool.push_back(t.e0);
        c->pool.push_back(t.e1);
    }
    c->pending.clear();
    if (ncls) *ncls = K_NCLASS;
    for (int k = 0; k < K_NCLASS && k < maxc; k++) {
        if (launches) launches[k] = c->t_launch[k];
        if (ms) ms[k] = c->t_ms[k];
        c->t_launch[k] = 0;
        c->t_ms[k] = 0;
    }
    return CROCCO_OK;
}

}  // extern "C"
