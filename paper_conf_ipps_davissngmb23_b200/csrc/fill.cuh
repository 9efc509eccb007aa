// fill.cuh -- ghost fill box operations (FillPatch / BC_Fill).
// Part of libcrocco (sm_100a, fp64). Formulas restate the paper's method as
// read in DESIGN.md sec. 3 (citations: PAPER.md line numbers); no code is
// shared with oracle/.
#pragma once
#include "common.cuh"
#include "amr.cuh"  // LevelTab

namespace crocco {

// ---------------------------------------------------------------------------
// Ghost fill: generic strided box copy / BC op (FillPatch, BC_Fill;
// PAPER.md:83, 108-109).  dst(t) = sign_c * src(src_base + t.src_stride) or a
// constant; src strides may be 0 (extrapolation) or negative (mirror).
// ---------------------------------------------------------------------------
struct BoxOp {
    const double *src;
    double *dst;
    int64_t sbase, sst[3], scs;  // src element of box origin (comp 0), strides, comp stride
    int64_t dbase, dst_[3], dcs;
    int ext[3];
    int ncomp;
    int mode;        // BOX_COPY / BOX_CONST / BOX_WALL / BOX_SLIP / BOX_SPLIT
    double val[5];   // constant state (CONST) / left state (SPLIT)
    const double *met;  // SLIP / SPLIT: metric row m^d (comp 0) indexed like src
    int64_t mcs;
    int axis;           // SPLIT: tangential axis (0..2) of the box, global index g0 + local
    int64_t g0;
    double s;           // split position at the fill time
    int right_mode;     // SPLIT: BOX_CONST (rval) or BOX_SLIP
    double rval[5];
};
enum { BOX_COPY = 0, BOX_CONST = 1, BOX_WALL = 2, BOX_SLIP = 3, BOX_SPLIT = 4 };
constexpr int MAX_OPS = 16;
struct BoxOps {
    BoxOp op[MAX_OPS];
    int nops;
};

// inviscid reflecting wall: momentum reflected about the plane normal to m^d/|m^d|
__device__ __forceinline__ void slip_reflect(const BoxOp &o, int64_t sp, double v[5]) {
    const double mx = o.met[sp], my = o.met[o.mcs + sp], mz = o.met[2 * o.mcs + sp];
    const double mm = sqrt(mx * mx + my * my + mz * mz);
    const double nx = mx / mm, ny = my / mm, nz = mz / mm;
    const double md = v[1] * nx + v[2] * ny + v[3] * nz;
    v[1] = v[1] - 2.0 * md * nx;
    v[2] = v[2] - 2.0 * md * ny;
    v[3] = v[3] - 2.0 * md * nz;
}

__global__ void __launch_bounds__(256) k_boxops(const __grid_constant__ BoxOps ops) {
    const BoxOp &o = ops.op[blockIdx.y];
    const int64_t tot = (int64_t)o.ext[0] * o.ext[1] * o.ext[2];
    for (int64_t t = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; t < tot;
         t += (int64_t)gridDim.x * blockDim.x) {
        const int a = (int)(t % o.ext[0]);
        const int64_t r = t / o.ext[0];
        const int b = (int)(r % o.ext[1]);
        const int c = (int)(r / o.ext[1]);
        const int64_t dp = o.dbase + a * o.dst_[0] + b * o.dst_[1] + c * o.dst_[2];
        const int64_t sp = o.sbase + a * o.sst[0] + b * o.sst[1] + c * o.sst[2];
        int mode = o.mode;
        const double *cst = o.val;
        if (mode == BOX_SPLIT) {
            const int loc = o.axis == 0 ? a : (o.axis == 1 ? b : c);
            if ((double)(o.g0 + loc) + 0.5 < o.s) {
                mode = BOX_CONST;
            } else {
                mode = o.right_mode;
                cst = o.rval;
            }
        }
        if (mode == BOX_CONST) {
            for (int q = 0; q < o.ncomp; q++) o.dst[q * o.dcs + dp] = cst[q];
            continue;
        }
        if (mode == BOX_COPY) {
            for (int q = 0; q < o.ncomp; q++) o.dst[q * o.dcs + dp] = o.src[q * o.scs + sp];
            continue;
        }
        double v[5];
#pragma unroll
        for (int q = 0; q < 5; q++) v[q] = o.src[q * o.scs + sp];
        if (mode == BOX_WALL) {
            v[1] = -v[1];
            v[2] = -v[2];
            v[3] = -v[3];
        } else {
            slip_reflect(o, sp, v);
        }
#pragma unroll
        for (int q = 0; q < 5; q++) o.dst[q * o.dcs + dp] = v[q];
    }
}

// ---------------------------------------------------------------------------
// Single-pass ghost fill (one launch instead of three): for faces that are
// PERIODIC, EXTRAP, WALL or DIRICHLET and blocks that all live on this rank, the
// 3-phase fill (reading 16) of a ghost point equals resolving its source from the
// HIGHEST direction in which it is a ghost down to the lowest: phase d of the
// fill writes the point from its d-source, which is still a ghost in the lower
// directions and was written by an earlier phase.  Per direction: PERIODIC wraps,
// EXTRAP clamps, WALL mirrors about the face and flips the momentum sign,
// DIRICHLET ends the chain with the constant state.  Bitwise equal to the phases.
// ---------------------------------------------------------------------------
struct GatherArgs {
    LevelTab t;                 // the local blocks (pointers, layout, global size, gid -> local)
    int64_t org[AMR_MAX_LOCAL][3];  // global origin of each local block
    int bc[3][2];
    double dir[3][2][5];
};

__global__ void __launch_bounds__(256) k_fill_gather(const __grid_constant__ GatherArgs ga) {
    const LevelTab &T = ga.t;
    const Lay &L = T.L;
    const int n0 = T.bn[0], n1 = T.bn[1], n2 = T.bn[2];
    const int P0 = n0 + 2 * G, P1 = n1 + 2 * G;
    // ghost shell of one block: k-slabs (2G planes of P0 P1), j-slabs (2G x n2 x P0), i-slabs (2G x n2 x n1)
    const int64_t nK = (int64_t)2 * G * P0 * P1, nJ = (int64_t)2 * G * n2 * P0, nI = (int64_t)2 * G * n2 * n1;
    const int lb = blockIdx.y;
    double *dst = const_cast<double *>(T.p[lb]);
    const int64_t *org = ga.org[lb];
    for (int64_t t = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; t < nK + nJ + nI;
         t += (int64_t)gridDim.x * blockDim.x) {
        int i, j, k;
        if (t < nK) {
            const int a = (int)(t % P0);
            const int64_t r = t / P0;
            const int b = (int)(r % P1), c = (int)(r / P1);  // c in [0, 2G)
            i = a - G;
            j = b - G;
            k = c < G ? c - G : n2 + (c - G);
        } else if (t < nK + nJ) {
            const int64_t u = t - nK;
            const int a = (int)(u % P0);
            const int64_t r = u / P0;
            const int b = (int)(r % (2 * G)), c = (int)(r / (2 * G));
            i = a - G;
            j = b < G ? b - G : n1 + (b - G);
            k = c;
        } else {
            const int64_t u = t - nK - nJ;
            const int a = (int)(u % (2 * G));
            const int64_t r = u / (2 * G);
            const int b = (int)(r % n1), c = (int)(r / n1);
            i = a < G ? a - G : n0 + (a - G);
            j = b;
            k = c;
        }
        int64_t g[3] = {org[0] + i, org[1] + j, org[2] + k};
        bool flip = false, cst = false;
        double cv[5];
#pragma unroll
        for (int d = 2; d >= 0; d--) {
            if (cst) break;
            const int64_t N = T.N[d];
            if (g[d] >= 0 && g[d] < N) continue;
            const int side = g[d] < 0 ? 0 : 1;
            const int kind = ga.bc[d][side];
            if (kind == 0) {                   // PERIODIC
                g[d] = side == 0 ? g[d] + N : g[d] - N;
            } else if (kind == 1) {            // EXTRAP
                g[d] = side == 0 ? 0 : N - 1;
            } else if (kind == 3) {            // WALL: mirror about the face, momentum negated
                g[d] = side == 0 ? -1 - g[d] : 2 * N - 1 - g[d];
                flip = !flip;
            } else {                           // DIRICHLET: the constant state ends the chain
#pragma unroll
                for (int q = 0; q < 5; q++) cv[q] = ga.dir[d][side][q];
                cst = true;
            }
        }
        double v[5];
        if (cst) {
#pragma unroll
            for (int q = 0; q < 5; q++) v[q] = cv[q];
        } else {
            int sb[3];
#pragma unroll
            for (int d = 0; d < 3; d++) sb[d] = (int)(g[d] / T.bn[d]);
            const int sl = T.g2l[sb[0] + T.nb[0] * (sb[1] + T.nb[1] * sb[2])];
            const double *src = T.p[sl];
            const int64_t sp = at(L, (int)(g[0] - (int64_t)sb[0] * n0), (int)(g[1] - (int64_t)sb[1] * n1),
                                  (int)(g[2] - (int64_t)sb[2] * n2));
#pragma unroll
            for (int q = 0; q < 5; q++) v[q] = src[q * L.cs + sp];
        }
        if (flip) {
            v[1] = -v[1];
            v[2] = -v[2];
            v[3] = -v[3];
        }
        const int64_t dp = at(L, i, j, k);
#pragma unroll
        for (int q = 0; q < 5; q++) dst[q * L.cs + dp] = v[q];
    }
}

}  // namespace crocco
