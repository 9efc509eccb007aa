// fill.cuh -- ghost fill box operations (FillPatch / BC_Fill).
// Part of libcrocco (sm_100a, fp64). Formulas restate the paper's method as
// read in DESIGN.md sec. 3 (citations: PAPER.md line numbers); no code is
// shared with oracle/.
#pragma once
#include "common.cuh"

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

}  // namespace crocco
