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
    int mode;       // 0 copy, 1 constant
    int flip_mom;   // negate comps 1..3
    double val[5];
};
constexpr int MAX_OPS = 16;
struct BoxOps {
    BoxOp op[MAX_OPS];
    int nops;
};
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
        if (o.mode == 1) {
            for (int q = 0; q < o.ncomp; q++) o.dst[q * o.dcs + dp] = o.val[q];
        } else {
            const int64_t sp = o.sbase + a * o.sst[0] + b * o.sst[1] + c * o.sst[2];
            for (int q = 0; q < o.ncomp; q++) {
                double v = o.src[q * o.scs + sp];
                if (o.flip_mom && q >= 1 && q <= 3) v = -v;
                o.dst[q * o.dcs + dp] = v;
            }
        }
    }
}

}  // namespace crocco
