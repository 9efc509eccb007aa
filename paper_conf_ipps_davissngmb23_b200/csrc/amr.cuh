// amr.cuh -- two-level block-structured AMR kernels (the
// paper's v2.1 path: FillPatchTwoLevels with a trilinear interpolator and
// AverageDown; readings 24-26).
// Part of libcrocco (sm_100a, fp64); no code shared with oracle/.
//
// Refinement ratio 2, node-centred: fine node f of the fine level lies at coarse
// index c0 + f/2.  Both kernels are pure HBM gathers (a few dozen bytes per
// point, no reuse worth staging): one thread per written point, consecutive
// threads on consecutive i, so every load and store is a coalesced row access.
#pragma once
#include "common.cuh"

namespace crocco {

constexpr int AMR_MAX_LOCAL = 64;    // local blocks of the source level per call
constexpr int AMR_MAX_BLOCKS = 512;  // blocks of the source level (gid -> local table)

// The local blocks of one level (equal blocks, so one layout).
struct LevelTab {
    const double *p[AMR_MAX_LOCAL];
    int16_t g2l[AMR_MAX_BLOCKS];  // global block id -> local index, -1 when remote
    Lay L;
    int bn[3];     // block interior size
    int nb[3];     // blocks per direction
    int64_t N[3];  // global interior size
};

__device__ __forceinline__ int64_t floor_half(int64_t h) { return h >= 0 ? h / 2 : -((-h + 1) / 2); }

// Blocks of the same-level sibling patches of a fine level (reading 31): box [lo, hi) of the
// block's interior in this level's fine index space, its state array and layout.
constexpr int SIB_MAX_BLOCKS = 16;
struct SibTab {
    int n;
    int64_t lo[SIB_MAX_BLOCKS][3], hi[SIB_MAX_BLOCKS][3];
    const double *p[SIB_MAX_BLOCKS];
    Lay L[SIB_MAX_BLOCKS];
};
// sibling block holding fine point f (this level's fine index), or -1
__device__ __forceinline__ int sib_find(const SibTab &sb, const int64_t f[3]) {
    for (int s = 0; s < sb.n; s++)
        if (f[0] >= sb.lo[s][0] && f[0] < sb.hi[s][0] && f[1] >= sb.lo[s][1] && f[1] < sb.hi[s][1] &&
            f[2] >= sb.lo[s][2] && f[2] < sb.hi[s][2])
            return s;
    return -1;
}

// One ghost box of a fine block on a COARSE_FINE face.
struct CFOp {
    double *dst;
    int64_t dbase;  // element of the box origin (comp 0)
    int ext[3];
    int64_t fo[3];  // fine-level index of the box origin
};
constexpr int CF_MAX_OPS = 16;
struct CFOps {
    CFOp op[CF_MAX_OPS];
    int nops;
    int interp;     // 1: points outside the siblings interpolated; 0: sibling copies only
    Lay Lf;         // fine block layout
    int64_t c0[3];  // coarse index of fine node 0
};

// FillPatchTwoLevels, C/F ghosts (reading 25): trilinear in index space from the
// 8 coarse nodes around c0 + f/2 (weights 1, 1/2 or 0 per direction, corner order
// e0 fastest).  The coarse state's ghosts must be filled (they supply corners
// beyond block faces and outside the domain).
// A point inside a same-level sibling takes the sibling's value instead (FillBoundary between
// the level's patches, reading 31).
__global__ void __launch_bounds__(256) k_cf_interp(const __grid_constant__ CFOps ops,
                                                   const __grid_constant__ LevelTab ct,
                                                   const __grid_constant__ SibTab sb) {
    const CFOp &o = ops.op[blockIdx.y];
    const int64_t tot = (int64_t)o.ext[0] * o.ext[1] * o.ext[2];
    const Lay &Lc = ct.L;
    for (int64_t t = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; t < tot;
         t += (int64_t)gridDim.x * blockDim.x) {
        const int a = (int)(t % o.ext[0]);
        const int64_t r = t / o.ext[0];
        const int b = (int)(r % o.ext[1]);
        const int c = (int)(r / o.ext[1]);
        const int loc[3] = {a, b, c};
        const int64_t dp = o.dbase + a + b * ops.Lf.py + c * ops.Lf.pz;
        if (sb.n > 0) {
            const int64_t f[3] = {o.fo[0] + a, o.fo[1] + b, o.fo[2] + c};
            const int s = sib_find(sb, f);
            if (s >= 0) {
                const Lay &Ls = sb.L[s];
                const int64_t ps = at(Ls, (int)(f[0] - sb.lo[s][0]), (int)(f[1] - sb.lo[s][1]), (int)(f[2] - sb.lo[s][2]));
#pragma unroll
                for (int q = 0; q < 5; q++) o.dst[q * ops.Lf.cs + dp] = sb.p[s][q * Ls.cs + ps];
                continue;
            }
        }
        if (!ops.interp) continue;
        int64_t I[3];
        double tt[3];
        int bx[3];
#pragma unroll
        for (int d = 0; d < 3; d++) {
            const int64_t h = 2 * ops.c0[d] + o.fo[d] + loc[d];
            I[d] = floor_half(h);
            tt[d] = (double)(h - 2 * I[d]) * 0.5;
            const int64_t Ic = I[d] < 0 ? 0 : (I[d] >= ct.N[d] ? ct.N[d] - 1 : I[d]);  // owner block
            bx[d] = (int)(Ic / ct.bn[d]);
            I[d] -= (int64_t)bx[d] * ct.bn[d];  // block-local index (may reach into the ghosts)
        }
        const int l = ct.g2l[bx[0] + ct.nb[0] * (bx[1] + ct.nb[1] * bx[2])];
        const double *src = ct.p[l];
        double v[5] = {0.0, 0.0, 0.0, 0.0, 0.0};
#pragma unroll
        for (int e = 0; e < 8; e++) {
            const int e0 = e & 1, e1 = (e >> 1) & 1, e2 = (e >> 2) & 1;
            const double w0 = e0 ? tt[0] : 1.0 - tt[0];
            const double w1 = e1 ? tt[1] : 1.0 - tt[1];
            const double w2 = e2 ? tt[2] : 1.0 - tt[2];
            const double w = w0 * w1 * w2;  // dyadic: every product and w * U below is exact
            const int64_t p = at(Lc, (int)(I[0] + e0), (int)(I[1] + e1), (int)(I[2] + e2));
#pragma unroll
            for (int q = 0; q < 5; q++) v[q] = v[q] + w * src[q * Lc.cs + p];
        }
#pragma unroll
        for (int q = 0; q < 5; q++) o.dst[q * ops.Lf.cs + dp] = v[q];
    }
}

// AverageDown (reading 26): covered coarse node I <- trapezoid average of the fine
// data over its cell, sum_{c,b,a} w_a w_b w_c U_f(2(I - c0) + (a, b, c)) with
// w = (1/4, 1/2, 1/4), sum order c outer, a inner.  The fine level's same-level
// ghosts must be filled (fine nodes next to a fine block face).
struct ADOp {
    double *dst;     // coarse block state
    int64_t dbase;   // element of the box origin
    int ext[3];
    int64_t Io[3];   // coarse global index of the box origin
    const double *buf;  // non-null: averages received from the fine block's rank (box order, 5
                        // comps) -- the covered nodes of the box take them (the others keep dst)
};
struct ADOps {
    ADOp op[CF_MAX_OPS];
    int nops;
    Lay Lc;
    int64_t c0[3];
    int64_t Nf[3];   // fine level interior size
    int per[3];      // fine level spans direction d periodically
};
// With siblings (reading 31) the boxes hold the nodes whose central fine node lies in this level;
// a node is averaged when its 27 fine nodes lie in this level's interior or a sibling's.
__device__ __forceinline__ bool ad_covered(const ADOps &ops, const SibTab &sb, const int64_t f[3]) {
    if (sb.n == 0) return true;  // the host boxes are the covered set
    for (int cz = -1; cz <= 1; cz++)
        for (int cy = -1; cy <= 1; cy++)
            for (int cx = -1; cx <= 1; cx++) {
                const int64_t g[3] = {f[0] + cx, f[1] + cy, f[2] + cz};
                bool in = true;
                for (int d = 0; d < 3; d++) in = in && (ops.per[d] || (g[d] >= 0 && g[d] < ops.Nf[d]));
                if (!in && sib_find(sb, g) < 0) return false;
            }
    return true;
}

__global__ void __launch_bounds__(256) k_average_down(const __grid_constant__ ADOps ops,
                                                      const __grid_constant__ LevelTab ft,
                                                      const __grid_constant__ SibTab sb) {
    const ADOp &o = ops.op[blockIdx.y];
    const int64_t tot = (int64_t)o.ext[0] * o.ext[1] * o.ext[2];
    const Lay &Lf = ft.L;
    const double wt[3] = {0.25, 0.5, 0.25};
    for (int64_t t = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; t < tot;
         t += (int64_t)gridDim.x * blockDim.x) {
        const int a = (int)(t % o.ext[0]);
        const int64_t r = t / o.ext[0];
        const int b = (int)(r % o.ext[1]);
        const int c = (int)(r / o.ext[1]);
        const int loc[3] = {a, b, c};
        int64_t fc[3], fg[3];
        int bx[3];
#pragma unroll
        for (int d = 0; d < 3; d++) {
            const int64_t f = 2 * (o.Io[d] + loc[d] - ops.c0[d]);  // inside [0, N_f) by coverage
            fg[d] = f;
            bx[d] = (int)(f / ft.bn[d]);
            fc[d] = f - (int64_t)bx[d] * ft.bn[d];
        }
        if (!ad_covered(ops, sb, fg)) continue;
        const int64_t dp = o.dbase + a + b * ops.Lc.py + c * ops.Lc.pz;
        if (o.buf) {
#pragma unroll
            for (int q = 0; q < 5; q++) o.dst[q * ops.Lc.cs + dp] = o.buf[q * tot + t];
            continue;
        }
        const double *src = ft.p[ft.g2l[bx[0] + ft.nb[0] * (bx[1] + ft.nb[1] * bx[2])]];
        const int64_t pc = at(Lf, (int)fc[0], (int)fc[1], (int)fc[2]);
#pragma unroll
        for (int q = 0; q < 5; q++) {
            const double *s = src + q * Lf.cs + pc;
            double acc = 0.0;
#pragma unroll
            for (int cz = -1; cz <= 1; cz++)
#pragma unroll
                for (int cy = -1; cy <= 1; cy++)
#pragma unroll
                    for (int cx = -1; cx <= 1; cx++) {
                        const double w = wt[cx + 1] * wt[cy + 1] * wt[cz + 1];
                        acc = acc + w * s[cx + cy * Lf.py + cz * Lf.pz];
                    }
            o.dst[q * ops.Lc.cs + dp] = acc;
        }
    }
}

}  // namespace crocco
