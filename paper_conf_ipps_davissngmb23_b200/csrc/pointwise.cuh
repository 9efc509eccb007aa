// pointwise.cuh -- primitive recovery, viscous point fluxes, standalone RK update.
// Part of libcrocco (sm_100a, fp64). Formulas restate the paper's method as
// read in DESIGN.md sec. 3 (citations: PAPER.md line numbers); no code is
// shared with oracle/.
#pragma once
#include <type_traits>
#include "common.cuh"

namespace crocco {

// Primitive recovery on every padded point:
// u v w p c sqrt(rho) H T  (perfect gas, Eq. 2 single species).
__global__ void __launch_bounds__(256) k_prims(const double *__restrict__ U, double *__restrict__ P,
                                               Lay L, Phys ph) {
    const int P0 = L.n0 + 2 * G, P1 = L.n1 + 2 * G, P2 = L.n2 + 2 * G;
    const int64_t tid = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
    const int64_t tot = (int64_t)P0 * P1 * P2;
    if (tid >= tot) return;
    const int i = (int)(tid % P0) - G;
    const int64_t r = tid / P0;
    const int j = (int)(r % P1) - G;
    const int k = (int)(r / P1) - G;
    const int64_t p = at(L, i, j, k);
    const double rho = U[p], ru = U[L.cs + p], rv = U[2 * L.cs + p], rw = U[3 * L.cs + p],
                 E = U[4 * L.cs + p];
    const double ir = 1.0 / rho;
    const double u = ru * ir, v = rv * ir, w = rw * ir;
    const double pr = ph.gm1 * (E - 0.5 * (ru * u + rv * v + rw * w));
    const double c = sqrt(ph.gamma * pr * ir);
    P[PU * L.cs + p] = u;
    P[PV * L.cs + p] = v;
    P[PW * L.cs + p] = w;
    P[PP * L.cs + p] = pr;
    P[PC * L.cs + p] = c;
    P[PSR * L.cs + p] = sqrt(rho);
    P[PH * L.cs + p] = (E + pr) * ir;
    P[PT * L.cs + p] = pr * ir / ph.R;
}

// Viscous and heat point fluxes F^_v^d (reading 12) on the
// interior +-2 box: D4 gradients in computational space, chain rule with the
// metrics, Newtonian stress (Stokes), Fourier heat flux, contravariant flux.
// Output FV[4d+q][box index], q = momentum x,y,z, energy.
__device__ __forceinline__ double d4(const double *f, int64_t p, int64_t s) {
    return (8.0 * (f[p + s] - f[p - s]) - (f[p + 2 * s] - f[p - 2 * s])) * (1.0 / 12.0);
}
__device__ __forceinline__ double mu_of_T(const Phys &ph, double T) {
    if (ph.mu_law == 1) {
        const double t = T / ph.T_ref;
        return ph.mu_ref * t * sqrt(t) * (ph.T_ref + ph.S) / (T + ph.S);
    }
    return ph.mu_ref;
}
__global__ void __launch_bounds__(256) k_visc(const double *__restrict__ Pm,
                                              const double *__restrict__ M, double *__restrict__ FV,
                                              Lay L, VLay V, Phys ph) {
    const int64_t tid = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
    const int64_t tot = (int64_t)V.b0 * V.b1 * V.b2;
    if (tid >= tot) return;
    const int i = (int)(tid % V.b0) - 2;
    const int64_t r = tid / V.b0;
    const int j = (int)(r % V.b1) - 2;
    const int k = (int)(r / V.b1) - 2;
    const int64_t p = at(L, i, j, k);
    const int64_t st[3] = {1, L.py, L.pz};
    const int64_t cs = L.cs;
    double gc[4][3];
    const int fidx[4] = {PU, PV, PW, PT};
#pragma unroll
    for (int f = 0; f < 4; f++)
#pragma unroll
        for (int d = 0; d < 3; d++) gc[f][d] = d4(Pm + fidx[f] * cs, p, st[d]);
    const double J = M[p];
    double m[3][3];
#pragma unroll
    for (int d = 0; d < 3; d++)
#pragma unroll
        for (int a = 0; a < 3; a++) m[d][a] = M[(1 + 3 * d + a) * cs + p];
    double gx[4][3];
#pragma unroll
    for (int f = 0; f < 4; f++)
#pragma unroll
        for (int a = 0; a < 3; a++)
            gx[f][a] = J * (m[0][a] * gc[f][0] + m[1][a] * gc[f][1] + m[2][a] * gc[f][2]);
    const double T = Pm[PT * cs + p];
    const double mu = mu_of_T(ph, T);
    const double kap = mu * ph.cp_over_Pr;
    const double div = gx[0][0] + gx[1][1] + gx[2][2];
    double tau[3][3];
#pragma unroll
    for (int a = 0; a < 3; a++)
#pragma unroll
        for (int b = 0; b < 3; b++) tau[a][b] = mu * (gx[a][b] + gx[b][a]);
    const double dterm = (2.0 / 3.0) * mu * div;
    tau[0][0] -= dterm;
    tau[1][1] -= dterm;
    tau[2][2] -= dterm;
    const double vel[3] = {Pm[PU * cs + p], Pm[PV * cs + p], Pm[PW * cs + p]};
    double hb[3];  // u_a tau_ab - q_b, q_b = -kappa dT/dx_b
#pragma unroll
    for (int b = 0; b < 3; b++)
        hb[b] = vel[0] * tau[0][b] + vel[1] * tau[1][b] + vel[2] * tau[2][b] + kap * gx[3][b];
    const int64_t o = vat(V, i, j, k);
#pragma unroll
    for (int d = 0; d < 3; d++) {
#pragma unroll
        for (int a = 0; a < 3; a++)
            FV[(4 * d + a) * V.cs + o] = m[d][0] * tau[a][0] + m[d][1] * tau[a][1] + m[d][2] * tau[a][2];
        FV[(4 * d + 3) * V.cs + o] = m[d][0] * hb[0] + m[d][1] * hb[1] + m[d][2] * hb[2];
    }
}

// Same viscous point fluxes, fused with the primitive recovery: a CTA owns
// VTX (i) x 8 (j) columns of the interior +-2 box and marches a slab of VK
// planes in k.  Each thread keeps u, v, w, T of its own column for planes
// k-2..k+2 in registers (k-derivatives), and only the current plane k (with a
// 2-point i/j halo) is staged in shared memory (i/j-derivatives), double
// buffered so one barrier per plane suffices.
#ifndef CROCCO_VISC_MINB
#define CROCCO_VISC_MINB 1
#endif
#ifndef CROCCO_VISC_PREFETCH
#define CROCCO_VISC_PREFETCH 1  // load the next plane's U / metrics one step ahead (registers)
#endif
#ifndef CROCCO_VISC_ZDIV
#define CROCCO_VISC_ZDIV 1  // 1: D4_zeta of F^_v^zeta folded into k_visc_tiled (own-column queue) -> R
#endif
#ifndef CROCCO_VISC_XDIV
#define CROCCO_VISC_XDIV 1  // 1: D4_xi of F^_v^xi also taken here (tiles overlap by 2-column arms), the xi sweep
                            //    carries no viscous term and F^_v^xi never goes to HBM (requires ZDIV);
                            //    measured -1.0..-1.5 ms per 512^3 stage with 32 x 8 tiles
#endif
#ifndef CROCCO_VISC_TX
// XDIV: 32 x 8 tiles (arms cost 4/28 = 14 %; 16 x 8 with 33 % arms measured slower, 24 x 8 slower still);
// without XDIV: 16 x 8 tiles, two 4-warp CTAs per SM (measured 3 % faster than 32 x 8)
#define CROCCO_VISC_TX (CROCCO_VISC_XDIV ? 32 : 16)
#endif
#ifndef CROCCO_VISC_TY
#define CROCCO_VISC_TY 8
#endif
#ifndef CROCCO_VISC_XSHFL
// XDIV with 32-wide tiles: D4_xi of F^xi by warp shuffles (a warp = one tile row) instead of a
// shared-memory round trip (measured 6.61 -> 6.48 ms per 512^3 launch)
#define CROCCO_VISC_XSHFL (CROCCO_VISC_XDIV && CROCCO_VISC_TX == 32)
#endif
#ifndef CROCCO_VISC_VK
#define CROCCO_VISC_VK (CROCCO_VISC_ZDIV ? 64 : 32)  // slab depth (ZDIV recomputes 4 planes per slab)
#endif
constexpr int VTX = CROCCO_VISC_TX, VTY = CROCCO_VISC_TY, VK = CROCCO_VISC_VK;  // tile and slab
constexpr int VSX = CROCCO_VISC_XDIV ? VTX - 4 : VTX;  // tile stride in i (XDIV: 2-column arms each side)
constexpr int VHX = VTX + 4, VHY = VTY + 4;          // with halo
constexpr int VPL = VHX * VHY;                       // points per staged plane
constexpr int VHALO = VPL - VTX * VTY;               // halo points per plane
constexpr size_t VISC_SMEM = (size_t)2 * 4 * VPL * sizeof(double) +
                              (CROCCO_VISC_XDIV && !CROCCO_VISC_XSHFL ? (size_t)2 * 4 * VTX * VTY * sizeof(double) : 0);
// slab depth of k_visc_tiled (runtime): the longest of CROCCO_VISC_VKMAX / ... / 128 planes that still gives >= 8
// waves of one-CTA-per-SM tiles (each slab recomputes 4 boundary planes; 64 -> 256 measured
// 6.47 -> 6.22 ms per 512^3 launch), else CROCCO_VISC_VK
#ifndef CROCCO_VISC_VKMAX
#define CROCCO_VISC_VKMAX 256  // 512 measured slower at 512^3 (one slab per column: 8.3 waves, tail)
#endif
__host__ __device__ inline int visc_tiles_x(const Lay &L, const VLay &V);
// overlap: the stage runs the ghost-free tiles beside the fill (crocco_rk_stage), so the slab
// depth must leave at least one interior slab, (n2 - 4)/vk >= 2 (visc_interior_tiles)
inline int visc_slab(const Lay &L, const VLay &V, bool overlap = false) {
    const int nz = CROCCO_VISC_ZDIV ? L.n2 : V.b2;
    const int64_t txy = (int64_t)visc_tiles_x(L, V) * ((V.b1 + VTY - 1) / VTY);
    for (int vk = CROCCO_VISC_VKMAX; vk > VK; vk /= 2)
        if (txy * ((nz + vk - 1) / vk) >= 8 * 148 && (!overlap || (L.n2 - 4) / vk >= 2)) return vk;
    return VK;
}
// tiles in i of the viscous box (XDIV: central columns tile the interior [0, n0) with stride VSX)
__host__ __device__ inline int visc_tiles_x(const Lay &L, const VLay &V) {
    return CROCCO_VISC_XDIV ? (L.n0 + VSX - 1) / VSX : (V.b0 + VTX - 1) / VTX;
}

__device__ __forceinline__ void prim4(const double *__restrict__ U, int64_t cs, int64_t p, double gm1,
                                      double iR, double out[4]) {
    const double rho = U[p], ru = U[cs + p], rv = U[2 * cs + p], rw = U[3 * cs + p], E = U[4 * cs + p];
    const double ir = rcp_nr(rho);
    const double u = ru * ir, v = rv * ir, w = rw * ir;
    const double pr = gm1 * fma(-0.5, fma(ru, u, fma(rv, v, rw * w)), E);
    out[0] = u;
    out[1] = v;
    out[2] = w;
    out[3] = pr * ir * iR;
}

// Tiles of k_visc_tiled whose loads stay inside the interior [0, n) in every
// direction (no ghost point read): with ZDIV they may run while the ghost
// exchange is in flight (SURVEY 8(e) overlap).  Half-open ranges of tile indices.
struct VTiles {
    int x0, x1, y0, y1, z0, z1;
};
__host__ __device__ inline VTiles visc_interior_tiles(const Lay &L, int vk) {
    VTiles t;
    // x: loads i0-2 .. i0+VTX+1 with i0 = bx VSX - 2; y likewise (stride VTY); z: planes z0-4 .. z1+3
    t.x0 = (4 + VSX - 1) / VSX;
    t.x1 = (L.n0 - VTX) >= 0 ? (L.n0 - VTX) / VSX + 1 : 0;
    t.y0 = (4 + VTY - 1) / VTY;
    t.y1 = (L.n1 - VTY) >= 0 ? (L.n1 - VTY) / VTY + 1 : 0;
    t.z0 = (4 + vk - 1) / vk;
    t.z1 = (L.n2 - 4) / vk;
    if (t.x1 < t.x0) t.x1 = t.x0;
    if (t.y1 < t.y0) t.y1 = t.y0;
    if (t.z1 < t.z0) t.z1 = t.z0;
    return t;
}

// sel: 0 every tile, 1 the ghost-free interior tiles only, 2 every other tile
__global__ void __launch_bounds__(VTX * VTY, CROCCO_VISC_MINB) k_visc_tiled(const double *__restrict__ U,
                                                          const double *__restrict__ M,
                                                          double *__restrict__ FV, Lay L, VLay V,
                                                          Phys ph, double *__restrict__ R, int64_t rcs,
                                                          int sel, int vk) {
    extern __shared__ double vsm[];  // [buffer 2][value 4][VPL]
    const int tid = threadIdx.x;
    const int tx = tid % VTX, ty = tid / VTX;
    const int tilesx = visc_tiles_x(L, V), tilesy = (V.b1 + VTY - 1) / VTY;
    int b = blockIdx.x;
    int bx, by, bz;
    const VTiles it = visc_interior_tiles(L, vk);
    if (sel == 1) {
        const int nx = it.x1 - it.x0, ny = it.y1 - it.y0;
        bx = it.x0 + b % nx;
        b /= nx;
        by = it.y0 + b % ny;
        bz = it.z0 + b / ny;
    } else if (sel == 2) {
        // the complement of the interior box, enumerated compactly: whole tile planes of the
        // slabs outside [z0, z1), then the xy ring around [x0, x1) x [y0, y1) of the others
        const int nx = it.x1 - it.x0, ny = it.y1 - it.y0, nzi = it.z1 - it.z0;
        const int plane = tilesx * tilesy;
        const int tz = (L.n2 + vk - 1) / vk;
        const int nzs = tz - nzi;
        if (b < nzs * plane) {
            const int sl = b / plane, r = b % plane;
            bz = sl < it.z0 ? sl : sl + nzi;
            bx = r % tilesx;
            by = r / tilesx;
        } else {
            b -= nzs * plane;
            const int ring = plane - nx * ny;
            bz = it.z0 + b / ring;
            int r = b % ring;
            if (r < it.y0 * tilesx) {
                by = r / tilesx;
                bx = r % tilesx;
            } else if ((r -= it.y0 * tilesx) < ny * (tilesx - nx)) {
                by = it.y0 + r / (tilesx - nx);
                const int c = r % (tilesx - nx);
                bx = c < it.x0 ? c : c + nx;
            } else {
                r -= ny * (tilesx - nx);
                by = it.y1 + r / tilesx;
                bx = r % tilesx;
            }
        }
    } else {
        bx = b % tilesx;
        b /= tilesx;
        by = b % tilesy;
        bz = b / tilesy;
    }
    const int i0 = bx * VSX - 2, j0 = by * VTY - 2;      // first output point of the tile
#if CROCCO_VISC_XDIV
    double *fxs = vsm + 2 * 4 * VPL;  // [buffer 2][comp 4][VTX * VTY]: F^xi of the computed columns
    double xq[4] = {0.0, 0.0, 0.0, 0.0};  // D4_xi F^xi of plane k-2 (computed in the previous step)
#if CROCCO_VISC_XSHFL
    static_assert(VTX == 32, "XSHFL needs one tile row per warp");
    double xq1[4] = {0.0, 0.0, 0.0, 0.0};  // D4_xi F^xi of plane k-1
    (void)fxs;
#endif
#endif
#if CROCCO_VISC_ZDIV
    // slab of interior output planes [z0, z1); gradients / point fluxes on planes z0-2 .. z1+1
    const int z0 = bz * vk, z1 = min(z0 + vk, L.n2);
    const int k0 = z0 - 2, k1 = z1 + 2;
    double zq[5][4];  // F^zeta of the own column, planes k-4 .. k
#pragma unroll
    for (int o = 0; o < 5; o++)
#pragma unroll
        for (int q = 0; q < 4; q++) zq[o][q] = 0.0;
#else
    const int k0 = bz * vk - 2, k1 = min(k0 + vk, V.b2 - 2);
#endif
    const double iR = 1.0 / ph.R;
    // own column (clamped into the padded box for the idle threads of edge tiles)
    const int i = i0 + tx, j = j0 + ty;
    const bool own = i < V.b0 - 2 && j < V.b1 - 2;
    // the column whose outputs (F^eta, R) this thread writes: XDIV -> central columns only
    const bool central = CROCCO_VISC_XDIV ? (tx >= 2 && tx < VTX - 2 && i < L.n0) : true;
    const int gi = min(i, L.n0 + G - 1), gj = min(j, L.n1 + G - 1);
    // halo point handled by this thread (tid < VHALO): rows j0-2, j0-1, j0+8, j0+9 (36 each),
    // then columns i0-2, i0-1, i0+32, i0+33 of rows j0..j0+7
    int hx = 0, hy = 0;
    if (tid < 4 * VHX) {
        hx = tid % VHX;
        const int r = tid / VHX;
        hy = r < 2 ? r : VTY + r;        // 0,1 | 10,11
    } else if (tid < VHALO) {
        const int t = tid - 4 * VHX;      // 0..31
        const int c = t % 4;
        hy = 2 + t / 4;
        hx = c < 2 ? c : VTX + c;         // 0,1 | VTX+2, VTX+3
    }
    const int hgi = min(i0 - 2 + hx, L.n0 + G - 1), hgj = min(j0 - 2 + hy, L.n1 + G - 1);
    const int hidx = hy * VHX + hx;
    const int oidx = (ty + 2) * VHX + (tx + 2);

    double win[4][5];  // own u v w T at planes k-2 .. k+2
    for (int o = 0; o < 4; o++) {
        double q[4];
        prim4(U, L.cs, at(L, gi, gj, k0 - 2 + o), ph.gm1, iR, q);
#pragma unroll
        for (int f = 0; f < 4; f++) win[f][o + 1] = q[f];  // shifted into 0..3 by the first step
    }
#if CROCCO_VISC_PREFETCH
    // global operands of the step, loaded one step ahead: own U at plane k+2,
    // halo U at plane k, own metrics at plane k
    double cO[5], cH[5], cM[10];
    auto ld_own = [&](int kk, double o5[5]) {
        const int64_t q = at(L, gi, gj, kk);
#pragma unroll
        for (int c = 0; c < 5; c++) o5[c] = U[c * L.cs + q];
    };
    auto ld_halo = [&](int kk, double o5[5]) {
        if (tid < VHALO) {
            const int64_t q = at(L, hgi, hgj, kk);
#pragma unroll
            for (int c = 0; c < 5; c++) o5[c] = U[c * L.cs + q];
        }
    };
    auto ld_met = [&](int kk, double o10[10]) {
        const int64_t q = at(L, gi, gj, kk);
#pragma unroll
        for (int c = 0; c < 10; c++) o10[c] = M[c * L.cs + q];
    };
    auto prim_of = [&](const double u5[5], double q[4]) {
        const double ir = rcp_nr(u5[0]);
        const double u = u5[1] * ir, v = u5[2] * ir, w = u5[3] * ir;
        const double pr = ph.gm1 * fma(-0.5, fma(u5[1], u, fma(u5[2], v, u5[3] * w)), u5[4]);
        q[0] = u;
        q[1] = v;
        q[2] = w;
        q[3] = pr * ir * iR;
    };
    ld_own(k0 + 2, cO);
    ld_halo(k0, cH);
    ld_met(k0, cM);
#if CROCCO_VISC_PREFETCH >= 2
    // distance 2: the operands of plane k+1 are already in flight when plane k starts
    double mO[5], mH[5], mM[10];
    {
        const int k1n = min(k0 + 1, k1 - 1);
        ld_own(k1n + 2, mO);
        ld_halo(k1n, mH);
        ld_met(k1n, mM);
    }
#endif
#endif
    for (int k = k0; k < k1; k++) {
#if CROCCO_VISC_PREFETCH
        double nO[5], nH[5], nM[10];
        const int kn = min(k + CROCCO_VISC_PREFETCH, k1 - 1);  // clamp: the last steps reload
        ld_own(kn + 2, nO);
        ld_halo(kn, nH);
        ld_met(kn, nM);
        {
            double q[4];
            prim_of(cO, q);
#pragma unroll
            for (int f = 0; f < 4; f++) {
#pragma unroll
                for (int o = 0; o < 4; o++) win[f][o] = win[f][o + 1];
                win[f][4] = q[f];
            }
        }
        double *pl = vsm + (k & 1) * 4 * VPL;
#pragma unroll
        for (int f = 0; f < 4; f++) pl[f * VPL + oidx] = win[f][2];
        if (tid < VHALO) {
            double q[4];
            prim_of(cH, q);
#pragma unroll
            for (int f = 0; f < 4; f++) pl[f * VPL + hidx] = q[f];
        }
#else
        {   // own primitives of plane k+2, shift the window
            double q[4];
            prim4(U, L.cs, at(L, gi, gj, k + 2), ph.gm1, iR, q);
#pragma unroll
            for (int f = 0; f < 4; f++) {
#pragma unroll
                for (int o = 0; o < 4; o++) win[f][o] = win[f][o + 1];
                win[f][4] = q[f];
            }
        }
        double *pl = vsm + (k & 1) * 4 * VPL;
#pragma unroll
        for (int f = 0; f < 4; f++) pl[f * VPL + oidx] = win[f][2];
        if (tid < VHALO) {
            double q[4];
            prim4(U, L.cs, at(L, hgi, hgj, k), ph.gm1, iR, q);
#pragma unroll
            for (int f = 0; f < 4; f++) pl[f * VPL + hidx] = q[f];
        }
#endif
        __syncthreads();
#if CROCCO_VISC_XDIV
        double xn[4] = {0.0, 0.0, 0.0, 0.0};  // D4_xi F^xi of plane k-1 (staged in the previous step)
        double fxr[4] = {0.0, 0.0, 0.0, 0.0}; // XSHFL: F^xi of this column at plane k
        if (!CROCCO_VISC_XSHFL && central && k > k0) {
            const double *fb = fxs + ((k - 1) & 1) * 4 * VTX * VTY + ty * VTX + tx;
#pragma unroll
            for (int q = 0; q < 4; q++) {
                const double *c = fb + q * VTX * VTY;
                xn[q] = fma(8.0, c[1] - c[-1], -(c[2] - c[-2])) * (1.0 / 12.0);
            }
        }
#endif
        if (own) {
            double gc[4][3];
#pragma unroll
            for (int f = 0; f < 4; f++) {
                const double *c = pl + f * VPL + oidx;
                gc[f][0] = fma(8.0, c[1] - c[-1], -(c[2] - c[-2])) * (1.0 / 12.0);
                gc[f][1] = fma(8.0, c[VHX] - c[-VHX], -(c[2 * VHX] - c[-2 * VHX])) * (1.0 / 12.0);
                gc[f][2] = fma(8.0, win[f][3] - win[f][1], -(win[f][4] - win[f][0])) * (1.0 / 12.0);
            }
#if CROCCO_VISC_PREFETCH
            const double J = cM[0];
            double m[3][3];
#pragma unroll
            for (int d = 0; d < 3; d++)
#pragma unroll
                for (int a = 0; a < 3; a++) m[d][a] = cM[1 + 3 * d + a];
#else
            const int64_t p = at(L, i, j, k);
            const double J = M[p];
            double m[3][3];
#pragma unroll
            for (int d = 0; d < 3; d++)
#pragma unroll
                for (int a = 0; a < 3; a++) m[d][a] = M[(1 + 3 * d + a) * L.cs + p];
#endif
            double gx[4][3];
#pragma unroll
            for (int f = 0; f < 4; f++)
#pragma unroll
                for (int a = 0; a < 3; a++)
                    gx[f][a] = J * fma(m[0][a], gc[f][0], fma(m[1][a], gc[f][1], m[2][a] * gc[f][2]));
            const double T = win[3][2];
            const double mu = mu_of_T(ph, T);
            const double kap = mu * ph.cp_over_Pr;
            const double div = gx[0][0] + gx[1][1] + gx[2][2];
            double tau[3][3];
#pragma unroll
            for (int a = 0; a < 3; a++)
#pragma unroll
                for (int bb = 0; bb < 3; bb++) tau[a][bb] = mu * (gx[a][bb] + gx[bb][a]);
            const double dterm = (2.0 / 3.0) * mu * div;
            tau[0][0] -= dterm;
            tau[1][1] -= dterm;
            tau[2][2] -= dterm;
            const double vel[3] = {win[0][2], win[1][2], win[2][2]};
            double hb[3];
#pragma unroll
            for (int bb = 0; bb < 3; bb++)
                hb[bb] = fma(vel[0], tau[0][bb], fma(vel[1], tau[1][bb], fma(vel[2], tau[2][bb], kap * gx[3][bb])));
            const int64_t o = vat(V, i, j, k);
#if CROCCO_VISC_ZDIV
            // F^xi, F^eta of the interior planes to HBM (the xi / eta sweeps difference them);
            // F^zeta stays in the own column's queue and is differenced here (D4_zeta)
#if CROCCO_VISC_XDIV
#if CROCCO_VISC_XSHFL
#pragma unroll
            for (int a = 0; a < 3; a++)
                fxr[a] = fma(m[0][0], tau[a][0], fma(m[0][1], tau[a][1], m[0][2] * tau[a][2]));
            fxr[3] = fma(m[0][0], hb[0], fma(m[0][1], hb[1], m[0][2] * hb[2]));
#else
            {   // F^xi of this column for the xi-divergence of the next step (shared memory only)
                double *fb = fxs + (k & 1) * 4 * VTX * VTY + ty * VTX + tx;
#pragma unroll
                for (int a = 0; a < 3; a++)
                    fb[a * VTX * VTY] = fma(m[0][0], tau[a][0], fma(m[0][1], tau[a][1], m[0][2] * tau[a][2]));
                fb[3 * VTX * VTY] = fma(m[0][0], hb[0], fma(m[0][1], hb[1], m[0][2] * hb[2]));
            }
#endif
            if (k >= z0 && k < z1 && central) {  // F^eta only (the eta sweep differences it)
#pragma unroll
                for (int a = 0; a < 3; a++)
                    FV[a * V.cs + o] = fma(m[1][0], tau[a][0], fma(m[1][1], tau[a][1], m[1][2] * tau[a][2]));
                FV[3 * V.cs + o] = fma(m[1][0], hb[0], fma(m[1][1], hb[1], m[1][2] * hb[2]));
            }
#else
            if (k >= z0 && k < z1) {
#pragma unroll
                for (int d = 0; d < 2; d++) {
#pragma unroll
                    for (int a = 0; a < 3; a++)
                        FV[(4 * d + a) * V.cs + o] = fma(m[d][0], tau[a][0], fma(m[d][1], tau[a][1], m[d][2] * tau[a][2]));
                    FV[(4 * d + 3) * V.cs + o] = fma(m[d][0], hb[0], fma(m[d][1], hb[1], m[d][2] * hb[2]));
                }
            }
#endif
#pragma unroll
            for (int oq = 0; oq < 4; oq++)
#pragma unroll
                for (int q = 0; q < 4; q++) zq[oq][q] = zq[oq + 1][q];
#pragma unroll
            for (int a = 0; a < 3; a++) zq[4][a] = fma(m[2][0], tau[a][0], fma(m[2][1], tau[a][1], m[2][2] * tau[a][2]));
            zq[4][3] = fma(m[2][0], hb[0], fma(m[2][1], hb[1], m[2][2] * hb[2]));
            if (k - 2 >= z0 && central && i >= 0 && i < L.n0 && j >= 0 && j < L.n1) {
                const int64_t r = (int64_t)i + (int64_t)L.n0 * (j + (int64_t)L.n1 * (k - 2));
#pragma unroll
                for (int q = 0; q < 4; q++) {
                    const double zd = fma(8.0, zq[3][q] - zq[1][q], -(zq[4][q] - zq[0][q])) * (1.0 / 12.0);
#if CROCCO_VISC_XDIV
                    R[(1 + q) * rcs + r] = zd + xq[q];
#else
                    R[(1 + q) * rcs + r] = zd;
#endif
                }
            }
#else
#pragma unroll
            for (int d = 0; d < 3; d++) {
#pragma unroll
                for (int a = 0; a < 3; a++)
                    FV[(4 * d + a) * V.cs + o] = fma(m[d][0], tau[a][0], fma(m[d][1], tau[a][1], m[d][2] * tau[a][2]));
                FV[(4 * d + 3) * V.cs + o] = fma(m[d][0], hb[0], fma(m[d][1], hb[1], m[d][2] * hb[2]));
            }
#endif
        }
#if CROCCO_VISC_XDIV
#if CROCCO_VISC_XSHFL
        // D4_xi of plane k from the row's lanes (every lane of the warp takes part)
#pragma unroll
        for (int q = 0; q < 4; q++) {
            const double p1 = __shfl_down_sync(0xffffffffu, fxr[q], 1), m1 = __shfl_up_sync(0xffffffffu, fxr[q], 1);
            const double p2 = __shfl_down_sync(0xffffffffu, fxr[q], 2), m2 = __shfl_up_sync(0xffffffffu, fxr[q], 2);
            xn[q] = fma(8.0, p1 - m1, -(p2 - m2)) * (1.0 / 12.0);
        }
#pragma unroll
        for (int q = 0; q < 4; q++) {  // planes k-1 -> k-2, k -> k-1
            xq[q] = xq1[q];
            xq1[q] = xn[q];
        }
#else
#pragma unroll
        for (int q = 0; q < 4; q++) xq[q] = xn[q];  // plane k-1 -> written with plane k-1's zeta term next step
#endif
#endif
#if CROCCO_VISC_PREFETCH >= 2
#pragma unroll
        for (int c = 0; c < 5; c++) {
            cO[c] = mO[c];
            cH[c] = mH[c];
            mO[c] = nO[c];
            mH[c] = nH[c];
        }
#pragma unroll
        for (int c = 0; c < 10; c++) {
            cM[c] = mM[c];
            mM[c] = nM[c];
        }
#elif CROCCO_VISC_PREFETCH
#pragma unroll
        for (int c = 0; c < 5; c++) {
            cO[c] = nO[c];
            cH[c] = nH[c];
        }
#pragma unroll
        for (int c = 0; c < 10; c++) cM[c] = nM[c];
#endif
    }
}

// ---------------------------------------------------------------------------
// Viscous divergence (Viscous; reading 12), fused end to end:
//   R_visc(i,j,k) = sum_d D4_d F^_v^d   (momentum x, y, z and energy)
// with the point fluxes F^_v^d of the same D4-gradient / Stokes / Fourier
// construction as k_visc_tiled, evaluated where the divergence needs them and
// never stored to HBM.  A CTA owns DTX (i) x DTY (j) interior columns and
// marches a slab of DK output planes in k; per gradient plane g:
//   phase 1: u, v, w, T of plane g+2 on the tile + 2-point halo (5-plane ring
//            in shared memory) and of plane g on the 4-point i / j arms;
//   phase 2: full gradients at plane g on the own points and on the 2-point
//            i-arm / j-arm points; F^_v^xi (own + i-arm) and F^_v^eta (own +
//            j-arm) to shared memory, F^_v^zeta of the own column to a 5-plane
//            register queue;
//   phase 3: D4_xi + D4_eta of plane g (3-plane register queue); plane g-2 is
//            complete once D4_zeta of the queue is added -> R comps 1..4.
// The point flux of a point is computed by one function with explicitly
// rounded operations, so a point evaluated as a halo point of one tile equals
// the same point evaluated as an own point of its neighbour tile bit for bit
// (decomposition invariance).
// ---------------------------------------------------------------------------
#ifndef CROCCO_VISC_DIV
#define CROCCO_VISC_DIV 0  // 1: fused viscous divergence (k_visc_div, measured slower: smem-bound); 0: point fluxes
#endif
#ifndef CROCCO_VDIV_MINB
#define CROCCO_VDIV_MINB 2
#endif
#ifndef CROCCO_VDIV_TY
#define CROCCO_VDIV_TY 8
#endif
#ifndef CROCCO_VDIV_TX
#define CROCCO_VDIV_TX 16
#endif
#ifndef CROCCO_VDIV_K
#define CROCCO_VDIV_K 64
#endif
constexpr int DTX = CROCCO_VDIV_TX, DTY = CROCCO_VDIV_TY, DK = CROCCO_VDIV_K;  // tile (i x j), slab (k)
constexpr int DNT = DTX * DTY;                  // threads (one own column each)
constexpr int DBW = DTX + 4;                    // ring rows: tile + 2-point halo
constexpr int DNB = DBW * (DTY + 4);            // ring points per plane
constexpr int DNA = 4 * DTY + 4 * DTX;          // 4-point arm points (current plane only)
constexpr int DXW = DTX + 4;                    // F^xi rows: own + i-arm
constexpr int DYH = DTY + 4;                    // F^eta columns: own + j-arm
constexpr int DNX = DXW * DTY, DNY = DTX * DYH;
constexpr size_t VDIV_SMEM = (size_t)(5 * 4 * DNB + 4 * DNA + 5 * 4 * DNT + 4 * DNX + 4 * DNY) * sizeof(double);

// stress tensor / energy flux of a point from its computational-space gradient
// gc[f][d] = D4_d f (f = u, v, w, T), metrics Mp[0..9] = (J, m^xi, m^eta, m^zeta)
// and its u, v, w, T: returns tau (symmetric, 6) and hb = u_a tau_ab - q_b.
// Every operation is an explicit rounding (no contraction freedom).
__device__ __forceinline__ void visc_point(const double gc[4][3], const double Mp[10], double u, double v,
                                           double w, double T, const Phys &ph, double tau[6], double hb[3]) {
    double gx[4][3];
#pragma unroll
    for (int f = 0; f < 4; f++)
#pragma unroll
        for (int a = 0; a < 3; a++)
            gx[f][a] = __dmul_rn(Mp[0], fma(Mp[1 + a], gc[f][0], fma(Mp[4 + a], gc[f][1], __dmul_rn(Mp[7 + a], gc[f][2]))));
    double mu = ph.mu_ref;
    if (ph.mu_law == 1) {
        const double t = __dmul_rn(T, ph.iT_ref);
        mu = __dmul_rn(__dmul_rn(__dmul_rn(ph.mu_ref, t), sqrt_nr(t)), div_nr(ph.T_ref + ph.S, __dadd_rn(T, ph.S)));
    }
    const double kap = __dmul_rn(mu, ph.cp_over_Pr);
    const double dv = __dmul_rn(__dmul_rn(2.0 / 3.0, mu), __dadd_rn(__dadd_rn(gx[0][0], gx[1][1]), gx[2][2]));
    const double m2 = __dmul_rn(2.0, mu);
    tau[0] = __dsub_rn(__dmul_rn(m2, gx[0][0]), dv);                 // xx
    tau[1] = __dsub_rn(__dmul_rn(m2, gx[1][1]), dv);                 // yy
    tau[2] = __dsub_rn(__dmul_rn(m2, gx[2][2]), dv);                 // zz
    tau[3] = __dmul_rn(mu, __dadd_rn(gx[0][1], gx[1][0]));           // xy
    tau[4] = __dmul_rn(mu, __dadd_rn(gx[0][2], gx[2][0]));           // xz
    tau[5] = __dmul_rn(mu, __dadd_rn(gx[1][2], gx[2][1]));           // yz
    hb[0] = fma(u, tau[0], fma(v, tau[3], fma(w, tau[4], __dmul_rn(kap, gx[3][0]))));
    hb[1] = fma(u, tau[3], fma(v, tau[1], fma(w, tau[5], __dmul_rn(kap, gx[3][1]))));
    hb[2] = fma(u, tau[4], fma(v, tau[5], fma(w, tau[2], __dmul_rn(kap, gx[3][2]))));
}
// F^_v^d = m^d_b (tau_xb, tau_yb, tau_zb, hb_b), m^d = Mp[1+3d .. 3+3d]
__device__ __forceinline__ void visc_proj(const double *md, const double tau[6], const double hb[3],
                                          double out[4]) {
    out[0] = fma(md[0], tau[0], fma(md[1], tau[3], __dmul_rn(md[2], tau[4])));
    out[1] = fma(md[0], tau[3], fma(md[1], tau[1], __dmul_rn(md[2], tau[5])));
    out[2] = fma(md[0], tau[4], fma(md[1], tau[5], __dmul_rn(md[2], tau[2])));
    out[3] = fma(md[0], hb[0], fma(md[1], hb[1], __dmul_rn(md[2], hb[2])));
}
__device__ __forceinline__ double d4v(double fm2, double fm1, double fp1, double fp2) {
    return __dmul_rn(fma(8.0, __dsub_rn(fp1, fm1), -__dsub_rn(fp2, fm2)), 1.0 / 12.0);
}

__global__ void __launch_bounds__(DNT, CROCCO_VDIV_MINB) k_visc_div(const double *__restrict__ U,
                                                                   const double *__restrict__ M,
                                                                   double *__restrict__ R, int64_t rcs,
                                                                   Lay L, Phys ph) {
    extern __shared__ double dsm[];
    double *ring = dsm;                   // u v w T, tile + 2 halo: [plane mod 5][4][DNB]
    double *arms = ring + 5 * 4 * DNB;    // u v w T of the 4-point arms, current plane: [4][DNA]
    double *fz = arms + 4 * DNA;          // F^zeta of the own columns: [plane mod 5][4][DNT]
    double *fx = fz + 5 * 4 * DNT;        // F^xi  [4][DNX], index (a+2) + DXW b
    double *fy = fx + 4 * DNX;            // F^eta [4][DNY], index a + DTX (b+2)
    constexpr int NSB = (DNB + DNT - 1) / DNT;  // ring points per thread and plane
    static_assert(DNA <= DNT, "one arm point per thread");
    const int tid = threadIdx.x;
    const int tilesx = (L.n0 + DTX - 1) / DTX, tilesy = (L.n1 + DTY - 1) / DTY;
    int bb = blockIdx.x;
    const int bx = bb % tilesx;
    bb /= tilesx;
    const int by = bb % tilesy;
    const int bz = bb / tilesy;
    const int i0 = bx * DTX, j0 = by * DTY, k0 = bz * DK, k1 = min(k0 + DK, L.n2);
    const double iR = 1.0 / ph.R;
    auto ci = [&](int a) { return min(max(i0 + a, -G), L.n0 + G - 1); };
    auto cj = [&](int b) { return min(max(j0 + b, -G), L.n1 + G - 1); };
    auto slot = [](int k) { return ((k + 10) % 5); };
    auto rb = [](int a, int b) { return (a + 2) + DBW * (b + 2); };
    // arm point (a, b) outside the ring rectangle -> index in `arms`
    auto ai = [](int a, int b) {
        return (b >= 0 && b < DTY) ? (a < 0 ? a + 4 : a - DTX) + 4 * b
                                   : 4 * DTY + a + DTX * (b < 0 ? b + 4 : b - DTY);
    };
    // this thread's arm points (tid < DNA): the 4-point arm point it stages and the
    // 2-point arm point whose gradient / flux it evaluates; xarm: along i (F^xi) else j (F^eta)
    const bool xarm = tid < 4 * DTY;
    int sa, sb, ga, gb;
    if (xarm) {
        const int c = tid & 3;
        sa = c < 2 ? c - 4 : DTX + c;
        ga = c < 2 ? c - 2 : DTX + c - 2;
        sb = gb = tid >> 2;
    } else {
        const int u = tid - 4 * DTY, r = u / DTX;
        sa = ga = u % DTX;
        sb = r < 2 ? r - 4 : DTY + r;
        gb = r < 2 ? r - 2 : DTY + r - 2;
    }
    const bool arm = tid < DNA;
    const int oa = tid % DTX, ob = tid / DTX;  // own column
    const bool own = i0 + oa < L.n0 && j0 + ob < L.n1;

    auto ld5 = [&](int a, int b, int k, double o[5]) {
        const int64_t p = at(L, ci(a), cj(b), k);
#pragma unroll
        for (int c = 0; c < 5; c++) o[c] = U[c * L.cs + p];
    };
    auto ld10 = [&](int a, int b, int k, double o[10]) {
        const int64_t p = at(L, ci(a), cj(b), k);
#pragma unroll
        for (int c = 0; c < 10; c++) o[c] = M[c * L.cs + p];
    };
    // u, v, w, T of a conserved state into d[0], d[st], d[2 st], d[3 st]
    auto put = [&](const double u5[5], double *d, int st) {
        const double ir = rcp_nr(u5[0]);
        const double u = __dmul_rn(u5[1], ir), v = __dmul_rn(u5[2], ir), w = __dmul_rn(u5[3], ir);
        const double pr = __dmul_rn(ph.gm1, fma(-0.5, fma(u5[1], u, fma(u5[2], v, __dmul_rn(u5[3], w))), u5[4]));
        d[0] = u;
        d[st] = v;
        d[2 * st] = w;
        d[3 * st] = __dmul_rn(__dmul_rn(pr, ir), iR);
    };
    // gradient of u, v, w, T at (a, b) of plane k -> tau, hb.  ARM: the point is a
    // 2-point arm point whose i- or j-stencil reaches into the 4-point arms.
    auto grad = [&](auto armc, int a, int b, int k, const double Mp[10], double tau[6], double hb[3]) {
        constexpr bool ARM = std::decay_t<decltype(armc)>::value;
        const double *pl = ring + slot(k) * 4 * DNB;
        const int ix = rb(a, b);
        const double *cm1 = ring + slot(k - 1) * 4 * DNB + ix, *cp1 = ring + slot(k + 1) * 4 * DNB + ix;
        const double *cm2 = ring + slot(k - 2) * 4 * DNB + ix, *cp2 = ring + slot(k + 2) * 4 * DNB + ix;
        auto cur = [&](int f, int a2, int b2) -> double {
            if (ARM && (a2 < -2 || a2 > DTX + 1 || b2 < -2 || b2 > DTY + 1)) return arms[f * DNA + ai(a2, b2)];
            return pl[f * DNB + rb(a2, b2)];
        };
        double gc[4][3];
#pragma unroll
        for (int f = 0; f < 4; f++) {
            gc[f][0] = d4v(cur(f, a - 2, b), cur(f, a - 1, b), cur(f, a + 1, b), cur(f, a + 2, b));
            gc[f][1] = d4v(cur(f, a, b - 2), cur(f, a, b - 1), cur(f, a, b + 1), cur(f, a, b + 2));
            gc[f][2] = d4v(cm2[f * DNB], cm1[f * DNB], cp1[f * DNB], cp2[f * DNB]);
        }
        const double *c0 = pl + ix;
        visc_point(gc, Mp, c0[0], c0[DNB], c0[2 * DNB], c0[3 * DNB], ph, tau, hb);
    };

    double xq[3][4];  // D4_xi F^xi + D4_eta F^eta of the own column, planes g-2 .. g
#pragma unroll
    for (int o = 0; o < 3; o++)
#pragma unroll
        for (int q = 0; q < 4; q++) xq[o][q] = 0.0;

    // prologue: ring planes k0-4 .. k0-1
    for (int t = tid; t < 4 * DNB; t += DNT) {
        const int k = k0 - 4 + t / DNB, r = t % DNB;
        double u5[5];
        ld5(r % DBW - 2, r / DBW - 2, k, u5);
        put(u5, ring + slot(k) * 4 * DNB + r, DNB);
    }
    // global operands of step g, loaded one step ahead: ring points of plane g+2, the
    // arm point of plane g, the metrics of the own and the arm gradient point
    double nU[NSB + 1][5], nM[2][10];
    auto prefetch = [&](int g) {
        const bool xy = g >= k0 && g < k1;
#pragma unroll
        for (int s2 = 0; s2 < NSB; s2++) {
            const int t = tid + s2 * DNT;
            if (t < DNB) ld5(t % DBW - 2, t / DBW - 2, g + 2, nU[s2]);
        }
        if (xy && arm) ld5(sa, sb, g, nU[NSB]);
        ld10(oa, ob, g, nM[0]);
        if (xy && arm) ld10(ga, gb, g, nM[1]);
    };
    prefetch(k0 - 2);
    for (int g = k0 - 2; g <= k1 + 1; g++) {
        const bool xy = g >= k0 && g < k1;  // F^xi / F^eta of plane g needed
        double cU[NSB + 1][5], cM[2][10];
#pragma unroll
        for (int s2 = 0; s2 <= NSB; s2++)
#pragma unroll
            for (int c = 0; c < 5; c++) cU[s2][c] = nU[s2][c];
#pragma unroll
        for (int s2 = 0; s2 < 2; s2++)
#pragma unroll
            for (int c = 0; c < 10; c++) cM[s2][c] = nM[s2][c];
        if (g < k1 + 1) prefetch(g + 1);
        // phase 1
#pragma unroll
        for (int s2 = 0; s2 < NSB; s2++) {
            const int t = tid + s2 * DNT;
            if (t < DNB) put(cU[s2], ring + slot(g + 2) * 4 * DNB + t, DNB);
        }
        if (xy && arm) put(cU[NSB], arms + tid, DNA);
        __syncthreads();
        // phase 2: own point
        {
            double tau[6], hb[3], f[4];
            grad(std::false_type{}, oa, ob, g, cM[0], tau, hb);
            visc_proj(cM[0] + 7, tau, hb, f);
#pragma unroll
            for (int q = 0; q < 4; q++) fz[(slot(g) * 4 + q) * DNT + tid] = f[q];
            if (xy) {
                visc_proj(cM[0] + 1, tau, hb, f);
#pragma unroll
                for (int q = 0; q < 4; q++) fx[q * DNX + (oa + 2) + DXW * ob] = f[q];
                visc_proj(cM[0] + 4, tau, hb, f);
#pragma unroll
                for (int q = 0; q < 4; q++) fy[q * DNY + oa + DTX * (ob + 2)] = f[q];
            }
        }
        // phase 2: arm point (2-point halo of F^xi along i, of F^eta along j)
        if (xy && arm) {
            double tau[6], hb[3], f[4];
            grad(std::true_type{}, ga, gb, g, cM[1], tau, hb);
            visc_proj(xarm ? cM[1] + 1 : cM[1] + 4, tau, hb, f);
            if (xarm) {
#pragma unroll
                for (int q = 0; q < 4; q++) fx[q * DNX + (ga + 2) + DXW * gb] = f[q];
            } else {
#pragma unroll
                for (int q = 0; q < 4; q++) fy[q * DNY + ga + DTX * (gb + 2)] = f[q];
            }
        }
        __syncthreads();
        // phase 3
#pragma unroll
        for (int o = 0; o < 2; o++)
#pragma unroll
            for (int q = 0; q < 4; q++) xq[o][q] = xq[o + 1][q];
        if (xy) {
#pragma unroll
            for (int q = 0; q < 4; q++) {
                const double *x = fx + q * DNX + (oa + 2) + DXW * ob;
                const double *y = fy + q * DNY + oa + DTX * (ob + 2);
                xq[2][q] = __dadd_rn(d4v(x[-2], x[-1], x[1], x[2]), d4v(y[-2 * DTX], y[-DTX], y[DTX], y[2 * DTX]));
            }
        }
        const int k = g - 2;
        if (k >= k0 && own) {
            const int64_t r = (int64_t)(i0 + oa) + (int64_t)L.n0 * ((j0 + ob) + (int64_t)L.n1 * k);
#pragma unroll
            for (int q = 0; q < 4; q++) {
                const double *z = fz + q * DNT + tid;
                const double zd = d4v(z[slot(k - 2) * 4 * DNT], z[slot(k - 1) * 4 * DNT], z[slot(k + 1) * 4 * DNT],
                                      z[slot(k + 2) * 4 * DNT]);
                R[(1 + q) * rcs + r] = __dadd_rn(xq[0][q], zd);
            }
        }
    }
}

// ComputeDt (Eq. 3, 95 Alg. 1 l.9, 131, 169):
// lambda_i = J_i sum_d (|m^d_i . u_i| + c_i |m^d_i|) on interior points, maximum
// over the block by warp shuffles + shared memory, over blocks/launches by
// atomicMax on the 64-bit pattern (non-negative doubles order like their bit
// patterns, so the result is exact and independent of the reduction order).
__global__ void __launch_bounds__(256) k_cfl(const double *__restrict__ U, const double *__restrict__ M,
                                             Lay L, Phys ph, unsigned long long *__restrict__ out) {
    __shared__ double red[8];
    const int64_t tot = (int64_t)L.n0 * L.n1 * L.n2;
    double lmax = 0.0;
    for (int64_t t = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; t < tot;
         t += (int64_t)gridDim.x * blockDim.x) {
        const int i = (int)(t % L.n0);
        const int64_t r = t / L.n0;
        const int j = (int)(r % L.n1), k = (int)(r / L.n1);
        const int64_t p = at(L, i, j, k);
        const double rho = U[p];
        const double ir = 1.0 / rho;
        const double u = U[L.cs + p] * ir, v = U[2 * L.cs + p] * ir, w = U[3 * L.cs + p] * ir;
        const double pr = ph.gm1 * (U[4 * L.cs + p] - 0.5 * rho * fma(u, u, fma(v, v, w * w)));
        const double c = sqrt(ph.gamma * pr * ir);
        double sum = 0.0;
#pragma unroll
        for (int d = 0; d < 3; d++) {
            const double mx = M[(1 + 3 * d) * L.cs + p], my = M[(2 + 3 * d) * L.cs + p],
                         mz = M[(3 + 3 * d) * L.cs + p];
            sum += fabs(fma(mx, u, fma(my, v, mz * w))) + c * sqrt(fma(mx, mx, fma(my, my, mz * mz)));
        }
        // a non-finite local radius (NaN state, negative pressure -> NaN c) poisons the maximum
        // (+inf) instead of being dropped by fmax; the host then reports the blow-up
        const double lp = M[p] * sum;
        lmax = lp <= 1.7976931348623157e308 ? fmax(lmax, lp) : __longlong_as_double(0x7ff0000000000000LL);
    }
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) lmax = fmax(lmax, __shfl_xor_sync(0xffffffffu, lmax, o));
    if ((threadIdx.x & 31) == 0) red[threadIdx.x >> 5] = lmax;
    __syncthreads();
    if (threadIdx.x == 0) {
        double m = red[0];
        for (int w = 1; w < (int)(blockDim.x >> 5); w++) m = fmax(m, red[w]);
        atomicMax(out, (unsigned long long)__double_as_longlong(m));
    }
}

// Update alone, from a materialised rhs (crocco_rk_update).
// state check (SURVEY sec. 5 failure detection, a test / bench utility): count interior
// points with a non-finite component, rho <= 0 or p <= 0
__global__ void __launch_bounds__(256) k_check_state(const double *__restrict__ U, Lay L, const Phys ph,
                                                     unsigned long long *bad) {
    const int64_t tot = (int64_t)L.n0 * L.n1 * L.n2;
    unsigned cnt = 0;
    for (int64_t t = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; t < tot; t += (int64_t)gridDim.x * blockDim.x) {
        const int i = (int)(t % L.n0);
        const int64_t r = t / L.n0;
        const int64_t p = at(L, i, (int)(r % L.n1), (int)(r / L.n1));
        const double rho = U[p], mx = U[L.cs + p], my = U[2 * L.cs + p], mz = U[3 * L.cs + p], E = U[4 * L.cs + p];
        const double pr = ph.gm1 * (E - 0.5 * (mx * mx + my * my + mz * mz) / rho);
        const bool ok = isfinite(rho) && isfinite(mx) && isfinite(my) && isfinite(mz) && isfinite(E) &&
                        rho > 0.0 && pr > 0.0;
        cnt += ok ? 0u : 1u;
    }
    for (int o = 16; o > 0; o >>= 1) cnt += __shfl_down_sync(0xffffffffu, cnt, o);
    if ((threadIdx.x & 31) == 0 && cnt) atomicAdd(bad, (unsigned long long)cnt);
}

__global__ void __launch_bounds__(256) k_update(const double *__restrict__ Uin,
                                                double *__restrict__ Uout, double *__restrict__ dU,
                                                const double *__restrict__ rhs, Lay L, int stage,
                                                double A, double B, double dt) {
    const int i = blockIdx.x * blockDim.x + threadIdx.x;
    const int j = blockIdx.y;
    const int k = blockIdx.z;
    if (i >= L.n0) return;
    const int64_t p = at(L, i, j, k);
#pragma unroll
    for (int c = 0; c < 5; c++) {
        const int64_t q = c * L.cs + p;
        const double du = (stage == 0) ? dt * rhs[q] : A * dU[q] + dt * rhs[q];
        dU[q] = du;
        Uout[q] = Uin[q] + B * du;
    }
}

}  // namespace crocco
