// MEASURED AND REJECTED (round 2): bitwise equal to k_visc_tiled but 6.56 vs 6.23 ms per 512^3
// launch (profiles/r02_variants_visc_tma.jsonl): the viscous kernel is issue / shared-memory bound
// (ncu: long-scoreboard stalls 5 %, mio + short-scoreboard 22 %), so staging more bytes in flight
// does not pay and the shared-memory primitive ring adds LDS traffic.  Not compiled.
// visc_tma.cuh -- the viscous kernel fed by TMA (Viscous; reading 12).
//
// Same tiles, slabs, arithmetic and outputs as k_visc_tiled (pointwise.cuh): point fluxes
// F^_v^d of the interior +-2 box from D4 gradients, the D4_xi divergence by warp shuffles,
// the D4_zeta divergence from an own-column register queue, both written to R (comps 1..4),
// F^_v^eta to HBM for the eta sweep.  What differs is how the operands reach the SM: every
// plane step, one thread issues two TMA tile loads (cp.async.bulk.tensor, mbarrier
// completion) -- the conserved state of plane k+2 on the halo'd tile (5 x 12 x 36) and the
// 10 metric components of plane k on the 8 x 32 own columns -- VST stages ahead of use, so
// about VST x 37 KB per SM are in flight without holding a register; the primitives of the
// halo'd tile go to a 6-plane ring in shared memory, from which the i, j and k derivatives
// are taken (no own-column register window).  Every arithmetic expression is the one of
// k_visc_tiled, so the results are bitwise equal.
#pragma once
#include <cuda.h>
#include "pointwise.cuh"

namespace crocco {

constexpr int VST = 3;  // TMA stages in flight (U plane k+2 and metrics of plane k per stage)
constexpr int VPR = 6;  // planes of primitives kept (k-2 .. k+2 read, k+3 written next step)
constexpr int VUP = 5 * VPL;        // doubles of one staged U plane (5 comps x 12 x 36)
constexpr int VMP = 10 * VTX * VTY;  // doubles of one staged metric plane (10 comps x 8 x 32)
constexpr int VPP = 4 * VPL;        // doubles of one primitive plane (u v w T x 12 x 36)
constexpr size_t VISC_TMA_SMEM = (size_t)(VST * (VUP + VMP) + VPR * VPP) * sizeof(double) + VST * 8 + 128;

struct ViscTmaArgs {
    CUtensorMap tu;  // U: dims (pitch_y, n1 + 8, n2 + 8, 5), box (36, 12, 1, 5)
    CUtensorMap tm;  // metrics: dims (pitch_y, n1 + 8, n2 + 8, 10), box (32, 8, 1, 10)
};

__device__ __forceinline__ unsigned smem_u32(const void *p) { return (unsigned)__cvta_generic_to_shared(p); }
__device__ __forceinline__ void mbar_init(uint64_t *bar, unsigned count) {
    asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(smem_u32(bar)), "r"(count) : "memory");
}
__device__ __forceinline__ void mbar_expect_tx(uint64_t *bar, unsigned bytes) {
    asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(smem_u32(bar)), "r"(bytes)
                 : "memory");
}
__device__ __forceinline__ void mbar_wait(uint64_t *bar, unsigned parity) {
    asm volatile(
        "{\n .reg .pred p;\n WAIT_%=:\n"
        " mbarrier.try_wait.parity.shared::cta.b64 p, [%0], %1;\n"
        " @!p bra WAIT_%=;\n}\n" ::"r"(smem_u32(bar)),
        "r"(parity)
        : "memory");
}
__device__ __forceinline__ void tma_load4(void *dst, const CUtensorMap *map, int x, int y, int z, int c,
                                          uint64_t *bar) {
    asm volatile(
        "cp.async.bulk.tensor.4d.shared::cluster.global.tile.mbarrier::complete_tx::bytes [%0], [%1, {%2, %3, %4, %5}], [%6];"
        ::"r"(smem_u32(dst)), "l"((uint64_t)map), "r"(x), "r"(y), "r"(z), "r"(c), "r"(smem_u32(bar))
        : "memory");
}

// sel: 0 every tile, 1 the ghost-free interior tiles only, 2 every other tile (as k_visc_tiled)
__global__ void __launch_bounds__(VTX * VTY, 1) k_visc_tma(const __grid_constant__ ViscTmaArgs ta,
                                                        const double *__restrict__ U, double *__restrict__ FV,
                                                        Lay L, VLay V, Phys ph, double *__restrict__ R,
                                                        int64_t rcs, int sel, int vk) {
    extern __shared__ __align__(128) unsigned char vsm_raw[];
    // 128-B aligned staging: [VST][U plane] [VST][metric plane] [VPR][primitive plane] [VST] mbarriers
    double *base = (double *)(((uintptr_t)vsm_raw + 127) & ~(uintptr_t)127);
    double *ust = base;
    double *mst = ust + VST * VUP;
    double *prg = mst + VST * VMP;
    uint64_t *bar = (uint64_t *)(prg + VPR * VPP);
    const int tid = threadIdx.x;
    const int tx = tid % VTX, ty = tid / VTX;
    const int tilesx = visc_tiles_x(L), tilesy = (V.b1 + VTY - 1) / VTY;
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
    const int i0 = bx * VSX - 2, j0 = by * VTY - 2;  // first output point of the tile
    const int z0 = bz * vk, z1 = min(z0 + vk, L.n2);
    const int k0 = z0 - 2, k1 = z1 + 2;              // planes of point fluxes: k0 .. k1-1
    const int nst = k1 - k0;
    // tensor coordinates (elements of the padded arrays): x = i + 16 (row lead), y = j + G, z = k + G
    const int tux = i0 - 2 + 16, tuy = j0 - 2 + G, tmx = i0 + 16, tmy = j0 + G;
    constexpr unsigned STAGE_BYTES = (unsigned)((VUP + VMP) * sizeof(double));
    auto issue = [&](int s) {  // stage s: U of plane k0+s+2 and metrics of plane k0+s
        uint64_t *bb = bar + s % VST;
        mbar_expect_tx(bb, STAGE_BYTES);
        tma_load4(ust + (s % VST) * VUP, &ta.tu, tux, tuy, k0 + s + 2 + G, 0, bb);
        tma_load4(mst + (s % VST) * VMP, &ta.tm, tmx, tmy, k0 + s + G, 0, bb);
    };
    if (tid == 0) {
        for (int s = 0; s < VST; s++) mbar_init(bar + s, 1);
        asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
        asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
        for (int s = 0; s < VST && s < nst; s++) issue(s);
    }
    const double iR = 1.0 / ph.R;
    auto prim_of = [&](const double u5[5], double q[4]) {
        const double ir = rcp_nr(u5[0]);
        const double u = u5[1] * ir, v = u5[2] * ir, w = u5[3] * ir;
        const double pr = ph.gm1 * fma(-0.5, fma(u5[1], u, fma(u5[2], v, u5[3] * w)), u5[4]);
        q[0] = u;
        q[1] = v;
        q[2] = w;
        q[3] = pr * ir * iR;
    };
    // prologue: primitives of planes k0-2 .. k0+1 on the halo'd tile, straight from global memory
    // (points clamped into the padded box as in k_visc_tiled: those values only reach discarded columns)
    for (int o = 0; o < 4; o++) {
        const int kk = k0 - 2 + o;
        double *pp = prg + ((kk + 2 * VPR) % VPR) * VPP;
        for (int p = tid; p < VPL; p += VTX * VTY) {
            const int hx = p % VHX, hy = p / VHX;
            const int gi = min(i0 - 2 + hx, L.n0 + G - 1), gj = min(j0 - 2 + hy, L.n1 + G - 1);
            const int64_t q = at(L, gi, gj, kk);
            double u5[5], pv[4];
#pragma unroll
            for (int c = 0; c < 5; c++) u5[c] = U[c * L.cs + q];
            prim_of(u5, pv);
#pragma unroll
            for (int f = 0; f < 4; f++) pp[f * VPL + p] = pv[f];
        }
    }
    // own column and output flags (as k_visc_tiled)
    const int i = i0 + tx, j = j0 + ty;
    const bool own = i < V.b0 - 2 && j < V.b1 - 2;
    const bool central = tx >= 2 && tx < VTX - 2 && i < L.n0;
    const int oidx = (ty + 2) * VHX + (tx + 2);
    double xq[4] = {0.0, 0.0, 0.0, 0.0};   // D4_xi F^xi of plane k-2
    double xq1[4] = {0.0, 0.0, 0.0, 0.0};  // D4_xi F^xi of plane k-1
    double zq[5][4];                        // F^zeta of the own column, planes k-4 .. k
#pragma unroll
    for (int o = 0; o < 5; o++)
#pragma unroll
        for (int q = 0; q < 4; q++) zq[o][q] = 0.0;
    for (int s = 0; s < nst; s++) {
        const int k = k0 + s;
        mbar_wait(bar + s % VST, (unsigned)(s / VST) & 1u);  // U(k+2), metrics(k) landed
        // primitives of plane k+2 on the halo'd tile -> ring slot (k+2) mod VPR (written over plane
        // k-4, last read in step k-2, before the barrier of step k-1)
        {
            const double *us = ust + (s % VST) * VUP;
            double *pp = prg + ((k + 2 + 2 * VPR) % VPR) * VPP;
            for (int p = tid; p < VPL; p += VTX * VTY) {
                double u5[5], pv[4];
#pragma unroll
                for (int c = 0; c < 5; c++) u5[c] = us[c * VPL + p];
                prim_of(u5, pv);
#pragma unroll
                for (int f = 0; f < 4; f++) pp[f * VPL + p] = pv[f];
            }
        }
        double cM[10];  // own metrics of plane k (read before the barrier: the slot is refilled after it)
#pragma unroll
        for (int c = 0; c < 10; c++) cM[c] = mst[(s % VST) * VMP + c * (VTX * VTY) + tid];
        __syncthreads();
        if (tid == 0 && s + VST < nst) {  // stage s+VST into the slot this step emptied
            asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
            issue(s + VST);
        }
        const double *pl = prg + ((k + 2 * VPR) % VPR) * VPP;
        const double *pm1 = prg + ((k - 1 + 2 * VPR) % VPR) * VPP, *pp1 = prg + ((k + 1 + 2 * VPR) % VPR) * VPP;
        const double *pm2 = prg + ((k - 2 + 2 * VPR) % VPR) * VPP, *pp2 = prg + ((k + 2 + 2 * VPR) % VPR) * VPP;
        double fxr[4] = {0.0, 0.0, 0.0, 0.0};  // F^xi of this column at plane k
        if (own) {
            double gc[4][3];
#pragma unroll
            for (int f = 0; f < 4; f++) {
                const double *c = pl + f * VPL + oidx;
                gc[f][0] = fma(8.0, c[1] - c[-1], -(c[2] - c[-2])) * (1.0 / 12.0);
                gc[f][1] = fma(8.0, c[VHX] - c[-VHX], -(c[2 * VHX] - c[-2 * VHX])) * (1.0 / 12.0);
                const int o = f * VPL + oidx;
                gc[f][2] = fma(8.0, pp1[o] - pm1[o], -(pp2[o] - pm2[o])) * (1.0 / 12.0);
            }
            const double J = cM[0];
            double m[3][3];
#pragma unroll
            for (int d = 0; d < 3; d++)
#pragma unroll
                for (int a = 0; a < 3; a++) m[d][a] = cM[1 + 3 * d + a];
            double gx[4][3];
#pragma unroll
            for (int f = 0; f < 4; f++)
#pragma unroll
                for (int a = 0; a < 3; a++)
                    gx[f][a] = J * fma(m[0][a], gc[f][0], fma(m[1][a], gc[f][1], m[2][a] * gc[f][2]));
            const double T = pl[3 * VPL + oidx];
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
            const double vel[3] = {pl[oidx], pl[VPL + oidx], pl[2 * VPL + oidx]};
            double hb[3];
#pragma unroll
            for (int bb = 0; bb < 3; bb++)
                hb[bb] = fma(vel[0], tau[0][bb], fma(vel[1], tau[1][bb], fma(vel[2], tau[2][bb], kap * gx[3][bb])));
            const int64_t o = vat(V, i, j, k);
#pragma unroll
            for (int a = 0; a < 3; a++)
                fxr[a] = fma(m[0][0], tau[a][0], fma(m[0][1], tau[a][1], m[0][2] * tau[a][2]));
            fxr[3] = fma(m[0][0], hb[0], fma(m[0][1], hb[1], m[0][2] * hb[2]));
            if (k >= z0 && k < z1 && central) {  // F^eta only (the eta sweep differences it)
#pragma unroll
                for (int a = 0; a < 3; a++)
                    FV[a * V.cs + o] = fma(m[1][0], tau[a][0], fma(m[1][1], tau[a][1], m[1][2] * tau[a][2]));
                FV[3 * V.cs + o] = fma(m[1][0], hb[0], fma(m[1][1], hb[1], m[1][2] * hb[2]));
            }
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
                    R[(1 + q) * rcs + r] = zd + xq[q];
                }
            }
        }
        // D4_xi of plane k from the row's lanes (every lane of the warp takes part)
        double xn[4];
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
    }
}

}  // namespace crocco
