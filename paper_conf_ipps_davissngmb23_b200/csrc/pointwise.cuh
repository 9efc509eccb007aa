// pointwise.cuh -- the viscous kernel (point fluxes + two of the three D4
// divergences), ComputeDt's reduction, the state check and the standalone RK
// update.  Part of libcrocco (sm_100a, fp64).  Formulas restate the paper's
// method as read in DESIGN.md sec. 3 (citations: PAPER.md line numbers); no code
// is shared with oracle/.
#pragma once
#include "common.cuh"

namespace crocco {

// Viscous and heat point fluxes F^_v^d (reading 12): D4
// gradients in computational space, chain rule with the metrics, Newtonian
// stress (Stokes), Fourier heat flux, contravariant flux F^_v^d = m^d_b (tau_.b,
// u_a tau_ab - q_b).
__device__ __forceinline__ double mu_of_T(const Phys &ph, double T) {
    if (ph.mu_law == 1) {
        const double t = T / ph.T_ref;
        return ph.mu_ref * t * sqrt(t) * (ph.T_ref + ph.S) / (T + ph.S);
    }
    return ph.mu_ref;
}

// k_visc_tiled: the point fluxes fused with the primitive recovery and with the
// D4_xi and D4_zeta divergences.  A CTA owns VTX (i) x VTY (j) columns of the
// interior +-2 box and marches a slab of vk interior planes in k (plus 2 planes
// on each side).  Each thread keeps u, v, w, T of its own column for planes
// k-2..k+2 in registers (k-derivatives); only the current plane (with a 2-point
// i/j halo) is staged in shared memory (i/j-derivatives), double buffered so one
// barrier per plane suffices; the next plane's U and metrics are loaded into
// registers one step ahead.
//   - tiles advance by VSX = VTX - 4 columns in i, so every tile carries 2-column
//     arms on both sides; a warp is one 32-column tile row and the 28 central
//     lanes take D4_xi of F^_v^xi by warp shuffles from lanes +-1, +-2;
//   - F^_v^zeta enters a 5-plane register queue of the own column and its D4_zeta
//     is added; D4_xi + D4_zeta go to R (comps 1..4) together;
//   - only F^_v^eta (4 comps) goes to HBM, for the eta sweep's interface flux.
// Measured choices: 32 x 8 tiles (16 x 8 with 33 % arm work and
// 24 x 8 slower); shuffles instead of a shared-memory round trip for D4_xi (6.61 ->
// 6.48 ms per 512^3 launch); prefetch distance 1 (2: 254 registers, 7.26 ms).
constexpr int VTX = 32, VTY = 8, VK = 64;  // tile and default slab depth
constexpr int VSX = VTX - 4;               // tile stride in i (2-column arms each side)
constexpr int VHX = VTX + 4, VHY = VTY + 4;  // with halo
constexpr int VPL = VHX * VHY;               // points per staged plane
constexpr int VHALO = VPL - VTX * VTY;       // halo points per plane
constexpr size_t VISC_SMEM = (size_t)2 * 4 * VPL * sizeof(double);
// slab depth of k_visc_tiled (run time): the longest of VISC_VKMAX / ... / 128 planes that still
// gives >= 8 waves of one-CTA-per-SM tiles (each slab recomputes 4 boundary planes; 64 -> 256
// measured 6.47 -> 6.22 ms per 512^3 launch; 512 slower: one slab per column, 8.3 waves), else VK
constexpr int VISC_VKMAX = 256;
__host__ __device__ inline int visc_tiles_x(const Lay &L) { return (L.n0 + VSX - 1) / VSX; }
// overlap: the stage runs the ghost-free tiles beside the fill (crocco_rk_stage), so the slab
// depth must leave at least one interior slab, (n2 - 4)/vk >= 2 (visc_interior_tiles)
// Small boxes (fewer than two waves of tiles at VK): shorter slabs down to VISC_VKMIN planes, so
// the marching chains shorten and more SMs take part (64^3: 27 tiles of 68 planes -> 216 of 12).
constexpr int VISC_VKMIN = 8;
inline int visc_slab(const Lay &L, const VLay &V, bool overlap = false) {
    const int64_t txy = (int64_t)visc_tiles_x(L) * ((V.b1 + VTY - 1) / VTY);
    for (int vk = VISC_VKMAX; vk > VK; vk /= 2)
        if (txy * ((L.n2 + vk - 1) / vk) >= 8 * 148 && (!overlap || (L.n2 - 4) / vk >= 2)) return vk;
    int vk = VK;
    while (vk > VISC_VKMIN && txy * ((L.n2 + vk - 1) / vk) < 2 * 148) vk /= 2;
    return vk;
}

// Tiles of k_visc_tiled whose loads stay inside the interior [0, n) in every
// direction (no ghost point read): they may run while the ghost exchange is in
// flight (SURVEY 8(e) overlap).  Half-open ranges of tile indices.
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
// MUL: the viscosity law (ph.mu_law) as a template parameter (the Sutherland branch's sqrt and division
// otherwise sit in every launch's code)
template <int MUL>
__global__ void __launch_bounds__(VTX * VTY, 1) k_visc_tiled(const double *__restrict__ U,
                                                          const double *__restrict__ M,
                                                          double *__restrict__ FV, Lay L, VLay V,
                                                          Phys ph, double *__restrict__ R, int64_t rcs,
                                                          int sel, int vk) {
    extern __shared__ double vsm[];  // [buffer 2][value 4][VPL]
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
    double xq[4] = {0.0, 0.0, 0.0, 0.0};   // D4_xi F^xi of plane k-2 (computed two steps back)
    double xq1[4] = {0.0, 0.0, 0.0, 0.0};  // D4_xi F^xi of plane k-1
    // slab of interior output planes [z0, z1); gradients / point fluxes on planes z0-2 .. z1+1
    const int z0 = bz * vk, z1 = min(z0 + vk, L.n2);
    const int k0 = z0 - 2, k1 = z1 + 2;
    double zq[5][4];  // F^zeta of the own column, planes k-4 .. k
#pragma unroll
    for (int o = 0; o < 5; o++)
#pragma unroll
        for (int q = 0; q < 4; q++) zq[o][q] = 0.0;
    const double iR = 1.0 / ph.R;
    // own column (clamped into the padded box for the idle threads of edge tiles)
    const int i = i0 + tx, j = j0 + ty;
    const bool own = i < V.b0 - 2 && j < V.b1 - 2;
    // the column whose outputs (F^eta, R) this thread writes: the central columns only
    const bool central = tx >= 2 && tx < VTX - 2 && i < L.n0;
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

    // u v w T of a conserved state (perfect gas, Eq. 2 single species)
    auto prim_of = [&](const double u5[5], double q[4]) {
        const double ir = rcp_nr(u5[0]);
        const double u = u5[1] * ir, v = u5[2] * ir, w = u5[3] * ir;
        const double pr = ph.gm1 * fma(-0.5, fma(u5[1], u, fma(u5[2], v, u5[3] * w)), u5[4]);
        q[0] = u;
        q[1] = v;
        q[2] = w;
        q[3] = pr * ir * iR;
    };
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
    double win[4][5];  // own u v w T at planes k-2 .. k+2
    for (int o = 0; o < 4; o++) {
        double u5[5], q[4];
        ld_own(k0 - 2 + o, u5);
        prim_of(u5, q);
#pragma unroll
        for (int f = 0; f < 4; f++) win[f][o + 1] = q[f];  // shifted into 0..3 by the first step
    }
    // global operands of the step, loaded one step ahead: own U at plane k+2,
    // halo U at plane k, own metrics at plane k
    double cO[5], cH[5], cM[10];
    ld_own(k0 + 2, cO);
    ld_halo(k0, cH);
    ld_met(k0, cM);
    for (int k = k0; k < k1; k++) {
        double nO[5], nH[5], nM[10];
        const int kn = min(k + 1, k1 - 1);  // clamp: the last step reloads
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
        __syncthreads();
        double fxr[4] = {0.0, 0.0, 0.0, 0.0};  // F^xi of this column at plane k
        {   // every thread evaluates (idle edge columns on clamped loads; their F^xi is masked below,
            // their F^eta / R stores are predicated): no divergent branch, -0.04 ms per 512^3 launch
            double gc[4][3];
#pragma unroll
            for (int f = 0; f < 4; f++) {
                const double *c = pl + f * VPL + oidx;
                gc[f][0] = fma(8.0, c[1] - c[-1], -(c[2] - c[-2])) * (1.0 / 12.0);
                gc[f][1] = fma(8.0, c[VHX] - c[-VHX], -(c[2 * VHX] - c[-2 * VHX])) * (1.0 / 12.0);
                gc[f][2] = fma(8.0, win[f][3] - win[f][1], -(win[f][4] - win[f][0])) * (1.0 / 12.0);
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
            const double T = win[3][2];
            const double mu = MUL == 1 ? mu_of_T(ph, T) : ph.mu_ref;
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
#pragma unroll
            for (int a = 0; a < 3; a++)
                fxr[a] = fma(m[0][0], tau[a][0], fma(m[0][1], tau[a][1], m[0][2] * tau[a][2]));
            fxr[3] = fma(m[0][0], hb[0], fma(m[0][1], hb[1], m[0][2] * hb[2]));
#pragma unroll
            for (int q = 0; q < 4; q++) fxr[q] = own ? fxr[q] : 0.0;
            if (k >= z0 && k < z1 && central && own) {  // F^eta only (the eta sweep differences it)
#pragma unroll
                for (int a = 0; a < 3; a++)
                    FV[a * V.cs + o] = fma(m[1][0], tau[a][0], fma(m[1][1], tau[a][1], m[1][2] * tau[a][2]));
                FV[3 * V.cs + o] = fma(m[1][0], hb[0], fma(m[1][1], hb[1], m[1][2] * hb[2]));
            }
            // F^zeta stays in the own column's queue and is differenced here (D4_zeta)
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
#pragma unroll
        for (int c = 0; c < 5; c++) {
            cO[c] = nO[c];
            cH[c] = nH[c];
        }
#pragma unroll
        for (int c = 0; c < 10; c++) cM[c] = nM[c];
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
