// kernels.cuh -- sm_100a device code of libcrocco (CRoCCo v2.0 hot path).
//
// Every formula here restates the paper's method as read in DESIGN.md sec. 3;
// citations are PAPER.md line numbers.  Nothing here is shared with oracle/.
// All arithmetic is fp64 on the CUDA-core FP64 pipe (no tensor cores: the
// path is a nonlinear stencil, not a contraction).  FMA contraction is left on
// (-fmad=true); parity with the (non-contracted) oracle is tested to 1e-11.
#pragma once
#include <cstdint>

namespace crocco {

constexpr int G = 4;    // state / metric ghost width (reading 7)
constexpr int GC = 10;  // coordinate ghost width (reading 7)

// ---------------------------------------------------------------------------
// Parameters passed by value (__grid_constant__-friendly PODs)
// ---------------------------------------------------------------------------
struct Phys {
    double gamma, gm1, igm1, R, Pr, cp_over_Pr;  // cp/Pr = gamma R /((gamma-1) Pr)
    int mu_law;
    double mu_ref, T_ref, S;
    double eps;
    int terms, dir_mask;
};

struct Lay {             // padded block layout (elements)
    int n0, n1, n2;
    int64_t off, py, pz, cs;
};

__host__ __device__ inline int64_t at(const Lay &L, int i, int j, int k) {
    return L.off + (int64_t)i + (int64_t)j * L.py + (int64_t)k * L.pz;
}

// ---------------------------------------------------------------------------
// WENO-SYMBO reconstruction at the +1/2 interface (PAPER.md:50 -> ref [9];
// reading 8).  One-divide form: alpha_k ~ C_k prod_{m!=k} (eps+beta_m)^2,
// mathematically identical to alpha_k = C_k/(eps+beta_k)^2.
// ---------------------------------------------------------------------------
__device__ __forceinline__ double weno_symbo(double v0, double v1, double v2, double v3, double v4,
                                             double v5, double eps) {
    constexpr double C0 = 0.094647545896, C1 = 0.428074212384, C2 = 0.408289331408,
                     C3 = 0.068988910311;
    constexpr double k1312 = 13.0 / 12.0;
    // six times the candidate reconstructions
    const double q0 = 2.0 * v0 - 7.0 * v1 + 11.0 * v2;
    const double q1 = -v1 + 5.0 * v2 + 2.0 * v3;
    const double q2 = 2.0 * v2 + 5.0 * v3 - v4;
    const double q3 = 11.0 * v3 - 7.0 * v4 + 2.0 * v5;
    double t1, t2;
    t1 = v0 - 2.0 * v1 + v2;
    t2 = v0 - 4.0 * v1 + 3.0 * v2;
    const double b0 = k1312 * t1 * t1 + 0.25 * t2 * t2;
    t1 = v1 - 2.0 * v2 + v3;
    t2 = v1 - v3;
    const double b1 = k1312 * t1 * t1 + 0.25 * t2 * t2;
    t1 = v2 - 2.0 * v3 + v4;
    t2 = 3.0 * v2 - 4.0 * v3 + v4;
    const double b2 = k1312 * t1 * t1 + 0.25 * t2 * t2;
    t1 = v3 - 2.0 * v4 + v5;
    t2 = -5.0 * v3 + 8.0 * v4 - 3.0 * v5;
    double b3 = k1312 * t1 * t1 + 0.25 * t2 * t2;
    b3 = fmax(fmax(b0, b1), fmax(b2, b3));  // downwind stencil never preferred
    double e0 = eps + b0, e1 = eps + b1, e2 = eps + b2, e3 = eps + b3;
    e0 *= e0;
    e1 *= e1;
    e2 *= e2;
    e3 *= e3;
    const double e01 = e0 * e1, e23 = e2 * e3;
    const double a0 = C0 * e1 * e23;
    const double a1 = C1 * e0 * e23;
    const double a2 = C2 * e01 * e3;
    const double a3 = C3 * e01 * e2;
    const double num = a0 * q0 + a1 * q1 + a2 * q2 + a3 * q3;
    const double den = 6.0 * (a0 + a1 + a2 + a3);
    return num / den;
}

// ---------------------------------------------------------------------------
// Characteristic WENO interface flux F^_{i+1/2} (
// readings 8-11).  Inputs are read from the conserved state U, the primitive
// buffer P (u v w p c sqrt(rho) H T) and the metric row m^d, at the 6 points
// i-2..i+3 (index p0 + l*s).  Pulliam-Chaussee eigenvectors at the Roe state
// of (i, i+1) for the unit normal of the frozen interface metric R6(m^d);
// local Lax-Friedrichs splitting per characteristic field.
// The projected flux uses L_s.F_n(U_l) = theta_l (L_s.U_l) + p_l k_{s,l}
// (F_n(U) = theta U + p (0, n, theta)), which is an exact identity.
// ---------------------------------------------------------------------------
enum { PU = 0, PV = 1, PW = 2, PP = 3, PC = 4, PSR = 5, PH = 6, PT = 7, NPRIM = 8 };

#ifndef CROCCO_FLUX_MINB
#define CROCCO_FLUX_MINB 1   // min resident CTAs/SM for k_flux (register cap)
#endif
#ifndef CROCCO_FLUX_USMEM
#define CROCCO_FLUX_USMEM 0  // 1: keep the 6x5 stencil states in shared memory, not registers
#endif
constexpr int FLUX_THREADS = 128;

__device__ __forceinline__ void iface_flux(const double *__restrict__ U,
                                           const double *__restrict__ Pm,
                                           const double *__restrict__ M, int64_t cs, int64_t p0,
                                           int64_t s, int d, const Phys &ph, double F[5],
                                           double *Us) {
    const double gm1 = ph.gm1;
    // frozen interface metric (reading 6): R6 = (1,-8,37,37,-8,1)/60
    const double *Md = M + (int64_t)(1 + 3 * d) * cs;
    double mh[3];
#pragma unroll
    for (int a = 0; a < 3; a++) {
        const double *m = Md + a * cs + p0;
        mh[a] = (37.0 * (m[2 * s] + m[3 * s]) - 8.0 * (m[s] + m[4 * s]) + (m[0] + m[5 * s])) *
                (1.0 / 60.0);
    }
    const double s2 = mh[0] * mh[0] + mh[1] * mh[1] + mh[2] * mh[2];
    const double imag = rsqrt(s2);
    const double mag = s2 * imag;
    const double nx = mh[0] * imag, ny = mh[1] * imag, nz = mh[2] * imag;

    // Roe average of points i (l=2) and i+1 (l=3) in sqrt(rho) form
    const int64_t pL = p0 + 2 * s, pR = p0 + 3 * s;
    const double srL = Pm[PSR * cs + pL], srR = Pm[PSR * cs + pR];
    const double iden = 1.0 / (srL + srR);
    const double ut = (srL * Pm[PU * cs + pL] + srR * Pm[PU * cs + pR]) * iden;
    const double vt = (srL * Pm[PV * cs + pL] + srR * Pm[PV * cs + pR]) * iden;
    const double wt = (srL * Pm[PW * cs + pL] + srR * Pm[PW * cs + pR]) * iden;
    const double Ht = (srL * Pm[PH * cs + pL] + srR * Pm[PH * cs + pR]) * iden;
    const double rt = srL * srR;
    const double q2 = ut * ut + vt * vt + wt * wt;
    const double c2 = gm1 * (Ht - 0.5 * q2);
    const double ict = rsqrt(c2);
    const double ct = c2 * ict;
    const double ic2 = ict * ict;
    const double irt = 1.0 / rt;
    const double tht = nx * ut + ny * vt + nz * wt;
    const double phi2 = 0.5 * gm1 * q2;
    constexpr double SQ12 = 0.70710678118654752440;
    const double alph = rt * ict * SQ12;   // rho/(sqrt2 c)
    const double beta = irt * ict * SQ12;  // 1/(sqrt2 rho c)

    // stencil points: state, normal velocity, pressure; LLF speeds
#if CROCCO_FLUX_USMEM
#define UL(l, c) Us[((l) * 5 + (c)) * FLUX_THREADS]
#else
    double Ul[6][5];
#define UL(l, c) Ul[l][c]
#endif
    double th[6], pl[6];
    double lam0 = 0.0, lam3 = 0.0, lam4 = 0.0;
#pragma unroll
    for (int l = 0; l < 6; l++) {
        const int64_t q = p0 + l * s;
#pragma unroll
        for (int c = 0; c < 5; c++) UL(l, c) = U[c * cs + q];
        const double t = nx * Pm[PU * cs + q] + ny * Pm[PV * cs + q] + nz * Pm[PW * cs + q];
        const double cl = Pm[PC * cs + q];
        th[l] = t;
        pl[l] = Pm[PP * cs + q];
        lam0 = fmax(lam0, fabs(t));
        lam3 = fmax(lam3, fabs(t + cl));
        lam4 = fmax(lam4, fabs(t - cl));
    }

    double f0 = 0.0, f1 = 0.0, f2 = 0.0, f3 = 0.0, f4 = 0.0;
    const double onemp = 1.0 - phi2 * ic2;
    const double gic2 = gm1 * ic2;
    const double nv[3] = {nx, ny, nz};
    // n x u~ (for the entropy/vorticity rows)
    const double cx = ny * wt - nz * vt, cy = nz * ut - nx * wt, cz = nx * vt - ny * ut;
    const double cr[3] = {cx, cy, cz};
#pragma unroll
    for (int sf = 0; sf < 5; sf++) {
        double L0, L1, L2, L3, L4;     // row s of T^{-1}
        double R0, R1, R2, R3, R4;     // column s of T
        double lam;
        double kA, kB;                 // k_{s,l} = kA + kB*theta_l
        if (sf < 3) {
            const double na = nv[sf];
            L0 = na * onemp + cr[sf] * irt;
            // -eps_{s b c} n_c / rho contributions, written out per s
            if (sf == 0) {
                L1 = na * gic2 * ut;
                L2 = nz * irt + na * gic2 * vt;
                L3 = -ny * irt + na * gic2 * wt;
                R1 = na * ut;
                R2 = na * vt + nz * rt;
                R3 = na * wt - ny * rt;
                R4 = na * phi2 * ph.igm1 + rt * (nz * vt - ny * wt);
            } else if (sf == 1) {
                L1 = -nz * irt + na * gic2 * ut;
                L2 = na * gic2 * vt;
                L3 = nx * irt + na * gic2 * wt;
                R1 = na * ut - nz * rt;
                R2 = na * vt;
                R3 = na * wt + nx * rt;
                R4 = na * phi2 * ph.igm1 + rt * (nx * wt - nz * ut);
            } else {
                L1 = ny * irt + na * gic2 * ut;
                L2 = -nx * irt + na * gic2 * vt;
                L3 = na * gic2 * wt;
                R1 = na * ut + ny * rt;
                R2 = na * vt - nx * rt;
                R3 = na * wt;
                R4 = na * phi2 * ph.igm1 + rt * (ny * ut - nx * vt);
            }
            L4 = -na * gic2;
            R0 = na;
            lam = lam0;
            kA = na * gic2 * tht;   // n_s (g-1) theta~/c^2 - theta_l n_s (g-1)/c^2
            kB = -na * gic2;
        } else {
            const double sg = (sf == 3) ? 1.0 : -1.0;
            L0 = beta * (phi2 - sg * ct * tht);
            L1 = sg * beta * (nx * ct - sg * gm1 * ut);
            L2 = sg * beta * (ny * ct - sg * gm1 * vt);
            L3 = sg * beta * (nz * ct - sg * gm1 * wt);
            L4 = beta * gm1;
            R0 = alph;
            R1 = alph * (ut + sg * nx * ct);
            R2 = alph * (vt + sg * ny * ct);
            R3 = alph * (wt + sg * nz * ct);
            R4 = alph * ((phi2 + c2) * ph.igm1 + sg * ct * tht);
            lam = (sf == 3) ? lam3 : lam4;
            kA = beta * (sg * ct - gm1 * tht);
            kB = beta * gm1;
        }
        double gp[6], gm[6];
        const double hl = 0.5 * lam;
#pragma unroll
        for (int l = 0; l < 6; l++) {
            const double w = L0 * UL(l, 0) + L1 * UL(l, 1) + L2 * UL(l, 2) + L3 * UL(l, 3) +
                             L4 * UL(l, 4);
            const double g = th[l] * w + pl[l] * (kA + kB * th[l]);
            gp[l] = 0.5 * g + hl * w;
            gm[l] = 0.5 * g - hl * w;
        }
        const double gh = weno_symbo(gp[0], gp[1], gp[2], gp[3], gp[4], gp[5], ph.eps) +
                          weno_symbo(gm[5], gm[4], gm[3], gm[2], gm[1], gm[0], ph.eps);
        f0 += R0 * gh;
        f1 += R1 * gh;
        f2 += R2 * gh;
        f3 += R3 * gh;
        f4 += R4 * gh;
    }
    F[0] = mag * f0;
    F[1] = mag * f1;
    F[2] = mag * f2;
    F[3] = mag * f3;
    F[4] = mag * f4;
}

// ---------------------------------------------------------------------------
// Kernels
// ---------------------------------------------------------------------------

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

// Interface fluxes of direction D for every interface i+1/2, i in [-1, n_D-1],
// of the interior lines; written to Fd[c][interface index] (WENOx/y/z,
// PAPER.md:110-112).  Each interface is computed exactly once.
template <int D>
__global__ void __launch_bounds__(FLUX_THREADS, CROCCO_FLUX_MINB) k_flux(const double *__restrict__ U,
                                              const double *__restrict__ Pm,
                                              const double *__restrict__ M, double *__restrict__ Fd,
                                              int64_t fcs, Lay L, Phys ph) {
    int i, j, k;
    int64_t out;
    if (D == 0) {
        const int64_t t = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
        const int ne = L.n0 + 1;
        const int64_t tot = (int64_t)ne * L.n1 * L.n2;
        if (t >= tot) return;
        const int e = (int)(t % ne);
        const int64_t line = t / ne;
        j = (int)(line % L.n1);
        k = (int)(line / L.n1);
        i = e - 1;
        out = t;
    } else if (D == 1) {
        i = blockIdx.y * blockDim.x + threadIdx.x;
        const int64_t y = (int64_t)blockIdx.x * blockDim.y + threadIdx.y;
        const int ne = L.n1 + 1;
        if (i >= L.n0 || y >= (int64_t)ne * L.n2) return;
        const int e = (int)(y % ne);
        k = (int)(y / ne);
        j = e - 1;
        out = i + (int64_t)L.n0 * y;
    } else {
        i = blockIdx.y * blockDim.x + threadIdx.x;
        const int64_t y = (int64_t)blockIdx.x * blockDim.y + threadIdx.y;
        if (i >= L.n0 || y >= (int64_t)L.n1 * (L.n2 + 1)) return;
        j = (int)(y % L.n1);
        const int e = (int)(y / L.n1);
        k = e - 1;
        out = i + (int64_t)L.n0 * y;
    }
    const int64_t s = (D == 0) ? 1 : (D == 1 ? L.py : L.pz);
    const int64_t p0 = at(L, i, j, k) - 2 * s;
    double F[5];
#if CROCCO_FLUX_USMEM
    __shared__ double sU[30 * FLUX_THREADS];
    double *Us = sU + threadIdx.x + blockDim.x * threadIdx.y;
#else
    double *Us = nullptr;
#endif
    iface_flux(U, Pm, M, L.cs, p0, s, D, ph, F, Us);
#pragma unroll
    for (int c = 0; c < 5; c++) Fd[c * fcs + out] = F[c];
#undef UL
}

// Viscous and heat point fluxes F^_v^d (reading 12) on the
// interior +-2 box: D4 gradients in computational space, chain rule with the
// metrics, Newtonian stress (Stokes), Fourier heat flux, contravariant flux.
// Output FV[4d+q][box index], q = momentum x,y,z, energy.
struct VLay {
    int b0, b1, b2;  // (n+4) box dims
    int64_t cs;
};
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
    const int64_t o = (i + 2) + (int64_t)V.b0 * ((j + 2) + (int64_t)V.b1 * (k + 2));
#pragma unroll
    for (int d = 0; d < 3; d++) {
#pragma unroll
        for (int a = 0; a < 3; a++)
            FV[(4 * d + a) * V.cs + o] = m[d][0] * tau[a][0] + m[d][1] * tau[a][1] + m[d][2] * tau[a][2];
        FV[(4 * d + 3) * V.cs + o] = m[d][0] * hb[0] + m[d][1] * hb[1] + m[d][2] * hb[2];
    }
}

// RHS assembly + Williamson update (PAPER.md:114 Update; reading 13):
// R = -sum_d (F_{i+1/2} - F_{i-1/2}) + sum_d D4_d F_v^d ;  rhs = J R.
// mode 0: write rhs.  mode 1: dU <- A dU + dt rhs ; U_out = U_in + B dU.
struct Asm {
    const double *F[3];
    int64_t fcs[3];
    const double *FV;
    VLay V;
    const double *M;
    const double *Uin;
    double *Uout;
    double *dU;
    double *rhs;
    double A, B, dt;
    int stage, mode, inv_mask, visc;
};
__global__ void __launch_bounds__(256) k_assemble(Asm a, Lay L) {
    const int i = blockIdx.x * blockDim.x + threadIdx.x;
    const int j = blockIdx.y;
    const int k = blockIdx.z;
    if (i >= L.n0) return;
    const int64_t p = at(L, i, j, k);
    double R[5] = {0.0, 0.0, 0.0, 0.0, 0.0};
    // inviscid flux differences; interface index of i-1/2 and i+1/2
    if (a.inv_mask & 1) {
        const int64_t lo = (int64_t)i + (int64_t)(L.n0 + 1) * (j + (int64_t)L.n1 * k);
#pragma unroll
        for (int c = 0; c < 5; c++) R[c] -= a.F[0][c * a.fcs[0] + lo + 1] - a.F[0][c * a.fcs[0] + lo];
    }
    if (a.inv_mask & 2) {
        const int64_t lo = (int64_t)i + (int64_t)L.n0 * (j + (int64_t)(L.n1 + 1) * k);
#pragma unroll
        for (int c = 0; c < 5; c++)
            R[c] -= a.F[1][c * a.fcs[1] + lo + L.n0] - a.F[1][c * a.fcs[1] + lo];
    }
    if (a.inv_mask & 4) {
        const int64_t lo = (int64_t)i + (int64_t)L.n0 * (j + (int64_t)L.n1 * k);
        const int64_t st = (int64_t)L.n0 * L.n1;
#pragma unroll
        for (int c = 0; c < 5; c++) R[c] -= a.F[2][c * a.fcs[2] + lo + st] - a.F[2][c * a.fcs[2] + lo];
    }
    if (a.visc) {
        const int64_t o = (i + 2) + (int64_t)a.V.b0 * ((j + 2) + (int64_t)a.V.b1 * (k + 2));
        const int64_t st[3] = {1, a.V.b0, (int64_t)a.V.b0 * a.V.b1};
#pragma unroll
        for (int q = 0; q < 4; q++)
#pragma unroll
            for (int d = 0; d < 3; d++) R[1 + q] += d4(a.FV + (4 * d + q) * a.V.cs, o, st[d]);
    }
    const double J = a.M[p];
    if (a.mode == 0) {
#pragma unroll
        for (int c = 0; c < 5; c++) a.rhs[c * L.cs + p] = J * R[c];
    } else {
#pragma unroll
        for (int c = 0; c < 5; c++) {
            const int64_t q = c * L.cs + p;
            const double r = J * R[c];
            const double du = (a.stage == 0) ? a.dt * r : a.A * a.dU[q] + a.dt * r;
            a.dU[q] = du;
            a.Uout[q] = a.Uin[q] + a.B * du;
        }
    }
}

// Update alone, from a materialised rhs (crocco_rk_update).
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

// ---------------------------------------------------------------------------
// Grid metrics (InitGridMetrics; readings 5-6).
//   dx[3a+d] = D6_d x_a on interior +-7 (coordinate layout),
//   m^d_a = D6_{d+2}[(D6_{d+1} x_{a+1}) x_{a+2}] - D6_{d+1}[(D6_{d+2} x_{a+1}) x_{a+2}],
//   J = 1/det(dx), on the padded box interior +-4.
// ---------------------------------------------------------------------------
__device__ __forceinline__ double d6(const double *f, int64_t p, int64_t s) {
    return (45.0 * (f[p + s] - f[p - s]) - 9.0 * (f[p + 2 * s] - f[p - 2 * s]) +
            (f[p + 3 * s] - f[p - 3 * s])) *
           (1.0 / 60.0);
}
__global__ void __launch_bounds__(256) k_coord_deriv(const double *__restrict__ X,
                                                     double *__restrict__ DX, Lay C) {
    const int W = G + 3;
    const int b0 = C.n0 + 2 * W, b1 = C.n1 + 2 * W, b2 = C.n2 + 2 * W;
    const int64_t tid = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
    if (tid >= (int64_t)b0 * b1 * b2) return;
    const int i = (int)(tid % b0) - W;
    const int64_t r = tid / b0;
    const int j = (int)(r % b1) - W;
    const int k = (int)(r / b1) - W;
    const int64_t p = at(C, i, j, k);
    const int64_t st[3] = {1, C.py, C.pz};
#pragma unroll
    for (int a = 0; a < 3; a++)
#pragma unroll
        for (int d = 0; d < 3; d++) DX[(3 * a + d) * C.cs + p] = d6(X + a * C.cs, p, st[d]);
}
__global__ void __launch_bounds__(128) k_metric(const double *__restrict__ X,
                                                const double *__restrict__ DX,
                                                double *__restrict__ M, Lay C, Lay L) {
    const int b0 = L.n0 + 2 * G, b1 = L.n1 + 2 * G, b2 = L.n2 + 2 * G;
    const int64_t tid = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
    if (tid >= (int64_t)b0 * b1 * b2) return;
    const int i = (int)(tid % b0) - G;
    const int64_t r = tid / b0;
    const int j = (int)(r % b1) - G;
    const int k = (int)(r / b1) - G;
    const int64_t pc = at(C, i, j, k);
    const int64_t pm = at(L, i, j, k);
    const int64_t st[3] = {1, C.py, C.pz};
#pragma unroll
    for (int d = 0; d < 3; d++)
#pragma unroll
        for (int a = 0; a < 3; a++) {
            const int d1 = (d + 1) % 3, d2 = (d + 2) % 3, a1 = (a + 1) % 3, a2 = (a + 2) % 3;
            const double *x2 = X + a2 * C.cs;
            const double *g1 = DX + (3 * a1 + d1) * C.cs;
            const double *g2 = DX + (3 * a1 + d2) * C.cs;
            auto prod1 = [&](int64_t q) { return g1[q] * x2[q]; };
            auto prod2 = [&](int64_t q) { return g2[q] * x2[q]; };
            const int64_t s2 = st[d2], s1 = st[d1];
            const double t1 = (45.0 * (prod1(pc + s2) - prod1(pc - s2)) -
                               9.0 * (prod1(pc + 2 * s2) - prod1(pc - 2 * s2)) +
                               (prod1(pc + 3 * s2) - prod1(pc - 3 * s2))) *
                              (1.0 / 60.0);
            const double t2 = (45.0 * (prod2(pc + s1) - prod2(pc - s1)) -
                               9.0 * (prod2(pc + 2 * s1) - prod2(pc - 2 * s1)) +
                               (prod2(pc + 3 * s1) - prod2(pc - 3 * s1))) *
                              (1.0 / 60.0);
            M[(1 + 3 * d + a) * L.cs + pm] = t1 - t2;
        }
    double A[3][3];
#pragma unroll
    for (int a = 0; a < 3; a++)
#pragma unroll
        for (int d = 0; d < 3; d++) A[a][d] = DX[(3 * a + d) * C.cs + pc];
    const double det = A[0][0] * (A[1][1] * A[2][2] - A[1][2] * A[2][1]) -
                       A[0][1] * (A[1][0] * A[2][2] - A[1][2] * A[2][0]) +
                       A[0][2] * (A[1][0] * A[2][1] - A[1][1] * A[2][0]);
    M[pm] = 1.0 / det;
}

}  // namespace crocco
