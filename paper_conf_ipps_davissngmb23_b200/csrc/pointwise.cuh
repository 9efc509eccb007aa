// pointwise.cuh -- primitive recovery, viscous point fluxes, standalone RK update.
// Part of libcrocco (sm_100a, fp64). Formulas restate the paper's method as
// read in DESIGN.md sec. 3 (citations: PAPER.md line numbers); no code is
// shared with oracle/.
#pragma once
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

}  // namespace crocco
