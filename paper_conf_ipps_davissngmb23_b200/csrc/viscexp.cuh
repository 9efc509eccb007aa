// viscexp.cuh -- the paper's 27-component metric set and the expanded (non-conservative)
// viscous form ("first and second order grid metrics ... a 27-component
// MultiFab"; readings 27-28).  A variant selected by
// crocco_phys.visc_form = 1; the default path is the conservative point-flux form.
// Part of libcrocco (sm_100a, fp64); no code shared with oracle/.
//
//   first metrics   xi_{a,j} = J m^a_j
//   second metrics  xi_{a,jk} = sum_b xi_{b,k} D6_b(xi_{a,j}),  j <= k, comp 6a + pair
//   V = div F_v at interior points by the chain rule (reading 28); R[1..4] = V / J so that
//   the sweeps' final rhs = J R adds V to the inviscid part.
#pragma once
#include "common.cuh"
#include "metrics.cuh"

namespace crocco {

__device__ __forceinline__ int pair_index(int j, int k) {  // (00, 01, 02, 11, 12, 22)
    const int lo = j < k ? j : k, hi = j < k ? k : j;
    return lo == 0 ? hi : (lo == 1 ? 2 + hi : 5);
}

// second metrics of the interior points, compact layout M2[q * rcs + i + n0 (j + n1 k)]
__global__ void __launch_bounds__(128) k_metric2(const double *__restrict__ M, double *__restrict__ M2,
                                                 Lay L, int64_t rcs) {
    const int64_t tid = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
    if (tid >= (int64_t)L.n0 * L.n1 * L.n2) return;
    const int i = (int)(tid % L.n0);
    const int64_t r = tid / L.n0;
    const int j = (int)(r % L.n1), k = (int)(r / L.n1);
    const int64_t p = at(L, i, j, k);
    const int64_t st[3] = {1, L.py, L.pz};
    auto xi = [&](int a, int c, int64_t q) { return M[q] * M[(1 + 3 * a + c) * L.cs + q]; };
    double x1[3][3];
#pragma unroll
    for (int b = 0; b < 3; b++)
#pragma unroll
        for (int c = 0; c < 3; c++) x1[b][c] = xi(b, c, p);
#pragma unroll
    for (int a = 0; a < 3; a++)
#pragma unroll
        for (int jj = 0; jj < 3; jj++) {
            double dx[3];  // D6_b of xi_{a,jj}
#pragma unroll
            for (int b = 0; b < 3; b++) {
                const int64_t s = st[b];
                dx[b] = (45.0 * (xi(a, jj, p + s) - xi(a, jj, p - s)) - 9.0 * (xi(a, jj, p + 2 * s) - xi(a, jj, p - 2 * s)) +
                         (xi(a, jj, p + 3 * s) - xi(a, jj, p - 3 * s))) *
                        (1.0 / 60.0);
            }
#pragma unroll
            for (int kk = jj; kk < 3; kk++)
                M2[(6 * a + pair_index(jj, kk)) * rcs + tid] = x1[0][kk] * dx[0] + x1[1][kk] * dx[1] + x1[2][kk] * dx[2];
        }
}

// u, v, w, T of every point of the padded box (P4[f * cs + p])
__global__ void __launch_bounds__(256) k_prims4(const double *__restrict__ U, double *__restrict__ P4, Lay L,
                                                const Phys ph) {
    const int64_t p = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
    if (p >= L.cs) return;
    const double rho = U[p], ir = 1.0 / rho;
    const double u = U[L.cs + p] * ir, v = U[2 * L.cs + p] * ir, w = U[3 * L.cs + p] * ir;
    const double pr = ph.gm1 * (U[4 * L.cs + p] - 0.5 * rho * (u * u + v * v + w * w));
    P4[p] = u;
    P4[L.cs + p] = v;
    P4[2 * L.cs + p] = w;
    P4[3 * L.cs + p] = pr * ir / ph.R;
}

__device__ __forceinline__ double d4c(const double *f, int64_t p, int64_t s) {
    return (8.0 * (f[p + s] - f[p - s]) - (f[p + 2 * s] - f[p - 2 * s])) * (1.0 / 12.0);
}
__device__ __forceinline__ double d2c(const double *f, int64_t p, int64_t s) {
    return (16.0 * (f[p + s] + f[p - s]) - (f[p + 2 * s] + f[p - 2 * s]) - 30.0 * f[p]) * (1.0 / 12.0);
}

// expanded viscous divergence (reading 28) of the interior points -> R comps 1..4 = V / J
__global__ void __launch_bounds__(128) k_visc_exp(const double *__restrict__ P4, const double *__restrict__ M,
                                                  const double *__restrict__ M2, double *__restrict__ R,
                                                  int64_t rcs, Lay L, const Phys ph) {
    const int64_t tid = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
    if (tid >= (int64_t)L.n0 * L.n1 * L.n2) return;
    const int i = (int)(tid % L.n0);
    const int64_t r = tid / L.n0;
    const int j = (int)(r % L.n1), k = (int)(r / L.n1);
    const int64_t p = at(L, i, j, k);
    const int64_t st[3] = {1, L.py, L.pz};
    const double J = M[p];
    double xi[3][3];
#pragma unroll
    for (int a = 0; a < 3; a++)
#pragma unroll
        for (int c = 0; c < 3; c++) xi[a][c] = J * M[(1 + 3 * a + c) * L.cs + p];
    double gx[4][3];     // d phi / d x_c
    double hx[4][6];     // d2 phi / d x_j d x_k, pair index (T: diagonal pairs only used)
#pragma unroll
    for (int f = 0; f < 4; f++) {
        const double *F = P4 + f * L.cs;
        double p1[3], p2[3][3];
#pragma unroll
        for (int a = 0; a < 3; a++) p1[a] = d4c(F, p, st[a]);
#pragma unroll
        for (int a = 0; a < 3; a++) p2[a][a] = d2c(F, p, st[a]);
#pragma unroll
        for (int lo = 0; lo < 3; lo++)
#pragma unroll
            for (int hi = lo + 1; hi < 3; hi++) {
                const int64_t sh = st[hi], sl = st[lo];
                const double m = (8.0 * (d4c(F, p + sh, sl) - d4c(F, p - sh, sl)) -
                                  (d4c(F, p + 2 * sh, sl) - d4c(F, p - 2 * sh, sl))) *
                                 (1.0 / 12.0);
                p2[lo][hi] = p2[hi][lo] = m;
            }
#pragma unroll
        for (int c = 0; c < 3; c++) gx[f][c] = xi[0][c] * p1[0] + xi[1][c] * p1[1] + xi[2][c] * p1[2];
#pragma unroll
        for (int q = 0; q < 6; q++) {
            const int jj = q < 3 ? 0 : (q < 5 ? 1 : 2);
            const int kk = q < 3 ? q : (q < 5 ? q - 2 : 2);
            double s = 0.0;
#pragma unroll
            for (int a = 0; a < 3; a++)
#pragma unroll
                for (int c = 0; c < 3; c++) s += xi[a][jj] * xi[c][kk] * p2[a][c];
#pragma unroll
            for (int a = 0; a < 3; a++) s += M2[(6 * a + q) * rcs + tid] * p1[a];
            hx[f][q] = s;
        }
    }
    const double T = P4[3 * L.cs + p];
    double mu, mup;
    if (ph.mu_law == 1) {
        const double t = T * ph.iT_ref;
        mu = ph.mu_ref * t * sqrt(t) * (ph.T_ref + ph.S) / (T + ph.S);
        mup = mu * (1.5 / T - 1.0 / (T + ph.S));
    } else {
        mu = ph.mu_ref;
        mup = 0.0;
    }
    const double div = gx[0][0] + gx[1][1] + gx[2][2];
    double dtau[3];
#pragma unroll
    for (int a = 0; a < 3; a++) {
        const double lap = hx[a][0] + hx[a][3] + hx[a][5];
        const double gdiv = hx[0][pair_index(0, a)] + hx[1][pair_index(1, a)] + hx[2][pair_index(2, a)];
        double s = mu * (lap + gdiv * (1.0 / 3.0));
#pragma unroll
        for (int c = 0; c < 3; c++) {
            double sym = gx[a][c] + gx[c][a];
            if (a == c) sym -= (2.0 / 3.0) * div;
            s += mup * gx[3][c] * sym;
        }
        dtau[a] = s;
    }
    const double u = P4[p], v = P4[L.cs + p], w = P4[2 * L.cs + p];
    double diss = 0.0;
#pragma unroll
    for (int a = 0; a < 3; a++)
#pragma unroll
        for (int c = 0; c < 3; c++) {
            double tau = mu * (gx[a][c] + gx[c][a]);
            if (a == c) tau -= (2.0 / 3.0) * mu * div;
            diss += tau * gx[a][c];
        }
    const double lapT = hx[3][0] + hx[3][3] + hx[3][5];
    const double gT2 = gx[3][0] * gx[3][0] + gx[3][1] * gx[3][1] + gx[3][2] * gx[3][2];
    const double kap_mu = ph.cp_over_Pr;  // kappa = mu c_p / Pr
    const double VE = u * dtau[0] + v * dtau[1] + w * dtau[2] + diss + kap_mu * (mu * lapT + mup * gT2);
    const double iJ = 1.0 / J;
    R[1 * rcs + tid] = dtau[0] * iJ;
    R[2 * rcs + tid] = dtau[1] * iJ;
    R[3 * rcs + tid] = dtau[2] * iJ;
    R[4 * rcs + tid] = VE * iJ;
}

}  // namespace crocco
