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

// Expanded viscous divergence (reading 28) of the interior points -> R comps 1..4 = V / J, tiled:
// a CTA owns XTX x XTY interior columns and marches a slab of planes in k.  Per plane, u, v, w, T of the halo'd tile (XTX + 4) x (XTY + 4) go into a 6-plane ring in
// shared memory (from U, no primitive array); D4_i and D4_j of the own column enter 5-plane
// register queues (the (i,k) and (j,k) mixed derivatives are D4_k of them), D4_i of the plane
// on the halo rows is staged once more for the (i,j) mixed derivative; first metrics and the 18
// second metrics are read once per point; the next plane's U is staged by cp.async one plane
// ahead.  Per point: D4 first, 5-point D2 and D4-of-D4 mixed computational derivatives, the chain
// rule with the first and second metrics, Sutherland mu' terms (round 2: 12.0 ms per 512^3 launch
// against 19.1 ms for the round-1 global-load pair k_prims4 + k_visc_exp,
// profiles/r02_variants_visc_exp_tiled.jsonl).
constexpr int XTX = 32, XTY = 8;
constexpr int XHX = XTX + 4, XHY = XTY + 4, XPL = XHX * XHY;
constexpr int XNP = 6;  // ring planes: k-2 .. k+2 read while plane k+3 is written
constexpr size_t VISC_EXP_SMEM = (size_t)(XNP * 4 * XPL + 4 * XTX * XHY + 2 * 5 * XPL) * sizeof(double);
constexpr int XVK = 64;  // slab depth (4 extra planes per slab)

__global__ void __launch_bounds__(XTX * XTY, 1) k_visc_exp_tiled(const double *__restrict__ U,
                                                              const double *__restrict__ M,
                                                              const double *__restrict__ M2,
                                                              double *__restrict__ R, int64_t rcs, Lay L,
                                                              const Phys ph) {
    extern __shared__ double xsm[];
    double *ring = xsm;                     // [slot][field][XPL]
    double *dI = xsm + XNP * 4 * XPL;       // [field][XHY][XTX]: D4_i at the own columns, halo rows
    double *ust = dI + 4 * XTX * XHY;       // [2][comp][XPL]: U of the next plane, cp.async one plane ahead
    const int tid = threadIdx.x, tx = tid % XTX, ty = tid / XTX;
    const int tilesx = (L.n0 + XTX - 1) / XTX, tilesy = (L.n1 + XTY - 1) / XTY;
    int b = blockIdx.x;
    const int bx = b % tilesx;
    b /= tilesx;
    const int by = b % tilesy, bz = b / tilesy;
    const int i0 = bx * XTX, j0 = by * XTY;
    const int z0 = bz * XVK, z1 = min(z0 + XVK, L.n2);
    const int i = i0 + tx, j = j0 + ty;
    const bool own = i < L.n0 && j < L.n1;
    const double iR = 1.0 / ph.R;
    auto slot = [&](int k) { return ring + ((k + 2 * XNP) % XNP) * 4 * XPL; };
    auto stage_plane = [&](int k) {  // cp.async of U of plane k on the halo'd tile (clamped into the box)
        double *us = ust + (k & 1) * 5 * XPL;
        for (int p = tid; p < XPL; p += XTX * XTY) {
            const int hx = p % XHX, hy = p / XHX;
            const int gi = min(i0 - 2 + hx, L.n0 + G - 1), gj = min(j0 - 2 + hy, L.n1 + G - 1);
            const int64_t q = at(L, gi, gj, k);
#pragma unroll
            for (int c = 0; c < 5; c++) {
                const unsigned d = (unsigned)__cvta_generic_to_shared(us + c * XPL + p);
                asm volatile("cp.async.ca.shared.global [%0], [%1], 8;\n" ::"r"(d), "l"(U + c * L.cs + q) : "memory");
            }
        }
        asm volatile("cp.async.commit_group;\n" ::: "memory");
    };
    auto load_plane = [&](int k) {  // u v w T of plane k on the halo'd tile from the staged U (own copies)
        double *pl = slot(k);
        const double *us = ust + (k & 1) * 5 * XPL;
        for (int p = tid; p < XPL; p += XTX * XTY) {
            const double rho = us[p], ir = 1.0 / rho;
            const double u = us[XPL + p] * ir, v = us[2 * XPL + p] * ir, w = us[3 * XPL + p] * ir;
            const double pr = ph.gm1 * (us[4 * XPL + p] - 0.5 * rho * (u * u + v * v + w * w));
            pl[p] = u;
            pl[XPL + p] = v;
            pl[2 * XPL + p] = w;
            pl[3 * XPL + p] = pr * ir / ph.R;
        }
    };
    (void)iR;
    auto d4 = [](double m2, double m1, double p1, double p2) {
        return (8.0 * (p1 - m1) - (p2 - m2)) * (1.0 / 12.0);
    };
    auto d2 = [](double m2, double m1, double c, double p1, double p2) {
        return (16.0 * (p1 + m1) - (p2 + m2) - 30.0 * c) * (1.0 / 12.0);
    };
    const int oc = (ty + 2) * XHX + (tx + 2);  // own point in a plane
    double qi[4][5], qj[4][5];                 // D4_i F, D4_j F of the own column, planes k-2 .. k+2
#pragma unroll
    for (int f = 0; f < 4; f++)
#pragma unroll
        for (int o = 0; o < 5; o++) qi[f][o] = qj[f][o] = 0.0;
    stage_plane(z0 - 2);
    for (int kk = z0 - 2; kk <= z1 + 1; kk++) {
        if (kk + 1 <= z1 + 1) {
            stage_plane(kk + 1);
            asm volatile("cp.async.wait_group 1;\n" ::: "memory");  // plane kk landed (this thread's copies)
        } else {
            asm volatile("cp.async.wait_group 0;\n" ::: "memory");
        }
        // this iteration's output plane k = kk - 2: its metrics and second metrics requested first,
        // so their latency overlaps the plane staging and the barriers
        double mv[10], m2v[18];
        const bool outp = kk - 2 >= z0 && own;
        if (outp) {
            const int64_t pq = at(L, i, j, kk - 2);
            const int64_t tq = (int64_t)i + (int64_t)L.n0 * (j + (int64_t)L.n1 * (kk - 2));
#pragma unroll
            for (int c = 0; c < 10; c++) mv[c] = M[c * L.cs + pq];
#pragma unroll
            for (int c = 0; c < 18; c++) m2v[c] = M2[c * rcs + tq];
        }
        load_plane(kk);
        __syncthreads();
        {   // queues: D4_i, D4_j of the own column at plane kk
            const double *pl = slot(kk);
#pragma unroll
            for (int f = 0; f < 4; f++) {
                const double *c = pl + f * XPL + oc;
#pragma unroll
                for (int o = 0; o < 4; o++) {
                    qi[f][o] = qi[f][o + 1];
                    qj[f][o] = qj[f][o + 1];
                }
                qi[f][4] = d4(c[-2], c[-1], c[1], c[2]);
                qj[f][4] = d4(c[-2 * XHX], c[-XHX], c[XHX], c[2 * XHX]);
            }
        }
        const int k = kk - 2;  // output plane (planes k-2 .. k+2 are in the ring)
        if (k < z0) continue;  // (uniform across the CTA)
        {   // D4_i at plane k on the own columns of every halo row
            const double *pl = slot(k);
            for (int p = tid; p < XTX * XHY; p += XTX * XTY) {
                const int cx = p % XTX, hy = p / XTX;
#pragma unroll
                for (int f = 0; f < 4; f++) {
                    const double *c = pl + f * XPL + hy * XHX + cx + 2;
                    dI[f * XTX * XHY + p] = d4(c[-2], c[-1], c[1], c[2]);
                }
            }
        }
        __syncthreads();
        if (!own) continue;
        const int64_t tcomp = (int64_t)i + (int64_t)L.n0 * (j + (int64_t)L.n1 * k);
        const double J = mv[0];
        double xi[3][3];
#pragma unroll
        for (int a = 0; a < 3; a++)
#pragma unroll
            for (int c = 0; c < 3; c++) xi[a][c] = J * mv[1 + 3 * a + c];
        const double *pm2 = slot(k - 2), *pm1 = slot(k - 1), *p0 = slot(k), *pp1 = slot(k + 1), *pp2 = slot(k + 2);
        // computational first derivatives P1[f][a] and second derivatives P2[f][pair] of u, v, w, T
        double P1[4][3], P2[4][6];
#pragma unroll
        for (int f = 0; f < 4; f++) {
            const int o = f * XPL + oc;
            const double *c = p0 + o;
            P1[f][0] = qi[f][2];
            P1[f][1] = qj[f][2];
            P1[f][2] = d4(pm2[o], pm1[o], pp1[o], pp2[o]);
            P2[f][0] = d2(c[-2], c[-1], c[0], c[1], c[2]);
            P2[f][3] = d2(c[-2 * XHX], c[-XHX], c[0], c[XHX], c[2 * XHX]);
            P2[f][5] = d2(pm2[o], pm1[o], c[0], pp1[o], pp2[o]);
            const double *di = dI + f * XTX * XHY + (ty + 2) * XTX + tx;
            P2[f][1] = d4(di[-2 * XTX], di[-XTX], di[XTX], di[2 * XTX]);  // D4_j(D4_i F)
            P2[f][2] = d4(qi[f][0], qi[f][1], qi[f][3], qi[f][4]);         // D4_k(D4_i F)
            P2[f][4] = d4(qj[f][0], qj[f][1], qj[f][3], qj[f][4]);         // D4_k(D4_j F)
        }
        double gx[4][3], hx[4][6];
#pragma unroll
        for (int f = 0; f < 4; f++)
#pragma unroll
            for (int cc = 0; cc < 3; cc++) gx[f][cc] = xi[0][cc] * P1[f][0] + xi[1][cc] * P1[f][1] + xi[2][cc] * P1[f][2];
        // d2/dx_j dx_k = sum_ab xi_{a,j} xi_{b,k} phi_ab + sum_a xi_{a,jk} phi_a, the symmetric phi_ab
        // grouped into the 6 computational pairs (coefficients shared by the four fields)
#pragma unroll
        for (int q = 0; q < 6; q++) {
            const int jj = q < 3 ? 0 : (q < 5 ? 1 : 2);
            const int kq = q < 3 ? q : (q < 5 ? q - 2 : 2);
            double w[6];
#pragma unroll
            for (int u = 0; u < 6; u++) {
                const int a = u < 3 ? 0 : (u < 5 ? 1 : 2);
                const int cc = u < 3 ? u : (u < 5 ? u - 2 : 2);
                w[u] = a == cc ? xi[a][jj] * xi[a][kq] : fma(xi[a][jj], xi[cc][kq], xi[cc][jj] * xi[a][kq]);
            }
            double m2[3];
#pragma unroll
            for (int a = 0; a < 3; a++) m2[a] = m2v[6 * a + q];
#pragma unroll
            for (int f = 0; f < 4; f++) {
                if (f == 3 && (q == 1 || q == 2 || q == 4)) {  // T: only the Laplacian is used
                    hx[f][q] = 0.0;
                    continue;
                }
                double sm = m2[0] * P1[f][0];
                sm = fma(m2[1], P1[f][1], sm);
                sm = fma(m2[2], P1[f][2], sm);
#pragma unroll
                for (int u = 0; u < 6; u++) sm = fma(w[u], P2[f][u], sm);
                hx[f][q] = sm;
            }
        }
        const double T = p0[3 * XPL + oc];
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
            double sm = mu * (lap + gdiv * (1.0 / 3.0));
#pragma unroll
            for (int cc = 0; cc < 3; cc++) {
                double sym = gx[a][cc] + gx[cc][a];
                if (a == cc) sym -= (2.0 / 3.0) * div;
                sm += mup * gx[3][cc] * sym;
            }
            dtau[a] = sm;
        }
        const double u = p0[oc], v = p0[XPL + oc], w = p0[2 * XPL + oc];
        double diss = 0.0;
#pragma unroll
        for (int a = 0; a < 3; a++)
#pragma unroll
            for (int cc = 0; cc < 3; cc++) {
                double tau = mu * (gx[a][cc] + gx[cc][a]);
                if (a == cc) tau -= (2.0 / 3.0) * mu * div;
                diss += tau * gx[a][cc];
            }
        const double lapT = hx[3][0] + hx[3][3] + hx[3][5];
        const double gT2 = gx[3][0] * gx[3][0] + gx[3][1] * gx[3][1] + gx[3][2] * gx[3][2];
        const double VE = u * dtau[0] + v * dtau[1] + w * dtau[2] + diss + ph.cp_over_Pr * (mu * lapT + mup * gT2);
        const double iJ = 1.0 / J;
        R[1 * rcs + tcomp] = dtau[0] * iJ;
        R[2 * rcs + tcomp] = dtau[1] * iJ;
        R[3 * rcs + tcomp] = dtau[2] * iJ;
        R[4 * rcs + tcomp] = VE * iJ;
    }
}

}  // namespace crocco
