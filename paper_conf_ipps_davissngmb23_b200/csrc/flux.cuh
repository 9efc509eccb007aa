// flux.cuh -- total interface flux of one direction: characteristic WENO-SYMBO
// inviscid flux (WENOx/y/z; readings 8-11) minus the
// viscous interface flux whose difference is the 4th-order central divergence
// (Viscous; reading 12).
//
// Inviscid part at interface i+1/2 of direction d, from the points i-2..i+3:
//   m^ = R6(m^d) = (m_{i-2} - 8m_{i-1} + 37m_i + 37m_{i+1} - 8m_{i+2} + m_{i+3})/60,
//   n = m^/|m^|; Roe state of (i, i+1); Pulliam-Chaussee T, T^-1 for n;
//   g_{s,l} = L_s.F_n(U_l), w_{s,l} = L_s.U_l, lambda_s = max_l |eig_s(l)|,
//   g^_s = W(g+lambda w) + W_mirror(g-lambda w)  [the 1/2 of the LLF split is
//   folded: W(v/2; eps) = W(v; 4 eps)/2, so the sum is halved at the end],
//   F^ = |m^| T g^.
// L_s.F_n(U_l) is evaluated as theta_l (L_s.U_l) + p_l k_{s,l} using the exact
// identity F_n(U) = theta U + p (0, n, theta); for the entropy / vorticity fields
// (k = ng (theta~ - theta_l)) the per-point products pm_l = p_l (theta~ - theta_l) are formed once
// and shared by the three fields (acoustic fields first in the field loop).
// Viscous part: with the point fluxes f = F^_v^d (k_visc),
//   h_{i+1/2} = [7(f_i + f_{i+1}) - (f_{i-1} + f_{i+2})]/12,
//   h_{i+1/2} - h_{i-1/2} = D4 f_i  (exactly, in exact arithmetic).
#pragma once
#include "common.cuh"
#include "weno.cuh"

namespace crocco {

// bit D: the three 6-point maxima of direction D as depth-3 trees instead of 6-deep chains (bitwise
// equal); round 1: zeta only (zeta -0.2 ms, xi +0.3 ms); on the final round-2 kernels all three
// directions (with the shared-memory flux carry, sweep.cuh)
constexpr int LAM_TREE = 7;

struct FluxIn {
    const double *__restrict__ U;
    const double *__restrict__ M;
    const double *__restrict__ FV;  // point viscous fluxes of this direction (4 comps) or null
    int64_t cs;                     // component stride of U / M
    int64_t vcs;                    // component stride of FV
};

// Stencil accessor (SAcc): conserved state U(l, c), primitives P(l, k) (k = PU..PH),
// the metric row m^d M(l, a) and the point viscous flux of direction d FV(l, q)
// (q = momentum x, y, z, energy) at stencil point l = 0..5 (points i-2..i+3).
// shared-memory ring of a warp: value v of ring point q in column col at
// sv[v * VS + (q & (NR-1)) * PS + col]; values: U (5), metric row (3), [F^_v (4) when the
// sweep carries a viscous term], primitives (7)
enum { SV_U = 0, SV_M = 5, SV_FV = 8 };
__host__ __device__ constexpr int sv_p(bool visc) { return visc ? 12 : 8; }   // first primitive
__host__ __device__ constexpr int sv_n(bool visc) { return sv_p(visc) + 7; }  // values per point
// CS = 0: point-major slots (q & (NR-1)) * PS + col (eta / zeta: a chunk of points is contiguous per
// column row); CS > 0: column-major col * CS + (q & (NR-1)) (xi: consecutive points of a line
// contiguous, CS padded so a warp's 32 reads take the minimum two wavefronts)
template <int NR, int PS, bool VISC, int CS = 0>
struct SAcc {
    static constexpr int SV_P = sv_p(VISC);
    const double *sv;
    int q0, col;
    static constexpr int VS = CS ? PS * CS : NR * PS;
    __device__ __forceinline__ double at_(int v, int l) const {
        if constexpr (CS != 0) return sv[v * VS + col * CS + ((q0 + l) & (NR - 1))];
        else return sv[v * VS + ((q0 + l) & (NR - 1)) * PS + col];
    }
    __device__ __forceinline__ double U(int l, int c) const { return at_(SV_U + c, l); }
    __device__ __forceinline__ double P(int l, int k) const { return at_(SV_P + k, l); }
    __device__ __forceinline__ double M(int l, int a) const { return at_(SV_M + a, l); }
    __device__ __forceinline__ double FV(int l, int q) const { return at_(SV_FV + q, l); }
    __device__ __forceinline__ double IS(int l) const { return P(l, PIS); }  // 1/sqrt(rho)
    __device__ __forceinline__ double H(int l) const { return P(l, PH); }    // total enthalpy
};

// Interface quantities that need no primitive of the outermost stencil points: frozen
// metric, normal and |m^|/2 (R6 of the staged metric rows) and the Roe state of points i,
// i+1 with the eigenvector scalars.  k_sweep_s evaluates them before it stores the newest
// chunk's primitives (independent chains for the scheduler), then calls flux_fields.
struct FluxSetup {
    double nx, ny, nz, hmag;           // unit normal, |m^|/2 (LLF 1/2 folded here)
    double ut, vt, wt, rt, irt;        // Roe velocity, density and its reciprocal
    double ct, c2, ic2, ict, tht, phi2;  // Roe sound speed, c^2, 1/c^2, 1/c, n.u~, (gamma-1)|u~|^2/2
};
template <class Acc>
__device__ __forceinline__ void flux_setup(const Acc &A, const Phys &ph, FluxSetup &su) {
    const double gm1 = ph.gm1;
    double mh[3];
#pragma unroll
    for (int a = 0; a < 3; a++)
        mh[a] = fma(37.0, A.M(2, a) + A.M(3, a), fma(-8.0, A.M(1, a) + A.M(4, a), A.M(0, a) + A.M(5, a))) *
                (1.0 / 60.0);
    const double s2 = fma(mh[0], mh[0], fma(mh[1], mh[1], mh[2] * mh[2]));
    const double imag = rsqrt_nr(s2);
    su.hmag = 0.5 * s2 * imag;
    const double nx = mh[0] * imag, ny = mh[1] * imag, nz = mh[2] * imag;
    su.nx = nx;
    su.ny = ny;
    su.nz = nz;

    // Roe average of points i (l=2), i+1 (l=3), sqrt(rho) weights
    const double isL = A.IS(2), isR = A.IS(3);
    const double srL = A.U(2, 0) * isL, srR = A.U(3, 0) * isR;
    const double iden = rcp_nr(srL + srR);
    const double wL = srL * iden, wR = srR * iden;
    const double ut = fma(wL, A.P(2, PU), wR * A.P(3, PU));
    const double vt = fma(wL, A.P(2, PV), wR * A.P(3, PV));
    const double wt = fma(wL, A.P(2, PW), wR * A.P(3, PW));
    const double Ht = fma(wL, A.H(2), wR * A.H(3));
    const double rt = srL * srR;
    const double q2 = fma(ut, ut, fma(vt, vt, wt * wt));
    const double c2 = gm1 * fma(-0.5, q2, Ht);
    const double ict = rsqrt_nr(c2);
    const double irt = isL * isR;  // 1/rho~
    su.ut = ut;
    su.vt = vt;
    su.wt = wt;
    su.rt = rt;
    su.irt = irt;
    su.c2 = c2;
    su.ct = c2 * ict;
    su.ic2 = ict * ict;
    su.tht = fma(nx, ut, fma(ny, vt, nz * wt));
    su.phi2 = 0.5 * gm1 * q2;
    su.ict = ict;
}

// Total interface flux F = F^_inv - h_v of direction D at interface i+1/2 from the setup above.
// A: stencil accessor (SAcc).
template <int D, class Acc, bool LIM = false>
__device__ __forceinline__ void flux_fields(const Acc &A, const FluxSetup &su, bool inv, bool visc,
                                            const Phys &ph, double F[5]) {
    F[0] = F[1] = F[2] = F[3] = F[4] = 0.0;
    if (inv) {
        const double gm1 = ph.gm1;
        const double nx = su.nx, ny = su.ny, nz = su.nz, hmag = su.hmag;
        const double ut = su.ut, vt = su.vt, wt = su.wt, rt = su.rt, irt = su.irt;
        const double ct = su.ct, c2 = su.c2, ic2 = su.ic2, ict = su.ict, tht = su.tht, phi2 = su.phi2;

        // stencil points (the states are re-read from the ring per field: holding the 6 x 5
        // states in registers measured slower)
#define UL(l, c) A.U(l, c)
        double th[6], pl[6];
        double lam0 = 0.0, lam3 = 0.0, lam4 = 0.0;
        constexpr bool lam_tree = (LAM_TREE >> D) & 1;
        double a0[6], a3[6], a4[6];
#pragma unroll
        for (int l = 0; l < 6; l++) {
            const double t = fma(nx, A.P(l, PU), fma(ny, A.P(l, PV), nz * A.P(l, PW)));
            const double cl = A.P(l, PC);
            th[l] = t;
            pl[l] = A.P(l, PP);
            if constexpr (lam_tree) {
                a0[l] = fabs(t);
                a3[l] = fabs(t + cl);
                a4[l] = fabs(t - cl);
            } else {
                lam0 = maxnn(lam0, fabs(t));
                lam3 = maxnn(lam3, fabs(t + cl));
                lam4 = maxnn(lam4, fabs(t - cl));
            }
        }
        if constexpr (lam_tree) {
            lam0 = maxnn(maxnn(maxnn(a0[0], a0[1]), maxnn(a0[2], a0[3])), maxnn(a0[4], a0[5]));
            lam3 = maxnn(maxnn(maxnn(a3[0], a3[1]), maxnn(a3[2], a3[3])), maxnn(a3[4], a3[5]));
            lam4 = maxnn(maxnn(maxnn(a4[0], a4[1]), maxnn(a4[2], a4[3])), maxnn(a4[4], a4[5]));
        }
        const double eps_b = 4.0 * WENO_BSCALE * ph.eps;  // b-units (weno.cuh) x 4 (folded 1/2)
        // acoustic rows are used as L_s / beta, beta = 1/(sqrt2 rho~ c~): W is homogeneous,
        // W(v; eps) = beta W(v / beta; eps / beta^2), so those fields take eps (and the absolute
        // limiter threshold) times 1/beta^2 = 2 rho~^2 c~^2; the factor beta returns in the back projection
        const double ib2 = (2.0 * rt * rt) * c2;
        const double epsA = eps_b * ib2;
        const double onemp = fma(-phi2, ic2, 1.0);
        const double gic2 = gm1 * ic2;
        const double cx = ny * wt - nz * vt, cy = nz * ut - nx * wt, cz = nx * vt - ny * ut;
        const double ph1 = phi2 * ph.igm1;
        double f0 = 0.0, f1 = 0.0, f2 = 0.0, f3 = 0.0, f4 = 0.0;
        // the five WENO-pair divisions are issued after the field loop (independent chains;
        // inside the loop measured slower); the loop is unrolled (rolled: +14 %)
        double gb[5], gn[5], gd[5];
#pragma unroll
        for (int it = 0; it < 5; it++) {
            // acoustic fields first; then p_l becomes pm_l = p_l (theta~ - theta_l), so the
            // entropy / vorticity fields' p_l (kB theta_l + kA) = ng pm_l (kA = ng theta~, kB = -ng)
            const int sf = it < 2 ? it + 3 : it - 2;
            if (it == 2) {
#pragma unroll
                for (int l = 0; l < 6; l++) pl[l] *= tht - th[l];
            }
            double L0, L1, L2, L3, L4, lam, kA, kB;
            if (sf < 3) {
                const double na = sf == 0 ? nx : (sf == 1 ? ny : nz);
                const double cr = sf == 0 ? cx : (sf == 1 ? cy : cz);
                const double ng = na * gic2;
                L0 = fma(na, onemp, cr * irt);
                if (sf == 0) {
                    L1 = ng * ut;
                    L2 = fma(nz, irt, ng * vt);
                    L3 = fma(-ny, irt, ng * wt);
                } else if (sf == 1) {
                    L1 = fma(-nz, irt, ng * ut);
                    L2 = ng * vt;
                    L3 = fma(nx, irt, ng * wt);
                } else {
                    L1 = fma(ny, irt, ng * ut);
                    L2 = fma(-nx, irt, ng * vt);
                    L3 = ng * wt;
                }
                L4 = -ng;
                lam = lam0;
                kA = ng * tht;
                kB = -ng;
            } else {
                const double sc = (sf == 3) ? ct : -ct;
                L0 = fma(-sc, tht, phi2);
                L1 = fma(sc, nx, -gm1 * ut);
                L2 = fma(sc, ny, -gm1 * vt);
                L3 = fma(sc, nz, -gm1 * wt);
                L4 = gm1;
                lam = (sf == 3) ? lam3 : lam4;
                kA = fma(-gm1, tht, sc);
                kB = gm1;
            }
            double gp[6], gm[6];
#pragma unroll
            for (int l = 0; l < 6; l++) {
                const double w =
                    fma(L0, UL(l, 0), fma(L1, UL(l, 1), fma(L2, UL(l, 2), fma(L3, UL(l, 3), L4 * UL(l, 4)))));
                const double g = sf < 3 ? fma(th[l], w, -kB * pl[l]) : fma(th[l], w, pl[l] * fma(kB, th[l], kA));
                gp[l] = fma(lam, w, g);
                gm[l] = fma(-lam, w, g);
            }
            const WenoFrac wf = sf < 3 ? weno_pair_frac<LIM>(gp, gm, eps_b, ph.wC, &ph, ph.aal_b)
                                       : weno_pair_frac<LIM>(gp, gm, epsA, ph.wC, &ph, ph.aal_b * ib2);
            gb[sf] = wf.base;
            gn[sf] = wf.num;
            gd[sf] = wf.den;
        }
        double gh[5];
#pragma unroll
        for (int sf = 0; sf < 5; sf++) gh[sf] = fma(div_nr(gn[sf], gd[sf]), 1.0 / 6.0, gb[sf]);
        // back projection F^/|m^| = sum_s gh_s R_s in closed form (the right eigenvectors R_s of
        // the columns written out above, summed symbolically):
        //   entropy / vorticity fields, G = (gh_0, gh_1, gh_2), s = n.G, c = rho~ (n x G):
        //     (s, u~ s + c, |u~|^2/2 s + u~.c)
        //   acoustic pair, S = alpha (gh_3 + gh_4), Dd = alpha c~ (gh_3 - gh_4), with alpha = rho~/(sqrt2 c~)
        //   and gh_{3,4} = beta x (the values computed from L_s / beta): alpha beta = 1/(2 c~^2):
        //     S (1, u~, H~) + Dd (0, n, n.u~),  H~ = (phi2 + c~^2)/(gamma-1)
        {
            const double sG = fma(nx, gh[0], fma(ny, gh[1], nz * gh[2]));
            const double cgx = rt * fma(ny, gh[2], -nz * gh[1]);
            const double cgy = rt * fma(nz, gh[0], -nx * gh[2]);
            const double cgz = rt * fma(nx, gh[1], -ny * gh[0]);
            const double S = (0.5 * ic2) * (gh[3] + gh[4]);
            const double Dd = (0.5 * ict) * (gh[3] - gh[4]);
            const double Ht = (phi2 + c2) * ph.igm1;
            const double sS = sG + S;
            f0 = sS;
            f1 = fma(ut, sS, fma(Dd, nx, cgx));
            f2 = fma(vt, sS, fma(Dd, ny, cgy));
            f3 = fma(wt, sS, fma(Dd, nz, cgz));
            f4 = fma(ph1, sG, fma(ut, cgx, fma(vt, cgy, fma(wt, cgz, fma(S, Ht, Dd * tht)))));
        }
#undef UL
        F[0] = hmag * f0;
        F[1] = hmag * f1;
        F[2] = hmag * f2;
        F[3] = hmag * f3;
        F[4] = hmag * f4;
    }
    if (visc) {
        // h_{i+1/2} = [7(f_i + f_{i+1}) - (f_{i-1} + f_{i+2})]/12 for momentum x,y,z and energy
#pragma unroll
        for (int q = 0; q < 4; q++) {
            const double h = fma(7.0, A.FV(2, q) + A.FV(3, q), -(A.FV(1, q) + A.FV(4, q))) * (1.0 / 12.0);
            F[1 + q] -= h;
        }
    }
}

}  // namespace crocco
