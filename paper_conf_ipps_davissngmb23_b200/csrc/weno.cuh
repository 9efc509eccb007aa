// weno.cuh -- WENO-SYMBO reconstruction (PAPER.md:50 -> ref [9]; reading 8).
//
// W(v_{-2..3}) reconstructs the value at the +1/2 interface from 4 candidate
// (optimal weights C: SYMBO by default, SYMOO selectable, reading 22)
// 3-point stencils (the 4th one downwind), Jiang-Shu smoothness indicators with
// beta_3 <- max(beta_0..beta_3), weights alpha_k = C_k/(eps+beta_k)^2.
//
// Evaluated in difference form (algebraically identical):
//   d_m = v_{m-1} - v_{m-2}  (d0 = v_{-1}-v_{-2}, ..., d4 = v_3-v_2)
//   q_k = v_0 + r_k/6, r = (5d1-2d0, d1+2d2, 4d2-d3, 6d2-5d3+2d4)
//   (12/13) beta_k = b_k = s_k^2 + (3/13) f_k^2, s = second differences,
//   f = one-sided first differences (3d1-d0, d1+d2, d3-3d2, 5d3-3d4)
//   alpha_k ~ C_k prod_{m != k} (lam eps + b_m)^2 with lam = 12/13   (one division)
// so W = v_0 + num/(6 den), num = sum alpha_k r_k, den = sum alpha_k.
// Callers pass eps_b = the epsilon in the units of b (see flux.cuh).
#pragma once
#include "common.cuh"

namespace crocco {

constexpr double WENO_BSCALE = 12.0 / 13.0;  // b_k = WENO_BSCALE * beta_k

struct WenoFrac {
    double base, num, den;  // W = base + num/(6 den)
};

// The host passes C / C0 (the weights' ratios are all that
// enter W), so alpha_0 needs no multiply, and e_k = eps + b_k is formed inside the
// FMA chain of b_k; max_k(eps + b_k) = eps + max_k b_k (monotone), so the
// downwind-stencil rule is unchanged.
// LIM: the limiters of reading 23 (ph.lim / ph.arl / ph.aal_b, common.cuh): linear weights
// alpha_k = C_k when max b < arl min b (bit 0) or max b < aal_b (bit 1), b after the
// downwind substitution; aal: the absolute threshold in the units of b of the values passed (the
// caller scales it with the values, see flux.cuh)
template <bool LIM = false>
__device__ __forceinline__ WenoFrac weno_symbo_frac(double v0, double v1, double v2, double v3,
                                                    double v4, double v5, double eps_b,
                                                    const double C[4], const Phys *lp = nullptr,
                                                    double aal = 0.0) {
    const double C0 = C[0], C1 = C[1], C2 = C[2], C3 = C[3];
    constexpr double K3 = 3.0 / 13.0;
    const double d0 = v1 - v0, d1 = v2 - v1, d2 = v3 - v2, d3 = v4 - v3, d4 = v5 - v4;
    const double s0 = d1 - d0, s1 = d2 - d1, s2 = d3 - d2, s3 = d4 - d3;
    const double f0 = fma(3.0, d1, -d0);
    const double f1 = d1 + d2;
    const double f2 = fma(-3.0, d2, d3);
    const double f3 = fma(5.0, d3, -3.0 * d4);
    const double r0 = fma(2.0, f0, -d1);         // 5 d1 - 2 d0
    const double r1 = fma(2.0, d2, d1);
    const double r2 = fma(4.0, d2, -d3);
    const double r3 = fma(6.0, d2, -f3) - d4;    // 6 d2 - 5 d3 + 2 d4
    bool lin = false;
    double e0, e1, e2, e3;
    if constexpr (LIM) {
        const double b0 = fma(K3 * f0, f0, s0 * s0);
        const double b1 = fma(K3 * f1, f1, s1 * s1);
        const double b2 = fma(K3 * f2, f2, s2 * s2);
        double b3 = fma(K3 * f3, f3, s3 * s3);
        b3 = maxnn(maxnn(b0, b1), maxnn(b2, b3));
        const double bmin = minnn(minnn(b0, b1), b2);  // b3 is the maximum
        lin = ((lp->lim & 1) && b3 < lp->arl * bmin) || ((lp->lim & 2) && b3 < aal);
        e0 = eps_b + b0;
        e1 = eps_b + b1;
        e2 = eps_b + b2;
        e3 = eps_b + b3;
    } else {
        // eps folded into the FMA chain of the smoothness indicators
        e0 = fma(s0, s0, fma(K3 * f0, f0, eps_b));
        e1 = fma(s1, s1, fma(K3 * f1, f1, eps_b));
        e2 = fma(s2, s2, fma(K3 * f2, f2, eps_b));
        e3 = fma(s3, s3, fma(K3 * f3, f3, eps_b));
        // downwind stencil never preferred (continuous max, parity-safe)
        e3 = maxnn(maxnn(e0, e1), maxnn(e2, e3));
    }
    e0 *= e0;
    e1 *= e1;
    e2 *= e2;
    e3 *= e3;
    // alpha_0 = C0 e1 e2 e3, alpha_1 = C1 e0 e2 e3, alpha_2 = C2 e0 e1 e3, alpha_3 = C3 e0 e1 e2
    double e01 = e0 * e1, e23 = e2 * e3;
    double x0 = e1;  // C0 = 1 (the host normalises C)
    double x1 = C1 * e0, x2 = C2 * e3, x3 = C3 * e2;
    if constexpr (LIM) {
        if (lin) {  // linear optimal weights: alpha_k = C_k
            x0 = C0;
            x1 = C1;
            x2 = C2;
            x3 = C3;
            e01 = e23 = 1.0;
        }
    }
    WenoFrac w;
    w.base = v2;
    w.num = fma(e23, fma(x0, r0, x1 * r1), e01 * fma(x2, r2, x3 * r3));
    w.den = fma(e23, x0 + x1, e01 * (x2 + x3));
    return w;
}

// W^+ of (vp0..vp5) plus W^- of the mirrored (vm5..vm0), as one fraction:
// (b+ + b-) + [(n+ d- + n- d+)/(d+ d-)]/6  -- one division per characteristic field; the pair's
// den is d+ d- (the 1/6 enters the caller's final FMA, one multiply less than 6 (d+ d-)).
// Range: the alpha products stay inside fp64 for |v| up to ~1e9.
template <bool LIM = false>
__device__ __forceinline__ WenoFrac weno_pair_frac(const double vp[6], const double vm[6], double eps_b,
                                                   const double C[4], const Phys *lp = nullptr, double aal = 0.0) {
    const WenoFrac a = weno_symbo_frac<LIM>(vp[0], vp[1], vp[2], vp[3], vp[4], vp[5], eps_b, C, lp, aal);
    const WenoFrac b = weno_symbo_frac<LIM>(vm[5], vm[4], vm[3], vm[2], vm[1], vm[0], eps_b, C, lp, aal);
    WenoFrac w;
    w.base = a.base + b.base;
    w.num = fma(a.num, b.den, b.num * a.den);
    w.den = a.den * b.den;  // the 1/6 is applied by the caller: W = base + (num/den)/6
    return w;
}
}  // namespace crocco
