// common.cuh -- shared PODs, layouts and constants of the libcrocco kernels.
// All arithmetic in libcrocco is fp64 on the CUDA-core FP64 pipe (the path is a
// nonlinear stencil, not a contraction, so no tensor cores).  FMA contraction
// is on; parity with the non-contracted oracle is tested to 1e-11.
#pragma once
#include <cstdint>

namespace crocco {

constexpr int G = 4;    // state / metric ghost width (reading 7)
constexpr int GC = 10;  // coordinate ghost width (reading 7)

struct Phys {
    double gamma, gm1, igm1, R, Pr, cp_over_Pr;  // cp/Pr = gamma R /((gamma-1) Pr)
    int mu_law;
    double mu_ref, T_ref, S, iT_ref;
    double eps;
    int terms, dir_mask;
    double wC[4];  // WENO optimal weights (SYMBO or SYMOO)
    int lim;       // WENO limiters (reading 23): bit 0 relative, bit 1 absolute
    double arl;    // relative threshold (scale-free)
    double aal_b;  // absolute threshold in the units of the kernels' b_k (weno.cuh)
    int visc_form; // 0 conservative point-flux viscous form, 1 expanded form (viscexp.cuh)
};

struct Lay {  // padded block layout (elements)
    int n0, n1, n2;
    int64_t off, py, pz, cs;
};

__host__ __device__ inline int64_t at(const Lay &L, int i, int j, int k) {
    return L.off + (int64_t)i + (int64_t)j * L.py + (int64_t)k * L.pz;
}

struct VLay {  // viscous point-flux box (interior +-2); rows padded to 16 elements
    int b0, b1, b2;
    int64_t py, pz, cs;
};

__host__ __device__ inline int64_t vat(const VLay &V, int i, int j, int k) {
    return (int64_t)(i + 2) + V.py * (j + 2) + V.pz * (k + 2);
}

// Branch-free reciprocal / reciprocal square root: hardware approximation
// (MUFU.RCP64H / MUFU.RSQ64H, relative error <= 2^-20, profiles/r01_approx.txt) + one
// third-order correction (error ~ e^3 <= 2^-60, i.e. rounding level) + (for x/y) one
// residual correction -- used instead of the IEEE div/sqrt sequences, whose slow-path
// branches cost issue slots, and shorter than two Newton steps (3 / 5 dependent FP64
// operations instead of 4 / 6) for the positive, normal-range operands of this path
// (densities, sound speeds, metric norms, WENO weight sums).
__device__ __forceinline__ double rcp_nr(double y) {
    double r;
    asm("rcp.approx.ftz.f64 %0, %1;" : "=d"(r) : "d"(y));
    const double e = fma(-y, r, 1.0);   // y r = 1 - e
    return fma(r, fma(e, e, e), r);     // r (1 + e + e^2) = (1 - e^3)/y
}
// x/y: one Newton step on the 2^-20 hardware reciprocal (2^-40) then the residual
// correction q + r (x - y q), which is (near) correctly rounded -- measured exact on
// 2^24 log-uniform samples (tools/approx_acc.cu, profiles/r01_approx.txt)
__device__ __forceinline__ double div_nr(double x, double y) {
    double r;
    asm("rcp.approx.ftz.f64 %0, %1;" : "=d"(r) : "d"(y));
    r = fma(r, fma(-y, r, 1.0), r);
    const double q = x * r;
    return fma(r, fma(-y, q, x), q);
}
__device__ __forceinline__ double rsqrt_nr(double x) {
    double r;
    asm("rsqrt.approx.ftz.f64 %0, %1;" : "=d"(r) : "d"(x));
    const double e = fma(-x * r, r, 1.0);           // x r^2 = 1 - e
    return fma(r * e, fma(0.375, e, 0.5), r);       // r (1 + e/2 + 3 e^2/8) = x^-1/2 (1 + O(e^3))
}
__device__ __forceinline__ double sqrt_nr(double x) {  // x > 0
    const double r = rsqrt_nr(x);
    const double s = x * r;
    return fma(0.5 * r, fma(-s, s, x), s);  // one Newton correction of s
}

// max / min of two non-negative finite doubles: one DSETP.MAX + selects.  (Round 1 compared the
// bit patterns on the integer pipe -- ISETP.U32 + ISETP.EX + 2 SEL per maximum; round 2 measured
// the FP64 compare 0.33 ms per 512^3 stage faster, bitwise the same results: the LLF speeds and
// the WENO-SYMBO downwind maxima are on the critical path, and the integer pair is the longer
// chain.)
__device__ __forceinline__ double maxnn(double a, double b) { return a > b ? a : b; }
__device__ __forceinline__ double minnn(double a, double b) { return a < b ? a : b; }

// asynchronous global -> shared copies (sm_80+ cp.async; the sweeps' rings, the viscous kernels' staging)
__device__ __forceinline__ void cp_async8(double *dst, const double *src) {
    const unsigned d = (unsigned)__cvta_generic_to_shared(dst);
    asm volatile("cp.async.ca.shared.global [%0], [%1], 8;\n" ::"r"(d), "l"(src) : "memory");
}
__device__ __forceinline__ void cp_async16(double *dst, const double *src) {
    const unsigned d = (unsigned)__cvta_generic_to_shared(dst);
    asm volatile("cp.async.cg.shared.global [%0], [%1], 16;\n" ::"r"(d), "l"(src) : "memory");
}
// predicated forms: when !ok nothing is read (src-size 0; the caller still passes a valid address)
// and the destination is zero-filled -- no branch around the copy
__device__ __forceinline__ void cp_async8z(double *dst, const double *src, bool ok) {
    const unsigned d = (unsigned)__cvta_generic_to_shared(dst);
    asm volatile("cp.async.ca.shared.global [%0], [%1], 8, %2;\n" ::"r"(d), "l"(src), "r"(ok ? 8u : 0u) : "memory");
}
__device__ __forceinline__ void cp_async16z(double *dst, const double *src, bool ok) {
    const unsigned d = (unsigned)__cvta_generic_to_shared(dst);
    asm volatile("cp.async.cg.shared.global [%0], [%1], 16, %2;\n" ::"r"(d), "l"(src), "r"(ok ? 16u : 0u) : "memory");
}
__device__ __forceinline__ void cp_async_commit() { asm volatile("cp.async.commit_group;\n" ::: "memory"); }
__device__ __forceinline__ void cp_async_wait_all() { asm volatile("cp.async.wait_group 0;\n" ::: "memory"); }

// primitive components staged per ring point by the sweeps (sweep.cuh)
// (PIS = 1/sqrt(rho): the Roe weights use sqrt(rho) = rho / sqrt(rho), 1/rho~ = PIS_L PIS_R)
enum { PU = 0, PV = 1, PW = 2, PP = 3, PC = 4, PIS = 5, PH = 6 };

}  // namespace crocco
