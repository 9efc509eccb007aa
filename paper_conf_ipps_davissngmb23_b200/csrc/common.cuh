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
    double mu_ref, T_ref, S;
    double eps;
    int terms, dir_mask;
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

// primitive buffer components (k_prims)
enum { PU = 0, PV = 1, PW = 2, PP = 3, PC = 4, PSR = 5, PH = 6, PT = 7, NPRIM = 8 };

}  // namespace crocco
