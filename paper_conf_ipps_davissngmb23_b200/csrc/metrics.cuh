// metrics.cuh -- grid metrics and Jacobian (InitGridMetrics).
// Part of libcrocco (sm_100a, fp64). Formulas restate the paper's method as
// read in DESIGN.md sec. 3 (citations: PAPER.md line numbers); no code is
// shared with oracle/.
#pragma once
#include "common.cuh"

namespace crocco {

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
