// relative error of rcp.approx.ftz.f64 / rsqrt.approx.ftz.f64 (MUFU.RCP64H / RSQ64H) and of
// 1 / 2 Newton steps, over log-uniform positive inputs; max over 2^24 samples
#include <cstdio>
#include <cmath>
__device__ unsigned long long h(unsigned long long x) { x ^= x >> 33; x *= 0xff51afd7ed558ccdULL; x ^= x >> 33; x *= 0xc4ceb9fe1a85ec53ULL; x ^= x >> 33; return x; }
__global__ void k(double *out) {
  double e[6] = {0,0,0,0,0,0};
  for (int it = 0; it < 64; it++) {
    unsigned long long t = (unsigned long long)(blockIdx.x * blockDim.x + threadIdx.x) * 64 + it;
    double u = (h(t) >> 11) * (1.0 / 9007199254740992.0);
    double y = exp2(-200.0 + 400.0 * u);
    double r; asm("rcp.approx.ftz.f64 %0, %1;" : "=d"(r) : "d"(y));
    double ex = 1.0 / y;
    e[0] = fmax(e[0], fabs(r - ex) / ex);
    double r1 = fma(r, fma(-y, r, 1.0), r);
    e[1] = fmax(e[1], fabs(r1 - ex) / ex);
    double q = 3.7 * r1; double q1 = fma(r1, fma(-y, q, 3.7), q); double exq = 3.7 / y;
    e[2] = fmax(e[2], fabs(q1 - exq) / exq);
    double s; asm("rsqrt.approx.ftz.f64 %0, %1;" : "=d"(s) : "d"(y));
    double exs = 1.0 / sqrt(y);
    e[3] = fmax(e[3], fabs(s - exs) / exs);
    double hh = 0.5 * y; double s1 = s * fma(-hh * s, s, 1.5);
    e[4] = fmax(e[4], fabs(s1 - exs) / exs);
    double s2 = s1 * fma(-hh * s1, s1, 1.5);
    e[5] = fmax(e[5], fabs(s2 - exs) / exs);
  }
  for (int i = 0; i < 6; i++) atomicMax((unsigned long long *)&out[i], (unsigned long long)__double_as_longlong(e[i]));
}
int main() {
  double *d; cudaMalloc(&d, 6 * sizeof(double)); cudaMemset(d, 0, 6 * sizeof(double));
  k<<<1024, 256>>>(d); double hst[6]; cudaMemcpy(hst, d, sizeof hst, cudaMemcpyDeviceToHost);
  const char *nm[6] = {"rcp_approx", "rcp_1newton", "div_1newton_corr", "rsqrt_approx", "rsqrt_1newton", "rsqrt_2newton"};
  for (int i = 0; i < 6; i++) printf("%-18s max rel err %.3e (2^%.1f)\n", nm[i], hst[i], log2(hst[i] + 1e-300));
}
