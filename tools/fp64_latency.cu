// DFMA throughput vs (warps per SM, independent chains per thread): how much ILP the
// FP64 pipe needs on B200 (informs the sweep-kernel occupancy/ILP trade-off)
#include <cstdio>
template <int ILP>
__global__ void k(double *out, int iters, double a, double b) {
    double x[ILP];
#pragma unroll
    for (int c = 0; c < ILP; c++) x[c] = threadIdx.x + c;
    for (int i = 0; i < iters; i++) {
#pragma unroll
        for (int u = 0; u < 8; u++) {
#pragma unroll
            for (int c = 0; c < ILP; c++) x[c] = fma(x[c], a, b);
        }
    }
    double s = 0;
#pragma unroll
    for (int c = 0; c < ILP; c++) s += x[c];
    out[blockIdx.x * blockDim.x + threadIdx.x] = s;
}
template <int ILP>
void run(double *out, int sms, int warps) {
    int thr = 32 * warps, iters = 20000 / ILP;
    cudaEvent_t e0, e1; cudaEventCreate(&e0); cudaEventCreate(&e1);
    k<ILP><<<sms, thr>>>(out, 10, 0.999999, 1e-7);
    cudaEventRecord(e0);
    k<ILP><<<sms, thr>>>(out, iters, 0.999999, 1e-7);
    cudaEventRecord(e1); cudaEventSynchronize(e1);
    float ms; cudaEventElapsedTime(&ms, e0, e1);
    double fmas_per_sm_clk = (double)thr * iters * 8 * ILP / (ms * 1e-3 * 1.965e9);
    printf("warps/SM %2d ILP %d: %.1f DFMA/clk/SM\n", warps, ILP, fmas_per_sm_clk);
}
int main() {
    int sms; cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
    double *out; cudaMalloc(&out, sizeof(double) * sms * 1024);
    for (int w : {4, 8, 12, 16}) { run<1>(out, sms, w); run<2>(out, sms, w); run<4>(out, sms, w); run<8>(out, sms, w); }
}
