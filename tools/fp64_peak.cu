// FP64 (non-tensor) DFMA throughput microbenchmark for the roofline peak.
// 148 SMs x N warps, 8 independent DFMA chains per thread; reports TFLOP/s (FMA = 2 flop).
#include <cstdio>
#include <cuda_runtime.h>
__global__ void k(double *out, int iters, double a, double b) {
    double x0 = threadIdx.x, x1 = x0 + 1, x2 = x0 + 2, x3 = x0 + 3, x4 = x0 + 4, x5 = x0 + 5, x6 = x0 + 6, x7 = x0 + 7;
    for (int i = 0; i < iters; i++) {
#pragma unroll
        for (int u = 0; u < 16; u++) {
            x0 = fma(x0, a, b); x1 = fma(x1, a, b); x2 = fma(x2, a, b); x3 = fma(x3, a, b);
            x4 = fma(x4, a, b); x5 = fma(x5, a, b); x6 = fma(x6, a, b); x7 = fma(x7, a, b);
        }
    }
    out[blockIdx.x * blockDim.x + threadIdx.x] = x0 + x1 + x2 + x3 + x4 + x5 + x6 + x7;
}
int main() {
    int sms = 0; cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
    int clk = 0; cudaDeviceGetAttribute(&clk, cudaDevAttrClockRate, 0);
    double *out; cudaMalloc(&out, sizeof(double) * sms * 32 * 1024);
    cudaEvent_t e0, e1; cudaEventCreate(&e0); cudaEventCreate(&e1);
    for (int warps = 4; warps <= 32; warps *= 2) {
        int thr = 32 * warps, iters = 4000;
        k<<<sms, thr>>>(out, 100, 0.999999, 1e-7);
        cudaEventRecord(e0);
        for (int r = 0; r < 5; r++) k<<<sms, thr>>>(out, iters, 0.999999, 1e-7);
        cudaEventRecord(e1); cudaEventSynchronize(e1);
        float ms; cudaEventElapsedTime(&ms, e0, e1);
        double fl = 5.0 * sms * thr * (double)iters * 16 * 8 * 2;
        printf("{\"sms\": %d, \"warps_per_sm\": %d, \"tflops\": %.3f, \"max_clock_mhz\": %d}\n", sms, warps, fl / ms / 1e9, clk / 1000);
    }
    return 0;
}
