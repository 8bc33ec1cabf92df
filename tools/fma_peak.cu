// fma_peak.cu -- measured fp32 FMA-pipe peak of this B200 (the ALU roofline
// denominator for the scan kernels, VERDICT r1 "measured FMA peak").
//
//   nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o fma_peak tools/fma_peak.cu && ./fma_peak
//
// Every thread runs 8 independent FFMA chains (enough ILP to cover the FMA
// latency at full occupancy); grid = 148 SMs x 8 CTAs x 256 threads. Prints
// one JSON line: TFLOP/s (2 flop per FFMA), best of 10 runs timed with CUDA
// events, and the SM clock the driver reports.
#include <cstdio>
#include <cuda_runtime.h>

__global__ void __launch_bounds__(256) k_fma(float* out, int iters, float a, float b) {
    float x0 = threadIdx.x, x1 = x0 + 1, x2 = x0 + 2, x3 = x0 + 3, x4 = x0 + 4, x5 = x0 + 5, x6 = x0 + 6, x7 = x0 + 7;
    for (int i = 0; i < iters; ++i) {
#pragma unroll
        for (int u = 0; u < 16; ++u) {
            x0 = __fmaf_rn(x0, a, b); x1 = __fmaf_rn(x1, a, b); x2 = __fmaf_rn(x2, a, b); x3 = __fmaf_rn(x3, a, b);
            x4 = __fmaf_rn(x4, a, b); x5 = __fmaf_rn(x5, a, b); x6 = __fmaf_rn(x6, a, b); x7 = __fmaf_rn(x7, a, b);
        }
    }
    out[blockIdx.x * blockDim.x + threadIdx.x] = x0 + x1 + x2 + x3 + x4 + x5 + x6 + x7;
}

int main() {
    cudaDeviceProp p;
    cudaGetDeviceProperties(&p, 0);
    const int blocks = p.multiProcessorCount * 8, threads = 256, iters = 4096;
    float* out;
    cudaMalloc(&out, sizeof(float) * blocks * threads);
    cudaEvent_t e0, e1;
    cudaEventCreate(&e0);
    cudaEventCreate(&e1);
    k_fma<<<blocks, threads>>>(out, iters, 0.999f, 0.001f);
    cudaDeviceSynchronize();
    float best = 1e30f;
    for (int r = 0; r < 10; ++r) {
        cudaEventRecord(e0);
        k_fma<<<blocks, threads>>>(out, iters, 0.999f, 0.001f);
        cudaEventRecord(e1);
        cudaEventSynchronize(e1);
        float ms;
        cudaEventElapsedTime(&ms, e0, e1);
        if (ms < best) best = ms;
    }
    const double ffma = (double)blocks * threads * iters * 16 * 8;
    const double tflops = 2.0 * ffma / (best * 1e-3) / 1e12;
    int clk = 0;
    cudaDeviceGetAttribute(&clk, cudaDevAttrClockRate, 0);
    const double nominal = 2.0 * p.multiProcessorCount * 128 * (clk * 1e3) / 1e12;  // TFLOP/s at the max SM clock (clk in kHz)
    printf("{\"fp32_fma_tflops\": %.2f, \"ms\": %.4f, \"ffma\": %.4g, \"sms\": %d, \"sm_max_mhz\": %.0f, "
           "\"nominal_tflops_at_max_clock\": %.2f, \"frac_of_nominal\": %.3f, \"gpu\": \"%s\"}\n",
           tflops, best, ffma, p.multiProcessorCount, clk / 1e3, nominal, tflops / nominal, p.name);
    return cudaGetLastError() != cudaSuccess;
}
