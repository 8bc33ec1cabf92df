// Microbenchmark: GPU kernel stores into page-locked (mapped) host memory
// vs device memory, two store patterns of a kNN result array [n x k] int32:
//  (a) row per thread: thread q writes its k values (warp store = 32 rows x 4 B)
//  (b) row per warp-iteration: lanes write consecutive elements of one row
// and the cudaMemcpy D2H of the same bytes. Prints GB/s.
#include <cstdio>
#include <cuda_runtime.h>
__global__ void rows_per_thread(int* out, int n, int k) {
    int q = blockIdx.x * blockDim.x + threadIdx.x;
    if (q >= n) return;
    int row = (int)((q * 2654435761u) % (unsigned)n);  // scattered rows, like original query order
    for (int r = 0; r < k; ++r) out[(size_t)row * k + r] = q + r;
}
__global__ void rows_per_warp(int* out, int n, int k) {
    int lane = threadIdx.x & 31;
    int w = (blockIdx.x * blockDim.x + threadIdx.x) >> 5;
    int q0 = w * 32;
    for (int i = 0; i < 32; ++i) {
        int q = q0 + i;
        if (q >= n) break;
        int row = (int)((q * 2654435761u) % (unsigned)n);
        if (lane < k) out[(size_t)row * k + lane] = q + lane;
    }
}
int main() {
    const int n = 434874, k = 20;
    size_t bytes = (size_t)n * k * 4;
    int *h, *hd, *d;
    cudaHostAlloc(&h, bytes, cudaHostAllocMapped);
    cudaHostGetDevicePointer(&hd, h, 0);
    cudaMalloc(&d, bytes);
    cudaEvent_t a, b;
    cudaEventCreate(&a); cudaEventCreate(&b);
    float ms;
    for (int rep = 0; rep < 2; ++rep) {
        for (int dst = 0; dst < 2; ++dst) {
            int* o = dst ? hd : d;
            cudaEventRecord(a);
            rows_per_thread<<<(n + 255) / 256, 256>>>(o, n, k);
            cudaEventRecord(b); cudaEventSynchronize(b); cudaEventElapsedTime(&ms, a, b);
            if (rep) printf("{\"pattern\": \"row-per-thread\", \"dst\": \"%s\", \"ms\": %.4f, \"GBps\": %.1f}\n", dst ? "host" : "device", ms, bytes / ms / 1e6);
            cudaEventRecord(a);
            rows_per_warp<<<(n / 32 + 8) / 8 + 1, 256>>>(o, n, k);
            cudaEventRecord(b); cudaEventSynchronize(b); cudaEventElapsedTime(&ms, a, b);
            if (rep) printf("{\"pattern\": \"row-per-warp\", \"dst\": \"%s\", \"ms\": %.4f, \"GBps\": %.1f}\n", dst ? "host" : "device", ms, bytes / ms / 1e6);
        }
        cudaEventRecord(a);
        cudaMemcpyAsync(h, d, bytes, cudaMemcpyDeviceToHost);
        cudaEventRecord(b); cudaEventSynchronize(b); cudaEventElapsedTime(&ms, a, b);
        if (rep) printf("{\"pattern\": \"cudaMemcpy D2H\", \"ms\": %.4f, \"GBps\": %.1f}\n", ms, bytes / ms / 1e6);
    }
    printf("{\"err\": \"%s\"}\n", cudaGetErrorString(cudaGetLastError()));
    return 0;
}
