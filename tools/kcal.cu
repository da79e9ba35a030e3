// Calibration: event-bracketed time of an empty kernel, a plain 16-B copy
// kernel and cudaMemcpyAsync D2D at small sizes (what "launch-bound" costs).
#include <cstdio>
#include <cuda_runtime.h>
__global__ void empty_k() {}
__global__ void copy_k(const uint4 *__restrict__ s, uint4 *__restrict__ d, size_t n) {
    for (size_t i = blockIdx.x * (size_t)blockDim.x + threadIdx.x; i < n; i += (size_t)gridDim.x * blockDim.x) d[i] = s[i];
}
__global__ void spin_k(long long ns) { long long t0 = clock64(); while (clock64() - t0 < ns) {} }
int main() {
    size_t bytes[] = {4616840, 102228128, 173135312};
    cudaStream_t st; cudaStreamCreate(&st);
    cudaEvent_t a, b; cudaEventCreate(&a); cudaEventCreate(&b);
    char *s, *d, *fl; cudaMalloc(&s, 200 << 20); cudaMalloc(&d, 200 << 20); cudaMalloc(&fl, 256 << 20);
    float ms;
    for (int rep = 0; rep < 2; rep++) {
        spin_k<<<1, 1, 0, st>>>(200000); cudaEventRecord(a, st); empty_k<<<144, 512, 0, st>>>(); cudaEventRecord(b, st);
        cudaEventSynchronize(b); cudaEventElapsedTime(&ms, a, b); printf("empty 144x512: %.2f us\n", ms * 1e3);
        spin_k<<<1, 1, 0, st>>>(200000); cudaEventRecord(a, st); for (int i = 0; i < 10; i++) empty_k<<<144, 512, 0, st>>>(); cudaEventRecord(b, st);
        cudaEventSynchronize(b); cudaEventElapsedTime(&ms, a, b); printf("10 x empty back-to-back: %.2f us each\n", ms * 1e2);
        for (size_t by : bytes) {
            size_t n = by / 16;
            for (int flush = 0; flush < 2; flush++) {
                if (flush) cudaMemsetAsync(fl, 1, 256 << 20, st);
                spin_k<<<1, 1, 0, st>>>(200000); cudaEventRecord(a, st);
                int grid = (int)((n + 511) / 512); if (grid > 296) grid = 296;
                copy_k<<<grid, 512, 0, st>>>((uint4 *)s, (uint4 *)d, n); cudaEventRecord(b, st);
                cudaEventSynchronize(b); cudaEventElapsedTime(&ms, a, b);
                printf("copy_k %zu B flush=%d: %.2f us (%.0f GB/s)\n", by, flush, ms * 1e3, 2.0 * by / (ms * 1e-3) / 1e9);
                if (flush) cudaMemsetAsync(fl, 1, 256 << 20, st);
                spin_k<<<1, 1, 0, st>>>(200000); cudaEventRecord(a, st);
                cudaMemcpyAsync(d, s, by, cudaMemcpyDeviceToDevice, st); cudaEventRecord(b, st);
                cudaEventSynchronize(b); cudaEventElapsedTime(&ms, a, b);
                printf("memcpyD2D %zu B flush=%d: %.2f us (%.0f GB/s)\n", by, flush, ms * 1e3, 2.0 * by / (ms * 1e-3) / 1e9);
            }
        }
    }
    return 0;
}
