// H2D bandwidth vs how the pinned host buffer was allocated.
#include <algorithm>
#include <cstdio>
#include <cstdint>
#include <cstdlib>
#include <cstring>
#include <sys/mman.h>
#include <cuda_runtime.h>
static float h2d(void *h, void *d, size_t n, cudaStream_t st) {
    cudaEvent_t a, b; cudaEventCreate(&a); cudaEventCreate(&b);
    float t[31];
    for (int i = 0; i < 31; i++) {
        cudaEventRecord(a, st); cudaMemcpyAsync(d, h, n, cudaMemcpyHostToDevice, st); cudaEventRecord(b, st);
        cudaEventSynchronize(b); cudaEventElapsedTime(&t[i], a, b);
    }
    std::sort(t, t + 31);
    printf("[min %.3f med %.3f max %.3f ms] ", t[0], t[15], t[30]);
    return t[15];
}
int main() {
    cudaStream_t st; cudaStreamCreate(&st);
    void *d; cudaMalloc(&d, 512 << 20);
    size_t sizes[] = {4 << 20, 16 << 20, 64 << 20, 256 << 20};
    for (size_t n : sizes) {
        void *h1; cudaHostAlloc(&h1, n, cudaHostAllocDefault); memset(h1, 1, n);
        void *h2 = malloc(n); memset(h2, 1, n); cudaHostRegister(h2, n, cudaHostRegisterDefault);
        void *h3 = mmap(nullptr, n + (2 << 20), PROT_READ | PROT_WRITE, MAP_PRIVATE | MAP_ANONYMOUS, -1, 0);
        h3 = (void *)(((uintptr_t)h3 + (2 << 20) - 1) & ~(uintptr_t)((2 << 20) - 1));
        madvise(h3, n, MADV_HUGEPAGE); memset(h3, 1, n); cudaHostRegister(h3, n, cudaHostRegisterDefault);
        float t1 = h2d(h1, d, n, st), t2 = h2d(h2, d, n, st), t3 = h2d(h3, d, n, st);
        printf("%4zu MB  cudaHostAlloc %6.1f GB/s   malloc+register %6.1f GB/s   2MB-huge+register %6.1f GB/s\n",
               n >> 20, n / t1 / 1e6, n / t2 / 1e6, n / t3 / 1e6);
        cudaFreeHost(h1); cudaHostUnregister(h2); free(h2); cudaHostUnregister(h3);
    }
    FILE *f = fopen("/sys/kernel/mm/transparent_hugepage/enabled", "r"); char buf[256] = {0};
    if (f) { fgets(buf, sizeof buf, f); fclose(f); }
    printf("THP: %s", buf);
    return 0;
}
