// vgen.cu -- harness kernel (NOT part of the method): writes VGEN(seed, v, t, e)
// into a producer tensor on the GPU, standing in for the training step's
// optimizer write between model versions.  Same counter-based generator as
// synth.vgen_numpy (see synth/__init__.py for the definition); no state is
// shared with the CPU side, both compute it from (seed, v, t, e).
#include <cstdint>
#include <cuda_runtime.h>

namespace {

__device__ __forceinline__ uint64_t splitmix64(uint64_t x) {
    uint64_t z = x + 0x9E3779B97F4A7C15ull;
    z = (z ^ (z >> 30)) * 0xBF58476D1CE4E5B9ull;
    z = (z ^ (z >> 27)) * 0x94D049BB133111EBull;
    return z ^ (z >> 31);
}

uint64_t splitmix64_host(uint64_t x) {
    uint64_t z = x + 0x9E3779B97F4A7C15ull;
    z = (z ^ (z >> 30)) * 0xBF58476D1CE4E5B9ull;
    z = (z ^ (z >> 27)) * 0x94D049BB133111EBull;
    return z ^ (z >> 31);
}

template <int DT>
__global__ void vgen_kernel(uint8_t *out, uint64_t key, uint64_t nelem) {
    for (uint64_t e = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; e < nelem; e += (uint64_t)gridDim.x * blockDim.x) {
        const uint64_t h = splitmix64(key + e);
        const uint64_t sign = h >> 63, ex = (h >> 32) & 3;
        if (DT == 0) {
            reinterpret_cast<uint32_t *>(out)[e] = (uint32_t)((sign << 31) | ((119 + ex) << 23) | (h & 0x7FFFFF));
        } else if (DT == 1) {
            reinterpret_cast<uint16_t *>(out)[e] = (uint16_t)((sign << 15) | ((119 + ex) << 7) | (h & 0x7F));
        } else if (DT == 2) {
            reinterpret_cast<uint16_t *>(out)[e] = (uint16_t)((sign << 15) | ((7 + ex) << 10) | (h & 0x3FF));
        } else {
            out[e] = (uint8_t)(h & 0xFF);
        }
    }
}

}  // namespace

extern "C" int vgen_fill(void *dev_ptr, uint64_t seed, uint64_t version, uint64_t t, int32_t dtype, uint64_t nelem,
                         void *stream) {
    if (nelem == 0) return 0;
    const uint64_t key = splitmix64_host(seed ^ splitmix64_host((version << 20) ^ t));
    const int block = 256;
    uint64_t want = (nelem + block - 1) / block;
    const int grid = (int)(want > 148 * 16 ? 148 * 16 : want);
    cudaStream_t st = (cudaStream_t)stream;
    uint8_t *p = (uint8_t *)dev_ptr;
    switch (dtype) {
        case 0: vgen_kernel<0><<<grid, block, 0, st>>>(p, key, nelem); break;
        case 1: vgen_kernel<1><<<grid, block, 0, st>>>(p, key, nelem); break;
        case 2: vgen_kernel<2><<<grid, block, 0, st>>>(p, key, nelem); break;
        case 3: vgen_kernel<3><<<grid, block, 0, st>>>(p, key, nelem); break;
        default: return -1;
    }
    return cudaGetLastError() == cudaSuccess ? 0 : -3;
}

__global__ void empty_kernel() {}

// Calibration for bench.py: an empty 148x512 launch.
extern "C" int launch_empty(void *stream) {
    empty_kernel<<<148, 512, 0, (cudaStream_t)stream>>>();
    return cudaGetLastError() == cudaSuccess ? 0 : -3;
}

// Flush L2 between timed steps: write `bytes` (> L2) of scratch.
extern "C" int l2_flush(void *dev_ptr, uint64_t bytes, void *stream) {
    return cudaMemsetAsync(dev_ptr, (int)(bytes & 0xFF), bytes, (cudaStream_t)stream) == cudaSuccess ? 0 : -3;
}

namespace {
__global__ void l2_read_kernel(const uint4 *p, uint64_t n, uint32_t *sink) {
    uint32_t x = 0;
    for (uint64_t i = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; i < n; i += (uint64_t)gridDim.x * blockDim.x) {
        const uint4 v = __ldcg(p + i);
        x ^= v.x ^ v.y ^ v.z ^ v.w;
    }
    if (x == 0x9E3779B9u) *sink = x;  // keeps the loads; never true for the memset pattern
}
}  // namespace

// Clean flush: write the first half of the buffer (each half > L2), then read
// the second half, so the first half's dirty lines are written back HERE and
// L2 ends up holding clean, unrelated lines -- the state ncu's cache control
// leaves before a kernel.  The timed kernel then pays no write-back of
// harness data.
extern "C" int l2_flush_clean(void *dev_ptr, uint64_t bytes, void *stream) {
    const uint64_t half = bytes / 2 / 16 * 16;
    cudaStream_t st = (cudaStream_t)stream;
    if (cudaMemsetAsync(dev_ptr, 0x5A, half, st) != cudaSuccess) return -3;
    uint8_t *second = (uint8_t *)dev_ptr + half;
    l2_read_kernel<<<148 * 4, 512, 0, st>>>((const uint4 *)second, half / 16, (uint32_t *)second);
    return cudaGetLastError() == cudaSuccess ? 0 : -3;
}

// Harness helpers for bench.py's e2e leg: pinned host buffers and copies
// through the CUDA runtime directly (torch's pinned copy path measured
// erratic H2D throughput on this VM, profiles/r01/h2dcal.log).
extern "C" void *host_alloc(uint64_t bytes) {
    void *p = nullptr;
    return cudaHostAlloc(&p, bytes, cudaHostAllocPortable) == cudaSuccess ? p : nullptr;
}
extern "C" int host_free(void *p) { return cudaFreeHost(p) == cudaSuccess ? 0 : -3; }
extern "C" int copy_async(void *dst, const void *src, uint64_t bytes, int kind, void *stream) {
    return cudaMemcpyAsync(dst, src, bytes, (cudaMemcpyKind)kind, (cudaStream_t)stream) == cudaSuccess ? 0 : -3;
}
