// kernels.cu -- sm_100a kernels of the model-update hot path.
//
//   pack_seal      (K2): gather the T scattered parameter tensors into
//                  the contiguous versioned snapshot and seal every chunk with
//                  {version, cks}.  "snapshot ... blocks the training until
//                  completion" (PAPER.md s4.4 P:1700-1703) -> this is t_p.
//   install_verify (K6): read the snapshot (local, NVLink-peer-mapped
//                  or DRAM-staged), recompute every chunk's cks, scatter into
//                  the INACTIVE slot's T tensors and, when every seal matched,
//                  flip the consumer's version word from the device: "the
//                  updated model is written to an alternative copy ... then
//                  the primary copy and alternative copy are swapped
//                  atomically" (s4.2 P:1214-1227) -> this is t_c.
//
// Both are warp-per-work-item streaming kernels: 128-bit loads/stores, U
// vectors in flight per lane, one persistent-ish grid sized to the SM count.
// HBM-bound: algorithmic bytes per launch = 2 * (sum of tensor bytes).
#include "vp_internal.h"

namespace vp {

namespace {

constexpr int kWarpsPerBlock = 16;   // 512 threads
constexpr int kBlocksPerSM = 2;      // 1024 threads / SM resident
constexpr int kUnroll = 4;           // 16-B vectors in flight per lane per step

__device__ __forceinline__ uint4 ld_stream(const void *p) {
    uint4 r;
    asm volatile("ld.global.nc.L1::no_allocate.v4.u32 {%0,%1,%2,%3}, [%4];"
                 : "=r"(r.x), "=r"(r.y), "=r"(r.z), "=r"(r.w)
                 : "l"(p));
    return r;
}

__device__ __forceinline__ void st_v4(void *p, const uint4 &v) {
    asm volatile("st.global.v4.u32 [%0], {%1,%2,%3,%4};" ::"l"(p), "r"(v.x), "r"(v.y), "r"(v.z), "r"(v.w)
                 : "memory");
}

// sum over the 4 words of a 16-B vector whose first word has global index g
__device__ __forceinline__ uint64_t cks_vec(const uint4 &v, uint32_t g) {
    const uint32_t m0 = (2u * g + 1u) * kCksK;
    const uint32_t d = 2u * kCksK;
    const uint32_t m1 = m0 + d, m2 = m1 + d, m3 = m2 + d;
    return (uint64_t)(v.x * m0) + (uint64_t)(v.y * m1) + (uint64_t)(v.z * m2) + (uint64_t)(v.w * m3);
}

__device__ __forceinline__ uint64_t warp_sum(uint64_t x) {
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) x += __shfl_xor_sync(0xffffffffu, x, o);
    return x;
}

// Copy bytes [b0, n) of an item word by word (any alignment); words are
// little-endian u32 of the packed buffer, zero-extended past n.
__device__ __forceinline__ uint64_t copy_words_bytewise(const uint8_t *__restrict__ src, uint8_t *__restrict__ dst,
                                                        uint32_t b0, uint32_t n, uint64_t p0, uint32_t lane,
                                                        bool inject_first) {
    uint64_t acc = 0;
    for (uint32_t w = b0 / 4 + lane; w * 4 < n; w += 32) {
        uint32_t word = 0;
#pragma unroll
        for (int k = 0; k < 4; k++) {
            uint32_t b = w * 4 + k;
            if (b < n) word |= (uint32_t)src[b] << (8 * k);
        }
        if (inject_first && w * 4 == b0) word ^= 0x10u;
#pragma unroll
        for (int k = 0; k < 4; k++) {
            uint32_t b = w * 4 + k;
            if (b < n) dst[b] = (uint8_t)(word >> (8 * k));
        }
        const uint32_t g = (uint32_t)((p0 + w * 4) >> 2);
        acc += (uint64_t)(word * ((2u * g + 1u) * kCksK));
    }
    return acc;
}

// Copy one work item (src -> dst, n bytes, packed offset p0); returns the
// lane's partial checksum of the packed-space words it moved.
__device__ __forceinline__ uint64_t copy_item(const uint8_t *__restrict__ src, uint8_t *__restrict__ dst, uint32_t n,
                                              uint64_t p0, uint32_t lane, bool inject) {
    uint64_t acc = 0;
    const bool aligned = (((uintptr_t)src | (uintptr_t)dst) & 15u) == 0;
    if (!aligned) return copy_words_bytewise(src, dst, 0, n, p0, lane, inject);
    const uint32_t nvec = n >> 4;
    const uint32_t g0 = (uint32_t)(p0 >> 2);
    for (uint32_t base = 0; base < nvec; base += 32 * kUnroll) {
        uint4 r[kUnroll];
#pragma unroll
        for (int u = 0; u < kUnroll; u++) {
            const uint32_t i = base + u * 32 + lane;
            if (i < nvec) r[u] = ld_stream(src + (size_t)i * 16);
        }
        if (inject && base == 0 && lane == 0) r[0].x ^= 0x10u;
#pragma unroll
        for (int u = 0; u < kUnroll; u++) {
            const uint32_t i = base + u * 32 + lane;
            if (i < nvec) {
                st_v4(dst + (size_t)i * 16, r[u]);
                acc += cks_vec(r[u], g0 + 4u * i);
            }
        }
    }
    if (n & 15u) acc += copy_words_bytewise(src, dst, nvec * 16, n, p0, lane, inject && nvec == 0);
    return acc;
}

template <bool kPack>
__device__ __forceinline__ void finish_item(const Item &it, uint64_t lane_acc, uint32_t lane, const Scratch &s,
                                            Seal *seals_out, const Seal *seals_in, uint64_t version,
                                            uint32_t nchunks, bool *last_chunk) {
    const uint64_t item_cks = warp_sum(lane_acc);
    *last_chunk = false;
    if (lane == 0) {
        const uint32_t c = it.chunk;
        atomicAdd((unsigned long long *)&s.acc[c], (unsigned long long)item_cks);
        __threadfence();
        const uint32_t prev = atomicAdd(&s.cnt[c], 1u);
        if (prev == it.chunk_items - 1) {
            __threadfence();
            const uint64_t total = atomicExch((unsigned long long *)&s.acc[c], 0ull);
            s.cnt[c] = 0;
            if (kPack) {
                volatile Seal *so = seals_out + c;
                so->cks = total;
                __threadfence();
                so->version = version;
            } else {
                const volatile Seal *si = seals_in + c;
                const uint64_t ev = si->version, ec = si->cks;
                if (ev != version) atomicOr(s.err, kErrVersion);
                else if (ec != total) atomicOr(s.err, kErrChecksum);
            }
            __threadfence();
            const uint32_t d = atomicAdd(s.done, 1u);
            *last_chunk = (d == nchunks - 1);
        }
    }
}

__device__ __forceinline__ void finalize_install(const InstallArgs &a) {
    __threadfence();
    const uint32_t e = atomicExch(a.s.err, 0u);
    *a.s.done = 0;
    const int32_t st = (e & kErrVersion) ? -4 : ((e & kErrChecksum) ? -5 : 0);
    if (a.status_h) *a.status_h = st;
    __threadfence_system();
    if (st == 0 && a.state_h) *a.state_h = (a.version << 1) | (uint64_t)a.target;  // the atomic swap
    if (a.pin_h) *a.pin_h = 0;  // snapshot no longer read by this consumer
    __threadfence_system();
}

__global__ void __launch_bounds__(kWarpsPerBlock * 32, kBlocksPerSM) pack_seal_kernel(const PackArgs a) {
    const uint32_t lane = threadIdx.x & 31u;
    const uint32_t warps = gridDim.x * (blockDim.x >> 5);
    for (uint32_t w = blockIdx.x * (blockDim.x >> 5) + (threadIdx.x >> 5); w < a.nitems; w += warps) {
        const Item it = a.items[w];
        const uint8_t *src = a.src[it.tensor] + it.tensor_off;
        uint8_t *dst = a.packed + it.packed_off;
        const uint64_t acc = copy_item(src, dst, it.nbytes, it.packed_off, lane, false);
        bool last;
        finish_item<true>(it, acc, lane, a.s, a.seals, nullptr, a.version, a.nchunks, &last);
        if (lane == 0 && last) *a.s.done = 0;  // every chunk sealed: reset for the next launch
    }
}

__global__ void __launch_bounds__(kWarpsPerBlock * 32, kBlocksPerSM) install_verify_kernel(const InstallArgs a) {
    const uint32_t lane = threadIdx.x & 31u;
    if (a.nitems == 0) {  // empty model: nothing to copy, still swap
        if (blockIdx.x == 0 && threadIdx.x == 0) finalize_install(a);
        return;
    }
    const uint32_t warps = gridDim.x * (blockDim.x >> 5);
    for (uint32_t w = blockIdx.x * (blockDim.x >> 5) + (threadIdx.x >> 5); w < a.nitems; w += warps) {
        const Item it = a.items[w];
        const uint8_t *src = a.packed + it.packed_off;
        uint8_t *dst = a.dst[it.tensor] + it.tensor_off;
        const uint64_t acc = copy_item(src, dst, it.nbytes, it.packed_off, lane, w == a.fault_item);
        bool last;
        finish_item<false>(it, acc, lane, a.s, nullptr, a.seals, a.version, a.nchunks, &last);
        if (lane == 0 && last) finalize_install(a);
    }
}

}  // namespace

Geometry pick_geometry(uint32_t nitems, int device) {
    static int sms = 0;
    if (sms == 0) {
        if (cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, device) != cudaSuccess || sms <= 0) sms = 148;
    }
    Geometry g;
    g.block = kWarpsPerBlock * 32;
    const uint32_t want = (nitems + kWarpsPerBlock - 1) / kWarpsPerBlock;
    const uint32_t cap = (uint32_t)sms * kBlocksPerSM;
    g.grid = (int)(want < 1 ? 1 : (want > cap ? cap : want));
    return g;
}

cudaError_t launch_pack(const PackArgs &a, const Geometry &g, cudaStream_t st) {
    if (a.nitems == 0) return cudaSuccess;
    pack_seal_kernel<<<g.grid, g.block, 0, st>>>(a);
    return cudaGetLastError();
}

cudaError_t launch_install(const InstallArgs &a, const Geometry &g, cudaStream_t st) {
    install_verify_kernel<<<g.grid, g.block, 0, st>>>(a);
    return cudaGetLastError();
}

}  // namespace vp
