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
// vectors in flight per lane, a grid of at most 2 blocks per SM.  HBM-bound:
// algorithmic bytes per launch = 2 * (sum of tensor bytes).  Checksums are
// carried per work item (item seal = cks + version * kVerMix) so neither kernel
// needs a cross-block reduction on its critical path; the chunk seals
// {version, cks} of DESIGN.md R16 are reduced from them by seal_reduce on a
// side stream.
#include "vp_internal.h"

#include <atomic>

namespace vp {

namespace {

#ifndef VP_WARPS_PER_BLOCK
#define VP_WARPS_PER_BLOCK 8
#endif
#ifndef VP_BLOCKS_PER_SM
#define VP_BLOCKS_PER_SM 2
#endif
#ifndef VP_UNROLL
#define VP_UNROLL 8
#endif
#ifndef VP_FUSED_UNROLL
#define VP_FUSED_UNROLL 8
#endif
#ifndef VP_FUSED_BLOCKS
#define VP_FUSED_BLOCKS 2
#endif
#ifndef VP_FUSED_READBACK
#define VP_FUSED_READBACK 1
#endif
#ifndef VP_WARP_PROF
#define VP_WARP_PROF 0  // tools/warp_prof.py builds a side variant with per-warp timestamps
#endif
#ifndef VP_DYNAMIC
#define VP_DYNAMIC 1  // A/B: profiles/r01/ktime_dynamic_ab.log
#endif
constexpr int kWarpsPerBlock = VP_WARPS_PER_BLOCK;  // 256 threads
constexpr int kBlocksPerSM = VP_BLOCKS_PER_SM;      // 512 threads / SM resident (128-reg budget)
constexpr int kUnroll = VP_UNROLL;                  // 16-B vectors in flight per lane per step
constexpr int kFusedUnroll = VP_FUSED_UNROLL;       // publish_fused_kernel's own geometry
constexpr int kFusedBlocks = VP_FUSED_BLOCKS;

__device__ __forceinline__ uint4 ld_stream(const void *p) {
    uint4 r;
    asm volatile("ld.global.nc.L1::no_allocate.v4.u32 {%0,%1,%2,%3}, [%4];"
                 : "=r"(r.x), "=r"(r.y), "=r"(r.z), "=r"(r.w)
                 : "l"(p));
    return r;
}

__device__ __forceinline__ uint64_t l2_evict_first_policy() {
    uint64_t pol;
    asm volatile("createpolicy.fractional.L2::evict_first.b64 %0, 1.0;" : "=l"(pol));
    return pol;
}

// The same with an L2 cache policy (createpolicy): read-once data evicted first
__device__ __forceinline__ uint4 ld_stream_pol(const void *p, uint64_t pol) {
    uint4 r;
    asm volatile("ld.global.nc.L1::no_allocate.L2::cache_hint.v4.u32 {%0,%1,%2,%3}, [%4], %5;"
                 : "=r"(r.x), "=r"(r.y), "=r"(r.z), "=r"(r.w)
                 : "l"(p), "l"(pol));
    return r;
}

__device__ __forceinline__ uint4 ld_cg(const void *p) {  // L2-coherent (data written during this grid)
    uint4 r;
    asm volatile("ld.global.cg.v4.u32 {%0,%1,%2,%3}, [%4];"
                 : "=r"(r.x), "=r"(r.y), "=r"(r.z), "=r"(r.w)
                 : "l"(p));
    return r;
}

__device__ __forceinline__ void st_release(uint64_t *p, uint64_t v) {
    asm volatile("st.release.gpu.global.u64 [%0], %1;" ::"l"(p), "l"(v) : "memory");
}

__device__ __forceinline__ void st_release_sys(uint64_t *p, uint64_t v) {
    asm volatile("st.release.sys.global.u64 [%0], %1;" ::"l"(p), "l"(v) : "memory");
}

__device__ __forceinline__ uint64_t ld_acquire_sys(const uint64_t *p) {
    uint64_t v;
    asm volatile("ld.acquire.sys.global.u64 %0, [%1];" : "=l"(v) : "l"(p) : "memory");
    return v;
}

__device__ __forceinline__ uint64_t ld_acquire(const uint64_t *p) {
    uint64_t v;
    asm volatile("ld.acquire.gpu.global.u64 %0, [%1];" : "=l"(v) : "l"(p) : "memory");
    return v;
}

__device__ __forceinline__ void st_v4(void *p, const uint4 &v) {
    asm volatile("st.global.v4.u32 [%0], {%1,%2,%3,%4};" ::"l"(p), "r"(v.x), "r"(v.y), "r"(v.z), "r"(v.w)
                 : "memory");
}

// CKS terms of the 4 words of a 16-B vector whose first word has global index g:
// sum_k w_k * ((2(g+k)+1) * K) mod 2^32   (R16)
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

// Work distribution of the streaming kernels.  Each warp's first item is
// static (its global warp id); after that, items are claimed from a per-launch
// counter, one item ahead, so the atomic's round trip overlaps the current
// item's stream.  This balances the tail (item sizes differ at tensor and
// chunk borders, SMs progress at different rates).  Claimed index = raw -
// base + nwarps; the grid's last block resets the counter (base 0).  With
// nitems <= nwarps there is no second round and no claim.  Used by the fused
// and install kernels; the pack stays static (measured faster, see there).
struct WorkQueue {
    unsigned int *ctr;
    uint32_t base, nwarps, nitems;
    bool dyn;
    uint32_t pending;  // lane 0: raw value of the claim in flight
    __device__ __forceinline__ WorkQueue(unsigned int *c, uint32_t b, uint32_t nw, uint32_t n)
        : ctr(c), base(b), nwarps(nw), nitems(n), dyn(VP_DYNAMIC && c != nullptr && n > nw), pending(0) {}
    __device__ __forceinline__ void claim(uint32_t lane) {
        if (dyn && lane == 0) pending = atomicAdd(ctr, 1u);
    }
    // the item after w: the claim made one item ago (or the static stride)
    __device__ __forceinline__ uint32_t next(uint32_t w, uint32_t lane) {
        if (!dyn) return w + nwarps;
        const uint32_t k = __shfl_sync(0xffffffffu, pending - base, 0);
        return k < nitems ? k + nwarps : nitems;  // k >= nitems: wrapped / exhausted
    }
};

// Copy bytes [b0, n) of an item word by word (any alignment); words are
// little-endian u32 of the packed buffer, zero-extended past n.
template <bool kCoherent>
__device__ __forceinline__ uint64_t copy_words_bytewise(const uint8_t *__restrict__ src, uint8_t *__restrict__ dst,
                                                        uint32_t b0, uint32_t n, uint64_t p0, uint32_t lane,
                                                        bool inject_first) {
    uint64_t acc = 0;
    for (uint32_t w = b0 / 4 + lane; w * 4 < n; w += 32) {
        uint32_t word = 0;
#pragma unroll
        for (int k = 0; k < 4; k++) {
            const uint32_t b = w * 4 + k;
            if (b < n) word |= (uint32_t)(kCoherent ? __ldcg(src + b) : src[b]) << (8 * k);
        }
        if (inject_first && w * 4 == b0) word ^= 0x10u;
#pragma unroll
        for (int k = 0; k < 4; k++) {
            const uint32_t b = w * 4 + k;
            if (b < n) dst[b] = (uint8_t)(word >> (8 * k));
        }
        const uint32_t g = (uint32_t)((p0 + w * 4) >> 2);
        acc += (uint64_t)(word * ((2u * g + 1u) * kCksK));
    }
    return acc;
}

// Copy one work item (src -> dst, n bytes, packed offset p0); returns the
// lane's partial checksum of the packed-space words it moved.
// pol != 0 (non-coherent loads only): L2 cache policy of the source loads
template <bool kCoherent, int U = kUnroll>
__device__ __forceinline__ uint64_t copy_item(const uint8_t *__restrict__ src, uint8_t *__restrict__ dst, uint32_t n,
                                              uint64_t p0, uint32_t lane, bool inject, uint64_t pol = 0) {
    uint64_t acc = 0;
    const bool aligned = (((uintptr_t)src | (uintptr_t)dst) & 15u) == 0;
    if (!aligned) return copy_words_bytewise<kCoherent>(src, dst, 0, n, p0, lane, inject);
    const uint32_t nvec = n >> 4;
    const uint32_t g0 = (uint32_t)(p0 >> 2);
    for (uint32_t base = 0; base < nvec; base += 32 * U) {
        uint4 r[U];
#pragma unroll
        for (int u = 0; u < U; u++) {
            const uint32_t i = base + u * 32 + lane;
            if (i < nvec)
                r[u] = kCoherent ? ld_cg(src + (size_t)i * 16)
                                 : (pol ? ld_stream_pol(src + (size_t)i * 16, pol) : ld_stream(src + (size_t)i * 16));
        }
        if (inject && base == 0 && lane == 0) r[0].x ^= 0x10u;
#pragma unroll
        for (int u = 0; u < U; u++) {
            const uint32_t i = base + u * 32 + lane;
            if (i < nvec) {
                st_v4(dst + (size_t)i * 16, r[u]);
                acc += cks_vec(r[u], g0 + 4u * i);
            }
        }
    }
    if (n & 15u) acc += copy_words_bytewise<kCoherent>(src, dst, nvec * 16, n, p0, lane, inject && nvec == 0);
    return acc;
}

// Fused copy for the SYNC in-process publish: per U-vector step, stream the
// tensor piece into the snapshot, immediately read those snapshot bytes back
// (same lane, same addresses -> ordered; an L2 hit), and store them into each
// consumer's slot.  Returns the pack checksum; cks_c[k] is the checksum of
// what consumer k received (the read-back, after any injected fault).
template <int U = kUnroll, int kC = kMaxFused>
__device__ __forceinline__ uint64_t copy_item_fused(const uint8_t *__restrict__ src, uint8_t *__restrict__ snap,
                                                    const uint64_t *dst, uint32_t ncons, uint32_t n, uint64_t p0,
                                                    uint32_t lane, uint32_t inject_mask, uint64_t *cks_c) {
    uint64_t acc = 0;
    bool aligned = (((uintptr_t)src | (uintptr_t)snap) & 15u) == 0;
#pragma unroll
    for (int k = 0; k < kC; k++)
        if (k < (int)ncons) aligned &= (dst[k] & 15u) == 0;
    if (!aligned) {  // rare: word path, pack then one read-back per consumer
        acc = copy_words_bytewise<false>(src, snap, 0, n, p0, lane, false);
        __syncwarp();
#pragma unroll
        for (int k = 0; k < kC; k++)
            if (k < (int)ncons)
                cks_c[k] += copy_words_bytewise<true>(snap, (uint8_t *)dst[k], 0, n, p0, lane, (inject_mask >> k) & 1u);
        return acc;
    }
    const uint32_t nvec = n >> 4;
    const uint32_t g0 = (uint32_t)(p0 >> 2);
    for (uint32_t base = 0; base < nvec; base += 32 * U) {
        uint4 r[U];
#pragma unroll
        for (int u = 0; u < U; u++) {
            const uint32_t i = base + u * 32 + lane;
            if (i < nvec) r[u] = ld_stream(src + (size_t)i * 16);
        }
#pragma unroll
        for (int u = 0; u < U; u++) {
            const uint32_t i = base + u * 32 + lane;
            if (i < nvec) {
                st_v4(snap + (size_t)i * 16, r[u]);
                acc += cks_vec(r[u], g0 + 4u * i);
            }
        }
#if VP_FUSED_READBACK
#pragma unroll
        for (int u = 0; u < U; u++) {  // read back what this lane stored
            const uint32_t i = base + u * 32 + lane;
            if (i < nvec) r[u] = ld_cg(snap + (size_t)i * 16);
        }
#endif
#pragma unroll
        for (int k = 0; k < kC; k++) {
            if (k >= (int)ncons) break;
#pragma unroll
            for (int u = 0; u < U; u++) {
                const uint32_t i = base + u * 32 + lane;
                if (i < nvec) {
                    uint4 x = r[u];
                    if (u == 0 && base == 0 && lane == 0 && ((inject_mask >> k) & 1u)) x.x ^= 0x10u;
                    st_v4((uint8_t *)dst[k] + (size_t)i * 16, x);
                    cks_c[k] += cks_vec(x, g0 + 4u * i);
                }
            }
        }
    }
    if (n & 15u) {
        acc += copy_words_bytewise<false>(src, snap, nvec * 16, n, p0, lane, false);
        __syncwarp();
#pragma unroll
        for (int k = 0; k < kC; k++)
            if (k < (int)ncons)
                cks_c[k] += copy_words_bytewise<true>(snap, (uint8_t *)dst[k], nvec * 16, n, p0, lane,
                                                      ((inject_mask >> k) & 1u) && nvec == 0);
    }
    return acc;
}

// pack: stream every item tensor -> packed, write its item seal.  No atomics,
// no fences: the consumer's kernel is ordered after this one by the stream /
// event, which makes every store visible.
#ifndef VP_PACK_UNROLL_SMALL
#define VP_PACK_UNROLL_SMALL 16  // pack_seal's vectors per lane for snapshots <= 1 GiB (profiles/r02/pack_ab.log)
#endif

// Item seals are released in batches of kRelBatch items per warp (pack_seal_kernel below).
#ifndef VP_PACK_REL_BATCH
#define VP_PACK_REL_BATCH 4
#endif
constexpr int kRelBatch = VP_PACK_REL_BATCH;

__device__ __forceinline__ void st_relaxed_sys(uint64_t *p, uint64_t v) {
    asm volatile("st.relaxed.sys.global.u64 [%0], %1;" ::"l"(p), "l"(v) : "memory");
}

__device__ __forceinline__ void st_relaxed_gpu(uint64_t *p, uint64_t v) {
    asm volatile("st.relaxed.gpu.global.u64 [%0], %1;" ::"l"(p), "l"(v) : "memory");
}

// ---------------------------------------------------------------------------
// Push delivery (VIPER_FANOUT_PUSH): the pack stores every item into
// its local snapshot AND straight into each consumer's peer-mapped staging
// (NVLink stores: fire-and-forget, so the warp streams at the link rate), then
// releases the item's seal at system scope in every staging.  Consumers install
// from their own HBM, item by item behind these seals.
__device__ __forceinline__ uint64_t copy_item_push(const uint8_t *__restrict__ src, uint8_t *__restrict__ snap,
                                                   const PushArgs &a, uint64_t off, uint32_t n, uint32_t lane) {
    bool aligned = (((uintptr_t)src | (uintptr_t)snap) & 15u) == 0;
    if (!aligned) {  // rare (unaligned source tensor): word path, then copy the snapshot piece out
        const uint64_t acc = copy_words_bytewise<false>(src, snap, 0, n, off, lane, false);
        __syncwarp();
        for (uint32_t k = 0; k < a.ndst; k++) copy_words_bytewise<true>(snap, a.dst[k] + off, 0, n, off, lane, false);
        return acc;
    }
    uint64_t acc = 0;
    const uint32_t nvec = n >> 4;
    const uint32_t g0 = (uint32_t)(off >> 2);
    for (uint32_t base = 0; base < nvec; base += 32 * kUnroll) {
        uint4 r[kUnroll];
#pragma unroll
        for (int u = 0; u < kUnroll; u++) {
            const uint32_t i = base + u * 32 + lane;
            if (i < nvec) r[u] = ld_stream(src + (size_t)i * 16);
        }
#pragma unroll
        for (int u = 0; u < kUnroll; u++) {
            const uint32_t i = base + u * 32 + lane;
            if (i < nvec) {
                st_v4(snap + (size_t)i * 16, r[u]);
                acc += cks_vec(r[u], g0 + 4u * i);
            }
        }
        for (uint32_t k = 0; k < a.ndst; k++) {
            uint8_t *d = a.dst[k] + off;
#pragma unroll
            for (int u = 0; u < kUnroll; u++) {
                const uint32_t i = base + u * 32 + lane;
                if (i < nvec) st_v4(d + (size_t)i * 16, r[u]);
            }
        }
    }
    if (n & 15u) {  // < 16-B tensor tail (packed offsets are 16-B aligned, the tail is not)
        acc += copy_words_bytewise<false>(src, snap, nvec * 16, n, off, lane, false);
        __syncwarp();
        for (uint32_t k = 0; k < a.ndst; k++) copy_words_bytewise<true>(snap, a.dst[k] + off, nvec * 16, n, off, lane, false);
    }
    return acc;
}

// Seals released in batches of kRelBatch items per warp, as in pack_seal
// (one system-scope fence per batch instead of one per item and consumer).
__global__ void __launch_bounds__(kWarpsPerBlock * 32, kBlocksPerSM) pack_push_kernel(const PushArgs a) {
    const uint32_t lane = threadIdx.x & 31u;
    const uint32_t nwarps = gridDim.x * kWarpsPerBlock;
    uint32_t pend_idx[kRelBatch];
    int npend = 0;
    auto release = [&]() {
        if (lane == 0 && npend) {
            asm volatile("fence.acq_rel.sys;" ::: "memory");  // the batch's data + cks words, everywhere
#pragma unroll
            for (int j = 0; j < kRelBatch; j++)
                if (j < npend) {
                    st_relaxed_sys(&a.p.iseal[pend_idx[j]].version, a.p.version);
                    for (uint32_t k = 0; k < a.ndst; k++) st_relaxed_sys(&a.dst_iseal[k][pend_idx[j]].version, a.p.version);
                }
        }
        npend = 0;
    };
    uint32_t w = blockIdx.x * kWarpsPerBlock + (threadIdx.x >> 5);
    Item nxt{};
    if (w < a.p.nitems) nxt = a.p.items[w];
    for (; w < a.p.nitems; w += nwarps) {
        const Item it = nxt;
        if (w + nwarps < a.p.nitems) nxt = a.p.items[w + nwarps];
        const uint64_t part = warp_sum(copy_item_push((const uint8_t *)it.ptr, a.p.packed + it.packed_off, a,
                                                      it.packed_off, it.nbytes, lane));
        __syncwarp();  // every lane's stores are ordered before lane 0's fence
        if (lane == 0) {
            const uint64_t mixed = part + a.p.version * kVerMix;
            a.p.iseal[it.gidx].mixed = mixed;
            for (uint32_t k = 0; k < a.ndst; k++) a.dst_iseal[k][it.gidx].mixed = mixed;  // the consumers' copies
        }
        pend_idx[npend++] = it.gidx;
        if (npend == kRelBatch) release();
    }
    release();
}

// ---------------------------------------------------------------------------
// NVLS multicast delivery (VIPER_FANOUT_NVLS): the snapshot lives in
// memory bound to one multicast object on every rank; the pack stores each
// 16-B vector once to the multicast address (multimem.st) and NVSwitch writes
// it into the producer's snapshot and every consumer's staging.  The item seal
// follows with a system-scope release through the same multicast address.
__device__ __forceinline__ void mc_st_v4(void *p, const uint4 &v) {
    asm volatile("multimem.st.global.v4.f32 [%0], {%1,%2,%3,%4};" ::"l"(p), "r"(v.x), "r"(v.y), "r"(v.z), "r"(v.w)
                 : "memory");
}

__device__ __forceinline__ void mc_st_u32(void *p, uint32_t v) {
    asm volatile("multimem.st.global.b32 [%0], %1;" ::"l"(p), "r"(v) : "memory");
}

__device__ __forceinline__ void mc_st_u64(void *p, uint64_t v) {
    asm volatile("multimem.st.global.b64 [%0], %1;" ::"l"(p), "l"(v) : "memory");
}

__device__ __forceinline__ void mc_st_relaxed_sys_u64(void *p, uint64_t v) {
    asm volatile("multimem.st.relaxed.sys.global.b64 [%0], %1;" ::"l"(p), "l"(v) : "memory");
}

__global__ void __launch_bounds__(kWarpsPerBlock * 32, kBlocksPerSM) pack_nvls_kernel(const NvlsArgs a) {
    const uint32_t lane = threadIdx.x & 31u;
    const uint32_t nwarps = gridDim.x * kWarpsPerBlock;
    uint32_t pend_idx[kRelBatch];  // seals released in batches (pack_seal)
    int npend = 0;
    auto release = [&]() {
        if (lane == 0 && npend) {
            asm volatile("fence.acq_rel.sys;" ::: "memory");
#pragma unroll
            for (int j = 0; j < kRelBatch; j++)
                if (j < npend) mc_st_relaxed_sys_u64(&a.mc_iseal[pend_idx[j]].version, a.version);
        }
        npend = 0;
    };
    uint32_t w0 = blockIdx.x * kWarpsPerBlock + (threadIdx.x >> 5);
    Item nxt{};
    if (w0 < a.nitems) nxt = a.items[w0];
    for (uint32_t w = w0; w < a.nitems; w += nwarps) {
        const Item it = nxt;
        if (w + nwarps < a.nitems) nxt = a.items[w + nwarps];
        const uint8_t *src = (const uint8_t *)it.ptr;
        uint8_t *dst = a.mc_packed + it.packed_off;
        const uint32_t n = it.nbytes;
        uint64_t acc = 0;
        uint32_t done = 0;
        if (((uintptr_t)src & 15u) == 0) {
            const uint32_t nvec = n >> 4;
            const uint32_t g0 = (uint32_t)(it.packed_off >> 2);
            for (uint32_t base = 0; base < nvec; base += 32 * kUnroll) {
                uint4 r[kUnroll];
#pragma unroll
                for (int u = 0; u < kUnroll; u++) {
                    const uint32_t i = base + u * 32 + lane;
                    if (i < nvec) r[u] = ld_stream(src + (size_t)i * 16);
                }
#pragma unroll
                for (int u = 0; u < kUnroll; u++) {
                    const uint32_t i = base + u * 32 + lane;
                    if (i < nvec) {
                        mc_st_v4(dst + (size_t)i * 16, r[u]);
                        acc += cks_vec(r[u], g0 + 4u * i);
                    }
                }
            }
            done = nvec * 16;
        }
        // word path (unaligned source or < 16-B tail): whole little-endian words;
        // the bytes past n in the last word are padding, which is zero by LAY
        for (uint32_t wd = done / 4 + lane; wd * 4 < n; wd += 32) {
            uint32_t word = 0;
#pragma unroll
            for (int k = 0; k < 4; k++) {
                const uint32_t b = wd * 4 + k;
                if (b < n) word |= (uint32_t)src[b] << (8 * k);
            }
            mc_st_u32(dst + wd * 4, word);
            const uint32_t g = (uint32_t)((it.packed_off + wd * 4) >> 2);
            acc += (uint64_t)(word * ((2u * g + 1u) * kCksK));
        }
        const uint64_t part = warp_sum(acc);
        __syncwarp();
        if (lane == 0) mc_st_u64(&a.mc_iseal[it.gidx].mixed, part + a.version * kVerMix);
        pend_idx[npend++] = it.gidx;
        if (npend == kRelBatch) release();
    }
    release();
}

// pack: stream every item tensor -> packed and seal it.  The seals are what a
// pipelined install waits on: a PDL-chained install on this GPU (gpu scope) or,
// under early notification, consumers on OTHER GPUs (kSys: system scope).  A
// release costs lane 0 a fence (MEMBAR.GPU / MEMBAR.SYS) that stalls the warp,
// and the system-scope one is expensive: one per 8-KiB item made the pack 1.4-
// 1.8x slower (profiles/r02/pack_release_ab.log).  So the seals are released
// in batches of kRelBatch items per warp: lane 0 writes the batch's cks words,
// issues ONE fence, then the versions as relaxed stores (the fence + relaxed
// store pair is a release: a consumer that acquires a version sees its item's
// data and cks).  Items stay the pipeline's unit; a seal just becomes visible
// up to kRelBatch - 1 items later.  The __syncwarp after each item orders
// every lane's stores before lane 0's fence.  Static strided items (measured
// faster than the work counter here: Llama-3 8B 5.05 vs 6.0 ms,
// profiles/r01/ktime_dynamic_ab.log), descriptors prefetched one item ahead.
template <int U, bool kSys>
__global__ void __launch_bounds__(kWarpsPerBlock * 32, kBlocksPerSM) pack_seal_kernel(const PackArgs a) {
    // let a programmatically-dependent install grid start now: it consumes
    // items as their ready flags flip (item-granular pack -> install pipeline)
    asm volatile("griddepcontrol.launch_dependents;");
    const uint32_t lane = threadIdx.x & 31u;
    const uint32_t nwarps = gridDim.x * kWarpsPerBlock;
    uint32_t w = blockIdx.x * kWarpsPerBlock + (threadIdx.x >> 5);
    uint32_t pend_idx[kRelBatch];
    int npend = 0;
    auto release = [&]() {  // lane 0: one fence for the batch, then its versions
        if (lane == 0 && npend) {
            if (kSys) asm volatile("fence.acq_rel.sys;" ::: "memory");
            else asm volatile("fence.acq_rel.gpu;" ::: "memory");
#pragma unroll
            for (int k = 0; k < kRelBatch; k++)
                if (k < npend) {
                    if (kSys) st_relaxed_sys(&a.iseal[pend_idx[k]].version, a.version);
                    else st_relaxed_gpu(&a.iseal[pend_idx[k]].version, a.version);
                }
        }
        npend = 0;
    };
    Item nxt{};
    if (w < a.nitems) nxt = a.items[w];
    for (; w < a.nitems; w += nwarps) {
        const Item it = nxt;  // descriptor prefetched one item ahead: its load overlaps this item's stream
        if (w + nwarps < a.nitems) nxt = a.items[w + nwarps];
        const uint64_t part = warp_sum(copy_item<false, U>((const uint8_t *)it.ptr, a.packed + it.packed_off,
                                                           it.nbytes, it.packed_off, lane, false));
        __syncwarp();  // every lane's stores are ordered before lane 0's fence
        if (lane == 0) a.iseal[it.gidx].mixed = part + a.version * kVerMix;  // before the fence, too
        pend_idx[npend++] = it.gidx;
        if (npend == kRelBatch) release();
    }
    release();
}

// the pack instantiation for a snapshot of `bytes` (sys: seals released at system scope)
static const void *pack_fn(uint64_t bytes, bool sys = false) {
    const bool big = bytes > (1ull << 30);
    if (sys)
        return big ? (const void *)pack_seal_kernel<8, true> : (const void *)pack_seal_kernel<VP_PACK_UNROLL_SMALL, true>;
    return big ? (const void *)pack_seal_kernel<8, false> : (const void *)pack_seal_kernel<VP_PACK_UNROLL_SMALL, false>;
}

// chunk seals {version, sum of item checksums} -- one warp per chunk, off the
// critical path (side stream); they are what DESIGN.md R16 / the oracle define.
__global__ void seal_reduce_kernel(const SealReduceArgs a) {
    const uint32_t lane = threadIdx.x & 31u;
    const uint32_t c = blockIdx.x * (blockDim.x >> 5) + (threadIdx.x >> 5);
    if (c >= a.nchunks) return;
    if (a.share_n > 1 && c % a.share_n != a.share_me) return;  // another producer's chunk
    const uint32_t lo = a.chunk_first[c], hi = a.chunk_first[c + 1];
    uint64_t s = 0;
    for (uint32_t i = lo + lane; i < hi; i += 32) s += a.iseal[i].mixed - a.version * kVerMix;
    s = warp_sum(s);
    if (lane == 0) {
        a.seals[c].cks = s;
        a.seals[c].version = a.version;
    }
}

// Checksum of one item read in place (no copy): the CKS terms of the packed
// words it covers (any alignment; words zero-extended past n).
__device__ __forceinline__ uint64_t cks_item_inplace(const uint8_t *__restrict__ src, uint32_t n, uint64_t p0,
                                                     uint32_t lane) {
    uint64_t acc = 0;
    uint32_t done = 0;
    if (((uintptr_t)src & 15u) == 0) {
        const uint32_t nvec = n >> 4;
        const uint32_t g0 = (uint32_t)(p0 >> 2);
        for (uint32_t base = 0; base < nvec; base += 32 * kUnroll) {
            uint4 r[kUnroll];
#pragma unroll
            for (int u = 0; u < kUnroll; u++) {
                const uint32_t i = base + u * 32 + lane;
                if (i < nvec) r[u] = ld_cg(src + (size_t)i * 16);
            }
#pragma unroll
            for (int u = 0; u < kUnroll; u++) {
                const uint32_t i = base + u * 32 + lane;
                if (i < nvec) acc += cks_vec(r[u], g0 + 4u * i);
            }
        }
        done = nvec * 16;
    }
    for (uint32_t w = done / 4 + lane; w * 4 < n; w += 32) {
        uint32_t word = 0;
#pragma unroll
        for (int k = 0; k < 4; k++) {
            const uint32_t b = w * 4 + k;
            if (b < n) word |= (uint32_t)__ldcg(src + b) << (8 * k);
        }
        const uint32_t g = (uint32_t)((p0 + w * 4) >> 2);
        acc += (uint64_t)(word * ((2u * g + 1u) * kCksK));
    }
    return acc;
}

// Chunk seals {version, cks} (R16) of a consumer slot as it is laid
// out in place (viper_view_seals): the same CKS as the producer's snapshot
// seals, computed from the installed tensors, so a consumer can prove its
// replica byte-exact against the oracle's seals without a host copy.  `seals`
// must be zeroed; item checksums are summed with 64-bit atomics (the sum is
// commutative, so the result is exact in any order).
__global__ void __launch_bounds__(kWarpsPerBlock * 32) view_seal_kernel(const ViewSealArgs a) {
    const uint32_t lane = threadIdx.x & 31u;
    const uint32_t nwarps = gridDim.x * kWarpsPerBlock;
    for (uint32_t w = blockIdx.x * kWarpsPerBlock + (threadIdx.x >> 5); w < a.nitems; w += nwarps) {
        const Item it = a.items[w];
        const uint64_t part = warp_sum(cks_item_inplace((const uint8_t *)it.ptr, it.nbytes, it.packed_off, lane));
        if (lane == 0) {
            atomicAdd((unsigned long long *)&a.seals[it.chunk].cks, (unsigned long long)part);
            a.seals[it.chunk].version = a.version;
        }
    }
}

// Grid completion word: low 32 bits count finished blocks, high 32 bits carry
// error bits.  Both halves live in ONE 64-bit word updated only by 64-bit
// atomics, so the last block's arrival returns every error reported before
// it.  This saves the separate error exchange (one L2 round trip) on the
// critical path.
__device__ __forceinline__ void report_err(unsigned long long *flags, uint32_t bits) {
    atomicOr(flags, (unsigned long long)bits << 32);
}

// Thread 0 of each block, after __syncthreads: release this block's stores
// (bar.sync + a gpu-scope release is cumulative over the block) and count it.
// Returns true in the last block, with the grid's error bits, and resets the word.
__device__ __forceinline__ bool grid_arrive(unsigned long long *flags, uint32_t *err) {
    unsigned long long old;
    asm volatile("atom.acq_rel.gpu.global.add.u64 %0, [%1], 1;" : "=l"(old) : "l"(flags) : "memory");
    if ((uint32_t)old != gridDim.x - 1) return false;
    *err = (uint32_t)(old >> 32);
    *flags = 0;  // every block has arrived: nobody else touches it in this grid
    return true;
}

// A seal wait should stop: the host aborted the install (abort_h) or another
// warp of this grid already timed out (its error bit is in the completion word).
// abort_h is host memory: a read is a PCIe round trip, so the waits below ask
// only once per kAbortPollMask + 1 polls (about every 250 us of waiting) --
// asked on every poll, a thousand waiting warps flooded PCIe and slowed the
// pipelined GPT-2 XL install 40-fold (profiles/r02/pipeline_overlap.log).
constexpr uint32_t kAbortPollMask = 255;
__device__ __forceinline__ bool wait_aborted(const InstallArgs &a) {
    if ((*(volatile unsigned long long *)a.flags >> 32) & kErrTimeout) return true;
    return a.abort_h && *a.abort_h;
}

// lane 0's seal spin, one step: sleep with exponential backoff (32 ns .. 1 us);
// true when the wait must end (kItemWaitNs passed, or aborted).
__device__ __forceinline__ bool wait_step(const InstallArgs &a, uint32_t &backoff, uint64_t &waited, uint32_t &polls) {
    __nanosleep(backoff);
    waited += backoff;
    if (backoff < 1024) backoff <<= 1;
    if ((++polls & kAbortPollMask) != 0) return false;
    return waited > kItemWaitNs || wait_aborted(a);
}

// End of an install grid: the last block to finish publishes the result and,
// when every item matched, swaps the version word from the device.
__device__ __forceinline__ void install_finish(const InstallArgs &a, bool bad) {
    if (bad) report_err(a.flags, kErrChecksum);
    __syncthreads();
    uint32_t e;
    if (threadIdx.x == 0 && grid_arrive(a.flags, &e)) {
        const int32_t st = (e & kErrTimeout) ? -6 : ((e & kErrChecksum) ? -5 : 0);
        // Every block's slot stores are GPU-visible (released by its arrival,
        // acquired by this one), which is all a reader on this GPU needs: it
        // launches its kernels after the host saw the flip.  When the slot
        // lives on ANOTHER GPU (an in-process SYNC install launched on the
        // producer's stream), a system-scope fence -- cumulative over what
        // this thread observed -- orders every block's peer stores before the
        // swap becomes visible.
        if (a.sys_swap) asm volatile("fence.acq_rel.sys;" ::: "memory");
        // the pin first: the host takes the status / swap as "done" and may
        // pin its next snapshot at once, which a late clear would undo
        if (a.pin_h) *a.pin_h = 0;  // snapshot no longer read by this consumer (every block has arrived)
        if (a.ctr) *a.ctr = 0;      // work counter: every warp stopped claiming
        if (a.status_h) *a.status_h = st;
        if (st == 0 && a.state_h) *a.state_h = (a.version << 1) | (uint64_t)a.target;  // the atomic swap
    }
}

// install: stream every item packed -> slot tensor, recompute its seal and
// compare with the producer's; the last block to finish publishes the result
// and, if every item matched, swaps the version word from the device.
__global__ void __launch_bounds__(kWarpsPerBlock * 32, kBlocksPerSM) install_verify_kernel(const InstallArgs a) {
    const uint32_t lane = threadIdx.x & 31u;
    const uint32_t nwarps = gridDim.x * kWarpsPerBlock;
    bool bad = false;
    uint32_t w = blockIdx.x * kWarpsPerBlock + (threadIdx.x >> 5);
    WorkQueue q(a.ctr, 0, nwarps, a.nitems);  // reset by the last block (install_finish)
    // Items staged for the peers (scatter-allgather owner / chain link) have
    // their seals released in batches of kRelBatch (one system-scope fence per
    // batch, as in pack_seal), but never held across a wait: a warp that is
    // about to wait for a seal first releases what it holds, so two consumers
    // can never wait on each other's pending seals.
    uint32_t rp_idx[kRelBatch];
    int rp_n = 0;
    auto release_staged = [&]() {
        if (lane == 0 && rp_n) {
            asm volatile("fence.acq_rel.sys;" ::: "memory");
#pragma unroll
            for (int j = 0; j < kRelBatch; j++)
                if (j < rp_n) st_relaxed_sys(&a.sa_iseal_out[rp_idx[j]].version, a.version);
        }
        rp_n = 0;
    };
    auto ready = [&](const ISeal *x) {  // warp-uniform: lane 0's first look at a seal
        int r = 0;
        if (lane == 0) r = ld_acquire_sys(&x->version) == a.version;
        return __shfl_sync(0xffffffffu, r, 0) != 0;
    };
    if (w < a.nitems) q.claim(lane);
    while (w < a.nitems) {
        const Item it = a.items[w];
        // Item-granular pipeline: with PDL the install grid runs concurrently
        // with the pack grid (all of whose blocks are resident by then, so
        // this cannot deadlock); wait for item w's ready flag, then stream it
        // with L2-coherent loads.  Without PDL the flag is already set.
        const uint8_t *src = a.packed + it.packed_off;
        const ISeal *is = a.iseal + w;
        if (a.mp_n > 1) {  // data-parallel producers: the chunk's owner packed it
            const uint32_t p = it.chunk % a.mp_n;
            src = a.mp_snap[p] + it.packed_off;
            is = a.mp_iseal[p] + w;
        }
        // Fan-out among consumers: `peer` is the consumer this item is pulled
        // from (-1 = the producer); `republish` = also stage it (+ seal,
        // release.sys) for the consumers that pull it from here.
        //   scatter-allgather: chunk c is owned by consumer c % N, which pulls
        //                      it from the producer; the others pull from it;
        //   chain:             consumer i pulls everything from consumer i-1
        //                      (0 from the producer) and stages it for i+1.
        int peer = -1;
        bool republish = false;
        if (a.sa_n) {
            if (a.chain) {
                peer = (int)a.sa_me - 1;
                republish = a.sa_me + 1 < a.sa_n;
            } else if (it.chunk % a.sa_n == a.sa_me) {
                republish = true;
            } else {
                peer = (int)(it.chunk % a.sa_n);
            }
        }
        if (peer >= 0) {
            if (!ready(a.sa_isrc[peer] + w)) release_staged();
            int ok = 0;
            if (lane == 0) {
                const ISeal *ps = a.sa_isrc[peer] + w;
                uint32_t backoff = 64, polls = 0;
                int64_t spent = 0;
                for (;;) {
                    if (ld_acquire_sys(&ps->version) == a.version) { ok = 1; break; }
                    __nanosleep(backoff);
                    spent += backoff;
                    if (backoff < 2048) backoff <<= 1;
                    // the peer is not installing this version (skipped it or
                    // finished without it): take the item from the producer.
                    // (The pin word is host memory: asked every 16th poll.)
                    if (spent > 20000 && (++polls & 15) == 0 && *a.sa_owner_pin[peer] != a.version) break;
                    if (spent > 50000000) break;  // 50 ms: never hang, fall back
                }
            }
            ok = __shfl_sync(0xffffffffu, ok, 0);
            if (ok) {
                src = a.sa_src[peer] + it.packed_off;
                is = a.sa_isrc[peer] + w;
            } else {
                peer = -1;  // producer copy (re-published only where this consumer stages it anyway)
            }
        }
        // (system scope: the producer may be another GPU pipelining its pack)
        if (rp_n && !ready(is)) release_staged();
        uint64_t expect = 0;
        if (lane == 0) {
            uint32_t backoff = 32, polls = 0;
            uint64_t waited = 0;
            while (ld_acquire_sys(&is->version) != a.version) {
                // never hang on a vanished producer: give up after kItemWaitNs,
                // when the host aborts, or when another warp timed out
                if (wait_step(a, backoff, waited, polls)) {
                    report_err(a.flags, kErrTimeout);
                    break;
                }
            }
            expect = is->mixed;
        }
        __syncwarp();
        // One pass, or two when a peer's staged copy failed its seal: the
        // second pass heals from the producer (pinned by this consumer) and
        // verifies against the producer's own seal.  (A loop, not a second
        // inlined copy: the kernel stays within its 128-register budget.)
        bool from_peer = peer >= 0;
        for (;;) {
            uint64_t part, staged = 0;
            if (republish) {
                // src -> slot, then the slot bytes just stored are read back
                // into this consumer's staging (what its peers will pull)
                uint64_t dsts[kMaxFused] = {(uint64_t)(a.sa_stage_out + it.packed_off), 0, 0, 0};
                uint64_t got[kMaxFused] = {0, 0, 0, 0};
                part = warp_sum(copy_item_fused(src, (uint8_t *)it.ptr, dsts, 1, it.nbytes, it.packed_off, lane,
                                                w == a.fault_item ? 1u : 0u, got));
                staged = warp_sum(got[0]);
            } else {
                part = warp_sum(copy_item<true>(src, (uint8_t *)it.ptr, it.nbytes, it.packed_off, lane,
                                                w == a.fault_item));  // injected on every pass: never healed
            }
            // expect is valid in lane 0 only: take the (warp-uniform) decision there
            if (__shfl_sync(0xffffffffu, (int)(from_peer && part + a.version * kVerMix != expect), 0)) {
                src = a.packed + it.packed_off;
                if (lane == 0) expect = a.iseal[w].mixed;
                from_peer = false;
                continue;
            }
            __syncwarp();  // every lane's staging stores before lane 0's (batched) release
            if (lane == 0) {
                if (republish) {  // peers may pull item w from this consumer's staging once released
                    a.sa_iseal_out[w].mixed = expect;
                    if (staged + a.version * kVerMix != expect) bad = true;
                }
                if (part + a.version * kVerMix != expect) bad = true;
            }
            if (republish) {
                rp_idx[rp_n++] = w;
                if (rp_n == kRelBatch) release_staged();
            }
            break;
        }
        w = q.next(w, lane);
        if (w < a.nitems) q.claim(lane);
    }
    release_staged();
    install_finish(a, bad);
}

// install_direct: the install of one version from ONE source -- the local or
// NVLink-peer-mapped snapshot, or this GPU's staging (push / NVLS / CE / DRAM
// tier) -- with the pack's structure: static item striding, and the next
// item's descriptor fetched one item ahead.
//   kPipe = false: the snapshot is COMPLETE before the grid starts (not
//     PDL-chained, not early-notified).  The next item's seal {cks, version}
//     is fetched one item ahead too, so a warp's only dependent round trip per
//     item is its data, and the data is immutable for the grid's lifetime (the
//     consumer pins it): non-coherent streaming loads.  A seal that does not
//     show `version` (it cannot, but the kernel never trusts that) falls back
//     to the acquire spin.
//   kPipe = true: the item pipeline behind a pack that is still running
//     (PDL on this GPU, early notification across GPUs): lane 0 acquires the
//     item's seal at system scope before the warp streams it, with
//     L2-coherent loads.  Only direct installs; scatter-allgather / chain /
//     data-parallel producers keep install_verify_kernel.
// U = 16-B vectors per lane in flight: 16 for snapshots <= 1 GiB, 8 above
// (ncu cold sweep, profiles/r02/install_sweep.json).
__device__ __forceinline__ ISeal ld_seal(const ISeal *p) {
    ISeal s;
    asm volatile("ld.global.cg.v2.u64 {%0,%1}, [%2];" : "=l"(s.mixed), "=l"(s.version) : "l"(p));
    return s;
}

#ifndef VP_ID_BLOCKS
#define VP_ID_BLOCKS 2
#endif
constexpr int kIdBlocks = VP_ID_BLOCKS;  // install_direct's resident blocks per SM

// lane 0: wait until item w's seal shows the version (acquire, system scope:
// the producer may be another GPU); returns its cks.  Never hangs.
__device__ __forceinline__ uint64_t acquire_seal(const InstallArgs &a, uint32_t w) {
    uint32_t backoff = 32, polls = 0;
    uint64_t waited = 0;
    while (ld_acquire_sys(&a.iseal[w].version) != a.version) {
        if (wait_step(a, backoff, waited, polls)) {
            report_err(a.flags, kErrTimeout);
            break;
        }
    }
    return a.iseal[w].mixed;
}

template <int U, bool kPipe>
__global__ void __launch_bounds__(kWarpsPerBlock * 32, kIdBlocks) install_direct_kernel(const InstallArgs a) {
    const uint32_t lane = threadIdx.x & 31u;
    const uint32_t nwarps = gridDim.x * kWarpsPerBlock;
    bool bad = false;
    uint32_t w = blockIdx.x * kWarpsPerBlock + (threadIdx.x >> 5);
    // a snapshot that fits in L2 was usually just written there: read it with
    // an evict-first policy so the slot stores do not push out the lines not
    // read yet (as the TMA install does, profiles/r01/tma_l2_hint_ab.log)
    const uint64_t pol = (!kPipe && a.l2_once) ? l2_evict_first_policy() : 0;
    Item nxt{};
    ISeal nseal{};
    if (w < a.nitems) {
        nxt = a.items[w];
        if (!kPipe && lane == 0) nseal = ld_seal(a.iseal + w);
    }
    for (; w < a.nitems; w += nwarps) {
        const Item it = nxt;
        uint64_t expect = 0;
        if (lane == 0) expect = (kPipe || nseal.version != a.version) ? acquire_seal(a, w) : nseal.mixed;
        if (kPipe) __syncwarp();  // the data loads below follow lane 0's acquire
        const uint32_t wn = w + nwarps;  // prefetch: its loads overlap this item's stream
        if (wn < a.nitems) {
            nxt = a.items[wn];
            if (!kPipe && lane == 0) nseal = ld_seal(a.iseal + wn);
        }
        const uint64_t part = warp_sum(copy_item<kPipe, U>(a.packed + it.packed_off, (uint8_t *)it.ptr, it.nbytes,
                                                           it.packed_off, lane, w == a.fault_item, pol));
        if (lane == 0 && part + a.version * kVerMix != expect) bad = true;
    }
    install_finish(a, bad);
}

// the instantiation for a snapshot of `bytes`
static const void *install_direct_fn(uint64_t bytes, bool pipe) {
    const bool big = bytes > (1ull << 30);
    if (pipe) return big ? (const void *)install_direct_kernel<8, true> : (const void *)install_direct_kernel<16, true>;
    return big ? (const void *)install_direct_kernel<8, false> : (const void *)install_direct_kernel<16, false>;
}

// SYNC in-process publish, pack + install fused per warp.  Lane l re-reads
// exactly the snapshot bytes it stored (same thread, so ordered) with L2
// loads, installs them and recomputes the item checksum; the seal check is
// against the value just sealed.  No cross-warp dependency inside the grid.
#if VP_WARP_PROF
// tools/warp_prof.py (profiling builds only): per warp {start, end, items, bytes}
__device__ unsigned long long g_warp_prof[8192 * 4];
__device__ unsigned long long g_prof_end;  // the last block, after the swap
__device__ __forceinline__ unsigned long long gtimer() {
    unsigned long long t;
    asm volatile("mov.u64 %0, %globaltimer;" : "=l"(t));
    return t;
}
#endif

#ifndef VP_FUSED_PREFETCH
#define VP_FUSED_PREFETCH 0  // 1: next item's descriptors loaded one item ahead (A/B)
#endif
#ifndef VP_FUSED1_BLOCKS
#define VP_FUSED1_BLOCKS VP_FUSED_BLOCKS
#endif
// kC = the consumers compiled in: 1 (the common SYNC 1 -> 1 update: fewer
// registers) or kMaxFused.
template <int kC>
__global__ void __launch_bounds__(kWarpsPerBlock * 32, kC == 1 ? VP_FUSED1_BLOCKS : kFusedBlocks)
    publish_fused_kernel(const FusedArgs a) {
    const uint32_t lane = threadIdx.x & 31u;
    const uint32_t nwarps = gridDim.x * kWarpsPerBlock;
    uint32_t bad = 0;
    uint32_t w = blockIdx.x * kWarpsPerBlock + (threadIdx.x >> 5);
#if VP_WARP_PROF
    const uint32_t gw = w;
    const unsigned long long prof_t0 = gtimer();
    unsigned long long prof_items = 0, prof_bytes = 0;
#endif
#if VP_FUSED_PREFETCH
    // The next item is known one item ahead (its claim was issued two items
    // ahead), so its descriptors -- the producer item and each consumer's slot
    // address -- load while this item streams.  The first two items of a warp
    // are static (w, w + nwarps); claims then start at 2 * nwarps.
    unsigned int *ctr = reinterpret_cast<unsigned int *>(a.flags + 1);
    const bool dyn = a.nitems > 2 * nwarps;
    uint32_t wn = w + nwarps;
    uint32_t pend = 0;
    Item it_n{};
    uint64_t cptr_n[kC];
    auto load_desc = [&](uint32_t x, Item &d, uint64_t *cp) {
        if (x >= a.nitems) return;
        d = a.items[x];
#pragma unroll
        for (int k = 0; k < kC; k++) cp[k] = k < (int)a.ncons ? a.cons[k].items[x].ptr : 0;
    };
    load_desc(w, it_n, cptr_n);
    while (w < a.nitems) {
        const Item it = it_n;
        uint64_t cptr[kC];
#pragma unroll
        for (int k = 0; k < kC; k++) cptr[k] = cptr_n[k];
        if (dyn && lane == 0 && wn < a.nitems) pend = atomicAdd(ctr, 1u);  // the item after wn
        load_desc(wn, it_n, cptr_n);
        uint32_t inject = 0;
#pragma unroll
        for (int k = 0; k < kC; k++)
            if (k < (int)a.ncons && w == a.cons[k].fault_item) inject |= 1u << k;
#else
    WorkQueue q(reinterpret_cast<unsigned int *>(a.flags + 1), 0, nwarps, a.nitems);  // reset by the last block
    if (w < a.nitems) q.claim(lane);
    while (w < a.nitems) {
        const Item it = a.items[w];
        uint64_t cptr[kC];  // only the slot address differs between the lists
        uint32_t inject = 0;
#pragma unroll
        for (int k = 0; k < kC; k++) {
            cptr[k] = k < (int)a.ncons ? a.cons[k].items[w].ptr : 0;
            if (k < (int)a.ncons && w == a.cons[k].fault_item) inject |= 1u << k;
        }
#endif
        uint64_t got[kC];
#pragma unroll
        for (int k = 0; k < kC; k++) got[k] = 0;
        const uint64_t part = warp_sum(copy_item_fused<kFusedUnroll, kC>((const uint8_t *)it.ptr, a.packed + it.packed_off,
                                                                         cptr, a.ncons, it.nbytes, it.packed_off, lane,
                                                                         inject, got));
        const uint64_t sealed = part + a.version * kVerMix;
        if (lane == 0) {  // no concurrent reader in this path: a plain store (grid end publishes it)
            a.iseal[w].mixed = sealed;
            a.iseal[w].version = a.version;
        }
#pragma unroll
        for (int k = 0; k < kC; k++) {
            if (k >= (int)a.ncons) break;
            if (warp_sum(got[k]) + a.version * kVerMix != sealed) bad |= 1u << k;
        }
#if VP_WARP_PROF
        prof_items++;
        prof_bytes += it.nbytes;
#endif
#if VP_FUSED_PREFETCH
        w = wn;
        if (w < a.nitems) {
            if (dyn) {
                const uint32_t k2 = __shfl_sync(0xffffffffu, pend, 0);
                wn = k2 < a.nitems - 2 * nwarps ? k2 + 2 * nwarps : a.nitems;
            } else {
                wn = w + nwarps;
            }
        }
#else
        w = q.next(w, lane);
        if (w < a.nitems) q.claim(lane);
#endif
    }
#if VP_WARP_PROF
    if (lane == 0 && gw < 8192) {
        g_warp_prof[gw * 4 + 0] = prof_t0;
        g_warp_prof[gw * 4 + 1] = gtimer();
        g_warp_prof[gw * 4 + 2] = prof_items;
        g_warp_prof[gw * 4 + 3] = prof_bytes;
    }
#endif
    if (lane == 0 && bad) report_err(a.flags, bad);
    __syncthreads();
    uint32_t e;
    if (threadIdx.x == 0 && grid_arrive(a.flags, &e)) {
        *reinterpret_cast<unsigned int *>(a.flags + 1) = 0;  // work counter: every warp stopped claiming
        if (a.sys_swap) asm volatile("fence.acq_rel.sys;" ::: "memory");  // peer slots: see install_finish
        for (uint32_t k = 0; k < a.ncons; k++) {
            const FusedCons &c = a.cons[k];
            const int32_t st = (e >> k) & 1u ? -5 : 0;
            if (c.status_h) *c.status_h = st;
            if (st == 0 && c.state_h) *c.state_h = (a.version << 1) | (uint64_t)c.target;  // the swap
            if (c.pin_h) *c.pin_h = 0;
        }
#if VP_WARP_PROF
        g_prof_end = gtimer();
#endif
    }
}

// ---------------------------------------------------------------------------
// pack_seal, TMA bulk-copy variant (VIPER_FLAG_TMA): per warp, a ring of
// kTmaStages shared-memory stages of kTmaStage bytes.  Lane 0 streams each
// item's 16-B-aligned body through the ring with cp.async.bulk (global ->
// shared, mbarrier complete_tx) and cp.async.bulk (shared -> global,
// bulk_group); all lanes checksum the stage from shared memory in between.
// Unaligned items / <16-B tails use the register path.  Used without PDL:
// the consumer's kernel starts after this grid completed, which makes every
// bulk store visible.
constexpr int kTmaStages = 3;
constexpr uint32_t kTmaStage = 4096;
constexpr int kTmaWarps = 8;

__device__ __forceinline__ uint32_t smem_u32(const void *p) {
    return static_cast<uint32_t>(__cvta_generic_to_shared(p));
}

__device__ __forceinline__ void mbar_init(uint64_t *bar) {
    asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" ::"r"(smem_u32(bar)) : "memory");
}

__device__ __forceinline__ void mbar_expect_tx(uint64_t *bar, uint32_t bytes) {
    asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(smem_u32(bar)), "r"(bytes) : "memory");
}

__device__ __forceinline__ void mbar_wait(uint64_t *bar, uint32_t parity) {
    asm volatile(
        "{\n\t.reg .pred p;\n"
        "WAIT_%=:\n\t"
        "mbarrier.try_wait.parity.shared::cta.b64 p, [%0], %1;\n\t"
        "@!p bra WAIT_%=;\n}" ::"r"(smem_u32(bar)),
        "r"(parity)
        : "memory");
}

__device__ __forceinline__ void bulk_g2s(void *smem, const void *gmem, uint32_t bytes, uint64_t *bar) {
    asm volatile("cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];"
                 ::"r"(smem_u32(smem)), "l"(gmem), "r"(bytes), "r"(smem_u32(bar))
                 : "memory");
}

#ifndef VP_TMA_HINTS
#define VP_TMA_HINTS 1  // 0: compile the L2 hints out (A/B, profiles/r01/tma_l2_hint_ab.log)
#endif
// L2 policy for data read exactly once (the pack's parameter tensors, the
// install's snapshot): evict it first, so it does not push out data that is
// read again soon (the snapshot the install or the D2H reads next).

// pol == 0: no hint (models larger than L2 gain nothing from it and lose a little)
__device__ __forceinline__ void bulk_g2s_once(void *smem, const void *gmem, uint32_t bytes, uint64_t *bar,
                                              uint64_t pol) {
#if VP_TMA_HINTS
    if (pol) {
        asm volatile(
            "cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes.L2::cache_hint [%0], [%1], %2, [%3], "
            "%4;" ::"r"(smem_u32(smem)),
            "l"(gmem), "r"(bytes), "r"(smem_u32(bar)), "l"(pol)
            : "memory");
        return;
    }
#endif
    bulk_g2s(smem, gmem, bytes, bar);
}

__device__ __forceinline__ void bulk_s2g(void *gmem, const void *smem, uint32_t bytes) {
    asm volatile("cp.async.bulk.global.shared::cta.bulk_group [%0], [%1], %2;" ::"l"(gmem), "r"(smem_u32(smem)),
                 "r"(bytes)
                 : "memory");
    asm volatile("cp.async.bulk.commit_group;" ::: "memory");
}

template <int N>
__device__ __forceinline__ void bulk_wait_read() {
    asm volatile("cp.async.bulk.wait_group.read %0;" ::"n"(N) : "memory");
}

struct TmaCursor {  // position in this warp's (item, stage-sized piece) sequence
    uint32_t w;     // item index
    uint32_t off;   // byte offset inside the item's TMA body
};

__device__ __forceinline__ uint32_t tma_body(const Item &it) {
    // TMA needs 16-B aligned addresses and sizes; the rest goes through registers
    return ((it.ptr | it.packed_off) & 15u) ? 0u : (it.nbytes & ~15u);
}

__global__ void __launch_bounds__(kTmaWarps * 32, 2) pack_seal_tma_kernel(const PackArgs a) {
    extern __shared__ __align__(128) uint8_t tma_smem[];
    const uint32_t lane = threadIdx.x & 31u, wib = threadIdx.x >> 5;
    const uint64_t pol = a.l2_once ? l2_evict_first_policy() : 0;  // parameter tensors: read once
    uint8_t *stage = tma_smem + wib * (kTmaStages * kTmaStage);
    uint64_t *bar = reinterpret_cast<uint64_t *>(tma_smem + kTmaWarps * kTmaStages * kTmaStage) + wib * kTmaStages;
    if (lane == 0) {
        for (int s = 0; s < kTmaStages; s++) mbar_init(bar + s);
        asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
    }
    __syncwarp();
    const uint32_t nwarps = gridDim.x * kTmaWarps;
    const uint32_t w0 = blockIdx.x * kTmaWarps + wib;
    // loader cursor: the next piece to bring in; skips items without a TMA body
    TmaCursor ld{w0, 0};
    auto next_piece = [&](TmaCursor &c, Item &it, uint32_t &bytes) -> bool {
        while (c.w < a.nitems) {
            it = a.items[c.w];
            const uint32_t body = tma_body(it);
            if (c.off < body) {
                bytes = min(kTmaStage, body - c.off);
                return true;
            }
            c.w += nwarps;
            c.off = 0;
        }
        return false;
    };
    uint32_t issued = 0, phase_bits = 0;
    // prologue: fill the ring
    for (int s = 0; s < kTmaStages; s++) {
        Item it;
        uint32_t bytes;
        if (!next_piece(ld, it, bytes)) break;
        if (lane == 0) {
            mbar_expect_tx(bar + s, bytes);
            bulk_g2s_once(stage + s * kTmaStage, (const uint8_t *)it.ptr + ld.off, bytes, bar + s, pol);
        }
        ld.off += bytes;
        issued++;
    }
    uint32_t consumed = 0;
    for (uint32_t w = w0; w < a.nitems; w += nwarps) {
        const Item it = a.items[w];
        const uint32_t body = tma_body(it);
        uint64_t acc = 0;
        for (uint32_t off = 0; off < body; off += kTmaStage) {
            const uint32_t bytes = min(kTmaStage, body - off);
            const int s = consumed % kTmaStages;
            mbar_wait(bar + s, (phase_bits >> s) & 1u);
            phase_bits ^= 1u << s;
            const uint8_t *buf = stage + s * kTmaStage;
            const uint32_t g0 = (uint32_t)((it.packed_off + off) >> 2);
            for (uint32_t i = lane; i < bytes / 16; i += 32)
                acc += cks_vec(*reinterpret_cast<const uint4 *>(buf + i * 16), g0 + 4u * i);
            __syncwarp();
            if (lane == 0) {
                asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
                bulk_s2g(a.packed + it.packed_off + off, buf, bytes);
            }
            consumed++;
            // refill this stage with the piece kTmaStages ahead once its store has read it
            Item nit;
            uint32_t nbytes;
            if (next_piece(ld, nit, nbytes)) {
                if (lane == 0) {
                    bulk_wait_read<0>();
                    mbar_expect_tx(bar + s, nbytes);
                    bulk_g2s_once(stage + s * kTmaStage, (const uint8_t *)nit.ptr + ld.off, nbytes, bar + s, pol);
                }
                ld.off += nbytes;
                issued++;
            }
        }
        if (body < it.nbytes)  // unaligned item or <16-B tail: register path
            acc += (body == 0) ? copy_item<false>((const uint8_t *)it.ptr, a.packed + it.packed_off, it.nbytes,
                                                  it.packed_off, lane, false)
                               : copy_words_bytewise<false>((const uint8_t *)it.ptr + 0, a.packed + it.packed_off,
                                                            body, it.nbytes, it.packed_off, lane, false);
        const uint64_t part = warp_sum(acc);
        if (lane == 0) {
            a.iseal[it.gidx].mixed = part + a.version * kVerMix;
            a.iseal[it.gidx].version = a.version;  // visible to the next kernel (no PDL with this variant)
        }
    }
    if (lane == 0) asm volatile("cp.async.bulk.wait_group 0;" ::: "memory");
    (void)issued;
}

// install_verify, TMA bulk-copy variant (direct installs not PDL-chained to
// their pack: ASYNC, DRAM tier, cross-process).  Snapshot pieces stream
// through the same per-warp shared-memory ring: cp.async.bulk global ->
// shared, checksum from shared memory, cp.async.bulk shared -> slot tensor.
// The grid's last block swaps the version once every bulk store completed.
__global__ void __launch_bounds__(kTmaWarps * 32, 2) install_verify_tma_kernel(const InstallArgs a) {
    extern __shared__ __align__(128) uint8_t tma_smem[];
    const uint32_t lane = threadIdx.x & 31u, wib = threadIdx.x >> 5;
    const uint64_t pol = a.l2_once ? l2_evict_first_policy() : 0;  // the snapshot: read once
    uint8_t *stage = tma_smem + wib * (kTmaStages * kTmaStage);
    uint64_t *bar = reinterpret_cast<uint64_t *>(tma_smem + kTmaWarps * kTmaStages * kTmaStage) + wib * kTmaStages;
    if (lane == 0) {
        for (int s = 0; s < kTmaStages; s++) mbar_init(bar + s);
        asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
    }
    __syncwarp();
    const uint32_t nwarps = gridDim.x * kTmaWarps;
    const uint32_t w0 = blockIdx.x * kTmaWarps + wib;
    auto body_of = [&](const Item &it) -> uint32_t {
        return ((it.ptr | it.packed_off) & 15u) ? 0u : (it.nbytes & ~15u);
    };
    TmaCursor ld{w0, 0};
    auto next_piece = [&](TmaCursor &c, Item &it, uint32_t &bytes) -> bool {
        while (c.w < a.nitems) {
            it = a.items[c.w];
            const uint32_t body = body_of(it);
            if (c.off < body) {
                bytes = min(kTmaStage, body - c.off);
                return true;
            }
            c.w += nwarps;
            c.off = 0;
        }
        return false;
    };
    for (int s = 0; s < kTmaStages; s++) {  // prologue: fill the ring
        Item it;
        uint32_t bytes;
        if (!next_piece(ld, it, bytes)) break;
        if (lane == 0) {
            mbar_expect_tx(bar + s, bytes);
            bulk_g2s_once(stage + s * kTmaStage, a.packed + it.packed_off + ld.off, bytes, bar + s, pol);
        }
        ld.off += bytes;
    }
    uint32_t consumed = 0, phase_bits = 0;
    bool bad = false;
    for (uint32_t w = w0; w < a.nitems; w += nwarps) {
        const Item it = a.items[w];
        // Only complete snapshots come here (not PDL-chained, not early-notified):
        // the seal is already there, so it is loaded now and checked when the
        // item is done instead of stalling lane 0 -- which issues the warp's
        // bulk copies -- on a round trip per item (the acquire spin below is
        // the never-hang fallback, not the expected path).
        ISeal sl{};
        if (lane == 0) sl = ld_seal(a.iseal + w);
        const uint32_t body = body_of(it);
        uint64_t acc = 0;
        for (uint32_t off = 0; off < body; off += kTmaStage) {
            const uint32_t bytes = min(kTmaStage, body - off);
            const int s = consumed % kTmaStages;
            mbar_wait(bar + s, (phase_bits >> s) & 1u);
            phase_bits ^= 1u << s;
            uint8_t *buf = stage + s * kTmaStage;
            if (w == a.fault_item && off == 0 && lane == 0) buf[0] ^= 0x10;  // fault injection (tests)
            __syncwarp();
            const uint32_t g0 = (uint32_t)((it.packed_off + off) >> 2);
            for (uint32_t i = lane; i < bytes / 16; i += 32)
                acc += cks_vec(*reinterpret_cast<const uint4 *>(buf + i * 16), g0 + 4u * i);
            __syncwarp();
            if (lane == 0) {
                asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
                bulk_s2g((uint8_t *)it.ptr + off, buf, bytes);
            }
            consumed++;
            Item nit;
            uint32_t nbytes;
            if (next_piece(ld, nit, nbytes)) {
                if (lane == 0) {
                    bulk_wait_read<0>();
                    mbar_expect_tx(bar + s, nbytes);
                    bulk_g2s_once(stage + s * kTmaStage, a.packed + nit.packed_off + ld.off, nbytes, bar + s, pol);
                }
                ld.off += nbytes;
            }
        }
        if (body < it.nbytes)
            acc += (body == 0) ? copy_item<true>(a.packed + it.packed_off, (uint8_t *)it.ptr, it.nbytes, it.packed_off,
                                                 lane, w == a.fault_item)
                               : copy_words_bytewise<true>(a.packed + it.packed_off, (uint8_t *)it.ptr, body,
                                                           it.nbytes, it.packed_off, lane, false);
        const uint64_t part = warp_sum(acc);
        if (lane == 0) {
            const uint64_t expect = sl.version == a.version ? sl.mixed : acquire_seal(a, w);
            if (part + a.version * kVerMix != expect) bad = true;
        }
    }
    if (lane == 0)  // slot stores complete, then ordered before the generic-proxy release below
        asm volatile("cp.async.bulk.wait_group 0;\n\tfence.proxy.async.global;" ::: "memory");
    __syncwarp();
    install_finish(a, bad);
}

// ---------------------------------------------------------------------------
// publish_fused, TMA bulk-copy variant (SYNC in-process).  Per warp, a ring of
// kFtStages shared-memory stages of kFtStage bytes (>= the default 8 KiB item
// cap, so an item is one piece).  Lane 0 brings each item's piece in with
// cp.async.bulk (global -> shared, mbarrier complete_tx); all lanes checksum
// it from shared memory (the item seal); lane 0 then issues bulk stores of
// the SAME stage into the snapshot and into every consumer's inactive slot
// (one bulk group per piece).  Install verification (R21'): once an
// item's bulk group has completed -- checked one item later, so the wait
// overlaps the next item's stream -- the warp reads the installed slot bytes
// back (L2 hits) and recomputes their checksum against the seal.  Items that
// are not 16-B aligned (or have a <16-B tail) take the register path
// (copy_item_fused) inline.  Static strided items.
#ifndef VP_FT_WARPS
#define VP_FT_WARPS 4
#endif
#ifndef VP_FT_STAGES
#define VP_FT_STAGES 3
#endif
#ifndef VP_FT_STAGE
#define VP_FT_STAGE 8192
#endif
#ifndef VP_FT_READBACK
#define VP_FT_READBACK 1
#endif
constexpr int kFtWarps = VP_FT_WARPS;
constexpr int kFtStages = VP_FT_STAGES;
constexpr uint32_t kFtStage = VP_FT_STAGE;

__device__ __forceinline__ void bulk_s2g_nc(void *gmem, const void *smem, uint32_t bytes) {  // no commit
    asm volatile("cp.async.bulk.global.shared::cta.bulk_group [%0], [%1], %2;" ::"l"(gmem), "r"(smem_u32(smem)),
                 "r"(bytes)
                 : "memory");
}

// 16-B-aligned TMA body of fused item w (0: the whole item takes the register path)
__device__ __forceinline__ uint32_t fused_tma_body(const FusedArgs &a, const Item &it, uint32_t w) {
    uint64_t m = it.ptr | it.packed_off | it.nbytes;
#pragma unroll
    for (int k = 0; k < kMaxFused; k++)
        if (k < (int)a.ncons) m |= a.cons[k].items[w].ptr;
    return (m & 15u) ? 0u : it.nbytes;
}

// Read consumer k's installed copy of item w back and checksum it (after the
// item's bulk stores completed).  Returns the bit mask of consumers whose copy
// does not match `sealed`.  Fault injection flips the first word first.
__device__ __forceinline__ uint32_t fused_verify_slots(const FusedArgs &a, uint32_t w, uint64_t sealed,
                                                       uint32_t lane) {
    const Item it = a.items[w];
    const uint32_t nvec = it.nbytes >> 4;
    const uint32_t g0 = (uint32_t)(it.packed_off >> 2);
    uint32_t bad = 0;
#pragma unroll
    for (int k = 0; k < kMaxFused; k++) {
        if (k >= (int)a.ncons) break;
        const uint8_t *dst = (const uint8_t *)a.cons[k].items[w].ptr;
        if (w == a.cons[k].fault_item) {
            if (lane == 0) *(volatile uint32_t *)dst ^= 0x10u;
            __syncwarp();
        }
        uint64_t c = 0;
        for (uint32_t base = 0; base < nvec; base += 32 * kFusedUnroll) {
            uint4 r[kFusedUnroll];
#pragma unroll
            for (int u = 0; u < kFusedUnroll; u++) {
                const uint32_t i = base + u * 32 + lane;
                if (i < nvec) r[u] = ld_cg(dst + (size_t)i * 16);
            }
#pragma unroll
            for (int u = 0; u < kFusedUnroll; u++) {
                const uint32_t i = base + u * 32 + lane;
                if (i < nvec) c += cks_vec(r[u], g0 + 4u * i);
            }
        }
        if (warp_sum(c) + a.version * kVerMix != sealed) bad |= 1u << k;
    }
    return bad;
}

__global__ void __launch_bounds__(kFtWarps * 32, 2) publish_fused_tma_kernel(const FusedArgs a) {
    extern __shared__ __align__(128) uint8_t tma_smem[];
    const uint32_t lane = threadIdx.x & 31u, wib = threadIdx.x >> 5;
    uint8_t *stage = tma_smem + wib * (kFtStages * kFtStage);
    uint64_t *bar = reinterpret_cast<uint64_t *>(tma_smem + kFtWarps * kFtStages * kFtStage) + wib * kFtStages;
    if (lane == 0) {
        for (int s = 0; s < kFtStages; s++) mbar_init(bar + s);
        asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
    }
    __syncwarp();
    const uint32_t nwarps = gridDim.x * kFtWarps;
    const uint32_t w0 = blockIdx.x * kFtWarps + wib;
    TmaCursor ld{w0, 0};
    auto next_piece = [&](TmaCursor &c, Item &it, uint32_t &bytes) -> bool {
        while (c.w < a.nitems) {
            it = a.items[c.w];
            const uint32_t body = fused_tma_body(a, it, c.w);
            if (c.off < body) {
                bytes = min(kFtStage, body - c.off);
                return true;
            }
            c.w += nwarps;
            c.off = 0;
        }
        return false;
    };
    for (int s = 0; s < kFtStages; s++) {  // prologue: fill the ring
        Item it;
        uint32_t bytes;
        if (!next_piece(ld, it, bytes)) break;
        if (lane == 0) {
            mbar_expect_tx(bar + s, bytes);
            bulk_g2s(stage + s * kFtStage, (const uint8_t *)it.ptr + ld.off, bytes, bar + s);
        }
        ld.off += bytes;
    }
    uint32_t consumed = 0, phase_bits = 0, bad = 0;
    uint32_t pw = 0xffffffffu;  // previous TMA item: verified once its bulk group completed
    uint64_t psealed = 0;
    for (uint32_t w = w0; w < a.nitems; w += nwarps) {
        const Item it = a.items[w];
        const uint32_t body = fused_tma_body(a, it, w);
        if (body == 0) {  // register path, verified inline (copy_item_fused's read-back)
            uint64_t cptr[kMaxFused];
            uint32_t inject = 0;
#pragma unroll
            for (int k = 0; k < kMaxFused; k++) {
                cptr[k] = k < (int)a.ncons ? a.cons[k].items[w].ptr : 0;
                if (k < (int)a.ncons && w == a.cons[k].fault_item) inject |= 1u << k;
            }
            uint64_t got[kMaxFused] = {0, 0, 0, 0};
            const uint64_t sealed =
                warp_sum(copy_item_fused<kFusedUnroll>((const uint8_t *)it.ptr, a.packed + it.packed_off, cptr,
                                                       a.ncons, it.nbytes, it.packed_off, lane, inject, got)) +
                a.version * kVerMix;
            if (lane == 0) {
                a.iseal[w].mixed = sealed;
                a.iseal[w].version = a.version;
            }
#pragma unroll
            for (int k = 0; k < kMaxFused; k++) {
                if (k >= (int)a.ncons) break;
                if (warp_sum(got[k]) + a.version * kVerMix != sealed) bad |= 1u << k;
            }
            continue;
        }
        uint64_t acc = 0;
        uint32_t npieces = 0;
        for (uint32_t off = 0; off < body; off += kFtStage) {
            const uint32_t bytes = min(kFtStage, body - off);
            const int s = consumed % kFtStages;
            mbar_wait(bar + s, (phase_bits >> s) & 1u);
            phase_bits ^= 1u << s;
            const uint8_t *buf = stage + s * kFtStage;
            const uint32_t g0 = (uint32_t)((it.packed_off + off) >> 2);
            for (uint32_t i = lane; i < bytes / 16; i += 32)
                acc += cks_vec(*reinterpret_cast<const uint4 *>(buf + i * 16), g0 + 4u * i);
            __syncwarp();
            if (lane == 0) {
                asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
                bulk_s2g_nc(a.packed + it.packed_off + off, buf, bytes);
                for (uint32_t k = 0; k < a.ncons; k++) bulk_s2g_nc((uint8_t *)a.cons[k].items[w].ptr + off, buf, bytes);
                asm volatile("cp.async.bulk.commit_group;" ::: "memory");
            }
            consumed++;
            npieces++;
            Item nit;
            uint32_t nbytes;
            if (next_piece(ld, nit, nbytes)) {  // refill this stage once the stores have read it
                if (lane == 0) {
                    bulk_wait_read<0>();
                    mbar_expect_tx(bar + s, nbytes);
                    bulk_g2s(stage + s * kFtStage, (const uint8_t *)nit.ptr + ld.off, nbytes, bar + s);
                }
                ld.off += nbytes;
            }
        }
        const uint64_t sealed = warp_sum(acc) + a.version * kVerMix;
        if (lane == 0) {  // no concurrent reader in this path: a plain store (grid end publishes it)
            a.iseal[w].mixed = sealed;
            a.iseal[w].version = a.version;
        }
        if (VP_FT_READBACK && pw != 0xffffffffu) {
            // the previous item's group completed once at most this item's
            // `npieces` groups are still pending
            if (lane == 0) {
                if (npieces == 1) asm volatile("cp.async.bulk.wait_group 1;" ::: "memory");
                else asm volatile("cp.async.bulk.wait_group 0;" ::: "memory");
                asm volatile("fence.proxy.async.global;" ::: "memory");
            }
            __syncwarp();
            bad |= fused_verify_slots(a, pw, psealed, lane);
        }
        pw = w;
        psealed = sealed;
    }
    if (lane == 0) asm volatile("cp.async.bulk.wait_group 0;\n\tfence.proxy.async.global;" ::: "memory");
    __syncwarp();
    if (VP_FT_READBACK && pw != 0xffffffffu) bad |= fused_verify_slots(a, pw, psealed, lane);
    if (lane == 0 && bad) report_err(a.flags, bad);
    __syncthreads();
    uint32_t e;
    if (threadIdx.x == 0 && grid_arrive(a.flags, &e)) {
        if (a.sys_swap) asm volatile("fence.acq_rel.sys;" ::: "memory");  // peer slots: see install_finish
        for (uint32_t k = 0; k < a.ncons; k++) {
            const FusedCons &c = a.cons[k];
            const int32_t st = (e >> k) & 1u ? -5 : 0;
            if (c.status_h) *c.status_h = st;
            if (st == 0 && c.state_h) *c.state_h = (a.version << 1) | (uint64_t)c.target;  // the swap
            if (c.pin_h) *c.pin_h = 0;
        }
    }
}

}  // namespace

#if VP_WARP_PROF
extern "C" int vp_debug_warp_prof(unsigned long long *out, int nwarps) {
    cudaError_t e = cudaMemcpyFromSymbol(out, g_warp_prof, sizeof(unsigned long long) * 4 * (size_t)nwarps);
    if (e == cudaSuccess) e = cudaMemcpyFromSymbol(out + 4 * (size_t)nwarps, g_prof_end, sizeof(unsigned long long));
    return (int)e;
}
#endif

// Per-device launch facts, cached once per (kernel, device): the SM count and
// the dynamic shared-memory opt-in (cudaFuncSetAttribute applies to the
// current device only).  Lock-free; a race just repeats idempotent calls.
constexpr int kMaxDevices = 64;

static int sm_count(int device) {
    static std::atomic<int> cache[kMaxDevices];
    const int d = device >= 0 && device < kMaxDevices ? device : 0;
    int n = cache[d].load(std::memory_order_relaxed);
    if (n > 0) return n;
    if (cudaDeviceGetAttribute(&n, cudaDevAttrMultiProcessorCount, device) != cudaSuccess || n <= 0) n = 148;
    cache[d].store(n, std::memory_order_relaxed);
    return n;
}

// The launch runs on the CURRENT device (a SYNC publish launches a consumer's
// install on the producer's stream), so both facts are keyed on it, not on
// the endpoint's device.
static int launch_device() {
    int d = 0;
    cudaGetDevice(&d);
    return d;
}

template <typename Kernel>
static cudaError_t opt_in_smem(Kernel kernel, size_t smem, int /*endpoint device*/, std::atomic<uint64_t> &done) {
    const int device = launch_device();
    const uint64_t bit = 1ull << (device >= 0 && device < kMaxDevices ? device : 0);
    if (done.load(std::memory_order_acquire) & bit) return cudaSuccess;
    const cudaError_t e = cudaFuncSetAttribute(kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
    if (e == cudaSuccess) done.fetch_or(bit, std::memory_order_acq_rel);
    return e;  // not cached on failure: the next launch retries and reports again
}

static int grid_for(uint32_t nitems, int warps_per_block, int sms, int blocks_per_sm) {
    const uint32_t want = (nitems + warps_per_block - 1) / warps_per_block;
    const uint32_t cap = (uint32_t)sms * blocks_per_sm;
    return (int)(want < 1 ? 1 : (want > cap ? cap : want));
}

constexpr size_t kTmaSmem = (size_t)kTmaWarps * kTmaStages * kTmaStage + kTmaWarps * kTmaStages * sizeof(uint64_t);

FusedLaunch fused_tma_launch(uint32_t nitems, int device) {
    static std::atomic<uint64_t> opted{0};
    FusedLaunch l{};
    l.func = (const void *)publish_fused_tma_kernel;
    l.smem = kFtWarps * kFtStages * kFtStage + kFtWarps * kFtStages * sizeof(uint64_t);
    l.err = opt_in_smem(publish_fused_tma_kernel, l.smem, device, opted);
    l.grid = grid_for(nitems, kFtWarps, sm_count(launch_device()), 2);
    l.block = kFtWarps * 32;
    return l;
}

Geometry pick_geometry(uint32_t nitems, int device, int max_sms) {
    const int sms = sm_count(launch_device());
    Geometry g;
    g.items = nitems;
    g.block = kWarpsPerBlock * 32;
    g.grid = grid_for(nitems, kWarpsPerBlock, max_sms > 0 && max_sms < sms ? max_sms : sms, kBlocksPerSM);
    return g;
}

cudaError_t launch_pack(const PackArgs &a, const Geometry &g, cudaStream_t st) {
    if (a.nitems == 0) return cudaSuccess;
    void *args[] = {(void *)&a};
    return cudaLaunchKernel(pack_fn(a.s_packed, a.sys_release), dim3(g.grid), dim3(g.block), args, 0, st);
}

const void *fused_kernel_fn(uint32_t ncons) {
    return ncons <= 1 ? (const void *)publish_fused_kernel<1> : (const void *)publish_fused_kernel<kMaxFused>;
}

Geometry fused_geometry(const Geometry &g, int device, uint32_t ncons) {
    // same block shape, up to kFusedBlocks resident blocks per SM
    Geometry f = g;
    f.grid = grid_for(g.items, kWarpsPerBlock, sm_count(launch_device()), ncons <= 1 ? VP_FUSED1_BLOCKS : kFusedBlocks);
    return f;
}

cudaError_t launch_fused(const FusedArgs &a, const Geometry &g, cudaStream_t st) {
    if (a.ncons <= 1) publish_fused_kernel<1><<<g.grid, g.block, 0, st>>>(a);
    else publish_fused_kernel<kMaxFused><<<g.grid, g.block, 0, st>>>(a);
    return cudaGetLastError();
}

LaunchSpec pack_launch(const PackArgs &a, const Geometry &g, bool tma, int device) {
    LaunchSpec l{};
    if (tma) {
        static std::atomic<uint64_t> opted{0};
        l.func = (const void *)pack_seal_tma_kernel;
        l.err = opt_in_smem(pack_seal_tma_kernel, kTmaSmem, device, opted);
        l.grid = grid_for(a.nitems, kTmaWarps, sm_count(launch_device()), 2);
        l.block = kTmaWarps * 32;
        l.smem = kTmaSmem;
    } else {
        l.func = pack_fn(a.s_packed, a.sys_release);
        l.grid = g.grid;
        l.block = g.block;
    }
    return l;
}

LaunchSpec install_launch(const InstallArgs &a, const Geometry &g, bool tma, int device, int max_sms, bool direct,
                          uint64_t s_packed, bool pipe) {
    LaunchSpec l{};
    if (direct && !tma) {
        const int sms = sm_count(launch_device());
        l.func = install_direct_fn(s_packed, pipe);
        l.grid = grid_for(a.nitems, kWarpsPerBlock, max_sms > 0 && max_sms < sms ? max_sms : sms, kIdBlocks);
        l.block = g.block;
    } else if (tma) {
        static std::atomic<uint64_t> opted{0};
        const int sms = sm_count(launch_device());
        l.func = (const void *)install_verify_tma_kernel;
        l.err = opt_in_smem(install_verify_tma_kernel, kTmaSmem, device, opted);
        l.grid = grid_for(a.nitems, kTmaWarps, max_sms > 0 && max_sms < sms ? max_sms : sms, 2);
        l.block = kTmaWarps * 32;
        l.smem = kTmaSmem;
    } else {
        l.func = (const void *)install_verify_kernel;
        l.grid = g.grid;
        l.block = g.block;
    }
    return l;
}

LaunchSpec push_launch(const Geometry &g) {
    LaunchSpec l{};
    l.func = (const void *)pack_push_kernel;
    l.grid = g.grid;
    l.block = g.block;
    return l;
}

LaunchSpec nvls_launch(const Geometry &g) {
    LaunchSpec l{};
    l.func = (const void *)pack_nvls_kernel;
    l.grid = g.grid;
    l.block = g.block;
    return l;
}

LaunchSpec seal_reduce_launch(const SealReduceArgs &a) {
    LaunchSpec l{};
    l.func = (const void *)seal_reduce_kernel;
    l.grid = (int)((a.nchunks + 7) / 8);
    l.block = 256;
    return l;
}

// Load every kernel of the library into the current device's context now,
// at registration, instead of at its first launch (CUDA lazy loading).  A lazy
// load must wait for work already queued on the device, so the first launch
// of an install behind a stream that waits for a producer (DRAM-tier piece
// flags, an early-notified pack) could block the host thread for as long as
// that producer takes -- forever if it died.  Once per device.
cudaError_t preload_kernels() {
    static std::atomic<uint64_t> done{0};
    const int dev = launch_device();
    const uint64_t bit = 1ull << (dev >= 0 && dev < kMaxDevices ? dev : 0);
    if (done.load(std::memory_order_acquire) & bit) return cudaSuccess;
    const void *fns[] = {pack_fn(0), pack_fn(~0ull), pack_fn(0, true), pack_fn(~0ull, true),
                         (const void *)seal_reduce_kernel,
                         (const void *)install_verify_kernel,    install_direct_fn(0, false),
                         install_direct_fn(~0ull, false),        install_direct_fn(0, true),
                         install_direct_fn(~0ull, true),
                         fused_kernel_fn(1), fused_kernel_fn(kMaxFused), (const void *)pack_seal_tma_kernel,
                         (const void *)install_verify_tma_kernel, (const void *)publish_fused_tma_kernel,
                         (const void *)view_seal_kernel,         (const void *)pack_push_kernel,
                         (const void *)pack_nvls_kernel};
    for (const void *f : fns) {
        cudaFuncAttributes fa;
        const cudaError_t e = cudaFuncGetAttributes(&fa, f);
        if (e != cudaSuccess) return e;
    }
    // and the dynamic shared-memory opt-in of the TMA kernels (idempotent)
    const size_t ft = kFtWarps * kFtStages * kFtStage + kFtWarps * kFtStages * sizeof(uint64_t);
    cudaError_t e = cudaFuncSetAttribute(pack_seal_tma_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)kTmaSmem);
    if (e == cudaSuccess)
        e = cudaFuncSetAttribute(install_verify_tma_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)kTmaSmem);
    if (e == cudaSuccess)
        e = cudaFuncSetAttribute(publish_fused_tma_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)ft);
    if (e != cudaSuccess) return e;
    done.fetch_or(bit, std::memory_order_acq_rel);
    return cudaSuccess;
}

cudaError_t launch_view_seals(const ViewSealArgs &a, cudaStream_t st) {
    if (a.nitems == 0) return cudaSuccess;
    int dev = 0;
    cudaGetDevice(&dev);
    view_seal_kernel<<<grid_for(a.nitems, kWarpsPerBlock, sm_count(dev), kBlocksPerSM), kWarpsPerBlock * 32, 0, st>>>(
        a);
    return cudaGetLastError();
}

cudaError_t launch_install(const InstallArgs &a, const Geometry &g, cudaStream_t st, bool pdl, bool direct,
                           uint64_t s_packed) {
    cudaLaunchConfig_t cfg{};
    cfg.gridDim = dim3(g.grid);
    cfg.blockDim = dim3(g.block);
    cfg.stream = st;
    cudaLaunchAttribute attr[1];
    attr[0].id = cudaLaunchAttributeProgrammaticStreamSerialization;
    attr[0].val.programmaticStreamSerializationAllowed = 1;
    cfg.attrs = attr;
    cfg.numAttrs = pdl ? 1 : 0;
    if (!direct) return cudaLaunchKernelEx(&cfg, install_verify_kernel, a);
    const int sms = sm_count(launch_device());
    cfg.gridDim = dim3(grid_for(a.nitems, kWarpsPerBlock, sms, kIdBlocks));
    void *args[] = {(void *)&a};
    return cudaLaunchKernelExC(&cfg, install_direct_fn(s_packed, true), args);
}

}  // namespace vp
