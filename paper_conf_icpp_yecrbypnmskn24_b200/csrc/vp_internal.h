// vp_internal.h -- internal types shared by the kernels and the host runtime of
// libviper.so (never exported; the public boundary is include/viper.h).
#pragma once
#include <cstdint>
#include <cuda_runtime.h>

namespace vp {

// One warp work item: a <= item_max byte piece of one tensor that lies inside
// one seal chunk.  `ptr` is the absolute device address of the piece in the
// tensor (producer: its parameter; consumer: the slot's copy), so a warp needs
// one dependent load (the item) before it streams data.
struct Item {
    uint64_t ptr;          // tensor-side address of this piece
    uint64_t packed_off;   // byte offset in the packed buffer (16-B aligned)
    uint32_t nbytes;       // bytes of this piece (multiple of 16 except a tensor tail)
    uint32_t chunk;        // seal chunk index
    uint32_t tensor;       // tensor index
    uint32_t gidx;         // index in the full work list (item seals are indexed by it)
};
static_assert(sizeof(Item) == 32, "Item must stay 32 B");

struct Seal {
    uint64_t version;
    uint64_t cks;
};

// Item seal: cks(item) + version * kVerMix, then the item's version as a
// ready flag (written with release semantics after the item's data).
struct ISeal {
    uint64_t mixed;
    uint64_t version;
};
static_assert(sizeof(ISeal) == 16, "ISeal must stay 16 B");

// CKS weight constant (R16): term_g = w_g * ((2g+1)*K) mod 2^32.
constexpr uint32_t kCksK = 0x9E3779B1u;
// Item seal = cks(item) + version * kVerMix (mod 2^64): binds every item's
// checksum to the version, so stale-but-consistent data fails verification.
constexpr uint64_t kVerMix = 0x9E3779B97F4A7C15ull;

enum : uint32_t { kErrChecksum = 1u, kErrTimeout = 2u };
// an install waits at most this long for one item's ready flag (producer gone)
constexpr uint64_t kItemWaitNs = 30ull * 1000000000ull;

struct PackArgs {
    const Item *items;          // producer list (ptr = parameter tensor piece)
    uint32_t nitems;
    uint8_t *packed;            // snapshot buffer
    ISeal *iseal;               // [nitems] item seals + ready flags (written)
    uint64_t version;
    uint32_t sys_release;       // release the ready flags at system scope (consumers
                                // on other GPUs pipeline behind this pack)
    uint32_t l2_once;           // TMA variant: load the tensors with an L2 evict-first hint
                                // (set when the snapshot fits in L2, so it stays there)
    uint64_t s_packed;          // packed size (selects the kernel instantiation)
};

// Push delivery (VIPER_FANOUT_PUSH): the pack also stores every item into
// each consumer's peer-mapped staging slot and releases its seal there.
constexpr int kMaxPush = 8;
struct PushArgs {
    PackArgs p;                 // the local pack (snapshot + item seals)
    uint32_t ndst;              // consumers
    uint8_t *dst[kMaxPush];     // consumer k's staging for this snapshot slot (peer-mapped)
    ISeal *dst_iseal[kMaxPush]; // consumer k's staging item seals
};

// NVLS multicast delivery (VIPER_FANOUT_NVLS): stores go to the multicast
// address of the snapshot slot; NVSwitch replicates them to every bound rank.
struct NvlsArgs {
    const Item *items;
    uint32_t nitems;
    uint8_t *mc_packed;         // multicast VA of snapshot slot b
    ISeal *mc_iseal;            // multicast VA of its item seals
    uint64_t version;
};

struct SealReduceArgs {
    const uint32_t *chunk_first;  // [nchunks + 1] item ranges of the chunks
    uint32_t nchunks;
    const ISeal *iseal;
    Seal *seals;                  // [nchunks] {version, cks} (written)
    uint64_t version;
    uint32_t share_n, share_me;   // multi-producer: only chunks c % share_n == share_me
};

// viper_view_seals: chunk seals of a consumer slot, computed in place.
struct ViewSealArgs {
    const Item *items;          // the slot's work list (ptr = slot tensor piece)
    uint32_t nitems;
    Seal *seals;                // [nchunks], zeroed by the caller; {version, cks} (written)
    uint64_t version;
};
cudaError_t launch_view_seals(const ViewSealArgs &a, cudaStream_t st);
// load every kernel into the current device's context (no lazy load at a launch)
cudaError_t preload_kernels();

struct InstallArgs {
    const Item *items;          // consumer list of the target slot (ptr = slot tensor piece)
    uint32_t nitems;
    const uint8_t *packed;      // source: snapshot (local or peer-mapped) or DRAM staging
    const ISeal *iseal;         // expected item seals + ready flags (same origin as packed)
    uint64_t version;
    uint32_t target;            // slot being written
    uint32_t fault_item;        // item whose first word is flipped (fault injection); ~0u = none
    unsigned long long *flags;  // [1] low 32 bits: blocks finished; high 32: error bits (self-resetting)
    unsigned int *ctr;          // work counter (kernels.cu WorkQueue), reset by the last block; NULL = static
    // Host-mapped control words (cudaHostAlloc/cudaHostRegister mapped).  The
    // last block writes *status_h, clears *pin_h and, when every item matched,
    // flips *state_h = (version << 1) | target: the atomic version swap.
    volatile int32_t *status_h;
    volatile uint64_t *pin_h;
    volatile uint64_t *state_h;
    const volatile int32_t *abort_h;  // host-mapped: nonzero = stop waiting for seals (report a timeout)
    // Scatter-allgather fan-out (sa_n > 0): item x is owned by consumer
    // chunk(x) % sa_n.  Owned items come from the producer (`packed`) and are
    // also written to this consumer's staging (+ seal, release.sys) for its
    // peers; the others are pulled from the owner's staging once its seal
    // shows `version`, falling back to the producer when the owner is not
    // installing this version.
    // Chain fan-out (sa_n > 0, chain = 1): consumer i pulls every item from
    // consumer i-1's staging (consumer 0 from the producer) and stages it for
    // consumer i+1 (all but the last), with the same seals and fallbacks.
    uint32_t sa_n, sa_me, chain;
    // Multi-producer fan-in (mp_n > 1): item x comes from producer
    // chunk(x) % mp_n (data-parallel replicas each pack their share)
    uint32_t mp_n;
    const uint8_t *const *mp_snap;               // [mp_n] producers' snapshot slot (device-mapped)
    const ISeal *const *mp_iseal;                // [mp_n] producers' item seals
    uint8_t *sa_stage_out;
    ISeal *sa_iseal_out;
    const uint8_t *const *sa_src;                // [sa_n] peers' staging (device-mapped)
    const ISeal *const *sa_isrc;                 // [sa_n] peers' staging seals
    const volatile uint64_t *const *sa_owner_pin;  // [sa_n] peers' pin words (host-mapped)
    uint32_t l2_once;           // TMA variant: load the snapshot with an L2 evict-first hint
    uint32_t sys_swap;          // the slot is on another GPU than the kernel: system-scope fence before the swap
};

// SYNC in-process publish (K2+K6 fused): each warp packs its item,
// then reads that snapshot piece back (L2) and installs + verifies it into up
// to kMaxFused consumers' inactive slots; the last block swaps their versions.
constexpr int kMaxFused = 4;
struct FusedCons {
    const Item *items;          // consumer list of its target slot
    uint32_t target;
    uint32_t fault_item;
    volatile int32_t *status_h;
    volatile uint64_t *pin_h;
    volatile uint64_t *state_h;
};
struct FusedArgs {
    const Item *items;          // producer list
    uint32_t nitems;
    uint32_t ncons;
    uint8_t *packed;
    ISeal *iseal;
    uint64_t version;
    unsigned long long *flags;  // [1] low 32: blocks finished; high 32: bit k = consumer k failed (self-resetting);
                                // flags + 1: the work counter (kernels.cu WorkQueue), reset by the last block
    FusedCons cons[kMaxFused];
    uint32_t sys_swap;          // a consumer slot is on another GPU: system-scope fence before the swaps
};

struct Geometry {
    int grid, block;
    uint32_t items = 0;
};
Geometry fused_geometry(const Geometry &g, int device, uint32_t ncons);  // publish_fused_kernel's grid (own occupancy)
Geometry pick_geometry(uint32_t nitems, int device, int max_sms = 0);  // max_sms > 0: at most that many SMs

cudaError_t launch_pack(const PackArgs &a, const Geometry &g, cudaStream_t st);
cudaError_t launch_fused(const FusedArgs &a, const Geometry &g, cudaStream_t st);
const void *fused_kernel_fn(uint32_t ncons);  // for the one-node launch graph (runtime.cpp)
// A kernel launch as data (function, geometry, dynamic shared memory) for the
// one-node launch graphs of runtime.cpp; err != cudaSuccess: not launchable.
struct LaunchSpec {
    const void *func;
    int grid, block;
    size_t smem;
    cudaError_t err;
};
using FusedLaunch = LaunchSpec;
// TMA bulk-copy variant of the fused kernel
FusedLaunch fused_tma_launch(uint32_t nitems, int device);
// pack_seal (register, geometry g) or pack_seal_tma; seal_reduce
LaunchSpec pack_launch(const PackArgs &a, const Geometry &g, bool tma, int device);
LaunchSpec seal_reduce_launch(const SealReduceArgs &a);
// pack_push / pack_nvls (register streaming, geometry g)
LaunchSpec push_launch(const Geometry &g);
LaunchSpec nvls_launch(const Geometry &g);
// install_verify (register, geometry g, not PDL-chained), install_verify_tma, or
// install_direct (direct = a complete snapshot from one source, register streaming)
LaunchSpec install_launch(const InstallArgs &a, const Geometry &g, bool tma, int device, int max_sms,
                          bool direct = false, uint64_t s_packed = 0, bool pipe = false);
#ifndef VP_INSTALL_TMA_DEFAULT
#define VP_INSTALL_TMA_DEFAULT 1
#endif
// complete-snapshot installs <= 1 GiB use the TMA kernel (else install_direct).  Cold (ncu) the two tie
// within 3%; right behind the pack that wrote the snapshot into L2 (CUDA events), TMA's asynchronous bulk
// stores ride out the write-back of the dirty snapshot better: ResNet-50 34.2 vs 38.3 us
// (profiles/r02/install_sweep.json, profiles/r02/ktime_install_ab.log)
constexpr bool kInstallTmaDefault = VP_INSTALL_TMA_DEFAULT != 0;
#ifndef VP_FUSED_TMA_DEFAULT
#define VP_FUSED_TMA_DEFAULT 0
#endif
// SYNC in-process publishes use the TMA fused kernel (VIPER_FUSED_TMA=0/1 overrides)
constexpr bool kFusedTmaDefault = VP_FUSED_TMA_DEFAULT != 0;
constexpr uint64_t kFusedTmaMaxBytes = 1ull << 30;  // auto-selection limit (packed bytes)
// pdl: the install directly follows the pack on `st` (programmatic dependent launch);
// direct: one source (install_direct_kernel, pipelined), else install_verify_kernel
cudaError_t launch_install(const InstallArgs &a, const Geometry &g, cudaStream_t st, bool pdl, bool direct = false,
                           uint64_t s_packed = 0);

}  // namespace vp
