// vp_internal.h -- internal types shared by the kernels and the host runtime of
// libviper.so (never exported; the public boundary is include/viper.h).
#pragma once
#include <cstdint>
#include <cuda_runtime.h>

namespace vp {

// One warp work item: a <= item_max byte piece of one tensor that lies inside
// one seal chunk.  The same list drives pack (tensor -> packed) and install
// (packed -> slot tensor): LAY depends only on the sizes, never on pointers.
struct Item {
    uint64_t packed_off;   // byte offset in the packed buffer (16-B aligned)
    uint64_t tensor_off;   // byte offset inside the tensor
    uint32_t nbytes;       // bytes of this piece (multiple of 16 except a tensor tail)
    uint32_t tensor;       // tensor index
    uint32_t chunk;        // seal chunk index
    uint32_t chunk_items;  // number of items of that chunk (last-arriver test)
};
static_assert(sizeof(Item) == 32, "Item must stay 32 B");

struct Seal {
    uint64_t version;
    uint64_t cks;
};

// Checksum weight constant (R16 / CKS): term_g = w_g * ((2g+1)*K) mod 2^32.
constexpr uint32_t kCksK = 0x9E3779B1u;

// Per-launch scratch that the kernels leave zeroed when they finish
// (self-resetting: no memset launch between versions).
struct Scratch {
    uint64_t *acc;      // [nchunks] running checksum of the chunk
    uint32_t *cnt;      // [nchunks] items finished in the chunk
    uint32_t *done;     // [1] chunks finished
    uint32_t *err;      // [1] error bits of this launch
};

enum : uint32_t { kErrChecksum = 1u, kErrVersion = 2u };

struct PackArgs {
    const Item *items;
    uint32_t nitems, nchunks;
    const uint8_t *const *src;  // [T] producer tensor base pointers (device)
    uint8_t *packed;            // snapshot buffer
    Seal *seals;                // [nchunks] written {version, cks}
    Scratch s;
    uint64_t version;
};

struct InstallArgs {
    const Item *items;
    uint32_t nitems, nchunks;
    uint8_t *const *dst;        // [T] target slot tensor base pointers (device)
    const uint8_t *packed;      // source: snapshot (local or peer-mapped) or staging
    const Seal *seals;          // expected seals (same origin as packed)
    Scratch s;
    uint64_t version;
    uint32_t target;            // slot being written
    uint32_t fault_item;        // item whose first byte is flipped (fault injection); ~0u = none
    // Host-mapped control words (cudaHostAlloc/cudaHostRegister mapped).
    // The last finishing warp writes *status_h, clears *pin_h and, on success,
    // flips *state_h = (version << 1) | target: the atomic version swap.
    volatile int32_t *status_h;
    volatile uint64_t *pin_h;
    volatile uint64_t *state_h;
};

// Work-list geometry chosen on the host (kernels.cu).
struct Geometry {
    int grid, block;
};
Geometry pick_geometry(uint32_t nitems, int device);

cudaError_t launch_pack(const PackArgs &a, const Geometry &g, cudaStream_t st);
cudaError_t launch_install(const InstallArgs &a, const Geometry &g, cudaStream_t st);

}  // namespace vp
