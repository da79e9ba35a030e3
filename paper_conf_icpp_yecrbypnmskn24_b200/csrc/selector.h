// selector.h -- the Transfer Selector's decision (Fig. 7, PAPER.md P:1776-1784;
// DESIGN.md s1 "Transfer Selector"), free of CUDA so that CPU tests drive it
// with synthetic records (selftest.cpp, viper_debug_resolve_tier) exactly as
// the cross-process bootstrap (xproc.cpp) uses it.
//
// Every rank contributes one TierRec to the first bootstrap allgather: the
// tier it asked for, its GPU's PCI bus id and the PCI bus ids its GPU can
// peer-access (itself first).  Every rank then resolves VIPER_TIER_AUTO from
// the same gathered array, so all ranks reach the same answer.
#pragma once
#include <cstdint>
#include <cstring>

#include "viper.h"

namespace vp {

constexpr uint32_t kTierMagic = 0x56495452u;  // "VITR"
constexpr int kMaxReach = 16;

struct TierRec {
    uint32_t magic;  // kTierMagic; 0 = a rank that failed before the bootstrap
    int32_t tier, nreach, pad;
    char pci[16];
    char reach[kMaxReach][16];
};
static_assert(sizeof(TierRec) == 288, "TierRec is exchanged between processes: keep its layout");

// Rank a's GPU can read rank b's GPU memory.  Records of failed ranks decide
// nothing (those ranks fail the registration in the next round anyway).
inline bool tier_reaches(const TierRec *all, int a, int b) {
    if (all[a].magic != kTierMagic || all[b].magic != kTierMagic) return true;
    for (int k = 0; k < all[a].nreach && k < kMaxReach; k++)
        if (strncmp(all[a].reach[k], all[b].pci, 16) == 0) return true;
    return false;
}

// `requested` unless it is VIPER_TIER_AUTO; then the GPU tier when every
// consumer reaches every producer (ranks [producer_rank, producer_rank + M))
// and -- with chain / scatter-allgather fan-out, where consumers also pull
// from each other -- every other consumer; with push / NVLS fan-out, where
// the producer writes into the consumers' memory, every producer must also
// reach every consumer; else the DRAM tier.  Otherwise the producers' own
// reach does not matter: nobody pulls from a consumer into a producer.
inline int32_t resolve_tier(const TierRec *all, int world, int producer_rank, int M, int32_t fanout,
                            int32_t requested) {
    if (requested != VIPER_TIER_AUTO) return requested;
    auto producer = [&](int r) { return r >= producer_rank && r < producer_rank + M; };
    const bool peers = fanout == VIPER_FANOUT_CHAIN || fanout == VIPER_FANOUT_SCATTER_ALLGATHER;
    const bool writes = fanout == VIPER_FANOUT_PUSH || fanout == VIPER_FANOUT_NVLS;
    for (int c = 0; c < world; c++) {
        if (producer(c)) continue;
        for (int r = 0; r < world; r++) {
            if (r != c && (producer(r) || peers) && !tier_reaches(all, c, r)) return VIPER_TIER_DRAM;
            if (writes && producer(r) && !tier_reaches(all, r, c)) return VIPER_TIER_DRAM;
        }
    }
    return VIPER_TIER_GPU;
}

}  // namespace vp
