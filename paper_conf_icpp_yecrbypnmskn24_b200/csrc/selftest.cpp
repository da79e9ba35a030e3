// selftest.cpp -- CUDA-free drivers of the version protocol (protocol.h,
// pin_latest) over a real shared-memory segment, so multi-process CPU tests
// (tests/test_protocol_mp.py, gloo world size 2) exercise the same host logic
// the engine runs between producer and consumer processes.
//
// Model: the "snapshot" is two slots of K u64 words; publish(v) waits until
// slot v&1 is unpinned, fills it with v, names it in pub_state.  A consumer
// pins the latest snapshot, copies it into its own double buffer (two slots
// of K words, ref-counted) and swaps its state word; readers acquire a slot,
// check that every word equals the slot's version, release.  A torn or
// mixed-version read shows up as a word != version.
#include <fcntl.h>
#include <sys/mman.h>
#include <unistd.h>

#include <cstring>
#include <new>

#include "protocol.h"
#include "runtime.h"
#include "selector.h"

using namespace vp;

namespace {

struct Seg {
    void *base;
    size_t bytes;
    uint64_t words;
    Ctrl *ctrl;
    uint64_t *snap;  // [2][words]
    uint64_t *cons;  // [kMaxConsumers][2][words]
    uint64_t last_v;
};

size_t seg_bytes(uint64_t words) {
    return (sizeof(Ctrl) + 4095) / 4096 * 4096 + sizeof(uint64_t) * words * 2 * (1 + kMaxConsumers);
}

Seg *map_seg(const char *path, uint64_t words, bool create) {
    const size_t bytes = seg_bytes(words);
    const int fd = shm_open(path, create ? (O_CREAT | O_EXCL | O_RDWR) : O_RDWR, 0600);
    if (fd < 0) return nullptr;
    if (create && ftruncate(fd, (off_t)bytes) != 0) {
        close(fd);
        return nullptr;
    }
    void *p = mmap(nullptr, bytes, PROT_READ | PROT_WRITE, MAP_SHARED, fd, 0);
    close(fd);
    if (p == MAP_FAILED) return nullptr;
    Seg *s = new Seg{p, bytes, words, (Ctrl *)p, nullptr, nullptr, 0};
    s->snap = (uint64_t *)((uint8_t *)p + (sizeof(Ctrl) + 4095) / 4096 * 4096);
    s->cons = s->snap + 2 * words;
    if (create) {
        memset(p, 0, bytes);
        new (p) Ctrl();
        s->ctrl->magic = kCtrlMagic;
    }
    return s;
}

}  // namespace

extern "C" {

viper_status viper_debug_proto_create(const char *path, uint64_t words, int32_t ncons, void **out) {
    Seg *s = map_seg(path, words, true);
    if (!s) return set_error(VIPER_E_NOMEM, "shm %s", path);
    s->ctrl->ncons.store(ncons);
    for (int i = 0; i < ncons; i++) s->ctrl->cons[i].active.store(1);
    *out = s;
    return VIPER_OK;
}

viper_status viper_debug_proto_open(const char *path, uint64_t words, void **out) {
    Seg *s = map_seg(path, words, false);
    if (!s || s->ctrl->magic != kCtrlMagic) return set_error(VIPER_E_PEER, "shm %s", path);
    *out = s;
    return VIPER_OK;
}

viper_status viper_debug_proto_close(void *h, int32_t unlink_it, const char *path) {
    Seg *s = (Seg *)h;
    munmap(s->base, s->bytes);
    if (unlink_it && path) shm_unlink(path);
    delete s;
    return VIPER_OK;
}

// Producer: publish version v into snapshot slot v & 1 (a3 + slot reuse).
viper_status viper_debug_proto_publish(void *h, uint64_t v) {
    Seg *s = (Seg *)h;
    if (v <= s->last_v) return set_error(VIPER_E_VERSION, "versions increase");
    const int b = (int)(v & 1);
    const uint64_t old_v = v >= 2 ? v - 2 : 0;
    int who = -1;
    if (old_v && !wait_unpinned(s->ctrl, old_v, 10ll * 1000000000ll, &who))
        return set_error(VIPER_E_TIMEOUT, "consumer %d pinned v%llu", who, (unsigned long long)old_v);
    volatile uint64_t *slot = s->snap + b * s->words;
    for (uint64_t i = 0; i < s->words; i++) slot[i] = v;  // the "pack"
    std::atomic_thread_fence(std::memory_order_seq_cst);
    s->ctrl->pub_state.store((v << 1) | (uint64_t)b);
    s->ctrl->pub_seq.fetch_add(1);
    futex_wake_all(&s->ctrl->pub_seq);
    s->last_v = v;
    return VIPER_OK;
}

// Consumer cidx: install the latest published version into its double buffer
// (a6 + a7).  *installed = the version installed, 0 if nothing new.
// *torn_snapshot counts snapshot words that changed while pinned.
viper_status viper_debug_proto_install(void *h, int32_t cidx, uint64_t *installed, uint64_t *torn_snapshot) {
    Seg *s = (Seg *)h;
    ConsRec *r = &s->ctrl->cons[cidx];
    *installed = 0;
    uint64_t v;
    int b;
    if (!pin_latest(s->ctrl, r, &v, &b)) return VIPER_OK;
    const uint64_t cur = r->state.load();
    if (cur && (cur >> 1) >= v) {
        r->pin.store(0);
        return VIPER_OK;
    }
    const int target = install_target(r);
    if (!wait_readers_gone(r, target, 10ll * 1000000000ll)) {
        r->pin.store(0);
        return set_error(VIPER_E_TIMEOUT, "readers kept slot %d", target);
    }
    volatile uint64_t *src = s->snap + b * s->words;
    volatile uint64_t *dst = s->cons + ((uint64_t)cidx * 2 + target) * s->words;
    uint64_t bad = 0;
    for (uint64_t i = 0; i < s->words; i++) {
        const uint64_t x = src[i];
        bad += x != v;
        dst[i] = x;
    }
    std::atomic_thread_fence(std::memory_order_seq_cst);
    if (!bad) r->state.store((v << 1) | (uint64_t)target);  // the swap
    r->pin.store(0);
    r->done_version.store(v);
    *installed = bad ? 0 : v;
    *torn_snapshot = bad;
    return VIPER_OK;
}

// Reader on consumer cidx (a8): acquire, verify every word == version, release.
viper_status viper_debug_proto_read(void *h, int32_t cidx, uint64_t *version, uint64_t *torn) {
    Seg *s = (Seg *)h;
    ConsRec *r = &s->ctrl->cons[cidx];
    const uint64_t st = try_acquire_slot(r, 0);
    *version = 0;
    *torn = 0;
    if (!st) return VIPER_OK;
    const int slot = (int)(st & 1);
    const uint64_t v = st >> 1;
    volatile uint64_t *p = s->cons + ((uint64_t)cidx * 2 + slot) * s->words;
    uint64_t bad = 0;
    for (int pass = 0; pass < 2; pass++)  // twice: the slot must not change while pinned
        for (uint64_t i = 0; i < s->words; i++) bad += p[i] != v;
    release_slot(r, slot);
    *version = v;
    *torn = bad;
    return VIPER_OK;
}

// Transfer Selector (selector.h) on synthetic gathered records.
viper_status viper_debug_resolve_tier(const void *records, int32_t world, int32_t producer_rank,
                                      int32_t nproducers, int32_t fanout, int32_t requested, int32_t *out) {
    const int M = nproducers > 1 ? nproducers : 1;
    if (!records || !out || world < 1 || producer_rank < 0 || producer_rank + M > world)
        return set_error(VIPER_E_INVAL, "bad arguments");
    *out = resolve_tier((const TierRec *)records, world, producer_rank, M, fanout, requested);
    return VIPER_OK;
}

}  // extern "C"
