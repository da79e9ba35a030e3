// protocol.h -- the host-side version protocol (SURVEY s8(a) a3/a7/a8,
// DESIGN.md s7), free of CUDA so that it is exercised by CPU multi-process
// tests (selftest.cpp) and a ThreadSanitizer build (tests/tsan_protocol.cpp)
// exactly as the engine uses it.
//
//   producer slot reuse  pub_state <- newer; fence; scan pins   (wait_unpinned)
//   consumer snapshot pin pin <- v; fence; re-read pub_state     (pin_latest)
//   writer (install)     wait ref[target] == 0                   (wait_readers_gone)
//   reader               s <- state; ref[slot]++; re-read state  (try_acquire_slot)
// All seq_cst std::atomic on words that may live in a shared-memory segment.
#pragma once
#include <errno.h>
#include <sched.h>
#include <signal.h>

#include <atomic>
#include <cstdint>

#include "runtime.h"

namespace vp {

// Failure detection: a consumer whose process no longer exists is marked
// inactive (its pin and refcounts no longer hold anything back).
inline bool consumer_alive(ConsRec *r) {
    const int32_t pid = r->pid.load();
    if (pid <= 0) return true;  // in-process consumer
    if (kill(pid, 0) == -1 && errno == ESRCH) {
        r->active.store(0);
        return false;
    }
    return true;
}

// Producer: before overwriting the snapshot slot that holds old_v, wait until
// no active consumer pins old_v.  Returns false (and *who) on timeout.
inline bool wait_unpinned(Ctrl *ctrl, uint64_t old_v, int64_t timeout_ns, int *who) {
    const int nc = ctrl->ncons.load();
    for (int i = 0; i < nc; i++) {
        const int64_t w0 = now_ns();
        uint32_t spins = 0;
        while (ctrl->cons[i].active.load() && ctrl->cons[i].pin.load() == old_v) {
            if (now_ns() - w0 > timeout_ns) {
                if (who) *who = i;
                return false;
            }
            if ((++spins & 0xFFFF) == 0 && !consumer_alive(&ctrl->cons[i])) break;
            __builtin_ia32_pause();
        }
    }
    return true;
}

// Consumer: pin the latest published snapshot (v, slot b).  The Dekker pair of
// wait_unpinned: pin <- v; re-read pub_state; undo if it moved.
inline bool pin_latest(Ctrl *ctrl, ConsRec *r, uint64_t *v, int *b) {
    for (;;) {
        const uint64_t ps = ctrl->pub_state.load();
        if (ps == 0) return false;
        r->pin.store(ps >> 1);
        if (ctrl->pub_state.load() == ps) {
            *v = ps >> 1;
            *b = (int)(ps & 1);
            return true;
        }
        r->pin.store(0);
    }
}

// Multi-producer: the version every producer published (all pub_m equal).
inline bool all_published(Ctrl *ctrl, int M, uint64_t *word) {
    const uint64_t w0 = ctrl->pub_m[0].load();
    for (int j = 1; j < M; j++)
        if (ctrl->pub_m[j].load() != w0) return false;
    *word = w0;
    return w0 != 0;
}

// Multi-producer pin: v once every producer published it, re-validated after the pin.
inline bool pin_latest_m(Ctrl *ctrl, ConsRec *r, int M, uint64_t *v, int *b) {
    for (int tries = 0; tries < 1000; tries++) {
        uint64_t w;
        if (!all_published(ctrl, M, &w)) {
            sched_yield();
            continue;
        }
        r->pin.store(w >> 1);
        uint64_t w2;
        if (all_published(ctrl, M, &w2) && w2 == w) {
            *v = w >> 1;
            *b = (int)(w & 1);
            return true;
        }
        r->pin.store(0);
    }
    return false;
}

// Writer: the alternative copy is written only once no reader pins it.
inline bool wait_readers_gone(ConsRec *r, int target, int64_t timeout_ns) {
    const int64_t t0 = now_ns();
    while (r->ref[target].load() != 0) {
        if (now_ns() - t0 > timeout_ns) return false;
        sched_yield();
    }
    return true;
}

// Reader: pin the active slot; returns the state word (version << 1 | slot)
// with ref[slot] held, or 0 when nothing >= min_version is installed.
inline uint64_t try_acquire_slot(ConsRec *r, uint64_t min_version) {
    for (;;) {
        const uint64_t s = r->state.load();
        if (s == 0 || (s >> 1) < min_version) return 0;
        const int slot = (int)(s & 1);
        r->ref[slot].fetch_add(1);
        if (r->state.load() == s) return s;
        r->ref[slot].fetch_sub(1);  // swapped under us: retry
    }
}

inline void release_slot(ConsRec *r, int slot) { r->ref[slot].fetch_sub(1); }

// The slot an install writes: the inactive one (slot 0 before the first install).
inline int install_target(ConsRec *r) {
    const uint64_t cur = r->state.load();
    return cur == 0 ? 0 : (int)(1 - (cur & 1));
}

}  // namespace vp
