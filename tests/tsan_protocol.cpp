// tsan_protocol.cpp -- ThreadSanitizer driver of the engine's host version
// protocol (paper_conf_icpp_yecrbypnmskn24_b200/csrc/protocol.h, the same
// header libviper.so compiles; SURVEY s4 T3 "host TSan build of the
// protocol").  Test infrastructure, built and run by tests/test_tsan_protocol.py.
//
// One producer publishes versions 1..V into a two-slot snapshot (plain
// stores); each consumer pins the latest snapshot, waits until no reader holds
// its inactive slot, copies the snapshot into it (plain loads and stores) and
// swaps its state word; readers acquire a slot, read every word (plain loads)
// and release it.  The data words are NOT atomic: any ordering the protocol
// fails to establish between a writer and a reader is a data race that TSan
// reports (exit 66), and any mixed-version read shows up as a torn count.
//
// -DMUTANT=1 drops the writer's wait for readers (wait_readers_gone) and
// -DMUTANT=2 drops the producer's pin scan (wait_unpinned): both must fail.
#include <cstdio>
#include <cstdlib>
#include <ctime>
#include <thread>
#include <vector>

#include "../paper_conf_icpp_yecrbypnmskn24_b200/csrc/protocol.h"

#ifndef MUTANT
#define MUTANT 0
#endif
#if MUTANT == 2
#define WAIT_UNPINNED(ctrl, v) true
#else
#define WAIT_UNPINNED(ctrl, v) wait_unpinned((ctrl), (v), 10ll * 1000000000ll, nullptr)
#endif

namespace vp {
int64_t now_ns() {  // libviper.so's definition lives in runtime.cpp (CUDA); same clock
    timespec ts;
    clock_gettime(CLOCK_MONOTONIC, &ts);
    return (int64_t)ts.tv_sec * 1000000000ll + ts.tv_nsec;
}
}  // namespace vp

using namespace vp;

int main(int argc, char **argv) {
    const uint64_t V = argc > 1 ? strtoull(argv[1], nullptr, 10) : 20000;
    const int NC = 2, NR = 2, K = 64;
    Ctrl *ctrl = new Ctrl();
    ctrl->ncons.store(NC);
    for (int i = 0; i < NC; i++) ctrl->cons[i].active.store(1);
    std::vector<uint64_t> snap(2 * K, 0), slots((size_t)NC * 2 * K, 0);
    std::atomic<bool> done{false};
    std::atomic<uint64_t> torn{0}, regress{0}, reads{0}, installs{0};

    std::thread producer([&] {
        uint64_t snap_version[2] = {0, 0};
        for (uint64_t v = 1; v <= V; v++) {
            const int b = (int)(v & 1);
            if (snap_version[b] && !WAIT_UNPINNED(ctrl, snap_version[b])) {
                fprintf(stderr, "producer: pin wait timed out\n");
                exit(2);
            }
            for (int k = 0; k < K; k++) snap[b * K + k] = v;  // the pack
            snap_version[b] = v;
            ctrl->pub_state.store((v << 1) | (uint64_t)b);  // publish
            std::this_thread::yield();  // let installs interleave with publishes
        }
        done.store(true);
    });

    std::vector<std::thread> consumers, readers;
    for (int i = 0; i < NC; i++) {
        consumers.emplace_back([&, i] {
            ConsRec *r = &ctrl->cons[i];
            uint64_t attempted = 0;
            for (;;) {
                uint64_t v;
                int b;
                if (!pin_latest(ctrl, r, &v, &b)) continue;
                if (v <= attempted) {
                    r->pin.store(0);
                    if (done.load() && v == V) break;
                    continue;
                }
                const int target = install_target(r);
#if MUTANT != 1
                if (!wait_readers_gone(r, target, 10ll * 1000000000ll)) {
                    fprintf(stderr, "consumer %d: readers never left\n", i);
                    exit(2);
                }
#endif
                uint64_t *dst = &slots[((size_t)i * 2 + target) * K];
                for (int k = 0; k < K; k++) dst[k] = snap[b * K + k];  // the install
                r->state.store((v << 1) | (uint64_t)target);            // the swap
                r->pin.store(0);
                attempted = v;
                installs.fetch_add(1);
            }
        });
        for (int j = 0; j < NR; j++) {
            readers.emplace_back([&, i] {
                ConsRec *r = &ctrl->cons[i];
                uint64_t last = 0;
                for (;;) {
                    const bool finished = done.load() && (r->state.load() >> 1) == V;
                    const uint64_t s = try_acquire_slot(r, 1);
                    if (s) {
                        const int slot = (int)(s & 1);
                        const uint64_t *src = &slots[((size_t)i * 2 + slot) * K];
                        uint64_t bad = 0;
                        for (int k = 0; k < K; k++) bad += src[k] != (s >> 1);
                        release_slot(r, slot);
                        if (bad) torn.fetch_add(1);
                        if ((s >> 1) < last) regress.fetch_add(1);
                        last = s >> 1;
                        reads.fetch_add(1);
                    }
                    if (finished) break;
                }
            });
        }
    }
    producer.join();
    for (auto &t : consumers) t.join();
    for (auto &t : readers) t.join();
    uint64_t last_state = 0;
    for (int i = 0; i < NC; i++) last_state += (ctrl->cons[i].state.load() >> 1) == V;
    printf("TSAN_PROTOCOL versions=%llu installs=%llu reads=%llu torn=%llu regress=%llu final_ok=%d\n",
           (unsigned long long)V, (unsigned long long)installs.load(), (unsigned long long)reads.load(),
           (unsigned long long)torn.load(), (unsigned long long)regress.load(), (int)(last_state == (uint64_t)NC));
    delete ctrl;
    return (torn.load() || regress.load() || last_state != (uint64_t)NC) ? 1 : 0;
}
