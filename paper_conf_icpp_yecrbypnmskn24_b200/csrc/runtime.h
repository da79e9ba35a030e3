// runtime.h -- host-side engine state of libviper.so (internal).
//
// Control plane: a Ctrl block in pinned, device-mapped
// host memory (in-process channel) or in a POSIX shared-memory segment
// registered with CUDA (cross-process channel) holds
//   pub_state  = (version << 1) | snapshot_slot   -- what the producer published
//   per consumer: state = (version << 1) | slot    -- what it serves (flipped by
//                 the install kernel from the device), pin (snapshot version it
//                 is reading), ref[2] (readers per slot), done_version/done_seq.
// All host-side accesses are seq_cst std::atomic; the device writes state,
// pin and status with system-scope fenced stores (kernels.cu finalize_install).
#pragma once
#include <atomic>
#include <condition_variable>
#include <cstdint>
#include <map>
#include <mutex>
#include <string>
#include <thread>
#include <unordered_map>
#include <vector>

#include "../../include/viper.h"
#include "vp_internal.h"

namespace vp {

constexpr int kMaxConsumers = 16;
constexpr int kMaxPieces = 256;     // DRAM tier: D2H / H2D pipeline granularity (whole chunks)
constexpr int kMaxProducers = 8;   // data-parallel producers (multi-producer fan-in)
constexpr uint64_t kCtrlMagic = 0x5649504552435431ull;  // "VIPERCT1"

// Fan-outs that exist only across processes (one producer, GPU tier).
inline bool xproc_only_fanout(int32_t f) {
    return f == VIPER_FANOUT_NVLS || f == VIPER_FANOUT_PUSH || f == VIPER_FANOUT_CE || f == VIPER_FANOUT_NCCL;
}
// Consumers receive the snapshot into a device staging buffer by a copy ahead of
// the install (DRAM tier: H2D; copy engine: peer copy; NCCL: broadcast).
inline bool copy_staged(int32_t tier, int32_t f) {
    return tier == VIPER_TIER_DRAM || f == VIPER_FANOUT_CE || f == VIPER_FANOUT_NCCL;
}
// Consumers install from a local staging buffer the producer writes into
// (push: peer stores; NVLS: multicast stores).
inline bool staged_fanout(int32_t f) { return f == VIPER_FANOUT_NVLS || f == VIPER_FANOUT_PUSH; }

// A public call runs on the model's GPU and leaves the caller's current device
// as it found it (a process driving several GPUs, e.g. torch's current device,
// must not see it change under a publish / release / unregister).
struct DeviceGuard {
    int prev = -1;
    cudaError_t err = cudaSuccess;
    explicit DeviceGuard(int dev) {
        if (cudaGetDevice(&prev) != cudaSuccess) prev = -1;
        if (prev != dev) err = cudaSetDevice(dev);
    }
    ~DeviceGuard() {
        int cur = -1;
        if (prev >= 0 && cudaGetDevice(&cur) == cudaSuccess && cur != prev) cudaSetDevice(prev);
    }
    DeviceGuard(const DeviceGuard &) = delete;
    DeviceGuard &operator=(const DeviceGuard &) = delete;
};

struct alignas(64) ConsRec {
    std::atomic<uint64_t> state;         // (v << 1) | slot, 0 = nothing installed (device-written)
    std::atomic<uint64_t> pin;           // snapshot version being read, 0 = none (device-cleared)
    std::atomic<int32_t> status;         // result of the last install kernel (device-written)
    std::atomic<int32_t> active;
    std::atomic<int64_t> ref[2];         // readers pinning each slot
    std::atomic<uint64_t> done_version;  // last version processed (installed or failed)
    std::atomic<uint32_t> done_seq;      // futex word, bumped after each install attempt
    std::atomic<int32_t> waiters;        // threads sleeping on done_seq
    std::atomic<int32_t> last_status;
    std::atomic<int32_t> pid;            // consumer process (failure detection), 0 = in-process
    std::atomic<uint64_t> p1_done;       // scatter-allgather: phase-1 version finished
    std::atomic<uint64_t> p2_done;       // scatter-allgather: phase-2 version finished
    std::atomic<int32_t> abort;          // host -> install kernel: stop waiting for item seals (the
                                         // update thread gave up: producer gone, unregister, deadline)
};

struct alignas(64) Ctrl {
    uint64_t magic;
    std::atomic<uint64_t> pub_state;     // (v << 1) | snapshot slot, 0 = none
    std::atomic<uint32_t> pub_seq;       // futex word, bumped on each publish
    std::atomic<uint32_t> closing;
    std::atomic<int64_t> pub_time_ns;    // CLOCK_MONOTONIC of the last publish notification
    std::atomic<int32_t> ncons;
    ConsRec cons[kMaxConsumers];
    // DRAM tier: piece i of snapshot slot b is in host staging once
    // dram_flag[b][i] >= v (written by the producer's copy stream with
    // cuStreamWriteValue64; consumers' copy streams wait with cuStreamWaitValue64)
    alignas(64) std::atomic<uint64_t> dram_flag[2][kMaxPieces];
    // multi-producer: producer j's (v << 1) | slot; consumers install v once
    // every producer published it
    alignas(64) std::atomic<uint64_t> pub_m[kMaxProducers];
    std::atomic<int32_t> nprod;
    std::atomic<int32_t> early_notify;   // producer names v before its pack completed
    std::atomic<int32_t> prod_pid;       // cross-process producer (liveness), 0 = in-process
    std::atomic<int64_t> pub_entry_ns;   // CLOCK_MONOTONIC at the entry of the last viper_publish
};

// Pointer-free work item (the device lists add each endpoint's tensor address).
struct BaseItem {
    uint64_t tensor_off, packed_off;
    uint32_t nbytes, chunk, tensor;
};

struct Manifest {
    int32_t n = 0;
    std::vector<uint64_t> nbytes, offsets;
    uint64_t s_packed = 0, chunk_bytes = 0;
    uint32_t align = 0;
    std::vector<BaseItem> items;
    std::vector<uint32_t> chunk_first;  // [nchunks + 1]
    uint64_t item_max = 0;
    uint32_t nchunks = 0;
    uint32_t *d_chunk_first = nullptr;
    // DRAM-tier pieces: [byte_lo, byte_hi) and [item_lo, item_hi), whole chunks
    std::vector<uint64_t> piece_lo, piece_hi;
    std::vector<uint32_t> piece_ilo, piece_ihi;
};

struct Channel;
struct Flusher;

// One kernel launched through a one-node CUDA graph whose node parameters are
// updated per launch: measured cheaper on the host than a direct launch on
// this VM (profiles/r01/launchcal.log: 2.3 vs 4.5 us).  The graph is rebuilt
// when the kernel function changes.
struct OneNodeGraph {
    cudaGraph_t g = nullptr;
    cudaGraphExec_t x = nullptr;
    cudaGraphNode_t n = nullptr;
    const void *func = nullptr;
    cudaError_t launch(const cudaKernelNodeParams &kp, cudaStream_t st);
    void destroy();
};

// Where a consumer reads snapshot slot b from: the producer's device buffers
// (same process, or CUDA-IPC peer-mapped over NVLink), the host staging of the
// DRAM tier (pinned; a shared-memory segment across processes), and -- in
// process only -- the event that marks slot b complete.
struct SnapSource {
    const uint8_t *snap[2] = {nullptr, nullptr};
    const ISeal *iseal[2] = {nullptr, nullptr};
    const uint8_t *h_stage[2] = {nullptr, nullptr};
    const ISeal *h_iseal[2] = {nullptr, nullptr};
    cudaEvent_t ev_ready[2] = {nullptr, nullptr};
};

struct ViewTicket {
    int32_t slot;
};

}  // namespace vp

struct viper_model {
    std::string name;
    int32_t role = 0, device = 0;
    viper_config cfg{};
    vp::Manifest man;
    vp::Geometry geo{};
    uint32_t *d_flags = nullptr;       // 64 B: [0, 8) grid completion (blocks | error bits), [8, 12) install / fused
                                       // work counter (kernels.cu WorkQueue)
    vp::Channel *chan = nullptr;       // in-process channel (registry entry)
    vp::Ctrl *ctrl = nullptr;          // host view of the control block
    vp::Ctrl *ctrl_dev = nullptr;      // device view (mapped)
    bool xproc = false;
    std::atomic<bool> closed{false};

    // ---------------- producer
    std::vector<void *> src_ptrs;
    vp::Item *d_items = nullptr;                     // producer list / consumer slot-0 list
    uint8_t *d_snap[2] = {nullptr, nullptr};
    vp::ISeal *d_iseal[2] = {nullptr, nullptr};      // item seals + ready flags per snapshot slot
    vp::Seal *d_seal[2] = {nullptr, nullptr};        // chunk seals per snapshot slot
    cudaEvent_t ev_sealed[2] = {nullptr, nullptr};   // chunk seals of slot b reduced
    void *snap_alloc = nullptr;
    cudaEvent_t ev_ready[2] = {nullptr, nullptr};   // snapshot slot b complete
    cudaEvent_t ev_packed = nullptr;
    cudaEvent_t ev_notify = nullptr;   // producer, early notification: the stream reached the pack
    cudaEvent_t ev_t[2] = {nullptr, nullptr};        // VIPER_FLAG_TIMING: around the kernel
    bool timing_pending = false;
    bool last_fused = false;                         // last publish used publish_fused_kernel
    vp::OneNodeGraph g_fused, g_pack, g_seal;        // per-publish launches through one-node graphs
    vp::OneNodeGraph g_inst;                         // consumer: installs not PDL-chained (install_mu held)
    cudaStream_t side = nullptr;                     // DRAM-tier D2H stream
    uint8_t *h_stage[2] = {nullptr, nullptr};        // DRAM tier (pinned)
    vp::ISeal *h_iseal[2] = {nullptr, nullptr};
    void *h_stage_alloc = nullptr;
    uint64_t snap_version[2] = {0, 0};
    uint64_t last_version = 0;
    int cur_snap = 1;

    // ---------------- consumer
    int32_t cidx = -1;
    bool prod_same_gpu = false;  // consumer (cross-process): the producer runs on this GPU too
    vp::ConsRec *rec = nullptr, *rec_dev = nullptr;
    std::vector<void *> slot_ptrs[2];
    vp::Item *d_slot_items[2] = {nullptr, nullptr};  // consumer work lists per slot
    void *slot1_alloc = nullptr;
    uint8_t *d_stage = nullptr;                      // DRAM tier device staging
    vp::ISeal *d_stage_iseal = nullptr;
    void *stage_alloc = nullptr;
    cudaStream_t ustream = nullptr;
    std::thread upd;
    std::atomic<bool> stop{false};
    std::mutex install_mu;
    uint64_t attempted = 0;
    std::atomic<bool> fault_next{false};
    std::mutex cb_mu;
    void (*cb)(uint64_t, viper_status, void *) = nullptr;
    void *cb_user = nullptr;
    std::mutex views_mu;
    std::unordered_map<uint64_t, vp::ViewTicket> views;
    uint64_t next_ticket = 1;

    // ---------------- cross-process (xproc.cpp)
    vp::SnapSource xsrc;                             // consumer: peer-mapped producer buffers
    void *shm_base = nullptr;                        // mapped control segment (+ DRAM staging)
    size_t shm_bytes = 0;
    std::string shm_name;
    bool shm_owner = false;
    bool shm_registered = false;
    void *peer_snap_base = nullptr;                  // cudaIpcOpenMemHandle result
    int32_t nconsumers_x = 0;                        // xproc: consumers in the channel
    void *sa_alloc = nullptr;                        // scatter-allgather: my staging [2][S] + seals [2][n]
    void *sa_peer_base[vp::kMaxConsumers] = {};          // peers' staging (IPC-opened)
    void *d_sa_tab = nullptr;                        // device tables: src[2][N], isrc[2][N], pin[N]
    uint64_t sa_S = 0, sa_IS = 0;
    int32_t rank = 0, world = 1;
    bool early_notify = false;                       // producer: consumers pipeline behind the pack
    vp::Flusher *flusher = nullptr;                  // producer: background flush (flush.cpp)
    int32_t nprod = 1, pidx = 0;                     // data-parallel producers / this producer's index
    uint32_t pack_nitems = 0;                        // items this producer packs (its chunk share)
    void *peer_snap_m[vp::kMaxProducers] = {};        // consumer: every producer's snapshot (IPC)
    void *d_mp_tab = nullptr;                        // consumer: snap[2][M], iseal[2][M]
    // push / NVLS (staged fan-outs): consumers install from their own staging
    vp::SnapSource stage_src;                        // consumer: staging slot b + its item seals
    void *push_peer_base[vp::kMaxPush] = {};         // producer (push): consumers' staging (IPC-opened)
    uint8_t *push_dst[2][vp::kMaxPush] = {};         // producer (push): consumer k's staging slot b
    vp::ISeal *push_iseal[2][vp::kMaxPush] = {};
    int32_t npush = 0;
    // NVLS (nvls.cpp): one multicast object; driver handles kept as integers
    uint64_t nvls_mc = 0, nvls_phys = 0, nvls_va = 0, nvls_uc = 0;
    size_t nvls_bytes = 0;
    int nvls_fd = -1, nvls_listen = -1;
    bool nvls_have_mc = false, nvls_have_phys = false, nvls_bound = false, nvls_uc_mapped = false,
         nvls_mc_mapped = false;
    void *nccl_comm = nullptr;                       // VIPER_FANOUT_NCCL: the communicator (ncclComm_t)
    int32_t nccl_root = 0;                           // the producer's rank in it
    uint8_t *nvls_mc_snap[2] = {nullptr, nullptr};   // producer: multicast VA of snapshot slot b
    vp::ISeal *nvls_mc_iseal[2] = {nullptr, nullptr};

    // ---------------- stats
    std::mutex stats_mu;
    viper_stats stats{};
};

namespace vp {

// Locking (in-process channel):
//   mu   guards `consumers`; a SYNC publish holds it for its whole duration, so
//        a consumer cannot be torn down while the producer installs into it.
//   pmu  leaf lock for `producer`; update threads read it while holding their
//        own install_mu, so a producer teardown that nulls it and then cycles
//        every consumer's install_mu knows no install still uses its buffers.
struct Channel {
    std::string name;
    Ctrl *ctrl = nullptr, *ctrl_dev = nullptr;
    std::mutex mu, pmu;
    viper_model *producer = nullptr;
    std::vector<viper_model *> consumers;
    int refs = 0;
    std::vector<uint64_t> nbytes;  // manifest check
    int32_t tier = -1;             // every endpoint of an in-process channel uses one tier
};

struct PreparedInstall {
    viper_model *c = nullptr;
    InstallArgs a{};
    double waited_us = 0;
};

// runtime.cpp helpers used by other translation units
viper_status set_error(viper_status st, const char *fmt, ...);
int64_t now_ns();
void futex_wake_all(std::atomic<uint32_t> *w);
void futex_wait(std::atomic<uint32_t> *w, uint32_t expected, int64_t timeout_us);
viper_status build_manifest(Manifest &m, const viper_tensor *t, int32_t n, uint64_t chunk_bytes, uint32_t align,
                            int device, uint64_t force_item_max = 0);
viper_status upload_items(const Manifest &m, const std::vector<void *> &ptrs, Item **d_out, uint32_t share_n,
                          uint32_t share_me, uint32_t *count);
std::atomic<uint64_t> &pub_word(viper_model *p);
viper_status prepare_install(viper_model *c, const SnapSource &src, uint64_t v, int b, PreparedInstall *pi);
viper_status launch_prepared(PreparedInstall &pi, const SnapSource &src, int b, cudaStream_t st, bool wait_ready,
                             bool pdl);
viper_status enqueue_install(viper_model *c, const SnapSource &src, uint64_t v, int b, cudaStream_t st,
                             bool wait_ready);
viper_status finish_install(viper_model *c, uint64_t v, double t_install_us);
void update_loop(viper_model *c);
viper_status alloc_producer(viper_model *m, const viper_tensor *tensors);
viper_status alloc_consumer(viper_model *m, const viper_tensor *tensors);
SnapSource source_of(const viper_model *p);

// stream memory operations (driver entry points, resolved at first use)
viper_status stream_wait_geq(cudaStream_t st, const void *dev_addr, uint64_t v);
viper_status stream_write(cudaStream_t st, void *dev_addr, uint64_t v);

// flush.cpp
viper_status flush_start(viper_model *m, const char *dir);
viper_status flush_enqueue(viper_model *p, uint64_t v, int b);
void flush_stop(viper_model *m);
void flush_stats(viper_model *m, uint64_t *flushed, uint64_t *skipped, uint64_t *last);

// xproc.cpp
viper_status xproc_register(viper_model *m, const viper_tensor *tensors, const viper_bootstrap *bs);
viper_status xproc_install(viper_model *c, uint64_t v, int b);   // consumer update thread
viper_status xproc_notify(viper_model *p, uint64_t v, int b, bool sync, bool already = false);  // producer
viper_status xproc_notify_early(viper_model *p, uint64_t v, int b, cudaStream_t st);           // producer
void xproc_abort(const viper_bootstrap *bs, viper_status st);  // failed before the bootstrap
void xproc_free(viper_model *m);

// nvls.cpp (VIPER_FANOUT_NVLS); every failure is VIPER_E_UNSUPPORTED / _PEER
viper_status nvls_probe(int device);
viper_status nvls_create(viper_model *m, int nranks, size_t bytes, char *sock_name, size_t cap);  // producer
viper_status nvls_serve(viper_model *m, int nconsumers);                                          // producer
viper_status nvls_join(viper_model *m, const char *sock_name, size_t bytes);                      // consumer
viper_status nvls_bind(viper_model *m, bool map_mc);                                              // every rank
void nvls_free(viper_model *m);

// nccl_fanout.cpp (VIPER_FANOUT_NCCL, the NCCL-broadcast baseline as an engine transport)
viper_status nccl_probe(void *unique_id_out);  // unique_id_out: 128 B (producer) or NULL
viper_status nccl_init(viper_model *m, const void *unique_id, int world, int rank);
viper_status nccl_broadcast_version(viper_model *m, void *snap, void *iseal, int root, cudaStream_t st);
void nccl_free(viper_model *m);

}  // namespace vp
