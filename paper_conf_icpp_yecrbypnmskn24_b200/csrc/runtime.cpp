// runtime.cpp -- the Model Weights Handler (PAPER.md s4.4 P:1671-1800, Fig. 7)
// rebuilt for one process per B200: registration / manifest,
// publish = snapshot + notify, the consumer's update thread that
// installs into the alternative copy and swaps atomically (P:1214-1227,
// P:1424-1428), and the reader-side acquire/release.
//
// Every byte moves in the kernels of kernels.cu; this file only decides what
// to launch, when, and on which stream.  There is no CPU data path.
#include "runtime.h"
#include "protocol.h"

#include <cuda.h>  // types of the driver entry points (no libcuda link)
#include <nvtx3/nvToolsExt.h>  // header-only; ranges cost nothing unless a tool attaches
#include <errno.h>
#include <linux/futex.h>
#include <signal.h>
#include <sched.h>
#include <sys/syscall.h>
#include <time.h>
#include <unistd.h>

#include <algorithm>
#include <climits>
#include <cstdarg>
#include <cstdio>
#include <cstring>
#include <new>

namespace vp {

extern int64_t g_trace[16];
static thread_local std::string t_err;

viper_status set_error(viper_status st, const char *fmt, ...) {
    char buf[512];
    va_list ap;
    va_start(ap, fmt);
    vsnprintf(buf, sizeof buf, fmt, ap);
    va_end(ap);
    t_err = buf;
    return st;
}

#define CUDA_TRY(x)                                                                                  \
    do {                                                                                             \
        cudaError_t e_ = (x);                                                                        \
        if (e_ != cudaSuccess)                                                                       \
            return set_error(VIPER_E_CUDA, "%s failed: %s (%s:%d)", #x, cudaGetErrorString(e_), __FILE__, \
                             __LINE__);                                                              \
    } while (0)

int64_t now_ns() {
    timespec ts;
    clock_gettime(CLOCK_MONOTONIC, &ts);
    return (int64_t)ts.tv_sec * 1000000000ll + ts.tv_nsec;
}

// Shared (non-private) futexes: they also work on words in a shm segment.
void futex_wake_all(std::atomic<uint32_t> *w) {
    syscall(SYS_futex, reinterpret_cast<uint32_t *>(w), FUTEX_WAKE, INT_MAX, nullptr, nullptr, 0);
}

void futex_wait(std::atomic<uint32_t> *w, uint32_t expected, int64_t timeout_us) {
    timespec ts, *tp = nullptr;
    if (timeout_us >= 0) {
        ts.tv_sec = timeout_us / 1000000;
        ts.tv_nsec = (timeout_us % 1000000) * 1000;
        tp = &ts;
    }
    syscall(SYS_futex, reinterpret_cast<uint32_t *>(w), FUTEX_WAIT, expected, tp, nullptr, 0);
}

static inline void cpu_relax() { __builtin_ia32_pause(); }

// NVTX range per stage (publish / install), visible in nsys and usable as an
// ncu --nvtx filter.
struct NvtxRange {
    explicit NvtxRange(const char *name) { nvtxRangePushA(name); }
    ~NvtxRange() { nvtxRangePop(); }
};

// Optional per-update JSON lines (SURVEY s5 metrics): VIPER_LOG=<path>.
static FILE *g_log = nullptr;
static std::mutex g_log_mu;
static std::once_flag g_log_once;

static void log_update(const char *role, const viper_model *m, uint64_t v, viper_status st, double host_us,
                       double extra_us, const char *extra_name) {
    std::call_once(g_log_once, [] {
        if (const char *p = getenv("VIPER_LOG")) g_log = fopen(p, "a");
    });
    if (!g_log) return;
    std::lock_guard<std::mutex> lk(g_log_mu);
    fprintf(g_log,
            "{\"t_ns\":%lld,\"role\":\"%s\",\"model\":\"%s\",\"version\":%llu,\"status\":%d,"
            "\"bytes\":%llu,\"tier\":%d,\"fanout\":%d,\"mode\":%d,\"host_us\":%.3f,\"%s\":%.3f}\n",
            (long long)now_ns(), role, m->name.c_str(), (unsigned long long)v, st,
            (unsigned long long)m->man.s_packed, m->cfg.tier, m->cfg.fanout, m->cfg.mode, host_us, extra_name, extra_us);
    fflush(g_log);
}

typedef CUresult (*PFN_wait64)(CUstream, CUdeviceptr, cuuint64_t, unsigned int);
typedef CUresult (*PFN_write64)(CUstream, CUdeviceptr, cuuint64_t, unsigned int);
static PFN_wait64 g_wait64 = nullptr;
static PFN_write64 g_write64 = nullptr;
static std::once_flag g_memops_once;

static void resolve_memops() {
    cudaDriverEntryPointQueryResult q;
    if (cudaGetDriverEntryPoint("cuStreamWaitValue64", (void **)&g_wait64, cudaEnableDefault, &q) != cudaSuccess ||
        q != cudaDriverEntryPointSuccess)
        g_wait64 = nullptr;
    if (cudaGetDriverEntryPoint("cuStreamWriteValue64", (void **)&g_write64, cudaEnableDefault, &q) != cudaSuccess ||
        q != cudaDriverEntryPointSuccess)
        g_write64 = nullptr;
}

viper_status stream_wait_geq(cudaStream_t st, const void *dev_addr, uint64_t v) {
    std::call_once(g_memops_once, resolve_memops);
    if (!g_wait64) return set_error(VIPER_E_UNSUPPORTED, "cuStreamWaitValue64 unavailable");
    const CUresult r = g_wait64((CUstream)st, (CUdeviceptr)dev_addr, v, CU_STREAM_WAIT_VALUE_GEQ);
    return r == CUDA_SUCCESS ? VIPER_OK : set_error(VIPER_E_CUDA, "cuStreamWaitValue64 failed (%d)", (int)r);
}

viper_status stream_write(cudaStream_t st, void *dev_addr, uint64_t v) {
    std::call_once(g_memops_once, resolve_memops);
    if (!g_write64) return set_error(VIPER_E_UNSUPPORTED, "cuStreamWriteValue64 unavailable");
    const CUresult r = g_write64((CUstream)st, (CUdeviceptr)dev_addr, v, CU_STREAM_WRITE_VALUE_DEFAULT);
    return r == CUDA_SUCCESS ? VIPER_OK : set_error(VIPER_E_CUDA, "cuStreamWriteValue64 failed (%d)", (int)r);
}

// ------------------------------------------------------------------ manifest
// LAY (R16) + the warp work list.  Items never cross a seal chunk
// and are at most item_max bytes; splits fall on 16-B multiples of the tensor.
viper_status build_manifest(Manifest &m, const viper_tensor *t, int32_t n, uint64_t chunk_bytes,
                                   uint32_t align, int device, uint64_t force_item_max) {
    m.n = n;
    m.nbytes.resize(n);
    m.offsets.resize(n);
    m.chunk_bytes = chunk_bytes;
    m.align = align;
    uint64_t off = 0;
    for (int32_t i = 0; i < n; i++) {
        m.nbytes[i] = t[i].nbytes;
        m.offsets[i] = off;
        off = (off + t[i].nbytes + align - 1) / align * align;
    }
    m.s_packed = off;
    m.nchunks = (uint32_t)((m.s_packed + chunk_bytes - 1) / chunk_bytes);
    int sms = 148;
    cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, device);
    // item size: enough items for ~4 per resident warp, 2 KiB .. 8 KiB, 512-B
    // multiple (VIPER_ITEM_MAX / VIPER_ITEM_MIN override, for sweeps).  Small
    // items keep the fused kernel's read-back L2-resident and balance the tail.
    // ~4 items per resident warp (16 warps / SM: kernels.cu geometry)
    uint64_t target = m.s_packed / ((uint64_t)sms * 16 * 4) + 1;
    uint64_t cap = 8192;  // sweep: profiles/r01/item_sweep.log (best for the fused kernel)
    if (const char *e = getenv("VIPER_ITEM_MAX")) cap = std::max<uint64_t>(512, strtoull(e, nullptr, 10) / 512 * 512);
    uint64_t item_max = std::min<uint64_t>(std::max<uint64_t>((target + 511) / 512 * 512, 2048), cap);
    if (const char *e = getenv("VIPER_ITEM_MIN")) item_max = std::max<uint64_t>(item_max, strtoull(e, nullptr, 10) / 512 * 512);
    if (force_item_max) item_max = force_item_max;  // restore: the partition the seals were made with
    if (item_max > chunk_bytes) item_max = chunk_bytes;
    m.item_max = item_max;
    m.items.clear();
    std::vector<uint32_t> per_chunk(m.nchunks, 0);
    for (int32_t i = 0; i < n; i++) {
        uint64_t done = 0;
        while (done < m.nbytes[i]) {
            const uint64_t p = m.offsets[i] + done;
            const uint64_t chunk = p / chunk_bytes;
            const uint64_t chunk_end = (chunk + 1) * chunk_bytes;
            const uint64_t len = std::min<uint64_t>({item_max, m.nbytes[i] - done, chunk_end - p});
            m.items.push_back(BaseItem{done, p, (uint32_t)len, (uint32_t)chunk, (uint32_t)i});
            per_chunk[chunk]++;
            done += len;
        }
    }
    m.chunk_first.assign(m.nchunks + 1, 0);
    for (uint32_t c = 0; c < m.nchunks; c++) {
        if (per_chunk[c] == 0) return set_error(VIPER_E_INVAL, "chunk %u has no data (align > chunk?)", c);
        m.chunk_first[c + 1] = m.chunk_first[c] + per_chunk[c];
    }
    if (m.items.size() >= (size_t)UINT32_MAX) return set_error(VIPER_E_INVAL, "too many work items");
    // DRAM-tier pipeline pieces: whole chunks, about S/64 clamped to
    // [8 MiB, 64 MiB] (VIPER_DRAM_PIECE overrides, for sweeps), at most kMaxPieces
    {
        uint64_t want = std::min<uint64_t>(std::max<uint64_t>(m.s_packed / 64, 8ull << 20), 64ull << 20);
        if (const char *e = getenv("VIPER_DRAM_PIECE")) want = std::max<uint64_t>(strtoull(e, nullptr, 10), 1);
        want = std::max<uint64_t>(want, (m.s_packed + kMaxPieces - 1) / kMaxPieces);
        const uint64_t per = std::max<uint64_t>(1, (want + chunk_bytes - 1) / chunk_bytes);  // chunks per piece
        m.piece_lo.clear(); m.piece_hi.clear(); m.piece_ilo.clear(); m.piece_ihi.clear();
        for (uint64_t c = 0; c < m.nchunks; c += per) {
            const uint64_t ce = std::min<uint64_t>(m.nchunks, c + per);
            m.piece_lo.push_back(c * chunk_bytes);
            m.piece_hi.push_back(std::min<uint64_t>(ce * chunk_bytes, m.s_packed));
            m.piece_ilo.push_back(m.chunk_first[c]);
            m.piece_ihi.push_back(m.chunk_first[ce]);
        }
        if (m.piece_lo.size() > (size_t)kMaxPieces) return set_error(VIPER_E_INVAL, "too many DRAM pieces");
    }
    CUDA_TRY(cudaMalloc(&m.d_chunk_first, m.chunk_first.size() * sizeof(uint32_t)));
    CUDA_TRY(cudaMemcpy(m.d_chunk_first, m.chunk_first.data(), m.chunk_first.size() * sizeof(uint32_t),
                        cudaMemcpyHostToDevice));
    return VIPER_OK;
}

// Device work list of one endpoint: the base items with that endpoint's tensor
// addresses folded in.
viper_status upload_items(const Manifest &m, const std::vector<void *> &ptrs, Item **d_out, uint32_t share_n,
                          uint32_t share_me, uint32_t *count) {
    *d_out = nullptr;
    std::vector<Item> v;
    v.reserve(m.items.size());
    for (size_t k = 0; k < m.items.size(); k++) {
        const BaseItem &b = m.items[k];
        if (share_n > 1 && b.chunk % share_n != share_me) continue;  // another producer's chunk
        v.push_back(Item{(uint64_t)(uintptr_t)ptrs[b.tensor] + b.tensor_off, b.packed_off, b.nbytes, b.chunk, b.tensor,
                         (uint32_t)k});
    }
    if (count) *count = (uint32_t)v.size();
    if (v.empty()) return VIPER_OK;
    CUDA_TRY(cudaMalloc((void **)d_out, v.size() * sizeof(Item)));
    CUDA_TRY(cudaMemcpy(*d_out, v.data(), v.size() * sizeof(Item), cudaMemcpyHostToDevice));
    return VIPER_OK;
}

// ------------------------------------------------------- in-process registry
static std::mutex g_reg_mu;
static std::map<std::string, Channel *> g_reg;

static viper_status channel_open(const std::string &name, const Manifest &man, int32_t tier, Channel **out) {
    std::lock_guard<std::mutex> lk(g_reg_mu);
    auto it = g_reg.find(name);
    Channel *ch;
    if (it == g_reg.end()) {
        ch = new Channel();
        ch->name = name;
        ch->nbytes = man.nbytes;
        void *p = nullptr;
        CUDA_TRY(cudaHostAlloc(&p, sizeof(Ctrl), cudaHostAllocMapped | cudaHostAllocPortable));
        memset(p, 0, sizeof(Ctrl));
        ch->ctrl = new (p) Ctrl();
        ch->ctrl->magic = kCtrlMagic;
        void *d = nullptr;
        CUDA_TRY(cudaHostGetDevicePointer(&d, p, 0));
        ch->ctrl_dev = (Ctrl *)d;
        ch->tier = tier;
        g_reg[name] = ch;
    } else {
        ch = it->second;
        if (ch->nbytes != man.nbytes)
            return set_error(VIPER_E_INVAL, "model '%s': tensor list differs from the other endpoints", name.c_str());
        // a DRAM-tier consumer reads the producer's host staging, which only a
        // DRAM-tier producer fills
        if (ch->tier != tier)
            return set_error(VIPER_E_INVAL, "model '%s': tier %d, the other endpoints use tier %d", name.c_str(), tier,
                             ch->tier);
    }
    ch->refs++;
    *out = ch;
    return VIPER_OK;
}

static viper_model *channel_producer(Channel *ch) {
    if (!ch) return nullptr;
    std::lock_guard<std::mutex> lk(ch->pmu);
    return ch->producer;
}

static void channel_close(Channel *ch) {
    std::lock_guard<std::mutex> lk(g_reg_mu);
    if (--ch->refs > 0) return;
    g_reg.erase(ch->name);
    cudaFreeHost(ch->ctrl);
    delete ch;
}

cudaError_t OneNodeGraph::launch(const cudaKernelNodeParams &kp, cudaStream_t st) {
    cudaError_t e;
    if (x && func != kp.func) destroy();
    if (!x) {
        if ((e = cudaGraphCreate(&g, 0)) == cudaSuccess && (e = cudaGraphAddKernelNode(&n, g, nullptr, 0, &kp)) == cudaSuccess)
            e = cudaGraphInstantiate(&x, g, 0);
        if (e != cudaSuccess) {
            destroy();  // nothing half-built is kept; the next launch starts over
            return e;
        }
        func = kp.func;
    } else if ((e = cudaGraphExecKernelNodeSetParams(x, n, &kp)) != cudaSuccess) {
        return e;
    }
    return cudaGraphLaunch(x, st);
}

void OneNodeGraph::destroy() {
    if (x) cudaGraphExecDestroy(x);
    if (g) cudaGraphDestroy(g);
    x = nullptr;
    g = nullptr;
    n = nullptr;
    func = nullptr;
}

// The snapshot fits in L2 (with room to spare): then the TMA kernels load
// data they read only once with an L2 evict-first hint, so the snapshot the
// next reader takes stays in L2 (profiles/r01/tma_l2_hint_ab.log: ResNet-50
// TMA install 40-42 -> 34 us; models larger than L2 lose a little, so off).
static bool fits_l2(int device, uint64_t bytes) {
    static std::atomic<int64_t> l2[64];
    const int d = device >= 0 && device < 64 ? device : 0;
    int64_t v = l2[d].load(std::memory_order_relaxed);
    if (v == 0) {
        int b = 0;
        if (cudaDeviceGetAttribute(&b, cudaDevAttrL2CacheSize, device) != cudaSuccess || b <= 0) b = 126 << 20;
        l2[d].store(v = b, std::memory_order_relaxed);
    }
    return bytes <= (uint64_t)v * 7 / 8;
}

static const bool g_no_graph = getenv("VIPER_NO_GRAPH") && atoi(getenv("VIPER_NO_GRAPH"));  // direct launches

// A LaunchSpec with one by-value argument struct, through a one-node graph
// (or directly with VIPER_NO_GRAPH=1).
template <typename Args>
static cudaError_t launch_spec(OneNodeGraph &og, const LaunchSpec &l, const Args &a, cudaStream_t st) {
    if (l.err != cudaSuccess) return l.err;
    void *args[] = {(void *)&a};
    if (g_no_graph) return cudaLaunchKernel(l.func, dim3(l.grid), dim3(l.block), args, l.smem, st);
    cudaKernelNodeParams kp{};
    kp.func = (void *)l.func;
    kp.gridDim = dim3(l.grid);
    kp.blockDim = dim3(l.block);
    kp.sharedMemBytes = (unsigned)l.smem;
    kp.kernelParams = args;
    return og.launch(kp, st);
}

// --------------------------------------------------------------- install path
void fire_callback(viper_model *c, uint64_t v, viper_status st) {
    void (*cb)(uint64_t, viper_status, void *);
    void *user;
    {
        std::lock_guard<std::mutex> lk(c->cb_mu);
        cb = c->cb;
        user = c->cb_user;
    }
    if (cb) cb(v, st, user);
}

// Pin the latest published snapshot (Dekker pair with the producer's
// pub_state store -> pin scan).  Returns false when
// nothing is published.
// Host half of an install of snapshot slot b (version v) of producer p into
// the inactive slot of consumer c: wait until no reader pins the target (a7)
// and build the kernel arguments.  Caller holds c->install_mu.
viper_status prepare_install(viper_model *c, const SnapSource &src, uint64_t v, int b, PreparedInstall *pi) {
    ConsRec *r = c->rec;
    const int target = install_target(r);
    const int64_t t0 = now_ns();
    if (!wait_readers_gone(r, target, 10ll * 1000000000ll))
        return set_error(VIPER_E_TIMEOUT, "readers kept slot %d pinned for 10 s", target);
    pi->c = c;
    pi->waited_us = (now_ns() - t0) / 1e3;
    InstallArgs &a = pi->a;
    a = InstallArgs{};
    // DRAM tier / copy-engine baseline: the install reads this GPU's staging,
    // filled by the copies launch_prepared enqueues ahead of the kernel
    const bool staged = copy_staged(c->cfg.tier, c->cfg.fanout);
    a.items = c->d_slot_items[target];
    a.nitems = (uint32_t)c->man.items.size();
    a.packed = staged ? c->d_stage : src.snap[b];
    a.iseal = staged ? c->d_stage_iseal : src.iseal[b];
    a.version = v;
    a.target = (uint32_t)target;
    a.fault_item = ~0u;
    if (c->fault_next.exchange(false) && a.nitems) a.fault_item = a.nitems / 2;
    a.flags = (unsigned long long *)c->d_flags;
    a.ctr = (unsigned int *)((uint8_t *)c->d_flags + 8);  // [8, 12): the install's work counter
    a.status_h = (volatile int32_t *)&c->rec_dev->status;
    a.pin_h = (volatile uint64_t *)&c->rec_dev->pin;
    a.state_h = (volatile uint64_t *)&c->rec_dev->state;
    a.abort_h = (const volatile int32_t *)&c->rec_dev->abort;
    return VIPER_OK;
}

// Stream half: [wait for the snapshot] [DRAM tier: H2D staging] install kernel.
// pdl: the kernel directly follows the pack on st and consumes its items as
// they are sealed (kernels.cu, item-granular pipeline).
viper_status launch_prepared(PreparedInstall &pi, const SnapSource &src, int b, cudaStream_t st,
                                    bool wait_ready, bool pdl) {
    viper_model *c = pi.c;
    if (c->cfg.tier == VIPER_TIER_DRAM) {
        // Host-to-Host channel: host staging -> this GPU's
        // staging, piece by piece as the producer's D2H lands (GPU-side waits
        // on the pieces' flags: the D2H and this H2D overlap)
        const Manifest &mm = c->man;
        static const bool dbg = getenv("VIPER_DEBUG") != nullptr;
        if (dbg) {
            cudaPointerAttributes pa{};
            cudaPointerGetAttributes(&pa, src.h_stage[b]);
            fprintf(stderr, "[viper] DRAM install: %zu pieces, staging type %d\n", mm.piece_lo.size(), (int)pa.type);
        }
        for (size_t i = 0; i < mm.piece_lo.size(); i++) {
            viper_status s = stream_wait_geq(st, &c->ctrl_dev->dram_flag[b][i], pi.a.version);
            if (dbg) fprintf(stderr, "[viper]  piece %zu: wait enqueued (%d)\n", i, s);
            if (s) return s;
            CUDA_TRY(cudaMemcpyAsync(c->d_stage + mm.piece_lo[i], src.h_stage[b] + mm.piece_lo[i],
                                     mm.piece_hi[i] - mm.piece_lo[i], cudaMemcpyHostToDevice, st));
        }
        // the item seals travel once, behind the last piece (the producer
        // raises the last flag after their D2H); only the install reads them
        CUDA_TRY(cudaMemcpyAsync(c->d_stage_iseal, src.h_iseal[b], sizeof(ISeal) * mm.items.size(),
                                 cudaMemcpyHostToDevice, st));
        if (dbg) fprintf(stderr, "[viper]  copies enqueued\n");
        pdl = false;
    } else if (c->cfg.fanout == VIPER_FANOUT_CE) {
        // copy-engine baseline: the sealed snapshot (notified only
        // once the pack completed) -> this GPU's staging over the peer
        // mapping, then the same local install + verify
        CUDA_TRY(cudaMemcpyAsync(c->d_stage, src.snap[b], c->man.s_packed, cudaMemcpyDefault, st));
        CUDA_TRY(cudaMemcpyAsync(c->d_stage_iseal, src.iseal[b], sizeof(ISeal) * c->man.items.size(),
                                 cudaMemcpyDefault, st));
        pdl = false;
    } else if (c->cfg.fanout == VIPER_FANOUT_NCCL) {
        // NCCL baseline: receive the producer's broadcasts of v into the staging
        viper_status s = nccl_broadcast_version(c, c->d_stage, c->d_stage_iseal, c->nccl_root, st);
        if (s) return s;
        pdl = false;
    } else if (wait_ready && src.ev_ready[b]) {
        CUDA_TRY(cudaStreamWaitEvent(st, src.ev_ready[b], 0));
    }
    c->rec->status.store(1);  // "in flight"
    const bool timing = c->cfg.flags & VIPER_FLAG_TIMING;
    // TMA bulk-copy install: direct pulls whose snapshot is complete before the
    // kernel starts (not PDL-chained, no early notification), forced by
    // VIPER_FLAG_TMA or auto up to 1 GiB like the pack
    const bool direct = pi.a.sa_n == 0 && pi.a.mp_n <= 1;
    pi.a.l2_once = fits_l2(c->device, c->man.s_packed) ? 1u : 0u;
    const bool complete = !(pdl && !timing) && !c->ctrl->early_notify.load();
    // A complete snapshot from one source: TMA bulk copies or register
    // streaming with prefetched descriptors + seals (install_direct).
    // VIPER_INSTALL_KERNEL=tma|direct|verify overrides the automatic choice (A/B).
    static const char *ik = getenv("VIPER_INSTALL_KERNEL");
    const bool tma_auto = ik ? strcmp(ik, "tma") == 0 : kInstallTmaDefault && c->man.s_packed <= (1ull << 30);
    const bool tma = direct && complete && !(c->cfg.flags & VIPER_FLAG_NO_TMA) &&
                     ((c->cfg.flags & VIPER_FLAG_TMA) || tma_auto);
    // install_direct for every one-source install, complete or pipelined (the
    // old install_verify_kernel stays for fan-outs among consumers and
    // data-parallel producers, and as the A/B: VIPER_INSTALL_KERNEL=verify)
    const bool use_direct = direct && !tma && !(ik && strcmp(ik, "verify") == 0);
    int launch_dev = c->device;
    cudaGetDevice(&launch_dev);  // a SYNC publish launches on the producer's GPU
    pi.a.sys_swap = launch_dev != c->device ? 1u : 0u;
    // A pipelined install whose producer packs on this same GPU (ranks sharing
    // a GPU with early notification forced, e.g. under MPS, where the two
    // grids run concurrently) gets at most half of the SMs: its warps wait for
    // items the pack has not sealed yet, and a grid holding every SM would
    // keep the pack from ever being scheduled.
    int max_sms = c->cfg.install_sms;
    Geometry geo = c->geo;
    if (!complete && c->prod_same_gpu) {
        int sms = 148;
        cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, c->device);
        max_sms = max_sms > 0 ? std::min(max_sms, std::max(1, sms / 2)) : std::max(1, sms / 2);
        geo = pick_geometry(pi.a.nitems, c->device, max_sms);
    }
    if (timing) CUDA_TRY(cudaEventRecord(c->ev_t[0], st));
    if (pdl && !timing && !tma)  // PDL: a plain stream launch
        CUDA_TRY(launch_install(pi.a, c->geo, st, true, use_direct, c->man.s_packed));
    else
        CUDA_TRY(launch_spec(c->g_inst, install_launch(pi.a, geo, tma, c->device, max_sms, use_direct,
                                                       c->man.s_packed, !complete),
                             pi.a, st));
    if (timing) {
        CUDA_TRY(cudaEventRecord(c->ev_t[1], st));
        c->timing_pending = true;
    }
    std::lock_guard<std::mutex> lk(c->stats_mu);
    c->stats.writer_wait_us = pi.waited_us;
    return VIPER_OK;
}

viper_status enqueue_install(viper_model *c, const SnapSource &src, uint64_t v, int b, cudaStream_t st,
                                    bool wait_ready) {
    PreparedInstall pi;
    viper_status s = prepare_install(c, src, v, b, &pi);
    if (s) return s;
    return launch_prepared(pi, src, b, st, wait_ready, false);
}

// In-process source: the producer's own buffers.
SnapSource source_of(const viper_model *p) {
    SnapSource s;
    for (int b = 0; b < 2; b++) {
        s.snap[b] = p->d_snap[b];
        s.iseal[b] = p->d_iseal[b];
        s.h_stage[b] = p->h_stage[b];
        s.h_iseal[b] = p->h_iseal[b];
        s.ev_ready[b] = p->ev_ready[b];
    }
    return s;
}

// After the install kernel of v completed on the host's view of the stream.
// v is reported done (the SYNC producer may return) BEFORE the bookkeeping:
// under VIPER_FLAG_TIMING the kernel-time event is synchronised only after
// that, with stats_mu held throughout, so a stats reader still sees v's
// numbers and the timing costs the update nothing.
viper_status finish_install(viper_model *c, uint64_t v, double t_install_us) {
    ConsRec *r = c->rec;
    viper_status st = r->status.load();
    if (st == 1) st = set_error(VIPER_E_CUDA, "install kernel did not report");
    {
        std::lock_guard<std::mutex> lk(c->stats_mu);
        r->pin.store(0);
        r->last_status.store(st);
        r->done_version.store(v);
        r->done_seq.fetch_add(1);
        if (r->waiters.load() > 0) futex_wake_all(&r->done_seq);
        float dev_ms = -1.f;
        if (c->timing_pending && cudaEventSynchronize(c->ev_t[1]) == cudaSuccess &&
            cudaEventElapsedTime(&dev_ms, c->ev_t[0], c->ev_t[1]) == cudaSuccess)
            c->timing_pending = false;
        if (dev_ms >= 0) c->stats.t_install_dev_us = dev_ms * 1e3;
        c->stats.last_status = st;
        c->stats.t_install_us = t_install_us;
        if (st == VIPER_OK) {
            c->stats.installs++;
            c->stats.version = v;
        } else {
            c->stats.failures++;
        }
    }
    log_update("consumer", c, v, st, t_install_us, c->stats.writer_wait_us, "writer_wait_us");
    return st;
}

// The producer of a cross-process channel still exists (its pid in Ctrl).
static bool producer_alive(const viper_model *c) {
    if (!c->xproc) return true;
    if (c->ctrl->closing.load()) return false;
    const int32_t pid = c->ctrl->prod_pid.load();
    return pid <= 0 || !(kill(pid, 0) == -1 && errno == ESRCH);
}

// Wait for the install enqueued on c->ustream, bounded: poll the
// stream instead of blocking in cudaStreamSynchronize, and give up when the
// consumer is unregistering, the producer process is gone or 60 s passed.  A
// DRAM-tier install may sit in cuStreamWaitValue64 on a piece flag that a dead
// producer never raises: giving up releases those flags from the host and
// tells the kernel (rec->abort) to stop waiting for seals, so the stream
// drains and the install reports VIPER_E_PEER / VIPER_E_TIMEOUT.
static viper_status wait_install_bounded(viper_model *c, uint64_t v, int b) {
    const int64_t t0 = now_ns();
    static const bool dbg_wait = getenv("VIPER_DEBUG") != nullptr;
    if (dbg_wait) fprintf(stderr, "[viper] waiting for the install of v%llu (slot %d)\n", (unsigned long long)v, b);
    for (uint32_t spins = 0;; spins++) {
        // the install kernel's last block reports in the mapped status word
        // before the grid retires: the cheap, early signal (the stream query
        // below covers errors and launches that never report)
        if (const int32_t s = c->rec->status.load(); s != 1) {
            // success: the last block stores the swap right after the status,
            // so wait for that word instead of for the grid to retire (a
            // stream synchronisation adds microseconds to every SYNC update;
            // later work on this stream is ordered behind the grid anyway)
            if (s == VIPER_OK) {
                const int64_t ts = now_ns();
                while ((c->rec->state.load() >> 1) != v && now_ns() - ts < 1000000000ll) cpu_relax();
                if ((c->rec->state.load() >> 1) == v) return VIPER_OK;
            }
            const cudaError_t e = cudaStreamSynchronize(c->ustream);
            return e == cudaSuccess ? VIPER_OK : set_error(VIPER_E_CUDA, "install: %s", cudaGetErrorString(e));
        }
        const int64_t dt = now_ns() - t0;
        if ((spins & 63) == 63) {
            const cudaError_t e = cudaStreamQuery(c->ustream);
            if (e == cudaSuccess) return VIPER_OK;
            if (e != cudaErrorNotReady) return set_error(VIPER_E_CUDA, "install: %s", cudaGetErrorString(e));
        }
        if ((spins & 255) == 255) {
            viper_status why = VIPER_OK;
            if (c->stop.load()) why = set_error(VIPER_E_STATE, "install of v%llu abandoned: unregistering",
                                                (unsigned long long)v);
            else if (!producer_alive(c)) why = set_error(VIPER_E_PEER, "producer gone during the install of v%llu",
                                                         (unsigned long long)v);
            else if (dt > 60ll * 1000000000ll) why = set_error(VIPER_E_TIMEOUT, "install of v%llu did not finish in 60 s",
                                                             (unsigned long long)v);
            if (why != VIPER_OK) {
                static const bool dbg = getenv("VIPER_DEBUG") != nullptr;
                if (dbg) fprintf(stderr, "[viper] install of v%llu abandoned: %s\n", (unsigned long long)v, viper_last_error());
                c->rec->abort.store(1);
                if (c->cfg.tier == VIPER_TIER_DRAM)  // release the copy stream's flag waits
                    for (size_t i = 0; i < c->man.piece_lo.size(); i++) {
                        uint64_t cur = c->ctrl->dram_flag[b][i].load();
                        while (cur < v && !c->ctrl->dram_flag[b][i].compare_exchange_weak(cur, v)) {
                        }
                    }
                const cudaError_t se = cudaStreamSynchronize(c->ustream);  // bounded now: the kernel stops waiting
                if (dbg) fprintf(stderr, "[viper] drained after abort: %s\n", cudaGetErrorString(se));
                c->rec->abort.store(0);
                // the data may still have arrived complete (its seals verified
                // every item and the kernel swapped): then v IS installed
                if (se == cudaSuccess && c->rec->status.load() == VIPER_OK && (c->rec->state.load() >> 1) == v)
                    return VIPER_OK;
                return why;
            }
        }
        if (dt < 200000) cpu_relax();
        else usleep(dt < 10000000 ? 20 : 200);
    }
}

// How long an idle update thread spins on the control block before it sleeps
// on the futex (VIPER_SPIN_US overrides): a futex wake-up costs tens of us of
// scheduling latency, a spin costs a host core while it lasts.
static const int64_t kIdleSpinNs = getenv("VIPER_SPIN_US") ? atoll(getenv("VIPER_SPIN_US")) * 1000 : 50000;

void update_loop(viper_model *c) {
    cudaSetDevice(c->device);
    Ctrl *ctrl = c->ctrl;
    ConsRec *r = c->rec;
    while (!c->stop.load()) {
        const uint32_t seq = ctrl->pub_seq.load();
        uint64_t ps = ctrl->pub_state.load();
        if (c->nprod > 1 && !all_published(ctrl, c->nprod, &ps)) ps = 0;
        bool work;
        {
            // SYNC producers install inline; the thread only catches a consumer
            // up that registered after the last publish.
            std::lock_guard<std::mutex> lk(c->install_mu);
            if (c->xproc) {  // cross-process: this thread installs every version it sees
                work = ps != 0 && (ps >> 1) > c->attempted;
            } else {
                viper_model *p = channel_producer(c->chan);
                const bool async = p && p->cfg.mode == VIPER_ASYNC;
                work = p && ps != 0 && (ps >> 1) > c->attempted && (async || c->attempted == 0);
            }
        }
        if (!work) {
            // short spin (notification latency), then sleep on the futex.  The
            // spin also watches the published word itself: an early-notified
            // version is named by a stream memop on the producer's GPU, which
            // may land after the host wake-up that roused this thread.
            const int64_t t0 = now_ns();
            const uint64_t ps0 = ctrl->pub_state.load();
            bool got = false;
            while (now_ns() - t0 < kIdleSpinNs) {
                if (ctrl->pub_seq.load() != seq || ctrl->pub_state.load() != ps0 || c->stop.load()) {
                    got = true;
                    break;
                }
                cpu_relax();
            }
            if (!got) futex_wait(&ctrl->pub_seq, seq, 2000);
            continue;
        }
        std::unique_lock<std::mutex> lk(c->install_mu);
        uint64_t v;
        int b;
        if (!(c->nprod > 1 ? pin_latest_m(ctrl, r, c->nprod, &v, &b) : pin_latest(ctrl, r, &v, &b))) continue;
        if (v <= c->attempted) {
            r->pin.store(0);
            continue;
        }
        if (c->attempted && v > c->attempted + 1) {
            std::lock_guard<std::mutex> sl(c->stats_mu);
            c->stats.skipped += v - c->attempted - 1;  // latest-wins
        }
        c->attempted = v;
        const int64_t tp = ctrl->pub_time_ns.load();
        const int64_t te = ctrl->pub_entry_ns.load(std::memory_order_relaxed);
        const int64_t t0 = now_ns();
        NvtxRange nvtx("viper_install");
        viper_status st;
        static const bool dbg = getenv("VIPER_DEBUG") != nullptr;
        if (dbg) fprintf(stderr, "[viper] update thread: installing v%llu from slot %d\n", (unsigned long long)v, b);
        if (c->xproc) {
            st = xproc_install(c, v, b);
            if (dbg) fprintf(stderr, "[viper] update thread: enqueued v%llu: %d %s\n", (unsigned long long)v, st, t_err.c_str());
        } else {
            // install_mu is held through the stream sync below: a producer
            // teardown drains this before freeing the buffers read here
            viper_model *p = channel_producer(c->chan);
            st = p ? enqueue_install(c, source_of(p), v, b, c->ustream, true)
                   : set_error(VIPER_E_STATE, "producer gone");
        }
        if (st == VIPER_OK) st = wait_install_bounded(c, v, b);
        {
            std::lock_guard<std::mutex> sl(c->stats_mu);
            c->stats.t_notify_us = tp ? (t0 - tp) / 1e3 : 0.0;
            c->stats.t_pickup_us = te ? (t0 - te) / 1e3 : 0.0;
        }
        if (st == VIPER_OK) st = finish_install(c, v, (now_ns() - t0) / 1e3);
        else {
            r->status.store(st);
            finish_install(c, v, (now_ns() - t0) / 1e3);
        }
        lk.unlock();
        fire_callback(c, v, st);
    }
}

// ------------------------------------------------------------------ producer
// Wait until consumer c's install of v reported (mapped status word), without
// a stream synchronisation: the install kernel's last block writes status and
// then the version word.
viper_status wait_install_done(viper_model *c, uint64_t v, cudaStream_t st) {
    ConsRec *r = c->rec;
    const int64_t t0 = now_ns();
    for (uint32_t spins = 0;; spins++) {
        const int32_t s = r->status.load();
        if (s != 1) {
            if (s == VIPER_OK)
                while ((r->state.load() >> 1) != v) cpu_relax();
            return VIPER_OK;
        }
        if ((spins & 1023) == 1023) {
            const cudaError_t q = cudaStreamQuery(st);  // surfaces launch / device errors
            if (q != cudaSuccess && q != cudaErrorNotReady)
                return set_error(VIPER_E_CUDA, "install: %s", cudaGetErrorString(q));
            if (q == cudaSuccess && r->status.load() == 1) return set_error(VIPER_E_CUDA, "install kernel did not report");
            if (now_ns() - t0 > 60ll * 1000000000ll) return set_error(VIPER_E_TIMEOUT, "install did not finish");
        }
        cpu_relax();
    }
}

int64_t g_trace[16];  // debug: host timestamps of the last publish (viper_debug_trace)
static const bool g_trace_on = getenv("VIPER_TRACE") != nullptr;  // tools/trace_publish.py sets it
#define TRACE(i) (g_trace_on ? (void)(g_trace[i] = now_ns()) : (void)0)

// The fused kernel through its one-node graph: measured cheaper on the host
// than a direct launch (profiles/r01/launchcal.log).
static cudaError_t launch_fused_fast(viper_model *p, const FusedArgs &f, cudaStream_t st) {
    const bool no_graph = g_no_graph;
    static const int tma_env = getenv("VIPER_FUSED_TMA") ? atoi(getenv("VIPER_FUSED_TMA")) : -1;
    const int32_t fl = p->cfg.flags;
    const bool tma = tma_env >= 0                  ? tma_env != 0
                     : (fl & VIPER_FLAG_FUSED_TMA) ? true
                     : (fl & VIPER_FLAG_NO_TMA)    ? false
                                                   : kFusedTmaDefault && p->man.s_packed <= kFusedTmaMaxBytes;
    const Geometry fg = fused_geometry(p->geo, p->device, f.ncons);
    void *args[] = {(void *)&f};
    cudaKernelNodeParams kp{};
    if (tma) {
        const FusedLaunch l = fused_tma_launch(f.nitems, p->device);
        if (l.err != cudaSuccess) return l.err;
        kp.func = (void *)l.func;
        kp.gridDim = dim3(l.grid);
        kp.blockDim = dim3(l.block);
        kp.sharedMemBytes = (unsigned)l.smem;
        if (no_graph) return cudaLaunchKernel(l.func, kp.gridDim, kp.blockDim, args, l.smem, st);
    } else {
        if (no_graph) return launch_fused(f, fg, st);
        kp.func = (void *)fused_kernel_fn(f.ncons);
        kp.gridDim = dim3(fg.grid);
        kp.blockDim = dim3(fg.block);
    }
    kp.kernelParams = args;
    return p->g_fused.launch(kp, st);
}

std::atomic<uint64_t> &pub_word(viper_model *p) {
    return p->nprod > 1 ? p->ctrl->pub_m[p->pidx] : p->ctrl->pub_state;
}

static viper_status producer_publish(viper_model *p, uint64_t v, cudaStream_t st) {
    NvtxRange nvtx("viper_publish");
    const int64_t t0 = now_ns();
    if (g_trace_on) g_trace[0] = t0;
    if (v == 0 || v <= p->last_version)
        return set_error(VIPER_E_VERSION, "publish(%llu) after %llu: versions strictly increase from 1",
                         (unsigned long long)v, (unsigned long long)p->last_version);
    Ctrl *ctrl = p->ctrl;
    ctrl->pub_entry_ns.store(t0, std::memory_order_relaxed);
    if (p->xproc && p->last_version) {
        // ASYNC cross-process: the previous version's notification (a host
        // function after its pack) must have named it before slot reuse
        const int64_t w0 = now_ns();
        while ((pub_word(p).load() >> 1) != p->last_version) {
            if (now_ns() - w0 > 60ll * 1000000000ll) return set_error(VIPER_E_TIMEOUT, "previous publish stuck");
            sched_yield();
        }
    }
    const int b = p->cur_snap ^ 1;
    const uint64_t old_v = p->snap_version[b];
    // Slot b still holds old_v: wait until no consumer reads it (latest-only
    // buffer).  pub_state already names a newer version, so late
    // pinners of old_v fail their re-validation.
    if (old_v) {
        int who = -1;
        if (!wait_unpinned(ctrl, old_v, 10ll * 1000000000ll, &who))
            return set_error(VIPER_E_TIMEOUT, "consumer %d kept snapshot v%llu pinned", who, (unsigned long long)old_v);
        // the DRAM-tier D2H of old_v must be finished before overwriting
        if (p->cfg.tier == VIPER_TIER_DRAM) CUDA_TRY(cudaStreamWaitEvent(st, p->ev_ready[b], 0));
        // ... and so must the side-stream seal reduction reading its item seals
        CUDA_TRY(cudaStreamWaitEvent(st, p->ev_sealed[b], 0));
    }
    TRACE(1);
    const bool dram = p->cfg.tier == VIPER_TIER_DRAM;
    const bool sync = p->cfg.mode == VIPER_SYNC;
    viper_status result = VIPER_OK;
    // SYNC: this thread delivers + installs for every local
    // consumer, then returns once each swapped (or failed).  The host half of
    // each install (reader wait, arguments) is done BEFORE the pack launch so
    // that the first install lands right behind it on the stream (PDL).  The
    // producer waits for these installs itself, so no snapshot pin is needed.
    std::vector<std::unique_lock<std::mutex>> locks;
    std::vector<PreparedInstall> prepared;
    const SnapSource psrc = source_of(p);
    std::unique_lock<std::mutex> chan_lock;
    if (sync && p->chan) {
        chan_lock = std::unique_lock<std::mutex>(p->chan->mu);  // consumers stay registered until we return
        const std::vector<viper_model *> cons = p->chan->consumers;
        for (viper_model *c : cons) {
            std::unique_lock<std::mutex> lk(c->install_mu);
            if (c->attempted >= v) continue;
            PreparedInstall pi;
            viper_status s = prepare_install(c, psrc, v, b, &pi);
            if (s != VIPER_OK) {
                result = s;
                continue;
            }
            c->attempted = v;
            prepared.push_back(pi);
            locks.push_back(std::move(lk));
        }
    }
    TRACE(2);
    if (p->xproc && p->early_notify) {  // v is named when the stream reaches the pack (xproc.cpp)
        viper_status s = xproc_notify_early(p, v, b, st);
        if (s) return s;
    } else if (p->xproc && sync && !dram) {
        // SYNC, named only once the pack completed: wake the consumers' update
        // threads now, so they are spinning on the published word (not asleep
        // on the futex, tens of us to wake) when it lands.  A pack longer than
        // their spin sends them back to sleep; the notification wakes them.
        ctrl->pub_seq.fetch_add(1);
        futex_wake_all(&ctrl->pub_seq);
    }
    const bool timing = p->cfg.flags & VIPER_FLAG_TIMING;
    std::vector<viper_model *> launched;
    // TMA bulk-copy pack: forced by the flag, or auto for packs no install is
    // PDL-chained to (profiles/r01: faster up to ~1 GB, slightly slower above)
    const bool tma_auto = !(p->cfg.flags & VIPER_FLAG_NO_TMA) && (!sync || dram || p->xproc) &&
                          p->man.s_packed <= (1ull << 30);
    const bool tma = ((p->cfg.flags & VIPER_FLAG_TMA) || tma_auto) && !p->early_notify && !staged_fanout(p->cfg.fanout);
    const bool fuse = sync && !dram && !prepared.empty() && prepared.size() <= (size_t)kMaxFused &&
                      !(p->cfg.flags & (VIPER_FLAG_NO_FUSE | VIPER_FLAG_TMA));
    if (fuse) {
        // one kernel: pack + seal + install + verify + swap for every local consumer
        FusedArgs f{};
        f.items = p->d_items;
        f.nitems = (uint32_t)p->man.items.size();
        f.ncons = (uint32_t)prepared.size();
        f.packed = p->d_snap[b];
        f.iseal = p->d_iseal[b];
        f.version = v;
        f.flags = (unsigned long long *)p->d_flags;
        for (size_t k = 0; k < prepared.size(); k++) {
            const InstallArgs &ia = prepared[k].a;
            f.cons[k] = FusedCons{ia.items, ia.target, ia.fault_item, ia.status_h, ia.pin_h, ia.state_h};
            if (prepared[k].c->device != p->device) f.sys_swap = 1;
            prepared[k].c->rec->status.store(1);
            std::lock_guard<std::mutex> lk(prepared[k].c->stats_mu);
            prepared[k].c->stats.writer_wait_us = prepared[k].waited_us;
        }
        if (timing) CUDA_TRY(cudaEventRecord(p->ev_t[0], st));
        TRACE(8);
        CUDA_TRY(launch_fused_fast(p, f, st));
        TRACE(9);
        if (timing) {
            CUDA_TRY(cudaEventRecord(p->ev_t[1], st));
            p->timing_pending = true;
        }
        for (PreparedInstall &pi : prepared) launched.push_back(pi.c);
        prepared.clear();
    } else {
        PackArgs a{};
        a.items = p->d_items;
        a.nitems = p->pack_nitems;  // this producer's chunk share (all items with one producer)
        a.packed = p->d_snap[b];
        a.iseal = p->d_iseal[b];
        a.version = v;
        static const bool force_sys = getenv("VIPER_TEST_SYS_RELEASE") && atoi(getenv("VIPER_TEST_SYS_RELEASE"));
        a.sys_release = (p->early_notify || force_sys) ? 1u : 0u;  // (force: A/B of the seal release cost)
        a.s_packed = p->man.s_packed;
        a.l2_once = fits_l2(p->device, p->man.s_packed) ? 1u : 0u;
        if (timing) CUDA_TRY(cudaEventRecord(p->ev_t[0], st));
        // a PDL-chained install must follow a plain stream launch; every
        // other pack goes through its one-node graph (cheaper on the host)
        const bool pdl_follows = sync && !dram && !tma && !prepared.empty();
        if (p->cfg.fanout == VIPER_FANOUT_PUSH && a.nitems) {
            // push: the same pack also stores every item into each consumer's staging
            PushArgs pa{};
            pa.p = a;
            pa.ndst = (uint32_t)p->npush;
            for (int k = 0; k < p->npush; k++) {
                pa.dst[k] = p->push_dst[b][k];
                pa.dst_iseal[k] = p->push_iseal[b][k];
            }
            CUDA_TRY(launch_spec(p->g_pack, push_launch(p->geo), pa, st));
        } else if (p->cfg.fanout == VIPER_FANOUT_NVLS && a.nitems) {
            // NVLS: one store per vector to the multicast address (snapshot + every consumer)
            NvlsArgs na{};
            na.items = a.items;
            na.nitems = a.nitems;
            na.mc_packed = p->nvls_mc_snap[b];
            na.mc_iseal = p->nvls_mc_iseal[b];
            na.version = v;
            CUDA_TRY(launch_spec(p->g_pack, nvls_launch(p->geo), na, st));
        } else if (pdl_follows) {
            CUDA_TRY(launch_pack(a, p->geo, st));
        } else if (a.nitems) {
            CUDA_TRY(launch_spec(p->g_pack, pack_launch(a, p->geo, tma, p->device), a, st));
        }
        if (timing) {
            CUDA_TRY(cudaEventRecord(p->ev_t[1], st));
            p->timing_pending = true;
        }
    }
    p->last_fused = fuse;
    auto launch_all = [&]() {
        for (PreparedInstall &pi : prepared) {
            // PDL item pipeline behind the register-path pack only (the TMA
            // pack's stores are visible at grid completion)
            viper_status s = launch_prepared(pi, psrc, b, st, dram, !dram && !tma && launched.empty());
            if (s != VIPER_OK) {
                result = s;
                continue;
            }
            launched.push_back(pi.c);
        }
    };
    if (sync && !dram) launch_all();
    TRACE(3);
    if (!dram) CUDA_TRY(cudaEventRecord(p->ev_ready[b], st));
    p->snap_version[b] = v;
    p->cur_snap = b;
    p->last_version = v;
    if (!p->xproc) {
        // in process, consumers order themselves after ev_ready[b]
        pub_word(p).store((v << 1) | (uint64_t)b);
        ctrl->pub_time_ns.store(now_ns());
        if (!sync) {  // ASYNC: wake the update threads now; their installs wait on ev_ready[b] (and,
                      // DRAM tier, on the pieces' flags) on the GPU, so the rest of this call overlaps them
            ctrl->pub_seq.fetch_add(1);
            futex_wake_all(&ctrl->pub_seq);
        }
    }
    // side stream: everything that only needs the finished pack
    CUDA_TRY(cudaEventRecord(p->ev_packed, st));
    CUDA_TRY(cudaStreamWaitEvent(p->side, p->ev_packed, 0));
    if (p->xproc && !sync && !p->early_notify) {
        // remote consumers read slot b without events: name v once the pack is
        // complete (host function on the side stream; DRAM-tier consumers
        // then follow the per-piece flags below)
        viper_status s = xproc_notify(p, v, b, false);
        if (s != VIPER_OK) result = s;
    }
    if (dram) {
        // snapshot -> pinned host, piece by piece on the side
        // stream (the caller's stream is blocked only by the pack); each piece
        // raises its flag for the consumers' H2D
        const Manifest &mm = p->man;
        const size_t np = mm.piece_lo.size();
        // VIPER_TEST_DRAM_STALL=1 (tests): the producer named v but never
        // delivers it (no copy, no flag), as one that died mid-transfer
        static const bool stall = getenv("VIPER_TEST_DRAM_STALL") && atoi(getenv("VIPER_TEST_DRAM_STALL"));
        for (size_t i = 0; i < np && !stall; i++) {
            CUDA_TRY(cudaMemcpyAsync(p->h_stage[b] + mm.piece_lo[i], p->d_snap[b] + mm.piece_lo[i],
                                     mm.piece_hi[i] - mm.piece_lo[i], cudaMemcpyDeviceToHost, p->side));
            if (i + 1 == np)  // item seals once, before the last flag (one copy instead of one per piece)
                CUDA_TRY(cudaMemcpyAsync(p->h_iseal[b], p->d_iseal[b], sizeof(ISeal) * mm.items.size(),
                                         cudaMemcpyDeviceToHost, p->side));
            viper_status s = stream_write(p->side, &p->ctrl_dev->dram_flag[b][i], v);
            if (s) return s;
        }
        CUDA_TRY(cudaEventRecord(p->ev_ready[b], p->side));
    }
    // chunk seals (R16) from the item seals
    SealReduceArgs ra{};
    ra.chunk_first = p->man.d_chunk_first;
    ra.nchunks = p->man.nchunks;
    ra.iseal = p->d_iseal[b];
    ra.seals = p->d_seal[b];
    ra.version = v;
    ra.share_n = (uint32_t)p->nprod;
    ra.share_me = (uint32_t)p->pidx;
    if (ra.nchunks) CUDA_TRY(launch_spec(p->g_seal, seal_reduce_launch(ra), ra, p->side));
    if (p->flusher) {  // background flush of this version, off the training stream
        viper_status s = flush_enqueue(p, v, b);
        if (s) return s;
    }
    CUDA_TRY(cudaEventRecord(p->ev_sealed[b], p->side));
    TRACE(4);
    if (sync && dram) launch_all();

    if (p->cfg.fanout == VIPER_FANOUT_NCCL) {
        // NCCL baseline: broadcast v to the consumers' staging.  Enqueued after
        // ev_packed (the notification that lets the consumers join waits on it)
        // and as the very last step before that notification, so no early
        // error return can leave the collective waiting for consumers that
        // were never told about v.
        viper_status s = nccl_broadcast_version(p, p->d_snap[b], p->d_iseal[b], p->rank, st);
        if (s) return s;
    }
    if (p->xproc) {
        if (sync) {  // name v once the pack completed, then wait for every consumer
            viper_status s = xproc_notify(p, v, b, true, p->early_notify);
            if (s != VIPER_OK) result = s;
        }
    } else if (sync) {
        const int64_t ti = now_ns();
        for (viper_model *c : launched) {
            viper_status s = wait_install_done(c, v, st);
            TRACE(5);
            if (s != VIPER_OK) {
                c->rec->status.store(s);
                if (result == VIPER_OK) result = s;
            }
            s = finish_install(c, v, (now_ns() - ti) / 1e3);
            if (s != VIPER_OK && result == VIPER_OK) result = s;
        }
        TRACE(6);
        locks.clear();
        for (viper_model *c : launched) fire_callback(c, v, c->rec->last_status.load());
    }
    {
        std::lock_guard<std::mutex> lk(p->stats_mu);
        p->stats.version = v;
        p->stats.t_publish_us = (now_ns() - t0) / 1e3;
        p->stats.last_status = result;
    }
    TRACE(7);
    log_update("producer", p, v, result, (now_ns() - t0) / 1e3, p->last_fused ? 1.0 : 0.0, "fused");
    return result;
}

// -------------------------------------------------------------- registration
static viper_status check_tensors(const viper_tensor *t, int32_t n) {
    if (n < 0 || (n > 0 && !t)) return set_error(VIPER_E_INVAL, "bad tensor list");
    for (int32_t i = 0; i < n; i++) {
        if (t[i].nbytes && !t[i].dev_ptr) return set_error(VIPER_E_INVAL, "tensor %d: null dev_ptr", i);
        if (t[i].dtype < VIPER_F32 || t[i].dtype > VIPER_BYTES) return set_error(VIPER_E_INVAL, "tensor %d: dtype", i);
        if (t[i].nbytes > 0xFFFFFFFFull * 64) return set_error(VIPER_E_INVAL, "tensor %d too large", i);
    }
    return VIPER_OK;
}

static void free_model(viper_model *m) {
    if (!m) return;
    if (m->upd.joinable()) {
        m->stop.store(true);
        if (m->ctrl) {
            m->ctrl->pub_seq.fetch_add(1);
            futex_wake_all(&m->ctrl->pub_seq);
        }
        m->upd.join();
    }
    if (m->chan) {
        Channel *ch = m->chan;
        if (m->role == VIPER_PRODUCER) {
            {
                std::lock_guard<std::mutex> lk(ch->pmu);
                if (ch->producer == m) ch->producer = nullptr;
            }
            // drain installs that may still read this producer's buffers; the
            // consumers cannot disappear meanwhile: their teardown takes ch->mu
            std::lock_guard<std::mutex> lk(ch->mu);
            for (viper_model *c : ch->consumers) {
                std::lock_guard<std::mutex> il(c->install_mu);
            }
        } else {
            std::lock_guard<std::mutex> lk(ch->mu);  // waits for an in-flight SYNC publish
            auto &v = ch->consumers;
            v.erase(std::remove(v.begin(), v.end(), m), v.end());
        }
    }
    DeviceGuard dg(m->device);
    cudaDeviceSynchronize();
    flush_stop(m);
    if (m->rec) m->rec->active.store(0);
    if (m->xproc) xproc_free(m);
    if (m->chan) channel_close(m->chan);
    cudaFree(m->man.d_chunk_first);
    cudaFree(m->d_items);
    cudaFree(m->d_slot_items[0]);
    cudaFree(m->d_slot_items[1]);
    cudaFree(m->d_flags);
    cudaFree(m->snap_alloc);
    cudaFree(m->slot1_alloc);
    cudaFree(m->stage_alloc);
    if (m->h_stage_alloc) cudaFreeHost(m->h_stage_alloc);
    for (auto *evs : {m->ev_ready, m->ev_sealed, m->ev_t})
        for (int k = 0; k < 2; k++)
            if (evs[k]) cudaEventDestroy(evs[k]);
    if (m->ev_packed) cudaEventDestroy(m->ev_packed);
    if (m->ev_notify) cudaEventDestroy(m->ev_notify);
    m->g_fused.destroy();
    m->g_pack.destroy();
    m->g_seal.destroy();
    m->g_inst.destroy();
    if (m->side) cudaStreamDestroy(m->side);
    if (m->ustream) cudaStreamDestroy(m->ustream);
    delete m;
}

static uint64_t al256(uint64_t x) { return (x + 255) / 256 * 256; }

// Producer-side buffers: two snapshot slots (the latest + the one being
// filled), their item seals and chunk seals, the events and side stream.
viper_status alloc_producer(viper_model *m, const viper_tensor *tensors) {
    const uint64_t S = al256(m->man.s_packed);
    const uint64_t IS = al256(sizeof(ISeal) * std::max<size_t>(m->man.items.size(), 1));
    const uint64_t CS = al256(sizeof(Seal) * std::max<uint32_t>(m->man.nchunks, 1));
    for (int32_t i = 0; i < m->man.n; i++) m->src_ptrs.push_back(tensors[i].dev_ptr);
    viper_status st = upload_items(m->man, m->src_ptrs, &m->d_items, (uint32_t)m->nprod, (uint32_t)m->pidx,
                                   &m->pack_nitems);
    if (st) return st;
    const size_t bytes = 2 * (S + IS + CS);
    CUDA_TRY(cudaMalloc(&m->snap_alloc, bytes));
    CUDA_TRY(cudaMemset(m->snap_alloc, 0, bytes));  // padding bytes stay 0 forever
    uint8_t *p = (uint8_t *)m->snap_alloc;
    for (int b = 0; b < 2; b++) {
        m->d_snap[b] = p + b * S;
        m->d_iseal[b] = (ISeal *)(p + 2 * S + b * IS);
        m->d_seal[b] = (Seal *)(p + 2 * S + 2 * IS + b * CS);
    }
    for (auto &e : m->ev_ready) CUDA_TRY(cudaEventCreateWithFlags(&e, cudaEventDisableTiming));
    for (auto &e : m->ev_sealed) CUDA_TRY(cudaEventCreateWithFlags(&e, cudaEventDisableTiming));
    for (auto &e : m->ev_t) CUDA_TRY(cudaEventCreate(&e));
    CUDA_TRY(cudaEventCreateWithFlags(&m->ev_packed, cudaEventDisableTiming));
    CUDA_TRY(cudaEventCreateWithFlags(&m->ev_notify, cudaEventDisableTiming));
    CUDA_TRY(cudaStreamCreateWithFlags(&m->side, cudaStreamNonBlocking));
    CUDA_TRY(cudaMalloc(&m->d_flags, 64));
    CUDA_TRY(cudaMemset(m->d_flags, 0, 64));
    if (m->cfg.tier == VIPER_TIER_DRAM && !m->xproc) {  // cross-process: in the shm segment (xproc.cpp)
        CUDA_TRY(cudaHostAlloc(&m->h_stage_alloc, 2 * (S + IS), cudaHostAllocPortable));
        uint8_t *h = (uint8_t *)m->h_stage_alloc;
        for (int b = 0; b < 2; b++) {
            m->h_stage[b] = h + b * S;
            m->h_iseal[b] = (ISeal *)(h + 2 * S + b * IS);
        }
    }
    return VIPER_OK;
}

// Consumer-side buffers: slot 1 (unless supplied), per-slot work lists,
// completion flags, DRAM-tier staging, the update stream.
viper_status alloc_consumer(viper_model *m, const viper_tensor *tensors) {
    viper_status st;
    const uint64_t S = m->man.s_packed;
    for (int32_t i = 0; i < m->man.n; i++) m->slot_ptrs[0].push_back(tensors[i].dev_ptr);
    if (m->cfg.slot1) {
        for (int32_t i = 0; i < m->man.n; i++) {
            if (m->cfg.slot1[i].nbytes != m->man.nbytes[i] || (m->man.nbytes[i] && !m->cfg.slot1[i].dev_ptr))
                return set_error(VIPER_E_INVAL, "slot1 tensor %d does not match", i);
            m->slot_ptrs[1].push_back(m->cfg.slot1[i].dev_ptr);
        }
    } else {
        CUDA_TRY(cudaMalloc(&m->slot1_alloc, std::max<uint64_t>(S, 256)));
        for (int32_t i = 0; i < m->man.n; i++) m->slot_ptrs[1].push_back((uint8_t *)m->slot1_alloc + m->man.offsets[i]);
    }
    for (int s = 0; s < 2; s++)
        if ((st = upload_items(m->man, m->slot_ptrs[s], &m->d_slot_items[s], 1, 0, nullptr))) return st;
    CUDA_TRY(cudaMalloc(&m->d_flags, 64));
    CUDA_TRY(cudaMemset(m->d_flags, 0, 64));
    if (copy_staged(m->cfg.tier, m->cfg.fanout)) {
        const uint64_t IS = al256(sizeof(ISeal) * std::max<size_t>(m->man.items.size(), 1));
        CUDA_TRY(cudaMalloc(&m->stage_alloc, al256(S) + IS));
        m->d_stage = (uint8_t *)m->stage_alloc;
        m->d_stage_iseal = (ISeal *)(m->d_stage + al256(S));
    }
    CUDA_TRY(cudaStreamCreateWithFlags(&m->ustream, cudaStreamNonBlocking));
    for (auto &e : m->ev_t) CUDA_TRY(cudaEventCreate(&e));
    return VIPER_OK;
}

// In-process endpoints on two GPUs: the producer's kernels write consumer slots
// (fused SYNC kernel, SYNC installs on the producer's stream) and a consumer's
// kernels read the producer's snapshot, so both directions need peer access.
// The DRAM tier moves everything through host memory and needs none.
static viper_status link_devices(int a, int b, int32_t tier) {
    if (a == b || tier == VIPER_TIER_DRAM) return VIPER_OK;
    int cur = 0;
    cudaGetDevice(&cur);
    viper_status st = VIPER_OK;
    for (int k = 0; k < 2 && st == VIPER_OK; k++) {
        const int x = k ? b : a, y = k ? a : b;
        int can = 0;
        if (cudaDeviceCanAccessPeer(&can, x, y) != cudaSuccess || !can) {
            st = set_error(VIPER_E_UNSUPPORTED, "GPU tier: device %d cannot access device %d (use the DRAM tier)", x, y);
            break;
        }
        cudaSetDevice(x);
        const cudaError_t e = cudaDeviceEnablePeerAccess(y, 0);
        if (e == cudaErrorPeerAccessAlreadyEnabled) cudaGetLastError();
        else if (e != cudaSuccess) st = set_error(VIPER_E_CUDA, "cudaDeviceEnablePeerAccess(%d -> %d): %s", x, y, cudaGetErrorString(e));
    }
    cudaSetDevice(cur);
    return st;
}

// Transfer Selector, in process (VIPER_TIER_AUTO): the tier of the model's
// existing endpoints; for the first one, the GPU tier when this GPU can
// peer-access every visible GPU (or is the only one) -- a process-wide fact,
// so endpoints registering concurrently decide alike -- else the DRAM tier.
static int32_t select_tier_local(const std::string &name, int device) {
    {
        std::lock_guard<std::mutex> lk(g_reg_mu);
        auto it = g_reg.find(name);
        if (it != g_reg.end()) return it->second->tier;
    }
    int ndev = 0;
    cudaGetDeviceCount(&ndev);
    for (int d = 0; d < ndev; d++) {
        int can = 0;
        if (d != device && (cudaDeviceCanAccessPeer(&can, device, d) != cudaSuccess || !can)) return VIPER_TIER_DRAM;
    }
    return VIPER_TIER_GPU;
}

static viper_status register_local(viper_model *m, const viper_tensor *tensors) {
    if (m->cfg.tier == VIPER_TIER_AUTO) m->cfg.tier = select_tier_local(m->name, m->device);
    viper_status st = channel_open(m->name, m->man, m->cfg.tier, &m->chan);
    if (st) return st;
    m->ctrl = m->chan->ctrl;
    m->ctrl_dev = m->chan->ctrl_dev;
    if (m->role == VIPER_PRODUCER) {
        viper_status ps = alloc_producer(m, tensors);
        if (ps == VIPER_OK && m->cfg.flush_dir) ps = flush_start(m, m->cfg.flush_dir);
        if (ps) return ps;
        // chan->mu orders this against consumers registering concurrently
        // (each side links to the endpoints it sees; lock order mu -> pmu)
        std::lock_guard<std::mutex> ck(m->chan->mu);
        for (viper_model *c : m->chan->consumers)
            if ((ps = link_devices(m->device, c->device, m->cfg.tier))) return ps;
        std::lock_guard<std::mutex> lk(m->chan->pmu);  // visible only once fully built
        if (m->chan->producer) return set_error(VIPER_E_STATE, "model '%s' already has a producer", m->name.c_str());
        m->chan->producer = m;
        return VIPER_OK;
    }
    if ((st = alloc_consumer(m, tensors))) return st;
    {
        std::lock_guard<std::mutex> lk(m->chan->mu);
        if (viper_model *p = channel_producer(m->chan))
            if ((st = link_devices(p->device, m->device, m->cfg.tier))) return st;
        // reuse the record of a consumer that unregistered (no reader left on
        // it), so restarting consumers never exhaust the kMaxConsumers records;
        // ncons stays the high-water mark the scans cover
        int idx = -1;
        const int n = m->ctrl->ncons.load();
        for (int i = 0; i < n && idx < 0; i++) {
            ConsRec &r = m->ctrl->cons[i];
            if (!r.active.load() && r.ref[0].load() == 0 && r.ref[1].load() == 0) idx = i;
        }
        if (idx < 0 && n >= kMaxConsumers)
            return set_error(VIPER_E_INVAL, "more than %d live consumers", kMaxConsumers);
        if (idx < 0) idx = n;
        m->cidx = idx;
        m->rec = &m->ctrl->cons[idx];
        m->rec_dev = &m->ctrl_dev->cons[idx];
        m->rec->state.store(0);
        m->rec->pin.store(0);
        m->rec->status.store(0);
        m->rec->done_version.store(0);
        m->rec->last_status.store(0);
        m->rec->abort.store(0);
        m->rec->active.store(1);
        if (idx == n) m->ctrl->ncons.store(idx + 1);
        m->chan->consumers.push_back(m);
    }
    m->upd = std::thread(update_loop, m);
    return VIPER_OK;
}

}  // namespace vp

using namespace vp;

// =================================================================== C-ABI
extern "C" {


// Every tensor must be device (or managed) memory of the model's device: a
// tensor on another GPU would otherwise be read over the peer mapping, or fault.
static viper_status check_tensor_devices(const viper_tensor *t, int32_t n, int device) {
    for (int32_t i = 0; i < n; i++) {
        if (!t[i].nbytes) continue;
        cudaPointerAttributes pa{};
        if (cudaPointerGetAttributes(&pa, t[i].dev_ptr) != cudaSuccess) {
            cudaGetLastError();
            return set_error(VIPER_E_INVAL, "tensor %d: not a CUDA allocation", i);
        }
        if (pa.type == cudaMemoryTypeManaged) continue;
        if (pa.type != cudaMemoryTypeDevice)
            return set_error(VIPER_E_INVAL, "tensor %d: not device memory (there is no host path)", i);
        if (pa.device != device)
            return set_error(VIPER_E_INVAL, "tensor %d lives on device %d, the model on device %d", i, pa.device, device);
    }
    return VIPER_OK;
}

static viper_status register_impl(const char *model_name, int32_t role, const viper_tensor *tensors, int32_t n,
                                  const viper_config *cfg, const viper_bootstrap *bs, viper_model **out,
                                  bool *joined) {
    {
        if (!out) return set_error(VIPER_E_INVAL, "out is NULL");
        *out = nullptr;
        if (!model_name || !*model_name) return set_error(VIPER_E_INVAL, "empty model name");
        if (role != VIPER_PRODUCER && role != VIPER_CONSUMER) return set_error(VIPER_E_INVAL, "bad role %d", role);
        viper_status st = check_tensors(tensors, n);
        if (st) return st;
        viper_config c{};
        if (cfg) c = *cfg;
        if (c.chunk_bytes == 0) c.chunk_bytes = 2ull << 20;
        if (c.align == 0) c.align = 256;
        if (c.align < 16 || (c.align & (c.align - 1))) return set_error(VIPER_E_INVAL, "align must be a power of 2 >= 16");
        if (c.chunk_bytes % 256 || c.chunk_bytes % c.align) return set_error(VIPER_E_INVAL, "chunk_bytes must be a multiple of 256 and align");
        if (c.tier != VIPER_TIER_GPU && c.tier != VIPER_TIER_DRAM && c.tier != VIPER_TIER_AUTO)
            return set_error(VIPER_E_INVAL, "bad tier");
        if (c.mode != VIPER_SYNC && c.mode != VIPER_ASYNC) return set_error(VIPER_E_INVAL, "bad mode");
        if (c.install_sms < 0) return set_error(VIPER_E_INVAL, "install_sms must be >= 0");
        if (c.fanout != VIPER_FANOUT_DIRECT && c.fanout != VIPER_FANOUT_CHAIN &&
            c.fanout != VIPER_FANOUT_SCATTER_ALLGATHER && !xproc_only_fanout(c.fanout))
            return set_error(VIPER_E_UNSUPPORTED, "fanout %d not supported", c.fanout);
        if (xproc_only_fanout(c.fanout) && !(bs && bs->world > 1))
            return set_error(VIPER_E_UNSUPPORTED, "fanout %d (NVLS / push / CE / NCCL) needs the cross-process channel",
                             c.fanout);
        int ndev = 0;
        if (cudaGetDeviceCount(&ndev) != cudaSuccess || ndev <= 0)
            return set_error(VIPER_E_CUDA, "no CUDA device (there is no CPU fallback)");
        if (c.device < 0 || c.device >= ndev) return set_error(VIPER_E_INVAL, "bad device %d", c.device);
        DeviceGuard dg(c.device);  // until this call returns (the update thread sets its own)
        if (dg.err != cudaSuccess) return set_error(VIPER_E_CUDA, "cudaSetDevice(%d): %s", c.device, cudaGetErrorString(dg.err));
        CUDA_TRY(preload_kernels());
        st = check_tensor_devices(tensors, n, c.device);
        if (st) return st;
        viper_model *m = new viper_model();
        m->name = model_name;
        m->role = role;
        m->device = c.device;
        m->cfg = c;
        st = build_manifest(m->man, tensors, n, c.chunk_bytes, c.align, c.device);
        if (!st) {
            m->geo = pick_geometry((uint32_t)m->man.items.size(), c.device,
                                   role == VIPER_CONSUMER ? c.install_sms : 0);
            if (bs && bs->world > 1) {
                m->xproc = true;
                *joined = true;
                st = xproc_register(m, tensors, bs);
            } else {
                st = register_local(m, tensors);
            }
        }
        if (st) {
            std::string keep = t_err;
            free_model(m);
            t_err = keep;
            return st;
        }
        {
            std::lock_guard<std::mutex> lk(m->stats_mu);
            m->stats.s_packed = m->man.s_packed;
            m->stats.nchunks = m->man.nchunks;
            m->stats.nitems = m->man.items.size();
        }
        *out = m;
        return VIPER_OK;
    }
}

viper_status viper_register_model(const char *model_name, int32_t role, const viper_tensor *tensors, int32_t n,
                                  const viper_config *cfg, const viper_bootstrap *bs, viper_model **out) {
    bool joined = false;
    viper_status st;
    try {
        st = register_impl(model_name, role, tensors, n, cfg, bs, out, &joined);
    } catch (const std::exception &e) {
        st = set_error(VIPER_E_NOMEM, "register: %s", e.what());
    }
    // failed before the bootstrap: still take part in its collectives, so the
    // other ranks fail with VIPER_E_PEER instead of waiting forever
    if (st != VIPER_OK && !joined && bs && bs->world > 1 && bs->allgather) xproc_abort(bs, st);
    return st;
}

viper_status viper_publish(viper_model *m, uint64_t version, void *cuda_stream) {
    if (!m || m->closed.load()) return set_error(VIPER_E_STATE, "model closed");
    if (m->role != VIPER_PRODUCER) return set_error(VIPER_E_STATE, "publish on a consumer");
    try {
        DeviceGuard dg(m->device);
        if (dg.err != cudaSuccess) return set_error(VIPER_E_CUDA, "cudaSetDevice");
        return producer_publish(m, version, (cudaStream_t)cuda_stream);
    } catch (const std::exception &e) {
        return set_error(VIPER_E_NOMEM, "publish: %s", e.what());
    }
}

viper_status viper_subscribe(viper_model *m, void (*on_update)(uint64_t, viper_status, void *), void *user) {
    if (!m || m->closed.load()) return set_error(VIPER_E_STATE, "model closed");
    if (m->role != VIPER_CONSUMER) return set_error(VIPER_E_STATE, "subscribe on a producer");
    std::lock_guard<std::mutex> lk(m->cb_mu);
    m->cb = on_update;
    m->cb_user = user;
    return VIPER_OK;
}

viper_status viper_acquire_latest(viper_model *m, uint64_t min_version, int64_t timeout_us, viper_view *out) {
    if (!m || !out || m->closed.load()) return set_error(VIPER_E_STATE, "model closed");
    if (m->role != VIPER_CONSUMER) return set_error(VIPER_E_STATE, "acquire on a producer");
    ConsRec *r = m->rec;
    const int64_t deadline = timeout_us < 0 ? INT64_MAX : now_ns() + timeout_us * 1000;
    for (;;) {
        const uint32_t seq = r->done_seq.load();
        const uint64_t s = r->state.load();
        if (s == 0 || (s >> 1) < min_version) {
            const int64_t now = now_ns();
            if (timeout_us == 0) return set_error(VIPER_E_NOVERSION, "no version >= %llu installed",
                                                  (unsigned long long)min_version);
            if (now >= deadline) return set_error(VIPER_E_TIMEOUT, "acquire timed out");
            const int64_t left_us = (deadline - now) / 1000;
            r->waiters.fetch_add(1);
            if (r->done_seq.load() == seq) futex_wait(&r->done_seq, seq, std::min<int64_t>(left_us, 1000));
            r->waiters.fetch_sub(1);
            continue;
        }
        const uint64_t got = try_acquire_slot(r, min_version);
        if (got) {
            const int slot = (int)(got & 1);
            std::lock_guard<std::mutex> lk(m->views_mu);
            const uint64_t t = m->next_ticket++;
            m->views[t] = ViewTicket{slot};
            out->version = got >> 1;
            out->slot = slot;
            out->ntensors = m->man.n;
            out->dev_ptrs = m->slot_ptrs[slot].data();
            out->ticket = t;
            return VIPER_OK;
        }
    }
}

struct ReleaseCtx {
    ConsRec *r;
    int slot;
};

static void CUDART_CB release_host_fn(void *p) {
    ReleaseCtx *c = (ReleaseCtx *)p;
    c->r->ref[c->slot].fetch_sub(1);
    delete c;
}

viper_status viper_release(viper_model *m, const viper_view *view, void *cuda_stream) {
    if (!m || !view || m->closed.load()) return set_error(VIPER_E_STATE, "model closed");
    if (m->role != VIPER_CONSUMER) return set_error(VIPER_E_STATE, "release on a producer");
    int slot;
    {
        std::lock_guard<std::mutex> lk(m->views_mu);
        auto it = m->views.find(view->ticket);
        if (it == m->views.end() || it->second.slot != view->slot)
            return set_error(VIPER_E_STATE, "unknown or already released view (ticket %llu)",
                             (unsigned long long)view->ticket);
        slot = it->second.slot;
        m->views.erase(it);
    }
    if (cuda_stream) {
        DeviceGuard dg(m->device);
        ReleaseCtx *c = new ReleaseCtx{m->rec, slot};
        cudaError_t e = cudaLaunchHostFunc((cudaStream_t)cuda_stream, release_host_fn, c);
        if (e != cudaSuccess) {
            delete c;
            m->rec->ref[slot].fetch_sub(1);
            return set_error(VIPER_E_CUDA, "cudaLaunchHostFunc: %s", cudaGetErrorString(e));
        }
        return VIPER_OK;
    }
    m->rec->ref[slot].fetch_sub(1);
    return VIPER_OK;
}

viper_status viper_wait_installed(viper_model *m, uint64_t v, int64_t timeout_us) {
    if (!m || m->closed.load()) return set_error(VIPER_E_STATE, "model closed");
    if (m->role != VIPER_CONSUMER) return set_error(VIPER_E_STATE, "wait_installed on a producer");
    ConsRec *r = m->rec;
    const int64_t deadline = timeout_us < 0 ? INT64_MAX : now_ns() + timeout_us * 1000;
    for (;;) {
        const uint32_t seq = r->done_seq.load();
        if ((r->state.load() >> 1) >= v) return VIPER_OK;
        if (r->done_version.load() >= v && r->last_status.load() != VIPER_OK) return r->last_status.load();
        const int64_t now = now_ns();
        if (now >= deadline) return set_error(VIPER_E_TIMEOUT, "version %llu not installed in time", (unsigned long long)v);
        r->waiters.fetch_add(1);
        if (r->done_seq.load() == seq) futex_wait(&r->done_seq, seq, std::min<int64_t>((deadline - now) / 1000, 1000));
        r->waiters.fetch_sub(1);
    }
}

viper_status viper_get_stats(viper_model *m, viper_stats *out) {
    if (!m || !out) return set_error(VIPER_E_INVAL, "null");
    if (m->role == VIPER_PRODUCER && m->timing_pending && cudaEventQuery(m->ev_t[1]) == cudaSuccess) {
        float ms = 0;
        if (cudaEventElapsedTime(&ms, m->ev_t[0], m->ev_t[1]) == cudaSuccess) {
            std::lock_guard<std::mutex> lk(m->stats_mu);
            if (m->last_fused) m->stats.t_fused_dev_us = ms * 1e3;
            else m->stats.t_pack_dev_us = ms * 1e3;
        }
        m->timing_pending = false;
    }
    std::lock_guard<std::mutex> lk(m->stats_mu);
    *out = m->stats;
    out->nconsumers = m->ctrl ? m->ctrl->ncons.load() : 0;
    flush_stats(m, &out->flushed, &out->flush_skipped, &out->flush_last);
    out->tier = m->cfg.tier;
    out->fanout = m->cfg.fanout;
    return VIPER_OK;
}

viper_status viper_layout(viper_model *m, uint64_t *s_packed, uint64_t *offsets, int32_t n) {
    if (!m) return set_error(VIPER_E_INVAL, "null model");
    if (s_packed) *s_packed = m->man.s_packed;
    if (offsets) {
        if (n < m->man.n) return set_error(VIPER_E_INVAL, "offsets array too small");
        for (int32_t i = 0; i < m->man.n; i++) offsets[i] = m->man.offsets[i];
    }
    return VIPER_OK;
}

viper_status viper_debug_buffers(viper_model *m, void **dev_packed, void **dev_seals, uint64_t *nchunks) {
    if (!m) return set_error(VIPER_E_INVAL, "null model");
    if (nchunks) *nchunks = m->man.nchunks;
    if (m->role == VIPER_PRODUCER) {
        const int b = m->cur_snap;
        if (m->ev_sealed[b]) CUDA_TRY(cudaEventSynchronize(m->ev_sealed[b]));
        if (dev_packed) *dev_packed = m->d_snap[b];
        if (dev_seals) *dev_seals = m->d_seal[b];
    } else {
        if (dev_packed) *dev_packed = m->d_stage;
        if (dev_seals) *dev_seals = nullptr;
    }
    return VIPER_OK;
}

viper_status viper_view_seals(viper_model *m, const viper_view *view, void *dev_seals_out, void *cuda_stream) {
    if (!m || !view || m->closed.load()) return set_error(VIPER_E_STATE, "model closed");
    if (m->role != VIPER_CONSUMER) return set_error(VIPER_E_STATE, "view_seals on a producer");
    if (!dev_seals_out && m->man.nchunks) return set_error(VIPER_E_INVAL, "dev_seals_out is NULL");
    {
        std::lock_guard<std::mutex> lk(m->views_mu);
        auto it = m->views.find(view->ticket);
        if (it == m->views.end() || it->second.slot != view->slot)
            return set_error(VIPER_E_STATE, "unknown or released view (ticket %llu)", (unsigned long long)view->ticket);
    }
    DeviceGuard dg(m->device);
    if (dg.err != cudaSuccess) return set_error(VIPER_E_CUDA, "cudaSetDevice");
    const cudaStream_t st = (cudaStream_t)cuda_stream;
    if (m->man.nchunks) CUDA_TRY(cudaMemsetAsync(dev_seals_out, 0, sizeof(Seal) * m->man.nchunks, st));
    ViewSealArgs a{};
    a.items = m->d_slot_items[view->slot];
    a.nitems = (uint32_t)m->man.items.size();
    a.seals = (Seal *)dev_seals_out;
    a.version = view->version;
    CUDA_TRY(launch_view_seals(a, st));
    return VIPER_OK;
}

viper_status viper_debug_trace(int64_t *out, int32_t n) {
    for (int i = 0; i < n && i < 16; i++) out[i] = g_trace[i];
    return VIPER_OK;
}

viper_status viper_debug_fault_next(viper_model *m) {
    if (!m || m->role != VIPER_CONSUMER) return set_error(VIPER_E_STATE, "consumer only");
    m->fault_next.store(true);
    return VIPER_OK;
}

viper_status viper_unregister(viper_model *m) {
    if (!m) return set_error(VIPER_E_INVAL, "null model");
    if (m->closed.exchange(true)) return set_error(VIPER_E_STATE, "double unregister");
    free_model(m);
    return VIPER_OK;
}

const char *viper_strerror(viper_status st) {
    switch (st) {
        case VIPER_OK: return "VIPER_OK";
        case VIPER_E_INVAL: return "VIPER_E_INVAL";
        case VIPER_E_NOMEM: return "VIPER_E_NOMEM";
        case VIPER_E_CUDA: return "VIPER_E_CUDA";
        case VIPER_E_VERSION: return "VIPER_E_VERSION";
        case VIPER_E_CHECKSUM: return "VIPER_E_CHECKSUM";
        case VIPER_E_TIMEOUT: return "VIPER_E_TIMEOUT";
        case VIPER_E_NOVERSION: return "VIPER_E_NOVERSION";
        case VIPER_E_STATE: return "VIPER_E_STATE";
        case VIPER_E_UNSUPPORTED: return "VIPER_E_UNSUPPORTED";
        case VIPER_E_PEER: return "VIPER_E_PEER";
        default: return "VIPER_E_UNKNOWN";
    }
}

const char *viper_last_error(void) { return t_err.c_str(); }
const char *viper_version(void) { return "viper-b200 0.1 (sm_100a)"; }

}  // extern "C"
