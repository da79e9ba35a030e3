// xproc.cpp -- the cross-process channel: one process per GPU (PAPER.md s4.4
// "GPU-to-GPU memory and Host-to-Host memory" channels), rebuilt
// for one NVSwitch node:
//
//   bootstrap   two allgathers over the caller's process group (records, then
//               statuses) -- the only use of a collective on this path;
//   control     the producer creates a shared-memory segment holding the Ctrl
//               block (+ the DRAM-tier host staging); every rank maps it and
//               registers it with CUDA (mapped), so install kernels flip their
//               consumer's version word from the device;
//   data        consumers CUDA-IPC-map the producer's snapshot allocation and
//               their install kernel pulls it over NVLink (peer loads), or
//               copies it from the shared host staging (DRAM tier);
//   notify      pub_state + a shared futex, written once slot b is complete
//               (SYNC: after an event sync; ASYNC: a host function on the
//               producer's side stream) -- "proactively informing consumers of
//               model updates".
#include <fcntl.h>
#include <sys/mman.h>
#include <sys/stat.h>
#include <sys/statvfs.h>
#include <unistd.h>

#include <climits>
#include <cstring>
#include <new>
#include <random>

#include "protocol.h"
#include "runtime.h"
#include "selector.h"

namespace vp {

namespace {

constexpr uint32_t kPeerMagic = 0x56495052u;  // "VIPR"

struct PeerRec {
    uint32_t magic;
    int32_t role, rank, device, pid, status, tier, fanout;
    uint64_t s_packed, nitems, nchunks, manifest_hash;
    uint64_t snap_off[2], iseal_off[2];      // inside the producer's IPC allocation
    uint64_t shm_bytes, stage_off[2], hiseal_off[2];  // inside the shm segment (DRAM tier)
    char shm_path[128];                      // "/name" (POSIX shm) or an absolute file path
    cudaIpcMemHandle_t snap_handle;
    cudaIpcMemHandle_t sa_handle;            // consumer staging (scatter-allgather)
    int32_t cidx;
    char pci[32];                            // PCI bus id of the rank's GPU
    char nvls_sock[64];                      // producer, NVLS: abstract socket serving the multicast fd
    uint64_t nvls_bytes;                     // producer, NVLS: size of the multicast object
    char nccl_id[128];                       // producer, NCCL fan-out: the ncclUniqueId
};

uint64_t fnv1a(const void *p, size_t n, uint64_t h = 0xcbf29ce484222325ull) {
    const uint8_t *b = (const uint8_t *)p;
    for (size_t i = 0; i < n; i++) h = (h ^ b[i]) * 0x100000001b3ull;
    return h;
}

uint64_t manifest_hash(const Manifest &m) {
    uint64_t h = fnv1a(m.nbytes.data(), m.nbytes.size() * sizeof(uint64_t));
    h = fnv1a(&m.align, sizeof m.align, h);
    return fnv1a(&m.chunk_bytes, sizeof m.chunk_bytes, h);
}

size_t page_up(size_t x) { return (x + 4095) / 4096 * 4096; }

bool is_posix_shm(const char *path) { return path[0] == '/' && strchr(path + 1, '/') == nullptr; }

// Create the segment: POSIX shm when /dev/shm has room, else a file in /tmp
// (a MAP_SHARED file mapping is shared the same way).
viper_status create_segment(viper_model *m, size_t bytes, char *path_out, size_t cap) {
    std::random_device rd;
    std::string base;
    for (char ch : m->name) base += (isalnum((unsigned char)ch) ? ch : '_');
    if (base.size() > 40) base.resize(40);
    char tag[64];
    snprintf(tag, sizeof tag, "viper-%s-%d-%08x", base.c_str(), (int)getpid(), (unsigned)rd());
    struct statvfs sv;
    const bool shm_ok = statvfs("/dev/shm", &sv) == 0 && (uint64_t)sv.f_bavail * sv.f_frsize > bytes + (64u << 20);
    int fd;
    if (shm_ok) {
        snprintf(path_out, cap, "/%s", tag);
        fd = shm_open(path_out, O_CREAT | O_EXCL | O_RDWR, 0600);
    } else {
        snprintf(path_out, cap, "/tmp/%s", tag);
        fd = open(path_out, O_CREAT | O_EXCL | O_RDWR, 0600);
    }
    if (fd < 0) return set_error(VIPER_E_NOMEM, "cannot create control segment %s", path_out);
    if (ftruncate(fd, (off_t)bytes) != 0) {
        close(fd);
        return set_error(VIPER_E_NOMEM, "ftruncate(%s, %zu) failed", path_out, bytes);
    }
    void *p = mmap(nullptr, bytes, PROT_READ | PROT_WRITE, MAP_SHARED, fd, 0);
    close(fd);
    if (p == MAP_FAILED) return set_error(VIPER_E_NOMEM, "mmap(%s) failed", path_out);
    m->shm_base = p;
    m->shm_bytes = bytes;
    m->shm_name = path_out;
    m->shm_owner = true;
    return VIPER_OK;
}

viper_status open_segment(viper_model *m, const char *path, size_t bytes) {
    const int fd = is_posix_shm(path) ? shm_open(path, O_RDWR, 0600) : open(path, O_RDWR);
    if (fd < 0) return set_error(VIPER_E_PEER, "cannot open control segment %s", path);
    void *p = mmap(nullptr, bytes, PROT_READ | PROT_WRITE, MAP_SHARED, fd, 0);
    close(fd);
    if (p == MAP_FAILED) return set_error(VIPER_E_PEER, "mmap(%s) failed", path);
    m->shm_base = p;
    m->shm_bytes = bytes;
    m->shm_name = path;
    return VIPER_OK;
}

#define CUDA_TRY(x)                                                                                          \
    do {                                                                                                     \
        cudaError_t e_ = (x);                                                                                \
        if (e_ != cudaSuccess)                                                                               \
            return set_error(VIPER_E_CUDA, "%s failed: %s (%s:%d)", #x, cudaGetErrorString(e_), __FILE__, __LINE__); \
    } while (0)

viper_status map_control(viper_model *m) {
    CUDA_TRY(cudaHostRegister(m->shm_base, m->shm_bytes, cudaHostRegisterPortable | cudaHostRegisterMapped));
    m->shm_registered = true;
    void *d = nullptr;
    CUDA_TRY(cudaHostGetDevicePointer(&d, m->shm_base, 0));
    m->ctrl = (Ctrl *)m->shm_base;
    m->ctrl_dev = (Ctrl *)d;
    return VIPER_OK;
}

struct NotifyCtx {
    Ctrl *ctrl;
    std::atomic<uint64_t> *pub;  // pub_state, or pub_m[j] for data-parallel producer j
    uint64_t word;
};

void CUDART_CB notify_fn(void *p) {  // host function: no CUDA calls here
    NotifyCtx *n = (NotifyCtx *)p;
    n->pub->store(n->word);
    n->ctrl->pub_time_ns.store(now_ns());
    n->ctrl->pub_seq.fetch_add(1);
    futex_wake_all(&n->ctrl->pub_seq);
    delete n;
}

struct WakeCtx {
    Ctrl *ctrl;
};

void CUDART_CB wake_fn(void *p) {  // host function: wake sleeping consumers (the word is already set)
    WakeCtx *w = (WakeCtx *)p;
    w->ctrl->pub_time_ns.store(now_ns());
    w->ctrl->pub_seq.fetch_add(1);
    futex_wake_all(&w->ctrl->pub_seq);
    delete w;
}

viper_status open_sa_peers(viper_model *m, const std::vector<PeerRec> &all, const viper_bootstrap *bs) {
    const int N = m->nconsumers_x;
    std::vector<const uint8_t *> src(2 * N), isrc(2 * N);
    std::vector<const volatile uint64_t *> pins(N);
    int j = 0;
    for (int r = 0; r < bs->world; r++) {
        if (all[r].role == VIPER_PRODUCER) continue;
        uint8_t *base;
        if (j == m->cidx) {
            base = (uint8_t *)m->sa_alloc;
        } else {
            CUDA_TRY(cudaIpcOpenMemHandle(&m->sa_peer_base[j], all[r].sa_handle, cudaIpcMemLazyEnablePeerAccess));
            base = (uint8_t *)m->sa_peer_base[j];
        }
        for (int b = 0; b < 2; b++) {
            src[b * N + j] = base + b * m->sa_S;
            isrc[b * N + j] = base + 2 * m->sa_S + b * m->sa_IS;
        }
        pins[j] = (const volatile uint64_t *)&m->ctrl_dev->cons[j].pin;
        j++;
    }
    const size_t bytes = (4 * N + N) * sizeof(void *);
    CUDA_TRY(cudaMalloc(&m->d_sa_tab, bytes));
    std::vector<const void *> tab;
    for (auto p : src) tab.push_back(p);
    for (auto p : isrc) tab.push_back(p);
    for (auto p : pins) tab.push_back((const void *)p);
    CUDA_TRY(cudaMemcpy(m->d_sa_tab, tab.data(), bytes, cudaMemcpyHostToDevice));
    return VIPER_OK;
}

// Data-parallel producers: map every producer's snapshot allocation and
// upload the per-slot tables the install kernel indexes by chunk % M.
viper_status open_producers(viper_model *m, const std::vector<PeerRec> &all, const viper_bootstrap *bs) {
    const int M = m->nprod;
    std::vector<const void *> tab(4 * M);
    for (int j = 0; j < M; j++) {
        const PeerRec &pj = all[bs->producer_rank + j];
        void *base;
        if (j == 0) {
            base = m->peer_snap_base;  // opened above for producer 0
        } else {
            CUDA_TRY(cudaIpcOpenMemHandle(&m->peer_snap_m[j], pj.snap_handle, cudaIpcMemLazyEnablePeerAccess));
            base = m->peer_snap_m[j];
        }
        for (int b = 0; b < 2; b++) {
            tab[b * M + j] = (const uint8_t *)base + pj.snap_off[b];
            tab[2 * M + b * M + j] = (const uint8_t *)base + pj.iseal_off[b];
        }
    }
    CUDA_TRY(cudaMalloc(&m->d_mp_tab, tab.size() * sizeof(void *)));
    CUDA_TRY(cudaMemcpy(m->d_mp_tab, tab.data(), tab.size() * sizeof(void *), cudaMemcpyHostToDevice));
    return VIPER_OK;
}

// Pre-round of the bootstrap: VIPER_TIER_AUTO -> GPU when every consumer's
// GPU reaches every producer's GPU (same GPU or peer access), else DRAM.
// Records of ranks that failed before the bootstrap (magic 0) decide nothing:
// those ranks fail the registration in the next round anyway.
// VIPER_TEST_NO_PEER=1 (tests): this rank reports that it reaches no GPU.
int32_t select_tier_xproc(const viper_model *m, const viper_bootstrap *bs, int M, bool *comm_ok) {
    TierRec me{};
    me.magic = kTierMagic;
    me.tier = m->cfg.tier;
    cudaDeviceGetPCIBusId(me.pci, sizeof me.pci, m->device);
    const char *hook = getenv("VIPER_TEST_NO_PEER");
    if (!(hook && atoi(hook))) {
        memcpy(me.reach[me.nreach++], me.pci, sizeof me.pci);
        int ndev = 0;
        cudaGetDeviceCount(&ndev);
        for (int d = 0; d < ndev && me.nreach < kMaxReach; d++) {
            int can = 0;
            if (d == m->device || cudaDeviceCanAccessPeer(&can, m->device, d) != cudaSuccess || !can) continue;
            cudaDeviceGetPCIBusId(me.reach[me.nreach++], 16, d);
        }
    }
    std::vector<TierRec> all(bs->world);
    *comm_ok = bs->allgather(&me, all.data(), sizeof(TierRec), bs->user) == 0;
    if (!*comm_ok) return m->cfg.tier;
    return resolve_tier(all.data(), bs->world, bs->producer_rank, M, m->cfg.fanout, m->cfg.tier);
}

}  // namespace

viper_status xproc_register(viper_model *m, const viper_tensor *tensors, const viper_bootstrap *bs) {
    if (!bs->allgather) return set_error(VIPER_E_INVAL, "bootstrap.allgather is NULL");
    const int M = bs->nproducers > 1 ? bs->nproducers : 1;
    viper_status bad = VIPER_OK;
    if (bs->rank < 0 || bs->rank >= bs->world || bs->producer_rank < 0 || bs->producer_rank >= bs->world)
        bad = set_error(VIPER_E_INVAL, "bad bootstrap ranks");
    else if (M > kMaxProducers || bs->producer_rank + M > bs->world)
        bad = set_error(VIPER_E_INVAL, "bad nproducers %d", bs->nproducers);
    else if (bs->world - M > kMaxConsumers)
        bad = set_error(VIPER_E_INVAL, "more than %d consumers", kMaxConsumers);
    if (bad) {  // still take part in the bootstrap collectives: the peers fail instead of hanging
        xproc_abort(bs, bad);  // (does not touch the error text)
        return bad;
    }
    bool comm_ok = true;
    m->cfg.tier = select_tier_xproc(m, bs, M, &comm_ok);  // Transfer Selector
    if (!comm_ok) return set_error(VIPER_E_PEER, "bootstrap allgather failed");
    m->rank = bs->rank;
    m->world = bs->world;
    m->nconsumers_x = bs->world - M;
    m->nprod = M;
    const bool producer = m->role == VIPER_PRODUCER;
    const bool is_prod_rank = bs->rank >= bs->producer_rank && bs->rank < bs->producer_rank + M;
    m->pidx = is_prod_rank ? bs->rank - bs->producer_rank : 0;
    const bool dram = m->cfg.tier == VIPER_TIER_DRAM;
    PeerRec me{};
    me.magic = kPeerMagic;
    me.role = m->role;
    me.rank = bs->rank;
    me.device = m->device;
    me.pid = (int32_t)getpid();
    me.tier = m->cfg.tier;
    me.fanout = m->cfg.fanout;
    me.s_packed = m->man.s_packed;
    me.nitems = m->man.items.size();
    me.nchunks = m->man.nchunks;
    me.manifest_hash = manifest_hash(m->man);
    cudaDeviceGetPCIBusId(me.pci, sizeof me.pci, m->device);
    viper_status st = VIPER_OK;
    if (producer != is_prod_rank)
        st = set_error(VIPER_E_INVAL, "rank %d: role does not match bootstrap.producer_rank/nproducers", bs->rank);
    if (st == VIPER_OK && M > 1 && (m->cfg.tier != VIPER_TIER_GPU || m->cfg.fanout != VIPER_FANOUT_DIRECT))
        st = set_error(VIPER_E_UNSUPPORTED, "data-parallel producers: GPU tier, direct fan-out only");
    // VIPER_TEST_NVLS_UNICAST=1 (tests, one consumer): NVLS registration without
    // a multicast object -- the "multicast" address is the consumer's staging,
    // mapped by CUDA IPC, and the producer's snapshot IS that buffer, as its
    // share of the object would be.  On sm_100 multimem.st lowers to the same
    // global store as a unicast one (the multicast is in the address
    // mapping), so this runs pack_nvls_kernel and the consumer's NVLS install
    // path bit for bit, everything but the switch's replication.
    const char *emul_env = getenv("VIPER_TEST_NVLS_UNICAST");
    const bool nvls_emul = m->cfg.fanout == VIPER_FANOUT_NVLS && emul_env && atoi(emul_env);
    const bool nvls = m->cfg.fanout == VIPER_FANOUT_NVLS && !nvls_emul;
    const bool push = m->cfg.fanout == VIPER_FANOUT_PUSH || nvls_emul;
    if (st == VIPER_OK && xproc_only_fanout(m->cfg.fanout) && m->cfg.tier != VIPER_TIER_GPU)
        st = set_error(VIPER_E_UNSUPPORTED, "fan-out %d needs the GPU tier (the Transfer Selector chose DRAM)",
                       m->cfg.fanout);
    if (st == VIPER_OK && push && bs->world - M > kMaxPush)
        st = set_error(VIPER_E_UNSUPPORTED, "push fan-out: at most %d consumers", kMaxPush);
    if (st == VIPER_OK && nvls_emul && bs->world - M != 1)
        st = set_error(VIPER_E_UNSUPPORTED, "VIPER_TEST_NVLS_UNICAST: exactly one consumer");
    if (st == VIPER_OK && nvls && !producer) st = nvls_probe(m->device);  // reported in allgather #1
    const bool nccl = m->cfg.fanout == VIPER_FANOUT_NCCL;
    if (st == VIPER_OK && nccl && producer && m->cfg.mode != VIPER_SYNC)
        st = set_error(VIPER_E_UNSUPPORTED, "NCCL fan-out: SYNC only (broadcasts are a lock-step collective)");
    if (st == VIPER_OK && nccl) st = nccl_probe(producer ? (void *)me.nccl_id : nullptr);  // reported in #1
    const uint64_t S = (m->man.s_packed + 255) / 256 * 256;
    const uint64_t IS = (sizeof(ISeal) * std::max<size_t>(m->man.items.size(), 1) + 255) / 256 * 256;
    const size_t ctrl_bytes = page_up(sizeof(Ctrl));
    if (st == VIPER_OK && producer && m->cfg.flush_dir && M > 1)
        st = set_error(VIPER_E_UNSUPPORTED, "flush with data-parallel producers");
    if (st == VIPER_OK && producer) {
        st = alloc_producer(m, tensors);
        if (st == VIPER_OK && m->cfg.flush_dir) st = flush_start(m, m->cfg.flush_dir);
        const size_t bytes = ctrl_bytes + (dram ? 2 * (S + IS) : 0);
        if (st == VIPER_OK && m->pidx == 0) st = create_segment(m, bytes, me.shm_path, sizeof me.shm_path);
        if (st == VIPER_OK && m->pidx == 0) {
            memset(m->shm_base, 0, ctrl_bytes);
            Ctrl *c = new (m->shm_base) Ctrl();
            c->magic = kCtrlMagic;
            c->ncons.store(bs->world - M);
            c->nprod.store(M);
            c->prod_pid.store((int32_t)getpid());
            st = map_control(m);
        }
        if (st == VIPER_OK) {
            me.shm_bytes = bytes;
            uint8_t *h = (uint8_t *)m->shm_base + ctrl_bytes;
            for (int b = 0; b < 2; b++) {
                me.snap_off[b] = (uint64_t)(m->d_snap[b] - (uint8_t *)m->snap_alloc);
                me.iseal_off[b] = (uint64_t)((uint8_t *)m->d_iseal[b] - (uint8_t *)m->snap_alloc);
                if (dram && m->pidx == 0) {
                    me.stage_off[b] = ctrl_bytes + b * S;
                    me.hiseal_off[b] = ctrl_bytes + 2 * S + b * IS;
                    m->h_stage[b] = h + b * S;
                    m->h_iseal[b] = (ISeal *)(h + 2 * S + b * IS);
                }
            }
            const cudaError_t e = cudaIpcGetMemHandle(&me.snap_handle, m->snap_alloc);
            if (e != cudaSuccess) st = set_error(VIPER_E_CUDA, "cudaIpcGetMemHandle: %s", cudaGetErrorString(e));
        }
        if (st == VIPER_OK && nvls) {  // the multicast object: snapshot + item seals, both slots
            st = nvls_create(m, bs->world, 2 * (S + IS), me.nvls_sock, sizeof me.nvls_sock);
            me.nvls_bytes = m->nvls_bytes;
        }
    }
    // consumers stage what their peers pull from them: the chunks they own
    // (scatter-allgather) or everything (chain)
    const bool sa = m->cfg.fanout == VIPER_FANOUT_SCATTER_ALLGATHER || m->cfg.fanout == VIPER_FANOUT_CHAIN;
    if (st == VIPER_OK && !producer && (sa || push)) {  // push: the producer stores into this staging
        // my staging, double-buffered by snapshot slot
        m->sa_S = S;
        m->sa_IS = IS;
        cudaError_t e = cudaMalloc(&m->sa_alloc, 2 * (S + IS));
        if (e == cudaSuccess) e = cudaMemset(m->sa_alloc, 0, 2 * (S + IS));
        if (e == cudaSuccess) e = cudaIpcGetMemHandle(&me.sa_handle, m->sa_alloc);
        if (e != cudaSuccess) st = set_error(VIPER_E_CUDA, "scatter-allgather staging: %s", cudaGetErrorString(e));
    }
    me.status = st;
    // ---- allgather #1: every rank's record
    std::vector<PeerRec> all(bs->world);
    if (bs->allgather(&me, all.data(), sizeof(PeerRec), bs->user) != 0)
        return set_error(VIPER_E_PEER, "bootstrap allgather failed");
    const PeerRec &pr = all[bs->producer_rank];
    if (st == VIPER_OK) {
        for (int r = 0; r < bs->world; r++) {
            if (all[r].magic != kPeerMagic) st = set_error(VIPER_E_PEER, "rank %d sent a bad record", r);
            else if (all[r].status == VIPER_E_UNSUPPORTED)  // e.g. no multicast on that GPU: same answer everywhere
                st = set_error(VIPER_E_UNSUPPORTED, "rank %d: fan-out %d unsupported there", r, m->cfg.fanout);
            else if (all[r].status != VIPER_OK) st = set_error(VIPER_E_PEER, "rank %d failed to register", r);
            else if (all[r].manifest_hash != me.manifest_hash)
                st = set_error(VIPER_E_INVAL, "rank %d registered a different tensor list", r);
            else if (all[r].tier != me.tier || all[r].fanout != me.fanout)
                st = set_error(VIPER_E_INVAL, "rank %d uses another tier / fan-out", r);
        }
    }
    if (st == VIPER_OK && (nvls || nccl)) {  // NVLS / NCCL: one GPU per rank
        for (int r = 0; r < bs->world && st == VIPER_OK; r++)
            for (int q = r + 1; q < bs->world; q++)
                if (strncmp(all[r].pci, all[q].pci, sizeof me.pci) == 0) {
                    st = set_error(VIPER_E_UNSUPPORTED, "%s: ranks %d and %d share GPU %s", nvls ? "NVLS" : "NCCL",
                                   r, q, all[r].pci);
                    break;
                }
    }
    if (st == VIPER_OK && nvls) st = producer ? nvls_serve(m, bs->world - M) : nvls_join(m, pr.nvls_sock, pr.nvls_bytes);
    {
        // allgather #1b (every rank, every fan-out, so the rounds always match):
        // every GPU joined the multicast object before anyone binds memory
        PeerRec mid{};
        mid.magic = kPeerMagic;
        mid.status = st;
        std::vector<PeerRec> ms(bs->world);
        if (bs->allgather(&mid, ms.data(), sizeof(PeerRec), bs->user) != 0)
            return set_error(VIPER_E_PEER, "bootstrap allgather #1b failed");
        for (int r = 0; r < bs->world && st == VIPER_OK; r++)
            if (ms[r].status != VIPER_OK)
                st = set_error(ms[r].status == VIPER_E_UNSUPPORTED ? VIPER_E_UNSUPPORTED : VIPER_E_PEER,
                               "rank %d failed to register", r);
    }
    if (st == VIPER_OK && nccl) {  // every rank is known to be fine: the collective init cannot strand one
        m->nccl_root = bs->producer_rank;
        st = nccl_init(m, pr.nccl_id, bs->world, bs->rank);
    }
    if (st == VIPER_OK && nvls) {
        st = nvls_bind(m, producer);
        if (st == VIPER_OK) {
            uint8_t *uc = (uint8_t *)m->nvls_uc;
            for (int b = 0; b < 2; b++) {
                ISeal *is = (ISeal *)(uc + 2 * S + b * IS);
                if (producer) {  // the snapshot IS this GPU's share of the multicast object
                    m->d_snap[b] = uc + b * S;
                    m->d_iseal[b] = is;
                    m->nvls_mc_snap[b] = (uint8_t *)m->nvls_va + b * S;
                    m->nvls_mc_iseal[b] = (ISeal *)((uint8_t *)m->nvls_va + 2 * S + b * IS);
                } else {
                    m->stage_src.snap[b] = uc + b * S;
                    m->stage_src.iseal[b] = is;
                }
            }
        }
    }
    if (st == VIPER_OK && producer && push) {  // map every consumer's staging
        int k = 0;
        for (int r = 0; r < bs->world && st == VIPER_OK; r++) {
            if (all[r].role == VIPER_PRODUCER) continue;
            const cudaError_t e =
                cudaIpcOpenMemHandle(&m->push_peer_base[k], all[r].sa_handle, cudaIpcMemLazyEnablePeerAccess);
            if (e != cudaSuccess) {
                st = set_error(VIPER_E_PEER, "push: cudaIpcOpenMemHandle (rank %d): %s", r, cudaGetErrorString(e));
                break;
            }
            for (int b = 0; b < 2; b++) {
                m->push_dst[b][k] = (uint8_t *)m->push_peer_base[k] + b * S;
                m->push_iseal[b][k] = (ISeal *)((uint8_t *)m->push_peer_base[k] + 2 * S + b * IS);
            }
            k++;
        }
        m->npush = k;
        if (nvls_emul && st == VIPER_OK) {  // the snapshot and the "multicast" address: consumer 0's staging
            for (int b = 0; b < 2; b++) {
                m->d_snap[b] = m->nvls_mc_snap[b] = m->push_dst[b][0];
                m->d_iseal[b] = m->nvls_mc_iseal[b] = m->push_iseal[b][0];
            }
            m->npush = 0;
        }
    }
    if (st == VIPER_OK && producer && m->pidx > 0) {  // data-parallel producer j > 0: join the segment
        st = open_segment(m, pr.shm_path, pr.shm_bytes);
        if (st == VIPER_OK) st = map_control(m);
    }
    if (st == VIPER_OK && producer) {
        // every consumer on another GPU: publish v as soon as the pack is
        // launched; consumers pull items as their seals are released (.sys)
        bool other = true;
        for (int r = 0; r < bs->world; r++)
            if (all[r].role != VIPER_PRODUCER && strncmp(all[r].pci, me.pci, sizeof me.pci) == 0) other = false;
        const char *env = getenv("VIPER_EARLY_NOTIFY");
        m->early_notify = env ? atoi(env) != 0 : other;
        // the copy engine and NCCL move a sealed snapshot
        if (m->cfg.fanout == VIPER_FANOUT_CE || m->cfg.fanout == VIPER_FANOUT_NCCL) m->early_notify = false;
        if (m->pidx == 0) m->ctrl->early_notify.store(m->early_notify ? 1 : 0);
    }
    if (st == VIPER_OK && !producer) {
        int idx = 0;
        for (int r = 0; r < bs->rank; r++)
            if (all[r].role != VIPER_PRODUCER) idx++;
        m->cidx = idx;
        m->prod_same_gpu = strncmp(pr.pci, me.pci, sizeof me.pci) == 0;
        st = open_segment(m, pr.shm_path, pr.shm_bytes);
        if (st == VIPER_OK) st = map_control(m);
        if (st == VIPER_OK && m->ctrl->magic != kCtrlMagic) st = set_error(VIPER_E_PEER, "bad control segment");
        if (st == VIPER_OK) {
            m->rec = &m->ctrl->cons[idx];
            m->rec_dev = &m->ctrl_dev->cons[idx];
            const cudaError_t e =
                cudaIpcOpenMemHandle(&m->peer_snap_base, pr.snap_handle, cudaIpcMemLazyEnablePeerAccess);
            if (e != cudaSuccess)
                st = set_error(VIPER_E_PEER, "cudaIpcOpenMemHandle (producer rank %d): %s", bs->producer_rank,
                               cudaGetErrorString(e));
        }
        if (st == VIPER_OK) {
            for (int b = 0; b < 2; b++) {
                m->xsrc.snap[b] = (const uint8_t *)m->peer_snap_base + pr.snap_off[b];
                m->xsrc.iseal[b] = (const ISeal *)((const uint8_t *)m->peer_snap_base + pr.iseal_off[b]);
                if (dram) {
                    m->xsrc.h_stage[b] = (const uint8_t *)m->shm_base + pr.stage_off[b];
                    m->xsrc.h_iseal[b] = (const ISeal *)((const uint8_t *)m->shm_base + pr.hiseal_off[b]);
                }
            }
            st = alloc_consumer(m, tensors);
        }
        if (st == VIPER_OK && sa) st = open_sa_peers(m, all, bs);
        if (st == VIPER_OK && push) {  // install from the staging the producer pushes into
            for (int b = 0; b < 2; b++) {
                m->stage_src.snap[b] = (const uint8_t *)m->sa_alloc + b * S;
                m->stage_src.iseal[b] = (const ISeal *)((const uint8_t *)m->sa_alloc + 2 * S + b * IS);
            }
        }
        if (st == VIPER_OK && M > 1) st = open_producers(m, all, bs);
        if (st == VIPER_OK) {
            m->rec->pid.store((int32_t)getpid());
            m->rec->active.store(1);
        }
    }
    // ---- allgather #2: statuses (all ranks fail together)
    PeerRec fin{};
    fin.magic = kPeerMagic;
    fin.status = st;
    std::vector<PeerRec> sts(bs->world);
    if (bs->allgather(&fin, sts.data(), sizeof(PeerRec), bs->user) != 0)
        return set_error(VIPER_E_PEER, "bootstrap allgather #2 failed");
    if (st != VIPER_OK) return st;
    for (int r = 0; r < bs->world; r++)
        if (sts[r].status != VIPER_OK)
            return set_error(sts[r].status == VIPER_E_UNSUPPORTED ? VIPER_E_UNSUPPORTED : VIPER_E_PEER,
                             "rank %d failed to register", r);
    if (!producer) m->upd = std::thread(update_loop, m);
    return VIPER_OK;
}

void xproc_abort(const viper_bootstrap *bs, viper_status st) {
    {
        TierRec t{};  // the Transfer Selector round (magic 0: decides nothing)
        std::vector<TierRec> tall(bs->world > 0 ? bs->world : 1);
        if (bs->allgather(&t, tall.data(), sizeof(TierRec), bs->user) != 0) return;
    }
    PeerRec me{};
    me.magic = kPeerMagic;
    me.rank = bs->rank;
    me.status = st;
    std::vector<PeerRec> all(bs->world > 0 ? bs->world : 1);
    // allgathers #1, #1b and #2 of xproc_register
    for (int round = 0; round < 3; round++)
        if (bs->allgather(&me, all.data(), sizeof(PeerRec), bs->user) != 0) return;
}

// Consumer update thread (install_mu held, v pinned): pull slot b of the
// producer over the peer mapping (or from the shared DRAM staging).
viper_status xproc_install(viper_model *c, uint64_t v, int b) {
    if (c->nprod > 1) {
        PreparedInstall pi;
        viper_status s = prepare_install(c, c->xsrc, v, b, &pi);
        if (s) return s;
        const int M = c->nprod;
        const void *const *tab = (const void *const *)c->d_mp_tab;
        pi.a.mp_n = (uint32_t)M;
        pi.a.mp_snap = (const uint8_t *const *)(tab + b * M);
        pi.a.mp_iseal = (const ISeal *const *)(tab + 2 * M + b * M);
        return launch_prepared(pi, c->xsrc, b, c->ustream, false, false);
    }
    if (staged_fanout(c->cfg.fanout))  // push / NVLS: the producer wrote into this GPU's staging
        return enqueue_install(c, c->stage_src, v, b, c->ustream, false);
    const bool chain = c->cfg.fanout == VIPER_FANOUT_CHAIN;
    if ((c->cfg.fanout != VIPER_FANOUT_SCATTER_ALLGATHER && !chain) || c->nconsumers_x < 2 ||
        c->cfg.tier != VIPER_TIER_GPU)
        return enqueue_install(c, c->xsrc, v, b, c->ustream, false);
    PreparedInstall pi;
    viper_status s = prepare_install(c, c->xsrc, v, b, &pi);
    if (s) return s;
    const int N = c->nconsumers_x;
    const void *const *tab = (const void *const *)c->d_sa_tab;
    pi.a.sa_n = (uint32_t)N;
    pi.a.sa_me = (uint32_t)c->cidx;
    pi.a.chain = chain ? 1u : 0u;
    pi.a.sa_stage_out = (uint8_t *)c->sa_alloc + b * c->sa_S;
    pi.a.sa_iseal_out = (ISeal *)((uint8_t *)c->sa_alloc + 2 * c->sa_S + b * c->sa_IS);
    pi.a.sa_src = (const uint8_t *const *)(tab + b * N);
    pi.a.sa_isrc = (const ISeal *const *)(tab + 2 * N + b * N);
    pi.a.sa_owner_pin = (const volatile uint64_t *const *)(tab + 4 * N);
    return launch_prepared(pi, c->xsrc, b, c->ustream, false, false);
}

// Producer: name v in pub_state once the pack of slot b completed.  ASYNC:
// a host function on the side stream (enqueued right after the side stream's
// wait on the pack).  SYNC: an event sync, then wait for every consumer.
viper_status xproc_notify(viper_model *p, uint64_t v, int b, bool sync, bool already) {
    Ctrl *ctrl = p->ctrl;
    const uint64_t word = (v << 1) | (uint64_t)b;
    if (!sync) {
        NotifyCtx *n = new NotifyCtx{ctrl, &pub_word(p), word};
        const cudaError_t e = cudaLaunchHostFunc(p->side, notify_fn, n);
        if (e != cudaSuccess) {
            delete n;
            return set_error(VIPER_E_CUDA, "cudaLaunchHostFunc: %s", cudaGetErrorString(e));
        }
        return VIPER_OK;
    }
    if (!already) {
        CUDA_TRY(cudaEventSynchronize(p->ev_packed));
        pub_word(p).store(word);
        ctrl->pub_time_ns.store(now_ns());
        ctrl->pub_seq.fetch_add(1);
        futex_wake_all(&ctrl->pub_seq);
    }
    // SYNC: every active consumer processed v (installed or failed)
    viper_status worst = VIPER_OK;
    const int nc = ctrl->ncons.load();
    for (int i = 0; i < nc; i++) {
        ConsRec *r = &ctrl->cons[i];
        const int64_t t0 = now_ns();
        for (;;) {
            const uint32_t seq = r->done_seq.load();
            if (!r->active.load() || r->done_version.load() >= v) break;
            if (!consumer_alive(r)) {  // its process exited: stop waiting, report it
                if (worst == VIPER_OK) worst = set_error(VIPER_E_PEER, "consumer %d exited", i);
                break;
            }
            if (now_ns() - t0 > 60ll * 1000000000ll)
                return set_error(VIPER_E_TIMEOUT, "consumer %d did not install v%llu", i, (unsigned long long)v);
            if (now_ns() - t0 < 200000) {  // spin first: a futex wake-up costs tens of us
                __builtin_ia32_pause();
                continue;
            }
            r->waiters.fetch_add(1);
            if (r->done_seq.load() == seq && r->done_version.load() < v) futex_wait(&r->done_seq, seq, 1000);
            r->waiters.fetch_sub(1);
        }
        if (r->active.load() && r->done_version.load() == v && r->last_status.load() != VIPER_OK && worst == VIPER_OK)
            worst = set_error(r->last_status.load(), "consumer %d failed to install v%llu", i, (unsigned long long)v);
    }
    return worst;
}

// Early notification (every consumer on another GPU): consumers launch install
// grids that wait per item on the seals the pack releases at system scope, so
// pack, NVLink pull and install overlap.  v is named by a stream memop placed
// right BEFORE the pack: a consumer GPU starts spinning on item seals only
// once the training stream has drained its earlier work and reached the pack,
// not at host enqueue time.  Sleeping update threads are then woken by a host
// function on the side stream (it does not write the word, so a late wake-up
// never names an older version over a newer one).
viper_status xproc_notify_early(viper_model *p, uint64_t v, int b, cudaStream_t st) {
    void *dev_word = p->nprod > 1 ? (void *)&p->ctrl_dev->pub_m[p->pidx] : (void *)&p->ctrl_dev->pub_state;
    viper_status s = stream_write(st, dev_word, (v << 1) | (uint64_t)b);
    if (s) return s;
    CUDA_TRY(cudaEventRecord(p->ev_notify, st));
    CUDA_TRY(cudaStreamWaitEvent(p->side, p->ev_notify, 0));
    WakeCtx *w = new WakeCtx{p->ctrl};
    const cudaError_t e = cudaLaunchHostFunc(p->side, wake_fn, w);
    if (e != cudaSuccess) {
        delete w;
        return set_error(VIPER_E_CUDA, "cudaLaunchHostFunc: %s", cudaGetErrorString(e));
    }
    // ... and wake them from this thread now: when the stream is idle, the
    // memop lands within microseconds, while a host function runs on the CUDA
    // callback thread tens to hundreds of microseconds later
    // (profiles/r02/notify_path.json).  A thread woken before the word lands
    // spins on the word itself (update_loop); the host function above still
    // wakes it if the stream reaches the pack only later.
    p->ctrl->pub_seq.fetch_add(1);
    futex_wake_all(&p->ctrl->pub_seq);
    return VIPER_OK;
}

void xproc_free(viper_model *m) {
    if (m->role == VIPER_PRODUCER && m->ctrl) m->ctrl->closing.store(1);
    for (auto &p : m->sa_peer_base)
        if (p) cudaIpcCloseMemHandle(p), p = nullptr;
    for (auto &p : m->peer_snap_m)
        if (p) cudaIpcCloseMemHandle(p), p = nullptr;
    for (auto &p : m->push_peer_base)
        if (p) cudaIpcCloseMemHandle(p), p = nullptr;
    nvls_free(m);
    nccl_free(m);
    cudaFree(m->d_mp_tab);
    m->d_mp_tab = nullptr;
    cudaFree(m->d_sa_tab);
    cudaFree(m->sa_alloc);
    m->d_sa_tab = m->sa_alloc = nullptr;
    if (m->peer_snap_base) cudaIpcCloseMemHandle(m->peer_snap_base);
    m->peer_snap_base = nullptr;
    if (m->shm_registered) cudaHostUnregister(m->shm_base);
    m->shm_registered = false;
    if (m->shm_base) munmap(m->shm_base, m->shm_bytes);
    m->shm_base = nullptr;
    m->ctrl = nullptr;
    m->rec = nullptr;
    if (m->shm_owner) {
        if (is_posix_shm(m->shm_name.c_str())) shm_unlink(m->shm_name.c_str());
        else unlink(m->shm_name.c_str());
    }
}

}  // namespace vp
