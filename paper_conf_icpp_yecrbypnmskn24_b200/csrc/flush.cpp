// flush.cpp -- background flush of published versions to storage, and the
// verified restore that reads them back.
//
// "For fault tolerance, all historical DNN models are flushed to the PFS
// through a background thread to minimize the impact on training"
// (PAPER.md s4.4 P:1789-1800).  Here: after each publish the producer's side
// stream copies the sealed snapshot (packed bytes + item seals + chunk seals)
// into one of two pinned host buffers and a library thread writes it to
// <flush_dir>/<model>.v<version>.viper (write to a temp name, fsync, rename).
// If both buffers are still being written the version is skipped and counted
// (the training stream is never blocked by storage).
//
// viper_restore reads such a file back into caller tensors through the same
// install kernel as a live update: the item seals travel with the data and
// are re-verified on the GPU (VIPER_E_CHECKSUM on any mismatch).
#include <fcntl.h>
#include <sys/stat.h>
#include <unistd.h>

#include <condition_variable>
#include <cstdio>
#include <cstring>
#include <deque>

#include "runtime.h"

namespace vp {

namespace {

struct FlushHeader {
    char magic[8];           // "VIPERCK1"
    uint64_t version, s_packed, nitems, nchunks, chunk_bytes, item_max;
    uint32_t align;
    int32_t ntensors;
};

#define CUDA_TRY(x)                                                                                          \
    do {                                                                                                     \
        cudaError_t e_ = (x);                                                                                \
        if (e_ != cudaSuccess)                                                                               \
            return set_error(VIPER_E_CUDA, "%s failed: %s (%s:%d)", #x, cudaGetErrorString(e_), __FILE__, __LINE__); \
    } while (0)

size_t meta_bytes(const Manifest &m) {
    return sizeof(FlushHeader) + 2 * sizeof(uint64_t) * m.n + sizeof(ISeal) * m.items.size() +
           sizeof(Seal) * m.nchunks;
}

bool write_all(int fd, const void *p, size_t n) {
    const uint8_t *b = (const uint8_t *)p;
    while (n) {
        const ssize_t w = write(fd, b, n);
        if (w <= 0) return false;
        b += w;
        n -= (size_t)w;
    }
    return true;
}

bool read_all(int fd, void *p, size_t n) {
    uint8_t *b = (uint8_t *)p;
    while (n) {
        const ssize_t r = read(fd, b, n);
        if (r <= 0) return false;
        b += r;
        n -= (size_t)r;
    }
    return true;
}

}  // namespace

struct Flusher {
    std::string dir;
    void *host[2] = {nullptr, nullptr};
    size_t bytes = 0;
    std::atomic<int> busy[2];
    std::thread th;
    std::mutex mu;
    std::condition_variable cv;
    std::deque<std::pair<uint64_t, int>> q;
    bool stop = false;
    std::atomic<uint64_t> flushed{0}, skipped{0}, last{0};
};

struct FlushCb {
    Flusher *f;
    uint64_t v;
    int k;
};

static void CUDART_CB flush_ready(void *p) {  // host function: queue only
    FlushCb *c = (FlushCb *)p;
    {
        std::lock_guard<std::mutex> lk(c->f->mu);
        c->f->q.emplace_back(c->v, c->k);
    }
    c->f->cv.notify_one();
    delete c;
}

static void flush_loop(viper_model *m, Flusher *f) {
    for (;;) {
        std::pair<uint64_t, int> job;
        {
            std::unique_lock<std::mutex> lk(f->mu);
            f->cv.wait(lk, [&] { return f->stop || !f->q.empty(); });
            if (f->q.empty()) return;  // stop requested and drained
            job = f->q.front();
            f->q.pop_front();
        }
        char name[1024], tmp[1100];
        snprintf(name, sizeof name, "%s/%s.v%020llu.viper", f->dir.c_str(), m->name.c_str(),
                 (unsigned long long)job.first);
        snprintf(tmp, sizeof tmp, "%s.tmp", name);
        const int fd = open(tmp, O_CREAT | O_TRUNC | O_WRONLY, 0644);
        bool ok = fd >= 0 && write_all(fd, f->host[job.second], f->bytes) && fsync(fd) == 0;
        if (fd >= 0) close(fd);
        ok = ok && rename(tmp, name) == 0;
        if (ok) {
            f->flushed.fetch_add(1);
            f->last.store(job.first);
        } else {
            unlink(tmp);
            f->skipped.fetch_add(1);
        }
        f->busy[job.second].store(0);
    }
}

viper_status flush_start(viper_model *m, const char *dir) {
    struct stat sb;
    if (stat(dir, &sb) != 0 || !S_ISDIR(sb.st_mode)) return set_error(VIPER_E_INVAL, "flush_dir '%s' is not a directory", dir);
    Flusher *f = new Flusher();
    f->dir = dir;
    f->bytes = meta_bytes(m->man) + m->man.s_packed;
    for (int k = 0; k < 2; k++) {
        f->busy[k].store(0);
        if (cudaHostAlloc(&f->host[k], f->bytes, cudaHostAllocPortable) != cudaSuccess) {
            for (int j = 0; j < k; j++) cudaFreeHost(f->host[j]);
            delete f;
            return set_error(VIPER_E_NOMEM, "flush buffers (%zu B)", f->bytes);
        }
    }
    f->th = std::thread(flush_loop, m, f);
    m->flusher = f;
    return VIPER_OK;
}

// Producer, side stream, after the chunk-seal reduction of version v in slot b.
viper_status flush_enqueue(viper_model *p, uint64_t v, int b) {
    Flusher *f = p->flusher;
    int k = -1;
    for (int j = 0; j < 2 && k < 0; j++) {
        int zero = 0;
        if (f->busy[j].compare_exchange_strong(zero, 1)) k = j;
    }
    if (k < 0) {  // storage is behind: skip this version, never stall training
        f->skipped.fetch_add(1);
        return VIPER_OK;
    }
    const Manifest &m = p->man;
    uint8_t *h = (uint8_t *)f->host[k];
    FlushHeader hd{};
    memcpy(hd.magic, "VIPERCK1", 8);
    hd.version = v;
    hd.s_packed = m.s_packed;
    hd.nitems = m.items.size();
    hd.nchunks = m.nchunks;
    hd.chunk_bytes = m.chunk_bytes;
    hd.item_max = m.item_max;
    hd.align = m.align;
    hd.ntensors = m.n;
    size_t o = 0;
    memcpy(h + o, &hd, sizeof hd);
    o += sizeof hd;
    memcpy(h + o, m.nbytes.data(), sizeof(uint64_t) * m.n);
    o += sizeof(uint64_t) * m.n;
    memcpy(h + o, m.offsets.data(), sizeof(uint64_t) * m.n);
    o += sizeof(uint64_t) * m.n;
    CUDA_TRY(cudaMemcpyAsync(h + o, p->d_iseal[b], sizeof(ISeal) * m.items.size(), cudaMemcpyDeviceToHost, p->side));
    o += sizeof(ISeal) * m.items.size();
    CUDA_TRY(cudaMemcpyAsync(h + o, p->d_seal[b], sizeof(Seal) * m.nchunks, cudaMemcpyDeviceToHost, p->side));
    o += sizeof(Seal) * m.nchunks;
    CUDA_TRY(cudaMemcpyAsync(h + o, p->d_snap[b], m.s_packed, cudaMemcpyDeviceToHost, p->side));
    FlushCb *cb = new FlushCb{f, v, k};
    const cudaError_t e = cudaLaunchHostFunc(p->side, flush_ready, cb);
    if (e != cudaSuccess) {
        delete cb;
        f->busy[k].store(0);
        return set_error(VIPER_E_CUDA, "cudaLaunchHostFunc: %s", cudaGetErrorString(e));
    }
    return VIPER_OK;
}

void flush_stop(viper_model *m) {
    Flusher *f = m->flusher;
    if (!f) return;
    if (m->side) cudaStreamSynchronize(m->side);  // every queued copy + callback has run
    {
        std::lock_guard<std::mutex> lk(f->mu);
        f->stop = true;
    }
    f->cv.notify_all();
    f->th.join();
    for (auto h : f->host) cudaFreeHost(h);
    delete f;
    m->flusher = nullptr;
}

void flush_stats(viper_model *m, uint64_t *flushed, uint64_t *skipped, uint64_t *last) {
    Flusher *f = m->flusher;
    *flushed = f ? f->flushed.load() : 0;
    *skipped = f ? f->skipped.load() : 0;
    *last = f ? f->last.load() : 0;
}

}  // namespace vp

using namespace vp;

extern "C" viper_status viper_restore(const char *path, const viper_tensor *tensors, int32_t n, int32_t device,
                                      void *cuda_stream, uint64_t *version_out) {
    if (!path || (n > 0 && !tensors) || n < 0) return set_error(VIPER_E_INVAL, "bad arguments");
    const int fd = open(path, O_RDONLY);
    if (fd < 0) return set_error(VIPER_E_INVAL, "cannot open %s", path);
    FlushHeader hd{};
    std::vector<uint64_t> nb, off;
    bool ok = read_all(fd, &hd, sizeof hd) && memcmp(hd.magic, "VIPERCK1", 8) == 0 && hd.ntensors == n;
    if (ok) {
        nb.resize(n);
        off.resize(n);
        ok = read_all(fd, nb.data(), sizeof(uint64_t) * n) && read_all(fd, off.data(), sizeof(uint64_t) * n);
    }
    for (int32_t i = 0; ok && i < n; i++) ok = nb[i] == tensors[i].nbytes;
    if (!ok) {
        close(fd);
        return set_error(VIPER_E_INVAL, "%s: not a checkpoint of these %d tensors", path, n);
    }
    DeviceGuard dg(device);
    if (dg.err != cudaSuccess) {
        close(fd);
        return set_error(VIPER_E_CUDA, "cudaSetDevice(%d)", device);
    }
    Manifest man;
    viper_status st = build_manifest(man, tensors, n, hd.chunk_bytes, hd.align, device, hd.item_max);
    if (st == VIPER_OK && (man.items.size() != hd.nitems || man.nchunks != hd.nchunks || man.s_packed != hd.s_packed))
        st = set_error(VIPER_E_INVAL, "%s: layout does not match", path);
    void *host = nullptr, *dev = nullptr, *flags = nullptr, *status_host = nullptr;
    Item *items = nullptr;
    const size_t IS = sizeof(ISeal) * hd.nitems, CS = sizeof(Seal) * hd.nchunks;
    const size_t bytes = IS + CS + hd.s_packed;
    if (st == VIPER_OK && cudaHostAlloc(&host, bytes, cudaHostAllocDefault) != cudaSuccess)
        st = set_error(VIPER_E_NOMEM, "pinned staging %zu B", bytes);
    if (st == VIPER_OK && !read_all(fd, host, bytes)) st = set_error(VIPER_E_INVAL, "%s: truncated", path);
    close(fd);
    cudaStream_t s = (cudaStream_t)cuda_stream;
    if (st == VIPER_OK && (cudaMalloc(&dev, IS + hd.s_packed + 16) != cudaSuccess ||
                           cudaMalloc(&flags, 64) != cudaSuccess ||
                           cudaHostAlloc(&status_host, 64, cudaHostAllocMapped) != cudaSuccess))
        st = set_error(VIPER_E_NOMEM, "restore buffers");
    if (st == VIPER_OK) {
        std::vector<void *> ptrs(n);
        for (int32_t i = 0; i < n; i++) ptrs[i] = tensors[i].dev_ptr;
        st = upload_items(man, ptrs, &items, 1, 0, nullptr);
    }
    if (st == VIPER_OK) {
        uint8_t *d = (uint8_t *)dev;
        volatile int32_t *sh = (volatile int32_t *)status_host;
        *sh = 1;
        void *sh_dev = nullptr;
        cudaError_t e = cudaHostGetDevicePointer(&sh_dev, status_host, 0);
        if (e == cudaSuccess) e = cudaMemsetAsync(flags, 0, 64, s);
        if (e == cudaSuccess) e = cudaMemcpyAsync(d, host, IS, cudaMemcpyHostToDevice, s);
        if (e == cudaSuccess) e = cudaMemcpyAsync(d + IS, (uint8_t *)host + IS + CS, hd.s_packed, cudaMemcpyHostToDevice, s);
        if (e == cudaSuccess) {
            InstallArgs a{};
            a.items = items;
            a.nitems = (uint32_t)man.items.size();
            a.packed = d + IS;
            a.iseal = (const ISeal *)d;
            a.version = hd.version;
            a.fault_item = ~0u;
            a.flags = (unsigned long long *)flags;
            a.ctr = (unsigned int *)((uint8_t *)flags + 8);  // zeroed above
            a.status_h = (volatile int32_t *)sh_dev;
            e = launch_install(a, pick_geometry(a.nitems, device), s, false);
        }
        if (e == cudaSuccess) e = cudaStreamSynchronize(s);
        if (e != cudaSuccess) st = set_error(VIPER_E_CUDA, "restore: %s", cudaGetErrorString(e));
        else if (*sh != VIPER_OK) st = set_error(*sh, "%s: seal verification failed", path);
    }
    cudaFree(items);
    cudaFree(man.d_chunk_first);
    cudaFree(dev);
    cudaFree(flags);
    if (status_host) cudaFreeHost(status_host);
    if (host) cudaFreeHost(host);
    if (st == VIPER_OK && version_out) *version_out = hd.version;
    return st;
}
