// nvls.cpp -- NVSwitch multicast (NVLS) plumbing for VIPER_FANOUT_NVLS
// (SURVEY s8(e) option 1, K5; the paper's GPU-to-GPU channel, s4.4
// P:1677-1696, extended to one producer -> N consumers).
//
// One multicast object spans every rank's GPU.  Each rank binds a buffer of
// its own HBM (the producer: its snapshot; a consumer: its receive staging)
// to the object and maps it unicast; the producer also maps the multicast
// address.  The producer's pack (kernels.cu pack_nvls_kernel) stores every
// 16-B vector once to the multicast address, NVSwitch replicates it into
// every bound buffer, and each consumer installs from its own HBM.
//
// Setup (inside xproc_register, around its allgathers):
//   producer  nvls_create: probe, cuMulticastCreate(numDevices = world),
//             export a POSIX fd, listen on an abstract Unix socket
//   allgather #1 carries the socket name
//   producer  nvls_serve: hand the fd to every consumer (SCM_RIGHTS) and add
//             its own device; consumers nvls_join: receive, import, add device
//   allgather #1b (every rank, every fan-out): all devices are added
//   all       nvls_bind: cuMemCreate + cuMulticastBindMem + unicast map
//             (producer: + the multicast map)
//   allgather #2 (statuses) orders every bind before the first publish.
// Every driver call is resolved through cudaGetDriverEntryPoint (no libcuda
// link), and any failure becomes VIPER_E_UNSUPPORTED with the reason, so a box
// without multicast (no fabric manager, one GPU) reports it instead of failing
// obscurely.
#include <cuda.h>
#include <poll.h>
#include <sys/socket.h>
#include <sys/un.h>
#include <unistd.h>

#include <algorithm>
#include <cstring>
#include <mutex>
#include <random>

#include "runtime.h"

namespace vp {

namespace {

struct Drv {
    CUresult (*devGet)(CUdevice *, int);
    CUresult (*devAttr)(int *, CUdevice_attribute, CUdevice);
    CUresult (*mcCreate)(CUmemGenericAllocationHandle *, const CUmulticastObjectProp *);
    CUresult (*mcAddDevice)(CUmemGenericAllocationHandle, CUdevice);
    CUresult (*mcBindMem)(CUmemGenericAllocationHandle, size_t, CUmemGenericAllocationHandle, size_t, size_t,
                          unsigned long long);
    CUresult (*mcUnbind)(CUmemGenericAllocationHandle, CUdevice, size_t, size_t);
    CUresult (*mcGran)(size_t *, const CUmulticastObjectProp *, CUmulticastGranularity_flags);
    CUresult (*exportFd)(void *, CUmemGenericAllocationHandle, CUmemAllocationHandleType, unsigned long long);
    CUresult (*importFd)(CUmemGenericAllocationHandle *, void *, CUmemAllocationHandleType);
    CUresult (*memCreate)(CUmemGenericAllocationHandle *, size_t, const CUmemAllocationProp *, unsigned long long);
    CUresult (*memRelease)(CUmemGenericAllocationHandle);
    CUresult (*addrReserve)(CUdeviceptr *, size_t, size_t, CUdeviceptr, unsigned long long);
    CUresult (*addrFree)(CUdeviceptr, size_t);
    CUresult (*memMap)(CUdeviceptr, size_t, size_t, CUmemGenericAllocationHandle, unsigned long long);
    CUresult (*memUnmap)(CUdeviceptr, size_t);
    CUresult (*setAccess)(CUdeviceptr, size_t, const CUmemAccessDesc *, size_t);
    CUresult (*allocGran)(size_t *, const CUmemAllocationProp *, CUmemAllocationGranularity_flags);
    bool ok = false;
};

Drv g_drv;
std::once_flag g_drv_once;

template <typename F>
bool resolve(const char *name, F *fn) {
    cudaDriverEntryPointQueryResult q;
    void *p = nullptr;
    if (cudaGetDriverEntryPoint(name, &p, cudaEnableDefault, &q) != cudaSuccess || q != cudaDriverEntryPointSuccess ||
        !p)
        return false;
    *fn = reinterpret_cast<F>(p);
    return true;
}

void load_driver() {
    Drv &d = g_drv;
    d.ok = resolve("cuDeviceGet", &d.devGet) && resolve("cuDeviceGetAttribute", &d.devAttr) &&
           resolve("cuMulticastCreate", &d.mcCreate) && resolve("cuMulticastAddDevice", &d.mcAddDevice) &&
           resolve("cuMulticastBindMem", &d.mcBindMem) && resolve("cuMulticastUnbind", &d.mcUnbind) &&
           resolve("cuMulticastGetGranularity", &d.mcGran) && resolve("cuMemExportToShareableHandle", &d.exportFd) &&
           resolve("cuMemImportFromShareableHandle", &d.importFd) && resolve("cuMemCreate", &d.memCreate) &&
           resolve("cuMemRelease", &d.memRelease) && resolve("cuMemAddressReserve", &d.addrReserve) &&
           resolve("cuMemAddressFree", &d.addrFree) && resolve("cuMemMap", &d.memMap) &&
           resolve("cuMemUnmap", &d.memUnmap) && resolve("cuMemSetAccess", &d.setAccess) &&
           resolve("cuMemGetAllocationGranularity", &d.allocGran);
}

#define DRV_TRY(x)                                                                                            \
    do {                                                                                                      \
        CUresult r_ = (x);                                                                                    \
        if (r_ != CUDA_SUCCESS) return set_error(VIPER_E_UNSUPPORTED, "NVLS: %s failed (CUresult %d)", #x, (int)r_); \
    } while (0)

sockaddr_un sock_addr(const char *name, socklen_t *len) {
    sockaddr_un a{};
    a.sun_family = AF_UNIX;
    a.sun_path[0] = '\0';  // abstract namespace: nothing on the filesystem to clean up
    strncpy(a.sun_path + 1, name, sizeof(a.sun_path) - 2);
    *len = (socklen_t)(offsetof(sockaddr_un, sun_path) + 1 + strlen(name));
    return a;
}

viper_status send_fd(int sock, int fd) {
    char byte = 'F';
    iovec iov{&byte, 1};
    char ctl[CMSG_SPACE(sizeof(int))];
    memset(ctl, 0, sizeof ctl);
    msghdr msg{};
    msg.msg_iov = &iov;
    msg.msg_iovlen = 1;
    msg.msg_control = ctl;
    msg.msg_controllen = sizeof ctl;
    cmsghdr *c = CMSG_FIRSTHDR(&msg);
    c->cmsg_level = SOL_SOCKET;
    c->cmsg_type = SCM_RIGHTS;
    c->cmsg_len = CMSG_LEN(sizeof(int));
    memcpy(CMSG_DATA(c), &fd, sizeof(int));
    if (sendmsg(sock, &msg, 0) != 1) return set_error(VIPER_E_PEER, "NVLS: sendmsg(SCM_RIGHTS) failed");
    return VIPER_OK;
}

viper_status recv_fd(int sock, int *fd) {
    char byte;
    iovec iov{&byte, 1};
    char ctl[CMSG_SPACE(sizeof(int))];
    msghdr msg{};
    msg.msg_iov = &iov;
    msg.msg_iovlen = 1;
    msg.msg_control = ctl;
    msg.msg_controllen = sizeof ctl;
    if (recvmsg(sock, &msg, 0) != 1) return set_error(VIPER_E_PEER, "NVLS: recvmsg failed");
    cmsghdr *c = CMSG_FIRSTHDR(&msg);
    if (!c || c->cmsg_type != SCM_RIGHTS) return set_error(VIPER_E_PEER, "NVLS: no descriptor received");
    memcpy(fd, CMSG_DATA(c), sizeof(int));
    return VIPER_OK;
}

size_t round_up(size_t x, size_t g) { return (x + g - 1) / g * g; }

}  // namespace

// ---- descriptor hand-off (no CUDA): an abstract Unix socket + SCM_RIGHTS.
// fd_listen: a fresh name and a listening socket; fd_serve: hand `fd` to `n`
// fetchers (bounded by timeout_ms per fetcher); fd_fetch: connect (retrying
// until timeout_ns) and receive it.
viper_status fd_listen(char *name, size_t cap, int *listen_fd) {
    std::random_device rd;
    snprintf(name, cap, "viper-nvls-%d-%08x", (int)getpid(), (unsigned)rd());
    const int s = socket(AF_UNIX, SOCK_STREAM | SOCK_CLOEXEC, 0);
    if (s < 0) return set_error(VIPER_E_UNSUPPORTED, "NVLS: socket() failed");
    socklen_t len;
    sockaddr_un a = sock_addr(name, &len);
    if (bind(s, (sockaddr *)&a, len) != 0 || listen(s, 64) != 0) {
        close(s);
        return set_error(VIPER_E_UNSUPPORTED, "NVLS: cannot listen on @%s", name);
    }
    *listen_fd = s;
    return VIPER_OK;
}

viper_status fd_serve(int listen_fd, int fd, int n, int timeout_ms) {
    for (int k = 0; k < n; k++) {
        pollfd p{listen_fd, POLLIN, 0};
        if (poll(&p, 1, timeout_ms) != 1) return set_error(VIPER_E_PEER, "NVLS: fetcher %d did not connect", k);
        const int c = accept(listen_fd, nullptr, nullptr);
        if (c < 0) return set_error(VIPER_E_PEER, "NVLS: accept failed");
        viper_status st = send_fd(c, fd);
        close(c);
        if (st) return st;
    }
    return VIPER_OK;
}

viper_status fd_fetch(const char *name, int *fd, int64_t timeout_ns) {
    socklen_t len;
    sockaddr_un a = sock_addr(name, &len);
    const int64_t t0 = now_ns();
    int s = -1;
    for (;;) {
        s = socket(AF_UNIX, SOCK_STREAM | SOCK_CLOEXEC, 0);
        if (s >= 0 && connect(s, (sockaddr *)&a, len) == 0) break;
        if (s >= 0) close(s);
        s = -1;
        if (now_ns() - t0 > timeout_ns) return set_error(VIPER_E_PEER, "NVLS: cannot reach @%s", name);
        usleep(1000);
    }
    const viper_status st = recv_fd(s, fd);
    close(s);
    return st;
}

viper_status nvls_probe(int device) {
    std::call_once(g_drv_once, load_driver);
    if (!g_drv.ok) return set_error(VIPER_E_UNSUPPORTED, "NVLS: multicast driver entry points unavailable");
    CUdevice d;
    DRV_TRY(g_drv.devGet(&d, device));
    int mc = 0;
    DRV_TRY(g_drv.devAttr(&mc, CU_DEVICE_ATTRIBUTE_MULTICAST_SUPPORTED, d));
    if (!mc) return set_error(VIPER_E_UNSUPPORTED, "NVLS: device %d reports no multicast support", device);
    return VIPER_OK;
}

// Producer: the multicast object for `nranks` GPUs covering `bytes`, exported
// as a POSIX fd, and an abstract Unix socket consumers fetch it from.
viper_status nvls_create(viper_model *m, int nranks, size_t bytes, char *sock_name, size_t cap) {
    viper_status st = nvls_probe(m->device);
    if (st) return st;
    CUmulticastObjectProp mp{};
    mp.numDevices = (unsigned)nranks;
    mp.handleTypes = CU_MEM_HANDLE_TYPE_POSIX_FILE_DESCRIPTOR;
    mp.size = bytes;
    size_t mg = 0, ag = 0;
    DRV_TRY(g_drv.mcGran(&mg, &mp, CU_MULTICAST_GRANULARITY_RECOMMENDED));
    CUmemAllocationProp ap{};
    ap.type = CU_MEM_ALLOCATION_TYPE_PINNED;
    ap.location.type = CU_MEM_LOCATION_TYPE_DEVICE;
    ap.location.id = m->device;
    DRV_TRY(g_drv.allocGran(&ag, &ap, CU_MEM_ALLOC_GRANULARITY_RECOMMENDED));
    const size_t g = std::max<size_t>(std::max<size_t>(mg, ag), 2u << 20);
    m->nvls_bytes = round_up(bytes, g);
    mp.size = m->nvls_bytes;
    CUmemGenericAllocationHandle h;
    DRV_TRY(g_drv.mcCreate(&h, &mp));
    m->nvls_mc = (uint64_t)h;
    m->nvls_have_mc = true;
    int fd = -1;
    DRV_TRY(g_drv.exportFd(&fd, h, CU_MEM_HANDLE_TYPE_POSIX_FILE_DESCRIPTOR, 0));
    m->nvls_fd = fd;
    return fd_listen(sock_name, cap, &m->nvls_listen);
}

// Producer: hand the fd to `nconsumers` connecting consumers, then add its own
// device.  Bounded: a consumer that never connects fails the registration.
viper_status nvls_serve(viper_model *m, int nconsumers) {
    viper_status st = fd_serve(m->nvls_listen, m->nvls_fd, nconsumers, 60000);
    if (st) return st;
    CUdevice d;
    DRV_TRY(g_drv.devGet(&d, m->device));
    DRV_TRY(g_drv.mcAddDevice((CUmemGenericAllocationHandle)m->nvls_mc, d));
    return VIPER_OK;
}

// Consumer: fetch the producer's multicast fd, import it, add this device.
viper_status nvls_join(viper_model *m, const char *sock_name, size_t bytes) {
    viper_status st = nvls_probe(m->device);
    if (st) return st;
    m->nvls_bytes = bytes;
    int fd = -1;
    st = fd_fetch(sock_name, &fd, 60ll * 1000000000ll);
    if (st) return st;
    CUmemGenericAllocationHandle h;
    const CUresult r = g_drv.importFd(&h, (void *)(intptr_t)fd, CU_MEM_HANDLE_TYPE_POSIX_FILE_DESCRIPTOR);
    close(fd);
    if (r != CUDA_SUCCESS) return set_error(VIPER_E_UNSUPPORTED, "NVLS: import of the multicast handle failed (%d)", (int)r);
    m->nvls_mc = (uint64_t)h;
    m->nvls_have_mc = true;
    CUdevice d;
    DRV_TRY(g_drv.devGet(&d, m->device));
    DRV_TRY(g_drv.mcAddDevice(h, d));
    return VIPER_OK;
}

// Every rank, after every device joined: back the object with this GPU's
// memory and map it (unicast; the producer also maps the multicast address).
viper_status nvls_bind(viper_model *m, bool map_mc) {
    CUmemAllocationProp ap{};
    ap.type = CU_MEM_ALLOCATION_TYPE_PINNED;
    ap.location.type = CU_MEM_LOCATION_TYPE_DEVICE;
    ap.location.id = m->device;
    CUmemGenericAllocationHandle phys;
    DRV_TRY(g_drv.memCreate(&phys, m->nvls_bytes, &ap, 0));
    m->nvls_phys = (uint64_t)phys;
    m->nvls_have_phys = true;
    DRV_TRY(g_drv.mcBindMem((CUmemGenericAllocationHandle)m->nvls_mc, 0, phys, 0, m->nvls_bytes, 0));
    m->nvls_bound = true;
    CUmemAccessDesc acc{};
    acc.location.type = CU_MEM_LOCATION_TYPE_DEVICE;
    acc.location.id = m->device;
    acc.flags = CU_MEM_ACCESS_FLAGS_PROT_READWRITE;
    CUdeviceptr uc = 0;
    DRV_TRY(g_drv.addrReserve(&uc, m->nvls_bytes, 0, 0, 0));
    m->nvls_uc = (uint64_t)uc;
    DRV_TRY(g_drv.memMap(uc, m->nvls_bytes, 0, phys, 0));
    m->nvls_uc_mapped = true;
    DRV_TRY(g_drv.setAccess(uc, m->nvls_bytes, &acc, 1));
    if (map_mc) {
        CUdeviceptr mc = 0;
        DRV_TRY(g_drv.addrReserve(&mc, m->nvls_bytes, 0, 0, 0));
        m->nvls_va = (uint64_t)mc;
        DRV_TRY(g_drv.memMap(mc, m->nvls_bytes, 0, (CUmemGenericAllocationHandle)m->nvls_mc, 0));
        m->nvls_mc_mapped = true;
        DRV_TRY(g_drv.setAccess(mc, m->nvls_bytes, &acc, 1));
    }
    // item seals must not show a stale version: start from zero
    if (cudaMemset((void *)uc, 0, m->nvls_bytes) != cudaSuccess)
        return set_error(VIPER_E_CUDA, "NVLS: cudaMemset of the bound buffer failed");
    return VIPER_OK;
}

void nvls_free(viper_model *m) {
    if (!g_drv.ok) return;
    if (m->nvls_mc_mapped) g_drv.memUnmap((CUdeviceptr)m->nvls_va, m->nvls_bytes);
    if (m->nvls_va) g_drv.addrFree((CUdeviceptr)m->nvls_va, m->nvls_bytes);
    if (m->nvls_uc_mapped) g_drv.memUnmap((CUdeviceptr)m->nvls_uc, m->nvls_bytes);
    if (m->nvls_uc) g_drv.addrFree((CUdeviceptr)m->nvls_uc, m->nvls_bytes);
    if (m->nvls_bound) {
        CUdevice d;
        if (g_drv.devGet(&d, m->device) == CUDA_SUCCESS)
            g_drv.mcUnbind((CUmemGenericAllocationHandle)m->nvls_mc, d, 0, m->nvls_bytes);
    }
    if (m->nvls_have_phys) g_drv.memRelease((CUmemGenericAllocationHandle)m->nvls_phys);
    if (m->nvls_have_mc) g_drv.memRelease((CUmemGenericAllocationHandle)m->nvls_mc);
    if (m->nvls_fd >= 0) close(m->nvls_fd);
    if (m->nvls_listen >= 0) close(m->nvls_listen);
    m->nvls_va = m->nvls_uc = 0;
    m->nvls_mc_mapped = m->nvls_uc_mapped = m->nvls_bound = m->nvls_have_phys = m->nvls_have_mc = false;
    m->nvls_fd = m->nvls_listen = -1;
}

}  // namespace vp

// ---- test hooks (include/viper.h): the descriptor hand-off alone, no CUDA
using namespace vp;
extern "C" {
viper_status viper_debug_fd_listen(char *name_out, int32_t cap, int32_t *listen_fd) {
    if (!name_out || cap < 32 || !listen_fd) return set_error(VIPER_E_INVAL, "bad arguments");
    int s = -1;
    const viper_status st = fd_listen(name_out, (size_t)cap, &s);
    *listen_fd = s;
    return st;
}
viper_status viper_debug_fd_serve(int32_t listen_fd, int32_t fd, int32_t n, int32_t timeout_ms) {
    const viper_status st = fd_serve(listen_fd, fd, n, timeout_ms);
    close(listen_fd);
    return st;
}
viper_status viper_debug_fd_fetch(const char *name, int32_t *fd_out, int64_t timeout_ms) {
    if (!name || !fd_out) return set_error(VIPER_E_INVAL, "bad arguments");
    int fd = -1;
    const viper_status st = fd_fetch(name, &fd, timeout_ms * 1000000ll);
    *fd_out = fd;
    return st;
}
}
