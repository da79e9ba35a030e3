// nccl_fanout.cpp -- VIPER_FANOUT_NCCL: NCCL broadcast as an engine transport,
// the baseline of SURVEY s8(b)/(e) ("NCCL broadcast is timed only as a
// baseline", north_star) run through the SAME seal, install, verify and swap
// as every other fan-out, so it compares like for like with them.
//
// The paper moves models with MPI_Send/Recv (s4.4 P:1689-1696); NCCL is the
// collective-library counterpart on one NVSwitch node.  A broadcast is a
// collective: every rank must issue the same sequence of them.  So this
// fan-out is SYNC only (a SYNC publish returns only after every consumer
// installed v, so consumers see every version, in order: the latest-wins skip
// of ASYNC would desynchronise the sequence) and never early-notified.
//
// Per publish: the producer enqueues, after its pack (and after ev_packed, so
// the notification that lets consumers join does not wait for them), two
// broadcasts rooted at itself -- the packed snapshot, then its item seals.
// Each consumer's update thread, once notified, enqueues the matching two
// broadcasts into its staging and then the usual local install + verify.
//
// libnccl is not linked: it is dlopen'ed ("libnccl.so.2", already loaded in a
// process that imported torch; VIPER_NCCL_LIB overrides) and every failure --
// no library, ranks sharing a GPU (NCCL refuses that), init errors -- becomes
// VIPER_E_UNSUPPORTED on every rank (xproc_register propagates it).
#include <dlfcn.h>
#include <nccl.h>  // types only (/usr/include); the functions come from dlsym

#include <cstring>
#include <mutex>

#include "runtime.h"

namespace vp {

namespace {

struct Nccl {
    ncclResult_t (*getUniqueId)(ncclUniqueId *);
    ncclResult_t (*commInitRank)(ncclComm_t *, int, ncclUniqueId, int);
    ncclResult_t (*broadcast)(const void *, void *, size_t, ncclDataType_t, int, ncclComm_t, cudaStream_t);
    ncclResult_t (*commDestroy)(ncclComm_t);
    const char *(*errorString)(ncclResult_t);
    bool ok = false;
};

Nccl g_nccl;
std::once_flag g_nccl_once;

template <typename F>
bool sym(void *h, const char *name, F *fn) {
    *fn = reinterpret_cast<F>(dlsym(h, name));
    return *fn != nullptr;
}

void load_nccl() {
    const char *env = getenv("VIPER_NCCL_LIB");
    void *h = dlopen(env ? env : "libnccl.so.2", RTLD_NOW | RTLD_GLOBAL);
    if (!h) return;
    Nccl &n = g_nccl;
    n.ok = sym(h, "ncclGetUniqueId", &n.getUniqueId) && sym(h, "ncclCommInitRank", &n.commInitRank) &&
           sym(h, "ncclBroadcast", &n.broadcast) && sym(h, "ncclCommDestroy", &n.commDestroy) &&
           sym(h, "ncclGetErrorString", &n.errorString);
}

viper_status nccl_err(const char *what, ncclResult_t r) {
    return set_error(VIPER_E_UNSUPPORTED, "NCCL fan-out: %s: %s", what, g_nccl.errorString ? g_nccl.errorString(r) : "?");
}

}  // namespace

// The library is usable (producer: and writes a fresh unique id).
viper_status nccl_probe(void *unique_id_out) {
    std::call_once(g_nccl_once, load_nccl);
    if (!g_nccl.ok) return set_error(VIPER_E_UNSUPPORTED, "NCCL fan-out: libnccl.so.2 not loadable (VIPER_NCCL_LIB)");
    if (unique_id_out) {
        const ncclResult_t r = g_nccl.getUniqueId((ncclUniqueId *)unique_id_out);
        if (r != ncclSuccess) return nccl_err("ncclGetUniqueId", r);
    }
    return VIPER_OK;
}

// Every rank, after the records were exchanged (collective over the world).
viper_status nccl_init(viper_model *m, const void *unique_id, int world, int rank) {
    ncclUniqueId id;
    memcpy(&id, unique_id, sizeof id);
    ncclComm_t comm = nullptr;
    const ncclResult_t r = g_nccl.commInitRank(&comm, world, id, rank);
    if (r != ncclSuccess) return nccl_err("ncclCommInitRank", r);
    m->nccl_comm = comm;
    return VIPER_OK;
}

// Both roles: the two broadcasts of one version on `st` (root: the producer's
// rank).  Producer: send = recv = its snapshot / seals; consumer: recv into
// its staging.
viper_status nccl_broadcast_version(viper_model *m, void *snap, void *iseal, int root, cudaStream_t st) {
    ncclComm_t comm = (ncclComm_t)m->nccl_comm;
    ncclResult_t r = g_nccl.broadcast(snap, snap, m->man.s_packed, ncclUint8, root, comm, st);
    if (r == ncclSuccess)
        r = g_nccl.broadcast(iseal, iseal, sizeof(ISeal) * m->man.items.size(), ncclUint8, root, comm, st);
    if (r != ncclSuccess) return set_error(VIPER_E_CUDA, "ncclBroadcast: %s", g_nccl.errorString(r));
    return VIPER_OK;
}

void nccl_free(viper_model *m) {
    if (m->nccl_comm && g_nccl.ok) g_nccl.commDestroy((ncclComm_t)m->nccl_comm);
    m->nccl_comm = nullptr;
}

}  // namespace vp
