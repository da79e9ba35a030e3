/*
 * viper.h -- C-ABI of libviper.so, the B200-native model-update hot path of
 * Viper's memory-first model transfer engine (Ye et al., ICPP '24).
 *
 * Citations are PAPER.md line ranges ("P:a-b") plus the section they sit in.
 * The paper's API (Fig. 4; s4.1 P:859-878) is a Python
 * `init(type)`, `save_weights(model_name, model_weights)` and
 * `load_weights(model_name) -> model_weights`; this ABI is that API made
 * explicit for one process per GPU:
 *
 *   init(type) + "create subscriptions if consumer"  -> viper_register_model
 *   save_weights                                      -> viper_publish
 *   push notification (s4.4 P:1802-1820)              -> viper_subscribe
 *   load_weights + double buffering (s4.2 P:1214-1227)-> viper_acquire_latest /
 *                                                        viper_release
 *   Inference Performance Predictor (s4.3)            -> viper_schedule
 *
 * Conventions (all calls):
 *   - Every call returns a viper_status: 0 = OK, < 0 = error.  No C++
 *     exception, abort or exit ever crosses the ABI.  viper_last_error()
 *     returns a thread-local human-readable detail for the last failure.
 *   - Pointers named dev_* are CUDA device pointers on cfg->device; all other
 *     pointers are host pointers.  Sizes are bytes unless stated.
 *   - `cuda_stream` arguments are cudaStream_t values passed as void*
 *     (NULL = the legacy default stream).
 *   - There is no CPU fallback: without a usable sm_100 device every call
 *     that needs the GPU returns VIPER_E_CUDA.
 *   - A call that works on the model's GPU switches to it and restores the
 *     calling thread's current CUDA device before it returns.
 */
#ifndef VIPER_H
#define VIPER_H

#include <stddef.h>
#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

typedef int32_t viper_status;
enum {
    VIPER_OK = 0,
    VIPER_E_INVAL = -1,       /* bad argument / descriptor / size                   */
    VIPER_E_NOMEM = -2,       /* device, pinned or shared memory allocation failed  */
    VIPER_E_CUDA = -3,        /* a CUDA call failed (detail in viper_last_error)    */
    VIPER_E_VERSION = -4,     /* publish(v) with v <= last published (v starts at 1)*/
    VIPER_E_CHECKSUM = -5,    /* a sealed chunk failed verification: v NOT installed,
                                 the previous version keeps serving                 */
    VIPER_E_TIMEOUT = -6,     /* a bounded wait expired                             */
    VIPER_E_NOVERSION = -7,   /* nothing (>= min_version) installed yet             */
    VIPER_E_STATE = -8,       /* wrong role, double release, unknown view, closed   */
    VIPER_E_UNSUPPORTED = -9, /* transport not available on this box / in this mode */
    VIPER_E_PEER = -10        /* peer process or GPU unreachable during bootstrap   */
};

typedef enum { VIPER_PRODUCER = 1, VIPER_CONSUMER = 2 } viper_role;

/* Element type of a tensor.  The path is dtype-agnostic: bytes are moved and
 * checksummed, never interpreted; the dtype is recorded in the manifest. */
typedef enum { VIPER_F32 = 0, VIPER_BF16 = 1, VIPER_F16 = 2, VIPER_BYTES = 3 } viper_dtype;

/* One contiguous parameter tensor ("model parameters (weights, biases)",
 * s2 P:426-431).  dev_ptr must stay allocated and shape-stable until
 * viper_unregister.  nbytes may be 0.  16-byte aligned dev_ptr takes the
 * vectorised path; other alignments are legal but slower. */
typedef struct {
    const char *name;      /* may be NULL */
    int32_t dtype;         /* viper_dtype */
    int32_t ndim;
    const int64_t *shape;  /* ndim entries, may be NULL when ndim == 0 */
    void *dev_ptr;
    uint64_t nbytes;
} viper_tensor;

/* Cross-process bootstrap (one process per GPU).  `allgather` must gather
 * `nbytes` from every rank into out[rank * nbytes] (e.g. a torch.distributed
 * all_gather on the bootstrap process group).  Pass NULL to viper_register_model
 * for an in-process channel: producer and consumers of the same model name in
 * the same process find each other by name (single-GPU loopback and tests). */
typedef struct {
    int32_t rank, world, producer_rank;
    int (*allgather)(const void *in, void *out, size_t nbytes, void *user);
    void *user;
    /* Data-parallel producers ("multiple producers running
     * data-parallel training"): ranks producer_rank ..
     * producer_rank + nproducers - 1 are producers holding identical replicas;
     * each publishes the same versions and packs only the chunks c with
     * c % nproducers == its index, consumers pull every chunk from its owner.
     * 0 or 1 = a single producer.  GPU tier, direct fan-out only. */
    int32_t nproducers;
} viper_bootstrap;

/* Storage tier (s4.4 P:1671-1720, Fig. 7). */
enum { VIPER_TIER_GPU = 0,   /* GPU-to-GPU memory: pull over NVLink peer mapping */
       VIPER_TIER_DRAM = 1,  /* Host-to-Host memory: staged through pinned DRAM  */
       VIPER_TIER_AUTO = 2 }; /* Transfer Selector (Fig. 7): decided
                                once at registration, the same on every endpoint.
                                Cross-process: the GPU tier when every consumer's
                                GPU can peer-access every producer's GPU (and,
                                with chain / scatter-allgather fan-out, every
                                other consumer's; or is the same GPU), else the
                                DRAM tier; every rank
                                must then ask for AUTO.  In process: the tier of
                                the model's existing endpoints, else the GPU tier
                                when this GPU can peer-access every visible GPU
                                (or is the only one).  viper_stats.tier reports
                                the choice. */
/* Fan-out of one producer to N consumers. */
enum { VIPER_FANOUT_DIRECT = 0,        /* every consumer pulls every chunk from the producer */
       VIPER_FANOUT_CHAIN = 1,         /* pipelined chain: consumer i pulls every item from
                                          consumer i-1 (consumer 0 from the producer) as
                                          soon as that item is sealed there, and stages it
                                          for consumer i+1.  Producer egress S; bound
                                          S/link + (N-1) items (SURVEY s8(e) option 3) */
       VIPER_FANOUT_SCATTER_ALLGATHER = 2, /* consumer i pulls chunks c = i (mod N) from the
                                             producer, the rest from its peers */
       VIPER_FANOUT_NVLS = 3,          /* NVSwitch multicast (SURVEY s8(e) option 1): every
                                          rank binds a staging buffer to one multicast
                                          object; the producer's pack stores each item
                                          once into the multicast address
                                          (multimem.st), the switch replicates it to every
                                          consumer, and each consumer installs from its own
                                          HBM.  Producer egress S.  Needs a GPU tier, one
                                          GPU per rank and cuMulticastCreate support
                                          (fabric manager); otherwise registration returns
                                          VIPER_E_UNSUPPORTED on every rank */
       VIPER_FANOUT_PUSH = 4,          /* push (SURVEY K3 deliver_push): the producer's
                                          pack stores every item into each consumer's
                                          peer-mapped staging as well as its snapshot
                                          (producer egress N x S, at most 8 consumers);
                                          consumers install from local HBM, item by item
                                          as the producer releases the item seals */
       VIPER_FANOUT_NCCL = 100,        /* baseline as an engine transport: after
                                          its pack the producer broadcasts the sealed snapshot
                                          and its item seals with NCCL (libnccl.so.2,
                                          dlopen'ed; VIPER_NCCL_LIB overrides); each consumer
                                          receives them into its staging and installs +
                                          verifies locally.  SYNC only (a broadcast is a
                                          lock-step collective), one GPU per rank; otherwise
                                          registration returns VIPER_E_UNSUPPORTED on every
                                          rank */
       VIPER_FANOUT_CE = 101           /* baseline: each consumer's update
                                          thread copies the sealed snapshot with the copy
                                          engine (cudaMemcpyAsync peer -> local staging)
                                          once the pack completed, then installs locally */
};
/* NVLS, PUSH, NCCL and CE are cross-process fan-outs (viper_bootstrap != NULL,
 * GPU tier, one producer); in process they return VIPER_E_UNSUPPORTED. */
/* Save mode (Fig. 3; s5.3 P:2143-2153). */
enum { VIPER_SYNC = 0,   /* publish returns after every consumer installed v (or failed) */
       VIPER_ASYNC = 1 };/* publish returns once the snapshot is enqueued on cuda_stream;
                            delivery and install proceed in the background       */

/* Flags (viper_config.flags). */
enum { VIPER_FLAG_TIMING = 2,   /* record CUDA events around the pack / install /
                                   fused kernels on their launch streams; the
                                   device times appear in viper_stats (bench.py) */
       VIPER_FLAG_NO_FUSE = 4,  /* producer: never use the fused SYNC kernel
                                   (pack and install as separate kernels)        */
       VIPER_FLAG_TMA = 8,      /* producer: pack with TMA bulk copies (implies
                                   NO_FUSE); consumer: install with TMA bulk copies
                                   (cp.async.bulk global<->shared) instead of 128-bit
                                   register streaming.  Without the flag TMA is
                                   picked automatically for models <= 1 GiB where it
                                   applies: packs no install is PDL-chained to
                                   (ASYNC, DRAM tier, cross-process) and direct
                                   installs of a completed snapshot               */
       VIPER_FLAG_NO_TMA = 16,  /* never auto-select the TMA kernels (the fused
                                   SYNC kernel streams through registers)         */
       VIPER_FLAG_FUSED_TMA = 32 }; /* producer: the fused SYNC kernel moves every
                                   16-B-aligned item with TMA bulk copies (one
                                   shared-memory stage stored into the snapshot
                                   and every consumer slot) and verifies the
                                   installed slot bytes by reading them back.
                                   Never auto-selected: it measured slower than
                                   the register fused kernel       */

typedef struct {
    int32_t tier;            /* VIPER_TIER_*                       (default GPU)    */
    int32_t fanout;          /* VIPER_FANOUT_*                     (default DIRECT) */
    int32_t mode;            /* VIPER_SYNC / VIPER_ASYNC           (default SYNC)   */
    uint64_t chunk_bytes;    /* seal granularity, multiple of 256 (0 -> 2 MiB)      */
    uint32_t align;          /* packed-layout alignment, power of 2 >= 16 (0 -> 256)*/
    int32_t device;          /* CUDA device ordinal of this process's GPU          */
    const viper_tensor *slot1; /* consumer: optional caller-owned second replica
                                  (same n, nbytes); NULL -> library allocates it  */
    int32_t flags;           /* VIPER_FLAG_*                                        */
    const char *flush_dir;   /* producer: background flush of every published version
                                to <flush_dir>/<model>.v<version>.viper ("all
                                historical DNN models are flushed ... through a
                                background thread").  Pinned double
                                buffer; a version is skipped (counted) when storage
                                is behind.  NULL = off.  Not with nproducers > 1.  */
    int32_t install_sms;     /* consumer: run its install kernel on at most this many SMs
                                (0 = all).  Bounds an update's share of the GPU while the
                                replica serves ("inference continues"): the
                                install takes longer, the other SMs stay with inference.
                                Applies to the consumer's own install kernel (ASYNC, DRAM
                                tier, cross-process), not to a SYNC in-process publish,
                                which installs inside the producer's fused kernel.     */
} viper_config;

typedef struct viper_model viper_model; /* opaque */

/* A pinned, immutable view of one installed version. */
typedef struct {
    uint64_t version;
    int32_t slot;            /* 0 = caller's tensors, 1 = the alternative copy */
    int32_t ntensors;
    void *const *dev_ptrs;   /* ntensors device pointers, library-owned, valid until
                                viper_release; readers must not write through them */
    uint64_t ticket;         /* opaque, checked by viper_release */
} viper_view;

/*
 * viper_register_model -- "init(type)" (s4.1 P:859-878) + the manifest the
 * Metadata DB holds {name, version, size, location}.
 *
 * Producer: `tensors` are the training replica's parameters (read-only to the
 * library).  Consumer: `tensors` are slot 0 of the inference replica (the
 * library writes them only while inactive and unpinned); cfg->slot1 or a
 * library allocation is slot 1.  Every participant must pass the same tensor
 * count and sizes in the same order (checked: VIPER_E_INVAL).
 *
 * Layout (R16): tensors keep registration order, offsets are
 * aligned to cfg->align, padding is zero, S_packed = align_up(end, align).
 * Library-owned: snapshot buffers (2 x S_packed on the producer), seals,
 * staging, flags, pinned host buffers, slot 1 (if not supplied).
 *
 * In-process (bs == NULL): the producer and its consumers must be on the same
 * device; consumers registered before a publish receive it.  Cross-process
 * (bs != NULL): collective over all bs->world ranks; rank bs->producer_rank
 * passes VIPER_PRODUCER, the others VIPER_CONSUMER.
 *
 * Returns VIPER_E_INVAL (bad args, size mismatch), VIPER_E_NOMEM,
 * VIPER_E_CUDA, VIPER_E_PEER (bootstrap failed), VIPER_E_UNSUPPORTED.
 */
viper_status viper_register_model(const char *model_name, int32_t role, const viper_tensor *tensors,
                                  int32_t n, const viper_config *cfg, const viper_bootstrap *bs,
                                  viper_model **out);

/*
 * viper_publish -- "save_weights" (Fig. 4; s4.2 P:1183-1200).
 * Producer only.  Snapshots the tensors (pack + per-chunk seal {version, cks},
 * DESIGN.md K2) on `cuda_stream`, after the caller's prior work on it, then
 * notifies subscribers (s4.4 P:1802-1812).  Versions strictly increase and
 * start at 1 (else VIPER_E_VERSION).  Only the latest version is buffered
 * (P:1786-1789): a slow consumer may skip versions, never go backwards.
 * SYNC: returns after every consumer installed v (or reports its failure,
 * e.g. VIPER_E_CHECKSUM).  ASYNC: returns after enqueueing; the caller may
 * modify its tensors once `cuda_stream` has passed this call.
 */
viper_status viper_publish(viper_model *m, uint64_t version, void *cuda_stream);

/*
 * viper_subscribe -- consumer only: "create subscriptions",
 * "proactively informing consumers of model updates".
 * on_update(version, status, user) runs on the library's update thread after
 * each install attempt (status VIPER_OK or an error); it must not block.
 * Pass NULL to remove.  Installs happen with or without a subscription.
 */
viper_status viper_subscribe(viper_model *m, void (*on_update)(uint64_t version, viper_status st, void *user),
                             void *user);

/*
 * viper_acquire_latest -- consumer only: pin the newest installed version
 * ("serve incoming inference queries with the latest model").
 * Waits up to timeout_us (0 = do not wait, <0 = forever) for a version >=
 * min_version.  The pinned slot is never written until viper_release.
 * Thread-safe.  VIPER_E_NOVERSION (timeout 0) / VIPER_E_TIMEOUT.
 */
viper_status viper_acquire_latest(viper_model *m, uint64_t min_version, int64_t timeout_us, viper_view *out);

/*
 * viper_release -- unpin a view.  cuda_stream != NULL: the unpin is enqueued
 * after the work already on that stream (readers launched kernels on the
 * slot).  Double release / unknown ticket -> VIPER_E_STATE.
 */
viper_status viper_release(viper_model *m, const viper_view *view, void *cuda_stream);

/* Wait until this consumer has installed a version >= v (or timeout). */
viper_status viper_wait_installed(viper_model *m, uint64_t v, int64_t timeout_us);

/* Statistics of the last update seen by this endpoint (all fields 0 if none). */
typedef struct {
    uint64_t version;          /* last version published (producer) / installed (consumer) */
    uint64_t s_packed;         /* packed bytes                                        */
    uint64_t nchunks, nitems;  /* seal chunks, warp work items                        */
    uint64_t installs, skipped, failures;  /* consumer counters                        */
    double t_publish_us;       /* producer: host time inside the last viper_publish   */
    double t_install_us;       /* consumer: host time of the last install (launch->done)*/
    double t_notify_us;        /* consumer: publish -> update-thread pickup            */
    double writer_wait_us;     /* consumer: time waiting for readers to leave a slot  */
    double t_pack_dev_us;      /* producer, VIPER_FLAG_TIMING: last pack_seal kernel (CUDA events) */
    double t_install_dev_us;   /* consumer, VIPER_FLAG_TIMING: last install_verify kernel          */
    double t_fused_dev_us;     /* producer, VIPER_FLAG_TIMING: last publish_fused kernel (SYNC,
                                  in-process: pack + install + verify + swap in one launch)     */
    int32_t last_status;
    int32_t nconsumers;
    uint64_t flushed, flush_skipped, flush_last;  /* producer with flush_dir        */
    int32_t tier;              /* tier in use (VIPER_TIER_AUTO resolved)               */
    int32_t fanout;            /* fan-out in use                                       */
    double t_pickup_us;        /* consumer: producer's viper_publish entry -> this update
                                  thread picked the version up (host CLOCK_MONOTONIC, shared by
                                  every process on the node)                           */
} viper_stats;
viper_status viper_get_stats(viper_model *m, viper_stats *out);

/* Layout queries (for tests / tooling): packed size, per-tensor offsets
 * (offsets may be NULL).  viper_debug_buffers: producer -> device pointers of
 * the most recent snapshot and of its chunk seals (2 x uint64 {version, cks}
 * per chunk, R16; waits until they are reduced); consumer -> its
 * DRAM-tier staging buffer (NULL on the GPU tier) and NULL seals. */
viper_status viper_layout(viper_model *m, uint64_t *s_packed, uint64_t *offsets, int32_t n);
viper_status viper_debug_buffers(viper_model *m, void **dev_packed, void **dev_seals, uint64_t *nchunks);

/*
 * viper_view_seals -- consumer: the chunk seals of a pinned view, computed on
 * the device from the installed slot tensors as they sit (no copy).  Output:
 * nchunks x {uint64 version = view->version, uint64 cks} in dev_seals_out, a
 * caller-owned device buffer of >= 16 * nchunks bytes on the model's device,
 * written in stream order on cuda_stream (the caller synchronises before
 * reading it).  cks is the CKS of DESIGN.md R16 over the packed layout (LAY,
 * zero padding), i.e. the value the producer sealed chunk c with, so equality
 * with the producer's (or the oracle's) chunk seals proves the replica
 * byte-exact up to the checksum's guarantees ("the updated model ... replaces
 * the previous model", s4.2 P:1208-1227).  The view must stay pinned until the
 * stream passes the call.  VIPER_E_STATE: producer / unknown view.
 */
viper_status viper_view_seals(viper_model *m, const viper_view *view, void *dev_seals_out, void *cuda_stream);

/* Test hook (T4 fault injection): the consumer's next install flips one
 * staged bit before verification -> VIPER_E_CHECKSUM, version not installed. */
viper_status viper_debug_fault_next(viper_model *m);

/*
 * viper_restore -- read a flushed version back (fault tolerance / resume).
 * Copies the file's packed snapshot to the GPU and installs it into
 * `tensors` (device pointers on `device`) with the install kernel, which
 * re-verifies every item seal: VIPER_E_CHECKSUM if the file was corrupted,
 * VIPER_E_INVAL if it does not describe these n tensors.  Synchronous on
 * cuda_stream; *version_out receives the file's version.
 */
viper_status viper_restore(const char *path, const viper_tensor *tensors, int32_t n, int32_t device,
                           void *cuda_stream, uint64_t *version_out);

/* Test hooks: the CUDA-free version protocol (protocol.h) over a POSIX shm
 * segment of `words` u64 per slot, for multi-process CPU tests.  publish(v)
 * fills snapshot slot v&1 after it is unpinned; install pins the latest
 * snapshot and swaps it into consumer cidx's double buffer; read acquires a
 * slot and counts words != its version (torn reads), then releases it. */
viper_status viper_debug_proto_create(const char *path, uint64_t words, int32_t ncons, void **out);
viper_status viper_debug_proto_open(const char *path, uint64_t words, void **out);
viper_status viper_debug_proto_close(void *h, int32_t unlink_it, const char *path);
viper_status viper_debug_proto_publish(void *h, uint64_t v);
viper_status viper_debug_proto_install(void *h, int32_t cidx, uint64_t *installed, uint64_t *torn_snapshot);
viper_status viper_debug_proto_read(void *h, int32_t cidx, uint64_t *version, uint64_t *torn);

/* Test hook: the Transfer Selector's decision (VIPER_TIER_AUTO, selector.h)
 * on `world` gathered 288-byte records {u32 magic 0x56495452, i32 tier,
 * i32 nreach, i32 pad, char pci[16], char reach[16][16]}, as every rank of the
 * cross-process bootstrap computes it.  *out = the tier in use.  Host only. */
viper_status viper_debug_resolve_tier(const void *records, int32_t world, int32_t producer_rank,
                                      int32_t nproducers, int32_t fanout, int32_t requested, int32_t *out);

/* Test hooks: the descriptor hand-off of NVLS registration (VIPER_FANOUT_NVLS),
 * with no CUDA: an abstract Unix socket and SCM_RIGHTS.  listen: a fresh name
 * (written to name_out, >= 32 bytes) and a listening socket; serve: hand `fd`
 * to `n` fetchers, waiting at most timeout_ms for each (VIPER_E_PEER when one
 * never connects), then close the socket; fetch: connect to `name` (retrying
 * up to timeout_ms) and receive a duplicate of the served descriptor. */
viper_status viper_debug_fd_listen(char *name_out, int32_t cap, int32_t *listen_fd);
viper_status viper_debug_fd_serve(int32_t listen_fd, int32_t fd, int32_t n, int32_t timeout_ms);
viper_status viper_debug_fd_fetch(const char *name, int32_t *fd_out, int64_t timeout_ms);

/* Tear down (joins the update thread, frees library-owned memory). */
viper_status viper_unregister(viper_model *m);

/* ------------------------------------------------------------------------
 * viper_schedule -- the Inference Performance Predictor (s4.3 P:1229-1669).
 * Host only, no GPU.  Fits the Training Loss Predictor families Exp2, Exp3,
 * Lin2, Expd3 to the warm-up losses, keeps the min-MSE family
 * (ties -> the paper's list order, R7), derives t_p = s_model /
 * bw_write and t_c = s_model / bw_read unless
 * t_p / t_c >= 0 are given, then runs Algorithm 2 (fixed interval,
 * P:1626-1649) or Algorithm 3 (greedy irregular; reading R3).
 * ---------------------------------------------------------------------- */
enum { VIPER_SCHED_FIXED = 0, VIPER_SCHED_GREEDY = 1 };
enum { VIPER_TLP_EXP2 = 0, VIPER_TLP_EXP3 = 1, VIPER_TLP_LIN2 = 2, VIPER_TLP_EXPD3 = 3 };

typedef struct {
    const double *losses;    /* warm-up training losses                              */
    const double *x;         /* their iteration ids (NULL -> 0..n-1)                  */
    int32_t n;               /* >= 3                                                  */
    int64_t s_iter, e_iter;  /* schedule window [s_iter, e_iter]                      */
    int64_t total_infers;    /* inference requests over the window                    */
    double t_train, t_infer; /* seconds per training iteration / per inference        */
    double s_model, bw_write, bw_read; /* bytes, bytes/s (used when t_p/t_c < 0)      */
    double t_p, t_c;         /* producer stall / consumer load seconds; < 0 -> derive */
    int32_t algo;            /* VIPER_SCHED_*                                         */
    double thresh;           /* greedy threshold; < 0 -> mean + std of |d loss| (R8)  */
    int32_t family;          /* -1 = fit; 0..3 = use `params` as given (no fit)       */
    double params[3];        /* used when family >= 0                                 */
} viper_sched_in;

typedef struct {
    int32_t family;          /* chosen VIPER_TLP_*                                    */
    double params[3];        /* a, b, c (unused entries 0)                            */
    double mse[4];           /* per family                                            */
    double t_p, t_c, thresh; /* the values used                                       */
    int64_t best_interval;   /* FIXED: the chosen interval; GREEDY: 0                 */
    int64_t *sched;          /* caller-allocated: checkpoint iterations               */
    int64_t sched_cap;       /* capacity of sched                                     */
    int64_t sched_len;       /* entries needed / written.  sched_cap < needed ->
                                VIPER_E_INVAL with sched_len = needed (size query)    */
    double predicted_cil;    /* Alg. 2 min t_l / Alg. 3 sum(i_l) + p_l * rem          */
} viper_sched_out;

viper_status viper_schedule(const viper_sched_in *in, viper_sched_out *out);

/* Static description of a status code ("VIPER_E_CHECKSUM", ...). */
const char *viper_strerror(viper_status st);
/* Thread-local detail of the last error on this thread ("" if none). */
const char *viper_last_error(void);
/* Library version string. */
const char *viper_version(void);

#ifdef __cplusplus
}
#endif
#endif /* VIPER_H */
