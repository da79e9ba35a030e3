/*
 * viper_oracle.c -- ORACLE (test infrastructure only; never on the product path).
 *
 * Only tests/, __graft_entry__.smoke() and bench.py's cpu_baseline / --impl
 * reference leg may load this library.  It shares no code, header, table or
 * constant generator with paper_conf_icpp_yecrbypnmskn24_b200/csrc: it is an
 * independent, plain, slow, obviously-correct CPU rendition of what one model
 * update computes, written from the paper and DESIGN.md's readings:
 *
 *   "the consumer will seamlessly replace the previous model with this new
 *    one" (s4.2)            -> a byte-exact state-dict copy
 *   "the updated model is written to an alternative copy, while the primary
 *    copy is used to serve inferences ... swapped atomically"
 *                                     (s4.2) -> double buffer + swap
 *   "only buffer and transfer the latest DNN model" (s4.4)
 *   checkpoint = "model parameters (weights, biases)"
 *
 * The packed layout (LAY), the chunk checksum (CKS) and the version-word
 * protocol are not in the paper (reading R16 in DESIGN.md): their plain
 * definitions are written out below exactly as DESIGN.md states them.
 *
 * Steps, in the paper's order for one update (s4.2 "Model Update" P:1183-1227):
 *   pack (snapshot the tensors) -> seal -> deliver (memcpy to each consumer's
 *   staging) -> verify -> wait until the alternative copy has no readers ->
 *   unpack into it -> atomic swap of the version word.
 * Everything is memcpy/memset and seq_cst C11 atomics; no blocking, fusion or
 * reordering beyond the definitions.
 */
#include <stdatomic.h>
#include <stdint.h>
#include <stdlib.h>
#include <string.h>
#include <sched.h>

#define OR_OK 0
#define OR_E_INVAL (-1)
#define OR_E_NOMEM (-2)
#define OR_E_VERSION (-4)
#define OR_E_CHECKSUM (-5)
#define OR_E_NOVERSION (-7)
#define OR_E_STATE (-8)

/* ---------------------------------------------------------------- LAY --
 * Reading R16: tensors keep registration order; off_0 = 0,
 * off_{t+1} = align_up(off_t + nbytes_t, align); S_packed = align_up(end, align).
 * Padding bytes are zero.  Returns S_packed. */
static uint64_t align_up(uint64_t x, uint64_t a) { return (x + a - 1) / a * a; }

uint64_t or_layout(int32_t n, const uint64_t *nbytes, uint32_t align, uint64_t *offsets) {
    uint64_t off = 0;
    for (int32_t i = 0; i < n; i++) {
        offsets[i] = off;
        off = align_up(off + nbytes[i], align);
    }
    return off;
}

/* ---------------------------------------------------------------- CKS --
 * Reading R16: view the packed buffer as little-endian u32 words
 * w_g (g = global word index mod 2^32), give each position the odd weight
 * m_g = (2g+1) * 0x9E3779B1 mod 2^32, and seal chunk c with
 *     cks_c = sum_{g in c} (w_g * m_g mod 2^32)   mod 2^64.
 * (SURVEY.md's XOR-with-index proposal missed ~7% of word swaps; see R16.)
 * `g0` is the global index of words[0]. */
uint64_t or_cks_words(const uint32_t *words, uint64_t nwords, uint64_t g0) {
    uint64_t sum = 0;
    for (uint64_t i = 0; i < nwords; i++) {
        uint32_t g = (uint32_t)(g0 + i);
        uint32_t m = (2u * g + 1u) * 0x9E3779B1u;
        uint32_t term = words[i] * m;
        sum += term;
    }
    return sum;
}

uint64_t or_nchunks(uint64_t s_packed, uint64_t chunk_bytes) {
    return (s_packed + chunk_bytes - 1) / chunk_bytes;
}

/* seals[2*c] = version, seals[2*c+1] = cks of chunk c. */
void or_seal(const uint8_t *packed, uint64_t s_packed, uint64_t chunk_bytes, uint64_t version,
             uint64_t *seals) {
    uint64_t nch = or_nchunks(s_packed, chunk_bytes);
    for (uint64_t c = 0; c < nch; c++) {
        uint64_t lo = c * chunk_bytes;
        uint64_t hi = lo + chunk_bytes < s_packed ? lo + chunk_bytes : s_packed;
        seals[2 * c] = version;
        seals[2 * c + 1] = or_cks_words((const uint32_t *)(packed + lo), (hi - lo) / 4, lo / 4);
    }
}

/* ------------------------------------------------------- pack / unpack -- */
void or_pack(int32_t n, const uint8_t *const *src, const uint64_t *nbytes, const uint64_t *offsets,
             uint8_t *packed, uint64_t s_packed) {
    memset(packed, 0, s_packed);
    for (int32_t i = 0; i < n; i++)
        if (nbytes[i]) memcpy(packed + offsets[i], src[i], nbytes[i]);
}

void or_unpack(int32_t n, uint8_t *const *dst, const uint64_t *nbytes, const uint64_t *offsets,
               const uint8_t *packed) {
    for (int32_t i = 0; i < n; i++)
        if (nbytes[i]) memcpy(dst[i], packed + offsets[i], nbytes[i]);
}

/* Returns OR_OK, OR_E_VERSION (a seal carries another version) or OR_E_CHECKSUM. */
int32_t or_verify(const uint8_t *packed, uint64_t s_packed, uint64_t chunk_bytes, uint64_t version,
                  const uint64_t *seals) {
    uint64_t nch = or_nchunks(s_packed, chunk_bytes);
    for (uint64_t c = 0; c < nch; c++) {
        uint64_t lo = c * chunk_bytes;
        uint64_t hi = lo + chunk_bytes < s_packed ? lo + chunk_bytes : s_packed;
        if (seals[2 * c] != version) return OR_E_VERSION;
        if (seals[2 * c + 1] != or_cks_words((const uint32_t *)(packed + lo), (hi - lo) / 4, lo / 4))
            return OR_E_CHECKSUM;
    }
    return OR_OK;
}

/* ------------------------------------------- double buffer + version word --
 * One consumer: two host copies of the T tensors (slot 0 = primary,
 * slot 1 = alternative), a 64-bit state word (version << 1) | active_slot
 * (0 = nothing installed), and one reader count per slot. */
typedef struct {
    int32_t n;
    uint64_t *nbytes, *offsets;
    uint64_t s_packed, chunk_bytes;
    uint8_t **slot[2];
    uint8_t *staging;
    uint64_t *seals;
    _Atomic uint64_t state;
    _Atomic int64_t ref[2];
    _Atomic uint64_t writes_while_pinned; /* writer-safety counter (must stay 0) */
    int32_t corrupt_next;                 /* fault injection: flip a staging byte */
} or_consumer;

typedef struct {
    int32_t n;
    uint64_t *nbytes, *offsets;
    uint64_t s_packed, chunk_bytes;
    uint8_t *packed;
    uint64_t *seals;
    uint64_t last_version;
    int32_t ncons;
    or_consumer **cons;
} or_producer;

static uint64_t *dup64(const uint64_t *a, int32_t n) {
    uint64_t *p = (uint64_t *)malloc(sizeof(uint64_t) * (n ? n : 1));
    if (p && n) memcpy(p, a, sizeof(uint64_t) * n);
    return p;
}

or_consumer *or_consumer_new(int32_t n, const uint64_t *nbytes, uint32_t align, uint64_t chunk_bytes) {
    or_consumer *c = (or_consumer *)calloc(1, sizeof(or_consumer));
    c->n = n;
    c->nbytes = dup64(nbytes, n);
    c->offsets = (uint64_t *)calloc(n ? n : 1, sizeof(uint64_t));
    c->s_packed = or_layout(n, nbytes, align, c->offsets);
    c->chunk_bytes = chunk_bytes;
    for (int s = 0; s < 2; s++) {
        c->slot[s] = (uint8_t **)calloc(n ? n : 1, sizeof(uint8_t *));
        for (int32_t i = 0; i < n; i++) c->slot[s][i] = (uint8_t *)calloc(nbytes[i] ? nbytes[i] : 1, 1);
    }
    c->staging = (uint8_t *)calloc(c->s_packed ? c->s_packed : 1, 1);
    c->seals = (uint64_t *)calloc(2 * (or_nchunks(c->s_packed, chunk_bytes) + 1), sizeof(uint64_t));
    atomic_store(&c->state, 0);
    atomic_store(&c->ref[0], 0);
    atomic_store(&c->ref[1], 0);
    atomic_store(&c->writes_while_pinned, 0);
    return c;
}

void or_consumer_free(or_consumer *c) {
    if (!c) return;
    for (int s = 0; s < 2; s++) {
        for (int32_t i = 0; i < c->n; i++) free(c->slot[s][i]);
        free(c->slot[s]);
    }
    free(c->staging); free(c->seals); free(c->nbytes); free(c->offsets); free(c);
}

or_producer *or_producer_new(int32_t n, const uint64_t *nbytes, uint32_t align, uint64_t chunk_bytes,
                             int32_t ncons, or_consumer **cons) {
    or_producer *p = (or_producer *)calloc(1, sizeof(or_producer));
    p->n = n;
    p->nbytes = dup64(nbytes, n);
    p->offsets = (uint64_t *)calloc(n ? n : 1, sizeof(uint64_t));
    p->s_packed = or_layout(n, nbytes, align, p->offsets);
    p->chunk_bytes = chunk_bytes;
    p->packed = (uint8_t *)calloc(p->s_packed ? p->s_packed : 1, 1);
    p->seals = (uint64_t *)calloc(2 * (or_nchunks(p->s_packed, chunk_bytes) + 1), sizeof(uint64_t));
    p->ncons = ncons;
    p->cons = (or_consumer **)calloc(ncons ? ncons : 1, sizeof(or_consumer *));
    for (int32_t i = 0; i < ncons; i++) p->cons[i] = cons[i];
    return p;
}

void or_producer_free(or_producer *p) {
    if (!p) return;
    free(p->packed); free(p->seals); free(p->nbytes); free(p->offsets); free(p->cons); free(p);
}

const uint8_t *or_producer_packed(const or_producer *p) { return p->packed; }
const uint64_t *or_producer_seals(const or_producer *p) { return p->seals; }
uint64_t or_producer_s_packed(const or_producer *p) { return p->s_packed; }

void or_consumer_corrupt_next(or_consumer *c) { c->corrupt_next = 1; }
uint64_t or_consumer_state(or_consumer *c) { return atomic_load(&c->state); }
uint64_t or_consumer_writes_while_pinned(or_consumer *c) { return atomic_load(&c->writes_while_pinned); }
uint8_t *or_consumer_slot_ptr(or_consumer *c, int32_t slot, int32_t t) { return c->slot[slot][t]; }

/* Install one delivered version into consumer c. */
int32_t or_install(or_consumer *c, uint64_t version) {
    if (c->corrupt_next && c->s_packed) {  /* fault injection: flip one bit in staging */
        c->staging[c->s_packed / 2] ^= 0x10;
        c->corrupt_next = 0;
    }
    int32_t st = or_verify(c->staging, c->s_packed, c->chunk_bytes, version, c->seals);
    if (st != OR_OK) return st;  /* not installed; the old version keeps serving */
    uint64_t cur = atomic_load(&c->state);
    int target = cur == 0 ? 0 : (int)(1 - (cur & 1));
    /* the alternative copy is written only once nobody reads it */
    while (atomic_load(&c->ref[target]) != 0) sched_yield();
    or_unpack(c->n, c->slot[target], c->nbytes, c->offsets, c->staging);
    if (atomic_load(&c->ref[target]) != 0) atomic_fetch_add(&c->writes_while_pinned, 1);
    atomic_store(&c->state, (version << 1) | (uint64_t)target); /* the atomic swap */
    return OR_OK;
}

/* One model update, producer side: pack, seal, deliver to every consumer,
 * install on every consumer.  Versions strictly increase, starting at 1. */
int32_t or_publish(or_producer *p, uint64_t version, const uint8_t *const *src) {
    if (version == 0 || version <= p->last_version) return OR_E_VERSION;
    p->last_version = version;
    or_pack(p->n, src, p->nbytes, p->offsets, p->packed, p->s_packed);
    or_seal(p->packed, p->s_packed, p->chunk_bytes, version, p->seals);
    uint64_t nch = or_nchunks(p->s_packed, p->chunk_bytes);
    int32_t worst = OR_OK;
    for (int32_t i = 0; i < p->ncons; i++) {
        or_consumer *c = p->cons[i];
        memcpy(c->staging, p->packed, p->s_packed);           /* deliver */
        memcpy(c->seals, p->seals, sizeof(uint64_t) * 2 * nch);
        int32_t st = or_install(c, version);
        if (st != OR_OK) worst = st;
    }
    return worst;
}

/* Reader side (a8): returns the pinned slot, its version via *version_out. */
int32_t or_acquire(or_consumer *c, uint64_t min_version, uint64_t *version_out, int32_t *slot_out) {
    for (;;) {
        uint64_t s = atomic_load(&c->state);
        if (s == 0 || (s >> 1) < min_version) return OR_E_NOVERSION;
        int slot = (int)(s & 1);
        atomic_fetch_add(&c->ref[slot], 1);
        if (atomic_load(&c->state) == s) {
            *version_out = s >> 1;
            *slot_out = slot;
            return OR_OK;
        }
        atomic_fetch_sub(&c->ref[slot], 1);  /* swapped under us: retry */
    }
}

int32_t or_release(or_consumer *c, int32_t slot) {
    if (slot < 0 || slot > 1) return OR_E_INVAL;
    int64_t prev = atomic_fetch_sub(&c->ref[slot], 1);
    if (prev <= 0) {
        atomic_fetch_add(&c->ref[slot], 1);
        return OR_E_STATE;
    }
    return OR_OK;
}
