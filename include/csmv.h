/*
 * csmv.h -- C ABI of the B200 (sm_100a) CSMV batched commit pipeline.
 *
 * CSMV (Nunes, Castro, Romano, IPDPS 2022; /root/reference/PAPER.md, cited
 * P:<line>) is a multi-versioned STM for GPUs with a client-server commit:
 * client warps run transactions over versioned boxes (VBoxes),
 * pre-validate them inside the warp and ship each warp's update
 * transactions as one batch to a persistent server that validates them
 * against recently committed write-sets held in shared memory (the ATR,
 * P:65) and hands back consecutive commit timestamps (CTS,
 * P:101); clients then write the new versions back and
 * advance the global timestamp GTS in commit order.
 *
 * "The CSMV library masks away from the programmer all the complexity
 * associated with the management of transactions and of activating the
 * (server) kernel": this header is that library's boundary.  The
 * transaction bodies are the paper's two benchmarks (Bank P:177-183,
 * MemcachedGPU P:185), selected by csmv_workload.kind and generated from a
 * counter-based generator (docs/GENERATOR.md) inside the kernel.
 *
 * Conventions
 *  - Every call is extern "C", takes plain pointers and sizes.  Functions
 *    returning int return CSMV_OK (0) or a negative CSMV_E* code; the
 *    message of the last error of the calling thread is csmv_last_error().
 *  - A handle is single-threaded (not re-entrant); one handle per device.
 *  - The library owns all device memory.  Host buffers passed in are read
 *    during the call (the caller keeps ownership); output buffers are
 *    caller-allocated host memory.
 *  - There is no CPU fallback: without an sm_100a device csmv_create
 *    returns NULL and csmv_last_error() says why.
 */
#ifndef CSMV_H
#define CSMV_H
#include <stdint.h>
#ifdef __cplusplus
extern "C" {
#endif

#define CSMV_ABI_VERSION 1

/* ---- error codes ---- */
#define CSMV_OK 0
#define CSMV_EINVAL (-1)    /* bad argument */
#define CSMV_ENOMEM (-2)    /* device allocation failed */
#define CSMV_ECUDA (-3)     /* CUDA runtime error / no sm_100a device */
#define CSMV_ESTATE (-4)    /* wrong call order (e.g. run before load) */
#define CSMV_ETIMEOUT (-5)  /* device watchdog fired (a spin loop overran) */
#define CSMV_EOVERFLOW (-6) /* caller buffer too small / timestamp space exhausted */

/* ---- workload descriptor ---- */
#define CSMV_KIND_BANK 0u
#define CSMV_KIND_KV 1u        /* P:185 (MemcachedGPU) */
#define CSMV_DIST_UNIFORM 0u
#define CSMV_DIST_ZIPF 1u
#define CSMV_LOG_NONE 0u       /* timed runs */
#define CSMV_LOG_DIGEST 1u     /* 32 B record per transaction */
#define CSMV_LOG_FULL 2u       /* + every value read */
#define CSMV_SERVER_CTA 0u     /* single-SM server (the paper's) */
#define CSMV_SERVER_CLUSTER 1u /* thread-block-cluster server (DSMEM) */
#define CSMV_SERVER_PART 2u    /* item-partitioned servers (NEXT-3): cluster_size =
                                  S = 2..8 independent server CTAs, server k owning the items that hash to k;
                                  a batch prepares at every server owning one of its items (validate that
                                  part, mark it pending), takes its CTS from one global counter once all
                                  voted yes, then decides at each (record, unmark).  Bank, per-warp batches */
#define CSMV_PUBLISH_CLIENT 0u /* client advances GTS when GTS == CTS-1 */
#define CSMV_PUBLISH_SERVER 1u /* a server warp advances GTS over finished write-backs */
#define CSMV_ATR_HASH 0u       /* item-indexed ATR (set-associative, smem) */
#define CSMV_ATR_LIST 1u       /* the paper's ATR: list of write-sets, collaborative validation */
#define CSMV_ATR_LIST_NOCV 2u  /* the list ATR, one lane per transaction (CSMV-NoCV) */

/* commit protocol (csmv_workload.commit) */
#define CSMV_COMMIT_CSMV 0u    /* the paper's client-server batched commit */
#define CSMV_COMMIT_ONLYCS 1u  /* CSMV-onlyCS ablation: the client-server design alone --
                                  list ATR scanned per transaction (no CV), no client pre-validation,
                                  one ATR insert per transaction, server-side write-back.  Bank only,
                                  single-CTA server; atr_mode is ignored */
#define CSMV_COMMIT_JVSTM 2u   /* JVSTM-GPU baseline: no server; every thread validates
                                  against a global-memory ATR, reserves its CTS with a global CAS,
                                  writes back and advances GTS in order itself.  Bank only */

#define CSMV_DBG_NO_PREVAL 1u  /* negative control: skip client pre-validation */
#define CSMV_DBG_NO_VALIDATE 2u/* negative control: server commits without validating */
#define CSMV_DBG_JITTER 4u     /* race widening: every client and server warp sleeps a seeded 0..2047 ns
                                  at each cross-warp protocol step (doorbell, response poll, write-back,
                                  publish, receiver sweep, payload load, lock entry, e_pre -> lastw) */
#define CSMV_DBG_PHASES 8u     /* per-phase client clocks (csmv_stats_t.client_phase_cycles) */
#define CSMV_DBG_KV_ITEMSETS 16u /* KV, A <= 16: ship PUT read/write sets item by item (the paper's literal
                                    form); default {set clock} u WS, which decides identically */
#define CSMV_DBG_ALT_COMMIT 32u /* bank, atr_mode HASH: swap the commit path -- the single-CTA server
                                   commits through the commit ring and one committer warp instead of the
                                   ticket-locked critical section, the cluster server the other way
                                   round; A/B only */

#define CSMV_DBG_KV_SEQREAD 128u /* KV: a PUT lane scans its set itself, way group by way group (A/B and
                                    parity cross-check of the default warp-cooperative one-trip read) */
#define CSMV_DBG_TRACE 64u     /* hot-chain trace: every committed update that writes csmv_workload.
                                   trace_item (bank: an account; KV: a set) logs a csmv_trace_rec with
                                   device-wide timestamps (globaltimer) -- csmv_get_trace */

#define CSMV_RECV_WARP 0u       /* a receiver warp sweeps the doorbells into a shared-memory dispatch
                                   queue; combining fills larger batches */
#define CSMV_RECV_SELF 1u       /* bank, single-CTA locked commit: every worker warp sweeps its own
                                   slice of the doorbells (no receiver warp, one more worker, no queue);
                                   lower latency -- helps hot-item chains (C3); other servers ignore it */

typedef struct csmv_workload {
    uint32_t kind;             /* CSMV_KIND_* */
    uint32_t dist;             /* CSMV_DIST_* for the items an update picks */
    uint32_t zipf_theta_milli; /* 990 = theta 0.99 */
    uint32_t p_update_ppm;     /* update probability, parts per million */
    uint32_t ro_period;        /* >0: tx % ro_period == ro_period-1 is read-only */
    uint32_t ro_reads;         /* bank ROT: 0 = total sum of all accounts, L = L-item scan */
    uint32_t amount_max;       /* bank transfer amount uniform in [1, amount_max] */
    uint32_t kv_ways;          /* KV associativity A */
    uint32_t kv_keys;          /* KV key space */
    uint32_t client_warps;     /* active client warps; 0 = full grid */
    uint32_t server;           /* CSMV_SERVER_* */
    uint32_t cluster_size;     /* cluster server CTAs (2..16) */
    uint32_t server_workers;   /* worker warps per server CTA (0 = default) */
    uint32_t server_combine;   /* batches a worker commits per critical section (1..8; 0 = 1) */
    uint32_t atr_capacity;     /* ATR entries (0 = default); rounded to the layout */
    uint32_t atr_mode;         /* CSMV_ATR_* */
    uint32_t publish;          /* CSMV_PUBLISH_* */
    uint32_t ro_streak;        /* 0: one transaction per lane per round (paper); R: a lane runs up to
                                  R read-only transactions per round, ahead of a pending update */
    uint32_t backoff_max;      /* 0: an aborted update retries every round (paper); B: an
                                  update rejected by the server sits out up to B rounds */
    uint32_t log_mode;         /* CSMV_LOG_* */
    uint32_t debug_flags;      /* CSMV_DBG_* */
    uint32_t watchdog_ms;      /* 0 = default (20000) */
    uint32_t commit;           /* CSMV_COMMIT_* (0 = the paper's CSMV) */
    uint32_t ro_adaptive;      /* 1: a lane stops its read-only run (at most ro_streak) as soon as the
                                  server has answered the warp's batch -- rounds track the server
                                  round trip (timing-dependent schedule; 0 = fixed, deterministic);
                                  2 (KV): also when the warp submitted nothing because its PUTs met
                                  versions newer than the snapshot, once GTS covers them */
    uint32_t server_recv;      /* CSMV_RECV_*: how the server's worker warps get requests */
    uint32_t client_group;     /* 0/1: one request per client warp (the paper's batch); G = 2, 4, 8:
                                  the G client warps of a group (same CTA) pre-validate against each other
                                  in shared memory (P:118 extended across warps) and submit ONE request of
                                  up to 32G conflict-free transactions, committed in one step of the
                                  critical section (CTA-level batch).  Bank, single-CTA ticket-locked
                                  server with a receiver warp, item-indexed ATR, CSMV commit */
    uint32_t trace_item;       /* CSMV_DBG_TRACE: bank account / KV set whose committed writers are traced;
                                  0xFFFFFFFF = the hottest (account 0 / the set of key 0: zipf rank 0) */
    uint32_t elide_ww;         /* 1: blind-write elision -- validate the read-set only, no separate
                                  write-write check; allowed only for workloads without blind writes: the
                                  bank (every transfer reads what it writes: RS = WS, so validating RS is
                                  the whole check); EINVAL for KV, whose PUTs write the value blindly */
    uint32_t retry_order;      /* CSMV_RETRY_*: client-side contention management of update retries
                                  (the paper leaves retry scheduling open) */
    uint32_t server_writeback; /* 1 = the server worker writes a committed update's versions back right
                                  after the critical section and publishes it (done flags; KV with
                                  publish CLIENT: the worker advances GTS itself), the new values and
                                  replacement slots travelling with the request -- as CSMV-onlyCS does
                                  (P:266); 0 = the client writes back.  KV: compact requests;
                                  bank: self-receiving workers (either publish mode); elsewhere ignored.
                                  With req_tagged (KV) the written words carry a check word of the
                                  round that the server verifies; the bank's take fenced requests */
    uint32_t req_tagged;       /* 0: a client fences its request's payload before ringing the doorbell
                                  and the server's receiver fences after seeing it (acquire); 1: no
                                  fences -- every payload word carries the request's round and the
                                  server re-reads the payload until all of it does (as the client does
                                  with the response).  Shorter request path (hot-item chains, C3/C4);
                                  costs server time when payloads arrive after their doorbell (C2).
                                  Taken by the bank's self-receiving workers (CSMV_RECV_SELF) and the
                                  KV filter workers, with item ids < 2^24; elsewhere ignored (fenced) */
} csmv_workload;

#define CSMV_RETRY_FREE 0u     /* every pending update attempts each round (optionally backoff_max) */
#define CSMV_RETRY_FIFO 1u     /* KV: PUTs on one cache set attempt in FIFO ticket order -- a PUT takes a
                                  ticket of its set when its lane adopts it and reads/submits only once the
                                  set's previous ticket committed and GTS covers that commit.  All PUTs on a
                                  set conflict (each reads and writes the set clock), so this only removes
                                  attempts that were certain to abort; validation is unchanged.  The schedule
                                  is timing-dependent (not for the 1-warp determinism tests) */

/* ---- statistics ---- */
#define CSMV_AB_PREVAL 0u      /* lost client pre-validation */
#define CSMV_AB_CONFLICT 1u    /* server validation failed */
#define CSMV_AB_EARLY 2u       /* client read a version newer than its snapshot (validation would fail) */
#define CSMV_AB_OVERFLOW 3u    /* ATR no longer covers the snapshot (bounded ATR) */
#define CSMV_AB_VERSION 4u     /* no version old enough */
#define CSMV_N_ABORT 5u

typedef struct csmv_stats {
    uint64_t committed_update;
    uint64_t committed_ro;
    uint64_t aborts[CSMV_N_ABORT][2]; /* [reason][0 = read-only, 1 = update] */
    uint64_t batches;          /* requests the server processed (a request = one warp's batch, or one
                                  client group's batches with client_group > 1) */
    uint64_t server_groups;    /* critical sections (each commits up to server_combine batches) */
    uint64_t rounds;           /* client warp rounds */
    uint64_t gts_start;
    uint64_t gts_final;
    uint64_t elapsed_ns;       /* fused kernel, CUDA events */
    uint64_t ro_checksum;      /* xor of read-only results (keeps them live) */
    uint64_t store_bytes;      /* device bytes of the version store */
    uint64_t store_bytes_paper;/* same items in the paper's VBox layout */
    uint64_t server_lock_cycles; /* cycles the commit critical section was held */
    uint64_t server_busy_cycles; /* cycles workers spent processing batches */
    uint64_t server_phase_cycles[8]; /* worker: queue wait, payload load, lock wait, critical section, respond */
    uint64_t cas_failures;     /* CSMV_COMMIT_JVSTM: failed CTS reservations (global CAS) */
    uint64_t client_phase_cycles[8]; /* CSMV_DBG_PHASES, summed over client warps (mean lane): read,
                                    pre-validation | JVSTM validation+CAS, submit, read-only txs,
                                    wait for server, write-back, GTS publish, divergence (JVSTM) */
    uint32_t client_warps;
    uint32_t server_ctas;
    uint32_t server_workers;
    uint32_t atr_entries;
    uint32_t sm_count;
    uint32_t kernel_launches;  /* kernels launched by the last csmv_run */
} csmv_stats_t;

/* One record per committed transaction, indexed by transaction number
 * (docs/GENERATOR.md section 5). cts = 0 marks a read-only transaction. */
typedef struct csmv_log_rec {
    uint32_t tx, snapshot, cts, attempts;
    uint64_t read_digest, aux;
} csmv_log_rec;

/* CSMV_DBG_TRACE record of one committed update writing the traced item:
 * its commit timestamp and snapshot, and globaltimer (ns, device-wide) at
 * the start of the client round (TXBegin), the doorbell, the response and
 * the end of its publish step (GTS advanced, or done flag stored). */
typedef struct csmv_trace_rec {
    uint32_t cts, snapshot;
    uint64_t t_begin, t_submit, t_response, t_publish;
    uint64_t t_claim, t_served; /* server side: the worker took the request / stored the response
                                   (0 where the commit path does not stamp them) */
    uint64_t t_snap, t_read;    /* client: snapshot taken (GTS read) / read-set read, before
                                   pre-validation and submit (0 where not stamped) */
    uint32_t n_readers;         /* KV: PUT lanes of the warp that read their set in that round */
    uint32_t n_kept;            /* transactions of the request that carried this commit */
} csmv_trace_rec;

typedef struct csmv csmv_t;

/* Version of this ABI (CSMV_ABI_VERSION); never fails. */
int csmv_abi_version(void);

/* Create a store of n_items 4-byte items (bank accounts), each a VBox of
 * n_versions in [1,16] versions.  Needs an sm_100a device
 * (the current CUDA device).  NULL on error (EINVAL, ENOMEM, ECUDA). */
csmv_t *csmv_create(uint64_t n_items, uint32_t n_versions);

/* Create a MemcachedGPU store: n_slots slots of `ways` ways, with
 * 16-byte keys, 32-byte values, per-slot LRU and per-set clocks, each a VBox
 * of n_versions versions.  n_slots must be a multiple of ways. */
csmv_t *csmv_create_kv(uint64_t n_slots, uint32_t ways, uint32_t n_versions);

/* Bank: install init_values[0..n) (host memory) as version ts = 0 of every
 * item and reset GTS to 0 -- the VBoxes' initial versions before any
 * transaction ("GTS ... keeps track of how many update
 * transactions committed so far").  The host buffer is copied during the
 * call (caller keeps ownership).  EINVAL if n != n_items or a null
 * argument; ECUDA on a copy/launch failure.  Also clears lastw and the
 * done flags, so runs restart at CTS 1. */
int csmv_load(csmv_t *h, const int32_t *init_values, uint64_t n);

/* KV: preload keys 0..n_keys-1 with PUT semantics (docs/GENERATOR.md
 * section 4; MemcachedGPU's set-associative cache) as version ts = 0
 * and reset GTS to 0.  Computed on the device
 * (count keys per set, bucket them, keep each set's A largest keys: a set's
 * r-th insertion takes way r mod A) in a device staging buffer of about
 * (13*S + 4*T + n_keys) * 4 bytes that the handle keeps for later loads
 * (grown when n_keys grows, freed by csmv_destroy).  EINVAL if n_keys is 0 or
 * >= 2^32; ECUDA on an allocation or launch failure. */
int csmv_load_kv(csmv_t *h, uint64_t n_keys);

/* Run on the given CUDA stream (a cudaStream_t, e.g. torch's current
 * stream); NULL = the legacy default stream.  Not from the paper: the
 * library activates its server and client kernel on the caller's stream
 * ("activating the (server) kernel").  The handle does not own the
 * stream.  EINVAL on a null handle; never fails otherwise. */
int csmv_set_stream(csmv_t *h, void *cuda_stream);

/* Run transactions 0..n_tx-1 of the workload to completion: every
 * transaction commits exactly once, aborted attempts are retried.
 * Blocking.  Continues from the current store and GTS.  ESTATE if not
 * loaded; ETIMEOUT if the device watchdog fired (the handle must then be
 * reloaded); EOVERFLOW if GTS + n_tx would exceed 2^32 - 2. */
int csmv_run(csmv_t *h, const csmv_workload *w, uint64_t n_tx, uint64_t seed);

/* Statistics of the last csmv_run: committed transactions, aborted attempts
 * by reason, elapsed time -- the paper's measures: throughput (TXs/sec) and
 * abort rate (Table V), and the store's memory next to the paper's
 * VBox size formula.  Copied into caller memory.  EINVAL on a null
 * argument. */
int csmv_stats(const csmv_t *h, csmv_stats_t *out);

/* Log of the last csmv_run (needs log_mode != NONE): n_tx records into buf
 * (cap records), one per transaction: its snapshot, CTS
 * and digests of what it read and wrote -- what the replaying oracle needs
 * to check opacity in CTS order.  ESTATE if the last run had no log;
 * EOVERFLOW if cap < n_tx; *n_out = records written. */
int csmv_get_log(const csmv_t *h, csmv_log_rec *buf, uint64_t cap, uint64_t *n_out);

/* FULL log values of the last run: n_tx * (*max_vals) u32 words, transaction
 * t's reads at [t * max_vals, ...) -- every value it observed.
 * Pass buf = NULL to query the size.  ESTATE if the last run was not FULL;
 * EOVERFLOW if cap_words is too small. */
int csmv_get_vals(const csmv_t *h, uint32_t *buf, uint64_t cap_words, uint32_t *max_vals);

/* Bank: copy the version store out as n_items * n_versions packed slots
 * (ts << 32) | (uint32_t)value, ts = 0xFFFFFFFF for an unused slot -- the
 * K versions each VBox keeps.  EINVAL on a KV store or a
 * null argument; EOVERFLOW if cap < n_items * n_versions. */
int csmv_dump_store(const csmv_t *h, uint64_t *rings_out, uint64_t cap);

/* KV: newest value of every item (P:185's key, value, LRU stamp and set
 * clock items): keys (n_slots*4 words), values (n_slots*8), lru (n_slots),
 * clocks (n_slots/ways).  Any may be NULL.  EINVAL on a bank store; ESTATE
 * if not loaded. */
int csmv_dump_kv(const csmv_t *h, uint32_t *keys, uint32_t *vals, uint32_t *lru,
                 uint32_t *clocks);

/* Copy transaction descriptors tx0..tx0+n-1 as the device generator sees
 * them (6 u32 per bank tx: is_update, src, dst, amt, start, len -- the
 * Bank's transfers and balance scans; 10 per KV tx), for the
 * generator parity check.  EINVAL on a bad workload. */
int csmv_gen_descs(csmv_t *h, const csmv_workload *w, uint64_t seed, uint64_t tx0,
                   uint64_t n, uint32_t *out);

/* CSMV_DBG_TRACE records of the last csmv_run (in completion order, at
 * most 2^18): copies min(cap, recorded) into buf; *n_out = records
 * recorded (may exceed cap).  ESTATE if the last run was not traced.
 * Diagnostic of the hot-item commit chain (every writer of
 * an item commits and publishes after the previous one). */
int csmv_get_trace(const csmv_t *h, csmv_trace_rec *buf, uint64_t cap, uint64_t *n_out);

/* The zipf CDF table the library built for (n, theta_milli) (the
 * skewed key popularity of the MemcachedGPU workload).  EINVAL on
 * n = 0 or a null buffer. */
int csmv_zipf_table(uint32_t n, uint32_t theta_milli, uint64_t *out);

/* Release everything the handle owns (device memory, events); accepts
 * NULL.  Waits for the handle's stream first. */
void csmv_destroy(csmv_t *h);

/* Message of the last error on this thread ("" if none); owned by the
 * library, valid until the thread's next failing call. */
const char *csmv_last_error(void);

#ifdef __cplusplus
}
#endif
#endif
