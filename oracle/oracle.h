/*
 * oracle.h -- CPU oracle for the CSMV batched commit pipeline.
 *
 * TEST INFRASTRUCTURE ONLY.  Only tests/, __graft_entry__.smoke() and
 * bench.py's cpu_baseline / --impl reference legs may load this library.
 * The product path (paper_conf_ipps_nunesc022_b200/) never includes, links
 * or calls anything under oracle/, and this code shares nothing with it:
 * its generator is its own implementation of docs/GENERATOR.md.
 *
 * Source of truth: /root/reference/PAPER.md (Nunes, Castro, Romano, "CSMV",
 * IPDPS 2022), cited as P:<line>.  Readings of silent / garbled passages are
 * the Q-numbers of SURVEY.md section 8(c), listed again in DESIGN.md.
 *
 * What it computes:
 *   - or_bank_check: the replaying checker.  CSMV produces an
 *     opaque history whose serialisation order is commit-timestamp
 *     (CTS) order for update transactions, with every read-only transaction
 *     placed at its snapshot.  Given the initial store, the
 *     descriptors and the (snapshot, CTS) of every committed transaction, the
 *     final store and every observed value are fully determined; the checker
 *     replays serially in CTS order and compares element by element.
 *   - or_bank_predict: the deterministic 1-client-warp
 *     schedule: a round-by-round CPU simulation of the protocol
 *     (snapshot, reads, client pre-validation, batched CTS, write-back,
 *     batched GTS advance) that predicts every snapshot, CTS and abort count.
 *
 * Parity pins: see tests/test_oracle_*.py.  Every function here is pinned
 * (worked example E0, closed forms, conservation, brute force); none is
 * "parity unpinned".
 */
#ifndef CSMV_ORACLE_H
#define CSMV_ORACLE_H
#include <stdint.h>
#ifdef __cplusplus
extern "C" {
#endif

/* ---- generator (docs/GENERATOR.md sections 1-2) ---- */
uint64_t or_mix64(uint64_t x);
uint64_t or_draw(uint64_t seed, uint64_t tx, uint64_t k);
uint64_t or_uniform(uint64_t u, uint64_t n);
int or_zipf_cdf(uint32_t n, uint32_t theta_milli, uint64_t *cdf_out);
uint32_t or_upper_bound(const uint64_t *cdf, uint32_t n, uint64_t u);

#define OR_EMPTY_TS 0xFFFFFFFFu   /* an unused version slot */
#define OR_DIST_UNIFORM 0u
#define OR_DIST_ZIPF 1u

/* ---- bank workload ---- */
typedef struct {
    uint32_t n_items;          /* N accounts (>= 2) */
    uint32_t n_versions;       /* K versions per VBox, 1..16 */
    uint32_t dist;             /* OR_DIST_UNIFORM / OR_DIST_ZIPF */
    uint32_t zipf_theta_milli; /* 990 = theta 0.99 */
    uint32_t p_update_ppm;     /* threshold mode */
    uint32_t ro_period;        /* >0: tx % p == p-1 is read-only (C1) */
    uint32_t ro_reads;         /* 0: total-sum ROT; L: L-item scan */
    uint32_t amount_max;       /* amount uniform in [1, amount_max] */
    uint32_t ro_streak;        /* predictor: 0 = one tx per lane per round; R = a lane
                                  runs up to R read-only txs per round until it
                                  holds an update (csmv_workload.ro_streak) */
} or_bank_cfg;

typedef struct {
    uint32_t is_update;
    uint32_t src, dst;   /* update: read-set = write-set = {src, dst} */
    int32_t amt;
    uint32_t start, len; /* read-only: items (start + j) % N, j < len */
} or_bank_desc;

typedef struct {
    uint32_t tx, snapshot, cts, attempts;
    uint64_t read_digest, aux;
} or_log_rec;

typedef struct {
    int ok;              /* 1 = history accepted */
    int code;            /* failure class, OR_E* below */
    uint64_t tx;         /* first divergent transaction */
    uint64_t expected, got;
    uint64_t replayed;   /* transactions replayed */
    double seconds;      /* wall time of the replay */
    char msg[200];
} or_report;

enum {
    OR_OK = 0,
    OR_E_MISSING = 1,    /* a tx has no commit record (R0) */
    OR_E_CTS = 2,        /* CTS set is not exactly {1..C} (R1) */
    OR_E_SNAPSHOT = 3,   /* snapshot out of range / not before CTS (R1) */
    OR_E_VALIDITY = 4,   /* committed despite a conflict (R3) */
    OR_E_READ = 5,       /* observed value differs from state at snapshot */
    OR_E_WRITE = 6,      /* written values differ */
    OR_E_RING = 7,       /* final version rings differ (R4) */
    OR_E_STATS = 8,      /* counters inconsistent with the log */
    OR_E_ARGS = 9
};

/* What the implementation under test claims (its csmv_stats). */
typedef struct {
    uint64_t committed_update, committed_ro;
    uint64_t gts_final;
    uint64_t total_aborts;
} or_claims;

int or_bank_gen(const or_bank_cfg *cfg, uint64_t seed, uint64_t tx0, uint64_t n,
                const uint64_t *zipf_cdf, or_bank_desc *out);

/* Replaying checker.  vals (FULL log, max_vals u32 per tx), rings (N*K
 * packed (ts<<32)|val u64, final store) and claims may be NULL. */
int or_bank_check(const or_bank_cfg *cfg, const int32_t *init, uint64_t n_tx,
                  const or_bank_desc *d, const or_log_rec *log,
                  const uint32_t *vals, uint32_t max_vals,
                  const uint64_t *rings, const or_claims *claims,
                  or_report *rep);

typedef struct {
    uint64_t rounds, batches;
    uint64_t aborts_preval;
    uint64_t committed_update, committed_ro;
    uint64_t gts_final;
    double seconds;
} or_pred_stats;

/* Deterministic 1-warp schedule (n_lanes lanes, lane l runs tx l, l+n_lanes,
 * ...).  Outputs the log, FULL values (may be NULL), final rings (N*K). */
int or_bank_predict(const or_bank_cfg *cfg, const int32_t *init, uint64_t n_tx,
                    const or_bank_desc *d, uint32_t n_lanes,
                    or_log_rec *log_out, uint32_t *vals_out, uint32_t max_vals,
                    uint64_t *rings_out, or_pred_stats *st);

/* VBox memory footprint in the paper's layout, 4 + (sizeof(X)+4)*K per item
 * (P:289). */
uint64_t or_vbox_bytes(uint64_t n_items, uint32_t value_bytes, uint32_t k);


/* ---- KV workload: MemcachedGPU, docs/GENERATOR.md section 4 ---- */
typedef struct {
    uint32_t n_slots;          /* S */
    uint32_t ways;             /* A (S % A == 0) */
    uint32_t n_keys;           /* key space */
    uint32_t n_versions;       /* K */
    uint32_t dist, zipf_theta_milli;
    uint32_t p_update_ppm;     /* PUT probability */
    uint32_t ro_streak;        /* predictor, as in or_bank_cfg */
} or_kv_cfg;

typedef struct {
    uint32_t is_update;        /* 1 = PUT, 0 = GET */
    uint32_t key;              /* key index k */
    uint32_t val[8];           /* PUT value words */
} or_kv_desc;

/* Current value of every KV item (newest version). */
typedef struct {
    uint32_t *keys;    /* S * 4 words: key of slot i */
    uint32_t *vals;    /* S * 8 words: value of slot i */
    uint32_t *lru;     /* S: LRU stamp of slot i */
    uint32_t *clocks;  /* S / A: clock of set t */
} or_kv_state;

void or_kv_key16(uint32_t k, uint32_t out[4]);
uint32_t or_kv_set(uint32_t k, uint32_t n_sets);
int or_kv_gen(const or_kv_cfg *cfg, uint64_t seed, uint64_t tx0, uint64_t n,
              const uint64_t *zipf_cdf, or_kv_desc *out);
/* Preload keys 0..n_keys-1 with PUT semantics (docs/GENERATOR.md 4). */
int or_kv_preload(const or_kv_cfg *cfg, or_kv_state *st);
/* Replaying checker: as or_bank_check, over the KV store; final_state (may
 * be NULL) is the implementation's newest value of every item. */
int or_kv_check(const or_kv_cfg *cfg, const or_kv_state *init, uint64_t n_tx,
                const or_kv_desc *d, const or_log_rec *log,
                const or_kv_state *final_state, const or_claims *claims,
                or_report *rep);
/* Deterministic 1-warp schedule; st_out receives the final store. */
int or_kv_predict(const or_kv_cfg *cfg, const or_kv_state *init, uint64_t n_tx,
                  const or_kv_desc *d, uint32_t n_lanes, or_log_rec *log_out,
                  or_kv_state *st_out, or_pred_stats *st);

#ifdef __cplusplus
}
#endif
#endif
