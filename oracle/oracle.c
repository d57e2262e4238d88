/*
 * oracle.c -- plain, slow, obviously-correct CPU oracle for CSMV.
 *
 * TEST INFRASTRUCTURE ONLY (see oracle.h).  Single-threaded C99; no
 * blocking, fusion or reordering beyond what PAPER.md states.
 *
 * Notation follows PAPER.md section III: GTS (global timestamp),
 * snapshot s, CTS (commit timestamp), read-set / write-set
 * (P:71), ATR, VBox with K versions.
 */
#define _POSIX_C_SOURCE 199309L
#include "oracle.h"

#include <math.h>
#include <stdio.h>
#include <stdlib.h>
#include <string.h>
#include <time.h>

static double now_s(void) {
    struct timespec t;
    clock_gettime(CLOCK_MONOTONIC, &t);
    return (double)t.tv_sec + 1e-9 * (double)t.tv_nsec;
}

/* ====================================================================== */
/* Generator: docs/GENERATOR.md sections 1-2 (input recipe, not the method) */
/* ====================================================================== */

uint64_t or_mix64(uint64_t x) {
    uint64_t z = x + 0x9E3779B97F4A7C15ull;
    z = (z ^ (z >> 30)) * 0xBF58476D1CE4E5B9ull;
    z = (z ^ (z >> 27)) * 0x94D049BB133111EBull;
    return z ^ (z >> 31);
}

uint64_t or_draw(uint64_t seed, uint64_t tx, uint64_t k) {
    return or_mix64(or_mix64(seed ^ (tx * 0xD1B54A32D192ED03ull)) + k);
}

uint64_t or_uniform(uint64_t u, uint64_t n) {
    return (uint64_t)(((unsigned __int128)u * (unsigned __int128)n) >> 64);
}

int or_zipf_cdf(uint32_t n, uint32_t theta_milli, uint64_t *cdf) {
    if (n == 0 || !cdf) return OR_E_ARGS;
    double theta = (double)theta_milli / 1000.0;
    double h = 0.0;
    for (uint32_t r = 1; r <= n; r++) h += pow((double)r, -theta);
    double s = 0.0;
    for (uint32_t i = 0; i < n; i++) {
        s += pow((double)(i + 1), -theta);
        double x = ldexp(s / h, 64);
        cdf[i] = (x >= 18446744073709551616.0) ? UINT64_MAX : (uint64_t)x;
    }
    cdf[n - 1] = UINT64_MAX;
    return OR_OK;
}

uint32_t or_upper_bound(const uint64_t *cdf, uint32_t n, uint64_t u) {
    /* first i with cdf[i] > u; plain binary search, clamped to n-1 */
    uint32_t lo = 0, hi = n;
    while (lo < hi) {
        uint32_t mid = lo + (hi - lo) / 2;
        if (cdf[mid] > u) hi = mid; else lo = mid + 1;
    }
    return lo < n ? lo : n - 1;
}

static uint32_t pick(uint32_t dist, const uint64_t *cdf, uint32_t n, uint64_t u) {
    if (dist == OR_DIST_ZIPF) return or_upper_bound(cdf, n, u);
    return (uint32_t)or_uniform(u, n);
}

static int is_update_tx(uint32_t ro_period, uint32_t p_update_ppm,
                        uint64_t seed, uint64_t tx) {
    if (ro_period > 0) return (tx % ro_period) != (uint64_t)(ro_period - 1);
    uint64_t thr = ((uint64_t)p_update_ppm << 32) / 1000000ull;
    return (or_draw(seed, tx, 0) >> 32) < thr;
}

/* Bank descriptors: docs/GENERATOR.md section 3. */
int or_bank_gen(const or_bank_cfg *c, uint64_t seed, uint64_t tx0, uint64_t n,
                const uint64_t *cdf, or_bank_desc *out) {
    if (!c || !out || c->n_items < 2) return OR_E_ARGS;
    if (c->dist == OR_DIST_ZIPF && !cdf) return OR_E_ARGS;
    uint32_t N = c->n_items;
    for (uint64_t i = 0; i < n; i++) {
        uint64_t tx = tx0 + i;
        or_bank_desc *d = &out[i];
        memset(d, 0, sizeof *d);
        d->is_update = (uint32_t)is_update_tx(c->ro_period, c->p_update_ppm, seed, tx);
        if (d->is_update) {
            d->src = pick(c->dist, cdf, N, or_draw(seed, tx, 1));
            d->dst = pick(c->dist, cdf, N, or_draw(seed, tx, 2));
            if (d->dst == d->src) d->dst = (d->src + 1) % N;
            d->amt = (int32_t)(1 + or_uniform(or_draw(seed, tx, 3), c->amount_max));
        } else if (c->ro_reads == 0) {
            d->start = 0;
            d->len = N;
        } else {
            d->start = (uint32_t)or_uniform(or_draw(seed, tx, 1), N);
            d->len = c->ro_reads;
        }
    }
    return OR_OK;
}

/* Digest of one 4-byte item (docs/GENERATOR.md section 5). */
static uint64_t dig1(uint32_t item, uint32_t val) {
    return or_mix64(((uint64_t)item << 32) ^ (uint64_t)val);
}

/* ====================================================================== */
/* VBox: K-version ring per item                         */
/* ====================================================================== */
/* A version is packed as (ts << 32) | (u32)value; an unused slot has
 * ts = OR_EMPTY_TS.  A new version replaces an unused slot if one exists
 * (lowest index), otherwise the oldest version (smallest ts): "the sooner
 * older versions are replaced by more recent ones". */

static uint64_t pack(uint32_t ts, uint32_t v) { return ((uint64_t)ts << 32) | v; }
static uint32_t ts_of(uint64_t s) { return (uint32_t)(s >> 32); }

static void vbox_init(uint64_t *ring, uint32_t K, int32_t v) {
    ring[0] = pack(0, (uint32_t)v);
    for (uint32_t j = 1; j < K; j++) ring[j] = pack(OR_EMPTY_TS, 0);
}

static void vbox_install(uint64_t *ring, uint32_t K, uint32_t cts, uint32_t v) {
    uint32_t victim = K;
    for (uint32_t j = 0; j < K && victim == K; j++)
        if (ts_of(ring[j]) == OR_EMPTY_TS) victim = j;
    if (victim == K) {
        victim = 0;
        for (uint32_t j = 1; j < K; j++)
            if (ts_of(ring[j]) < ts_of(ring[victim])) victim = j;
    }
    ring[victim] = pack(cts, v);
}

uint64_t or_vbox_bytes(uint64_t n, uint32_t value_bytes, uint32_t k) {
    /* "4+(sizeof(X)+4) x #versions bytes" per data item */
    return n * (4ull + ((uint64_t)value_bytes + 4ull) * (uint64_t)k);
}

/* ====================================================================== */
/* Bank replaying checker                               */
/* ====================================================================== */

static int fail(or_report *r, int code, uint64_t tx, uint64_t exp, uint64_t got,
                const char *what) {
    r->ok = 0;
    r->code = code;
    r->tx = tx;
    r->expected = exp;
    r->got = got;
    snprintf(r->msg, sizeof r->msg, "%s (tx %llu: expected %llu got %llu)", what,
             (unsigned long long)tx, (unsigned long long)exp,
             (unsigned long long)got);
    return code;
}

/* Evaluate read-only transaction `tx` against the current state, which is
 * the state at its snapshot (it observes the versions with the
 * largest timestamp not after its snapshot). */
static int check_rot(const or_bank_cfg *c, const int32_t *state, uint64_t tx,
                     const or_bank_desc *d, const or_log_rec *rec,
                     const uint32_t *vals, uint32_t max_vals, or_report *rep) {
    uint32_t N = c->n_items;
    int64_t sum = 0;
    uint64_t dg = 0;
    for (uint32_t j = 0; j < d->len; j++) {
        uint32_t x = (d->start + j) % N;
        int32_t v = state[x];
        if (vals && j < max_vals && vals[tx * (uint64_t)max_vals + j] != (uint32_t)v)
            return fail(rep, OR_E_READ, tx, (uint32_t)v,
                        vals[tx * (uint64_t)max_vals + j], "read-only value");
        sum += v;
        dg += dig1(x, (uint32_t)v);
    }
    if (rec->read_digest != dg)
        return fail(rep, OR_E_READ, tx, dg, rec->read_digest, "read-only read digest");
    if (rec->aux != (uint64_t)sum)
        return fail(rep, OR_E_READ, tx, (uint64_t)sum, rec->aux, "read-only sum");
    return OR_OK;
}

int or_bank_check(const or_bank_cfg *c, const int32_t *init, uint64_t n_tx,
                  const or_bank_desc *d, const or_log_rec *log,
                  const uint32_t *vals, uint32_t max_vals,
                  const uint64_t *rings, const or_claims *claims,
                  or_report *rep) {
    if (!c || !init || !rep || (n_tx && (!d || !log))) return OR_E_ARGS;
    memset(rep, 0, sizeof *rep);
    rep->ok = 1;
    double t0 = now_s();
    uint32_t N = c->n_items, K = c->n_versions;
    int rc = OR_OK;

    /* R0: every transaction committed exactly once. */
    uint64_t C = 0, R = 0;
    for (uint64_t t = 0; t < n_tx; t++) {
        if (log[t].tx != (uint32_t)t || log[t].attempts == 0)
            return fail(rep, OR_E_MISSING, t, t, log[t].tx, "missing commit record");
        if (d[t].is_update) C++; else R++;
    }

    /* R1: CTS of the updates are exactly {1..C} (P:65 GTS counts commits,
     * P:116 CTS = GTS+1, P:130 consecutive per batch); snapshots in [0, C]
     * and an update's snapshot precedes its CTS. */
    uint64_t *by_cts = (uint64_t *)malloc((C + 1) * sizeof(uint64_t));
    uint64_t *rot_cnt = (uint64_t *)calloc(C + 2, sizeof(uint64_t));
    uint64_t *rot_ord = (uint64_t *)malloc((R + 1) * sizeof(uint64_t));
    int32_t *state = (int32_t *)malloc((size_t)N * sizeof(int32_t));
    uint32_t *lastw = (uint32_t *)calloc(N, sizeof(uint32_t));
    uint64_t *ring = (uint64_t *)malloc((size_t)N * K * sizeof(uint64_t));
    if (!by_cts || !rot_cnt || !rot_ord || !state || !lastw || !ring) {
        rc = fail(rep, OR_E_ARGS, 0, 0, 0, "out of memory");
        goto out;
    }
    for (uint64_t i = 0; i <= C; i++) by_cts[i] = UINT64_MAX;
    for (uint64_t t = 0; t < n_tx; t++) {
        const or_log_rec *r = &log[t];
        if (d[t].is_update) {
            if (r->cts < 1 || r->cts > C || by_cts[r->cts] != UINT64_MAX) {
                rc = fail(rep, OR_E_CTS, t, C, r->cts, "CTS not a permutation of 1..C");
                goto out;
            }
            by_cts[r->cts] = t;
            if (r->snapshot >= r->cts) {
                rc = fail(rep, OR_E_SNAPSHOT, t, r->cts, r->snapshot,
                          "update snapshot not before its CTS");
                goto out;
            }
        } else {
            if (r->cts != 0) {
                rc = fail(rep, OR_E_CTS, t, 0, r->cts, "read-only tx with a CTS");
                goto out;
            }
            if (r->snapshot > C) {
                rc = fail(rep, OR_E_SNAPSHOT, t, C, r->snapshot, "snapshot beyond final GTS");
                goto out;
            }
            rot_cnt[r->snapshot + 1]++;
        }
    }
    /* bucket the read-only transactions by snapshot (counting sort) */
    for (uint64_t i = 1; i <= C + 1; i++) rot_cnt[i] += rot_cnt[i - 1];
    for (uint64_t t = 0; t < n_tx; t++)
        if (!d[t].is_update) rot_ord[rot_cnt[log[t].snapshot]++] = t;
    /* now rot_cnt[s] is the end of bucket s; bucket s starts at rot_cnt[s-1] */

    /* R2: initial state, one version (ts 0) per VBox. */
    for (uint32_t x = 0; x < N; x++) {
        state[x] = init[x];
        vbox_init(&ring[(size_t)x * K], K, init[x]);
    }
    uint64_t rpos = 0;
    /* ROTs at snapshot 0 */
    while (rpos < rot_cnt[0]) {
        uint64_t t = rot_ord[rpos++];
        if ((rc = check_rot(c, state, t, &d[t], &log[t], vals, max_vals, rep))) goto out;
    }

    /* R3: replay updates in CTS order. */
    for (uint64_t cts = 1; cts <= C; cts++) {
        uint64_t t = by_cts[cts];
        const or_bank_desc *T = &d[t];
        const or_log_rec *r = &log[t];
        uint32_t s = r->snapshot;
        /* Validity: no transaction that committed after T's snapshot wrote an
         * item T read or wrote.  In CTS order this is
         * lastw[x] <= s for every x in RS u WS. */
        uint32_t items[2] = {T->src, T->dst};
        for (int k = 0; k < 2; k++)
            if (lastw[items[k]] > s) {
                rc = fail(rep, OR_E_VALIDITY, t, s, lastw[items[k]],
                          "committed although a later commit wrote its read/write set");
                goto out;
            }
        /* Observed reads: state now equals state at s on RS (validity). */
        int32_t vs = state[T->src], vd = state[T->dst];
        if (vals && max_vals >= 2) {
            const uint32_t *v = &vals[t * (uint64_t)max_vals];
            if (v[0] != (uint32_t)vs) { rc = fail(rep, OR_E_READ, t, (uint32_t)vs, v[0], "update read src"); goto out; }
            if (v[1] != (uint32_t)vd) { rc = fail(rep, OR_E_READ, t, (uint32_t)vd, v[1], "update read dst"); goto out; }
        }
        uint64_t rd = dig1(T->src, (uint32_t)vs) + dig1(T->dst, (uint32_t)vd);
        if (r->read_digest != rd) { rc = fail(rep, OR_E_READ, t, rd, r->read_digest, "update read digest"); goto out; }
        /* Writes: the transfer, int32 wrap-around. */
        uint32_t ns = (uint32_t)vs - (uint32_t)T->amt;
        uint32_t nd = (uint32_t)vd + (uint32_t)T->amt;
        uint64_t wd = dig1(T->src, ns) + dig1(T->dst, nd);
        if (r->aux != wd) { rc = fail(rep, OR_E_WRITE, t, wd, r->aux, "update write digest"); goto out; }
        /* Apply: new versions tagged with the CTS. */
        state[T->src] = (int32_t)ns;
        state[T->dst] = (int32_t)nd;
        vbox_install(&ring[(size_t)T->src * K], K, (uint32_t)cts, ns);
        vbox_install(&ring[(size_t)T->dst * K], K, (uint32_t)cts, nd);
        lastw[T->src] = lastw[T->dst] = (uint32_t)cts;
        /* Read-only transactions whose snapshot is cts. */
        while (rpos < rot_cnt[cts]) {
            uint64_t u = rot_ord[rpos++];
            if ((rc = check_rot(c, state, u, &d[u], &log[u], vals, max_vals, rep))) goto out;
        }
    }

    /* R4: final version rings (exact, the replacement rule is deterministic
     * given the CTS order) and the claimed counters. */
    if (rings) {
        for (uint64_t i = 0; i < (uint64_t)N * K; i++)
            if (rings[i] != ring[i]) {
                rc = fail(rep, OR_E_RING, i / K, ring[i], rings[i], "final version ring (item in tx field)");
                goto out;
            }
    }
    if (claims) {
        uint64_t ab = 0;
        for (uint64_t t = 0; t < n_tx; t++) ab += (uint64_t)log[t].attempts - 1;
        if (claims->committed_update != C) { rc = fail(rep, OR_E_STATS, 0, C, claims->committed_update, "committed_update"); goto out; }
        if (claims->committed_ro != R) { rc = fail(rep, OR_E_STATS, 0, R, claims->committed_ro, "committed_ro"); goto out; }
        if (claims->gts_final != C) { rc = fail(rep, OR_E_STATS, 0, C, claims->gts_final, "gts_final"); goto out; }
        if (claims->total_aborts != ab) { rc = fail(rep, OR_E_STATS, 0, ab, claims->total_aborts, "aborts vs attempts"); goto out; }
    }
    rep->replayed = n_tx;
out:
    rep->seconds = now_s() - t0;
    free(by_cts); free(rot_cnt); free(rot_ord); free(state); free(lastw); free(ring);
    return rc;
}

/* ====================================================================== */
/* Deterministic 1-client-warp schedule                        */
/* ====================================================================== */
/* One client warp of n_lanes lanes; lane l runs transactions l, l+n_lanes,
 * ... in order, retrying an aborted one in the next round.
 * Per round:
 *   1. s <- GTS (begin; one snapshot per warp round);
 *   2. (a) a lane whose current transaction is an update reads it at s;
 *      (b) a lane whose current transaction is read-only runs it at s and
 *      finishes -- with ro_streak = R > 0 it keeps running its
 *      next read-only transactions (at most R per round) and stops at its
 *      next update, which waits for the next round; with ro_streak = 0 it
 *      runs exactly one transaction per round;
 *   3. client-side pre-validation: update lanes in lane order, a
 *      lane is dropped if it conflicts with an earlier kept lane
 *      (SURVEY Q5); dropped lanes abort;
 *   4. the batch goes to the server, which validates it against the ATR
 *      entries committed after s -- with one client warp all
 *      earlier commits are <= s, so none conflicts -- and reserves
 *      consecutive CTS s+1.. in lane order;
 *   5. write-back and GTS += n.
 * Nothing else can abort here: the newest version of every item is at or
 * below s (no version misses) and the window is empty. */
int or_bank_predict(const or_bank_cfg *c, const int32_t *init, uint64_t n_tx,
                    const or_bank_desc *d, uint32_t L,
                    or_log_rec *log, uint32_t *vals, uint32_t max_vals,
                    uint64_t *rings_out, or_pred_stats *st) {
    if (!c || !init || !st || L == 0 || L > 32 || (n_tx && (!d || !log))) return OR_E_ARGS;
    memset(st, 0, sizeof *st);
    double t0 = now_s();
    uint32_t N = c->n_items, K = c->n_versions;
    int32_t *state = (int32_t *)malloc((size_t)N * sizeof(int32_t));
    uint64_t *ring = (uint64_t *)malloc((size_t)N * K * sizeof(uint64_t));
    if (!state || !ring) { free(state); free(ring); return OR_E_ARGS; }
    for (uint32_t x = 0; x < N; x++) {
        state[x] = init[x];
        vbox_init(&ring[(size_t)x * K], K, init[x]);
    }
    /* lane state: pending update cu (NONE = UINT64_MAX) and read cursor cr */
    uint64_t cu[32], cr[32];
    uint32_t att_u[32], att_r[32];
    for (uint32_t l = 0; l < L; l++) { cu[l] = UINT64_MAX; cr[l] = l; att_u[l] = att_r[l] = 0; }
    uint32_t gts = 0;
    for (;;) {
        int any = 0;
        for (uint32_t l = 0; l < L; l++) any |= cu[l] != UINT64_MAX || cr[l] < n_tx;
        if (!any) break;
        st->rounds++;
        uint32_t s = gts;                                   /* step 1 */
        int cand[32] = {0};
        for (uint32_t l = 0; l < L; l++) {                  /* step 2a */
            if (cu[l] == UINT64_MAX && cr[l] < n_tx && d[cr[l]].is_update) {
                cu[l] = cr[l];
                cr[l] += L;
            }
            if (cu[l] != UINT64_MAX) {
                att_u[l]++;
                cand[l] = 1;
            }
        }
        for (uint32_t l = 0; l < L; l++) {                  /* step 2b */
            if (!c->ro_streak && cu[l] != UINT64_MAX) continue;
            uint32_t n_ro = 0;
            while (cr[l] < n_tx) {
                uint64_t t = cr[l];
                const or_bank_desc *T = &d[t];
                if (T->is_update) break;  /* adopted in a later round */
                if (c->ro_streak ? n_ro >= c->ro_streak : n_ro >= 1) break;
                att_r[l]++;
                n_ro++;
                int64_t sum = 0;
                uint64_t dg = 0;
                for (uint32_t j = 0; j < T->len; j++) {
                    uint32_t x = (T->start + j) % N;
                    if (vals && j < max_vals) vals[t * (uint64_t)max_vals + j] = (uint32_t)state[x];
                    sum += state[x];
                    dg += dig1(x, (uint32_t)state[x]);
                }
                log[t].tx = (uint32_t)t; log[t].snapshot = s; log[t].cts = 0;
                log[t].attempts = att_r[l]; log[t].read_digest = dg; log[t].aux = (uint64_t)sum;
                st->committed_ro++;
                att_r[l] = 0;
                cr[l] += L;
            }
        }
        int kept[32] = {0};                                 /* step 3 */
        int nk = 0;
        for (uint32_t j = 0; j < L; j++) {
            if (!cand[j]) continue;
            const or_bank_desc *B = &d[cu[j]];
            int conflict = 0;
            for (uint32_t i = 0; i < j && !conflict; i++) {
                if (!kept[i]) continue;
                const or_bank_desc *A = &d[cu[i]];
                /* RS = WS = {src, dst}: any shared item is a conflict */
                conflict = A->src == B->src || A->src == B->dst ||
                           A->dst == B->src || A->dst == B->dst;
            }
            if (conflict) { st->aborts_preval++; continue; }
            kept[j] = 1;
            nk++;
        }
        if (nk) st->batches++;
        uint32_t rank = 0;                                  /* steps 4-5 */
        for (uint32_t l = 0; l < L; l++) {
            if (!kept[l]) continue;
            uint64_t t = cu[l];
            const or_bank_desc *T = &d[t];
            uint32_t cts = s + 1 + rank++;
            int32_t vs = state[T->src], vd = state[T->dst];
            if (vals && max_vals >= 2) {
                vals[t * (uint64_t)max_vals + 0] = (uint32_t)vs;
                vals[t * (uint64_t)max_vals + 1] = (uint32_t)vd;
            }
            uint32_t ns = (uint32_t)vs - (uint32_t)T->amt;
            uint32_t nd = (uint32_t)vd + (uint32_t)T->amt;
            log[t].tx = (uint32_t)t; log[t].snapshot = s; log[t].cts = cts;
            log[t].attempts = att_u[l];
            log[t].read_digest = dig1(T->src, (uint32_t)vs) + dig1(T->dst, (uint32_t)vd);
            log[t].aux = dig1(T->src, ns) + dig1(T->dst, nd);
            state[T->src] = (int32_t)ns;
            state[T->dst] = (int32_t)nd;
            vbox_install(&ring[(size_t)T->src * K], K, cts, ns);
            vbox_install(&ring[(size_t)T->dst * K], K, cts, nd);
            st->committed_update++;
            att_u[l] = 0;
            cu[l] = UINT64_MAX;
        }
        gts = s + (uint32_t)nk;
    }
    st->gts_final = gts;
    if (rings_out) memcpy(rings_out, ring, (size_t)N * K * sizeof(uint64_t));
    st->seconds = now_s() - t0;
    free(state); free(ring);
    return OR_OK;
}
