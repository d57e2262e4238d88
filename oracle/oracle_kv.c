/*
 * oracle_kv.c -- CPU oracle for the MemcachedGPU workload of CSMV.
 *
 * TEST INFRASTRUCTURE ONLY (see oracle.h).  Plain C99, single-threaded.
 *
 * The mutable state is an A-way set-associative cache of S slots with an LRU
 * replacement policy, 16-byte keys and 32-byte values.  Every key,
 * value, per-slot LRU stamp and per-set clock is one versioned item (VBox,
 * P:63).  GET is a read-only transaction, PUT an update transaction that
 * scans the set and "issue[s] 4 write operations".  Readings of the
 * paper's silences are SURVEY Q16/Q27 and docs/GENERATOR.md section 4.
 */
#define _POSIX_C_SOURCE 199309L
#include "oracle.h"

#include <stdio.h>
#include <stdlib.h>
#include <string.h>
#include <time.h>

static double kv_now(void) {
    struct timespec t;
    clock_gettime(CLOCK_MONOTONIC, &t);
    return (double)t.tv_sec + 1e-9 * (double)t.tv_nsec;
}

/* ---- item ids (docs/GENERATOR.md 4) ---- */
#define MAXSET 1026u   /* 2A + 2 for A <= 512 */

typedef struct {
    uint32_t S, A, T;  /* slots, ways, sets */
} geom;

static uint32_t key_item(const geom *g, uint32_t i) { (void)g; return i; }
static uint32_t val_item(const geom *g, uint32_t i) { return g->S + i; }
static uint32_t lru_item(const geom *g, uint32_t i) { return 2u * g->S + i; }
static uint32_t clk_item(const geom *g, uint32_t t) { return 3u * g->S + t; }

void or_kv_key16(uint32_t k, uint32_t out[4]) {
    uint64_t a = or_mix64((uint64_t)k), b = or_mix64((uint64_t)k ^ 0x5555555555555555ull);
    out[0] = (uint32_t)a; out[1] = (uint32_t)(a >> 32);
    out[2] = (uint32_t)b; out[3] = (uint32_t)(b >> 32);
}

uint32_t or_kv_set(uint32_t k, uint32_t n_sets) {
    return (uint32_t)or_uniform(or_mix64((uint64_t)k ^ 0xA5A5A5A5A5A5A5A5ull), n_sets);
}

/* ---- digests (docs/GENERATOR.md 5) ---- */
static uint64_t dig_word(uint32_t item, uint32_t w, uint32_t word) {
    return or_mix64(((uint64_t)item << 35) ^ ((uint64_t)w << 32) ^ (uint64_t)word);
}
static uint64_t dig_u32(uint32_t item, uint32_t v) {
    return or_mix64(((uint64_t)item << 32) ^ (uint64_t)v);
}

/* ---- generator ---- */
int or_kv_gen(const or_kv_cfg *c, uint64_t seed, uint64_t tx0, uint64_t n,
              const uint64_t *cdf, or_kv_desc *out) {
    if (!c || !out || c->n_keys == 0) return OR_E_ARGS;
    if (c->dist == OR_DIST_ZIPF && !cdf) return OR_E_ARGS;
    uint64_t thr = ((uint64_t)c->p_update_ppm << 32) / 1000000ull;
    for (uint64_t i = 0; i < n; i++) {
        uint64_t tx = tx0 + i;
        or_kv_desc *d = &out[i];
        memset(d, 0, sizeof *d);
        d->is_update = (or_draw(seed, tx, 0) >> 32) < thr;
        uint64_t u = or_draw(seed, tx, 1);
        d->key = c->dist == OR_DIST_ZIPF ? or_upper_bound(cdf, c->n_keys, u)
                                         : (uint32_t)or_uniform(u, c->n_keys);
        if (d->is_update)
            for (uint32_t j = 0; j < 4; j++) {
                uint64_t v = or_draw(seed, tx, 4 + j);
                d->val[2 * j] = (uint32_t)v;
                d->val[2 * j + 1] = (uint32_t)(v >> 32);
            }
    }
    return OR_OK;
}

/* ---- transaction bodies on a state ---- */
typedef struct {
    uint32_t rs[MAXSET], nrs;   /* read-set, in read order */
    uint32_t ws[4], nws;        /* write-set (PUT) */
    uint64_t read_digest, aux;  /* aux: GET hit way+1 / 0; PUT write digest */
    uint32_t victim, clock_new; /* PUT */
} kv_effect;

static int key_eq(const uint32_t *a, const uint32_t *b) {
    return a[0] == b[0] && a[1] == b[1] && a[2] == b[2] && a[3] == b[3];
}
static int key_empty(const uint32_t *a) { return !(a[0] | a[1] | a[2] | a[3]); }

static void read_key(const geom *g, const or_kv_state *st, uint32_t slot, kv_effect *e) {
    uint32_t it = key_item(g, slot);
    e->rs[e->nrs++] = it;
    for (uint32_t w = 0; w < 4; w++) e->read_digest += dig_word(it, w, st->keys[4 * (size_t)slot + w]);
}

/* GET(k): scan the set's ways in order, stop at the matching key
 * (then read its value) or at the first empty way. */
static void kv_get(const geom *g, const or_kv_state *st, uint32_t k, kv_effect *e) {
    uint32_t kk[4];
    or_kv_key16(k, kk);
    uint32_t t = or_kv_set(k, g->T);
    e->nrs = e->nws = 0;
    e->read_digest = e->aux = 0;
    for (uint32_t w = 0; w < g->A; w++) {
        uint32_t slot = t * g->A + w;
        read_key(g, st, slot, e);
        const uint32_t *key = &st->keys[4 * (size_t)slot];
        if (key_eq(key, kk)) {
            uint32_t it = val_item(g, slot);
            e->rs[e->nrs++] = it;
            for (uint32_t j = 0; j < 8; j++) e->read_digest += dig_word(it, j, st->vals[8 * (size_t)slot + j]);
            e->aux = w + 1;
            return;
        }
        if (key_empty(key)) return;
    }
}

/* PUT(k, v): scan as GET; the victim is the matching or first empty
 * way, else the least recently updated way (all LRU stamps read, ties to
 * the lowest way); read the set clock c; write key, value, LRU = c+1 and
 * clock = c+1 ("4 write operations").  If apply, update the state. */
static void kv_put(const geom *g, or_kv_state *st, uint32_t k, const uint32_t val[8], int apply,
                   kv_effect *e) {
    uint32_t kk[4];
    or_kv_key16(k, kk);
    uint32_t t = or_kv_set(k, g->T);
    e->nrs = e->nws = 0;
    e->read_digest = e->aux = 0;
    uint32_t victim = UINT32_MAX;
    for (uint32_t w = 0; w < g->A && victim == UINT32_MAX; w++) {
        uint32_t slot = t * g->A + w;
        read_key(g, st, slot, e);
        const uint32_t *key = &st->keys[4 * (size_t)slot];
        if (key_eq(key, kk) || key_empty(key)) victim = slot;
    }
    if (victim == UINT32_MAX) {
        uint32_t best = 0;
        for (uint32_t w = 0; w < g->A; w++) {
            uint32_t slot = t * g->A + w;
            uint32_t it = lru_item(g, slot);
            e->rs[e->nrs++] = it;
            e->read_digest += dig_u32(it, st->lru[slot]);
            if (w == 0 || st->lru[slot] < best) {
                best = st->lru[slot];
                victim = slot;
            }
        }
    }
    uint32_t ci = clk_item(g, t);
    e->rs[e->nrs++] = ci;
    uint32_t c = st->clocks[t];
    e->read_digest += dig_u32(ci, c);
    uint32_t cn = c + 1;
    e->victim = victim;
    e->clock_new = cn;
    e->ws[0] = key_item(g, victim);
    e->ws[1] = val_item(g, victim);
    e->ws[2] = lru_item(g, victim);
    e->ws[3] = ci;
    e->nws = 4;
    uint64_t wd = 0;
    for (uint32_t j = 0; j < 4; j++) wd += dig_word(e->ws[0], j, kk[j]);
    for (uint32_t j = 0; j < 8; j++) wd += dig_word(e->ws[1], j, val[j]);
    wd += dig_u32(e->ws[2], cn) + dig_u32(ci, cn);
    e->aux = wd;
    if (apply) {
        memcpy(&st->keys[4 * (size_t)victim], kk, 16);
        memcpy(&st->vals[8 * (size_t)victim], val, 32);
        st->lru[victim] = cn;
        st->clocks[t] = cn;
    }
}

static int geom_of(const or_kv_cfg *c, geom *g) {
    if (!c || c->ways == 0 || c->n_slots == 0 || c->n_slots % c->ways) return OR_E_ARGS;
    if (2u * c->ways + 2u > MAXSET) return OR_E_ARGS;
    g->S = c->n_slots;
    g->A = c->ways;
    g->T = c->n_slots / c->ways;
    return OR_OK;
}

int or_kv_preload(const or_kv_cfg *c, or_kv_state *st) {
    geom g;
    if (geom_of(c, &g) || !st) return OR_E_ARGS;
    memset(st->keys, 0, (size_t)g.S * 16);
    memset(st->vals, 0, (size_t)g.S * 32);
    memset(st->lru, 0, (size_t)g.S * 4);
    memset(st->clocks, 0, (size_t)g.T * 4);
    kv_effect *e = (kv_effect *)malloc(sizeof *e);
    if (!e) return OR_E_ARGS;
    for (uint32_t k = 0; k < c->n_keys; k++) {
        uint32_t v[8];
        for (uint32_t j = 0; j < 4; j++) {
            uint64_t x = or_mix64((((uint64_t)k << 2) | j) ^ 0x3C3C3C3C3C3C3C3Cull);
            v[2 * j] = (uint32_t)x;
            v[2 * j + 1] = (uint32_t)(x >> 32);
        }
        kv_put(&g, st, k, v, 1, e);
    }
    free(e);
    return OR_OK;
}

/* ---- replaying checker (SURVEY 8(c) R0-R5 for the KV store) ---- */
static int kv_fail(or_report *r, int code, uint64_t tx, uint64_t exp, uint64_t got, const char *what) {
    r->ok = 0;
    r->code = code;
    r->tx = tx;
    r->expected = exp;
    r->got = got;
    snprintf(r->msg, sizeof r->msg, "%s (tx %llu: expected %llu got %llu)", what,
             (unsigned long long)tx, (unsigned long long)exp, (unsigned long long)got);
    return code;
}

static int state_alloc(const geom *g, or_kv_state *s) {
    s->keys = (uint32_t *)malloc((size_t)g->S * 16);
    s->vals = (uint32_t *)malloc((size_t)g->S * 32);
    s->lru = (uint32_t *)malloc((size_t)g->S * 4);
    s->clocks = (uint32_t *)malloc((size_t)g->T * 4);
    return s->keys && s->vals && s->lru && s->clocks;
}
static void state_copy(const geom *g, or_kv_state *d, const or_kv_state *s) {
    memcpy(d->keys, s->keys, (size_t)g->S * 16);
    memcpy(d->vals, s->vals, (size_t)g->S * 32);
    memcpy(d->lru, s->lru, (size_t)g->S * 4);
    memcpy(d->clocks, s->clocks, (size_t)g->T * 4);
}
static void state_free(or_kv_state *s) {
    free(s->keys); free(s->vals); free(s->lru); free(s->clocks);
}

static int check_get(const geom *g, const or_kv_state *st, uint64_t t, const or_kv_desc *d,
                     const or_log_rec *r, kv_effect *e, or_report *rep) {
    kv_get(g, st, d->key, e);
    if (r->read_digest != e->read_digest)
        return kv_fail(rep, OR_E_READ, t, e->read_digest, r->read_digest, "GET read digest");
    if (r->aux != e->aux) return kv_fail(rep, OR_E_READ, t, e->aux, r->aux, "GET hit way");
    return OR_OK;
}

int or_kv_check(const or_kv_cfg *c, const or_kv_state *init, uint64_t n_tx, const or_kv_desc *d,
                const or_log_rec *log, const or_kv_state *fin, const or_claims *claims,
                or_report *rep) {
    geom g;
    if (geom_of(c, &g) || !init || !rep || (n_tx && (!d || !log))) return OR_E_ARGS;
    memset(rep, 0, sizeof *rep);
    rep->ok = 1;
    double t0 = kv_now();
    int rc = OR_OK;
    uint64_t C = 0, R = 0;
    for (uint64_t t = 0; t < n_tx; t++) {                 /* R0 */
        if (log[t].tx != (uint32_t)t || log[t].attempts == 0)
            return kv_fail(rep, OR_E_MISSING, t, t, log[t].tx, "missing commit record");
        if (d[t].is_update) C++; else R++;
    }
    uint64_t n_items = 3ull * g.S + g.T;
    uint64_t *by_cts = (uint64_t *)malloc((C + 1) * sizeof(uint64_t));
    uint64_t *rot_cnt = (uint64_t *)calloc(C + 2, sizeof(uint64_t));
    uint64_t *rot_ord = (uint64_t *)malloc((R + 1) * sizeof(uint64_t));
    uint32_t *lastw = (uint32_t *)calloc(n_items, sizeof(uint32_t));
    kv_effect *e = (kv_effect *)malloc(sizeof *e);
    or_kv_state st = {0};
    int have = state_alloc(&g, &st);
    if (!by_cts || !rot_cnt || !rot_ord || !lastw || !e || !have) {
        rc = kv_fail(rep, OR_E_ARGS, 0, 0, 0, "out of memory");
        goto out;
    }
    for (uint64_t i = 0; i <= C; i++) by_cts[i] = UINT64_MAX;
    for (uint64_t t = 0; t < n_tx; t++) {                 /* R1 */
        const or_log_rec *r = &log[t];
        if (d[t].is_update) {
            if (r->cts < 1 || r->cts > C || by_cts[r->cts] != UINT64_MAX) {
                rc = kv_fail(rep, OR_E_CTS, t, C, r->cts, "CTS not a permutation of 1..C");
                goto out;
            }
            by_cts[r->cts] = t;
            if (r->snapshot >= r->cts) {
                rc = kv_fail(rep, OR_E_SNAPSHOT, t, r->cts, r->snapshot, "update snapshot not before its CTS");
                goto out;
            }
        } else {
            if (r->cts != 0) { rc = kv_fail(rep, OR_E_CTS, t, 0, r->cts, "read-only tx with a CTS"); goto out; }
            if (r->snapshot > C) { rc = kv_fail(rep, OR_E_SNAPSHOT, t, C, r->snapshot, "snapshot beyond final GTS"); goto out; }
            rot_cnt[r->snapshot + 1]++;
        }
    }
    for (uint64_t i = 1; i <= C + 1; i++) rot_cnt[i] += rot_cnt[i - 1];
    for (uint64_t t = 0; t < n_tx; t++)
        if (!d[t].is_update) rot_ord[rot_cnt[log[t].snapshot]++] = t;
    state_copy(&g, &st, init);                            /* R2 */
    uint64_t rpos = 0;
    while (rpos < rot_cnt[0]) {
        uint64_t t = rot_ord[rpos++];
        if ((rc = check_get(&g, &st, t, &d[t], &log[t], e, rep))) goto out;
    }
    for (uint64_t cts = 1; cts <= C; cts++) {             /* R3 */
        uint64_t t = by_cts[cts];
        const or_log_rec *r = &log[t];
        kv_put(&g, &st, d[t].key, d[t].val, 0, e);
        /* validity over RS u WS */
        for (uint32_t i = 0; i < e->nrs + e->nws; i++) {
            uint32_t x = i < e->nrs ? e->rs[i] : e->ws[i - e->nrs];
            if (lastw[x] > r->snapshot) {
                rc = kv_fail(rep, OR_E_VALIDITY, t, r->snapshot, lastw[x],
                             "committed although a later commit wrote its read/write set");
                goto out;
            }
        }
        if (r->read_digest != e->read_digest) { rc = kv_fail(rep, OR_E_READ, t, e->read_digest, r->read_digest, "PUT read digest"); goto out; }
        if (r->aux != e->aux) { rc = kv_fail(rep, OR_E_WRITE, t, e->aux, r->aux, "PUT write digest"); goto out; }
        kv_put(&g, &st, d[t].key, d[t].val, 1, e);
        for (uint32_t i = 0; i < e->nws; i++) lastw[e->ws[i]] = (uint32_t)cts;
        while (rpos < rot_cnt[cts]) {
            uint64_t u = rot_ord[rpos++];
            if ((rc = check_get(&g, &st, u, &d[u], &log[u], e, rep))) goto out;
        }
    }
    if (fin) {                                            /* R4 */
        for (uint64_t i = 0; i < (uint64_t)g.S * 4; i++)
            if (fin->keys[i] != st.keys[i]) { rc = kv_fail(rep, OR_E_RING, i / 4, st.keys[i], fin->keys[i], "final key (slot in tx field)"); goto out; }
        for (uint64_t i = 0; i < (uint64_t)g.S * 8; i++)
            if (fin->vals[i] != st.vals[i]) { rc = kv_fail(rep, OR_E_RING, i / 8, st.vals[i], fin->vals[i], "final value (slot in tx field)"); goto out; }
        for (uint64_t i = 0; i < g.S; i++)
            if (fin->lru[i] != st.lru[i]) { rc = kv_fail(rep, OR_E_RING, i, st.lru[i], fin->lru[i], "final LRU (slot in tx field)"); goto out; }
        for (uint64_t i = 0; i < g.T; i++)
            if (fin->clocks[i] != st.clocks[i]) { rc = kv_fail(rep, OR_E_RING, i, st.clocks[i], fin->clocks[i], "final clock (set in tx field)"); goto out; }
    }
    if (claims) {
        uint64_t ab = 0;
        for (uint64_t t = 0; t < n_tx; t++) ab += (uint64_t)log[t].attempts - 1;
        if (claims->committed_update != C) { rc = kv_fail(rep, OR_E_STATS, 0, C, claims->committed_update, "committed_update"); goto out; }
        if (claims->committed_ro != R) { rc = kv_fail(rep, OR_E_STATS, 0, R, claims->committed_ro, "committed_ro"); goto out; }
        if (claims->gts_final != C) { rc = kv_fail(rep, OR_E_STATS, 0, C, claims->gts_final, "gts_final"); goto out; }
        if (claims->total_aborts != ab) { rc = kv_fail(rep, OR_E_STATS, 0, ab, claims->total_aborts, "aborts vs attempts"); goto out; }
    }
    rep->replayed = n_tx;
out:
    rep->seconds = kv_now() - t0;
    free(by_cts); free(rot_cnt); free(rot_ord); free(lastw); free(e);
    if (have) state_free(&st);
    return rc;
}

/* ---- deterministic 1-client-warp schedule, as or_bank_predict ---- */
static int sets_conflict(const kv_effect *a, const kv_effect *b) {
    /* WS_a n (RS_b u WS_b) or WS_b n RS_a */
    for (uint32_t i = 0; i < a->nws; i++) {
        for (uint32_t j = 0; j < b->nrs; j++) if (a->ws[i] == b->rs[j]) return 1;
        for (uint32_t j = 0; j < b->nws; j++) if (a->ws[i] == b->ws[j]) return 1;
    }
    for (uint32_t i = 0; i < b->nws; i++)
        for (uint32_t j = 0; j < a->nrs; j++) if (b->ws[i] == a->rs[j]) return 1;
    return 0;
}

int or_kv_predict(const or_kv_cfg *c, const or_kv_state *init, uint64_t n_tx, const or_kv_desc *d,
                  uint32_t L, or_log_rec *log, or_kv_state *out, or_pred_stats *ps) {
    geom g;
    if (geom_of(c, &g) || !init || !ps || L == 0 || L > 32 || (n_tx && (!d || !log))) return OR_E_ARGS;
    memset(ps, 0, sizeof *ps);
    double t0 = kv_now();
    or_kv_state st = {0};
    kv_effect *eff = (kv_effect *)malloc(32 * sizeof(kv_effect));
    if (!state_alloc(&g, &st) || !eff) { free(eff); state_free(&st); return OR_E_ARGS; }
    state_copy(&g, &st, init);
    /* lane state as or_bank_predict: pending PUT cu, read cursor cr */
    uint64_t cu[32], cr[32];
    uint32_t att_u[32], att_r[32];
    for (uint32_t l = 0; l < L; l++) { cu[l] = UINT64_MAX; cr[l] = l; att_u[l] = att_r[l] = 0; }
    kv_effect *eg = &eff[L < 32 ? L : 31];  /* scratch for GETs */
    kv_effect get_tmp;
    if (L == 32) eg = &get_tmp;
    uint32_t gts = 0;
    for (;;) {
        int any = 0;
        for (uint32_t l = 0; l < L; l++) any |= cu[l] != UINT64_MAX || cr[l] < n_tx;
        if (!any) break;
        ps->rounds++;
        uint32_t s = gts;
        int cand[32] = {0};
        for (uint32_t l = 0; l < L; l++) {  /* pending PUTs read at s */
            if (cu[l] == UINT64_MAX && cr[l] < n_tx && d[cr[l]].is_update) {
                cu[l] = cr[l];
                cr[l] += L;
            }
            if (cu[l] != UINT64_MAX) {
                att_u[l]++;
                cand[l] = 1;
                kv_put(&g, &st, d[cu[l]].key, d[cu[l]].val, 0, &eff[l]);
            }
        }
        for (uint32_t l = 0; l < L; l++) {  /* GETs at s */
            if (!c->ro_streak && cu[l] != UINT64_MAX) continue;
            uint32_t n_ro = 0;
            while (cr[l] < n_tx) {
                uint64_t t = cr[l];
                if (d[t].is_update) break;
                if (c->ro_streak ? n_ro >= c->ro_streak : n_ro >= 1) break;
                att_r[l]++;
                n_ro++;
                kv_get(&g, &st, d[t].key, eg);
                log[t].tx = (uint32_t)t; log[t].snapshot = s; log[t].cts = 0; log[t].attempts = att_r[l];
                log[t].read_digest = eg->read_digest; log[t].aux = eg->aux;
                ps->committed_ro++;
                att_r[l] = 0;
                cr[l] += L;
            }
        }
        int kept[32] = {0};
        int nk = 0;
        for (uint32_t j = 0; j < L; j++) {
            if (!cand[j]) continue;
            int conflict = 0;
            for (uint32_t i = 0; i < j && !conflict; i++)
                if (kept[i]) conflict = sets_conflict(&eff[i], &eff[j]);
            if (conflict) { ps->aborts_preval++; continue; }
            kept[j] = 1;
            nk++;
        }
        if (nk) ps->batches++;
        uint32_t rank = 0;
        for (uint32_t l = 0; l < L; l++) {
            if (!kept[l]) continue;
            uint64_t t = cu[l];
            uint32_t cts = s + 1 + rank++;
            /* pairwise conflict-free: each kept PUT reads what it read at s */
            kv_put(&g, &st, d[t].key, d[t].val, 1, &eff[l]);
            log[t].tx = (uint32_t)t; log[t].snapshot = s; log[t].cts = cts; log[t].attempts = att_u[l];
            log[t].read_digest = eff[l].read_digest; log[t].aux = eff[l].aux;
            ps->committed_update++;
            att_u[l] = 0;
            cu[l] = UINT64_MAX;
        }
        gts = s + (uint32_t)nk;
    }
    ps->gts_final = gts;
    if (out) state_copy(&g, out, &st);
    ps->seconds = kv_now() - t0;
    state_free(&st);
    free(eff);
    return OR_OK;
}
