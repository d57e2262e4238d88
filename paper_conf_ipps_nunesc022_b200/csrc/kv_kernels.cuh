// kv_kernels.cuh -- client warp and server worker for the MemcachedGPU
// workload.  Included by kernel.cu after the shared helpers.
//
// GET(k) is a read-only transaction: scan the ways of set(k), stop at the
// matching key (then read its value) or at the first empty way; never
// touches LRU.  PUT(k, v) is an update: the same scan, then the
// LRU stamps of all ways if neither a match nor an empty way was found, the
// set clock c, and the paper's "4 write operations": key, value, LRU = c+1,
// clock = c+1 (docs/GENERATOR.md 4).  Read/write sets are variable-length,
// so the request carries per-lane id lists and the server validates them
// with the generic worker below.
#pragma once

namespace csmvd {

template <int NS>
__device__ void client_warp_kv(const KParams& p, uint64_t t_begin, uint32_t* scratch) {
  const uint32_t FULL = 0xFFFFFFFFu;
  const uint32_t lane = threadIdx.x & 31, wib = threadIdx.x >> 5;
  const uint32_t cw = wib * p.n_client_ctas + (blockIdx.x - 1);
  if (cw >= p.n_cw) return;
  const uint64_t T = (uint64_t)p.n_cw * 32;
  uint64_t cur = (uint64_t)cw * 32 + lane;
  uint32_t att = 0;
  ClientCounters cc;
  uint32_t round = 0;
  const uint32_t K = p.K, S = p.kv_S, A = p.kv_A, Tn = p.kv_T;
  const uint32_t lt = lanemask_lt();
  const uint32_t streak = p.ro_streak;
  // per-warp smem scratch, lane-minor: RS[kKvMaxRs][32], WS[4][32], NRS[32]
  uint32_t* RS = scratch + (size_t)wib * 32 * (kKvMaxRs + 5);
  uint32_t* WS = RS + kKvMaxRs * 32;
  uint32_t* NRS = WS + 4 * 32;
  uint32_t* my_ids = p.req_ids + (size_t)cw * p.maxid * 32;

  for (;;) {
    if (!__any_sync(FULL, cur < p.n_tx)) break;
    ++round;
    ++cc.n_rounds;
    uint32_t s = 0, err = 0;
    if (lane == 0) {
      s = ld_acquire(p.gts);  // TXBegin
      err = ld_relaxed(&p.ctl->error);
    }
    s = __shfl_sync(FULL, s, 0);
    if (__shfl_sync(FULL, err, 0)) break;

    int status = ST_NONE;
    KvTx d{};
    uint32_t kk[4] = {0, 0, 0, 0};
    uint32_t victim = 0, tset = 0, clk = 0, nrs = 0;
    uint64_t rdig = 0;
    uint32_t n_ro = 0;
    while (cur < p.n_tx) {
      d = gen_kv(p.gen, cur);
      kv_key16(d.key, kk);
      tset = kv_set(d.key, Tn);
      if (!d.is_update) {
        // ---- GET: a read-only transaction
        if (streak ? n_ro >= streak : n_ro >= 1) break;
        ++att;
        ++n_ro;
        uint64_t dg = 0;
        uint32_t hit = 0;
        int r = RD_OK;
        for (uint32_t w = 0; w < A; ++w) {
          const uint32_t slot = tset * A + w;
          uint32_t key[4];
          r = kv_read_mw<NS, 4>(p.kv_key + (size_t)slot * NS * 4, K, s, true, key);
          if (r != RD_OK) break;
#pragma unroll
          for (int j = 0; j < 4; ++j) dg += dig_word(slot, j, key[j]);
          if (key[0] == kk[0] && key[1] == kk[1] && key[2] == kk[2] && key[3] == kk[3]) {
            uint32_t val[8];
            r = kv_read_mw<NS, 8>(p.kv_val + (size_t)slot * NS * 8, K, s, true, val);
            if (r != RD_OK) break;
#pragma unroll
            for (int j = 0; j < 8; ++j) dg += dig_word(S + slot, j, val[j]);
            hit = w + 1;
            break;
          }
          if (!(key[0] | key[1] | key[2] | key[3])) break;
        }
        if (r != RD_OK) {
          cc.abort(CSMV_AB_VERSION, false);  // retried next round
          status = ST_ABORT;
          break;
        }
        if (p.log_mode) log_commit(p, cur, s, 0, att, dg, hit);
        ++cc.c_ro;
        cc.ro_ck ^= dg;
        cur += T;
        att = 0;
        continue;
      }
      if (!streak && n_ro) break;
      // ---- PUT: reads of an update transaction (RS tracked)
      ++att;
      int r = RD_OK;
      victim = 0xFFFFFFFFu;
      nrs = 0;
      rdig = 0;
      for (uint32_t w = 0; w < A && victim == 0xFFFFFFFFu; ++w) {
        const uint32_t slot = tset * A + w;
        uint32_t key[4];
        r = kv_read_mw<NS, 4>(p.kv_key + (size_t)slot * NS * 4, K, s, false, key);
        if (r != RD_OK) break;
        RS[nrs++ * 32 + lane] = slot;
#pragma unroll
        for (int j = 0; j < 4; ++j) rdig += dig_word(slot, j, key[j]);
        if ((key[0] == kk[0] && key[1] == kk[1] && key[2] == kk[2] && key[3] == kk[3]) ||
            !(key[0] | key[1] | key[2] | key[3]))
          victim = slot;
      }
      if (r == RD_OK && victim == 0xFFFFFFFFu) {
        uint32_t best = 0;
        for (uint32_t w = 0; w < A; ++w) {
          const uint32_t slot = tset * A + w;
          uint32_t l;
          r = kv_read_1<NS>(p.kv_lru + (size_t)slot * NS, K, s, l);
          if (r != RD_OK) break;
          RS[nrs++ * 32 + lane] = 2 * S + slot;
          rdig += dig1(2 * S + slot, l);
          if (w == 0 || l < best) {
            best = l;
            victim = slot;
          }
        }
      }
      if (r == RD_OK) {
        r = kv_read_1<NS>(p.kv_clk + (size_t)tset * NS, K, s, clk);
        if (r == RD_OK) {
          RS[nrs++ * 32 + lane] = 3 * S + tset;
          rdig += dig1(3 * S + tset, clk);
        }
      }
      if (r == RD_NEWER) {
        cc.abort(CSMV_AB_EARLY, true);
        status = ST_ABORT;
      } else if (r == RD_MISS) {
        cc.abort(CSMV_AB_VERSION, true);
        status = ST_ABORT;
      } else {
        WS[0 * 32 + lane] = victim;
        WS[1 * 32 + lane] = S + victim;
        WS[2 * 32 + lane] = 2 * S + victim;
        WS[3 * 32 + lane] = 3 * S + tset;
        NRS[lane] = nrs;
        status = ST_CAND;
      }
      break;
    }
    __syncwarp();

    // Client-side pre-validation: greedy in lane order; lane j is
    // dropped if WS_i n (RS_j u WS_j) or WS_j n RS_i is non-empty for an
    // earlier kept lane i.
    const uint32_t cand = __ballot_sync(FULL, status == ST_CAND);
    uint32_t kept = cand;
    if (!(p.debug & CSMV_DBG_NO_PREVAL)) {
      kept = 0;
      uint32_t rem = cand;
      while (rem) {
        const int i = __ffs(rem) - 1;
        kept |= 1u << i;
        bool conf = false;
        if (((rem >> lane) & 1u) && lane > (uint32_t)i) {
          const uint32_t nrs_i = NRS[i];
          for (int a = 0; a < 4; ++a) {
            const uint32_t x = WS[a * 32 + i];
            for (uint32_t b = 0; b < nrs; ++b) conf |= RS[b * 32 + lane] == x;
            for (int b = 0; b < 4; ++b) conf |= WS[b * 32 + lane] == x;
          }
          for (uint32_t b = 0; b < nrs_i; ++b) {
            const uint32_t y = RS[b * 32 + i];
            for (int a = 0; a < 4; ++a) conf |= WS[a * 32 + lane] == y;
          }
        }
        rem &= ~__ballot_sync(FULL, conf) & ~(1u << i);
      }
    }
    const bool mine = (kept >> lane) & 1u;
    if (status == ST_CAND && !mine) cc.abort(CSMV_AB_PREVAL, true);
    if (!kept) continue;

    // Batch submit: per-lane id list RS u WS (bit 31: in WS).
    if (mine) {
      uint32_t n = 0;
      for (uint32_t b = 0; b < nrs; ++b) {
        const uint32_t x = RS[b * 32 + lane];
        bool w = false;
#pragma unroll
        for (int a = 0; a < 4; ++a) w |= WS[a * 32 + lane] == x;
        my_ids[(size_t)n++ * 32 + lane] = x | (w ? kWriteBit : 0u);
      }
#pragma unroll
      for (int a = 0; a < 4; ++a) {
        const uint32_t x = WS[a * 32 + lane];
        bool in_rs = false;
        for (uint32_t b = 0; b < nrs; ++b) in_rs |= RS[b * 32 + lane] == x;
        if (!in_rs) my_ids[(size_t)n++ * 32 + lane] = x | kWriteBit;
      }
      p.req_cnt[(size_t)cw * 32 + lane] = n;
    }
    if (lane == 0) {
      p.req_hdr[cw].snapshot = s;
      p.req_hdr[cw].mask = kept;
    }
    __syncwarp();
    fence_gpu();
    uint32_t base = 0, cmask = 0, omask = 0;
    if (lane == 0) st_relaxed(&p.req_seq[cw], round);
    {
      uint32_t it = 0;
      bool ok = true;
      while (warp_ld_relaxed(&p.resp[cw].seq) != round) {
        if ((++it & 255u) == 0) {
          uint32_t bad = 0;
          if (lane == 0) bad = ld_relaxed(&p.ctl->error) || watchdog(p, t_begin, 1);
          if (__shfl_sync(FULL, bad, 0)) {
            ok = false;
            break;
          }
        }
        __nanosleep(64);
      }
      fence_gpu();
      if (ok) {
        base = ld_relaxed(&p.resp[cw].cts_base);
        cmask = ld_relaxed(&p.resp[cw].commit_mask);
        omask = ld_relaxed(&p.resp[cw].overflow_mask);
      }
    }
    uint32_t cts = 0;
    if (mine) {
      if ((cmask >> lane) & 1u) {
        // Client-side write-back: the paper's 4 writes.
        cts = base + __popc(cmask & lt);
        const uint32_t cn = clk + 1;
        kv_write_mw<NS, 4>(p.kv_key + (size_t)victim * NS * 4, K, cts, kk);
        kv_write_mw<NS, 8>(p.kv_val + (size_t)victim * NS * 8, K, cts, d.val);
        kv_write_1<NS>(p.kv_lru + (size_t)victim * NS, K, cts, cn);
        kv_write_1<NS>(p.kv_clk + (size_t)tset * NS, K, cts, cn);
        if (p.log_mode) {
          uint64_t wd = dig1(2 * S + victim, cn) + dig1(3 * S + tset, cn);
#pragma unroll
          for (int j = 0; j < 4; ++j) wd += dig_word(victim, j, kk[j]);
#pragma unroll
          for (int j = 0; j < 8; ++j) wd += dig_word(S + victim, j, d.val[j]);
          log_commit(p, cur, s, cts, att, rdig, wd);
        }
        ++cc.c_upd;
        cur += T;
        att = 0;
      } else {
        cc.abort(((omask >> lane) & 1u) ? CSMV_AB_OVERFLOW : CSMV_AB_CONFLICT, true);
      }
    }
    const uint32_t n = __popc(cmask);
    if (n) {
      if (p.publish == CSMV_PUBLISH_CLIENT) {
        __syncwarp();
        fence_gpu();
        uint32_t it = 0;
        while (warp_ld_relaxed(p.gts) != base - 1) {
          if ((++it & 255u) == 0) {
            uint32_t bad = 0;
            if (lane == 0) bad = ld_relaxed(&p.ctl->error) || watchdog(p, t_begin, 2);
            if (__shfl_sync(FULL, bad, 0)) break;
          }
          __nanosleep(32);
        }
        if (lane == 0) st_release(p.gts, base + n - 1);
      } else if (cts) {
        st_release(p.done_ring + (cts & ((1u << kDoneLog2) - 1)), cts);
      }
    }
  }
  client_flush(p, cc);
}

// Generic server worker (variable-length read/write sets): one batch per
// critical section.  Validation reads lastw inside the critical section, so
// it covers every commit up to the current tail exactly.
__device__ void server_worker_generic(const KParams& p, uint64_t* queue, uint32_t qn_log2, SrvShared* sh,
                                      uint64_t t_begin) {
  const uint32_t FULL = 0xFFFFFFFFu;
  const uint32_t lane = threadIdx.x & 31;
  const uint32_t lt = lanemask_lt();
  const uint32_t qmask = (1u << qn_log2) - 1;
  const uint32_t dmask = (1u << kDoneLog2) - 1;
  unsigned long long busy = 0, locked = 0, batches = 0;
  for (;;) {
    uint32_t slot = 0;
    if (lane == 0) slot = atomicAdd(&sh->q_head, 1u);
    slot = __shfl_sync(FULL, slot, 0);
    uint64_t ent;
    bool quit = false;
    for (;;) {
      ent = *(volatile uint64_t*)&queue[slot & qmask];
      if ((uint32_t)(ent >> 32) == (slot >> qn_log2) + 1) break;
      if (*(volatile uint32_t*)&sh->exit) {
        quit = true;
        break;
      }
      __nanosleep(64);
    }
    if (quit) break;
    const uint32_t cw = (uint32_t)ent;
    const long long t0 = clock64();
    const uint32_t sq = ld_relaxed(p.req_seq + cw);
    fence_gpu();
    const uint32_t s = ld_relaxed(&p.req_hdr[cw].snapshot);
    const uint32_t mask = ld_relaxed(&p.req_hdr[cw].mask);
    const bool mine = (mask >> lane) & 1u;
    const uint32_t cnt = mine ? ld_relaxed(p.req_cnt + (size_t)cw * 32 + lane) : 0u;
    uint32_t ids[kKvMaxId];
#pragma unroll
    for (uint32_t k = 0; k < kKvMaxId; ++k)
      ids[k] = (k < cnt) ? ld_relaxed(p.req_ids + ((size_t)cw * p.maxid + k) * 32 + lane) : 0u;
    uint32_t x = s;
#pragma unroll
    for (uint32_t k = 0; k < kKvMaxId; ++k) x ^= ids[k];
    if (__ballot_sync(FULL, x == 0x12345679u) == FULL) __nanosleep(1);
    // ---- critical section
    uint32_t ticket = 0;
    if (lane == 0) ticket = atomicAdd(&sh->next_ticket, 1u);
    ticket = __shfl_sync(FULL, ticket, 0);
    while (*(volatile uint32_t*)&sh->now_serving != ticket) __nanosleep(16);
    __syncwarp();
    fence_cta();
    const long long t1 = clock64();
    const uint32_t t0c = *(volatile uint32_t*)&sh->tail;
    uint32_t lw[kKvMaxId];
#pragma unroll
    for (uint32_t k = 0; k < kKvMaxId; ++k) lw[k] = (k < cnt) ? ld_relaxed(p.lastw + (ids[k] & ~kWriteBit)) : 0u;
    bool conflict = false;
#pragma unroll
    for (uint32_t k = 0; k < kKvMaxId; ++k) conflict |= lw[k] > s;
    if (p.debug & CSMV_DBG_NO_VALIDATE) conflict = false;
    const bool commit = mine && !conflict;
    const uint32_t cm = __ballot_sync(FULL, commit);
    const uint32_t n = __popc(cm);
    const uint32_t cts = t0c + 1 + __popc(cm & lt);
    if (p.publish == CSMV_PUBLISH_SERVER && n) {
      if (lane == 0) {
        uint32_t it = 0;
        while (t0c + n > sh->gts_seen + dmask) {
          sh->gts_seen = ld_relaxed(p.gts);
          if ((++it & 255u) == 0 && watchdog(p, t_begin, 4)) break;
        }
      }
      __syncwarp();
    }
    if (commit) {
#pragma unroll
      for (uint32_t k = 0; k < kKvMaxId; ++k)
        if (k < cnt && (ids[k] & kWriteBit)) p.lastw[ids[k] & ~kWriteBit] = cts;
    }
    __syncwarp();
    fence_cta();
    if (lane == 0) {
      sh->tail = t0c + n;
      fence_cta();
      *(volatile uint32_t*)&sh->now_serving = ticket + 1;
    }
    const long long t2 = clock64();
    if (lane == 0) {
      st_relaxed(&p.resp[cw].cts_base, t0c + 1);
      st_relaxed(&p.resp[cw].commit_mask, cm);
      st_relaxed(&p.resp[cw].overflow_mask, 0u);
      st_release(&p.resp[cw].seq, sq);
    }
    __syncwarp();
    busy += (unsigned long long)(clock64() - t0);
    locked += (unsigned long long)(t2 - t1);
    ++batches;
  }
  if (lane == 0) {
    atomicAdd(&p.stats->batches, batches);
    atomicAdd(&p.stats->groups, batches);
    atomicAdd(&p.stats->busy_cycles, busy);
    atomicAdd(&p.stats->lock_cycles, locked);
  }
}

// ---- setup and dump kernels
template <int NS>
__global__ void init_kv_rings(KParams p, const uint32_t* keys, const uint32_t* vals, const uint32_t* lru,
                              const uint32_t* clocks) {
  const uint64_t i = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x;
  if (i == 0) *p.gts = 0;
  if (i >= p.kv_S) return;
  const uint64_t E = (uint64_t)kEmptyTs << 32;
  for (int j = 0; j < NS; ++j) {
#pragma unroll
    for (int w = 0; w < 4; ++w) p.kv_key[(i * NS + j) * 4 + w] = j ? E : (uint64_t)keys[i * 4 + w];
#pragma unroll
    for (int w = 0; w < 8; ++w) p.kv_val[(i * NS + j) * 8 + w] = j ? E : (uint64_t)vals[i * 8 + w];
    p.kv_lru[i * NS + j] = j ? E : (uint64_t)lru[i];
    if (i < p.kv_T) p.kv_clk[i * NS + j] = j ? E : (uint64_t)clocks[i];
  }
}

template <int NS, int W>
__device__ __forceinline__ void newest_words(const uint64_t* ring, uint32_t* out) {
  int best = -1;
  uint32_t bts = 0;
  for (int j = 0; j < NS; ++j) {
    const uint32_t ts = (uint32_t)(ring[j * W] >> 32);
    if (ts != kEmptyTs && (best < 0 || ts > bts)) {
      best = j;
      bts = ts;
    }
  }
  for (int w = 0; w < W; ++w) out[w] = (uint32_t)ring[best * W + w];
}

template <int NS>
__global__ void kv_newest(KParams p, uint32_t* keys, uint32_t* vals, uint32_t* lru, uint32_t* clocks) {
  const uint64_t i = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x;
  if (i >= p.kv_S) return;
  newest_words<NS, 4>(p.kv_key + i * NS * 4, keys + i * 4);
  newest_words<NS, 8>(p.kv_val + i * NS * 8, vals + i * 8);
  newest_words<NS, 1>(p.kv_lru + i * NS, lru + i);
  if (i < p.kv_T) newest_words<NS, 1>(p.kv_clk + i * NS, clocks + i);
}

__global__ void gen_kv_descs_kernel(GenParams g, uint64_t tx0, uint64_t n, uint32_t* out) {
  const uint64_t i = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x;
  if (i >= n) return;
  const KvTx d = gen_kv(g, tx0 + i);
  uint32_t* o = out + i * 10;
  o[0] = d.is_update;
  o[1] = d.key;
  for (int j = 0; j < 8; ++j) o[2 + j] = d.val[j];
}

}  // namespace csmvd
