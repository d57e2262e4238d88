// client_kv.cuh -- the client warp of the MemcachedGPU workload.
//
// CSMV_KV_POLL_PREFETCH (A/B, default 0): poll the response with a load
// issued one GET step ahead instead of a blocking load per step.  It
// answers ~5 us sooner, yet C4 loses ~20 %: warps whose batch returns early
// start their next round (and re-scan the hot sets) sooner, and the herd on
// a hot set grows (tools/chain.py: restart 6.6 -> 16.9 us per link).
#ifndef CSMV_KV_POLL_PREFETCH
#define CSMV_KV_POLL_PREFETCH 0
#endif
// Same lane state machine and round phases as client_bank.cuh; GET is the
// read-only transaction, PUT the update transaction (docs/GENERATOR.md 4).
//
// Read-set representation.  By default (and always above kKvFullWays ways,
// up to 256) a PUT's read/write set is shipped as {set clock} u WS;
// with CSMV_DBG_KV_ITEMSETS (A <= 16) it is tracked item by item (smem
// scratch) and shipped whole, the paper's literal form.  The two decide
// identically: every item a PUT reads lies in its set t,
// every PUT on set t reads and writes clock[t], and nothing else writes an
// item of set t, so "a commit after s wrote an item of RS u WS" holds iff
// "a commit after s wrote clock[t]" -- validation and
// pre-validation (two PUTs conflict iff same set) decide exactly as
// with the full sets (DESIGN.md readings; the 1-warp tests compare both
// against the item-level reference predictor).
#pragma once

namespace csmvd {

// GET(k) at snapshot s: scan set(k), stop at the matching key (then read
// its value) or at the first empty way; never touches LRU.
template <int NS>
__device__ __forceinline__ int kv_get(const KParams& p, uint32_t key, uint32_t s, uint64_t& dg, uint32_t& hit) {
  const uint32_t K = p.K, S = p.kv_S, A = p.kv_A;
  uint32_t gk[4];
  kv_key16(key, gk);
  const uint32_t gset = kv_set(key, p.kv_T);
  dg = 0;
  hit = 0;
  // U ways in flight per lane (the scan stops at a match or an empty way;
  // the over-read of at most U-1 ways is the price of U x fewer round trips)
  constexpr int U = NS <= 4 ? 4 : (NS == 8 ? 2 : 1);
  for (uint32_t w0 = 0; w0 < A; w0 += U) {
    Ring<4> r[U][NS];
#pragma unroll
    for (int u = 0; u < U; ++u) {
      if (w0 + u < A) {
        const uint64_t* ring = p.kv_key + (size_t)(gset * A + w0 + u) * NS * 4;
#pragma unroll
        for (int j = 0; j < NS; ++j) r[u][j] = ld_ring<4>(ring + j * 4);
      }
    }
#pragma unroll
    for (int u = 0; u < U; ++u) {
      if (w0 + u >= A) break;
      const uint32_t slot = gset * A + w0 + u;
      uint32_t k4[4];
      int rr = kv_key_pick<NS>(p.kv_key + (size_t)slot * NS * 4, r[u], K, s, true, k4);
      if (rr != RD_OK) return rr;
#pragma unroll
      for (int j = 0; j < 4; ++j) dg += dig_word(slot, j, k4[j]);
      if (k4[0] == gk[0] && k4[1] == gk[1] && k4[2] == gk[2] && k4[3] == gk[3]) {
        uint32_t val[8];
        rr = kv_read_mw<NS, 8>(p.kv_val + (size_t)slot * NS * 8, K, s, true, val);
        if (rr != RD_OK) return rr;
#pragma unroll
        for (int j = 0; j < 8; ++j) dg += dig_word(S + slot, j, val[j]);
        hit = w0 + u + 1;
        return RD_OK;
      }
      if (!(k4[0] | k4[1] | k4[2] | k4[3])) return RD_OK;
    }
  }
  return RD_OK;
}

template <int NS>
__device__ void client_warp_kv(const KParams& p, uint64_t t_begin, uint32_t* scratch) {
  const uint32_t FULL = 0xFFFFFFFFu;
  const uint32_t lane = threadIdx.x & 31, wib = threadIdx.x >> 5;
  const uint32_t cw = wib * p.n_client_ctas + (blockIdx.x - p.n_server_ctas);
  if (cw >= p.n_cw) return;
  const uint64_t T = (uint64_t)p.n_cw * 32;
  uint64_t cu = kNoTx;
  uint64_t dk_id = kNoTx;  // cu whose key dk_key holds
  uint32_t dk_key = 0;
  uint64_t cr = (uint64_t)cw * 32 + lane;
  uint32_t att_u = 0, att_r = 0, hold = 0, n_srv_ab = 0;
  ClientCounters cc;
  uint32_t round = 0;
  const uint32_t K = p.K, S = p.kv_S, A = p.kv_A, Tn = p.kv_T;
  const uint32_t lt = lanemask_lt();
  const uint32_t streak = p.ro_streak;
  const bool compact = A > kKvFullWays || !(p.debug & CSMV_DBG_KV_ITEMSETS);
  PhaseClock pc((p.debug & CSMV_DBG_PHASES) != 0);
  Jitter jit(p, 1);
  const bool tracing = (p.debug & CSMV_DBG_TRACE) != 0;
  // per-warp smem scratch, lane-minor: RS[kKvMaxRs][32], WS[4][32], NRS[32]
  uint32_t* RS = scratch + (size_t)wib * 32 * (kKvMaxRs + 5);
  uint32_t* WS = RS + kKvMaxRs * 32;
  uint32_t* NRS = WS + 4 * 32;
  uint32_t* my_ids = p.req_ids + (size_t)cw * p.maxid * 32;

  for (;;) {
    if (!__any_sync(FULL, cu != kNoTx || cr < p.n_tx)) break;
    pc.start();
    ++round;
    ++cc.n_rounds;
    const uint64_t t_rb = tracing ? globaltimer() : 0;
    uint64_t t_sub = 0;
    uint32_t s = 0, err = 0;
    if (lane == 0) {
      s = ld_acquire(p.gts);  // TXBegin
      err = ld_relaxed(&p.ctl->error);
    }
    s = __shfl_sync(FULL, s, 0);
    if (__shfl_sync(FULL, err, 0)) break;

    // ---- A: the pending PUT reads at s (read-set tracked)
    int status = ST_NONE;
    KvTx d{};
    uint32_t kk[4] = {0, 0, 0, 0};
    uint32_t victim = 0, tset = 0, clk = 0, nrs = 0;
    uint64_t rdig = 0;
    uint32_t need = 0;  // a PUT that met a version newer than s retries once GTS >= need
    if (cu == kNoTx && cr < p.n_tx && gen_is_update(p.gen, cr)) {
      cu = cr;
      cr += T;
    }
    bool pending = false;  // a PUT to read this round
    if (cu != kNoTx) {
      if (hold) {
        --hold;
        status = ST_ABORT;
      } else {
        if (dk_id != cu) {  // the pending PUT's key, drawn once (not every retry round)
          dk_key = gen_kv_key(p.gen, cu);
          dk_id = cu;
        }
        d = gen_kv_k(p.gen, cu, dk_key);
        kv_key16(d.key, kk);
        tset = kv_set(d.key, Tn);
        ++att_u;
        pending = true;
      }
    }
    // Pre-validation before the reads ({set clock} u WS requests): two PUTs
    // conflict iff they share a set, and the lowest lane of a set is the one
    // pre-validation keeps (Q5) -- so the others lose now, without
    // scanning a set they cannot commit in.  (A lower lane whose read then
    // fails no longer lets the next lane of its set in: only an extra abort.
    // With one client warp no read fails, so the deterministic schedule is
    // the same.)  On a hot set this removes every duplicate scan of its ~80
    // sectors per warp round.
    bool reader = pending;
    if (compact && !(p.debug & CSMV_DBG_NO_PREVAL)) {
      const uint32_t pm = __ballot_sync(FULL, pending);
      const uint32_t peers = __match_any_sync(FULL, pending ? tset : 0xFFFFFFFFu);
      reader = pending && (peers & pm & lt) == 0;
    }
    if (pending && !reader) {
      cc.abort(CSMV_AB_PREVAL, true);
      status = ST_ABORT;
    }
    if (reader) {
      {
        int r = RD_OK;
        uint32_t seen = 0;  // newest version timestamp the reads met
        victim = 0xFFFFFFFFu;
        // the set clock first: every PUT on the set writes it, so a PUT
        // committed after s on this set shows here after one load and the
        // scans are skipped (the abort is the same: the clock is in RS)
        if (compact) {
          r = kv_read_1<NS>(p.kv_clk + (size_t)tset * NS, K, s, clk, &seen);
          if (r == RD_OK) rdig += dig1(3 * S + tset, clk);
        }
        // key scan, U ways in flight (as in kv_get), stop at match or empty;
        // the ways loaded past the stop are not read (not in RS)
        constexpr int U = NS <= 4 ? 4 : (NS == 8 ? 2 : 1);
        for (uint32_t w0 = 0; w0 < A && victim == 0xFFFFFFFFu && r == RD_OK; w0 += U) {
          Ring<4> rk[U][NS];
#pragma unroll
          for (int u = 0; u < U; ++u) {
            if (w0 + u < A) {
              const uint64_t* ring = p.kv_key + (size_t)(tset * A + w0 + u) * NS * 4;
#pragma unroll
              for (int j = 0; j < NS; ++j) rk[u][j] = ld_ring<4>(ring + j * 4);
            }
          }
#pragma unroll
          for (int u = 0; u < U; ++u) {
            if (w0 + u >= A || victim != 0xFFFFFFFFu || r != RD_OK) break;
            const uint32_t slot = tset * A + w0 + u;
            uint32_t key[4];
            r = kv_key_pick<NS>(p.kv_key + (size_t)slot * NS * 4, rk[u], K, s, false, key, &seen);
            if (r != RD_OK) break;
            if (!compact) RS[nrs++ * 32 + lane] = slot;
#pragma unroll
            for (int j = 0; j < 4; ++j) rdig += dig_word(slot, j, key[j]);
            if ((key[0] == kk[0] && key[1] == kk[1] && key[2] == kk[2] && key[3] == kk[3]) ||
                !(key[0] | key[1] | key[2] | key[3]))
              victim = slot;
          }
        }
        if (r == RD_OK && victim == 0xFFFFFFFFu) {
          // LRU scan of the full set; a one-word ring needs one pass (a newer
          // version anywhere aborts the PUT anyway)
          constexpr int UL = 4;
          uint32_t best = 0;
          for (uint32_t w0 = 0; w0 < A && r == RD_OK; w0 += UL) {
            Ring<NS> rl[UL];
#pragma unroll
            for (int u = 0; u < UL; ++u)
              if (w0 + u < A) rl[u] = ld_ring<NS>(p.kv_lru + (size_t)(tset * A + w0 + u) * NS);
#pragma unroll
            for (int u = 0; u < UL; ++u) {
              if (w0 + u >= A) break;
              const uint32_t slot = tset * A + w0 + u;
              const Sel q = select_version<NS>(rl[u], s);
              seen = max(seen, q.newest);
              if (q.newest > s) {
                r = RD_NEWER;
                break;
              }
              if (q.best < 0 || (uint32_t)q.best >= K) {
                r = RD_MISS;
                break;
              }
              const uint32_t l = (uint32_t)slot_at<NS>(rl[u], q.best);
              if (!compact) RS[nrs++ * 32 + lane] = 2 * S + slot;
              rdig += dig1(2 * S + slot, l);
              if (w0 + u == 0 || l < best) {
                best = l;
                victim = slot;
              }
            }
          }
        }
        if (r == RD_OK && !compact) {
          r = kv_read_1<NS>(p.kv_clk + (size_t)tset * NS, K, s, clk, &seen);
          if (r == RD_OK) {
            RS[nrs++ * 32 + lane] = 3 * S + tset;
            rdig += dig1(3 * S + tset, clk);
          }
        }
        if (r == RD_NEWER) {
          need = seen;  // retry once GTS covers the newer version (its commit is then visible)
          cc.abort(CSMV_AB_EARLY, true);
          status = ST_ABORT;
          if (p.backoff_max) hold = min(p.backoff_max, 1u << min(n_srv_ab++, 8u));
        } else if (r == RD_MISS) {
          need = s + 1;  // every version <= s is recycled: only a newer snapshot can read it
          cc.abort(CSMV_AB_VERSION, true);
          status = ST_ABORT;
        } else {
          if (!compact) {
            WS[0 * 32 + lane] = victim;
            WS[1 * 32 + lane] = S + victim;
            WS[2 * 32 + lane] = 2 * S + victim;
            WS[3 * 32 + lane] = 3 * S + tset;
            NRS[lane] = nrs;
          }
          status = ST_CAND;
        }
      }
    }
    __syncwarp();
    pc.mark(PH_READ);
    jit();  // versions read, not yet validated

    // ---- B: pre-validation: lane j is dropped if WS_i n (RS_j u WS_j)
    // or WS_j n RS_i is non-empty for an earlier kept lane i
    const uint32_t cand = __ballot_sync(FULL, status == ST_CAND);
    uint32_t kept = cand;
    if (!(p.debug & CSMV_DBG_NO_PREVAL) && compact) {
      kept = 0;
      uint32_t rem = cand;
      while (rem) {  // same set <=> conflicting read/write sets
        const int i = __ffs(rem) - 1;
        kept |= 1u << i;
        const uint32_t ti = __shfl_sync(FULL, tset, i);
        rem &= ~__ballot_sync(FULL, ((rem >> lane) & 1u) && lane > (uint32_t)i && tset == ti) & ~(1u << i);
      }
    } else if (!(p.debug & CSMV_DBG_NO_PREVAL)) {
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
    pc.mark(PH_PREVAL);
    if (kept && mine && compact) {
      my_ids[0 * 32 + lane] = (3 * S + tset) | kWriteBit;  // read and written: stands for the set
      my_ids[1 * 32 + lane] = victim | kWriteBit;
      my_ids[2 * 32 + lane] = (S + victim) | kWriteBit;
      my_ids[3 * 32 + lane] = (2 * S + victim) | kWriteBit;
      p.req_cnt[(size_t)cw * 32 + lane] = 4;
    } else if (kept && mine) {
      // request ids: RS u WS (bit 31: in WS)
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
    if (kept) {
      if (lane == 0) {
        p.req_hdr[cw].snapshot = s;
        p.req_hdr[cw].mask = kept;
        p.req_hdr[cw].round = round;
      }
      __syncwarp();
      fence_gpu();
      jit();  // payload written, doorbell not yet
      if (lane == 0) st_relaxed(&p.req_seq[cw], round);
      if (tracing) t_sub = globaltimer();
      pc.mark(PH_SUBMIT);
    }

    // ---- C: GETs at s while the batch is at the server, one
    // per active lane per step.  ro_adaptive ends the run early, warp-wide:
    // once the server has answered the warp's batch; with ro_adaptive = 2
    // also -- when the warp submitted nothing because its PUTs read versions
    // newer than s -- as soon as GTS covers the newest of those versions (a
    // retry can then read them).
    {
      const bool blocked = cu != kNoTx && status == ST_ABORT && need != 0;
      uint32_t need_min = blocked ? need : 0xFFFFFFFFu;
      need_min = __reduce_min_sync(FULL, need_min);
      bool run = streak || cu == kNoTx;
      const uint32_t lim = streak ? streak : 1u;
      uint64_t pf = 0;  // CSMV_KV_POLL_PREFETCH: the response's first word, prefetched one GET step ahead
      (void)pf;
      for (uint32_t n_ro = 0; n_ro < lim; ++n_ro) {
        bool has = run && cr < p.n_tx && !gen_kv_is_update(p.gen, cr);  // an update: the next round adopts it
        if (!__any_sync(FULL, has)) break;
        if (has) {
          const KvTx g = gen_kv(p.gen, cr);
          ++att_r;
          uint64_t dg;
          uint32_t hit;
          if (kv_get<NS>(p, g.key, s, dg, hit) != RD_OK) {
            cc.abort(CSMV_AB_VERSION, false);  // retried next round
            run = false;
          } else {
            if (p.log_mode) log_commit(p, cr, s, 0, att_r, dg, hit);
            ++cc.c_ro;
            cc.ro_ck ^= dg;
            cr += T;
            att_r = 0;
          }
        }
        if (p.ro_adaptive) {
          if (kept) {
#if CSMV_KV_POLL_PREFETCH
            if (__shfl_sync(FULL, (uint32_t)(pf >> 32), 0) == round) break;
            if (lane == 0) pf = ld_relaxed64(&p.resp[cw].base);
#else
            if ((uint32_t)(warp_ld_relaxed64(&p.resp[cw].base) >> 32) == round) break;
#endif
          }
          if (p.ro_adaptive >= 2 && !kept && need_min != 0xFFFFFFFFu && warp_ld_relaxed(p.gts) >= need_min) break;
        }
      }
    }
    __syncwarp();
    pc.mark(PH_ROT);
    if (!kept) continue;

    // ---- D: response, write-back, GTS
    uint32_t base = 0, cmask = 0, omask = 0;
    wait_response(p, cw, round, t_begin, base, cmask, omask, jit);
    const uint64_t t_resp = tracing ? globaltimer() : 0;
    if (p.commit == CSMV_COMMIT_ONLYCS) fence_gpu();  // acquire: the server's write-backs
    pc.mark(PH_WAIT);
    uint32_t cts = 0;
    jit();  // committed, versions not yet written back
    if (mine) {
      if ((cmask >> lane) & 1u) {
        // Client-side write-back: the paper's 4 writes.
        cts = base + __popc(cmask & lt);
        const uint32_t cn = clk + 1;
        // the four rings' slot timestamps in one round trip, then the stores
        uint64_t* rk = p.kv_key + (size_t)victim * NS * 4;
        uint64_t* rv = p.kv_val + (size_t)victim * NS * 8;
        uint64_t* rl = p.kv_lru + (size_t)victim * NS;
        uint64_t* rc = p.kv_clk + (size_t)tset * NS;
        uint32_t tk[NS], tv[NS], tl[NS], tc[NS];
        kv_ring_ts<NS, 4>(rk, K, tk);
        kv_ring_ts<NS, 8>(rv, K, tv);
        kv_ring_ts<NS, 1>(rl, K, tl);
        kv_ring_ts<NS, 1>(rc, K, tc);
        const uint32_t cn1[1] = {cn};
        kv_install<NS, 4>(rk, tk, K, cts, kk);
        kv_install<NS, 8>(rv, tv, K, cts, d.val);
        kv_install<NS, 1>(rl, tl, K, cts, cn1);
        kv_install<NS, 1>(rc, tc, K, cts, cn1);
        if (p.log_mode) {
          uint64_t wd = dig1(2 * S + victim, cn) + dig1(3 * S + tset, cn);
#pragma unroll
          for (int j = 0; j < 4; ++j) wd += dig_word(victim, j, kk[j]);
#pragma unroll
          for (int j = 0; j < 8; ++j) wd += dig_word(S + victim, j, d.val[j]);
          log_commit(p, cu, s, cts, att_u, rdig, wd);
        }
        ++cc.c_upd;
        cu = kNoTx;
        att_u = 0;
        n_srv_ab = 0;
      } else {
        const bool ovf = (omask >> lane) & 1u;
        cc.abort(ovf ? CSMV_AB_OVERFLOW : CSMV_AB_CONFLICT, true);
        if (!ovf && p.backoff_max) hold = min(p.backoff_max, 1u << min(n_srv_ab++, 8u));
      }
    }
    __syncwarp();
    pc.mark(PH_WRITEBACK);
    const uint32_t n = __popc(cmask);
    if (n) {
      jit();  // write-backs done, commit not yet published
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
    pc.mark(PH_PUBLISH);
    if (tracing && cts && tset == p.trace_item)
      trace_commit(p, cts, s, t_rb, t_sub, t_resp, globaltimer());
  }
  client_flush(p, cc);
  pc.flush(p);
}

}  // namespace csmvd
