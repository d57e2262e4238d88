// client_bank.cuh -- the client warp of the Bank workload.
// Included by kernel.cu after the shared client helpers.
//
// Lane state: at most one pending update transaction `cu` and a read cursor
// `cr` over the lane's own transactions (static assignment: lane l of client
// warp w runs tx (32w + l) + k*T).  A round (one snapshot s):
//   A  TXBegin s <- GTS; the pending update (adopting the next transaction if
//      it is an update) reads its items at s;
//   B  client-side pre-validation and the batch submit;
//   C  read-only transactions at s while the batch is at the server
//      (P:69): ro_streak = 0 -> one transaction per lane per round (the
//      paper's model: only lanes without a pending update run one); R > 0 ->
//      up to R of them, running ahead of a pending update, stopping at the
//      next update;
//   D  the response, client write-back, GTS advance.
// An update rejected by the server may sit out `backoff` rounds
// (backoff_max > 0); its lane keeps running read-only transactions.
//
// Commit-protocol ablations:
//   CSMV_COMMIT_ONLYCS  B skips pre-validation and ships the new values; the
//                       server validates, inserts and writes back one
//                       transaction at a time (server_worker_onlycs);
//   CSMV_COMMIT_JVSTM   no server: B is replaced by jv_commit, each lane
//                       validating against the global ATR and reserving its
//                       CTS with a global CAS, then writing back and
//                       advancing GTS in CTS order itself (lane-divergent).
#pragma once

namespace csmvd {

constexpr uint64_t kNoTx = ~0ull;

// JVSTM-GPU commit of one transaction with snapshot s and RS = WS = {a, b}
// (JVSTM's lock-free commit ported per thread): validate against
// every record of the global ATR after s, reserve CTS t+1 with
// a CAS on the ATR tail t, re-validating the records that appeared when the
// CAS fails, then publish the write-set record at entry t+1.  Returns the
// CTS, or 0 with `reason` set (CONFLICT; OVERFLOW when the ring no longer
// holds every record after s; -1 if the run is being torn down).  Entry c is
// overwritten only by CTS c + R, which needs tail >= c + R; the tail is <= t
// throughout a scan that ends in a successful CAS at t, so t - s < R proves
// every record read was the one of its CTS.
__device__ __forceinline__ uint32_t jv_commit(const KParams& p, uint32_t s, uint32_t a, uint32_t b, int& reason,
                                              uint32_t& fails, uint64_t t_begin) {
  const uint32_t R = 1u << p.jv_log2, M = R - 1;
  uint32_t t = ld_acquire(&p.ctl->jv_tail);
  uint32_t q = s;
  for (;;) {
    if (t - s >= R) {
      reason = CSMV_AB_OVERFLOW;
      return 0;
    }
    for (uint32_t c = q + 1; c - 1 < t; ++c) {  // records (q, t]
      uint32_t it = 0;
      while (ld_acquire(p.jv_tag + (c & M)) != c) {
        if ((++it & 1023u) == 0 && (ld_relaxed(&p.ctl->error) || watchdog(p, t_begin, 6))) {
          reason = -1;
          return 0;
        }
        __nanosleep(32);
      }
      const uint64_t e = ld_relaxed64(p.jv_ws + (c & M));
      const uint32_t w0 = (uint32_t)e, w1 = (uint32_t)(e >> 32);
      if (!(p.debug & CSMV_DBG_NO_VALIDATE) && (w0 == a || w0 == b || w1 == a || w1 == b)) {
        reason = CSMV_AB_CONFLICT;
        return 0;
      }
    }
    const uint32_t old = atomicCAS(&p.ctl->jv_tail, t, t + 1);
    if (old == t) break;
    ++fails;
    q = t;
    t = old;
  }
  const uint32_t cts = t + 1;
  st_relaxed64(p.jv_ws + (cts & M), ((uint64_t)b << 32) | a);
  st_release(p.jv_tag + (cts & M), cts);
  return cts;
}

// ---------------------------------------------------------------------------
// CTA-level batches (csmv_workload.client_group = G > 1).  The active client
// warps of a CTA form groups of up to G warps (warps gG .. gG+G-1).  Each
// round, after its own pre-validation, a warp publishes the kept
// lanes' (src, dst) in shared memory; after a group barrier every lane that
// is still kept checks them against the kept lanes of every lower warp of
// its group and drops out (PREVAL) on any overlap -- a conservative greedy in
// (warp, lane) order: the lower warps' sets are their own kept sets, so a
// transaction may be dropped for a conflict with one that is itself dropped
// (only an extra abort; the submitted batch is conflict-free either way).
// Each warp still writes its own request slot; the group's first warp rings
// ONE doorbell for all of them, and the server commits the whole group in
// one step of its critical section (server_worker, G sub-batches probed
// together) and answers each warp in its own response slot.  Group rounds
// are lock-step: a named barrier (id 1 + g) at the top of the round (the
// group continues while any warp has work, and stops on an error seen by
// any), one after the kept sets are published, one after the payloads are
// fenced.  Everything after that (read-only transactions, the response,
// write-back, publish) is per warp as before.
// ---------------------------------------------------------------------------
struct Group {
  uint32_t size = 1;     // warps in this warp's group (1: per-warp batches)
  uint32_t pos = 0;      // this warp's position in it
  uint32_t bar = 0;      // named barrier id
  uint32_t* flags = nullptr;  // [size] per-warp words (top-of-round vote / kept masks)
  uint2* ids = nullptr;       // [size][32] kept lanes' (src, dst)
  __device__ __forceinline__ void sync() const {
    asm volatile("bar.sync %0, %1;" ::"r"(bar), "r"(size * 32) : "memory");
  }
  // OR of `v` over the group's warps (lane 0 of each contributes)
  __device__ __forceinline__ uint32_t vote_or(uint32_t v, uint32_t slot) const {
    if ((threadIdx.x & 31) == 0) flags[slot * 8 + pos] = v;
    sync();
    uint32_t r = 0;
    for (uint32_t k = 0; k < size; ++k) r |= ((volatile uint32_t*)flags)[slot * 8 + k];
    return r;
  }
};

__device__ __forceinline__ Group make_group(const KParams& p, uint8_t* smem) {
  Group g;
  const uint32_t G = p.group > 1 ? p.group : 1u;
  if (G == 1) return g;
  const uint32_t wib = threadIdx.x >> 5, cta = blockIdx.x - p.n_server_ctas;
  // active warps of this CTA: w with w * n_client_ctas + cta < n_cw
  uint32_t n_act = cta < p.n_cw ? (p.n_cw - cta + p.n_client_ctas - 1) / p.n_client_ctas : 0u;
  if (n_act > (uint32_t)kWarps) n_act = kWarps;
  const uint32_t gi = wib / G;
  g.size = min(G, n_act - gi * G);
  g.pos = wib % G;
  g.bar = 1 + gi;
  uint8_t* base = smem + (size_t)gi * (G * 32 * sizeof(uint2) + 3 * 8 * sizeof(uint32_t));
  g.ids = reinterpret_cast<uint2*>(base);
  g.flags = reinterpret_cast<uint32_t*>(base + G * 32 * sizeof(uint2));
  return g;
}

template <int NS>
__device__ void client_warp(const KParams& p, uint64_t t_begin, uint8_t* smem) {
  const uint32_t FULL = 0xFFFFFFFFu;
  const uint32_t lane = threadIdx.x & 31;
  const uint32_t cw = (threadIdx.x >> 5) * p.n_client_ctas + (blockIdx.x - p.n_server_ctas);
  if (cw >= p.n_cw) return;
  const Group grp = make_group(p, smem);
  const bool grouped = grp.size > 1;
  // CSMV_SERVER_PART (server_part.cuh): the servers this warp's last batch
  // prepared at, whose decide acknowledgements are outstanding
  const bool part = p.part_log2 != 0;
  uint32_t dec_mask = 0, dec_round = 0, smask = 0;
  auto wait_acks = [&]() {  // every server's decide of the previous batch was processed
    if (!dec_mask) return;
    uint32_t it = 0;
    for (;;) {
      uint32_t a = dec_round;
      if (lane < 32 && ((dec_mask >> lane) & 1u)) a = ld_acquire(p.mdack + (size_t)lane * p.mstride + cw);
      if (__all_sync(FULL, a == dec_round)) break;
      if ((++it & 255u) == 0) {
        uint32_t bad = 0;
        if (lane == 0) bad = ld_relaxed(&p.ctl->error) || watchdog(p, t_begin, 13);
        if (__shfl_sync(FULL, bad, 0)) break;
      }
      __nanosleep(32);
    }
    dec_mask = 0;
  };
  const uint64_t T = (uint64_t)p.n_cw * 32;
  uint64_t cu = kNoTx;                       // pending update
  uint64_t du_id = kNoTx;                    // cu's descriptor, drawn once (not every retry round)
  BankTx du{};
  uint64_t cr = (uint64_t)cw * 32 + lane;    // read cursor
  uint32_t att_u = 0, att_r = 0, hold = 0, n_srv_ab = 0;
  ClientCounters cc;
  uint32_t round = 0;
  uint32_t* my_ids = p.req_ids + (size_t)cw * 2 * 32;
  const uint32_t K = p.K;
  const uint32_t lt = lanemask_lt();
  const uint32_t streak = p.ro_streak;
  PhaseClock pc((p.debug & CSMV_DBG_PHASES) != 0);
  Jitter jit(p, 1);
  const bool tracing = (p.debug & CSMV_DBG_TRACE) != 0;

  for (;;) {
    const bool work = __any_sync(FULL, cu != kNoTx || cr < p.n_tx);
    if (grouped) {  // lock-step group round: go on while any warp has work, stop on any error
      uint32_t e = 0;
      if (lane == 0) e = ld_relaxed(&p.ctl->error);
      e = __shfl_sync(FULL, e, 0);
      const uint32_t v = grp.vote_or((work ? 1u : 0u) | (e ? 2u : 0u), 0);
      if (v != 1u) break;
    } else if (!work) {
      break;
    }
    pc.start();
    ++round;
    ++cc.n_rounds;
    const uint64_t t_rb = tracing ? globaltimer() : 0;
    uint64_t t_sub = 0;
    uint32_t s = 0, err = 0;
    if (lane == 0) {
      s = ld_acquire(p.gts);  // TXBegin: snapshot
      err = ld_relaxed(&p.ctl->error);
    }
    s = __shfl_sync(FULL, s, 0);
    if (!grouped && __shfl_sync(FULL, err, 0)) break;
    // the trace's snapshot/read stamps are a build option for the bank
    // client (CSMV_BANK_STAMPS): two more 64-bit values live across the
    // round cost C2 ~1-2 % (profiles/r02/raw/r02bc_ab_load_stamps.txt)
#ifdef CSMV_BANK_STAMPS
    const uint64_t t_snap = tracing ? globaltimer() : 0;
#else
    const uint64_t t_snap = 0;
#endif

    // ---- A: the pending update reads at s
    int status = ST_NONE;
    BankTx d{};
    Ring<NS> rs{}, rd{};
    uint32_t vs = 0, vd = 0;
    if (cu == kNoTx && cr < p.n_tx && gen_is_update(p.gen, cr)) {
      cu = cr;
      cr += T;
    }
    if (cu != kNoTx) {
      if (hold) {
        --hold;
        status = ST_ABORT;  // sitting out (backoff)
      } else {
        if (du_id != cu) {
          du = gen_bank(p.gen, cu);
          du_id = cu;
        }
        d = du;
        ++att_u;
        rs = ld_ring<NS>(p.rings + (size_t)d.src * NS);
        rd = ld_ring<NS>(p.rings + (size_t)d.dst * NS);
        const Sel qs = select_version<NS>(rs, s), qd = select_version<NS>(rd, s);
        if (qs.newest > s || qd.newest > s) {
          cc.abort(CSMV_AB_EARLY, true);  // a commit after s wrote it: validation must fail
          status = ST_ABORT;
          if (p.backoff_max) hold = min(p.backoff_max, 1u << min(n_srv_ab++, 8u));
        } else if (qs.best < 0 || qd.best < 0) {
          cc.abort(CSMV_AB_VERSION, true);
          status = ST_ABORT;
        } else {
          vs = (uint32_t)slot_at<NS>(rs, qs.best);
          vd = (uint32_t)slot_at<NS>(rd, qd.best);
          status = ST_CAND;
        }
      }
    }

#ifdef CSMV_BANK_STAMPS
    const uint64_t t_read = tracing ? globaltimer() : 0;
#else
    const uint64_t t_read = 0;
#endif
    pc.mark(PH_READ);
    jit();  // versions read, not yet validated
    if (p.commit == CSMV_COMMIT_JVSTM) {
      // ---- B': decentralized commit, every lane on its own
      if (status == ST_CAND) {
        int reason = 0;
        const uint32_t cts = jv_commit(p, s, d.src, d.dst, reason, cc.cas_fail, t_begin);
        pc.mark(PH_PREVAL);
        if (cts) {
          const uint32_t ns = vs - (uint32_t)d.amt, nd = vd + (uint32_t)d.amt;
          write_back<NS>(p.rings + (size_t)d.src * NS, rs, K, cts, ns);
          write_back<NS>(p.rings + (size_t)d.dst * NS, rd, K, cts, nd);
          pc.mark(PH_WRITEBACK);
          if (p.log_mode) {
            log_commit(p, cu, s, cts, att_u, dig1(d.src, vs) + dig1(d.dst, vd), dig1(d.src, ns) + dig1(d.dst, nd));
            if (p.log_mode == CSMV_LOG_FULL && p.max_vals >= 2) {
              p.vals[cu * p.max_vals] = vs;
              p.vals[cu * p.max_vals + 1] = vd;
            }
          }
          // in-order GTS advance by this thread
          uint32_t it = 0;
          while (ld_relaxed(p.gts) != cts - 1) {
            if ((++it & 1023u) == 0 && (ld_relaxed(&p.ctl->error) || watchdog(p, t_begin, 7))) break;
            __nanosleep(32);
          }
          st_release(p.gts, cts);
          pc.mark(PH_PUBLISH);
          ++cc.c_upd;
          cu = kNoTx;
          att_u = 0;
        } else if (reason >= 0) {
          cc.abort(reason, true);
        }
        status = ST_NONE;  // decided here: not a pre-validation loser below
      }
      __syncwarp();
      pc.mark(PH_DIVERGENCE);
    }
    // ---- B: pre-validation, greedy in lane order (RS = WS = {src, dst})
    const uint32_t cand = p.commit == CSMV_COMMIT_JVSTM ? 0u : __ballot_sync(FULL, status == ST_CAND);
    uint32_t kept = cand;
    if (!(p.debug & CSMV_DBG_NO_PREVAL) && p.commit == CSMV_COMMIT_CSMV) {
      kept = 0;
      uint32_t rem = cand;
      while (rem) {
        const int i = __ffs(rem) - 1;
        const uint32_t a = __shfl_sync(FULL, d.src, i), b = __shfl_sync(FULL, d.dst, i);
        kept |= 1u << i;
        const bool conf = ((rem >> lane) & 1u) && lane > (uint32_t)i &&
                          (d.src == a || d.src == b || d.dst == a || d.dst == b);
        rem &= ~__ballot_sync(FULL, conf) & ~(1u << i);
      }
    }
    uint32_t gkept = kept;  // grouped: the group submits iff any of its warps kept a lane
    uint32_t watch = cw;    // the response slot that tells the read-only run the batch is answered
    if (grouped) {
      // cross-warp pre-validation against the kept lanes of the lower warps
      grp.ids[grp.pos * 32 + lane] = make_uint2(d.src, d.dst);
      grp.vote_or(kept, 1);  // publishes `kept` in flags[8 + pos]; the barrier orders the ids too
      bool conf = false;
      if ((kept >> lane) & 1u) {
        for (uint32_t w = 0; w < grp.pos; ++w) {
          uint32_t mk = ((volatile uint32_t*)grp.flags)[8 + w];
          while (mk) {
            const uint32_t j = __ffs(mk) - 1;
            mk &= mk - 1;
            const uint2 o = grp.ids[w * 32 + j];
            conf |= d.src == o.x || d.src == o.y || d.dst == o.x || d.dst == o.y;
          }
        }
      }
      kept &= ~__ballot_sync(FULL, conf);
    }
    const bool mine = (kept >> lane) & 1u;
    if (status == ST_CAND && !mine) cc.abort(CSMV_AB_PREVAL, true);
    if (p.commit != CSMV_COMMIT_JVSTM) pc.mark(PH_PREVAL);
    if (grouped) {
      // every warp writes its header (mask possibly 0: the server reads all G
      // slots of a group); the first warp rings the group's doorbell after
      // every payload is fenced
      if (mine) {
        put_req_id(p, my_ids + lane, d.src | kWriteBit, round);
        put_req_id(p, my_ids + 32 + lane, d.dst | kWriteBit, round);
      }
      if (lane == 0) put_req_hdr(p, cw, s, kept, round);
      __syncwarp();
      if (!p.req_tagged) fence_gpu();  // tagged: the server checks the round in every word instead
      gkept = grp.vote_or(kept, 2);
      // the server answers the warps that submitted something; all warps of
      // the group watch the first of them, so their rounds stay aligned
      for (uint32_t k = 0; k < grp.size; ++k)
        if (((volatile uint32_t*)grp.flags)[16 + k]) {
          watch = cw + (k - grp.pos) * p.n_client_ctas;
          break;
        }
      jit();  // payloads written, doorbell not yet
      if (gkept && grp.pos == 0 && lane == 0) st_relaxed(&p.req_seq[cw], round);
      if (tracing) t_sub = globaltimer();
      pc.mark(PH_SUBMIT);
    } else if (kept) {
      if (part) wait_acks();  // the servers still read this slot for the previous decide
      if (mine) {
        put_req_id(p, my_ids + lane, d.src | kWriteBit, round);
        put_req_id(p, my_ids + 32 + lane, d.dst | kWriteBit, round);
        if (p.commit == CSMV_COMMIT_ONLYCS || p.bank_swb) {  // the server writes back
          uint32_t* rv = p.req_vals + (size_t)cw * 128 + lane;
          const uint32_t na = vs - (uint32_t)d.amt, nb = vd + (uint32_t)d.amt;
          rv[0] = na;
          rv[32] = nb;
          // the slots the versions replace, fixed by this read (nothing writes
          // either account before this commit: it validated)
          if (p.bank_swb) {
            const uint32_t sl = ring_victim<NS>(rs, K) | (ring_victim<NS>(rd, K) << 8);
            rv[64] = sl;
            if (p.req_tagged) rv[96] = bank_swb_check(round, na, nb, sl);  // no fence: the server checks it
          }
        }
      }
      if (lane == 0) put_req_hdr(p, cw, s, kept, round);
      __syncwarp();
      if (!p.req_tagged) fence_gpu();  // tagged: the server checks the round in every word instead
      jit();  // payload written, doorbell not yet
      if (part) {  // the servers owning an item of the batch; prepared one at a time, lowest first
        smask = __reduce_or_sync(FULL, mine ? (1u << part_owner(d.src, p.part_log2)) |
                                                  (1u << part_owner(d.dst, p.part_log2))
                                            : 0u);
        if (lane == (uint32_t)(__ffs(smask) - 1)) st_relaxed(p.mreq_seq + (size_t)lane * p.mstride + cw, round);
      } else if (lane == 0) {
        st_relaxed(&p.req_seq[cw], round);
      }
      if (tracing) t_sub = globaltimer();
      pc.mark(PH_SUBMIT);
    }

    // ---- D (as a step callable from inside C): the server's answer
    // (P:101), client write-back, GTS.  With ro_adaptive the read-only
    // phase polls for the answer at every row group and runs D right away,
    // so a commit is written back and published about one L2 round trip
    // after its answer instead of after the whole read-only phase -- the
    // step every hot-item chain link waits for (tools/chain.py).  Not in
    // the deterministic (fixed) mode: there D stays after C.
    uint32_t cts = 0;
    uint64_t t_resp = 0;
    bool d_done = false;
    auto phase_d = [&](uint32_t base, uint32_t cmask, uint32_t omask) {
      t_resp = tracing ? globaltimer() : 0;
      if (p.commit == CSMV_COMMIT_ONLYCS) fence_gpu();  // acquire: the server's write-backs
      pc.mark(PH_WAIT);
      jit();  // committed, versions not yet written back
      if (mine) {
        if ((cmask >> lane) & 1u) {
          // Client-side write-back with CTS = base + rank.
          cts = base + __popc(cmask & lt);
          const uint32_t ns = vs - (uint32_t)d.amt, nd = vd + (uint32_t)d.amt;
          if (p.commit != CSMV_COMMIT_ONLYCS && !p.bank_swb) {
            write_back<NS>(p.rings + (size_t)d.src * NS, rs, K, cts, ns);
            write_back<NS>(p.rings + (size_t)d.dst * NS, rd, K, cts, nd);
            // lastw (the item-indexed ATR's exact level, server.cuh): written
            // here, before this commit is published, so GTS = g implies lastw
            // of every commit <= g.  Two commits writing one item are ordered
            // (the later one's snapshot covers the earlier one), so plain
            // stores leave lastw at the latest.
            st_relaxed(p.lastw + d.src, cts);
            st_relaxed(p.lastw + d.dst, cts);
          }
          if (p.log_mode) {
            log_commit(p, cu, s, cts, att_u, dig1(d.src, vs) + dig1(d.dst, vd), dig1(d.src, ns) + dig1(d.dst, nd));
            if (p.log_mode == CSMV_LOG_FULL && p.max_vals >= 2) {
              p.vals[cu * p.max_vals] = vs;
              p.vals[cu * p.max_vals + 1] = vd;
            }
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
      const uint32_t n = p.bank_swb ? 0u : __popc(cmask);  // server write-back: published by the server
      if (n) {
        jit();  // write-backs done, commit not yet published
        if (p.publish == CSMV_PUBLISH_CLIENT) {
          // Advance GTS by n once every earlier commit is visible:
          // spin until GTS == first CTS - 1 ("GTS 1" = GTS+1).
          __syncwarp();
          fence_gpu();
          uint32_t it = 0;
          while (warp_ld_relaxed(p.gts) != base - 1) {
            if ((++it & 255u) == 0) {
              uint32_t bad = 0;
              if (lane == 0) bad = ld_relaxed(&p.ctl->error) || watchdog(p, t_begin, 2);
              if (__shfl_sync(FULL, bad, 0)) break;
            }
            __nanosleep(CSMV_SLEEP_PUB);
          }
          if (lane == 0) st_release(p.gts, base + n - 1);  // release also orders the write-backs
        } else if (cts && p.commit != CSMV_COMMIT_ONLYCS) {
          st_release(p.done_ring + (cts & ((1u << kDoneLog2) - 1)), cts);
        }
      }
      pc.mark(PH_PUBLISH);
      d_done = true;
    };
    // CSMV_SERVER_PART: prepare server by server in increasing order (the
    // first was rung with the batch), each with only the lanes every earlier
    // one accepted -- a transaction holding marks at lower servers never
    // waits on one that needs them, so two spanning transactions cannot keep
    // aborting each other (with all prepares at once, ~10^4 in-flight
    // transfers on 4K accounts livelocked: each held the mark the other
    // needed); then the CTS from the global counter and a decide at every
    // server prepared.  A state machine (p_sm: servers still to prepare, the
    // lowest one rung) that the read-only phase advances at every row group,
    // like the early D of the other servers.
    uint32_t p_ok = kept, p_om = 0, p_sm = smask, p_rung = smask & (0u - smask);
    auto part_vote = [&](uint32_t& v, uint32_t& o) -> bool {  // the current server's vote, if in
      uint64_t w = 0;
      if (lane < 2) w = ld_relaxed64(&p.mresp[(size_t)(__ffs(p_sm) - 1) * p.mstride + cw].base + lane);
      const uint64_t w1 = __shfl_sync(FULL, w, 1), w0 = __shfl_sync(FULL, w, 0);
      if ((uint32_t)(w0 >> 32) != round || (uint32_t)(w1 >> 32) != round) return false;
      v = (uint32_t)w0;
      o = (uint32_t)w1;
      return true;
    };
    auto part_advance = [&](uint32_t v, uint32_t o) {
      p_ok &= v;
      p_om |= o;
      p_sm &= p_sm - 1;
      if (p_sm && p_ok) {  // the next server, with the surviving lanes
        const uint32_t k = __ffs(p_sm) - 1;
        if (lane == 0) p.req_hdr[cw].mask = p_ok;
        __syncwarp();
        fence_gpu();
        if (lane == k) st_relaxed(p.mreq_seq + (size_t)k * p.mstride + cw, round);
        p_rung |= 1u << k;
        return;
      }
      uint32_t base = 0;
      if (lane == 0 && p_ok) {
        base = atomicAdd(&p.ctl->cts_next, (uint32_t)__popc(p_ok)) + 1;  // the one global CTS sequence
        // done-ring room (server publish): CTS c reuses flag c & mask only once GTS >= c - 2^20
        for (uint32_t it = 0; base + __popc(p_ok) > ld_relaxed(p.gts) + (1u << kDoneLog2); ++it) {
          if ((it & 255u) == 255u && (ld_relaxed(&p.ctl->error) || watchdog(p, t_begin, 15))) break;
          __nanosleep(64);
        }
      }
      base = __shfl_sync(FULL, base, 0);
      if (lane == 0) {
        st_relaxed64(p.mdec + 2 * (size_t)cw, ((uint64_t)round << 32) | base);
        st_relaxed64(p.mdec + 2 * (size_t)cw + 1, ((uint64_t)round << 32) | p_ok);
      }
      __syncwarp();
      fence_gpu();
      if ((p_rung >> lane) & 1u) st_relaxed(p.mdec_seq + (size_t)lane * p.mstride + cw, round);
      dec_mask = p_rung;
      dec_round = round;
      phase_d(base, p_ok, p_om & ~p_ok);
    };
    const bool early_d = p.ro_adaptive && kept && p.commit == CSMV_COMMIT_CSMV && !part;
    // ro_adaptive: the watched response slot's first word is prefetched by
    // lane 0 one row group ahead (its latency hides behind the group's own
    // loads; a blocking poll would add an L2 round trip to every group);
    // `answered` once it carries this round's tag
    uint64_t pf = 0;
    bool answered = false;
    const uint32_t wslot = kept ? cw : watch;
    // the word that says the batch was answered
    const uint64_t* wword = &p.resp[wslot].base;
    auto poll = [&]() {
      if (!p.ro_adaptive || !gkept || d_done || answered) return;
      if (part) {  // advance the partitioned protocol by one step if its current vote is in
        if (__shfl_sync(FULL, (uint32_t)(pf >> 32), 0) == round) {
          uint32_t v, o;
          if (part_vote(v, o)) {
            part_advance(v, o);
            pf = 0;
          }
        } else if (lane == 0) {
          pf = ld_relaxed64(&p.mresp[(size_t)(__ffs(p_sm) - 1) * p.mstride + cw].base);
        }
        return;
      }
      if (__shfl_sync(FULL, (uint32_t)(pf >> 32), 0) == round) {
        answered = true;
        uint32_t b0, c0, o0;
        if (early_d && try_response(p, cw, round, b0, c0, o0)) phase_d(b0, c0, o0);
      } else if (lane == 0) {
        pf = ld_relaxed64(wword);
      }
    };

    // ---- C: read-only transactions at s.  A lane runs
    // its next read-only transactions up to the next update (at most
    // ro_streak; one if 0, and only without a pending update); a version
    // miss ends its run (retried next round).  The warp runs them depth by
    // depth -- every lane's first, then every lane's second, ... -- each one
    // scanned by the whole warp (rot_coop), so a round is not as long as
    // its longest lane's run.
    {
      const uint32_t lim = streak ? streak : 1u;
      bool run = streak || cu == kNoTx;
      for (uint32_t n_ro = 0; n_ro < lim; ++n_ro) {
        BankTx r{};
        bool has = false;
        if (run && cr < p.n_tx) has = gen_bank_ro(p.gen, cr, r.start, r.len);
        const uint32_t act = __ballot_sync(FULL, has);
        if (!act) break;
        if (has) ++att_r;
        bool ok;
        int64_t rsum;
        uint64_t rdig;
        rot_coop<NS>(p, act, r.start, r.len, s, cr, ok, rsum, rdig, poll);
        if (has) {
          if (ok) {
            if (p.log_mode) log_commit(p, cr, s, 0, att_r, rdig, (uint64_t)rsum);
            ++cc.c_ro;
            cc.ro_ck ^= (uint64_t)rsum;
            cr += T;
            att_r = 0;
          } else {
            cc.abort(CSMV_AB_VERSION, false);  // retried next round
            run = false;
          }
        }
        run = run && has;
        // ro_adaptive: the batch has been answered -> finish the round
        poll();
        if (p.ro_adaptive && gkept && (d_done || answered)) break;
      }
    }
    __syncwarp();
    pc.mark(PH_ROT);
    if (!kept) continue;  // grouped: the server answers only the warps that submitted something

    // ---- D, unless the read-only phase already ran it
    if (!d_done && part) {
      for (uint32_t it = 0; !d_done;) {  // the rest of the protocol, blocking
        uint32_t v = 0, o = 0;
        if (part_vote(v, o)) {
          part_advance(v, o);
          continue;
        }
        if ((++it & 255u) == 0) {
          uint32_t bad = 0;
          if (lane == 0) bad = ld_relaxed(&p.ctl->error) || watchdog(p, t_begin, 14);
          if (__shfl_sync(FULL, bad, 0)) break;
        }
        __nanosleep(CSMV_SLEEP_RESP);
      }
    } else if (!d_done) {
      uint32_t base = 0, cmask = 0, omask = 0;
      wait_response(p, cw, round, t_begin, base, cmask, omask, jit);
      phase_d(base, cmask, omask);
    }
    if (tracing && cts && (d.src == p.trace_item || d.dst == p.trace_item)) {
      uint64_t tc, tv;
      trace_srv_times(p, cw, round, t_sub, tc, tv);
      trace_commit(p, cts, s, t_rb, t_sub, t_resp, globaltimer(), tc, tv, t_snap, t_read, 0, __popc(kept));
    }
  }
  if (part) wait_acks();  // the servers have processed our last decide before we count as done
  client_flush(p, cc);
  pc.flush(p);
}

}  // namespace csmvd
