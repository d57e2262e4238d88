// client_kv.cuh -- the client warp of the MemcachedGPU workload.
//
// Same lane state machine and round phases as client_bank.cuh; GET is the
// read-only transaction, PUT the update transaction (docs/GENERATOR.md 4).
//
// Trace diagnostics (build knobs, CSMV_NVCC_EXTRA; CSMV_DBG_TRACE runs):
// CSMV_TRACE_SNAP_LATE stamps t_snap when the PUT read starts instead of
// after the snapshot; CSMV_TRACE_COOP_SPLIT when the cooperative read's
// loads have arrived; CSMV_TRACE_EVAL_END makes t_read the end of the first
// reader's evaluation (profiles/r02/raw/r02be_c4_chain_eval_split.txt).
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
// Resumable, one memory round trip per call, so that the warp can poll its
// response / GTS / ticket between trips (phase C): a GET in progress is
//   vslot == 0: the key scan, next way w0 (U ways in flight per call; the
//               over-read of at most U-1 ways past the stop is not read)
//   vslot != 0: the value of the matching slot vslot - 1 is next.
struct KvGet {
  uint32_t gk[4];
  uint32_t gset, w0, vslot, hit;
  uint64_t dg;
};

template <int NS>
__device__ __forceinline__ void kv_get_start(const KParams& p, uint32_t key, KvGet& g) {
  kv_key16(key, g.gk);
  g.gset = kv_set(key, p.kv_T);
  g.w0 = g.vslot = g.hit = 0;
  g.dg = 0;
}

// One step of a GET, split in two so that the warp can look at its polls
// (issued before the step's loads) while the loads are in flight:
// kv_get_issue puts the step's loads in flight into rb, kv_get_finish
// evaluates them; fin = the GET is complete (g.dg, g.hit final).
#ifndef CSMV_KV_GET_U
#define CSMV_KV_GET_U 2  // key ways per GET step at NS <= 4 (build knob for A/B: 2 beats 4 by ~12 % on C4, fewer spills)
#endif
template <int NS>
struct KvStep {
  static constexpr int U = NS <= 4 ? CSMV_KV_GET_U : (NS == 8 ? 2 : 1);  // key ways per step
  static constexpr int R = U * NS;                           // Ring<4> registers per step
  static constexpr bool kValOne = 2 * NS <= R;               // the value ring fits: one trip
};

template <int NS>
__device__ __forceinline__ void kv_get_issue(const KParams& p, const KvGet& g, Ring<4> (&rb)[KvStep<NS>::R]) {
  constexpr int U = KvStep<NS>::U;
  const uint32_t A = p.kv_A;
  if (g.vslot) {  // the whole value ring (8-word versions as two 4-word halves)
    if constexpr (KvStep<NS>::kValOne) {
      const uint64_t* ring = p.kv_val + (size_t)(g.vslot - 1) * NS * 8;
#pragma unroll
      for (int j = 0; j < 2 * NS; ++j) rb[j] = ld_ring<4>(ring + j * 4);
    }
    return;
  }
#pragma unroll
  for (int u = 0; u < U; ++u) {
    if (g.w0 + u < A) {
      const uint64_t* ring = p.kv_key + (size_t)(g.gset * A + g.w0 + u) * NS * 4;
#pragma unroll
      for (int j = 0; j < NS; ++j) rb[u * NS + j] = ld_ring<4>(ring + j * 4);
    }
  }
}

template <int NS>
__device__ __forceinline__ int kv_get_finish(const KParams& p, uint32_t s, KvGet& g,
                                             const Ring<4> (&rb)[KvStep<NS>::R], bool& fin) {
  constexpr int U = KvStep<NS>::U;
  const uint32_t K = p.K, S = p.kv_S, A = p.kv_A;
  fin = false;
  if (g.vslot) {  // + a re-read of the chosen version if a newer one is present (kv_key_pick)
    const uint32_t slot = g.vslot - 1;
    const uint64_t* ring = p.kv_val + (size_t)slot * NS * 8;
    uint32_t val[8];
    int rr;
    if constexpr (KvStep<NS>::kValOne) {
      Ring<8> rv[NS];
#pragma unroll
      for (int j = 0; j < NS; ++j)
#pragma unroll
        for (int w = 0; w < 4; ++w) {
          rv[j].s[w] = rb[2 * j].s[w];
          rv[j].s[4 + w] = rb[2 * j + 1].s[w];
        }
      rr = kv_key_pick<NS, 8>(ring, rv, K, s, true, val);
    } else {
      rr = kv_read_mw<NS, 8>(ring, K, s, true, val);
    }
    if (rr != RD_OK) return rr;
#pragma unroll
    for (int j = 0; j < 8; ++j)  // the log's digest; unlogged: the value folded into the checksum
      g.dg = p.log_mode ? g.dg + dig_word(S + slot, j, val[j]) : g.dg ^ ((uint64_t)val[j] << (32 * (j & 1)));
    fin = true;
    return RD_OK;
  }
  const uint32_t w0 = g.w0;
#pragma unroll
  for (int u = 0; u < U; ++u) {
    if (w0 + u >= A) break;
    const uint32_t slot = g.gset * A + w0 + u;
    Ring<4> ru[NS];
#pragma unroll
    for (int j = 0; j < NS; ++j) ru[j] = rb[u * NS + j];
    uint32_t k4[4];
    const int rr = kv_key_pick<NS>(p.kv_key + (size_t)slot * NS * 4, ru, K, s, true, k4);
    if (rr != RD_OK) return rr;
    if (p.log_mode) {  // the log's digest of every key read (S14)
#pragma unroll
      for (int j = 0; j < 4; ++j) g.dg += dig_word(slot, j, k4[j]);
    }
    if (k4[0] == g.gk[0] && k4[1] == g.gk[1] && k4[2] == g.gk[2] && k4[3] == g.gk[3]) {
      g.hit = w0 + u + 1;
      g.vslot = slot + 1;  // the value next
      return RD_OK;
    }
    if (!(k4[0] | k4[1] | k4[2] | k4[3])) {
      fin = true;
      return RD_OK;
    }
  }
  g.w0 = w0 + U;
  fin = g.w0 >= A;
  return RD_OK;
}

// A PUT's read of its set t at snapshot s by the whole warp (compact
// requests, A <= 16 ways, NS <= 8; every lane calls it with the same t, kk),
// split in an issue and an evaluation half so that the reads of several PUTs
// can be in flight together: lane w < A loads way w's whole key ring, lane
// 31 the set clock's ring; the LRU stamps cost a second trip, only when no
// way stops the scan.  It decides exactly as the sequential scan (the
// reader's own loop in client_warp_kv): the clock first, then ways in order
// up to the first one that matches the key, is empty, or cannot be read at s
// (NEWER / MISS: the PUT aborts with that reason); ways past the stop are
// not read (not in the digest); with no stop, the LRU stamps of all ways,
// the victim being the first least recently used way.  One lane per way
// keeps the evaluation to a handful of warp-wide operations (its latency is
// on the hot set's commit chain).  Results are warp-uniform.
template <int NS>
struct KvCoopLd {
  Ring<4> kr[NS];
  Ring<NS> cr;
};

template <int NS>
__device__ __forceinline__ void kv_put_read_issue(const KParams& p, uint32_t t, KvCoopLd<NS>& ld) {
  const uint32_t lane = threadIdx.x & 31, A = p.kv_A;
  if (lane < A) {
    const uint64_t* ring = p.kv_key + (size_t)(t * A + lane) * NS * 4;
#pragma unroll
    for (int j = 0; j < NS; ++j) ld.kr[j] = ld_ring<4>(ring + j * 4);
  }
  if (lane == 31) ld.cr = ld_ring<NS>(p.kv_clk + (size_t)t * NS);
}

template <int NS>
__device__ __forceinline__ void kv_put_read_eval(const KParams& p, uint32_t s, uint32_t t, const uint32_t (&kk)[4],
                                                 const KvCoopLd<NS>& ld, int& st, uint32_t& seen, uint32_t& victim,
                                                 int& iv, int& ic, uint32_t& clk, uint64_t& rdig) {
  const uint32_t FULL = 0xFFFFFFFFu;
  const uint32_t lane = threadIdx.x & 31;
  const uint32_t K = p.K, S = p.kv_S, A = p.kv_A;
  const bool lead = lane < A;  // this lane's way
  const uint32_t slot = t * A + lane;
  // the clock (lane 31): status and replacement slot in one word
  int cst = RD_OK, cic = 0;
  uint32_t cval = 0, cseen = 0;
  if (lane == 31) cst = kv_read_clk<NS>(ld.cr, K, s, cval, cseen, cic);
  const uint32_t cw = __shfl_sync(FULL, ((uint32_t)cst << 8) | (uint32_t)cic, 31);
  cst = (int)(cw >> 8);
  ic = (int)(cw & 0xFFu);
  clk = __shfl_sync(FULL, cval, 31);
  victim = 0xFFFFFFFFu;
  iv = 0;
  rdig = 0;
  // this lane's way: kv_key_pick with rot = false, and the slot a new
  // version would replace (the key, value and LRU rings' timestamps agree)
  int cand = -1;
  uint32_t cts = 0, newest = 0, torn_max = 0, key[4] = {0u, 0u, 0u, 0u}, lts[NS];
  bool torn = false;
#pragma unroll
  for (int j = 0; j < NS; ++j) {
    lts[j] = kEmptyTs;
    if (!lead || (uint32_t)j >= K) continue;
    const uint32_t t0 = (uint32_t)(ld.kr[j].s[0] >> 32);
    lts[j] = t0;
    bool intact = true;
#pragma unroll
    for (int x = 0; x < 4; ++x) {
      const uint32_t tw = (uint32_t)(ld.kr[j].s[x] >> 32);
      intact &= tw == t0;
      if (tw != kEmptyTs) newest = max(newest, tw);
      if (tw <= s) torn_max = max(torn_max, tw);
    }
    if (!intact) {
      torn = true;
      continue;
    }
    if (t0 != kEmptyTs && t0 <= s && (cand < 0 || t0 > cts)) {
      cand = j;
      cts = t0;
#pragma unroll
      for (int x = 0; x < 4; ++x) key[x] = (uint32_t)ld.kr[j].s[x];
    }
  }
  const int wst = newest > s ? RD_NEWER : ((cand < 0 || (torn && torn_max > cts)) ? RD_MISS : RD_OK);
  const bool match = key[0] == kk[0] && key[1] == kk[1] && key[2] == kk[2] && key[3] == kk[3];
  const bool empty = !(key[0] | key[1] | key[2] | key[3]);
  const int my_iv = kv_install_slot<NS>(lts, K);
  const uint32_t stops = __ballot_sync(FULL, lead && (wst != RD_OK || match || empty));
  const uint32_t ws = stops ? (uint32_t)__ffs(stops) - 1 : A;  // the scan's last way (A: none)
  const bool rd = lead && lane <= ws;  // the ways read: 0..ws (all of them when nothing stopped the scan)
  seen = max(__shfl_sync(FULL, cseen, 31), __reduce_max_sync(FULL, rd ? newest : 0u));
  st = cst;
  if (cst != RD_OK) return;
  // the stopping way's status and replacement slot
  const uint32_t sw = __shfl_sync(FULL, ((uint32_t)wst << 8) | (uint32_t)my_iv, stops ? ws : 0);
  if (stops && (sw >> 8) != RD_OK) {
    st = (int)(sw >> 8);
    return;
  }
  const bool lg = p.log_mode != 0;  // the read digest exists for the log (S14) only
  uint64_t dg = 0;
  if (rd && lg) {
#pragma unroll
    for (int x = 0; x < 4; ++x) dg += dig_word(slot, x, key[x]);
  }
  uint32_t vw = ws;  // victim way
  iv = (int)(sw & 0xFFu);
  if (!stops) {  // LRU stamps of every way; the first least recently used way is the victim
    int lst = RD_OK;
    uint32_t l = 0xFFFFFFFFu, ln = 0;
    if (lead) {
      const Ring<NS> lr = ld_ring<NS>(p.kv_lru + (size_t)slot * NS);
      const Sel q = select_version<NS>(lr, s);
      ln = q.newest;
      if (q.newest > s) lst = RD_NEWER;
      else if (q.best < 0 || (uint32_t)q.best >= K) lst = RD_MISS;
      else l = (uint32_t)slot_at<NS>(lr, q.best);
    }
    seen = max(seen, __reduce_max_sync(FULL, ln));
    const uint32_t bad = __ballot_sync(FULL, lead && lst != RD_OK);
    if (bad) {
      st = __shfl_sync(FULL, lst, __ffs(bad) - 1);
      return;
    }
    if (lead && lg) dg += dig1(2 * S + slot, l);
    const uint32_t lmin = __reduce_min_sync(FULL, l);
    vw = (uint32_t)__ffs(__ballot_sync(FULL, lead && l == lmin)) - 1;
    iv = __shfl_sync(FULL, my_iv, vw);
  }
  if (lg) {  // the digest of everything read, summed over the warp
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) dg += __shfl_xor_sync(FULL, dg, o);
    rdig = dg + dig1(3 * S + t, clk);
  }
  victim = t * A + vw;
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
  // CSMV_RETRY_FIFO: the pending PUT's ticket of its set (taken at adoption)
  const bool tickets = p.kv_tk_next != nullptr;
  uint32_t tk = 0;
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
#ifndef CSMV_TRACE_SNAP_LATE
    const uint64_t t_snap = tracing ? globaltimer() : 0;
#else
    uint64_t t_snap = 0;
#endif

    // ---- A: the pending PUT reads at s (read-set tracked)
    int status = ST_NONE;
    uint32_t kk[4] = {0, 0, 0, 0};
    uint32_t victim = 0, tset = 0, clk = 0, nrs = 0;
    int iv = 0, ic = 0;  // ring slots the PUT's versions replace: key/value/LRU rings, clock ring
    uint64_t rdig = 0;
    uint32_t need = 0;  // a PUT that met a version newer than s retries once GTS >= need
    bool adopted = false;
    if (cu == kNoTx && cr < p.n_tx && gen_is_update(p.gen, cr)) {
      cu = cr;
      cr += T;
      adopted = true;
    }
    if (tickets) {
      // CSMV_RETRY_FIFO: a PUT takes its set's next ticket when adopted; the
      // lanes of the warp adopting PUTs on one set take consecutive tickets
      // in lane order with one atomic (the set's lowest such lane adds)
      const uint32_t am = __ballot_sync(FULL, adopted);
      if (am) {
        if (adopted && dk_id != cu) {
          dk_key = gen_kv_key(p.gen, cu);
          dk_id = cu;
        }
        const uint32_t ts = adopted ? kv_set(dk_key, Tn) : 0xFFFFFFFFu;
        const uint32_t peers = __match_any_sync(FULL, ts) & am;
        const uint32_t leader = adopted ? (uint32_t)__ffs(peers) - 1 : lane;
        uint32_t b = 0;
        if (adopted && lane == leader) b = atomicAdd(p.kv_tk_next + ts, (uint32_t)__popc(peers));
        b = __shfl_sync(FULL, b, leader);
        if (adopted) tk = b + __popc(peers & lt);
      }
    }
    bool pending = false;  // a PUT to read this round
    bool tkwait = false;   // CSMV_RETRY_FIFO: an earlier ticket of the set is still being served
    if (cu != kNoTx) {
      if (hold) {
        --hold;
        status = ST_ABORT;
      } else {
        if (dk_id != cu) {  // the pending PUT's key, drawn once (not every retry round)
          dk_key = gen_kv_key(p.gen, cu);
          dk_id = cu;
        }
        // only the key now: the value's draws wait for the write-back
        tset = kv_set(dk_key, Tn);
        if (tickets) {
          // the turn of this ticket: the previous one committed (its CTS in
          // the low word) -- read only once the snapshot covers that commit
          const uint64_t sv = ld_relaxed64(p.kv_tk_serv + tset);
          if ((uint32_t)(sv >> 32) != tk) {
            tkwait = true;
            status = ST_WAIT;
          } else if ((uint32_t)sv > s) {
            need = (uint32_t)sv;
            status = ST_WAIT;
          }
        }
        if (status != ST_WAIT) {
          kv_key16(dk_key, kk);
          ++att_u;
          pending = true;
        }
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
    // compact requests on sets of up to 16 ways: the warp reads each
    // reader's set together, one memory round trip per reader
    const bool coop = NS <= 8 && compact && A <= 16 && !(p.debug & CSMV_DBG_KV_SEQREAD);
    int r_c = RD_OK;
    uint32_t seen_c = 0;
    const uint32_t n_readers = __popc(__ballot_sync(FULL, reader));
#ifdef CSMV_TRACE_EVAL_END
    uint64_t t_eval_end = 0;
#endif
#ifdef CSMV_TRACE_SNAP_LATE
    t_snap = tracing ? globaltimer() : 0;
#endif
    if (coop) {
      // up to kCoopMax readers' sets in flight together, then evaluated one by one
#ifndef CSMV_KV_COOP_MAX
#define CSMV_KV_COOP_MAX 1
#endif
      constexpr int kCoopMax = CSMV_KV_COOP_MAX;
      uint32_t rem = __ballot_sync(FULL, reader);
      while (rem) {
        int rls[kCoopMax];
        uint32_t tss[kCoopMax];
        KvCoopLd<NS> ld[kCoopMax];
#pragma unroll
        for (int i = 0; i < kCoopMax; ++i) {
          rls[i] = rem ? __ffs(rem) - 1 : -1;
          rem &= rem - 1;
          tss[i] = rls[i] >= 0 ? __shfl_sync(FULL, tset, rls[i]) : 0u;
          if (rls[i] >= 0) kv_put_read_issue<NS>(p, tss[i], ld[i]);
        }
#ifdef CSMV_TRACE_COOP_SPLIT  // diagnostics: t_snap = the loads have arrived (t_read - t_snap = evaluation)
        if (tracing) {
          uint64_t x = ld[0].cr.s[0];
#pragma unroll
          for (int j = 0; j < NS; ++j) x ^= ld[0].kr[j].s[0] ^ ld[0].kr[j].s[1] ^ ld[0].kr[j].s[2] ^ ld[0].kr[j].s[3];
          x = __reduce_or_sync(FULL, (uint32_t)x) ;
          t_snap = globaltimer() + (x == 0x9u ? 1 : 0);
        }
#endif
#pragma unroll
        for (int i = 0; i < kCoopMax; ++i) {
          if (rls[i] < 0) break;
          uint32_t k4[4];
#pragma unroll
          for (int x = 0; x < 4; ++x) k4[x] = __shfl_sync(FULL, kk[x], rls[i]);
          int st_, iv_, ic_;
          uint32_t seen_, vic_, clk_;
          uint64_t dg_;
          kv_put_read_eval<NS>(p, s, tss[i], k4, ld[i], st_, seen_, vic_, iv_, ic_, clk_, dg_);
#ifdef CSMV_TRACE_EVAL_END  // diagnostics: t_read - t_snap = the first reader's evaluation
          if (tracing && i == 0) t_eval_end = globaltimer() + (vic_ == 0x12345u ? 1 : 0);
#endif
          if (lane == (uint32_t)rls[i]) {
            r_c = st_;
            seen_c = seen_;
            victim = vic_;
            iv = iv_;
            ic = ic_;
            clk = clk_;
            rdig = dg_;
          }
        }
      }
    }
    if (reader) {
      {
        int r = RD_OK;
        uint32_t seen = 0;  // newest version timestamp the reads met
        if (coop) {
          r = r_c;
          seen = seen_c;
        } else {
        victim = 0xFFFFFFFFu;
        // The set clock's whole ring (one 64-bit word per version: one
        // load, no re-read) travels with the first group of key ways.  It
        // is evaluated first: every PUT on the set writes it, so a PUT
        // committed after s on this set shows there and the rest of the
        // scan is skipped (the abort is the same: the clock is in RS).
        const Ring<NS> rcl = ld_ring<NS>(p.kv_clk + (size_t)tset * NS);
        bool clk_done = false;
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
          if (compact && !clk_done) {
            clk_done = true;
            r = kv_read_clk<NS>(rcl, K, s, clk, seen, ic);
            if (r != RD_OK) break;
            rdig += dig1(3 * S + tset, clk);
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
                !(key[0] | key[1] | key[2] | key[3])) {
              victim = slot;
              // the key, value and LRU rings of a slot are written together by
              // every PUT (same CTS, same replacement rule) from identical
              // initial rings, so their slot timestamps are identical and the
              // key ring read here fixes the slot all three versions replace
              uint32_t ts[NS];
#pragma unroll
              for (int j = 0; j < NS; ++j) ts[j] = (uint32_t)(rk[u][j].s[0] >> 32);
              iv = kv_install_slot<NS>(ts, K);
            }
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
                uint32_t ts[NS];  // the LRU ring's slot timestamps = the key and value rings' (above)
#pragma unroll
                for (int j = 0; j < NS; ++j) ts[j] = (uint32_t)(rl[u].s[j] >> 32);
                iv = kv_install_slot<NS>(ts, K);
              }
            }
          }
        }
        if (r == RD_OK && !compact) {
          r = kv_read_clk<NS>(rcl, K, s, clk, seen, ic);
          if (r == RD_OK) {
            RS[nrs++ * 32 + lane] = 3 * S + tset;
            rdig += dig1(3 * S + tset, clk);
          }
        }
        }  // sequential read
        if (r == RD_NEWER) {
          need = seen;  // retry once GTS covers the newer version (its commit is then visible)
          cc.abort(CSMV_AB_EARLY, true);
          status = ST_ABORT;
          if (p.backoff_max && !tickets) hold = min(p.backoff_max, 1u << min(n_srv_ab++, 8u));
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
#ifdef CSMV_TRACE_EVAL_END
    const uint64_t t_read = t_eval_end;
#else
    const uint64_t t_read = tracing ? globaltimer() : 0;
#endif
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
      put_req_id(p, my_ids + 0 * 32 + lane, (3 * S + tset) | kWriteBit, round);  // read and written: the set
      put_req_id(p, my_ids + 1 * 32 + lane, victim | kWriteBit, round);
      put_req_id(p, my_ids + 2 * 32 + lane, (S + victim) | kWriteBit, round);
      put_req_id(p, my_ids + 3 * 32 + lane, (2 * S + victim) | kWriteBit, round);
      p.req_cnt[(size_t)cw * 32 + lane] = 4;
      if (p.kv_swb) {  // what the server needs to write the four versions back
        const KvTx d = gen_kv_k(p.gen, cu, dk_key);
        uint32_t* r = my_ids + kSwbRow * 32 + lane;
#pragma unroll
        for (int j = 0; j < 4; ++j) r[j * 32] = kk[j];
#pragma unroll
        for (int j = 0; j < 8; ++j) r[(4 + j) * 32] = d.val[j];
        r[12 * 32] = clk + 1;
        r[13 * 32] = (uint32_t)iv | ((uint32_t)ic << 8);
        if (p.req_tagged) {  // no fence before the doorbell: the server checks this word instead
          uint32_t w[kSwbRows];
#pragma unroll
          for (int j = 0; j < 4; ++j) w[j] = kk[j];
#pragma unroll
          for (int j = 0; j < 8; ++j) w[4 + j] = d.val[j];
          w[12] = clk + 1;
          w[13] = (uint32_t)iv | ((uint32_t)ic << 8);
          st_relaxed(r + kSwbRows * 32, swb_check(round, w, 1));
        }
      }
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
      if (lane == 0) put_req_hdr(p, cw, s, kept, round);
      __syncwarp();
      if (!p.req_tagged) fence_gpu();  // tagged: the server checks the round in every word instead
      jit();  // payload written, doorbell not yet
      if (lane == 0) st_relaxed(&p.req_seq[cw], round);
      if (tracing) t_sub = globaltimer();
      pc.mark(PH_SUBMIT);
    }

    bool have_resp = false;
    uint32_t base = 0, cmask = 0, omask = 0;
    // ---- C: GETs at s while the batch is at the server: each
    // active lane runs up to lim GETs, one after another, ending its run at
    // its next update or a VERSION miss (the same GETs per round as one GET
    // per lane per step).  The lanes advance one memory round trip per
    // iteration, each on its own GET, and the warp polls between trips: with
    // ro_adaptive the run ends early, warp-wide, once the server has
    // answered the warp's batch; with ro_adaptive = 2 also -- when the warp
    // submitted nothing because its PUTs read versions newer than s -- as
    // soon as GTS covers the newest of those versions (a retry can then read
    // them); and (CSMV_RETRY_FIFO) when a waiting PUT's turn comes.  A GET
    // cut short is not an attempt: it runs again in a later round.
    {
      const bool blocked = cu != kNoTx && (status == ST_ABORT || status == ST_WAIT) && need != 0;
      uint32_t need_min = blocked ? need : 0xFFFFFFFFu;
      need_min = __reduce_min_sync(FULL, need_min);
      const bool any_tkwait = __any_sync(FULL, tkwait);
      const bool poll_gts = p.ro_adaptive >= 2 && !kept && need_min != 0xFFFFFFFFu;
      bool run = streak || cu == kNoTx;
      const uint32_t lim = streak ? streak : 1u;
      uint32_t n_ro = 0;  // GETs this lane completed this round
      bool act = false;   // a GET in progress
      bool idle = true;   // no GET ran this round
      KvGet g;
      for (;;) {
        if (!act && run && n_ro < lim && cr < p.n_tx && !gen_kv_is_update(p.gen, cr)) {
          kv_get_start<NS>(p, gen_kv_key(p.gen, cr), g);  // an update: the next round adopts it
          ++att_r;
          act = true;
        }
        if (!__any_sync(FULL, act)) break;
        idle = false;
        // this trip's polls, issued before its loads and looked at while
        // they are in flight: lanes 0-2 the three response words (the
        // answer is then complete: no further load), lane 0 GTS, waiting
        // PUTs their set's ticket word
        uint64_t pv = 0, sv = 0;
        if (p.ro_adaptive) {
          if (kept) {
            if (lane < 3) pv = ld_relaxed64(&p.resp[cw].base + lane);
          } else if (poll_gts && lane == 0) {
            pv = ld_relaxed(p.gts);
          }
        }
        if (tkwait) sv = ld_relaxed64(p.kv_tk_serv + tset);
        Ring<4> rb[KvStep<NS>::R];
        if (act) kv_get_issue<NS>(p, g, rb);
        if (p.ro_adaptive) {
          if (kept) {
            const uint64_t b = __shfl_sync(FULL, pv, 0), c = __shfl_sync(FULL, pv, 1), o = __shfl_sync(FULL, pv, 2);
            if ((uint32_t)(b >> 32) == round && (uint32_t)(c >> 32) == round && (uint32_t)(o >> 32) == round) {
              have_resp = true;
              base = (uint32_t)b;
              cmask = (uint32_t)c;
              omask = (uint32_t)o;
              break;
            }
          } else if (poll_gts && (uint32_t)__shfl_sync(FULL, pv, 0) >= need_min) {
            break;
          }
        }
        if (any_tkwait && __any_sync(FULL, tkwait && (uint32_t)(sv >> 32) == tk)) break;  // a turn came
        if (act) {
          bool fin;
          if (kv_get_finish<NS>(p, s, g, rb, fin) != RD_OK) {
            cc.abort(CSMV_AB_VERSION, false);  // retried next round
            run = false;
            act = false;
          } else if (fin) {
            if (p.log_mode) log_commit(p, cr, s, 0, att_r, g.dg, g.hit);
            ++cc.c_ro;
            cc.ro_ck ^= g.dg;
            cr += T;
            att_r = 0;
            act = false;
            ++n_ro;
          }
        }
      }
      if (act) --att_r;  // cut short: not an attempt
      // nothing to submit, read or wait on the server for: back off before
      // the next round's polls (CSMV_RETRY_FIFO lanes waiting for a turn)
      if (tickets && !kept && idle) __nanosleep(256);
    }
    __syncwarp();
    pc.mark(PH_ROT);
    if (!kept) continue;

    // ---- D: response (unless phase C's poll already has it), write-back, GTS
    if (!have_resp) wait_response(p, cw, round, t_begin, base, cmask, omask, jit);
    const uint64_t t_resp = tracing ? globaltimer() : 0;
    if (p.commit == CSMV_COMMIT_ONLYCS) fence_gpu();  // acquire: the server's write-backs
    pc.mark(PH_WAIT);
    uint32_t cts = 0;
    jit();  // committed, versions not yet written back
    if (mine) {
      if ((cmask >> lane) & 1u) {
        // Client-side write-back: the paper's 4 writes.
        const KvTx d = gen_kv_k(p.gen, cu, dk_key);  // the PUT's value
        cts = base + __popc(cmask & lt);
        // CSMV_RETRY_FIFO: hand the set to the next ticket, which reads once GTS covers cts
        if (tickets) st_relaxed64(p.kv_tk_serv + tset, ((uint64_t)(tk + 1) << 32) | cts);
        const uint32_t cn = clk + 1;
        if (!p.kv_swb) {  // (server write-back: the worker has written them and published)
          // stores only: the slots were fixed by the read (the rings are as
          // read -- nothing wrote the set after s: this commit validated)
          uint64_t* rk = p.kv_key + (size_t)victim * NS * 4;
          uint64_t* rv = p.kv_val + (size_t)victim * NS * 8;
          uint64_t* rl = p.kv_lru + (size_t)victim * NS;
          uint64_t* rc = p.kv_clk + (size_t)tset * NS;
          const uint32_t cn1[1] = {cn};
          kv_install_at<4>(rk, iv, cts, kk);
          kv_install_at<8>(rv, iv, cts, d.val);
          kv_install_at<1>(rl, iv, cts, cn1);
          kv_install_at<1>(rc, ic, cts, cn1);
        }
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
        if (!ovf && p.backoff_max && !tickets) hold = min(p.backoff_max, 1u << min(n_srv_ab++, 8u));
      }
    }
    __syncwarp();
    pc.mark(PH_WRITEBACK);
    const uint32_t n = p.kv_swb ? 0u : __popc(cmask);  // server write-back: published by the server
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
    // the key of the lane's next update, drawn now (a zipf pick: a few
    // dependent loads) rather than when the next round adopts it
    if (cu == kNoTx && cr < p.n_tx && dk_id != cr && gen_is_update(p.gen, cr)) {
      dk_key = gen_kv_key(p.gen, cr);
      dk_id = cr;
    }
    if (tracing && cts && tset == p.trace_item) {
      uint64_t tc, tv;
      trace_srv_times(p, cw, round, t_sub, tc, tv);
      trace_commit(p, cts, s, t_rb, t_sub, t_resp, globaltimer(), tc, tv, t_snap, t_read, n_readers, __popc(kept));
    }
  }
  client_flush(p, cc);
  pc.flush(p);
}

}  // namespace csmvd
