// fused.cuh -- the fused persistent CSMV kernel for sm_100a: device code and
// launch templates, instantiated once per (workload kind, server kind) in
// fused_{bank,kv}_{cta,cl}.cu so that the four variants compile in parallel.
//
// One cooperative grid holds both roles of the paper's client-server split
// (P:99-105): CTAs 0..C-1 are the server (C = 1, the paper's one SM, or a
// thread-block cluster), the rest are client SMs.  Fusing the roles into one
// launch guarantees co-residency of a server that spins on its clients (the
// paper launches two kernels; separate kernels deadlock when a profiler
// serialises them).  CSMV_COMMIT_JVSTM launches clients only.
//
// Client warp, one round (client_bank.cuh / client_kv.cuh):
//   TXBegin     s <- GTS (one acquire load per warp round)
//   TXRead      newest version with ts <= s from the VBox ring
//   pre-validation of the warp's update lanes (shuffle/ballot)
//   submit the batch (request slot + doorbell)
//   read-only transactions at s while the batch is at the server
//   the response, client write-back of the new versions
//   ordered GTS advance by n (CSMV_PUBLISH_CLIENT) or a done
//   flag per CTS for the server publisher (CSMV_PUBLISH_SERVER)
//   aborted transactions retry with a fresh snapshot next round
//
// Server (server.cuh): a receiver warp per server CTA dispatches doorbells to
// worker warps; a worker validates whole batches (one lane per transaction,
// __ballot_sync) against the two-level item-indexed ATR (HBM lastw + smem
// recent-commit table; or the paper's list ATR), reserves consecutive CTS
// and records the write-sets inside a shared-memory ticket-locked critical
// section.  No global atomics on
// the commit path.
#pragma once
#include <cuda_runtime.h>

#include "kernel.cuh"
#include "ptx.cuh"

namespace csmvd {

enum : int { ST_NONE = 0, ST_RO_OK, ST_CAND, ST_UPD_OK, ST_ABORT, ST_WAIT };

// --------------------------------------------------------------------------
// VBox read (TXRead) and write-back
// --------------------------------------------------------------------------
struct Sel {
  int best;          // slot of the newest version with ts <= s, -1 if none
  uint32_t best_ts;
  uint32_t newest;   // largest ts present
};

template <int NS>
__device__ __forceinline__ Sel select_version(const Ring<NS>& r, uint32_t s) {
  Sel q{-1, 0u, 0u};
#pragma unroll
  for (int j = 0; j < NS; ++j) {
    uint32_t ts = (uint32_t)(r.s[j] >> 32);
    if (ts != kEmptyTs) {
      q.newest = max(q.newest, ts);
      if (ts <= s && (q.best < 0 || ts > q.best_ts)) {
        q.best = j;
        q.best_ts = ts;
      }
    }
  }
  return q;
}

template <int NS>
__device__ __forceinline__ uint64_t slot_at(const Ring<NS>& r, int j) {
  uint64_t v = r.s[0];
#pragma unroll
  for (int i = 1; i < NS; ++i) v = (j == i) ? r.s[i] : v;
  return v;
}

// Replace the first unused slot, else the oldest version.  The
// writer owns the item: the WW check orders all writers of an item
// and the ring is unchanged since this transaction read it.
// the slot a new version of ring r replaces: the first unused, else the oldest
template <int NS>
__device__ __forceinline__ int ring_victim(const Ring<NS>& r, uint32_t K) {
  int victim = -1;
#pragma unroll
  for (int j = 0; j < NS; ++j) {
    uint32_t ts = (uint32_t)(r.s[j] >> 32);
    if ((uint32_t)j < K && victim < 0 && ts == kEmptyTs) victim = j;
  }
  if (victim < 0) {
    victim = 0;
    uint32_t vts = (uint32_t)(r.s[0] >> 32);
#pragma unroll
    for (int j = 1; j < NS; ++j) {
      uint32_t ts = (uint32_t)(r.s[j] >> 32);
      if ((uint32_t)j < K && ts < vts) {
        victim = j;
        vts = ts;
      }
    }
  }
  return victim;
}

template <int NS>
__device__ __forceinline__ void write_back(uint64_t* ring, const Ring<NS>& r, uint32_t K,
                                           uint32_t cts, uint32_t val) {
  int victim = -1;
  uint32_t vts = kEmptyTs;
#pragma unroll
  for (int j = 0; j < NS; ++j) {
    uint32_t ts = (uint32_t)(r.s[j] >> 32);
    if ((uint32_t)j < K && victim < 0 && ts == kEmptyTs) victim = j;
  }
  if (victim < 0) {
    victim = 0;
    vts = (uint32_t)(r.s[0] >> 32);
#pragma unroll
    for (int j = 1; j < NS; ++j) {
      uint32_t ts = (uint32_t)(r.s[j] >> 32);
      if ((uint32_t)j < K && ts < vts) {
        victim = j;
        vts = ts;
      }
    }
  }
  st_relaxed64(ring + victim, ((uint64_t)cts << 32) | val);
}

// one relaxed load by lane 0, broadcast: keeps spin loops warp-uniform
__device__ __forceinline__ uint32_t warp_ld_relaxed(const uint32_t* p) {
  uint32_t v = 0;
  if ((threadIdx.x & 31) == 0) v = ld_relaxed(p);
  return __shfl_sync(0xFFFFFFFFu, v, 0);
}

__device__ __forceinline__ uint64_t warp_ld_relaxed64(const uint64_t* p) {
  uint64_t v = 0;
  if ((threadIdx.x & 31) == 0) v = ld_relaxed64(p);
  return __shfl_sync(0xFFFFFFFFu, v, 0);
}

__device__ __forceinline__ bool watchdog(const KParams& p, uint64_t t0, uint32_t where);

// CSMV_DBG_JITTER: race widening.  A warp-private counter-based stream
// (seeded by the run's seed and the warp's global index, the same in every
// lane, so the sleep is warp-uniform) draws a delay of 0..2047 ns at each
// protocol step that hands data to another SM or warp: a client's doorbell,
// response poll, write-back and GTS publish; a server's sweep, payload load,
// lock entry, commit step, the KV workers' e_pre -> lastw window and the
// publisher's sweep.  Off (one predicated branch) unless the flag is set.
struct Jitter {
  uint64_t s;
  bool on;
  __device__ Jitter(const KParams& p, uint32_t salt)
      : s(mix64(p.gen.seed ^ 0x6A17C0DEull ^ ((uint64_t)(blockIdx.x * kWarps + (threadIdx.x >> 5)) << 20) ^ salt)),
        on((p.debug & CSMV_DBG_JITTER) != 0) {}
  __device__ __forceinline__ void operator()() {
    if (on) {
      s = mix64(s);
      __nanosleep((uint32_t)(s >> 53));  // 0..2047 ns
    }
  }
};

// Non-blocking: the server's answer to request `round` of client warp cw,
// if all three words carry the round's tag yet.
// A request's header (ReqHdr): tagged, two 64-bit relaxed stores; else
// plain stores of the fields (a fence follows before the doorbell).
__device__ __forceinline__ void put_req_hdr(const KParams& p, uint32_t cw, uint32_t s, uint32_t mask, uint32_t round) {
  if (p.req_tagged) {
    st_relaxed64x2(reinterpret_cast<uint64_t*>(&p.req_hdr[cw]), ((uint64_t)round << 32) | s,
                   ((uint64_t)round << 32) | mask);
  } else {
    p.req_hdr[cw].snapshot = s;
    p.req_hdr[cw].mask = mask;
    p.req_hdr[cw].round = p.req_hdr[cw].round2 = round;
  }
}
// one id of a request: tagged, a relaxed store carrying the round; else a plain store
__device__ __forceinline__ void put_req_id(const KParams& p, uint32_t* a, uint32_t id, uint32_t round) {
  if (p.req_tagged) st_relaxed(a, id | id_tag(round));
  else *a = id;
}

// The three words of a response, loaded by lanes 0-2 at once (one L2 round
// trip, not three) and broadcast.
__device__ __forceinline__ void ld_response(const KParams& p, uint32_t cw, uint64_t& b, uint64_t& c, uint64_t& o) {
  const uint32_t lane = threadIdx.x & 31;
  uint64_t v = 0;
  if (lane < 3) v = ld_relaxed64(&p.resp[cw].base + lane);
  b = __shfl_sync(0xFFFFFFFFu, v, 0);
  c = __shfl_sync(0xFFFFFFFFu, v, 1);
  o = __shfl_sync(0xFFFFFFFFu, v, 2);
}

__device__ __forceinline__ bool try_response(const KParams& p, uint32_t cw, uint32_t round, uint32_t& base,
                                             uint32_t& cmask, uint32_t& omask) {
  uint64_t b, c, o;
  ld_response(p, cw, b, c, o);
  if ((uint32_t)(b >> 32) != round || (uint32_t)(c >> 32) != round || (uint32_t)(o >> 32) != round) return false;
  base = (uint32_t)b;
  cmask = (uint32_t)c;
  omask = (uint32_t)o;
  return true;
}

// Wait for the server's answer to request `round` of client warp cw (all
// three words tagged with round).  false if the run is being torn down.
__device__ __forceinline__ bool wait_response(const KParams& p, uint32_t cw, uint32_t round, uint64_t t_begin,
                                              uint32_t& base, uint32_t& cmask, uint32_t& omask, Jitter& jit) {
  const uint32_t FULL = 0xFFFFFFFFu;
  uint32_t it = 0;
  uint64_t b, c, o;
  for (;;) {
    jit();
    ld_response(p, cw, b, c, o);
    if ((uint32_t)(b >> 32) == round && (uint32_t)(c >> 32) == round && (uint32_t)(o >> 32) == round) break;
    if ((++it & 255u) == 0) {
      uint32_t bad = 0;
      if ((threadIdx.x & 31) == 0) bad = ld_relaxed(&p.ctl->error) || watchdog(p, t_begin, 1);
      if (__shfl_sync(FULL, bad, 0)) return false;
    }
    __nanosleep(CSMV_SLEEP_RESP);
  }
  base = (uint32_t)b;
  cmask = (uint32_t)c;
  omask = (uint32_t)o;
  return true;
}

__device__ __forceinline__ bool watchdog(const KParams& p, uint64_t t0, uint32_t where) {
  if (globaltimer() - t0 > p.watchdog_ns) {
    if (atomicCAS(&p.ctl->error, 0u, 1u) == 0u) p.ctl->where = where;
    return true;
  }
  return false;
}

// --------------------------------------------------------------------------
// Read-only transaction: L consecutive accounts (or all)
// --------------------------------------------------------------------------
// Exact warp sums by redux.sync: an int32 per lane as two 16-bit-wide
// halves (no 32-bit wrap), a u64 per lane (mod 2^64) as four 16-bit chunks.
__device__ __forceinline__ int64_t warp_sum_i32(int32_t v) {
  const int hi = __reduce_add_sync(0xFFFFFFFFu, v >> 16);
  const unsigned lo = __reduce_add_sync(0xFFFFFFFFu, (unsigned)v & 0xFFFFu);
  return (int64_t)hi * 65536 + (int64_t)lo;
}
__device__ __forceinline__ uint64_t warp_sum_u64(uint64_t v) {
  uint64_t r = 0;
#pragma unroll
  for (int k = 0; k < 4; ++k)
    r += (uint64_t)__reduce_add_sync(0xFFFFFFFFu, (unsigned)(v >> (16 * k)) & 0xFFFFu) << (16 * k);
  return r;
}

// Warp-cooperative read-only transactions: the lanes in
// `act` each own one read-only transaction at snapshot s -- tx, a scan of
// `len` accounts from `start` -- and the whole warp runs them one after
// another, 32 consecutive accounts per row (one coalesced 1 KiB load of
// 32-byte VBoxes), U rows in flight.  Each row is reduced across the warp
// (exact int64 sum, digest, any-miss) and added into its owner lane.  Same
// per-transaction result as one lane scanning alone; no lane waits for another lane's
// longer read-only run.
//
// `poll` is called at every row-group boundary (warp-uniform): the client
// uses it to finish its batch (write-back, publish) as soon as the server's
// answer is in, instead of after the whole read-only phase.
struct NoPoll {
  __device__ __forceinline__ void operator()() const {}
};

template <int NS, typename Poll = NoPoll>
__device__ __forceinline__ void rot_coop(const KParams& p, uint32_t act, uint32_t start, uint32_t len, uint32_t s,
                                         uint64_t tx, bool& ok, int64_t& sum, uint64_t& dg, Poll poll = Poll()) {
#ifndef CSMV_ROT_U
#define CSMV_ROT_U 8
#endif
  constexpr int U = NS <= 4 ? CSMV_ROT_U : (NS == 8 ? 4 : 2);
  const uint32_t FULL = 0xFFFFFFFFu;
  const uint32_t lane = threadIdx.x & 31;
  const uint32_t N = p.n_items;
  ok = true;
  sum = 0;
  dg = 0;
  const uint32_t L = __shfl_sync(FULL, len, act ? __ffs(act) - 1 : 0);  // the same for every transaction
  const uint32_t rows = (L + 31) / 32;
  const bool full_log = p.log_mode == CSMV_LOG_FULL;
  const bool long_scan = L > N;  // a scan longer than the store wraps more than once
  // owners are taken lowest lane first, `rows` rows each; (rem, cur, k) are
  // warp-uniform, so the shuffles below run under uniform branches
  uint32_t rem = act, cur = 0, k = rows, cur_start = 0;
  uint64_t cur_tx = 0;
  while (rem || k < rows) {
    Ring<NS> r[U];
    uint32_t xs[U], own[U], ev[U];
    uint64_t txo[U];
    bool on[U];
#pragma unroll
    for (int u = 0; u < U; ++u) {
      if (k >= rows && rem) {  // next owner
        cur = __ffs(rem) - 1;
        rem &= rem - 1;
        k = 0;
        cur_start = __shfl_sync(FULL, start, cur);
        if (full_log) cur_tx = __shfl_sync(FULL, tx, cur);
      }
      on[u] = k < rows;
      own[u] = cur;
      txo[u] = cur_tx;
      ev[u] = k * 32 + lane;
      uint32_t x = cur_start + ev[u];  // start < N; ev < L
      if (x >= N) x -= N;
      if (long_scan && x >= N) x %= N;
      xs[u] = x;
      if (on[u] && ev[u] < L) r[u] = ld_ring<NS>(p.rings + (size_t)x * NS);
      if (on[u]) ++k;
    }
    // version selection for every row first, so that the re-reads a newer
    // version calls for are in flight together (one L2 round trip per group)
    uint64_t vv[U], rv[U];
    bool miss_[U], re[U];
#pragma unroll
    for (int u = 0; u < U; ++u) {
      vv[u] = rv[u] = 0;
      miss_[u] = re[u] = false;
      if (on[u] && ev[u] < L) {
        const Sel q = select_version<NS>(r[u], s);
        if (q.best < 0) {
          miss_[u] = true;  // version recycled
        } else {
          vv[u] = slot_at<NS>(r[u], q.best);
          // A newer version exists, so write-backs may have overwritten slots
          // while we read.  Versions are evicted oldest first, so if the chosen
          // slot still holds the same version, no version in (best_ts, s] was
          // missed; otherwise the snapshot's version is gone.
          re[u] = q.newest > s;
          if (re[u]) rv[u] = ld_relaxed64(p.rings + (size_t)xs[u] * NS + q.best);
        }
      }
    }
#pragma unroll
    for (int u = 0; u < U; ++u) {
      if (!on[u]) break;  // warp-uniform
      const bool valid = ev[u] < L;
      const bool miss = miss_[u] || (re[u] && rv[u] != vv[u]);
      const uint32_t val = (uint32_t)vv[u];
      const bool rmiss = __any_sync(FULL, miss);
      const int64_t rs = warp_sum_i32(miss ? 0 : (int32_t)val);
      uint64_t rd = 0;
      if (p.log_mode) {
        rd = warp_sum_u64(valid && !miss ? dig1(xs[u], val) : 0ull);
        if (p.log_mode == CSMV_LOG_FULL && valid && ev[u] < p.max_vals) p.vals[txo[u] * p.max_vals + ev[u]] = val;
      }
      if (lane == own[u]) {
        ok = ok && !rmiss;
        sum += rs;
        dg += rd;
      }
    }
    poll();
  }
}

// --------------------------------------------------------------------------
// Client warp
// --------------------------------------------------------------------------
struct ClientCounters {
  uint32_t c_upd = 0, c_ro = 0, n_rounds = 0, cas_fail = 0;
  uint32_t ab[CSMV_N_ABORT][2];
  uint64_t ro_ck = 0;
  __device__ ClientCounters() {
#pragma unroll
    for (int i = 0; i < (int)CSMV_N_ABORT; ++i) ab[i][0] = ab[i][1] = 0;
  }
  __device__ __forceinline__ void abort(int reason, bool upd) {
#pragma unroll
    for (int i = 0; i < (int)CSMV_N_ABORT; ++i)
      if (reason == i) ++ab[i][upd ? 1 : 0];
  }
};

// Per-phase client clocks (CSMV_DBG_PHASES; the shape of Tables I and III,
// P:136-147).  Every lane accumulates; the flush reports the
// mean over lanes, so warp-convergent phases read as the warp's time and
// lane-divergent ones (JVSTM-GPU) as the mean lane's.
enum : int {
  PH_READ = 0,     // A: snapshot + update reads
  PH_PREVAL,       // B: pre-validation          | JVSTM: validation + CTS CAS
  PH_SUBMIT,       // B: request + doorbell      | JVSTM: ATR record insert
  PH_ROT,          // C: read-only transactions
  PH_WAIT,         // D: waiting for the server
  PH_WRITEBACK,    // D: write-back
  PH_PUBLISH,      // D: GTS advance / done flag
  PH_DIVERGENCE,   // JVSTM: a lane's wait from its own commit end to reconvergence
};

struct PhaseClock {
  unsigned long long ph[8];
  long long t;
  bool on;
  __device__ explicit PhaseClock(bool enabled) : t(0), on(enabled) {
#pragma unroll
    for (int i = 0; i < 8; ++i) ph[i] = 0;
  }
  __device__ __forceinline__ void start() {
    if (on) t = clock64();
  }
  __device__ __forceinline__ void mark(int k) {
    if (on) {
      const long long n = clock64();
#pragma unroll
      for (int i = 0; i < 8; ++i)
        if (i == k) ph[i] += (unsigned long long)(n - t);
      t = n;
    }
  }
  __device__ __forceinline__ void flush(const KParams& p) const {
    if (!on) return;
#pragma unroll
    for (int i = 0; i < 8; ++i) {
      unsigned long long v = ph[i];
#pragma unroll
      for (int o = 16; o; o >>= 1) v += __shfl_xor_sync(0xFFFFFFFFu, v, o);
      if ((threadIdx.x & 31) == 0 && v) atomicAdd(&p.stats->client_phase[i], v / 32);
    }
  }
};

// CSMV_DBG_TRACE: one record per committed writer of the traced item
// CSMV_DBG_TRACE, server side: the worker stamps when it claimed a request
// and when it stores the response into the response's spare word -- 16 bits
// of the round, then the low 24 bits of each globaltimer value (ns; the
// client rebuilds them next to its own submit time).  Stored before the
// round-tagged words; the client reads it after them, so a stale stamp is
// possible (diagnostics only) and shows as a round mismatch or an odd delta.
__device__ __forceinline__ uint64_t trace_now(const KParams& p) {
  return (p.debug & CSMV_DBG_TRACE) ? globaltimer() : 0ull;
}
__device__ __forceinline__ void trace_served(const KParams& p, uint32_t cw, uint32_t round, uint64_t t_claim) {
  if (p.debug & CSMV_DBG_TRACE)
    st_relaxed64(&p.resp[cw].pad, ((uint64_t)(round & 0xFFFFu) << 48) | ((t_claim & 0xFFFFFFull) << 24) |
                                      (globaltimer() & 0xFFFFFFull));
}
// the server stamps of warp cw's answered request `round` (0, 0 if absent)
__device__ __forceinline__ void trace_srv_times(const KParams& p, uint32_t cw, uint32_t round, uint64_t t_sub,
                                                uint64_t& tc, uint64_t& tv) {
  const uint64_t v = ld_relaxed64(&p.resp[cw].pad);
  tc = tv = 0;
  if ((uint32_t)(v >> 48) != (round & 0xFFFFu)) return;
  const uint64_t ref = t_sub - (1ull << 22);  // the claim may be stamped a little before t_sub is read
  auto rebuild = [&](uint64_t lo) {
    uint64_t t = (ref & ~0xFFFFFFull) | lo;
    if (t < ref) t += 1ull << 24;
    return t;
  };
  tc = rebuild((v >> 24) & 0xFFFFFFull);
  tv = rebuild(v & 0xFFFFFFull);
}

__device__ __forceinline__ void trace_commit(const KParams& p, uint32_t cts, uint32_t s, uint64_t tb, uint64_t ts,
                                             uint64_t tr, uint64_t tp, uint64_t tc = 0, uint64_t tv = 0,
                                             uint64_t tsn = 0, uint64_t trd = 0, uint32_t nrd = 0,
                                             uint32_t nkept = 0) {
  const uint32_t i = atomicAdd(&p.ctl->trace_n, 1u);
  if (i < kTraceCap) {
    csmv_trace_rec r;
    r.cts = cts;
    r.snapshot = s;
    r.t_begin = tb;
    r.t_submit = ts;
    r.t_response = tr;
    r.t_publish = tp;
    r.t_claim = tc;
    r.t_served = tv;
    r.t_snap = tsn;
    r.t_read = trd;
    r.n_readers = nrd;
    r.n_kept = nkept;
    p.trace[i] = r;
  }
}

__device__ __forceinline__ void log_commit(const KParams& p, uint64_t tx, uint32_t s, uint32_t cts,
                                           uint32_t att, uint64_t rdig, uint64_t aux) {
  csmv_log_rec rec;
  rec.tx = (uint32_t)tx;
  rec.snapshot = s;
  rec.cts = cts;
  rec.attempts = att;
  rec.read_digest = rdig;
  rec.aux = aux;
  p.log[tx] = rec;
}

// flush per-warp counters once (no global atomics on the commit path)
__device__ __forceinline__ void client_flush(const KParams& p, const ClientCounters& cc) {
  const uint32_t FULL = 0xFFFFFFFFu;
  const uint32_t lane = threadIdx.x & 31;
  const uint32_t s_upd = __reduce_add_sync(FULL, cc.c_upd), s_ro = __reduce_add_sync(FULL, cc.c_ro);
  const uint32_t s_cf = __reduce_add_sync(FULL, cc.cas_fail);
  uint32_t s_ab[CSMV_N_ABORT][2];
#pragma unroll
  for (int i = 0; i < (int)CSMV_N_ABORT; ++i) {
    s_ab[i][0] = __reduce_add_sync(FULL, cc.ab[i][0]);
    s_ab[i][1] = __reduce_add_sync(FULL, cc.ab[i][1]);
  }
  uint64_t ro_ck = cc.ro_ck;
#pragma unroll
  for (int o = 16; o; o >>= 1) ro_ck ^= __shfl_xor_sync(FULL, ro_ck, o);
  if (lane == 0) {
    atomicAdd(&p.stats->committed_update, (unsigned long long)s_upd);
    atomicAdd(&p.stats->committed_ro, (unsigned long long)s_ro);
    for (int i = 0; i < (int)CSMV_N_ABORT; ++i) {
      if (s_ab[i][0]) atomicAdd(&p.stats->aborts[i][0], (unsigned long long)s_ab[i][0]);
      if (s_ab[i][1]) atomicAdd(&p.stats->aborts[i][1], (unsigned long long)s_ab[i][1]);
    }
    atomicAdd(&p.stats->rounds, (unsigned long long)cc.n_rounds);
    if (s_cf) atomicAdd(&p.stats->cas_fail, (unsigned long long)s_cf);
    atomicXor(&p.stats->ro_checksum, (unsigned long long)ro_ck);
    __threadfence();
    atomicAdd(&p.ctl->done_warps, 1u);
  }
}

}  // namespace csmvd

#include "client_bank.cuh"

#include "kv.cuh"
#include "server.cuh"
#include "client_kv.cuh"
#include "server_part.cuh"

namespace csmvd {

template <int NS, int KIND, bool CL>
__global__ void __launch_bounds__(kBlock, 1) csmv_fused(const KParams p) {
  extern __shared__ __align__(16) uint8_t smem[];
  const uint64_t t_begin = globaltimer();
  if (blockIdx.x < p.n_server_ctas) {
    if constexpr (KIND == CSMV_KIND_BANK && !CL) {
      if (p.part_log2) {
        server_part_cta<NS>(p, smem, t_begin);
        return;
      }
    }
    server_cta<NS, KIND, CL>(p, smem, t_begin);
  }
  else if (p.pub_remote && blockIdx.x == p.n_server_ctas && (threadIdx.x >> 5) == kWarps - 1)
    server_publisher(p, nullptr, t_begin, p.gts_start);  // an idle client warp slot (host.cu)
  else if constexpr (KIND == CSMV_KIND_KV) client_warp_kv<NS>(p, t_begin, reinterpret_cast<uint32_t*>(smem));
  else client_warp<NS>(p, t_begin, smem);
}

template <int NS, int KIND, bool CL>
inline cudaError_t launch_ns(const KParams& p, uint32_t grid, size_t smem, cudaStream_t st, int* occ) {
  auto kern = csmv_fused<NS, KIND, CL>;
  cudaError_t e = cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
  if (e != cudaSuccess) return e;
#ifdef CSMV_CARVEOUT  // A/B: the shared-memory share of the unified L1 (percent)
  e = cudaFuncSetAttribute(kern, cudaFuncAttributePreferredSharedMemoryCarveout, CSMV_CARVEOUT);
  if (e != cudaSuccess) return e;
#endif
  if (CL) {
    e = cudaFuncSetAttribute(kern, cudaFuncAttributeNonPortableClusterSizeAllowed, 1);
    if (e != cudaSuccess) return e;
  }
  cudaLaunchConfig_t cfg = {};
  cudaLaunchAttribute at[2];
  at[0].id = cudaLaunchAttributeCooperative;
  at[0].val.cooperative = 1;
  at[1].id = cudaLaunchAttributeClusterDimension;
  at[1].val.clusterDim.x = CL ? p.n_server_ctas : 1;
  at[1].val.clusterDim.y = 1;
  at[1].val.clusterDim.z = 1;
  cfg.blockDim = dim3(kBlock);
  cfg.dynamicSmemBytes = smem;
  cfg.stream = st;
  cfg.attrs = at;
  cfg.numAttrs = CL ? 2 : 1;
  if (occ) {  // query: co-resident CTAs of this configuration
    if (CL) {
      cfg.gridDim = dim3(p.n_server_ctas);
      int ncl = 0;
      e = cudaOccupancyMaxActiveClusters(&ncl, kern, &cfg);
      *occ = ncl * (int)p.n_server_ctas;
      return e;
    }
    int b = 0;
    e = cudaOccupancyMaxActiveBlocksPerMultiprocessor(&b, kern, kBlock, smem);
    int dev = 0, sms = 0;
    cudaGetDevice(&dev);
    cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
    *occ = b * sms;
    return e;
  }
  cfg.gridDim = dim3(grid);
  return cudaLaunchKernelEx(&cfg, kern, p);
}

template <int KIND, bool CL>
inline cudaError_t launch_kind(const KParams& p, uint32_t nslot, uint32_t grid, size_t smem, cudaStream_t st,
                               int* occ) {
  switch (nslot) {
    case 2: return launch_ns<2, KIND, CL>(p, grid, smem, st, occ);
    case 4: return launch_ns<4, KIND, CL>(p, grid, smem, st, occ);
    case 8: return launch_ns<8, KIND, CL>(p, grid, smem, st, occ);
    case 16: return launch_ns<16, KIND, CL>(p, grid, smem, st, occ);
  }
  return cudaErrorInvalidValue;
}

// one per translation unit (fused_*.cu)
cudaError_t launch_fused_bank_cta(const KParams& p, uint32_t nslot, uint32_t grid, size_t smem, cudaStream_t st, int* occ);
cudaError_t launch_fused_bank_cl(const KParams& p, uint32_t nslot, uint32_t grid, size_t smem, cudaStream_t st, int* occ);
cudaError_t launch_fused_kv_cta(const KParams& p, uint32_t nslot, uint32_t grid, size_t smem, cudaStream_t st, int* occ);
cudaError_t launch_fused_kv_cl(const KParams& p, uint32_t nslot, uint32_t grid, size_t smem, cudaStream_t st, int* occ);

}  // namespace csmvd
