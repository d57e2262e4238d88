// kernel.cu -- the fused persistent CSMV kernel for sm_100a.
//
// One cooperative grid holds both roles of the paper's client-server split
// (P:99-105): CTA 0 is the server SM, CTAs 1..C are client SMs.  Fusing the
// roles into one launch guarantees co-residency of a server that spins on
// its clients (the paper launches two kernels; separate kernels deadlock when
// a profiler serialises them).
//
// Client warp, one round (section III):
//   TXBegin     s <- GTS (one acquire load per warp round)
//   TXRead      newest version with ts <= s from the VBox ring
//               read-only lanes finish here, no commit
//   pre-validation of the warp's update lanes (shuffle/ballot)
//   submit the batch (request slot + doorbell), wait for the response P:101
//   write-back of the new versions by the client
//   ordered GTS advance by n (CSMV_PUBLISH_CLIENT) or a done
//   flag per CTS for the server publisher (CSMV_PUBLISH_SERVER)
//   aborted lanes retry with a fresh snapshot next round
//
// Server CTA: worker warps each own a contiguous slice of client doorbells
// (receiving and working are merged per warp); a batch is
// validated by the whole warp (one lane per transaction, __ballot_sync /
// __match_any_sync) against the ATR, which lives in shared memory as an
// item-indexed set-associative table of (item, last CTS) covering every
// commit after the watermark W_low;
// consecutive CTS are reserved and the write-sets inserted inside one
// shared-memory critical section.  No global atomics on the
// commit path.
#include <cuda_runtime.h>

#include "kernel.cuh"
#include "ptx.cuh"

namespace csmvd {

enum : int { ST_NONE = 0, ST_RO_OK, ST_CAND, ST_UPD_OK, ST_ABORT };

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
template <int NS>
__device__ __forceinline__ bool rot_scan(const KParams& p, uint32_t start, uint32_t len, uint32_t s,
                                         uint64_t tx, int64_t& sum, uint64_t& dg) {
  constexpr int U = 4;
  sum = 0;
  dg = 0;
  const uint32_t N = p.n_items;
  uint32_t x = start;
  for (uint32_t j = 0; j < len; j += U) {
    Ring<NS> r[U];
    uint32_t xs[U];
#pragma unroll
    for (int u = 0; u < U; ++u) {
      xs[u] = x;
      if (j + u < len) r[u] = ld_ring<NS>(p.rings + (size_t)x * NS);
      x = (x + 1 == N) ? 0u : x + 1;
    }
#pragma unroll
    for (int u = 0; u < U; ++u) {
      if (j + u >= len) break;
      Sel q = select_version<NS>(r[u], s);
      if (q.best < 0) return false;  // version recycled
      uint64_t v = slot_at<NS>(r[u], q.best);
      if (q.newest > s) {
        // A newer version exists, so write-backs may have overwritten slots
        // while we read.  Versions are evicted oldest first, so if the chosen
        // slot still holds the same version, no version in (best_ts, s] was
        // missed; otherwise the snapshot's version is gone.
        if (ld_relaxed64(p.rings + (size_t)xs[u] * NS + q.best) != v) return false;
      }
      int32_t val = (int32_t)(uint32_t)v;
      sum += val;
      if (p.log_mode) {
        dg += dig1(xs[u], (uint32_t)val);
        if (p.log_mode == CSMV_LOG_FULL && j + u < p.max_vals)
          p.vals[tx * p.max_vals + j + u] = (uint32_t)val;
      }
    }
  }
  return true;
}

// --------------------------------------------------------------------------
// Client warp
// --------------------------------------------------------------------------
struct ClientCounters {
  uint32_t c_upd = 0, c_ro = 0, n_rounds = 0;
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
    atomicXor(&p.stats->ro_checksum, (unsigned long long)ro_ck);
    __threadfence();
    atomicAdd(&p.ctl->done_warps, 1u);
  }
}

}  // namespace csmvd

#include "client_bank.cuh"

namespace csmvd {

// --------------------------------------------------------------------------
// Server CTA
// --------------------------------------------------------------------------
struct SrvShared {
  uint32_t tail;         // last CTS assigned (the CTS counter)
  uint32_t next_ticket;  // ticket lock around validate+reserve+insert
  uint32_t now_serving;
  uint32_t gts_seen;     // publisher progress seen by workers (back-pressure)
  uint32_t q_head;       // next dispatch-queue slot a worker claims
  uint32_t exit;         // receiver: all clients finished
};

// ---------------------------------------------------------------------------
// The ATR, item-indexed and split in two levels:
//  * lastw[x] in HBM: CTS of the last commit that wrote x -- the exact
//    record of every committed write-set, all history;
//  * rt in shared memory: 4-way buckets of (cts << 32 | item) holding recent
//    writes plus, per bucket, evmax = the largest CTS ever evicted from it,
//    so that commits made after a worker prefetched lastw (CTS > e_pre) are
//    seen with on-chip latency.
// Invariant: if the latest write c of item y (bucket b) is not in b, then
// evmax[b] >= c (entries leave a bucket only through atomicExch, and the
// evictor records the evicted CTS with atomicMax).
// Validation of x for snapshot s (P:75 read-set, P:115 write-set), s <= e_pre:
//    conflict  iff  lastw[x] (as of e_pre) > s  or  some way holds (x, c), c > s
//    unknown   iff  not conflict and evmax[b] > e_pre -> abort, reason OVERFLOW
// ---------------------------------------------------------------------------
constexpr int kRtWays = 4;

__device__ __forceinline__ uint32_t rt_bucket(uint32_t key, uint32_t rt_log2) {
  return (key * 0x9E3779B1u) >> (32 - rt_log2);
}

struct RtProbe {
  int way;        // way to overwrite: the way holding x, else the oldest
  bool conflict;
  bool unknown;
};

__device__ __forceinline__ RtProbe rt_probe(const uint64_t* rt, const uint32_t* evmax, uint32_t bucket,
                                            uint32_t key, uint32_t s, uint32_t e_pre, uint32_t lastw) {
  const ulonglong2* e = reinterpret_cast<const ulonglong2*>(rt + (size_t)bucket * kRtWays);
  const ulonglong2 a = e[0], b = e[1];
  const uint32_t ev = evmax[bucket];
  const uint64_t w[4] = {a.x, a.y, b.x, b.y};
  RtProbe r;
  r.conflict = lastw > s;
  int hit = -1, old = 0;
  uint32_t oldc = 0xFFFFFFFFu;
#pragma unroll
  for (int i = 0; i < kRtWays; ++i) {
    const uint32_t k = (uint32_t)w[i], c = (uint32_t)(w[i] >> 32);
    if (k == key) {
      hit = i;
      r.conflict |= c > s;
    }
    if (c < oldc) {
      oldc = c;
      old = i;
    }
  }
  r.unknown = !r.conflict && ev > e_pre;
  r.way = hit >= 0 ? hit : old;
  return r;
}

// Record (key, cts) into `way` of its bucket; an evicted entry of another
// key raises evmax.  Exchanges by several lanes on one slot are serialised
// by the hardware and each evictor sees the value it replaced.
__device__ __forceinline__ void rt_record(uint64_t* rt, uint32_t* evmax, uint32_t bucket, int way,
                                          uint32_t key, uint32_t cts) {
  const unsigned long long old =
      atomicExch(reinterpret_cast<unsigned long long*>(rt + (size_t)bucket * kRtWays + way),
                 ((unsigned long long)cts << 32) | key);
  if ((uint32_t)old != key && (uint32_t)(old >> 32) != 0u) atomicMax(evmax + bucket, (uint32_t)(old >> 32));
}

// Receiver warp: sweeps every client doorbell with coalesced loads
// and dispatches new requests to the workers through a shared-memory queue
// (entry = lap << 32 | client warp; a worker that claimed slot i waits for
// lap i / QN + 1).  At most one request per client warp is outstanding, so
// QN >= n_cw slots never wrap onto an unconsumed entry.
__device__ void server_receiver(const KParams& p, uint32_t* last_seen, uint64_t* queue, uint32_t qn_log2,
                                SrvShared* sh, uint64_t t_begin) {
  const uint32_t FULL = 0xFFFFFFFFu;
  const uint32_t lane = threadIdx.x & 31;
  const uint32_t rows = (p.n_cw + 31) / 32;
  const uint32_t lt = lanemask_lt();
  const uint32_t qmask = (1u << qn_log2) - 1;
  uint32_t tail = 0;  // next queue slot to fill
  uint32_t idle = 0;
  for (;;) {
    bool found = false;
    for (uint32_t r0 = 0; r0 < rows; r0 += 8) {
      uint32_t seq[8];
#pragma unroll
      for (int k = 0; k < 8; ++k) {
        const uint32_t w = (r0 + k) * 32 + lane;
        seq[k] = (r0 + k < rows && w < p.n_cw) ? ld_relaxed(p.req_seq + w) : 0u;
      }
#pragma unroll
      for (int k = 0; k < 8; ++k) {
        const uint32_t w = (r0 + k) * 32 + lane;
        const bool pend = r0 + k < rows && w < p.n_cw && seq[k] != last_seen[w];
        const uint32_t pm = __ballot_sync(FULL, pend);
        if (pm) {
          found = true;
          if (pend) {
            const uint32_t pos = tail + __popc(pm & lt);
            last_seen[w] = seq[k];
            *(volatile uint64_t*)&queue[pos & qmask] = ((uint64_t)((pos >> qn_log2) + 1) << 32) | w;
          }
          tail += __popc(pm);
        }
      }
    }
    if (found) {
      idle = 0;
      continue;
    }
    if ((++idle & 15u) == 0) {
      uint32_t dw = 0, er = 0;
      if (lane == 0) {
        dw = ld_relaxed(&p.ctl->done_warps);
        er = ld_relaxed(&p.ctl->error);
        if (!er && dw < p.n_cw && watchdog(p, t_begin, 3)) er = 1;
      }
      dw = __shfl_sync(FULL, dw, 0);
      er = __shfl_sync(FULL, er, 0);
      if (dw >= p.n_cw || er) {
        if (lane == 0) *(volatile uint32_t*)&sh->exit = 1;
        return;
      }
    }
  }
}

// Server worker warp.  Claims up to kMaxCombine dispatched batches (the
// first blocking, the rest only if already queued), loads them outside the
// lock, and commits them inside ONE critical section, one after another in
// queue order -- exactly as if each had its own critical section: batch j
// is validated after batch j-1's write-set was recorded, and receives the
// next consecutive CTS range.
__device__ void server_worker(const KParams& p, uint64_t* rt, uint32_t* evmax, uint64_t* queue,
                              uint32_t qn_log2, SrvShared* sh, uint64_t t_begin) {
  constexpr int M = kMaxCombine;
  const uint32_t FULL = 0xFFFFFFFFu;
  const uint32_t lane = threadIdx.x & 31;
  const uint32_t lt = lanemask_lt();
  const uint32_t qmask = (1u << qn_log2) - 1;
  const uint32_t dmask = (1u << kDoneLog2) - 1;
  const uint32_t m_max = p.combine < 1 ? 1u : (p.combine > (uint32_t)M ? (uint32_t)M : p.combine);
  unsigned long long busy = 0, locked = 0, batches = 0, groups = 0;
  unsigned long long ph[8] = {0, 0, 0, 0, 0, 0, 0, 0};
  for (;;) {
    const long long tq = clock64();
    // ---- claim: first request blocking
    uint32_t slot = 0;
    if (lane == 0) slot = atomicAdd(&sh->q_head, 1u);
    slot = __shfl_sync(FULL, slot, 0);
    uint32_t cwv[M];
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
    cwv[0] = (uint32_t)ent;
    // ---- combine: grab further requests that are already queued
    uint32_t m = 1;
#pragma unroll
    for (int j = 1; j < M; ++j) {
      uint32_t got = 0xFFFFFFFFu;
      if (m == (uint32_t)j && m < m_max && lane == 0) {
        const uint32_t h = *(volatile uint32_t*)&sh->q_head;
        const uint64_t e = *(volatile uint64_t*)&queue[h & qmask];
        if ((uint32_t)(e >> 32) == (h >> qn_log2) + 1 && atomicCAS(&sh->q_head, h, h + 1) == h) got = (uint32_t)e;
      }
      got = __shfl_sync(FULL, got, 0);
      cwv[j] = got;
      if (got != 0xFFFFFFFFu && m == (uint32_t)j) m = j + 1;
    }
    const long long t0 = clock64();
    // ---- load the batches: doorbell (acquire pattern), header, ids
    uint32_t sq[M], sn[M], msk[M], id0[M], id1[M];
#pragma unroll
    for (int j = 0; j < M; ++j) sq[j] = (j < (int)m) ? ld_relaxed(p.req_seq + cwv[j]) : 0u;
    fence_gpu();
#pragma unroll
    for (int j = 0; j < M; ++j) {
      sn[j] = msk[j] = id0[j] = id1[j] = 0;
      if (j < (int)m) {
        sn[j] = ld_relaxed(&p.req_hdr[cwv[j]].snapshot);
        msk[j] = ld_relaxed(&p.req_hdr[cwv[j]].mask);
      }
    }
    bool mine[M];
#pragma unroll
    for (int j = 0; j < M; ++j) {
      mine[j] = (msk[j] >> lane) & 1u;
      if (mine[j]) {
        id0[j] = ld_relaxed(p.req_ids + (size_t)cwv[j] * 64 + lane) & ~kWriteBit;
        id1[j] = ld_relaxed(p.req_ids + (size_t)cwv[j] * 64 + 32 + lane) & ~kWriteBit;
      }
    }
    const uint32_t e_pre = *(volatile uint32_t*)&sh->tail;  // lastw covers every CTS <= e_pre
    fence_cta();
    uint32_t lw0[M], lw1[M], bk0[M], bk1[M];
    uint32_t xor_all = e_pre;
#pragma unroll
    for (int j = 0; j < M; ++j) {
      lw0[j] = lw1[j] = 0;
      if (mine[j]) {
        lw0[j] = ld_relaxed(p.lastw + id0[j]);
        lw1[j] = ld_relaxed(p.lastw + id1[j]);
      }
      bk0[j] = rt_bucket(id0[j], p.rt_log2);
      bk1[j] = rt_bucket(id1[j], p.rt_log2);
      xor_all ^= bk0[j] ^ bk1[j] ^ lw0[j] ^ lw1[j] ^ sn[j];
    }
    // The payload must have arrived before the lock is taken: a warp vote on
    // values derived from it makes the loads complete here.
    if (__ballot_sync(FULL, xor_all == 0x12345679u) == FULL) __nanosleep(1);
    const long long tl = clock64();
    // ---- critical section: validate, reserve CTS, record
    uint32_t ticket = 0;
    if (lane == 0) ticket = atomicAdd(&sh->next_ticket, 1u);
    ticket = __shfl_sync(FULL, ticket, 0);
    while (*(volatile uint32_t*)&sh->now_serving != ticket) __nanosleep(16);
    __syncwarp();
    fence_cta();
    const long long t1 = clock64();
    const uint32_t t0c = *(volatile uint32_t*)&sh->tail;
    uint32_t t = t0c;
    uint32_t cm[M], om[M], base[M];
#pragma unroll
    for (int j = 0; j < M; ++j) {
      cm[j] = om[j] = 0;
      base[j] = t + 1;
      if (j >= (int)m) continue;
      RtProbe q0{0, false, false}, q1{0, false, false};
      if (mine[j]) {
        q0 = rt_probe(rt, evmax, bk0[j], id0[j], sn[j], e_pre, lw0[j]);
        q1 = rt_probe(rt, evmax, bk1[j], id1[j], sn[j], e_pre, lw1[j]);
        if (bk1[j] == bk0[j] && q1.way == q0.way) q1.way = (q1.way + 1) & (kRtWays - 1);
      }
      bool ovf = mine[j] && (q0.unknown || q1.unknown);
      bool conflict = mine[j] && (q0.conflict || q1.conflict);
      if (p.debug & CSMV_DBG_NO_VALIDATE) ovf = conflict = false;
      const bool commit = mine[j] && !ovf && !conflict;
      cm[j] = __ballot_sync(FULL, commit);
      om[j] = __ballot_sync(FULL, ovf);
      const uint32_t c = t + 1 + __popc(cm[j] & lt);
      t += __popc(cm[j]);
      if (commit) {
        p.lastw[id0[j]] = c;
        p.lastw[id1[j]] = c;
        rt_record(rt, evmax, bk0[j], q0.way, id0[j], c);
        rt_record(rt, evmax, bk1[j], q1.way, id1[j], c);
      }
      __syncwarp();  // batch j's records precede batch j+1's probes
    }
    const long long ta = clock64();
    if (p.publish == CSMV_PUBLISH_SERVER && t != t0c) {
      // done-ring back-pressure: CTS c may reuse slot c & dmask only once
      // GTS >= c - 2^20
      if (lane == 0) {
        uint32_t it = 0;
        while (t > sh->gts_seen + dmask) {
          sh->gts_seen = ld_relaxed(p.gts);
          if ((++it & 255u) == 0 && watchdog(p, t_begin, 4)) break;
        }
      }
      __syncwarp();
    }
    fence_cta();
    if (lane == 0) {
      sh->tail = t;
      fence_cta();
      *(volatile uint32_t*)&sh->now_serving = ticket + 1;
    }
    const long long t2 = clock64();
    // ---- respond: one fence, then the payloads and sequence words
    if (lane == 0) {
#pragma unroll
      for (int j = 0; j < M; ++j) {
        if (j >= (int)m) break;
        st_relaxed(&p.resp[cwv[j]].cts_base, base[j]);
        st_relaxed(&p.resp[cwv[j]].commit_mask, cm[j]);
        st_relaxed(&p.resp[cwv[j]].overflow_mask, om[j]);
      }
      fence_gpu();
#pragma unroll
      for (int j = 0; j < M; ++j) {
        if (j >= (int)m) break;
        st_relaxed(&p.resp[cwv[j]].seq, sq[j]);
      }
    }
    __syncwarp();
    const long long t3 = clock64();
    busy += (unsigned long long)(t3 - t0);
    locked += (unsigned long long)(t2 - t1);
    ph[0] += (unsigned long long)(t0 - tq);
    ph[1] += (unsigned long long)(tl - t0);
    ph[2] += (unsigned long long)(t1 - tl);
    ph[3] += (unsigned long long)(t2 - t1);
    ph[4] += (unsigned long long)(t3 - t2);
    ph[5] += (unsigned long long)(ta - t1);
    batches += m;
    ++groups;
  }
  if (lane == 0) {
    for (int i = 0; i < 8; ++i) atomicAdd(&p.stats->phase[i], ph[i]);
    atomicAdd(&p.stats->batches, batches);
    atomicAdd(&p.stats->groups, groups);
    atomicAdd(&p.stats->busy_cycles, busy);
    atomicAdd(&p.stats->lock_cycles, locked);
  }
}

// CSMV_PUBLISH_SERVER: advance GTS over the prefix of CTS whose write-backs
// are done.  Same invariant as P:116 (GTS = c only once every commit <= c
// has written back), without a client-side serial chain.
__device__ void server_publisher(const KParams& p, SrvShared* sh, uint64_t t_begin) {
  const uint32_t FULL = 0xFFFFFFFFu;
  const uint32_t lane = threadIdx.x & 31;
  const uint32_t dmask = (1u << kDoneLog2) - 1;
  uint32_t g = *(volatile uint32_t*)&sh->tail;
  uint32_t spins = 0;
  for (;;) {
    uint32_t v[4];
#pragma unroll
    for (int k = 0; k < 4; ++k) v[k] = ld_relaxed(p.done_ring + ((g + 1 + k * 32 + lane) & dmask));
    uint32_t adv = 0;
#pragma unroll
    for (int k = 0; k < 4; ++k) {
      const uint32_t bad = __ballot_sync(FULL, v[k] != g + 1 + k * 32 + lane);
      if (adv == (uint32_t)k * 32) adv += bad ? (uint32_t)(__ffs(bad) - 1) : 32u;
    }
    if (adv) {
      fence_gpu();
      g += adv;
      if (lane == 0) st_release(p.gts, g);
      continue;
    }
    if ((++spins & 63u) == 0) {
      uint32_t dw = 0, er = 0;
      if (lane == 0) {
        dw = ld_relaxed(&p.ctl->done_warps);
        er = ld_relaxed(&p.ctl->error);
        if (!er && watchdog(p, t_begin, 5)) er = 1;
      }
      dw = __shfl_sync(FULL, dw, 0);
      er = __shfl_sync(FULL, er, 0);
      if (er) break;
      if (dw >= p.n_cw && g == *(volatile uint32_t*)&sh->tail) break;
    }
  }
}

}  // namespace csmvd

#include "kv.cuh"
#include "kv_kernels.cuh"

namespace csmvd {

template <int KIND>
__device__ void server_cta(const KParams& p, uint8_t* smem, uint64_t t_begin) {
  uint64_t* rt = reinterpret_cast<uint64_t*>(smem);
  const uint32_t rt_words = (uint32_t)kRtWays << p.rt_log2;
  const uint32_t qn_log2 = queue_log2(p.n_cw);
  uint64_t* queue = rt + rt_words;
  uint32_t* evmax = reinterpret_cast<uint32_t*>(queue + (1u << qn_log2));
  uint32_t* last_seen = evmax + (1u << p.rt_log2);
  const uint32_t ls_words = (p.n_cw + 31) / 32 * 32;
  SrvShared* sh = reinterpret_cast<SrvShared*>(last_seen + ls_words);
  for (uint32_t i = threadIdx.x; i < rt_words; i += blockDim.x) rt[i] = 0xFFFFFFFFull;  // cts 0, no item
  for (uint32_t i = threadIdx.x; i < (1u << p.rt_log2); i += blockDim.x) evmax[i] = 0;
  for (uint32_t i = threadIdx.x; i < (1u << qn_log2); i += blockDim.x) queue[i] = 0;
  for (uint32_t i = threadIdx.x; i < ls_words; i += blockDim.x) last_seen[i] = 0;
  if (threadIdx.x == 0) {
    const uint32_t g0 = *p.gts;
    sh->tail = g0;
    sh->next_ticket = 0;
    sh->now_serving = 0;
    sh->gts_seen = g0;
    sh->q_head = 0;
    sh->exit = 0;
  }
  __syncthreads();
  const uint32_t warp = threadIdx.x >> 5;
  if (warp == 0) {
    server_receiver(p, last_seen, queue, qn_log2, sh, t_begin);
  } else if (warp <= p.n_workers) {
    if constexpr (KIND == CSMV_KIND_KV) server_worker_generic(p, queue, qn_log2, sh, t_begin);
    else server_worker(p, rt, evmax, queue, qn_log2, sh, t_begin);
  } else if (warp == p.n_workers + 1 && p.publish == CSMV_PUBLISH_SERVER) {
    server_publisher(p, sh, t_begin);
  }
  __syncthreads();
  if (threadIdx.x == 0) p.ctl->tail_final = sh->tail;
}

template <int NS, int KIND>
__global__ void __launch_bounds__(kBlock, 1) csmv_fused(const KParams p) {
  extern __shared__ __align__(16) uint8_t smem[];
  const uint64_t t_begin = globaltimer();
  if (blockIdx.x == 0) server_cta<KIND>(p, smem, t_begin);
  else if constexpr (KIND == CSMV_KIND_KV) client_warp_kv<NS>(p, t_begin, reinterpret_cast<uint32_t*>(smem));
  else client_warp<NS>(p, t_begin);
}

template <int NS>
__global__ void init_rings(uint64_t* rings, const int32_t* init, uint64_t n, uint32_t* gts) {
  const uint64_t i = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x;
  if (i == 0) *gts = 0;
  if (i >= n) return;
  Ring<NS> r;
#pragma unroll
  for (int j = 0; j < NS; ++j) r.s[j] = (uint64_t)kEmptyTs << 32;
  r.s[0] = (uint64_t)(uint32_t)init[i];
  *reinterpret_cast<Ring<NS>*>(rings + i * NS) = r;
}

__global__ void gen_descs_kernel(GenParams g, uint64_t tx0, uint64_t n, uint32_t* out) {
  const uint64_t i = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x;
  if (i >= n) return;
  BankTx d = gen_bank(g, tx0 + i);
  uint32_t* o = out + i * 6;
  o[0] = d.is_update;
  o[1] = d.src;
  o[2] = d.dst;
  o[3] = (uint32_t)d.amt;
  o[4] = d.start;
  o[5] = d.len;
}

template <int NS, int KIND>
static cudaError_t launch_ns(const KParams& p, uint32_t grid, size_t smem, cudaStream_t st) {
  cudaError_t e =
      cudaFuncSetAttribute(csmv_fused<NS, KIND>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
  if (e != cudaSuccess) return e;
  void* args[] = {(void*)&p};
  return cudaLaunchCooperativeKernel((const void*)csmv_fused<NS, KIND>, dim3(grid), dim3(kBlock), args, smem, st);
}

template <int KIND>
static cudaError_t launch_kind(const KParams& p, uint32_t nslot, uint32_t grid, size_t smem, cudaStream_t st) {
  switch (nslot) {
    case 2: return launch_ns<2, KIND>(p, grid, smem, st);
    case 4: return launch_ns<4, KIND>(p, grid, smem, st);
    case 8: return launch_ns<8, KIND>(p, grid, smem, st);
    case 16: return launch_ns<16, KIND>(p, grid, smem, st);
  }
  return cudaErrorInvalidValue;
}

cudaError_t launch_fused(const KParams& p, uint32_t nslot, uint32_t grid, size_t smem, cudaStream_t st) {
  if (p.kind == CSMV_KIND_KV) return launch_kind<CSMV_KIND_KV>(p, nslot, grid, smem, st);
  return launch_kind<CSMV_KIND_BANK>(p, nslot, grid, smem, st);
}

template <int NS, int KIND>
static cudaError_t occ_ns(size_t smem, int* b) {
  cudaError_t e =
      cudaFuncSetAttribute(csmv_fused<NS, KIND>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
  if (e != cudaSuccess) return e;
  return cudaOccupancyMaxActiveBlocksPerMultiprocessor(b, csmv_fused<NS, KIND>, kBlock, smem);
}

cudaError_t fused_occupancy(uint32_t nslot, uint32_t kind, size_t smem, int* b) {
  if (kind == CSMV_KIND_KV) {
    switch (nslot) {
      case 2: return occ_ns<2, CSMV_KIND_KV>(smem, b);
      case 4: return occ_ns<4, CSMV_KIND_KV>(smem, b);
      case 8: return occ_ns<8, CSMV_KIND_KV>(smem, b);
      case 16: return occ_ns<16, CSMV_KIND_KV>(smem, b);
    }
    return cudaErrorInvalidValue;
  }
  switch (nslot) {
    case 2: return occ_ns<2, CSMV_KIND_BANK>(smem, b);
    case 4: return occ_ns<4, CSMV_KIND_BANK>(smem, b);
    case 8: return occ_ns<8, CSMV_KIND_BANK>(smem, b);
    case 16: return occ_ns<16, CSMV_KIND_BANK>(smem, b);
  }
  return cudaErrorInvalidValue;
}

cudaError_t launch_init_kv(const KParams& p, uint32_t nslot, const uint32_t* keys, const uint32_t* vals,
                           const uint32_t* lru, const uint32_t* clocks, cudaStream_t st) {
  const uint32_t blocks = (uint32_t)((p.kv_S + 255) / 256);
  switch (nslot) {
    case 2: init_kv_rings<2><<<blocks, 256, 0, st>>>(p, keys, vals, lru, clocks); break;
    case 4: init_kv_rings<4><<<blocks, 256, 0, st>>>(p, keys, vals, lru, clocks); break;
    case 8: init_kv_rings<8><<<blocks, 256, 0, st>>>(p, keys, vals, lru, clocks); break;
    case 16: init_kv_rings<16><<<blocks, 256, 0, st>>>(p, keys, vals, lru, clocks); break;
    default: return cudaErrorInvalidValue;
  }
  return cudaGetLastError();
}

cudaError_t launch_kv_newest(const KParams& p, uint32_t nslot, uint32_t* keys, uint32_t* vals, uint32_t* lru,
                             uint32_t* clocks, cudaStream_t st) {
  const uint32_t blocks = (uint32_t)((p.kv_S + 255) / 256);
  switch (nslot) {
    case 2: kv_newest<2><<<blocks, 256, 0, st>>>(p, keys, vals, lru, clocks); break;
    case 4: kv_newest<4><<<blocks, 256, 0, st>>>(p, keys, vals, lru, clocks); break;
    case 8: kv_newest<8><<<blocks, 256, 0, st>>>(p, keys, vals, lru, clocks); break;
    case 16: kv_newest<16><<<blocks, 256, 0, st>>>(p, keys, vals, lru, clocks); break;
    default: return cudaErrorInvalidValue;
  }
  return cudaGetLastError();
}

cudaError_t launch_gen_kv_descs(GenParams g, uint64_t tx0, uint64_t n, uint32_t* out, cudaStream_t st) {
  if (n == 0) return cudaSuccess;
  gen_kv_descs_kernel<<<(uint32_t)((n + 255) / 256), 256, 0, st>>>(g, tx0, n, out);
  return cudaGetLastError();
}

cudaError_t launch_init_rings(uint64_t* rings, uint32_t nslot, const int32_t* init, uint64_t n,
                              uint32_t* gts, cudaStream_t st) {
  const uint32_t blocks = (uint32_t)((n + 255) / 256) + 1;
  switch (nslot) {
    case 2: init_rings<2><<<blocks, 256, 0, st>>>(rings, init, n, gts); break;
    case 4: init_rings<4><<<blocks, 256, 0, st>>>(rings, init, n, gts); break;
    case 8: init_rings<8><<<blocks, 256, 0, st>>>(rings, init, n, gts); break;
    case 16: init_rings<16><<<blocks, 256, 0, st>>>(rings, init, n, gts); break;
    default: return cudaErrorInvalidValue;
  }
  return cudaGetLastError();
}

cudaError_t launch_gen_descs(GenParams g, uint64_t tx0, uint64_t n, uint32_t* out, cudaStream_t st) {
  if (n == 0) return cudaSuccess;
  gen_descs_kernel<<<(uint32_t)((n + 255) / 256), 256, 0, st>>>(g, tx0, n, out);
  return cudaGetLastError();
}

}  // namespace csmvd
