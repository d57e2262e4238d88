// server.cuh -- the commit server.
//
// Single-CTA server (CL = false, the paper's one server SM) or a
// thread-block-cluster server (CL = true): cluster 0 of the fused grid, C
// CTAs.  In the cluster server
//  * the recent-commit table (the on-chip level of the ATR) is striped over
//    the C CTAs' shared memory by bucket (bucket b lives in CTA b mod C) and
//    reached through distributed shared memory -- C times the capacity;
//  * the CTS counter, ticket lock and publisher live in CTA 0 (SURVEY H5:
//    validation + CTS reservation stay linearizable in one place);
//  * every CTA runs a receiver warp for its slice of the client doorbells and
//    its own worker warps, so receiving, payload loading and responding scale
//    with C.
// Included by kernel.cu after the shared helpers.
#pragma once
#include <cooperative_groups.h>

namespace csmvd {

namespace cg = cooperative_groups;

struct SrvShared {
  uint32_t tail;         // last CTS assigned (the CTS counter)   [CTA 0]
  uint32_t next_ticket;  // ticket lock around validate+reserve+insert        [CTA 0]
  uint32_t now_serving;  //                                                   [CTA 0]
  uint32_t gts_seen;     // publisher progress seen by workers (back-pressure) [CTA 0]
  uint32_t q_head;       // next dispatch-queue slot a worker claims          [per CTA]
  uint32_t exit;         // receiver: all clients finished                    [per CTA]
  uint32_t ring_head;    // commit ring: next slot a worker claims            [CTA 0]
  uint32_t ring_done;    // commit ring: slots the committer has finished     [CTA 0]
  uint32_t workers_left; // commit ring: worker warps still running          [CTA 0]
  uint32_t pad[7];
};
static_assert(sizeof(SrvShared) == 64, "control block is 64 B (server_smem_bytes)");

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

struct SrvCtx {
  uint64_t* rt;       // this CTA's stripe of buckets (kRtWays u64 each)
  uint32_t rt32;      // rt as a shared-window address
  uint32_t* evmax;    // this CTA's stripe of eviction watermarks
  uint32_t clog2;     // log2(server CTAs)
  SrvShared* sh;      // this CTA's control block
  SrvShared* sh0;     // CTA 0's control block (DSMEM in a cluster)
  uint64_t* queue;    // this CTA's dispatch queue
  uint32_t qn_log2;
  uint32_t* last_seen;
  uint32_t cw_lo, cw_hi;  // client warps this CTA's receiver serves
  uint32_t ring32;     // CTA 0's commit ring: shared (::cluster in a cluster) window address
};

// shared-memory stores/loads of the commit ring (explicit shared::cluster
// forms in a cluster: the payload goes to CTA 0 through DSMEM)
template <bool CL>
__device__ __forceinline__ void ring_st_v4(uint32_t a, uint4 v) {
  if constexpr (CL)
    asm volatile("st.shared::cluster.v4.u32 [%0], {%1, %2, %3, %4};" ::"r"(a), "r"(v.x), "r"(v.y), "r"(v.z), "r"(v.w)
                 : "memory");
  else
    asm volatile("st.shared.v4.u32 [%0], {%1, %2, %3, %4};" ::"r"(a), "r"(v.x), "r"(v.y), "r"(v.z), "r"(v.w)
                 : "memory");
}
// acquire load of a flag in this CTA's shared memory written (after a
// release fence) by a warp of this CTA (CL = false: a plain LDS) or of any
// CTA of the cluster
template <bool CL>
__device__ __forceinline__ uint32_t ring_ld_acquire(uint32_t a) {
  uint32_t v;
  if constexpr (CL) asm volatile("ld.acquire.cluster.shared::cta.u32 %0, [%1];" : "=r"(v) : "r"(a) : "memory");
  else asm volatile("ld.acquire.cta.shared::cta.u32 %0, [%1];" : "=r"(v) : "r"(a) : "memory");
  return v;
}

template <bool CL>
__device__ __forceinline__ uint64_t* rt_at(const SrvCtx& c, uint32_t b) {
  if constexpr (!CL) {
    return c.rt + (size_t)b * kRtWays;
  } else {
    const uint32_t owner = b & ((1u << c.clog2) - 1), local = b >> c.clog2;
    return cg::this_cluster().map_shared_rank(c.rt, owner) + (size_t)local * kRtWays;
  }
}

template <bool CL>
__device__ __forceinline__ uint32_t* ev_at(const SrvCtx& c, uint32_t b) {
  if constexpr (!CL) {
    return c.evmax + b;
  } else {
    const uint32_t owner = b & ((1u << c.clog2) - 1), local = b >> c.clog2;
    return cg::this_cluster().map_shared_rank(c.evmax, owner) + local;
  }
}

template <bool CL>
__device__ __forceinline__ void srv_fence() {
  if constexpr (CL) asm volatile("fence.acq_rel.cluster;" ::: "memory");
  else fence_cta();
}

struct RtProbe {
  int way;        // way to overwrite: the way holding x, else the oldest
  bool conflict;
  bool unknown;
};

// A bucket as loaded: its 4 ways and its eviction watermark.  Loading and
// evaluating are split so that callers can put several loads in flight.
struct RtBucket {
  ulonglong2 a, b;
  uint32_t ev;
};

template <bool CL>
__device__ __forceinline__ RtBucket rt_load(const SrvCtx& c, uint32_t bucket) {
  const ulonglong2* e = reinterpret_cast<const ulonglong2*>(rt_at<CL>(c, bucket));
  RtBucket q;
  q.a = e[0];
  q.b = e[1];
  q.ev = *ev_at<CL>(c, bucket);
  return q;
}

__device__ __forceinline__ RtProbe rt_eval(const RtBucket& q, uint32_t key, uint32_t s, uint32_t e_pre,
                                           uint32_t lastw) {
  const uint64_t w[4] = {q.a.x, q.a.y, q.b.x, q.b.y};
  const uint32_t ev = q.ev;
  RtProbe r;
  r.conflict = lastw > s;
  int hit = -1, old = 0;
  uint32_t oldc = 0xFFFFFFFFu;
#pragma unroll
  for (int i = 0; i < kRtWays; ++i) {
    const uint32_t k = (uint32_t)w[i], cc = (uint32_t)(w[i] >> 32);
    if (k == key) {
      hit = i;
      r.conflict |= cc > s;
    }
    if (cc < oldc) {
      oldc = cc;
      old = i;
    }
  }
  r.unknown = !r.conflict && ev > e_pre;
  r.way = hit >= 0 ? hit : old;
  return r;
}

template <bool CL>
__device__ __forceinline__ RtProbe rt_probe(const SrvCtx& c, uint32_t bucket, uint32_t key, uint32_t s,
                                            uint32_t e_pre, uint32_t lastw) {
  return rt_eval(rt_load<CL>(c, bucket), key, s, e_pre, lastw);
}

// Record (key, cts) into `way` of its bucket; an evicted entry of another
// key raises evmax.  Exchanges by several lanes on one slot are serialised
// by the hardware and each evictor sees the value it replaced.
template <bool CL>
__device__ __forceinline__ void rt_record(const SrvCtx& c, uint32_t bucket, int way, uint32_t key, uint32_t cts) {
  const unsigned long long old =
      atomicExch(reinterpret_cast<unsigned long long*>(rt_at<CL>(c, bucket) + way), ((unsigned long long)cts << 32) | key);
  if ((uint32_t)old != key && (uint32_t)(old >> 32) != 0u) atomicMax(ev_at<CL>(c, bucket), (uint32_t)(old >> 32));
}

// ---------------------------------------------------------------------------
// Recent-write filter (the on-chip level of the ATR for the bank worker).
// The same smem as the table above, read as 2^(rt_log2+3) u32 slots striped
// over the server CTAs: slot i holds the largest CTS of any committed write
// whose item hashes to i under one of kFiltK hash functions (a batch stores
// its LAST CTS for all of its writes, so lanes that share a slot store the
// same value and plain stores suffice -- the critical-section holder is the
// only writer).  Values only grow.  For a transaction with snapshot s,
// validated with lastw prefetched at tail e_pre >= s:
//    conflict  iff  lastw[x] > s                        (exact, every CTS <= e_pre)
//    unknown   iff  no conflict and min_k F[h_k(x)] > e_pre
// A write of x after e_pre raises all k slots of x above e_pre, so "no
// unknown" proves there was none; "unknown" aborts with the labelled reason
// OVERFLOW -- a true conflict inside the window, or a false
// positive with probability ~(k W / slots)^k for W writes in the window.
// Per item: k loads and k stores, no atomics, no eviction.
// ---------------------------------------------------------------------------
constexpr int kFiltK = 3;
#ifndef CSMV_BANK_FILT_K
#define CSMV_BANK_FILT_K 2
#endif
constexpr int kBankFiltK = CSMV_BANK_FILT_K;  // hashes the locked bank worker uses (<= kFiltK)
static_assert(kBankFiltK >= 1 && kBankFiltK <= kFiltK, "CSMV_BANK_FILT_K must be 1..kFiltK");

// KV requests in the compact {set clock} u WS form use the filter
__device__ __forceinline__ bool kv_filter_mode(const KParams& p) {
  return p.kv_A > kKvFullWays || !(p.debug & CSMV_DBG_KV_ITEMSETS);
}

// slot k of item x: multiplicative hashes with three odd constants
__device__ __forceinline__ uint32_t filt_slot(uint32_t x, int k, uint32_t slots_log2) {
  const uint32_t C[3] = {0x9E3779B1u, 0x85EBCA77u, 0xC2B2AE3Du};
  return (x * C[k]) >> (32 - slots_log2);
}
// the same hashes onto n slots (n not a power of two): the high word of h * n
__device__ __forceinline__ uint32_t filt_slot_n(uint32_t x, int k, uint32_t n) {
  const uint32_t C[3] = {0x9E3779B1u, 0x85EBCA77u, 0xC2B2AE3Du};
  return __umulhi(x * C[k], n);
}

// 32-bit shared-window address of filter slot i (a shared::cluster address
// of the owning CTA for the cluster server)
template <bool CL>
__device__ __forceinline__ uint32_t filt_addr(const SrvCtx& c, uint32_t i) {
  if constexpr (!CL) {
    return c.rt32 + 4u * i;
  } else {
    const uint32_t owner = i & ((1u << c.clog2) - 1), local = c.rt32 + 4u * (i >> c.clog2);
    uint32_t a;
    asm("mapa.shared::cluster.u32 %0, %1, %2;" : "=r"(a) : "r"(local), "r"(owner));
    return a;
  }
}
template <bool CL>
__device__ __forceinline__ uint32_t filt_ld(uint32_t a) {
  uint32_t v;
  if constexpr (CL) asm volatile("ld.shared::cluster.u32 %0, [%1];" : "=r"(v) : "r"(a) : "memory");
  else asm volatile("ld.shared.u32 %0, [%1];" : "=r"(v) : "r"(a) : "memory");
  return v;
}
template <bool CL>
__device__ __forceinline__ void filt_st(uint32_t a, uint32_t v) {
  if constexpr (CL) asm volatile("st.shared::cluster.u32 [%0], %1;" ::"r"(a), "r"(v) : "memory");
  else asm volatile("st.shared.u32 [%0], %1;" ::"r"(a), "r"(v) : "memory");
}

// The bank filter keeps 16-bit slots (twice the slots in the same shared
// memory, so far fewer false positives): slot i holds the low 16 bits of the
// last CTS stored into it, and slots are written in CTS order (by the
// critical-section holder / the committer).  With tail t and a window
// W = t - e_pre < 2^16, a slot written at c in (e_pre, t] has age
// (t - v) mod 2^16 = t - c < W; an older slot may alias into the window
// (probability ~W / 2^16), which is only a false positive.  So
//    unknown(x)  iff  W >= 2^16  or  max_k age(F[h_k(x)]) < W
// never misses a write of x after e_pre.
__device__ __forceinline__ uint32_t filt16_age(uint32_t t, uint32_t v) { return (t - v) & 0xFFFFu; }

template <bool CL>
__device__ __forceinline__ uint32_t filt16_addr(const SrvCtx& c, uint32_t i) {
  if constexpr (!CL) {
    return c.rt32 + 2u * i;
  } else {
    const uint32_t owner = i & ((1u << c.clog2) - 1), local = c.rt32 + 2u * (i >> c.clog2);
    uint32_t a;
    asm("mapa.shared::cluster.u32 %0, %1, %2;" : "=r"(a) : "r"(local), "r"(owner));
    return a;
  }
}
template <bool CL>
__device__ __forceinline__ uint32_t filt16_ld(uint32_t a) {
  uint16_t v;
  if constexpr (CL) asm volatile("ld.shared::cluster.u16 %0, [%1];" : "=h"(v) : "r"(a) : "memory");
  else asm volatile("ld.shared.u16 %0, [%1];" : "=h"(v) : "r"(a) : "memory");
  return v;
}
template <bool CL>
__device__ __forceinline__ void filt16_st(uint32_t a, uint32_t v) {
  const uint16_t h = (uint16_t)v;
  if constexpr (CL) asm volatile("st.shared::cluster.u16 [%0], %1;" ::"r"(a), "h"(h) : "memory");
  else asm volatile("st.shared.u16 [%0], %1;" ::"r"(a), "h"(h) : "memory");
}

// ---------------------------------------------------------------------------
// Receiver warp: sweeps its slice of the client doorbells with
// coalesced loads and dispatches new requests to this CTA's workers through
// a shared-memory queue (entry = lap << 32 | client warp; a worker that
// claimed slot i waits for lap i / QN + 1).  At most one request per client
// warp is outstanding, so QN >= slice slots never wrap onto an unconsumed
// entry.
// ---------------------------------------------------------------------------
static __device__ void server_receiver(const KParams& p, const SrvCtx& c, uint64_t t_begin) {
  const uint32_t FULL = 0xFFFFFFFFu;
  const uint32_t lane = threadIdx.x & 31;
  const uint32_t n = c.cw_hi - c.cw_lo;
  const uint32_t rows = (n + 31) / 32;
  const uint32_t lt = lanemask_lt();
  const uint32_t qmask = (1u << c.qn_log2) - 1;
  uint32_t tail = 0;
  uint32_t idle = 0;
  Jitter jit(p, 3);
  for (;;) {
    jit();
    bool found = false;
    for (uint32_t r0 = 0; r0 < rows; r0 += 8) {
      bool fenced = false;  // per group of 8 rows: each group's doorbells are loaded after the last fence
      uint32_t seq[8];
#pragma unroll
      for (int k = 0; k < 8; ++k) {
        const uint32_t i = (r0 + k) * 32 + lane;
        seq[k] = (r0 + k < rows && i < n) ? ld_relaxed(p.req_seq + c.cw_lo + i) : 0u;
      }
#pragma unroll
      for (int k = 0; k < 8; ++k) {
        const uint32_t i = (r0 + k) * 32 + lane;
        const bool pend = r0 + k < rows && i < n && seq[k] != c.last_seen[i];
        const uint32_t pm = __ballot_sync(FULL, pend);
        if (pm) {
          found = true;
          if (!fenced && !p.req_tagged) {  // acquire: the payloads of this group's doorbells
            fence_gpu();  // precede every worker's reads of them (queue -> fence.cta -> loads);
            fenced = true;  // tagged requests: the worker checks the round in every word instead
          }
          if (pend) {
            const uint32_t pos = tail + __popc(pm & lt);
            c.last_seen[i] = seq[k];
            // {slot tag, request round (low 16 bits) << 16 | client warp}
            *(volatile uint64_t*)&c.queue[pos & qmask] =
                ((uint64_t)((pos >> c.qn_log2) + 1) << 32) | ((seq[k] & 0xFFFFu) << 16) | (c.cw_lo + i);
          }
          tail += __popc(pm);
        }
      }
    }
    if (found) {
      idle = 0;
      continue;
    }
    // an idle sweep backs off briefly: the receiver shares the server SM's
    // issue slots and load pipe with the critical section
    if (CSMV_SLEEP_RECV) __nanosleep(CSMV_SLEEP_RECV);
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
        if (lane == 0) *(volatile uint32_t*)&c.sh->exit = 1;
        return;
      }
    }
  }
}

// Claim the next dispatched request of this CTA's queue (blocking): its
// client warp and (rq) the low 16 bits of its round.  Returns false when the
// receiver has finished.
__device__ __forceinline__ bool claim_request(const SrvCtx& c, uint32_t& cw, uint32_t* rq = nullptr) {
  const uint32_t FULL = 0xFFFFFFFFu;
  const uint32_t qmask = (1u << c.qn_log2) - 1;
  uint32_t slot = 0;
  if ((threadIdx.x & 31) == 0) slot = atomicAdd(&c.sh->q_head, 1u);
  slot = __shfl_sync(FULL, slot, 0);
  for (;;) {  // convergent wait: every lane polls the same word (broadcast LDS)
    const uint64_t ent = *(volatile uint64_t*)&c.queue[slot & qmask];
    if ((uint32_t)(ent >> 32) == (slot >> c.qn_log2) + 1) {
      cw = (uint32_t)ent & 0xFFFFu;
      if (rq) *rq = ((uint32_t)ent >> 16) & 0xFFFFu;
      return true;
    }
    if (*(volatile uint32_t*)&c.sh->exit) return false;
    __nanosleep(CSMV_SLEEP_QUEUE);
  }
}

// Ticket lock around the commit critical section, in CTA 0's shared memory.
// One CTA: acquire = ld.acquire.cta of now_serving (a plain LDS), release =
// st.release.cta (one MEMBAR.CTA) -- no fences beyond that.  Cluster: the
// DSMEM words with cluster-scope fences.
template <bool CL>
__device__ __forceinline__ uint32_t cs_enter(const SrvCtx& c) {
  uint32_t ticket = 0;
  if ((threadIdx.x & 31) == 0) ticket = atomicAdd(&c.sh0->next_ticket, 1u);
  ticket = __shfl_sync(0xFFFFFFFFu, ticket, 0);
  if constexpr (CL) {
    while (*(volatile uint32_t*)&c.sh0->now_serving != ticket) __nanosleep(16);
    __syncwarp();
    srv_fence<CL>();
  } else {
    const uint32_t a = (uint32_t)__cvta_generic_to_shared(&c.sh0->now_serving);
    for (;;) {
      uint32_t v;
      asm volatile("ld.acquire.cta.shared::cta.u32 %0, [%1];" : "=r"(v) : "r"(a) : "memory");
      if (v == ticket) break;
      if (CSMV_SLEEP_LOCK) __nanosleep(CSMV_SLEEP_LOCK);
    }
    __syncwarp();
  }
  return ticket;
}

template <bool CL>
__device__ __forceinline__ void cs_leave(const SrvCtx& c, uint32_t ticket, uint32_t new_tail) {
  __syncwarp();
  if constexpr (CL) {
    srv_fence<CL>();
    if ((threadIdx.x & 31) == 0) {
      *(volatile uint32_t*)&c.sh0->tail = new_tail;
      srv_fence<CL>();
      *(volatile uint32_t*)&c.sh0->now_serving = ticket + 1;
    }
  } else if ((threadIdx.x & 31) == 0) {
    // one fence orders every store of the section (the warp's, through the
    // __syncwarp above: filter slots, and the KV workers' lastw) before BOTH
    // the tail -- which KV workers read outside the lock as e_pre and then
    // load lastw under it -- and the lock handoff
    fence_cta();
    *(volatile uint32_t*)&c.sh0->tail = new_tail;
    *(volatile uint32_t*)&c.sh0->now_serving = ticket + 1;
  }
}

// done-ring back-pressure (CSMV_PUBLISH_SERVER): CTS t may reuse slot
// t & mask only once GTS >= t - 2^20
__device__ __forceinline__ void done_ring_room(const KParams& p, const SrvCtx& c, uint32_t t, uint64_t t_begin) {
  const uint32_t dmask = (1u << kDoneLog2) - 1;
  if ((threadIdx.x & 31) == 0) {
    uint32_t it = 0;
    while (t > *(volatile uint32_t*)&c.sh0->gts_seen + dmask) {
      *(volatile uint32_t*)&c.sh0->gts_seen = ld_relaxed(p.gts);
      if ((++it & 255u) == 0 && watchdog(p, t_begin, 4)) break;
    }
  }
  __syncwarp();
}

// ---------------------------------------------------------------------------
// The paper's ATR (CSMV_ATR_LIST / CSMV_ATR_LIST_NOCV, single-CTA server):
// a CTS-indexed ring of R write-set records in shared memory;
// entry c holds the write-set of the commit with CTS c.  A transaction with
// snapshot s is validated against the entries (s, t] -- every commit after
// its snapshot; if the ring no longer holds them all
// (t - s >= R) it aborts with the labelled reason OVERFLOW.
//  * LIST (collaborative validation): the transactions of
//    the batch are validated one after another; for each, every lane takes
//    the same read/write-set entries e_t (a broadcast) and stripes over the
//    ATR records, and __any_sync combines the lanes' findings;
//  * LIST_NOCV (CSMV-NoCV): each lane validates its own
//    transaction by scanning every record of the window itself.
// ---------------------------------------------------------------------------
__device__ __forceinline__ void atr_list_validate(const KParams& p, const SrvCtx& c, uint32_t s, uint32_t t,
                                                  bool mine, uint32_t a, uint32_t b, bool& ovf, bool& conflict) {
  const uint32_t FULL = 0xFFFFFFFFu;
  const uint32_t lane = threadIdx.x & 31;
  const uint32_t R = (uint32_t)kRtWays << (p.rt_log2 - p.clog2);
  const uint64_t* atr = c.rt;
  ovf = mine && (t - s >= R);
  conflict = false;
  if (p.atr_mode == CSMV_ATR_LIST) {
    uint32_t need = __ballot_sync(FULL, mine && !ovf), found = 0;
    while (need) {
      const int i = __ffs(need) - 1;
      need &= need - 1;
      const uint32_t ea = __shfl_sync(FULL, a, i), eb = __shfl_sync(FULL, b, i);
      bool f = false;
      for (uint32_t q = s + 1 + lane; q - 1 < t; q += 32) {  // q in (s, t], striped over lanes
        const uint64_t e = atr[q & (R - 1)];
        const uint32_t w0 = (uint32_t)e, w1 = (uint32_t)(e >> 32);
        f |= w0 == ea || w0 == eb || w1 == ea || w1 == eb;
      }
      if (__any_sync(FULL, f)) found |= 1u << i;
    }
    conflict = (found >> lane) & 1u;
  } else if (mine && !ovf) {
    for (uint32_t q = s + 1; q - 1 < t; ++q) {
      const uint64_t e = atr[q & (R - 1)];
      const uint32_t w0 = (uint32_t)e, w1 = (uint32_t)(e >> 32);
      conflict |= w0 == a || w0 == b || w1 == a || w1 == b;
    }
  }
}

// CSMV_RECV_SELF (bank, one CTA, ticket-locked commit): the worker warps
// receive for themselves -- no receiver warp, no dispatch queue
__device__ __forceinline__ bool kv_filter_mode(const KParams& p);

__device__ __forceinline__ bool server_self_recv(const KParams& p) {
  if (p.server_recv != CSMV_RECV_SELF || p.n_server_ctas != 1) return false;
  if (p.kind == CSMV_KIND_KV) return kv_filter_mode(p);  // the KV filter worker, one batch per claim
  return p.atr_mode == CSMV_ATR_HASH && p.commit == CSMV_COMMIT_CSMV && !(p.debug & CSMV_DBG_ALT_COMMIT);
}

// Self-receiving worker: sweep this worker's slice [lo, hi) of the client
// doorbells with coalesced loads and claim up to m_max new requests, lowest
// client warp first (P:103's receiver, folded into the worker).  Returns the
// number claimed; 0 once every client has finished (or on error).  At most
// one request per client warp is outstanding, and only this warp reads or
// writes last_seen[lo, hi).  GTS is read (relaxed) with the doorbells of
// each sweep; the acquire fence after a successful sweep orders it too, so
// `gts` is an acquired e_pre for the lastw prefetch with no further round
// trip (ld.relaxed; fence.acq_rel.gpu = acquire).
template <int M>
__device__ __forceinline__ uint32_t self_claim(const KParams& p, const SrvCtx& c, uint32_t lo, uint32_t hi,
                                               uint32_t m_max, uint32_t (&cwv)[M], uint32_t (&rqv)[M], uint64_t t_begin,
                                               uint32_t& gts) {
  const uint32_t FULL = 0xFFFFFFFFu;
  const uint32_t lane = threadIdx.x & 31;
  const uint32_t n = hi - lo, rows = (n + 31) / 32;
  for (uint32_t idle = 1;; ++idle) {
    uint32_t m = 0;
    uint32_t g = 0;
    // tagged requests: no fence after the sweep, so GTS is read with
    // acquire semantics here (the lastw prefetch is ordered after it)
    if (lane == 0) g = p.req_tagged ? ld_acquire(p.gts) : ld_relaxed(p.gts);
    for (uint32_t r0 = 0; r0 < rows && m < m_max; r0 += 4) {
      // the doorbells of up to 4 rows in flight at once: one L2 round trip
      uint32_t sqv[4];
#pragma unroll
      for (int k = 0; k < 4; ++k) {
        const uint32_t i = (r0 + k) * 32 + lane;
        sqv[k] = (r0 + k < rows && i < n) ? ld_relaxed(p.req_seq + lo + i) : 0u;
      }
#pragma unroll
      for (int k = 0; k < 4; ++k) {
        const uint32_t r = r0 + k, i = r * 32 + lane;
        if (r >= rows || m >= m_max) break;
        uint32_t pm = __ballot_sync(FULL, i < n && sqv[k] != c.last_seen[lo - c.cw_lo + i]);
#pragma unroll
        for (int j = 0; j < M; ++j) {
          if ((uint32_t)j == m && pm && m < m_max) {
            const uint32_t l = __ffs(pm) - 1;
            pm &= pm - 1;
            if (lane == l) c.last_seen[lo - c.cw_lo + i] = sqv[k];
            cwv[j] = lo + r * 32 + l;
            rqv[j] = __shfl_sync(FULL, sqv[k], l) & 0xFFFFu;
            m = j + 1;
          }
        }
      }
    }
    if (m) {
      if (!p.req_tagged) fence_gpu();  // acquire: the payloads of the doorbells just seen precede our loads of them
      gts = __shfl_sync(FULL, g, 0);
      return m;
    }
    if ((idle & 15u) == 0) {
      uint32_t fin = 0;
      if (lane == 0) {
        const uint32_t er = ld_relaxed(&p.ctl->error);
        fin = er || ld_relaxed(&p.ctl->done_warps) >= p.n_cw || watchdog(p, t_begin, 3);
      }
      if (__shfl_sync(FULL, fin, 0)) return 0;
    }
  }
}

// ---------------------------------------------------------------------------
// Bank worker warp.  Claims up to kMaxCombine dispatched batches (the first
// blocking, the rest only if already queued), loads them outside the lock,
// and commits them inside ONE critical section, one after another in queue
// order -- exactly as if each had its own critical section: batch j is
// validated after batch j-1's write-set was recorded, and receives the next
// consecutive CTS range.  A batch is validated by the whole warp,
// one lane per transaction, __ballot_sync for the commit mask.
//
// G > 1 (csmv_workload.client_group, CTA-level batches): a request is the
// G sub-batches of a client group (client_bank.cuh), mutually conflict-free
// by the clients' cross-warp pre-validation.  Up to M/G requests are combined;
// within one, the G sub-batches' filter probes are issued together and
// evaluated against the same window (none can conflict with another), their
// CTS ranges follow one another in warp order, and their filter slots are
// stored once with the request's last CTS: one step of the serial chain per
// request instead of one per sub-batch.
// ---------------------------------------------------------------------------
#ifndef CSMV_LASTW_ONE_TRIP
#define CSMV_LASTW_ONE_TRIP 1
#endif
constexpr bool kLastwOneTrip = CSMV_LASTW_ONE_TRIP;  // grouped requests: every lastw load of a group in flight at once

template <bool CL, bool SELF, int G = 1>
__device__ void server_worker(const KParams& p, const SrvCtx& c, uint64_t t_begin) {
#ifndef CSMV_G4_REQS
#define CSMV_G4_REQS 2
#endif
  constexpr int M = G == 4 ? 4 * CSMV_G4_REQS : kMaxCombine;  // sub-batches held per critical section
  constexpr int MR = M / G;  // requests per critical section
  static_assert(!SELF || G == 1, "self-receiving workers take per-warp batches");
  const uint32_t FULL = 0xFFFFFFFFu;
  const uint32_t lane = threadIdx.x & 31;
  const uint32_t lt = lanemask_lt();
  const uint32_t qmask = (1u << c.qn_log2) - 1;
  const uint32_t m_max = G > 1 ? max(1u, min(p.combine, (uint32_t)M) / G)
                              : (p.combine < 1 ? 1u : (p.combine > (uint32_t)M ? (uint32_t)M : p.combine));
  unsigned long long busy = 0, locked = 0, batches = 0, groups = 0;
  unsigned long long ph[8] = {0, 0, 0, 0, 0, 0, 0, 0};
  constexpr bool self = SELF;
  Jitter jit(p, 4);
  uint32_t my_lo = 0, my_hi = 0;
  if constexpr (SELF) {
    const uint32_t w = threadIdx.x >> 5, per = (c.cw_hi - c.cw_lo + p.n_workers - 1) / p.n_workers;
    my_lo = min(c.cw_lo + w * per, c.cw_hi);
    my_hi = min(my_lo + per, c.cw_hi);
  }
  uint32_t gts_claim = 0;  // SELF: GTS read with the doorbells (acquired by the claim's fence)
  for (;;) {
    const long long tq = clock64();
    uint32_t cwv[M], rqv[M];  // client warps, their rounds (low 16 bits: tagged requests)
    uint32_t m = 1;
    if constexpr (SELF) {
      m = self_claim<M>(p, c, my_lo, my_hi, m_max, cwv, rqv, t_begin, gts_claim);
      if (!m) break;
    } else {
      if (!claim_request(c, cwv[0], &rqv[0])) break;
    }
    const uint64_t t_claim = trace_now(p);
    // ---- combine: grab further requests that are already queued
#pragma unroll
    for (int j = 1; j < MR; ++j) {
      uint32_t got = 0xFFFFFFFFu;
      if (!self && m == (uint32_t)j && m < m_max && lane == 0) {
        const uint32_t h = *(volatile uint32_t*)&c.sh->q_head;
        const uint64_t e = *(volatile uint64_t*)&c.queue[h & qmask];
        if ((uint32_t)(e >> 32) == (h >> c.qn_log2) + 1 && atomicCAS(&c.sh->q_head, h, h + 1) == h) got = (uint32_t)e;
      }
      if (self) continue;
      got = __shfl_sync(FULL, got, 0);
      cwv[j] = got == 0xFFFFFFFFu ? got : got & 0xFFFFu;
      rqv[j] = got >> 16;
      if (got != 0xFFFFFFFFu && m == (uint32_t)j) m = j + 1;
    }
    const uint32_t m_req = m;
    if constexpr (G > 1) {
      // expand request r (its group's first warp) into sub-batches r*G + k:
      // the group's warps lead + k * n_client_ctas, as many as the CTA has
#pragma unroll
      for (int r = MR - 1; r >= 0; --r) {
        const uint32_t lead = cwv[r], cta = lead % p.n_client_ctas, w0 = lead / p.n_client_ctas, lq = rqv[r];
        const uint32_t n_act = min((uint32_t)kWarps, (p.n_cw - cta + p.n_client_ctas - 1) / p.n_client_ctas);
        const uint32_t gs = min((uint32_t)G, n_act - w0);
#pragma unroll
        for (int k = 0; k < G; ++k) {
          cwv[r * G + k] = ((uint32_t)r < m_req && (uint32_t)k < gs) ? lead + k * p.n_client_ctas : 0xFFFFFFFFu;
          rqv[r * G + k] = lq;  // a group's warps run their rounds in lock-step: one round for all
        }
      }
      m = m_req * G;
    }
    const long long t0 = clock64();
    jit();  // claimed, payload not yet loaded
    // ---- load the batches: header and ids together (the receiver's fence
    // ordered them after the doorbells; ours orders them after the queue)
    if (!self) fence_cta();
    uint32_t sq[M], sn[M], msk[M], id0[M], id1[M];
    // server write-back (self-receiving workers, csmv_workload.server_writeback):
    // the new balances and replacement slots, with the payload
    uint32_t wv0[SELF ? M : 1], wv1[SELF ? M : 1], wvi[SELF ? M : 1];
    if constexpr (SELF) {
#pragma unroll
      for (int j = 0; j < M; ++j) {
        wv0[j] = wv1[j] = wvi[j] = 0;
        if (p.bank_swb && j < (int)m) {
          const uint32_t* rv = p.req_vals + (size_t)cwv[j] * 128 + lane;
          if (!p.req_tagged) {  // tagged: loaded (and checked) with the payload below
            wv0[j] = ld_relaxed(rv);
            wv1[j] = ld_relaxed(rv + 32);
            wvi[j] = ld_relaxed(rv + 64);
          }
        }
      }
    }
    // fenced requests: every load in flight at once, no checks (the
    // receiver's or the claim's fence ordered them after the doorbells).
    // Tagged requests are taken by the self-receiving worker only (the
    // receiver-fed worker of C2 is server-bound: the check costs it ~2 %
    // even when off, so it is not compiled there)
    if (!SELF || !p.req_tagged) {
#pragma unroll
    for (int j = 0; j < M; ++j) {
      sq[j] = sn[j] = msk[j] = id0[j] = id1[j] = 0;
      if (j < (int)m && (G == 1 || cwv[j] != 0xFFFFFFFFu)) {
        sn[j] = ld_relaxed(&p.req_hdr[cwv[j]].snapshot);
        msk[j] = ld_relaxed(&p.req_hdr[cwv[j]].mask);
        sq[j] = ld_relaxed(&p.req_hdr[cwv[j]].round);
        id0[j] = ld_relaxed(p.req_ids + (size_t)cwv[j] * 64 + lane) & ~kWriteBit;
        id1[j] = ld_relaxed(p.req_ids + (size_t)cwv[j] * 64 + 32 + lane) & ~kWriteBit;
      }
    }
    } else
    // tagged requests: loaded again until every word carries the round of
    // the doorbell (the client did not fence the payload before it).  All
    // loads are issued before any is looked at (one round trip).
    for (uint32_t pass = 0;; ++pass) {
      uint64_t w0[M], w1[M];
#pragma unroll
      for (int j = 0; j < M; ++j) {
        w0[j] = w1[j] = 0;
        id0[j] = id1[j] = 0;
        if (j < (int)m && (G == 1 || cwv[j] != 0xFFFFFFFFu)) {
          const uint64_t* hw = reinterpret_cast<const uint64_t*>(&p.req_hdr[cwv[j]]);
          w0[j] = ld_relaxed64(hw);
          w1[j] = ld_relaxed64(hw + 1);
          id0[j] = ld_relaxed(p.req_ids + (size_t)cwv[j] * 64 + lane);
          id1[j] = ld_relaxed(p.req_ids + (size_t)cwv[j] * 64 + 32 + lane);
        }
      }
      // server write-back words: re-read with the payload, checked against the round
      uint32_t wck[SELF ? M : 1];
      if constexpr (SELF) {
#pragma unroll
        for (int j = 0; j < M; ++j) {
          wck[j] = 0;
          if (p.bank_swb && j < (int)m) {
            const uint32_t* rv = p.req_vals + (size_t)cwv[j] * 128 + lane;
            wv0[j] = ld_relaxed(rv);
            wv1[j] = ld_relaxed(rv + 32);
            wvi[j] = ld_relaxed(rv + 64);
            wck[j] = ld_relaxed(rv + 96);
          }
        }
      }
      bool stale = false;
      const uint32_t keep = p.req_tagged ? kIdItemMask : ~kWriteBit, tm = kIdTagMask << kIdItemBits;
#pragma unroll
      for (int j = 0; j < M; ++j) {
        sn[j] = (uint32_t)w0[j];
        sq[j] = (uint32_t)(w0[j] >> 32);
        msk[j] = (uint32_t)w1[j];
        const bool live = j < (int)m && (G == 1 || cwv[j] != 0xFFFFFFFFu);
        if (p.req_tagged && live) {
          const uint32_t tg = id_tag(rqv[j]);
          const bool mj = (msk[j] >> lane) & 1u;
          stale |= (sq[j] & 0xFFFFu) != rqv[j] || (uint32_t)(w1[j] >> 32) != sq[j] ||
                   (mj && ((id0[j] & tm) != tg || (id1[j] & tm) != tg));
          if constexpr (SELF) {
            if (p.bank_swb && mj) stale |= bank_swb_check(sq[j], wv0[j], wv1[j], wvi[j]) != wck[j];
          }
        }
        id0[j] &= keep;
        id1[j] &= keep;
      }
      if (!__any_sync(FULL, stale)) break;
      if ((pass & 1023u) == 1023u) {  // a lost payload would be a protocol error: let the watchdog see it
        uint32_t bad = 0;
        if (lane == 0) bad = ld_relaxed(&p.ctl->error) || watchdog(p, t_begin, 5);
        if (__shfl_sync(FULL, bad, 0)) break;
      }
    }
    bool mine[M];
#pragma unroll
    for (int j = 0; j < M; ++j) {
      mine[j] = (msk[j] >> lane) & 1u;
      if (!mine[j]) id0[j] = id1[j] = 0;
    }
    const bool hash = G > 1 || p.atr_mode == CSMV_ATR_HASH;
    // lastw covers every CTS <= e_pre: clients write lastw with their
    // write-back, before the commit is published, so e_pre = GTS (acquire;
    // self-receiving workers already hold one from their claim)
    const uint32_t e_pre = SELF ? gts_claim : (hash ? ld_acquire(p.gts) : *(volatile uint32_t*)&c.sh0->tail);
    if (!SELF) srv_fence<CL>();
    const bool novalid = (p.debug & CSMV_DBG_NO_VALIDATE) != 0;
    // HASH: the exact part of the validation (lastw, every CTS <= e_pre) and
    // the filter slot addresses are settled before the lock
    bool chk[M];
    uint32_t fa[M][kFiltK], fb[M][kFiltK];
    uint32_t xor_all = e_pre;
    const uint32_t fl2 = p.rt_log2 + 4;  // 16-bit filter slots
    // Self-receiving workers (latency-bound hot-item chains, C3): all 2M
    // lastw loads in one L2 round trip (idle lanes read lastw[0]).  With a
    // receiver (C2) they stay one round trip per batch: that latency is the
    // window in which further batches queue up to be combined
    // (profiles/r01/ab_late.md).
    uint32_t lwa[M], lwb[M];
#pragma unroll
    for (int j = 0; j < M; ++j) {
      lwa[j] = lwb[j] = 0;
      if ((SELF || (G > 1 && kLastwOneTrip)) && hash) {
        lwa[j] = ld_relaxed(p.lastw + id0[j]);
        lwb[j] = ld_relaxed(p.lastw + id1[j]);
      }
    }
#pragma unroll
    for (int j = 0; j < M; ++j) {
      uint32_t lw0 = lwa[j], lw1 = lwb[j];
      if (!(SELF || (G > 1 && kLastwOneTrip)) && mine[j] && hash) {
        lw0 = ld_relaxed(p.lastw + id0[j]);
        lw1 = ld_relaxed(p.lastw + id1[j]);
      }
      chk[j] = mine[j] && (novalid || (lw0 <= sn[j] && lw1 <= sn[j]));
#pragma unroll
      for (int k = 0; k < kFiltK; ++k) {
        fa[j][k] = filt16_addr<CL>(c, p.filt16_n ? filt_slot_n(id0[j], k, p.filt16_n) : filt_slot(id0[j], k, fl2));
        fb[j][k] = filt16_addr<CL>(c, p.filt16_n ? filt_slot_n(id1[j], k, p.filt16_n) : filt_slot(id1[j], k, fl2));
      }
      xor_all ^= lw0 ^ lw1 ^ sn[j];
    }
    // The payload must have arrived before the lock is taken: a warp vote on
    // values derived from it makes the loads complete here.
    if (__ballot_sync(FULL, xor_all == 0x12345679u) == FULL) __nanosleep(1);
    jit();  // lastw checked against e_pre, lock not yet taken
    const long long tl = clock64();
    // ---- critical section: validate, reserve CTS, record
    const uint32_t ticket = cs_enter<CL>(c);
    const long long t1 = clock64();
    const uint32_t t0c = *(volatile uint32_t*)&c.sh0->tail;
    uint32_t t = t0c;
    uint32_t cm[M], om[M], base[M];
    bool ovfl[M];
    if (hash) {
      // request r (sub-batches r*G .. r*G+G-1): a write after e_pre to one of
      // its items raised all of that item's slots above e_pre (earlier
      // requests of this section included; the sub-batches of one request
      // are conflict-free, so they need not see each other's stores)
#pragma unroll
      for (int r = 0; r < MR; ++r) {
#pragma unroll
        for (int k = 0; k < G; ++k) {
          const int j = r * G + k;
          cm[j] = om[j] = 0;
          ovfl[j] = false;
          base[j] = t + 1;
        }
        if ((uint32_t)r < m_req) {
          // every lane probes (a lane without a live transaction probes the
          // slots of item 0, a valid address): no predicated loads and no
          // zero-fill moves in the chain; chk masks the result
          uint32_t va[G][kFiltK], vb[G][kFiltK];
          bool cmt[G];
#pragma unroll
          for (int k = 0; k < G; ++k) {
#pragma unroll
            for (int q = 0; q < kBankFiltK; ++q) {
              va[k][q] = filt16_ld<CL>(fa[r * G + k][q]);
              vb[k][q] = filt16_ld<CL>(fb[r * G + k][q]);
            }
          }
          // slot v is recent iff its CTS lies in (e_pre, t]: (v - e_pre - 1) mod 2^16 < t - e_pre
          const uint32_t win = t - e_pre;  // commits the exact lastw check did not cover
#pragma unroll
          for (int k = 0; k < G; ++k) {
            const int j = r * G + k;
            bool ra = true, rb = true;
#pragma unroll
            for (int q = 0; q < kBankFiltK; ++q) {
              ra = ra && ((va[k][q] - e_pre - 1u) & 0xFFFFu) < win;
              rb = rb && ((vb[k][q] - e_pre - 1u) & 0xFFFFu) < win;
            }
            const bool ovf = chk[j] && !novalid && (win > 0xFFFFu || ra || rb);
            cmt[k] = chk[j] && !ovf;
            cm[j] = __ballot_sync(FULL, cmt[k]);
            ovfl[j] = ovf;  // the overflow mask is voted after the lock
            base[j] = t + 1;
            t += __popc(cm[j]);
          }
#pragma unroll
          for (int k = 0; k < G; ++k) {
            const int j = r * G + k;
            if (cmt[k]) {
#pragma unroll
              for (int q = 0; q < kBankFiltK; ++q) {  // the request's last CTS: equal values, race-free
                filt16_st<CL>(fa[j][q], t);
                filt16_st<CL>(fb[j][q], t);
              }
            }
          }
          __syncwarp();  // request r's records precede request r+1's probes
        }
      }
    } else {
#pragma unroll
      for (int j = 0; j < M; ++j) {
        cm[j] = om[j] = 0;
        base[j] = t + 1;
        if (j >= (int)m) continue;
        bool ovf = false, conflict = false;
        atr_list_validate(p, c, sn[j], t, mine[j], id0[j], id1[j], ovf, conflict);
        if (novalid) ovf = conflict = false;
        const bool commit = mine[j] && !ovf && !conflict;
        cm[j] = __ballot_sync(FULL, commit);
        om[j] = __ballot_sync(FULL, ovf);
        const uint32_t cts = t + 1 + __popc(cm[j] & lt);
        t += __popc(cm[j]);
        // the paper's ATR: the write-set of commit `cts` at entry cts
        if (commit) c.rt[cts & ((uint32_t)(kRtWays << (p.rt_log2 - p.clog2)) - 1)] = ((uint64_t)id1[j] << 32) | id0[j];
        __syncwarp();  // batch j's records precede batch j+1's validation
      }
    }
    const long long ta = clock64();
    if (p.publish == CSMV_PUBLISH_SERVER && t != t0c) done_ring_room(p, c, t, t_begin);
    cs_leave<CL>(c, ticket, t);
    const long long t2 = clock64();
    if constexpr (SELF) {
      // Server write-back (csmv_workload.server_writeback): each committed
      // transfer's two versions and lastw, then its done flag -- the
      // publisher advances GTS over them (the clients' invariant: GTS = g
      // implies lastw and the rings hold every commit <= g)
      if (p.bank_swb && t != t0c) {
        const uint32_t NS = p.K <= 2 ? 2u : p.K <= 4 ? 4u : p.K <= 8 ? 8u : 16u;  // ring slots (host nslot_for)
        jit();
#pragma unroll
        for (int j = 0; j < M; ++j) {
          if (j < (int)m && ((cm[j] >> lane) & 1u)) {
            const uint32_t cts = base[j] + __popc(cm[j] & lt);
            st_relaxed64(p.rings + (size_t)id0[j] * NS + (wvi[j] & 0xFFu), ((uint64_t)cts << 32) | wv0[j]);
            st_relaxed64(p.rings + (size_t)id1[j] * NS + ((wvi[j] >> 8) & 0xFFu), ((uint64_t)cts << 32) | wv1[j]);
            st_relaxed(p.lastw + id0[j], cts);
            st_relaxed(p.lastw + id1[j], cts);
            if (p.publish == CSMV_PUBLISH_SERVER) st_release(p.done_ring + (cts & ((1u << kDoneLog2) - 1)), cts);
          }
        }
        if (p.publish == CSMV_PUBLISH_CLIENT) {  // this worker advances GTS over its range, in CTS order
          __syncwarp();
          fence_gpu();
          if (lane == 0) {
            uint32_t it = 0;
            while (ld_relaxed(p.gts) != t0c) {
              if ((++it & 255u) == 0 && (ld_relaxed(&p.ctl->error) || watchdog(p, t_begin, 6))) break;
              __nanosleep(32);
            }
            st_release(p.gts, t);
          }
          __syncwarp();
        }
      }
    }
    if (hash) {
#pragma unroll
      for (int j = 0; j < M; ++j) om[j] = __ballot_sync(FULL, ovfl[j]);
    }
    // ---- respond: round-tagged words, no fence (kernel.cuh Resp);
    // only to warps that submitted something (a grouped warp with mask 0
    // waits for nothing, and a late word could land on its next request)
    if (lane < (uint32_t)m) {
#pragma unroll
      for (int j = 0; j < M; ++j) {
        if ((uint32_t)j == lane && msk[j] != 0) {
          trace_served(p, cwv[j], sq[j], t_claim);
          const uint64_t tag = (uint64_t)sq[j] << 32;
          st_relaxed64(&p.resp[cwv[j]].base, tag | base[j]);
          st_relaxed64(&p.resp[cwv[j]].commit, tag | cm[j]);
          st_relaxed64(&p.resp[cwv[j]].ovf, tag | om[j]);
        }
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
    batches += m_req;
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

// bank + recent-write filter: the cluster server commits through the commit
// ring (below), the single-CTA server under the ticket lock (server_worker);
// CSMV_DBG_ALT_COMMIT swaps them
__device__ __forceinline__ bool server_uses_ring(const KParams& p) {
  return p.kind == CSMV_KIND_BANK && p.atr_mode == CSMV_ATR_HASH && p.commit == CSMV_COMMIT_CSMV &&
         ((p.n_server_ctas > 1) != ((p.debug & CSMV_DBG_ALT_COMMIT) != 0));
}

// ---------------------------------------------------------------------------
// Bank commit through the commit ring (atr_mode HASH, the default).
// The order-dependent part of a commit -- filter probe, CTS assignment,
// filter update, lastw, respond -- is run by ONE committer warp
// in CTA 0, which owns the recent-write filter and the CTS counter outright:
// no lock, no lock handoff, and its filter accesses are local shared memory
// even in a cluster.  Worker warps (every server CTA) do everything that needs
// no order: claim dispatched batches, load them, prefetch lastw and settle the
// exact part of the validation (lastw[x] <= s for every CTS <= e_pre), compute
// the filter-slot addresses, and push the prepared batches into the ring in
// CTA 0's shared memory (DSMEM stores from the other CTAs of a cluster).  The
// committer takes the slots in ring order, so every batch is validated after
// the write-sets of all batches before it were recorded and receives the next
// consecutive CTS range -- as if each had held the lock in that order.
// G > 1 (client groups): a request's G batches go into G consecutive slots
// (requests never straddle: slots are claimed in whole requests) and the
// committer commits the G slots in one step of its chain.
// ---------------------------------------------------------------------------
template <bool CL, int G = 1>
__device__ void server_worker_cm(const KParams& p, const SrvCtx& c, uint64_t t_begin) {
  constexpr int M = kMaxCombine;
  constexpr int MR = M / G;  // requests per claim
  const uint32_t R = 1u << p.cm_ring_log2;
  const uint32_t FULL = 0xFFFFFFFFu;
  const uint32_t lane = threadIdx.x & 31;
  const uint32_t qmask = (1u << c.qn_log2) - 1;
  const uint32_t m_max = G > 1 ? max(1u, min(p.combine, (uint32_t)M) / G)
                              : (p.combine < 1 ? 1u : (p.combine > (uint32_t)M ? (uint32_t)M : p.combine));
  const uint32_t fl2 = p.rt_log2 - p.clog2 + 3;  // the filter: CTA 0's stripe, 8 << local_log2 32-bit slots
  const bool novalid = (p.debug & CSMV_DBG_NO_VALIDATE) != 0;
  unsigned long long busy = 0, batches = 0, groups = 0, ph0 = 0, ph1 = 0, ph4 = 0;
  Jitter jit(p, 5);
  for (;;) {
    const long long tq = clock64();
    uint32_t cwv[M];
    if (!claim_request(c, cwv[0])) break;
    uint32_t m = 1;
#pragma unroll
    for (int j = 1; j < MR; ++j) {
      uint32_t got = 0xFFFFFFFFu;
      if (m == (uint32_t)j && m < m_max && lane == 0) {
        const uint32_t h = *(volatile uint32_t*)&c.sh->q_head;
        const uint64_t e = *(volatile uint64_t*)&c.queue[h & qmask];
        if ((uint32_t)(e >> 32) == (h >> c.qn_log2) + 1 && atomicCAS(&c.sh->q_head, h, h + 1) == h) got = (uint32_t)e;
      }
      got = __shfl_sync(FULL, got, 0);
      cwv[j] = got == 0xFFFFFFFFu ? got : got & 0xFFFFu;  // the entry's client warp (server_receiver)
      if (got != 0xFFFFFFFFu && m == (uint32_t)j) m = j + 1;
    }
    const uint32_t m_req = m;
    if constexpr (G > 1) {  // request r -> its group's warps lead + k * n_client_ctas (see server_worker)
#pragma unroll
      for (int r = MR - 1; r >= 0; --r) {
        const uint32_t lead = cwv[r], cta = lead % p.n_client_ctas, w0 = lead / p.n_client_ctas;
        const uint32_t n_act = min((uint32_t)kWarps, (p.n_cw - cta + p.n_client_ctas - 1) / p.n_client_ctas);
        const uint32_t gs = min((uint32_t)G, n_act - w0);
#pragma unroll
        for (int k = 0; k < G; ++k)
          cwv[r * G + k] = ((uint32_t)r < m_req && (uint32_t)k < gs) ? lead + k * p.n_client_ctas : 0xFFFFFFFFu;
      }
      m = m_req * G;
    }
    const long long t0 = clock64();
    fence_cta();  // payload loads after the queue entries (the receiver fenced after the doorbells)
    uint32_t sq[M], sn[M], msk[M], id0[M], id1[M];
#pragma unroll
    for (int j = 0; j < M; ++j) {
      sq[j] = sn[j] = msk[j] = id0[j] = id1[j] = 0;
      if (j < (int)m && (G == 1 || cwv[j] != 0xFFFFFFFFu)) {
        sn[j] = ld_relaxed(&p.req_hdr[cwv[j]].snapshot);
        msk[j] = ld_relaxed(&p.req_hdr[cwv[j]].mask);
        sq[j] = ld_relaxed(&p.req_hdr[cwv[j]].round);
        id0[j] = ld_relaxed(p.req_ids + (size_t)cwv[j] * 64 + lane) & ~kWriteBit;
        id1[j] = ld_relaxed(p.req_ids + (size_t)cwv[j] * 64 + 32 + lane) & ~kWriteBit;
      }
    }
    bool mine[M];
#pragma unroll
    for (int j = 0; j < M; ++j) {
      mine[j] = (msk[j] >> lane) & 1u;
      if (!mine[j]) id0[j] = id1[j] = 0;
    }
    // m consecutive ring slots, in claim order
    uint32_t s0 = 0;
    if (lane == 0) s0 = atomicAdd(&c.sh0->ring_head, m);
    s0 = __shfl_sync(FULL, s0, 0);
    const long long tl = clock64();
    {  // room: slot s0+m-1 is free once the committer finished s0+m-1-R
      uint32_t it = 0;
      while ((int)(s0 + m - *(volatile uint32_t*)&c.sh0->ring_done) > (int)R) {
        if ((++it & 1023u) == 0 && (ld_relaxed(&p.ctl->error) || watchdog(p, t_begin, 8))) break;
        __nanosleep(32);
      }
      __syncwarp();
      srv_fence<CL>();  // the committer's reads of the slot's previous use precede our stores
    }
    // lastw prefetched only now: the window the filter must cover is then
    // the ring's depth, not the wait for room as well
    const uint32_t e_pre = ld_acquire(p.gts);  // lastw covers every CTS <= GTS (client write-back)
    srv_fence<CL>();
    jit();  // e_pre read, lastw not yet
    uint32_t chkm[M];
#pragma unroll
    for (int j = 0; j < M; ++j) {
      uint32_t lw0 = 0, lw1 = 0;
      if (mine[j]) {
        lw0 = ld_relaxed(p.lastw + id0[j]);
        lw1 = ld_relaxed(p.lastw + id1[j]);
      }
      chkm[j] = __ballot_sync(FULL, mine[j] && (novalid || (lw0 <= sn[j] && lw1 <= sn[j])));
    }
#pragma unroll
    for (int j = 0; j < M; ++j) {
      if (j < (int)m) {
        const uint32_t sl = c.ring32 + (uint32_t)sizeof(CmSlot) * ((s0 + j) & (R - 1));
        uint4 a, b;  // filter slots as byte offsets (the committer adds CTA 0's base)
        a.x = 4u * filt_slot(id0[j], 0, fl2);
        a.y = 4u * filt_slot(id0[j], 1, fl2);
        a.z = 4u * filt_slot(id0[j], 2, fl2);
        a.w = 4u * filt_slot(id1[j], 0, fl2);
        b.x = 4u * filt_slot(id1[j], 1, fl2);
        b.y = 4u * filt_slot(id1[j], 2, fl2);
        b.z = id0[j];
        b.w = id1[j];
        ring_st_v4<CL>(sl + (uint32_t)offsetof(CmSlot, w) + 16u * lane, a);
        ring_st_v4<CL>(sl + (uint32_t)offsetof(CmSlot, w) + 16u * (32 + lane), b);
        if (lane == 0) ring_st_v4<CL>(sl + 16u, make_uint4(chkm[j], msk[j], 0u, 0u));
        if (lane == 0) filt_st<CL>(sl + 4u, cwv[j]);
        if (lane == 0) filt_st<CL>(sl + 8u, sq[j]);
        if (lane == 0) filt_st<CL>(sl + 12u, novalid ? 0xFFFFFFFFu : e_pre);
      }
    }
    __syncwarp();
    srv_fence<CL>();  // payloads before flags
    if (lane < m) filt_st<CL>(c.ring32 + (uint32_t)sizeof(CmSlot) * ((s0 + lane) & (R - 1)), s0 + lane + 1);
    __syncwarp();
    const long long t3 = clock64();
    busy += (unsigned long long)(t3 - t0);
    ph0 += (unsigned long long)(t0 - tq);
    ph1 += (unsigned long long)(tl - t0);
    ph4 += (unsigned long long)(t3 - tl);
    batches += m_req;
    ++groups;
  }
  __syncwarp();
  if (lane == 0) {
    srv_fence<CL>();  // every flag we wrote precedes the count
    atomicSub(&c.sh0->workers_left, 1u);
    atomicAdd(&p.stats->phase[0], ph0);
    atomicAdd(&p.stats->phase[1], ph1);
    atomicAdd(&p.stats->phase[4], ph4);
    atomicAdd(&p.stats->batches, batches);
    atomicAdd(&p.stats->groups, groups);
    atomicAdd(&p.stats->busy_cycles, busy);
  }
}

// The committer warp (CTA 0).  `ring` is CTA 0's commit ring (local).  The
// next slot's flag and payload are loaded while the current batch is being
// committed, so the serial chain per batch is: filter loads -> commit mask
// -> CTS -> filter stores.
struct CmPayload {
  uint4 w0, w1;
  uint32_t cw, round, e_chk, chkm, msk;
};

template <bool CL>
__device__ __forceinline__ bool cm_try(CmSlot* sl, uint32_t seq, CmPayload& q) {
  const uint32_t f = ring_ld_acquire<CL>((uint32_t)__cvta_generic_to_shared(&sl->flag));
  const uint32_t lane = threadIdx.x & 31;
  q.w0 = sl->w[0][lane];
  q.w1 = sl->w[1][lane];
  const uint4 h = *reinterpret_cast<const uint4*>(sl);
  q.cw = h.y;
  q.round = h.z;
  q.e_chk = h.w;
  q.chkm = sl->chk;
  q.msk = sl->pad[0];
  return __shfl_sync(0xFFFFFFFFu, f, 0) == seq + 1;  // lane 0's view decides
}

// A slot's payload, loaded after its unit's flags were seen (acquire).
__device__ __forceinline__ void cm_load(const CmSlot* sl, CmPayload& q) {
  const uint32_t lane = threadIdx.x & 31;
  q.w0 = sl->w[0][lane];
  q.w1 = sl->w[1][lane];
  const uint4 h = *reinterpret_cast<const uint4*>(sl);
  q.cw = h.y;
  q.round = h.z;
  q.e_chk = h.w;
  q.chkm = sl->chk;
  q.msk = sl->pad[0];
}

template <bool CL, int G = 1>
__device__ void server_committer(const KParams& p, const SrvCtx& c, CmSlot* ring, uint64_t t_begin) {
  const uint32_t R = 1u << p.cm_ring_log2;
  const uint32_t FULL = 0xFFFFFFFFu;
  const uint32_t lane = threadIdx.x & 31;
  const uint32_t dmask = (1u << kDoneLog2) - 1;
  const bool srv_pub = p.publish == CSMV_PUBLISH_SERVER;
  const uint32_t fbase = c.rt32;  // the filter (this CTA's rt stripe); slots arrive as byte offsets
  uint32_t t = *(volatile uint32_t*)&c.sh->tail;
  uint32_t gseen = t;
  unsigned long long cs = 0, wait = 0;
  CmPayload q[G];  // the next unit: one batch, or a client group's G batches
  bool have = false;
  Jitter jit(p, 6);
  // A unit is ready when all its G flags are set.  Its G payloads were all
  // written by one worker warp before one release fence and its flags after
  // it, so one acquire (of the first flag) orders every payload load; the
  // other flags are checked relaxed.  (In a cluster the acquire is LDS +
  // CCTL.IVALL: one per unit instead of one per batch.)
  auto try_unit = [&](uint32_t first) {
    if constexpr (G == 1) {
      return cm_try<CL>(ring + (first & (R - 1)), first, q[0]);
    } else {
      uint32_t ok = 1;
      if (lane == 0) {
#pragma unroll
        for (int k = 1; k < G; ++k)
          ok &= *(volatile uint32_t*)&ring[(first + k) & (R - 1)].flag == first + k + 1;
        ok &= ring_ld_acquire<CL>((uint32_t)__cvta_generic_to_shared(&ring[first & (R - 1)].flag)) == first + 1;
      }
      if (!__shfl_sync(FULL, ok, 0)) return false;
#pragma unroll
      for (int k = 0; k < G; ++k) cm_load(ring + ((first + k) & (R - 1)), q[k]);
      return true;
    }
  };
  for (uint32_t next = 0;; next += G) {
    const long long tw = clock64();
    // wait for the unit starting at slot `next` (unless the prefetch found it ready)
    for (uint32_t it = 0; !have;) {
      have = try_unit(next);
      if (have) break;
      uint32_t done = 0;
      if (lane == 0 && *(volatile uint32_t*)&c.sh->workers_left == 0 &&
          *(volatile uint32_t*)&c.sh->ring_head == next)
        done = 1;
      if (lane == 0 && (++it & 4095u) == 0 && (ld_relaxed(&p.ctl->error) || watchdog(p, t_begin, 9))) done = 1;
      if (__shfl_sync(FULL, done, 0)) break;
    }
    if (!have) break;
    jit();
    const long long t1 = clock64();
    CmPayload cur[G];
#pragma unroll
    for (int k = 0; k < G; ++k) cur[k] = q[k];
    // every lane probes (non-live lanes carry item 0's slots, valid offsets);
    // chk masks the result -- no predicated loads in the chain
    uint32_t v[G][6];
#pragma unroll
    for (int k = 0; k < G; ++k) {
      v[k][0] = filt_ld<false>(fbase + cur[k].w0.x);
      v[k][1] = filt_ld<false>(fbase + cur[k].w0.y);
      v[k][2] = filt_ld<false>(fbase + cur[k].w0.z);
      v[k][3] = filt_ld<false>(fbase + cur[k].w0.w);
      v[k][4] = filt_ld<false>(fbase + cur[k].w1.x);
      v[k][5] = filt_ld<false>(fbase + cur[k].w1.y);
    }
    // prefetch the next unit (its payload is only used if all its flags were set)
    have = try_unit(next + G);
    // a write after e_pre to one of the items raised all of its slots above
    // e_pre (every earlier unit of the ring included; the batches of one
    // unit are conflict-free by the clients' pre-validation)
    // (32-bit slots here: the committer's chain is the cluster server's bound,
    // and the 16-bit age test costs more than its fewer false positives gain)
    bool commit[G];
    uint32_t cm[G], om[G], base[G];
#pragma unroll
    for (int k = 0; k < G; ++k) {
      const bool chk = (cur[k].chkm >> lane) & 1u;
      const uint32_t lo = max(min(v[k][0], min(v[k][1], v[k][2])), min(v[k][3], min(v[k][4], v[k][5])));
      const bool ovf = chk && lo > cur[k].e_chk;
      commit[k] = chk && !ovf;
      cm[k] = __ballot_sync(FULL, commit[k]);
      om[k] = __ballot_sync(FULL, ovf);
      base[k] = t + 1;
      t += __popc(cm[k]);
    }
    if (srv_pub && t > gseen + dmask) {  // done-ring back-pressure: CTS t may reuse slot t & mask once GTS >= t - 2^20
      for (uint32_t it = 0; t > gseen + dmask;) {
        gseen = __shfl_sync(FULL, ld_relaxed(p.gts), 0);
        if ((++it & 255u) == 0 && __shfl_sync(FULL, (uint32_t)(lane == 0 && watchdog(p, t_begin, 4)), 0)) break;
      }
    }
#pragma unroll
    for (int k = 0; k < G; ++k) {
      if (commit[k]) {  // the unit's last CTS: equal values for shared slots, race-free
        filt_st<false>(fbase + cur[k].w0.x, t);
        filt_st<false>(fbase + cur[k].w0.y, t);
        filt_st<false>(fbase + cur[k].w0.z, t);
        filt_st<false>(fbase + cur[k].w0.w, t);
        filt_st<false>(fbase + cur[k].w1.x, t);
        filt_st<false>(fbase + cur[k].w1.y, t);
      }
    }
    if (lane == 0) {  // respond: round-tagged words, no fence (kernel.cuh Resp); slot release
#pragma unroll
      for (int k = 0; k < G; ++k) {
        if (G == 1 || cur[k].msk != 0) {  // grouped: only the warps that submitted something
          const uint64_t tag = (uint64_t)cur[k].round << 32;
          st_relaxed64x2(&p.resp[cur[k].cw].base, tag | base[k], tag | cm[k]);
          st_relaxed64(&p.resp[cur[k].cw].ovf, tag | om[k]);
        }
      }
      *(volatile uint32_t*)&c.sh->ring_done = next + G;
    }
    if (lane == 0) *(volatile uint32_t*)&c.sh->tail = t;  // the CTS counter (read at exit)
    __syncwarp();  // this unit's filter stores precede the next unit's loads
    const long long t2 = clock64();
    wait += (unsigned long long)(t1 - tw);
    cs += (unsigned long long)(t2 - t1);
  }
  srv_fence<CL>();
  if (lane == 0) *(volatile uint32_t*)&c.sh->tail = t;
  if (lane == 0) {
    atomicAdd(&p.stats->phase[2], wait);
    atomicAdd(&p.stats->phase[3], cs);
    atomicAdd(&p.stats->lock_cycles, cs);
  }
}

// ---------------------------------------------------------------------------
// Generic worker (variable-length read/write sets, the KV workload): one
// batch per critical section, validated against the two-level ATR exactly
// like the bank worker's -- lastw prefetched before the lock (tail e_pre),
// commits after e_pre found in the recent-commit table.
// ---------------------------------------------------------------------------
template <bool CL>
__device__ void server_worker_generic(const KParams& p, const SrvCtx& c, uint64_t t_begin) {
  const uint32_t FULL = 0xFFFFFFFFu;
  const uint32_t lane = threadIdx.x & 31;
  const uint32_t lt = lanemask_lt();
  unsigned long long busy = 0, locked = 0, batches = 0;
  unsigned long long ph[8] = {0, 0, 0, 0, 0, 0, 0, 0};
  // {set clock} u WS requests (client_kv.cuh): ids[0] is the clock of the
  // PUT's set, read and written by every PUT of that set while nothing else
  // writes the set -- it alone decides validation (DESIGN.md readings)
  const bool compact = p.kv_A > kKvFullWays || !(p.debug & CSMV_DBG_KV_ITEMSETS);
  Jitter jit(p, 7);
  for (;;) {
    uint32_t cw;
    const long long tq = clock64();
    if (!claim_request(c, cw)) break;
    const uint64_t t_claim = trace_now(p);
    const long long t0 = clock64();
    fence_cta();  // after the receiver's acquire (see server_receiver)
    const uint32_t sq = ld_relaxed(&p.req_hdr[cw].round);
    const uint32_t s = ld_relaxed(&p.req_hdr[cw].snapshot);
    const uint32_t mask = ld_relaxed(&p.req_hdr[cw].mask);
    const uint32_t cnt_raw = ld_relaxed(p.req_cnt + (size_t)cw * 32 + lane);
    uint32_t ids[kKvMaxId];  // loaded with the header; rows past a lane's count are ignored
#pragma unroll
    for (uint32_t k = 0; k < kKvMaxId; ++k)
      ids[k] = (!compact || k < 4) ? ld_relaxed(p.req_ids + ((size_t)cw * p.maxid + k) * 32 + lane) : 0u;
    const bool mine = (mask >> lane) & 1u;
    const uint32_t cnt = mine ? cnt_raw : 0u;
    const uint32_t nval = compact ? min(cnt, 1u) : cnt;  // ids to validate
    const uint32_t e_pre = *(volatile uint32_t*)&c.sh0->tail;  // lastw covers every CTS <= e_pre
    srv_fence<CL>();
    jit();  // e_pre read, lastw not yet (the window cs_leave's fence covers)
    uint32_t lw[kKvMaxId];
    uint32_t x = s ^ e_pre;
#pragma unroll
    for (uint32_t k = 0; k < kKvMaxId; ++k) {
      lw[k] = (k < nval) ? ld_relaxed(p.lastw + (ids[k] & ~kWriteBit)) : 0u;
      x ^= ids[k] ^ lw[k];
    }
    if (__ballot_sync(FULL, x == 0x12345679u) == FULL) __nanosleep(1);  // payload complete before the lock
    jit();
    const long long tl = clock64();
    // ---- critical section
    const uint32_t ticket = cs_enter<CL>(c);
    const long long t1 = clock64();
    const uint32_t t0c = *(volatile uint32_t*)&c.sh0->tail;
    bool conflict = false, unknown = false;
    // four buckets in flight per step; warp-uniform exit after the longest set
#pragma unroll
    for (uint32_t k0 = 0; k0 < kKvMaxId; k0 += 4) {
      if (!__any_sync(FULL, k0 < nval)) break;
      RtBucket q[4];
#pragma unroll
      for (uint32_t u = 0; u < 4; ++u)
        if (k0 + u < kKvMaxId && k0 + u < nval) q[u] = rt_load<CL>(c, rt_bucket(ids[k0 + u] & ~kWriteBit, p.rt_log2));
#pragma unroll
      for (uint32_t u = 0; u < 4; ++u) {
        if (k0 + u < kKvMaxId && k0 + u < nval) {
          const RtProbe r = rt_eval(q[u], ids[k0 + u] & ~kWriteBit, s, e_pre, lw[k0 + u]);
          conflict |= r.conflict;
          unknown |= r.unknown;
        }
      }
    }
    if (p.debug & CSMV_DBG_NO_VALIDATE) conflict = unknown = false;
    const bool ovf = mine && !conflict && unknown;
    const bool commit = mine && !conflict && !unknown;
    const uint32_t cm = __ballot_sync(FULL, commit);
    const uint32_t om = __ballot_sync(FULL, ovf);
    const uint32_t n = __popc(cm);
    const uint32_t cts = t0c + 1 + __popc(cm & lt);
    const long long tv = clock64();
    if (p.publish == CSMV_PUBLISH_SERVER && n) done_ring_room(p, c, t0c + n, t_begin);
    if (commit) {
#pragma unroll
      for (uint32_t k = 0; k < kKvMaxId; ++k) {
        if (k < cnt && (ids[k] & kWriteBit)) {
          const uint32_t id = ids[k] & ~kWriteBit, b = rt_bucket(id, p.rt_log2);
          st_relaxed(p.lastw + id, cts);  // every written item, so lastw stays exact for any later run
          if (k < nval || !compact) {
            const RtProbe q = rt_probe<CL>(c, b, id, 0u, 0u, 0u);  // the way to (re)use
            rt_record<CL>(c, b, q.way, id, cts);
          }
        }
      }
    }
    const long long tr = clock64();
    cs_leave<CL>(c, ticket, t0c + n);
    const long long t2 = clock64();
    if (lane == 0) {  // round-tagged words, no fence (kernel.cuh Resp)
      trace_served(p, cw, sq, t_claim);
      const uint64_t tag = (uint64_t)sq << 32;
      st_relaxed64(&p.resp[cw].base, tag | (t0c + 1));
      st_relaxed64(&p.resp[cw].commit, tag | cm);
      st_relaxed64(&p.resp[cw].ovf, tag | om);
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
    ph[5] += (unsigned long long)(tv - t1);
    ph[6] += (unsigned long long)(tr - tv);
    ph[7] += (unsigned long long)(t2 - tr);
    ++batches;
  }
  if (lane == 0) {
    for (int i = 0; i < 8; ++i) atomicAdd(&p.stats->phase[i], ph[i]);
    atomicAdd(&p.stats->batches, batches);
    atomicAdd(&p.stats->groups, batches);
    atomicAdd(&p.stats->busy_cycles, busy);
    atomicAdd(&p.stats->lock_cycles, locked);
  }
}

// ---------------------------------------------------------------------------
// KV worker for {set clock} u WS requests (the default, client_kv.cuh):
// validation is decided by clock[t] alone (DESIGN.md readings), so each PUT
// validates one item -- exactly against lastw (every CTS <= e_pre, before
// the lock) and against the recent-write filter for the commits after e_pre
// (as the bank worker).  Only clocks enter the filter: nothing else is ever
// validated in this mode; lastw is written for all four written items.
// ---------------------------------------------------------------------------
template <int NS, bool CL, bool SELF = false>
__device__ void server_worker_kv_filter(const KParams& p, const SrvCtx& c, uint64_t t_begin) {
  const uint32_t FULL = 0xFFFFFFFFu;
  const uint32_t lane = threadIdx.x & 31;
  const uint32_t lt = lanemask_lt();
  const bool novalid = (p.debug & CSMV_DBG_NO_VALIDATE) != 0;
  const uint32_t fl2 = p.rt_log2 + 3;
  unsigned long long busy = 0, locked = 0, batches = 0;
  unsigned long long ph[8] = {0, 0, 0, 0, 0, 0, 0, 0};
  Jitter jit(p, 8);
  uint32_t my_lo = 0, my_hi = 0;  // SELF: this worker's slice of the doorbells
  if constexpr (SELF) {
    const uint32_t w = threadIdx.x >> 5, per = (c.cw_hi - c.cw_lo + p.n_workers - 1) / p.n_workers;
    my_lo = min(c.cw_lo + w * per, c.cw_hi);
    my_hi = min(my_lo + per, c.cw_hi);
  }
  for (;;) {
    uint32_t cw, rq = 0;
    const long long tq = clock64();
    if constexpr (SELF) {  // sweep own slice; the claim's acquire fence orders the payload loads
      uint32_t one[1], r1[1], g;
      if (!self_claim<1>(p, c, my_lo, my_hi, 1, one, r1, t_begin, g)) break;
      cw = one[0];
      rq = r1[0];
    } else {
      if (!claim_request(c, cw, &rq)) break;
      fence_cta();  // after the receiver's acquire (see server_receiver)
    }
    const uint64_t t_claim = trace_now(p);
    const long long t0 = clock64();
    uint32_t sq, s, mask, ids[4];
    // server write-back: the PUT's key, value, new LRU / clock value and
    // replacement slots, loaded with the payload (+ the check word when tagged)
    uint32_t wb[kSwbRows];
    // tagged requests: loaded again until every word carries the round of
    // the doorbell (the client did not fence the payload before it)
    for (uint32_t pass = 0;; ++pass) {
      const uint64_t* hw = reinterpret_cast<const uint64_t*>(&p.req_hdr[cw]);
      const uint64_t w0 = ld_relaxed64(hw), w1 = ld_relaxed64(hw + 1);
      s = (uint32_t)w0;
      sq = (uint32_t)(w0 >> 32);
      mask = (uint32_t)w1;
#pragma unroll
      for (int k = 0; k < 4; ++k) ids[k] = ld_relaxed(p.req_ids + ((size_t)cw * p.maxid + k) * 32 + lane);
      uint32_t wck = 0;
      if (p.kv_swb) {
#pragma unroll
        for (int k = 0; k < (int)kSwbRows; ++k)
          wb[k] = ld_relaxed(p.req_ids + ((size_t)cw * p.maxid + kSwbRow + k) * 32 + lane);
        if (p.req_tagged) wck = ld_relaxed(p.req_ids + ((size_t)cw * p.maxid + kSwbRow + kSwbRows) * 32 + lane);
      }
      if (!p.req_tagged) {
#pragma unroll
        for (int k = 0; k < 4; ++k) ids[k] &= ~kWriteBit;
        break;
      }
      const uint32_t tg = id_tag(rq), tm = kIdTagMask << kIdItemBits;
      bool stale = (sq & 0xFFFFu) != rq || (uint32_t)(w1 >> 32) != sq;
      if ((mask >> lane) & 1u) {
#pragma unroll
        for (int k = 0; k < 4; ++k) stale |= (ids[k] & tm) != tg;
        if (p.kv_swb) stale |= swb_check(sq, wb, 1) != wck;  // the write-back words of this round
      }
#pragma unroll
      for (int k = 0; k < 4; ++k) ids[k] &= kIdItemMask;
      if (!__any_sync(FULL, stale)) break;
      if ((pass & 1023u) == 1023u) {  // a lost payload would be a protocol error: let the watchdog see it
        uint32_t bad = 0;
        if (lane == 0) bad = ld_relaxed(&p.ctl->error) || watchdog(p, t_begin, 5);
        if (__shfl_sync(FULL, bad, 0)) break;
      }
    }
    const bool mine = (mask >> lane) & 1u;
    const uint32_t e_pre = *(volatile uint32_t*)&c.sh0->tail;  // lastw covers every CTS <= e_pre
    srv_fence<CL>();
    jit();  // e_pre read, lastw not yet (the window cs_leave's fence covers)
    const uint32_t lw = mine ? ld_relaxed(p.lastw + ids[0]) : 0u;
    const bool chk = mine && (novalid || lw <= s);
    uint32_t fa[kFiltK];
#pragma unroll
    for (int k = 0; k < kFiltK; ++k) fa[k] = filt_addr<CL>(c, filt_slot(ids[0], k, fl2));
    const uint32_t e_chk = novalid ? 0xFFFFFFFFu : e_pre;
    if (__ballot_sync(FULL, (s ^ lw ^ ids[1] ^ ids[2] ^ ids[3]) == 0x12345679u) == FULL) __nanosleep(1);
    jit();
    const long long tl = clock64();
    // ---- critical section
    const uint32_t ticket = cs_enter<CL>(c);
    const long long t1 = clock64();
    const uint32_t t0c = *(volatile uint32_t*)&c.sh0->tail;
    uint32_t v[kFiltK] = {0u, 0u, 0u};
    if (chk) {
#pragma unroll
      for (int k = 0; k < kFiltK; ++k) v[k] = filt_ld<CL>(fa[k]);
    }
    const bool ovf = chk && min(v[0], min(v[1], v[2])) > e_chk;
    const bool commit = chk && !ovf;
    const uint32_t cm = __ballot_sync(FULL, commit);
    const uint32_t om = __ballot_sync(FULL, ovf);
    const uint32_t n = __popc(cm);
    const long long tv = clock64();
    if (p.publish == CSMV_PUBLISH_SERVER && n) done_ring_room(p, c, t0c + n, t_begin);
    if (commit) {
      const uint32_t cts = t0c + 1 + __popc(cm & lt);
#pragma unroll
      for (int k = 0; k < kFiltK; ++k) filt_st<CL>(fa[k], t0c + n);  // the batch's last CTS
#pragma unroll
      for (int k = 0; k < 4; ++k) st_relaxed(p.lastw + ids[k], cts);
    }
    const long long tr = clock64();
    cs_leave<CL>(c, ticket, t0c + n);
    const long long t2 = clock64();
    if (p.kv_swb && n) {
      // Server write-back (csmv_workload.server_writeback): the four
      // versions of each committed PUT, then GTS advanced in CTS order
      // -- by this worker once GTS reaches its first CTS - 1, or through the
      // done flags and the publisher.  No lock is held: a later range's
      // worker waits for this one's publish, never the other way round.
      jit();
      if (commit) {
        const uint32_t cts = t0c + 1 + __popc(cm & lt);
        const uint32_t S = p.kv_S, victim = ids[1], tset = ids[0] - 3 * S;
        const int iv = (int)(wb[13] & 0xFFu), ic = (int)((wb[13] >> 8) & 0xFFu);
        const uint32_t kk[4] = {wb[0], wb[1], wb[2], wb[3]};
        const uint32_t vv[8] = {wb[4], wb[5], wb[6], wb[7], wb[8], wb[9], wb[10], wb[11]};
        const uint32_t cn1[1] = {wb[12]};
        kv_install_at<4>(p.kv_key + (size_t)victim * NS * 4, iv, cts, kk);
        kv_install_at<8>(p.kv_val + (size_t)victim * NS * 8, iv, cts, vv);
        kv_install_at<1>(p.kv_lru + (size_t)victim * NS, iv, cts, cn1);
        kv_install_at<1>(p.kv_clk + (size_t)tset * NS, ic, cts, cn1);
        if (p.publish == CSMV_PUBLISH_SERVER) st_release(p.done_ring + (cts & ((1u << kDoneLog2) - 1)), cts);
      }
      if (p.publish == CSMV_PUBLISH_CLIENT) {
        __syncwarp();
        fence_gpu();
        if (lane == 0) {
          uint32_t it = 0;
          while (ld_relaxed(p.gts) != t0c) {
            if ((++it & 255u) == 0 && (ld_relaxed(&p.ctl->error) || watchdog(p, t_begin, 6))) break;
            __nanosleep(32);
          }
          st_release(p.gts, t0c + n);
        }
      }
      __syncwarp();
    }
    if (lane == 0) {  // round-tagged words, no fence (kernel.cuh Resp)
      trace_served(p, cw, sq, t_claim);
      const uint64_t tag = (uint64_t)sq << 32;
      st_relaxed64(&p.resp[cw].base, tag | (t0c + 1));
      st_relaxed64(&p.resp[cw].commit, tag | cm);
      st_relaxed64(&p.resp[cw].ovf, tag | om);
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
    ph[5] += (unsigned long long)(tv - t1);
    ph[6] += (unsigned long long)(tr - tv);
    ph[7] += (unsigned long long)(t2 - tr);
    ++batches;
  }
  if (lane == 0) {
    for (int i = 0; i < 8; ++i) atomicAdd(&p.stats->phase[i], ph[i]);
    atomicAdd(&p.stats->batches, batches);
    atomicAdd(&p.stats->groups, batches);
    atomicAdd(&p.stats->busy_cycles, busy);
    atomicAdd(&p.stats->lock_cycles, locked);
  }
}

// ---------------------------------------------------------------------------
// CSMV-onlyCS worker: the client-server design with the paper's
// complementary mechanisms removed -- no collaborative validation (the lane
// of the transaction scans the list ATR alone), no batched ATR insert
// (each transaction is validated and, if it commits, inserted before the
// next one is looked at; this also catches the intra-batch conflicts the
// missing client pre-validation would have caught), and server-side
// write-back of the new versions (instead of the client's).  Bank,
// single-CTA server; the ATR is the CTS-indexed ring of CSMV_ATR_LIST.
// ---------------------------------------------------------------------------
template <int NS>
__device__ void server_worker_onlycs(const KParams& p, const SrvCtx& c, uint64_t t_begin) {
  const uint32_t FULL = 0xFFFFFFFFu;
  const uint32_t lane = threadIdx.x & 31;
  const uint32_t lt = lanemask_lt();
  const uint32_t R = (uint32_t)kRtWays << p.rt_log2;
  const uint32_t dmask = (1u << kDoneLog2) - 1;
  unsigned long long busy = 0, locked = 0, batches = 0;
  Jitter jit(p, 9);
  for (;;) {
    uint32_t cw;
    if (!claim_request(c, cw)) break;
    const long long t0 = clock64();
    fence_cta();  // after the receiver's acquire (see server_receiver)
    const uint32_t sq = ld_relaxed(&p.req_hdr[cw].round);
    const uint32_t s = ld_relaxed(&p.req_hdr[cw].snapshot);
    const uint32_t mask = ld_relaxed(&p.req_hdr[cw].mask);
    const bool mine = (mask >> lane) & 1u;
    uint32_t a = 0, b = 0, na = 0, nb = 0;
    if (mine) {
      a = ld_relaxed(p.req_ids + (size_t)cw * 64 + lane) & ~kWriteBit;
      b = ld_relaxed(p.req_ids + (size_t)cw * 64 + 32 + lane) & ~kWriteBit;
      na = ld_relaxed(p.req_vals + (size_t)cw * 128 + lane);
      nb = ld_relaxed(p.req_vals + (size_t)cw * 128 + 32 + lane);
    }
    if (__ballot_sync(FULL, (a ^ b ^ na ^ nb ^ s) == 0x12345679u) == FULL) __nanosleep(1);
    jit();
    const uint32_t ticket = cs_enter<false>(c);
    const long long t1 = clock64();
    const uint32_t base = *(volatile uint32_t*)&c.sh0->tail + 1;
    uint32_t t = base - 1, cm = 0, om = 0, rem = mask;
    while (rem) {  // one transaction at a time, in lane order
      const int i = __ffs(rem) - 1;
      rem &= rem - 1;
      uint32_t ok = 0, ovf = 0;
      if (lane == (uint32_t)i) {
        ovf = (t - s >= R) ? 1u : 0u;
        ok = ovf ? 0u : 1u;
        if (!(p.debug & CSMV_DBG_NO_VALIDATE)) {
          for (uint32_t q = s + 1; ok && q - 1 < t; ++q) {  // every commit after s
            const uint64_t e = c.rt[q & (R - 1)];
            const uint32_t w0 = (uint32_t)e, w1 = (uint32_t)(e >> 32);
            if (w0 == a || w0 == b || w1 == a || w1 == b) ok = 0;
          }
        }
        if (ok) c.rt[(t + 1) & (R - 1)] = ((uint64_t)b << 32) | a;  // insert this write-set alone
      }
      ok = __shfl_sync(FULL, ok, i);
      ovf = __shfl_sync(FULL, ovf, i);
      if (ok) {
        cm |= 1u << i;
        ++t;
      } else if (ovf) {
        om |= 1u << i;
      }
      __syncwarp();
    }
    if (p.publish == CSMV_PUBLISH_SERVER && t + 1 != base) done_ring_room(p, c, t, t_begin);
    cs_leave<false>(c, ticket, t);
    const long long t2 = clock64();
    // server-side write-back; every earlier writer of a and b has published
    // (the snapshot s covers it), so the ring read here is current
    if ((cm >> lane) & 1u) {
      const uint32_t cts = base + __popc(cm & lt);
      const Ring<NS> ra = ld_ring<NS>(p.rings + (size_t)a * NS), rb = ld_ring<NS>(p.rings + (size_t)b * NS);
      write_back<NS>(p.rings + (size_t)a * NS, ra, p.K, cts, na);
      write_back<NS>(p.rings + (size_t)b * NS, rb, p.K, cts, nb);
      if (p.publish == CSMV_PUBLISH_SERVER) st_release(p.done_ring + (cts & dmask), cts);
    }
    __syncwarp();
    fence_gpu();  // the write-backs precede the response (the client publishes GTS after it)
    if (lane == 0) {  // round-tagged words after the fence above
      const uint64_t tag = (uint64_t)sq << 32;
      st_relaxed64(&p.resp[cw].base, tag | base);
      st_relaxed64(&p.resp[cw].commit, tag | cm);
      st_relaxed64(&p.resp[cw].ovf, tag | om);
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

// ---------------------------------------------------------------------------
// CSMV_PUBLISH_SERVER: advance GTS over the prefix of CTS whose write-backs
// are done.  Same invariant as P:116 (GTS = c only once every commit <= c
// has written back), without a client-side serial chain.  CTA 0 only.
// ---------------------------------------------------------------------------
// With pub_remote it runs on an idle warp of the first client CTA instead
// (c == nullptr): its done-flag sweeps then use another SM's load pipe and
// issue slots than the critical section's, and it stops once the server has
// finished (ctl->srv_done, release) and GTS reached the final tail.
static __device__ void server_publisher(const KParams& p, const SrvCtx* c, uint64_t t_begin, uint32_t g0) {
  const uint32_t FULL = 0xFFFFFFFFu;
  const uint32_t lane = threadIdx.x & 31;
  const uint32_t dmask = (1u << kDoneLog2) - 1;
  uint32_t g = g0;
  uint32_t spins = 0;
  Jitter jit(p, 10);
  // one sweep looks at the next 32 * 4 * W flags: W 16-byte loads per lane in
  // flight, lane l of row k covering CTS g+1 + 4(32k + l) .. +3 (a sweep is
  // one L2 round trip, so this bounds GTS's advance rate)
  constexpr int W = 8;
  for (;;) {
    jit();
    const uint32_t g0 = g + 1;
    const uint32_t a0 = g0 & 3u;  // 16-byte loads need a 4-aligned first CTS: start at g0 - a0
    uint4 v[W];
#pragma unroll
    for (int k = 0; k < W; ++k)
      v[k] = ld_relaxed_v4(p.done_ring + ((g0 - a0 + 4u * (k * 32 + lane)) & dmask));
    uint32_t adv = 0;
    bool open = true;
#pragma unroll
    for (int k = 0; k < W; ++k) {
      const uint32_t e0 = g0 - a0 + 4u * (k * 32 + lane);
      const uint32_t w[4] = {v[k].x, v[k].y, v[k].z, v[k].w};
      int first_bad = 4;
#pragma unroll
      for (int i = 3; i >= 0; --i)
        if (w[i] != e0 + i && e0 + i >= g0) first_bad = i;  // flags before g0 are not looked at
      const uint32_t bad = __ballot_sync(FULL, first_bad < 4);
      if (open) {
        if (bad) {
          const int l = __ffs(bad) - 1;
          const uint32_t fb = __shfl_sync(FULL, (uint32_t)first_bad, l);
          adv = 4u * (k * 32 + l) + fb - a0;
          open = false;
        } else {
          adv = 4u * (k * 32 + 32) - a0;
        }
      }
    }
    if (adv) {
      fence_gpu();
      g += adv;
      if (lane == 0) st_release(p.gts, g);
      continue;
    }
    if (CSMV_SLEEP_PUBLISHER) __nanosleep(CSMV_SLEEP_PUBLISHER);
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
      if (c) {
        if (dw >= p.n_cw && g == *(volatile uint32_t*)&c->sh->tail) break;
      } else {
        uint32_t fin = 0;
        if (lane == 0 && dw >= p.n_cw) {
          if (p.part_log2) fin = g == ld_relaxed(&p.ctl->cts_next);  // every CTS is handed out by then
          else if (ld_acquire(&p.ctl->srv_done)) fin = g == ld_relaxed(&p.ctl->tail_final);
        }
        if (__shfl_sync(FULL, fin, 0)) break;
      }
    }
  }
}

// Shared-memory layout of one server CTA (every CTA of the fused grid gets
// the same dynamic allocation): rt stripe, evmax stripe, dispatch queue,
// last-seen doorbells of its slice, control block.
template <int NS, int KIND, bool CL>
__device__ void server_cta(const KParams& p, uint8_t* smem, uint64_t t_begin) {
  const uint32_t C = p.n_server_ctas;
  const uint32_t rank = CL ? cg::this_cluster().block_rank() : 0u;
  const uint32_t local_log2 = p.rt_log2 - p.clog2;
  // cluster + commit ring: CTA 0 is left to the committer (and publisher);
  // the client doorbells are sliced over CTAs 1..C-1
  const bool ring_cl = CL && server_uses_ring(p);
  const uint32_t nserve = ring_cl ? C - 1 : C, srank = ring_cl ? rank - 1 : rank;
  const uint32_t per = (p.n_cw + nserve - 1) / nserve;
  SrvCtx c;
  c.clog2 = p.clog2;
  c.cw_lo = (ring_cl && rank == 0) ? p.n_cw : min(srank * per, p.n_cw);
  c.cw_hi = min(c.cw_lo + per, p.n_cw);
  c.qn_log2 = queue_log2(per);
  c.rt = reinterpret_cast<uint64_t*>(smem);
  c.rt32 = (uint32_t)__cvta_generic_to_shared(c.rt);
  const uint32_t rt_words = rt_region_words(local_log2, p.filt16_n);
  c.queue = c.rt + rt_words;
  c.evmax = reinterpret_cast<uint32_t*>(c.queue + (1u << c.qn_log2));
  c.last_seen = c.evmax + (1u << p.ev_log2);
  const uint32_t ls_words = (per + 31) / 32 * 32;
  c.sh = reinterpret_cast<SrvShared*>(c.last_seen + ls_words);
  CmSlot* ring = reinterpret_cast<CmSlot*>(reinterpret_cast<uint8_t*>(c.sh) + sizeof(SrvShared));
  c.ring32 = (uint32_t)__cvta_generic_to_shared(ring);
  if constexpr (CL) {
    c.sh0 = cg::this_cluster().map_shared_rank(c.sh, 0);
    asm("mapa.shared::cluster.u32 %0, %1, 0;" : "=r"(c.ring32) : "r"(c.ring32));
  } else {
    c.sh0 = c.sh;
  }
  // bank + filter: the commit ring and one committer warp (unless the A/B flag asks for the lock)
  const bool cmring = server_uses_ring(p);
  const bool filt = KIND == CSMV_KIND_BANK ? p.atr_mode == CSMV_ATR_HASH : kv_filter_mode(p);
  const uint64_t rt_init = filt ? 0ull : 0xFFFFFFFFull;
  for (uint32_t i = threadIdx.x; i < rt_words; i += blockDim.x) c.rt[i] = rt_init;  // table: cts 0, no item; filter: 0
  for (uint32_t i = threadIdx.x; i < (1u << p.ev_log2); i += blockDim.x) c.evmax[i] = 0;
  for (uint32_t i = threadIdx.x; i < (1u << c.qn_log2); i += blockDim.x) c.queue[i] = 0;
  for (uint32_t i = threadIdx.x; i < ls_words; i += blockDim.x) c.last_seen[i] = 0;
  for (uint32_t i = threadIdx.x; i < (1u << p.cm_ring_log2); i += blockDim.x) ring[i].flag = 0;
  if (threadIdx.x == 0) {
    const uint32_t g0 = *p.gts;
    c.sh->tail = g0;
    c.sh->next_ticket = 0;
    c.sh->now_serving = 0;
    c.sh->gts_seen = g0;
    c.sh->q_head = 0;
    c.sh->exit = 0;
    c.sh->ring_head = 0;
    c.sh->ring_done = 0;
    c.sh->workers_left = p.n_workers * nserve;
  }
  if constexpr (CL) cg::this_cluster().sync();
  else __syncthreads();
  const uint32_t warp = threadIdx.x >> 5;
  const bool serving = !(ring_cl && rank == 0);
  if (!CL && server_self_recv(p)) {
    // warps 0..n_workers-1 self-receiving workers, then the publisher
    if (warp < p.n_workers) {
      if constexpr (KIND == CSMV_KIND_KV) server_worker_kv_filter<NS, CL, !CL>(p, c, t_begin);
      else server_worker<CL, !CL>(p, c, t_begin);
    } else if (warp == p.n_workers && p.publish == CSMV_PUBLISH_SERVER && !p.pub_remote) {
      server_publisher(p, &c, t_begin, c.sh->tail);
    }
  } else if (!serving && warp <= p.n_workers) {
    // CTA 0 of a ring cluster: no receiver, no workers
  } else if (warp == 0) {
    server_receiver(p, c, t_begin);
  } else if (warp <= p.n_workers) {
    if constexpr (KIND == CSMV_KIND_KV) {
      if (kv_filter_mode(p)) server_worker_kv_filter<NS, CL>(p, c, t_begin);
      else server_worker_generic<CL>(p, c, t_begin);
    }
    else if (!CL && p.commit == CSMV_COMMIT_ONLYCS) server_worker_onlycs<NS>(p, c, t_begin);
    else if (cmring && p.group == 2) server_worker_cm<CL, 2>(p, c, t_begin);
    else if (cmring && p.group == 4) server_worker_cm<CL, 4>(p, c, t_begin);
    else if (cmring) server_worker_cm<CL>(p, c, t_begin);
    else if (!CL && p.group == 2) server_worker<CL, false, 2>(p, c, t_begin);
    else if (!CL && p.group == 4) server_worker<CL, false, 4>(p, c, t_begin);
    else if (!CL && p.group == 8) server_worker<CL, false, 8>(p, c, t_begin);
    else server_worker<CL, false>(p, c, t_begin);
  } else if (warp == p.n_workers + 1 && rank == 0 && p.publish == CSMV_PUBLISH_SERVER && !p.pub_remote) {
    server_publisher(p, &c, t_begin, c.sh->tail);
  } else if (warp == kWarps - 1 && rank == 0 && cmring) {
    if (p.group == 2) server_committer<CL, 2>(p, c, ring, t_begin);
    else if (p.group == 4) server_committer<CL, 4>(p, c, ring, t_begin);
    else server_committer<CL>(p, c, ring, t_begin);
  }
  if constexpr (CL) cg::this_cluster().sync();
  else __syncthreads();
  if (rank == 0 && threadIdx.x == 0) {
    p.ctl->tail_final = c.sh->tail;
    st_release(&p.ctl->srv_done, 1u);  // the remote publisher may stop once GTS reaches tail_final
  }
}

}  // namespace csmvd
