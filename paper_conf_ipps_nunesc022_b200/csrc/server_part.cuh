// server_part.cuh -- item-partitioned commit over S independent server CTAs
// (CSMV_SERVER_PART; NEXT-3, the paper's first future-work item).
//
// Server k owns the items x with part_owner(x) == k and keeps, in its own
// shared memory, the part of the ATR for them: a 32-bit recent-write filter
// (slot = largest CTS of a decided write hashing there, two hashes) and the
// set of items with a pending prepare (exact item ids in 4-way buckets: a
// hashed counter table saturates -- ~10^4 prepared items are in flight).  One CTS sequence stays global (a counter
// in Ctl).  A client warp's batch goes through three messages
// (checked by exhaustive interleavings in
// the two-server model checker under tests/ before this code):
//   1 PREPARE at every server owning an item of the batch: for each lane
//     with an item here, validate that part -- lastw[x] <= s for the commits
//     up to e_pre = GTS, no filter slot set after e_pre (else OVERFLOW), no
//     pending prepare of another transaction on it (else CONFLICT) -- and if
//     clean mark its items pending; vote (lanes with nothing here vote yes);
//   2 the client ANDs the votes and takes CTS = ++counter for the survivors
//     (one L2 atomic per batch);
//   3 DECIDE at every prepared server: record the committed write-sets in the
//     filter (atomicMax: decides may arrive out of CTS order) and clear the
//     pending marks of every lane this server marked; acknowledge.
// Two conflicting transactions share an item, hence its server, whose
// pending marks keep them from being prepared at the same time; the later
// one prepares after the earlier decided -- so it either sees the earlier
// record (or lastw) and aborts, or its snapshot covers it -- and takes its
// CTS after the earlier one took its own.  Write-back, lastw and the GTS
// publish (done flags, server publisher) are as in the other servers.
//
// Each server CTA runs self-receiving worker warps (a slice of the client
// warps each, decides first), a ticket lock (cs_enter / cs_leave) around the
// filter and the pending counters, and server 0 the publisher (unless it
// runs on a client CTA).  Included by fused.cuh after server.cuh.
#pragma once

namespace csmvd {

__device__ __forceinline__ uint32_t part_filt_slot(uint32_t x, int k) {
  const uint32_t C[2] = {0x9E3779B1u, 0x85EBCA77u};
  return (x * C[k]) >> (32 - kPartFiltLog2);
}
__device__ __forceinline__ uint32_t part_pend_bucket(uint32_t x) {
  return (x * 0xC2B2AE3Du) >> (32 - (kPartPendLog2 - 2));
}
constexpr uint32_t kPendEmpty = 0xFFFFFFFFu;

struct PartCtx {
  uint32_t* filt;       // [2^kPartFiltLog2]
  uint32_t* pend;       // [2^kPartPendLog2] item ids with a pending prepare, 4-way buckets (kPendEmpty = free)
  uint32_t* seen_req;   // [n_cw] last prepare doorbell seen
  uint32_t* seen_dec;   // [n_cw] last decide doorbell seen
  uint32_t* marked;     // [n_cw] lanes this server marked pending at the client warp's last prepare
  SrvShared* sh;
  uint32_t k;           // this server
};

// pending set (under the server's lock; lanes of one batch never mark one item twice)
__device__ __forceinline__ bool pend_has(const uint32_t* pend, uint32_t x, bool& full) {
  const volatile uint32_t* b = pend + 4 * part_pend_bucket(x);
  const uint32_t q0 = b[0], q1 = b[1], q2 = b[2], q3 = b[3];
  full = q0 != kPendEmpty && q1 != kPendEmpty && q2 != kPendEmpty && q3 != kPendEmpty;
  return q0 == x || q1 == x || q2 == x || q3 == x;
}
__device__ __forceinline__ bool pend_insert(uint32_t* pend, uint32_t x) {
  uint32_t* b = pend + 4 * part_pend_bucket(x);
#pragma unroll
  for (int i = 0; i < 4; ++i)
    if (atomicCAS(b + i, kPendEmpty, x) == kPendEmpty) return true;
  return false;  // bucket full (other lanes of this batch took the last slots)
}
__device__ __forceinline__ void pend_erase(uint32_t* pend, uint32_t x) {
  volatile uint32_t* b = pend + 4 * part_pend_bucket(x);
#pragma unroll
  for (int i = 0; i < 4; ++i)
    if (b[i] == x) b[i] = kPendEmpty;
}

static __device__ void part_worker(const KParams& p, const PartCtx& c, uint64_t t_begin) {
  const uint32_t FULL = 0xFFFFFFFFu;
  const uint32_t lane = threadIdx.x & 31;
  const uint32_t warp = threadIdx.x >> 5;
  const uint32_t S = 1u << p.part_log2;
  const size_t off = (size_t)c.k * p.mstride;
  const uint32_t per = (p.n_cw + p.n_workers - 1) / p.n_workers;
  const uint32_t lo = min(warp * per, p.n_cw), hi = min(lo + per, p.n_cw), n = hi - lo, rows = (n + 31) / 32;
  const bool novalid = (p.debug & CSMV_DBG_NO_VALIDATE) != 0;
  unsigned long long batches = 0, decides = 0, locked = 0;
  Jitter jit(p, 11);
  uint32_t rr = 0, rl = 31;  // round robin: next row to look at, last lane served
  (void)S;
  for (uint32_t idle = 1;; ++idle) {
    // ---- sweep, round robin over rows and lanes (a fixed scan order starves
    // the last rows' clients -- and their decides, whose marks then block
    // everyone); in the chosen row a pending decide first (it unblocks others)
    uint32_t cw = 0xFFFFFFFFu, seq = 0;
    bool dec = false;
    for (uint32_t q = 0; q < rows && cw == 0xFFFFFFFFu; ++q) {
      const uint32_t r = (rr + q) % rows;
      const uint32_t i = lo + r * 32 + lane;
      const uint32_t sd = i < hi ? ld_relaxed(p.mdec_seq + off + i) : 0u;
      const uint32_t sr = i < hi ? ld_relaxed(p.mreq_seq + off + i) : 0u;
      const uint32_t pd = __ballot_sync(FULL, i < hi && sd != c.seen_dec[i]);
      const uint32_t pr = __ballot_sync(FULL, i < hi && sr != c.seen_req[i]);
      if (pd | pr) {
        dec = pd != 0;
        const uint32_t m = dec ? pd : pr;
        const uint32_t after = m & ~(0xFFFFFFFFu >> (31 - rl));  // lanes past the last one served
        const uint32_t l = __ffs(after ? after : m) - 1;
        seq = __shfl_sync(FULL, dec ? sd : sr, l);
        cw = lo + r * 32 + l;
        if (lane == l) (dec ? c.seen_dec : c.seen_req)[cw] = seq;
        rr = r + 1;
        rl = l;
      }
    }
    if (cw == 0xFFFFFFFFu) {
      if ((idle & 15u) == 0) {
        uint32_t fin = 0;
        if (lane == 0) {
          const uint32_t er = ld_relaxed(&p.ctl->error);
          fin = er || ld_acquire(&p.ctl->done_warps) >= p.n_cw || watchdog(p, t_begin, 12);
        }
        if (__shfl_sync(FULL, fin, 0)) break;
      }
      continue;
    }
    idle = 0;
    fence_gpu();  // acquire: the payload of the doorbell just seen precedes our loads of it
    jit();
    const uint32_t s = ld_relaxed(&p.req_hdr[cw].snapshot);
    const uint32_t msk = ld_relaxed(&p.req_hdr[cw].mask);
    const uint32_t a = ld_relaxed(p.req_ids + (size_t)cw * 64 + lane) & ~kWriteBit;
    const uint32_t b = ld_relaxed(p.req_ids + (size_t)cw * 64 + 32 + lane) & ~kWriteBit;
    const bool mine = (msk >> lane) & 1u;
    const bool oa = mine && part_owner(a, p.part_log2) == c.k, ob = mine && part_owner(b, p.part_log2) == c.k;
    if (dec) {
      // ---- DECIDE: record the committed write-sets, clear our marks, acknowledge
      const uint64_t w0 = ld_relaxed64(p.mdec + 2 * (size_t)cw), w1 = ld_relaxed64(p.mdec + 2 * (size_t)cw + 1);
      if ((uint32_t)(w0 >> 32) != seq || (uint32_t)(w1 >> 32) != seq) {  // the client overwrote it: protocol error
        if (lane == 0) atomicCAS(&p.ctl->error, 0u, 2u);
        break;
      }
      const uint32_t base = (uint32_t)w0, cm = (uint32_t)w1;
      // ownership from the ids alone: the mask may have shrunk since our
      // prepare (the client prepares later servers with the survivors only)
      const bool xa = part_owner(a, p.part_log2) == c.k, xb = part_owner(b, p.part_log2) == c.k;
      const uint32_t ticket = cs_enter<false>(SrvCtx{nullptr, 0, nullptr, 0, c.sh, c.sh});
      const long long t1 = clock64();
      const bool marked = (c.marked[cw] >> lane) & 1u;
      if (marked) {
        if (xa) pend_erase(c.pend, a);
        if (xb) pend_erase(c.pend, b);
      }
      if ((cm >> lane) & 1u) {  // committed lanes were marked at every owner of their items
        const uint32_t cts = base + __popc(cm & lanemask_lt());
#pragma unroll
        for (int k = 0; k < 2; ++k) {
          if (xa) atomicMax(c.filt + part_filt_slot(a, k), cts);
          if (xb) atomicMax(c.filt + part_filt_slot(b, k), cts);
        }
      }
      cs_leave<false>(SrvCtx{nullptr, 0, nullptr, 0, c.sh, c.sh}, ticket, 0u);
      locked += (unsigned long long)(clock64() - t1);
      __syncwarp();
      if (lane == 0) st_release(p.mdack + off + cw, seq);  // our payload loads precede the acknowledgement
      ++decides;
      continue;
    }
    // ---- PREPARE: validate our part of each lane, mark it pending, vote
    const uint32_t e_pre = ld_acquire(p.gts);  // lastw covers every CTS <= GTS (client write-back)
    const uint32_t la = oa ? ld_relaxed(p.lastw + a) : 0u, lb = ob ? ld_relaxed(p.lastw + b) : 0u;
    const bool here = oa || ob;
    const bool chk = here && (novalid || (la <= s && lb <= s));
    if (__ballot_sync(FULL, (la ^ lb ^ e_pre) == 0x12345679u) == FULL) __nanosleep(1);  // loads complete here
    const uint32_t ticket = cs_enter<false>(SrvCtx{nullptr, 0, nullptr, 0, c.sh, c.sh});
    const long long t1 = clock64();
    bool ovf = false, conf = false;
    if (chk && !novalid) {
#pragma unroll
      for (int x = 0; x < 2; ++x) {
        const bool o = x ? ob : oa;
        const uint32_t it = x ? b : a;
        if (o) {
          const uint32_t v = min(c.filt[part_filt_slot(it, 0)], c.filt[part_filt_slot(it, 1)]);
          ovf = ovf || v > e_pre;  // a decided write after e_pre may have hit it
          bool full = false;
          conf = conf || pend_has(c.pend, it, full) || full;  // another transaction is in flight on it
        }
      }
    }
    bool ok = chk && !ovf && !conf;
    __syncwarp();  // every lane's lookups precede any insertion
    if (ok) {  // mark; a lane that finds its bucket full after all takes its marks back and votes no
      const bool ia = !oa || pend_insert(c.pend, a);
      const bool ib = !ob || pend_insert(c.pend, b);
      if (!(ia && ib)) {
        if (oa && ia) pend_erase(c.pend, a);
        if (ob && ib) pend_erase(c.pend, b);
        ok = false;
        conf = true;
      }
    }
    const uint32_t okm = __ballot_sync(FULL, ok);
    const uint32_t om = __ballot_sync(FULL, chk && ovf && !conf && !ok);  // labelled OVERFLOW, the rest CONFLICT
    if (lane == 0) c.marked[cw] = okm;
    cs_leave<false>(SrvCtx{nullptr, 0, nullptr, 0, c.sh, c.sh}, ticket, 0u);
    locked += (unsigned long long)(clock64() - t1);
    // vote: lanes with nothing here vote yes
    const uint32_t herem = __ballot_sync(FULL, here);
    const uint32_t vote = okm | (msk & ~herem);
    if (lane == 0) {
      const uint64_t tag = (uint64_t)seq << 32;
      Resp* r = p.mresp + off + cw;
      st_relaxed64(&r->commit, tag | om);
      st_relaxed64(&r->ovf, tag);
      st_relaxed64(&r->base, tag | vote);
    }
    __syncwarp();
    ++batches;
  }
  if (lane == 0) {
    atomicAdd(&p.stats->batches, batches);
    atomicAdd(&p.stats->groups, batches + decides);
    atomicAdd(&p.stats->lock_cycles, locked);
  }
}

template <int NS>
__device__ void server_part_cta(const KParams& p, uint8_t* smem, uint64_t t_begin) {
  PartCtx c;
  c.k = blockIdx.x;
  c.filt = reinterpret_cast<uint32_t*>(smem);
  c.pend = c.filt + (1u << kPartFiltLog2);
  c.seen_req = c.pend + (1u << kPartPendLog2);
  const uint32_t nw = (p.n_cw + 31) / 32 * 32;
  c.seen_dec = c.seen_req + nw;
  c.marked = c.seen_dec + nw;
  c.sh = reinterpret_cast<SrvShared*>(c.marked + nw);
  for (uint32_t i = threadIdx.x; i < (1u << kPartFiltLog2); i += blockDim.x) c.filt[i] = 0;
  for (uint32_t i = threadIdx.x; i < (1u << kPartPendLog2); i += blockDim.x) c.pend[i] = kPendEmpty;
  for (uint32_t i = threadIdx.x; i < 3 * nw; i += blockDim.x) c.seen_req[i] = 0;
  if (threadIdx.x == 0) {
    c.sh->tail = 0;
    c.sh->next_ticket = 0;
    c.sh->now_serving = 0;
  }
  __syncthreads();
  const uint32_t warp = threadIdx.x >> 5;
  if (warp < p.n_workers) {
    part_worker(p, c, t_begin);
  } else if (warp == kWarps - 1 && c.k == 0 && p.publish == CSMV_PUBLISH_SERVER && !p.pub_remote) {
    server_publisher(p, nullptr, t_begin, p.gts_start);
  }
  __syncthreads();
  if (c.k == 0 && threadIdx.x == 0) {
    p.ctl->tail_final = ld_relaxed(&p.ctl->cts_next);
    st_release(&p.ctl->srv_done, 1u);
  }
}

}  // namespace csmvd
