// server_part.cuh -- item-partitioned commit over S independent server CTAs
// (CSMV_SERVER_PART; NEXT-3, the paper's first future-work item).
//
// Server k owns the items x with part_owner(x) == k (x mod S) and keeps, in
// its own shared memory, the part of the ATR for them: a 32-bit recent-write
// filter (slot = largest CTS of a decided write hashing there, two hashes)
// and one pending bit per owned item (bit x / S; folded when the partition
// has more than 2^20 items -- a false conflict then, never a missed one).
// One CTS sequence stays global (a counter in Ctl).  A client warp's batch
// goes through three messages (checked by exhaustive
// interleavings in the two-server model checker under tests/ before this
// code):
//   1 PREPARE at every server owning an item of the batch: for each lane
//     with an item here, claim the pending bit of each of its items here
//     (atomicOr; a bit already set is another transaction in flight on it:
//     CONFLICT, the lane gives back what it claimed), then validate that
//     part -- lastw[x] <= s for the commits up to e_pre = GTS, no filter slot
//     set after e_pre (else OVERFLOW, the claims given back); vote (lanes
//     with nothing here vote yes);
//   2 the client ANDs the votes and takes CTS = ++counter for the survivors
//     (one L2 atomic per batch);
//   3 DECIDE at every prepared server: record the committed write-sets in the
//     filter (atomicMax: decides may arrive out of CTS order), then clear
//     the pending bits of every lane this server marked; acknowledge.
// Two conflicting transactions share an item, hence its server and its
// pending bit, so they are never prepared at the same time; the later one
// claims the bit after the earlier one's decide cleared it, which follows
// (fence.cta) that decide's filter record -- so it sees the record (or
// lastw) and aborts, or its snapshot covers it -- and takes its CTS after
// the earlier one took its own.  No lock: the claims are the serialisation
// (the single server's critical section is a ticket lock, server.cuh).
// Write-back, lastw and the GTS publish (done flags, server publisher) are
// as in the other servers.
//
// Each server CTA runs self-receiving worker warps (a slice of the client
// warps each, round robin, decides first), and server 0 the publisher
// (unless it runs on a client CTA).  Included by fused.cuh after server.cuh.
#pragma once

namespace csmvd {

__device__ __forceinline__ uint32_t part_filt_slot(uint32_t x, int k) {
  const uint32_t C[2] = {0x9E3779B1u, 0x85EBCA77u};
  return (x * C[k]) >> (32 - kPartFiltLog2);
}
struct PartCtx {
  uint32_t* filt;       // [2^kPartFiltLog2]
  uint32_t* pend;       // [2^(part_bits_log2 - 5)] pending bit per owned item
  uint32_t* seen_req;   // [n_cw] last prepare doorbell seen
  uint32_t* seen_dec;   // [n_cw] last decide doorbell seen
  uint32_t* marked;     // [n_cw] lanes this server marked pending at the client warp's last prepare
  uint32_t k;           // this server
};

__device__ __forceinline__ uint32_t part_bit(const KParams& p, uint32_t x) {
  return (x >> p.part_log2) & ((1u << p.part_bits_log2) - 1);
}
// claim x's pending bit: true if it was free (now ours)
__device__ __forceinline__ bool pend_claim(const KParams& p, uint32_t* pend, uint32_t x) {
  const uint32_t i = part_bit(p, x), m = 1u << (i & 31);
  return (atomicOr(pend + (i >> 5), m) & m) == 0;
}
__device__ __forceinline__ void pend_release(const KParams& p, uint32_t* pend, uint32_t x) {
  const uint32_t i = part_bit(p, x);
  atomicAnd(pend + (i >> 5), ~(1u << (i & 31)));
}

static __device__ void part_worker(const KParams& p, const PartCtx& c, uint64_t t_begin) {
  const uint32_t FULL = 0xFFFFFFFFu;
  const uint32_t lane = threadIdx.x & 31;
  const uint32_t warp = threadIdx.x >> 5;
  const size_t off = (size_t)c.k * p.mstride;
  const uint32_t per = (p.n_cw + p.n_workers - 1) / p.n_workers;
  const uint32_t lo = min(warp * per, p.n_cw), hi = min(lo + per, p.n_cw), n = hi - lo, rows = (n + 31) / 32;
  const bool novalid = (p.debug & CSMV_DBG_NO_VALIDATE) != 0;
  unsigned long long batches = 0, decides = 0, locked = 0;
  Jitter jit(p, 11);
  uint32_t rr = 0, rl = 31;  // round robin: next row to look at, last lane served
  for (uint32_t idle = 1;; ++idle) {
    // ---- sweep, round robin over rows and lanes (a fixed scan order starves
    // the last rows' clients -- and their decides, whose marks then block
    // everyone); in the chosen row a pending decide first (it unblocks
    // others).  Up to 4 rows' doorbells in one L2 round trip.
    uint32_t cw = 0xFFFFFFFFu, seq = 0;
    bool dec = false;
    for (uint32_t q0 = 0; q0 < rows && cw == 0xFFFFFFFFu; q0 += 4) {
      uint32_t sd[4], sr[4];
#pragma unroll
      for (int k = 0; k < 4; ++k) {
        const uint32_t i = lo + ((rr + q0 + k) % rows) * 32 + lane;
        const bool v = q0 + k < rows && i < hi;
        sd[k] = v ? ld_relaxed(p.mdec_seq + off + i) : 0u;
        sr[k] = v ? ld_relaxed(p.mreq_seq + off + i) : 0u;
      }
#pragma unroll
      for (int k = 0; k < 4; ++k) {
        const uint32_t r = (rr + q0 + k) % rows, i = lo + r * 32 + lane;
        if (q0 + k >= rows || cw != 0xFFFFFFFFu) break;
        const uint32_t pd = __ballot_sync(FULL, i < hi && sd[k] != c.seen_dec[i]);
        const uint32_t pr = __ballot_sync(FULL, i < hi && sr[k] != c.seen_req[i]);
        if (pd | pr) {
          dec = pd != 0;
          const uint32_t m = dec ? pd : pr;
          const uint32_t after = m & ~(0xFFFFFFFFu >> (31 - rl));  // lanes past the last one served
          const uint32_t l = __ffs(after ? after : m) - 1;
          seq = __shfl_sync(FULL, dec ? sd[k] : sr[k], l);
          cw = lo + r * 32 + l;
          if (lane == l) (dec ? c.seen_dec : c.seen_req)[cw] = seq;
          rr = r + 1;
          rl = l;
        }
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
      const long long t1 = clock64();
      if ((cm >> lane) & 1u) {  // committed lanes were marked at every owner of their items
        const uint32_t cts = base + __popc(cm & lanemask_lt());
#pragma unroll
        for (int k = 0; k < 2; ++k) {
          if (xa) atomicMax(c.filt + part_filt_slot(a, k), cts);
          if (xb) atomicMax(c.filt + part_filt_slot(b, k), cts);
        }
      }
      __threadfence_block();  // the records precede the release of the bits (a later claimer sees them)
      if ((c.marked[cw] >> lane) & 1u) {
        if (xa) pend_release(p, c.pend, a);
        if (xb) pend_release(p, c.pend, b);
      }
      locked += (unsigned long long)(clock64() - t1);
      __syncwarp();
      if (lane == 0) st_release(p.mdack + off + cw, seq);  // our payload loads precede the acknowledgement
      ++decides;
      continue;
    }
    // ---- PREPARE: validate our part of each lane, mark it pending, vote
    // lastw covers every CTS <= GTS (client write-back); read again here, not
    // the sweep's value: with the clients' own GTS chain the sweep's e_pre
    // lags enough for the filter to reject most prepares (OVERFLOW storms)
    const uint32_t e_pre = ld_acquire(p.gts);
    const uint32_t la = oa ? ld_relaxed(p.lastw + a) : 0u, lb = ob ? ld_relaxed(p.lastw + b) : 0u;
    const bool here = oa || ob;
    const bool chk = here && (novalid || (la <= s && lb <= s));
    const long long t1 = clock64();
    bool ovf = false, conf = false;
    if (chk && !novalid) {
      // claims in increasing bit order: of two transactions wanting the same
      // two bits, one gets both (claimed in any order, each could hold one
      // and both abort -- 40-60 % aborts on C2 at 2-8 servers)
      const bool af = !ob || part_bit(p, a) < part_bit(p, b);
      const uint32_t x0 = af ? a : b, x1 = af ? b : a;
      const bool o0 = af ? oa : ob, o1 = af ? ob : oa;
      const bool g0 = !o0 || pend_claim(p, c.pend, x0);
      const bool g1 = g0 && (!o1 || pend_claim(p, c.pend, x1));
      const bool ga = af ? g0 : g1, gb = af ? g1 : g0;
      conf = !(ga && gb);
      __threadfence_block();  // our claims precede the filter reads (a decide that released a bit recorded first)
      if (!conf) {
#pragma unroll
        for (int x = 0; x < 2; ++x) {
          const bool o = x ? ob : oa;
          const uint32_t it = x ? b : a;
          if (o) ovf = ovf || min(c.filt[part_filt_slot(it, 0)], c.filt[part_filt_slot(it, 1)]) > e_pre;
        }
      }
      if (conf || ovf) {  // give back what this lane claimed
        if (oa && ga) pend_release(p, c.pend, a);
        if (ob && gb) pend_release(p, c.pend, b);
      }
    }
    const bool ok = chk && !ovf && !conf;
    const uint32_t okm = __ballot_sync(FULL, ok);
    const uint32_t om = __ballot_sync(FULL, chk && ovf && !conf);  // labelled OVERFLOW, the rest CONFLICT
    if (lane == 0) c.marked[cw] = novalid ? 0u : okm;
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
  const uint32_t pw = part_pend_words(p.part_bits_log2);
  c.seen_req = c.pend + pw;
  const uint32_t nw = (p.n_cw + 31) / 32 * 32;
  c.seen_dec = c.seen_req + nw;
  c.marked = c.seen_dec + nw;
  for (uint32_t i = threadIdx.x; i < (1u << kPartFiltLog2) + pw + 3 * nw; i += blockDim.x) c.filt[i] = 0;
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
