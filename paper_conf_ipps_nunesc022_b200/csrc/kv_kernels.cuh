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

}  // namespace csmvd

#include "client_kv.cuh"

namespace csmvd {

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
