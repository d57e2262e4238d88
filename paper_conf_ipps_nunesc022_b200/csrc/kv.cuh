// kv.cuh -- MemcachedGPU workload on the CSMV pipeline.
//
// The store is an A-way set-associative cache of S slots (T = S/A sets).
// Every key (16 B), value (32 B), per-slot LRU stamp and per-set clock is a
// versioned item (VBox) with K versions:
//   key ring   u64[S][NS][4]   value ring u64[S][NS][8]
//   lru ring   u64[S][NS]      clock ring u64[T][NS]
// A version of a multi-word item stores every 4-byte word as (ts << 32 |
// word): a reader accepts a version only if all its words carry the same ts,
// so a version being recycled by a concurrent write-back is detected without
// fences (a torn read shows two timestamps).  Item ids (docs/GENERATOR.md 4):
// key i, value S+i, LRU 2S+i, clock 3S+t.
#pragma once
#include "kernel.cuh"
#include "ptx.cuh"

namespace csmvd {

enum : int { RD_OK = 0, RD_MISS = 1, RD_NEWER = 2 };

__device__ __forceinline__ void kv_key16(uint32_t k, uint32_t (&out)[4]) {
  const uint64_t a = mix64((uint64_t)k), b = mix64((uint64_t)k ^ 0x5555555555555555ull);
  out[0] = (uint32_t)a;
  out[1] = (uint32_t)(a >> 32);
  out[2] = (uint32_t)b;
  out[3] = (uint32_t)(b >> 32);
}

__device__ __forceinline__ uint32_t kv_set(uint32_t k, uint32_t T) {
  return (uint32_t)uniform(mix64((uint64_t)k ^ 0xA5A5A5A5A5A5A5A5ull), T);
}

struct KvTx {
  uint32_t is_update;
  uint32_t key;
  uint32_t val[8];
};

__device__ __forceinline__ bool gen_kv_is_update(const GenParams& g, uint64_t tx) {
  return (draw(g.seed, tx, 0) >> 32) < g.upd_thresh;
}
__device__ __forceinline__ uint32_t gen_kv_key(const GenParams& g, uint64_t tx) {
  return gen_pick(g, draw(g.seed, tx, 1));  // a zipf pick is a binary search over the key CDF
}
// transaction tx with its key already drawn (gen_kv_key)
__device__ __forceinline__ KvTx gen_kv_k(const GenParams& g, uint64_t tx, uint32_t key) {
  KvTx d;
  d.is_update = gen_kv_is_update(g, tx);
  d.key = key;
#pragma unroll
  for (int j = 0; j < 4; ++j) {
    const uint64_t v = d.is_update ? draw(g.seed, tx, 4 + j) : 0ull;
    d.val[2 * j] = (uint32_t)v;
    d.val[2 * j + 1] = (uint32_t)(v >> 32);
  }
  return d;
}
__device__ __forceinline__ KvTx gen_kv(const GenParams& g, uint64_t tx) { return gen_kv_k(g, tx, gen_kv_key(g, tx)); }

__device__ __forceinline__ uint64_t dig_word(uint32_t item, uint32_t w, uint32_t word) {
  return mix64(((uint64_t)item << 35) ^ ((uint64_t)w << 32) ^ (uint64_t)word);
}

// Read a W-word item at snapshot s.  rot: a read-only transaction (a newer
// version is fine); otherwise any version newer than s means
// validation must fail (RD_NEWER).
// `seen` (optional) is raised to the newest version timestamp present.
template <int NS, int W>
__device__ __forceinline__ int kv_read_mw(const uint64_t* ring, uint32_t K, uint32_t s, bool rot,
                                          uint32_t (&out)[W], uint32_t* seen = nullptr) {
  uint32_t ts[NS];
#pragma unroll
  for (int j = 0; j < NS; ++j) ts[j] = ((uint32_t)j < K) ? (uint32_t)(ld_relaxed64(ring + j * W) >> 32) : kEmptyTs;
  int cand = -1;
  uint32_t cts = 0, newest = 0;
#pragma unroll
  for (int j = 0; j < NS; ++j) {
    if (ts[j] == kEmptyTs) continue;
    newest = max(newest, ts[j]);
    if (ts[j] <= s && (cand < 0 || ts[j] > cts)) {
      cand = j;
      cts = ts[j];
    }
  }
  if (seen) *seen = max(*seen, newest);
  if (!rot && newest > s) return RD_NEWER;
  if (cand < 0) return RD_MISS;
  // the payload read is the re-check: every word still tagged cts means the
  // version was intact after the scan (oldest-first recycling)
  if constexpr (W == 1) {
    const uint64_t v = ld_relaxed64(ring + cand);
    if ((uint32_t)(v >> 32) != cts) return rot ? RD_MISS : RD_NEWER;
    out[0] = (uint32_t)v;
  } else {
    const Ring<W> r = ld_ring<W>(ring + cand * W);
#pragma unroll
    for (int w = 0; w < W; ++w) {
      if ((uint32_t)(r.s[w] >> 32) != cts) return rot ? RD_MISS : RD_NEWER;
      out[w] = (uint32_t)r.s[w];
    }
  }
  return RD_OK;
}

// GET-side read of a key (W = 4) or value (W = 8) item at snapshot s from its whole ring,
// loaded in one pass (NS x 32 B, independent 256-bit loads) -- one memory
// round trip per way instead of kv_read_mw's two.  A slot counts only if
// all its words carry the same ts; a torn slot (a write-back in flight: its
// new words carry a CTS > s) that may hide the version visible at s makes
// the read a miss.  When a version newer than s is present the chosen slot
// is re-read (address-dependent on the first loads, so ordered after them):
// still intact means no version in (cts, s] was recycled meanwhile (oldest-
// first recycling) -- the argument of rot_coop (kernel.cu).
// rot = false (a PUT's read): any version newer than s -> RD_NEWER, as in
// kv_read_mw (a torn slot carries a newer ts, so it is covered too).
template <int NS, int W = 4>
__device__ __forceinline__ int kv_key_pick(const uint64_t* ring, const Ring<W> (&r)[NS], uint32_t K, uint32_t s,
                                           bool rot, uint32_t (&out)[W], uint32_t* seen = nullptr) {
  int cand = -1;
  uint32_t cts = 0, newest = 0, torn_max = 0;
  bool torn = false;
#pragma unroll
  for (int j = 0; j < NS; ++j) {
    if ((uint32_t)j >= K) continue;
    const uint32_t t0 = (uint32_t)(r[j].s[0] >> 32);
    bool intact = true;
#pragma unroll
    for (int w = 0; w < W; ++w) {
      const uint32_t tw = (uint32_t)(r[j].s[w] >> 32);
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
    }
  }
  if (seen) *seen = max(*seen, newest);
  if (!rot && newest > s) return RD_NEWER;
  if (cand < 0 || (torn && torn_max > cts)) return RD_MISS;
  if (newest > s) {
    const Ring<W> q = ld_ring<W>(ring + cand * W);
#pragma unroll
    for (int w = 0; w < W; ++w) {
      if ((uint32_t)(q.s[w] >> 32) != cts) return RD_MISS;
      out[w] = (uint32_t)q.s[w];
    }
    return RD_OK;
  }
#pragma unroll
  for (int j = 0; j < NS; ++j)
    if (j == cand) {
#pragma unroll
      for (int w = 0; w < W; ++w) out[w] = (uint32_t)r[j].s[w];
    }
  return RD_OK;
}

// The version timestamps of a W-word ring (one load per slot).
template <int NS, int W>
__device__ __forceinline__ void kv_ring_ts(const uint64_t* ring, uint32_t K, uint32_t (&ts)[NS]) {
#pragma unroll
  for (int j = 0; j < NS; ++j) ts[j] = ((uint32_t)j < K) ? (uint32_t)(ld_relaxed64(ring + j * W) >> 32) : 0u;
}

// The slot a new version replaces: the first unused slot, else the oldest
// (P:291), given the ring's slot timestamps.
template <int NS>
__device__ __forceinline__ int kv_install_slot(const uint32_t (&ts)[NS], uint32_t K) {
  int victim = -1;
#pragma unroll
  for (int j = 0; j < NS; ++j)
    if ((uint32_t)j < K && victim < 0 && ts[j] == kEmptyTs) victim = j;
  if (victim < 0) {
    victim = 0;
    uint32_t vts = ts[0];
#pragma unroll
    for (int j = 1; j < NS; ++j)
      if ((uint32_t)j < K && ts[j] < vts) {
        victim = j;
        vts = ts[j];
      }
  }
  return victim;
}

// Store version (cts, data) into slot `victim` of a W-word ring.
template <int W>
__device__ __forceinline__ void kv_install_at(uint64_t* ring, int victim, uint32_t cts, const uint32_t (&data)[W]) {
  uint64_t* dst = ring + victim * W;
#pragma unroll
  for (int w = 0; w < W; w += 4) {
    if (W - w >= 4) {
      asm volatile("st.relaxed.gpu.global.v4.u64 [%0], {%1,%2,%3,%4};" ::"l"(dst + w),
                   "l"(((uint64_t)cts << 32) | data[w]), "l"(((uint64_t)cts << 32) | data[w + 1]),
                   "l"(((uint64_t)cts << 32) | data[w + 2]), "l"(((uint64_t)cts << 32) | data[w + 3])
                   : "memory");
    } else {
      st_relaxed64(dst + w, ((uint64_t)cts << 32) | data[w]);
    }
  }
}

// Install version (cts, data) over kv_install_slot's slot.  The writer owns
// the item (WW check): nothing else writes it between the loads of
// ts and the store.
template <int NS, int W>
__device__ __forceinline__ void kv_install(uint64_t* ring, const uint32_t (&ts)[NS], uint32_t K, uint32_t cts,
                                           const uint32_t (&data)[W]) {
  kv_install_at<W>(ring, kv_install_slot<NS>(ts, K), cts, data);
}

// The set clock (or any one-word item) read by a PUT at snapshot s from its
// whole ring in one load: a slot's (ts, word) is one 64-bit word, so no
// re-read is needed; any version newer than s -> RD_NEWER (the PUT cannot
// commit).  *slot = the slot the PUT's own version will replace.
template <int NS>
__device__ __forceinline__ int kv_read_clk(const Ring<NS>& r, uint32_t K, uint32_t s, uint32_t& out, uint32_t& seen,
                                           int& slot) {
  uint32_t ts[NS];
#pragma unroll
  for (int j = 0; j < NS; ++j) ts[j] = (uint32_t)j < K ? (uint32_t)(r.s[j] >> 32) : kEmptyTs;
  int cand = -1;
  uint32_t cts = 0, newest = 0;
#pragma unroll
  for (int j = 0; j < NS; ++j) {
    if (ts[j] == kEmptyTs) continue;
    newest = max(newest, ts[j]);
    if (ts[j] <= s && (cand < 0 || ts[j] > cts)) {
      cand = j;
      cts = ts[j];
    }
  }
  seen = max(seen, newest);
  if (newest > s) return RD_NEWER;
  if (cand < 0) return RD_MISS;
  out = (uint32_t)slot_at<NS>(r, cand);
  slot = kv_install_slot<NS>(ts, K);
  return RD_OK;
}

template <int NS, int W>
__device__ __forceinline__ void kv_write_mw(uint64_t* ring, uint32_t K, uint32_t cts, const uint32_t (&data)[W]) {
  uint32_t ts[NS];
  kv_ring_ts<NS, W>(ring, K, ts);
  kv_install<NS, W>(ring, ts, K, cts, data);
}

// Single-word item (LRU stamp, set clock): only update transactions read them.
template <int NS>
__device__ __forceinline__ int kv_read_1(const uint64_t* ring, uint32_t K, uint32_t s, uint32_t& out,
                                         uint32_t* seen = nullptr) {
  uint32_t o[1];
  const int r = kv_read_mw<NS, 1>(ring, K, s, false, o, seen);
  out = o[0];
  return r;
}

template <int NS>
__device__ __forceinline__ void kv_write_1(uint64_t* ring, uint32_t K, uint32_t cts, uint32_t v) {
  const uint32_t d[1] = {v};
  kv_write_mw<NS, 1>(ring, K, cts, d);
}

struct KvRings {
  uint64_t* key;
  uint64_t* val;
  uint64_t* lru;
  uint64_t* clk;
};

}  // namespace csmvd
