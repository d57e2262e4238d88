// gen.cuh -- the CUDA path's own implementation of docs/GENERATOR.md
// (counter-based: a transaction's descriptor is a pure function of
// (seed, tx), computed in registers -- no descriptor array in HBM).
// The zipf CDF table is built on the host (host.cu) and read here.
#pragma once
#include <cstdint>

namespace csmvd {

__host__ __device__ __forceinline__ uint64_t mix64(uint64_t x) {
  uint64_t z = x + 0x9E3779B97F4A7C15ull;
  z = (z ^ (z >> 30)) * 0xBF58476D1CE4E5B9ull;
  z = (z ^ (z >> 27)) * 0x94D049BB133111EBull;
  return z ^ (z >> 31);
}

__host__ __device__ __forceinline__ uint64_t draw(uint64_t seed, uint64_t tx, uint64_t k) {
  return mix64(mix64(seed ^ (tx * 0xD1B54A32D192ED03ull)) + k);
}

__device__ __forceinline__ uint64_t uniform(uint64_t u, uint64_t n) { return __umul64hi(u, n); }

// first i with cdf[i] > u, clamped to n-1 (the table's last entry is
// 2^64-1).  The guide table narrows the search: with 2^m buckets of u,
// guide[b] = the pick at the start of bucket b and guide[2^m] = n-1, so the
// pick of any u in bucket b lies in [guide[b], guide[b+1]] (picks are
// monotone in u) -- the upper_bound over that range is the same as over
// the whole table (a couple of dependent loads instead of log2 n).
__device__ __forceinline__ uint32_t zipf_pick(const uint64_t* __restrict__ cdf, const uint32_t* __restrict__ guide,
                                              uint32_t m, uint32_t n, uint64_t u) {
  const uint32_t b = m ? (uint32_t)(u >> (64 - m)) : 0u;
  uint32_t lo = __ldg(guide + b), hi = __ldg(guide + b + 1);
  while (lo < hi) {  // the answer is in [lo, hi]: hi itself needs no test
    const uint32_t mid = (lo + hi) >> 1;
    if (__ldg(cdf + mid) > u) hi = mid; else lo = mid + 1;
  }
  return lo < n ? lo : n - 1;
}

struct GenParams {
  uint64_t seed;
  uint64_t upd_thresh;       // update iff (draw(.,0) >> 32) < upd_thresh
  const uint64_t* zipf_cdf;  // non-null iff zipf
  const uint32_t* zipf_guide;  // [2^guide_log2 + 1] (zipf_pick)
  uint32_t guide_log2;
  uint32_t n_items;          // bank: accounts; KV: key space
  uint32_t ro_period;
  uint32_t ro_reads;
  uint32_t amount_max;
};

struct BankTx {
  uint32_t is_update;
  uint32_t src, dst;
  int32_t amt;
  uint32_t start, len;
};

__device__ __forceinline__ uint32_t gen_pick(const GenParams& g, uint64_t u) {
  return g.zipf_cdf ? zipf_pick(g.zipf_cdf, g.zipf_guide, g.guide_log2, g.n_items, u) : (uint32_t)uniform(u, g.n_items);
}

__device__ __forceinline__ bool gen_is_update(const GenParams& g, uint64_t tx) {
  if (g.ro_period) return (tx % g.ro_period) != (uint64_t)(g.ro_period - 1);
  return (draw(g.seed, tx, 0) >> 32) < g.upd_thresh;
}

__device__ __forceinline__ BankTx gen_bank(const GenParams& g, uint64_t tx) {
  BankTx d;
  d.is_update = gen_is_update(g, tx);
  d.src = d.dst = 0;
  d.amt = 0;
  d.start = 0;
  d.len = 0;
  if (d.is_update) {
    d.src = gen_pick(g, draw(g.seed, tx, 1));
    d.dst = gen_pick(g, draw(g.seed, tx, 2));
    if (d.dst == d.src) d.dst = (d.src + 1 == g.n_items) ? 0 : d.src + 1;
    d.amt = (int32_t)(1 + uniform(draw(g.seed, tx, 3), g.amount_max));
  } else if (g.ro_reads == 0) {
    d.len = g.n_items;
  } else {
    d.start = (uint32_t)uniform(draw(g.seed, tx, 1), g.n_items);
    d.len = g.ro_reads;
  }
  return d;
}

// the read-only fields of transaction tx without the update's endpoint
// draws (zipf picks are a binary search): false if tx is an update
__device__ __forceinline__ bool gen_bank_ro(const GenParams& g, uint64_t tx, uint32_t& start, uint32_t& len) {
  start = len = 0;
  if (gen_is_update(g, tx)) return false;
  if (g.ro_reads == 0) {
    len = g.n_items;
  } else {
    start = (uint32_t)uniform(draw(g.seed, tx, 1), g.n_items);
    len = g.ro_reads;
  }
  return true;
}

// digest contribution of one 4-byte item (docs/GENERATOR.md section 5)
__device__ __forceinline__ uint64_t dig1(uint32_t item, uint32_t val) {
  return mix64(((uint64_t)item << 32) ^ (uint64_t)val);
}

}  // namespace csmvd
