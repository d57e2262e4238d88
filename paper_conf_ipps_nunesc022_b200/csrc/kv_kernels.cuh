// kv_kernels.cuh -- setup, dump and generator kernels of the MemcachedGPU
// workload; its client warp is client_kv.cuh.  Included by kernel.cu.
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
#include "fused.cuh"

namespace csmvd {

// ---- setup and dump kernels

// Device preload of keys 0..n-1 with PUT semantics (docs/GENERATOR.md 4),
// in three passes: count the keys of every set, scatter them into per-set
// buckets (bucket order is arbitrary), then one thread per set keeps the m =
// min(A, c) largest keys of its bucket.  Keys are inserted in key order and
// are pairwise distinct (mix64 is a bijection, and no key is all-zero: that
// would need k = mix64^-1(0) and k ^ 0x55.. = mix64^-1(0) at once), so a
// set's r-th insertion (0-based) fills way r mod A -- the first A fill the
// empty ways in order, each later one evicts the smallest LRU clock, the
// oldest insertion -- and the survivors are its last m insertions, i.e. its
// m largest keys, with ranks c-m .. c-1 and LRU clock rank+1.
__global__ void kv_preload_count(uint32_t n, uint32_t T, uint32_t* cnt) {
  for (uint32_t k = blockIdx.x * blockDim.x + threadIdx.x; k < n; k += gridDim.x * blockDim.x)
    atomicAdd(&cnt[kv_set(k, T)], 1u);
}

__global__ void kv_preload_scatter(uint32_t n, uint32_t T, const uint32_t* off, uint32_t* fill,
                                   uint32_t* bucket) {
  for (uint32_t k = blockIdx.x * blockDim.x + threadIdx.x; k < n; k += gridDim.x * blockDim.x) {
    const uint32_t t = kv_set(k, T);
    bucket[off[t] + atomicAdd(&fill[t], 1u)] = k;
  }
}

constexpr uint32_t kMaxWays = 256;

// keys/vals/lru/clocks: the plain-word layout init_kv_rings installs
// (zeroed by the caller: empty ways stay all-zero).
__global__ void kv_preload_place(uint32_t T, uint32_t A, const uint32_t* off, const uint32_t* cnt,
                                 const uint32_t* bucket, uint32_t* keys, uint32_t* vals, uint32_t* lru,
                                 uint32_t* clocks) {
  const uint32_t t = blockIdx.x * blockDim.x + threadIdx.x;
  if (t >= T) return;
  const uint32_t c = cnt[t], m = c < A ? c : A;
  const uint32_t* b = bucket + off[t];
  uint32_t top[kMaxWays];  // ascending: the m largest keys seen so far
  uint32_t n = 0;
  for (uint32_t i = 0; i < c; ++i) {
    const uint32_t x = b[i];
    uint32_t j;
    if (n < m) {
      j = n++;
    } else if (x > top[0]) {
      j = 0;
      while (j + 1 < n && top[j + 1] < x) {
        top[j] = top[j + 1];
        ++j;
      }
      top[j] = x;
      continue;
    } else {
      continue;
    }
    while (j > 0 && top[j - 1] > x) {
      top[j] = top[j - 1];
      --j;
    }
    top[j] = x;
  }
  for (uint32_t j = 0; j < n; ++j) {
    const uint32_t k = top[j], r = c - n + j;
    const uint64_t slot = (uint64_t)t * A + r % A;
    uint32_t kk[4];
    kv_key16(k, kk);
#pragma unroll
    for (int w = 0; w < 4; ++w) keys[slot * 4 + w] = kk[w];
#pragma unroll
    for (uint32_t w = 0; w < 4; ++w) {
      const uint64_t x = mix64((((uint64_t)k << 2) | w) ^ 0x3C3C3C3C3C3C3C3Cull);
      vals[slot * 8 + 2 * w] = (uint32_t)x;
      vals[slot * 8 + 2 * w + 1] = (uint32_t)(x >> 32);
    }
    lru[slot] = r + 1;
  }
  clocks[t] = c;
}

template <int NS>
__global__ void init_kv_rings(KParams p, const uint32_t* keys, const uint32_t* vals, const uint32_t* lru,
                              const uint32_t* clocks) {
  // one thread per ring word, grid-stride over each ring array in turn
  // (coalesced stores: the rings are [item][NS][W] u64)
  const uint64_t tid = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x, stride = (uint64_t)gridDim.x * blockDim.x;
  if (tid == 0) *p.gts = 0;
  const uint64_t E = (uint64_t)kEmptyTs << 32;
  const uint64_t S = p.kv_S, T = p.kv_T;
  for (uint64_t x = tid; x < S * NS * 4; x += stride) {
    const uint64_t i = x / (NS * 4), j = (x / 4) % NS;
    p.kv_key[x] = j ? E : (uint64_t)keys[i * 4 + (x & 3)];
  }
  for (uint64_t x = tid; x < S * NS * 8; x += stride) {
    const uint64_t i = x / (NS * 8), j = (x / 8) % NS;
    p.kv_val[x] = j ? E : (uint64_t)vals[i * 8 + (x & 7)];
  }
  for (uint64_t x = tid; x < S * NS; x += stride) p.kv_lru[x] = (x % NS) ? E : (uint64_t)lru[x / NS];
  for (uint64_t x = tid; x < T * NS; x += stride) p.kv_clk[x] = (x % NS) ? E : (uint64_t)clocks[x / NS];
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
