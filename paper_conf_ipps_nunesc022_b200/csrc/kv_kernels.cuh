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
