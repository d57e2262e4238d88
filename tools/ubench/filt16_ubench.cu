// Serial chain of the locked bank critical section, 32-bit vs 16-bit filter
// slots (one warp, idle SM): loads -> test -> ballot -> CTS -> stores.
//  mode 0: 32-bit slots, min/max test against e_pre
//  mode 1: 16-bit slots, age = (t - v) & 0xFFFF, max/min test against the window
//  mode 2: 16-bit slots, per-slot "recent" predicates combined with AND/OR
//  mode 3: 16-bit slots, ages of slot pairs with 16x2 SIMD (vsub2 / vmaxu2)
#include <cstdio>
#include <cstdint>
#include <cuda_runtime.h>
__device__ __forceinline__ uint32_t lds32(uint32_t a) { uint32_t v; asm volatile("ld.shared.u32 %0, [%1];" : "=r"(v) : "r"(a) : "memory"); return v; }
__device__ __forceinline__ void sts32(uint32_t a, uint32_t v) { asm volatile("st.shared.u32 [%0], %1;" ::"r"(a), "r"(v) : "memory"); }
__device__ __forceinline__ uint32_t lds16(uint32_t a) { uint16_t v; asm volatile("ld.shared.u16 %0, [%1];" : "=h"(v) : "r"(a) : "memory"); return v; }
__device__ __forceinline__ void sts16(uint32_t a, uint32_t v) { uint16_t h = (uint16_t)v; asm volatile("st.shared.u16 [%0], %1;" ::"r"(a), "h"(h) : "memory"); }
template <int MODE>
__global__ void k(unsigned long long* out, int iters) {
  extern __shared__ uint32_t sm[];
  for (uint32_t i = threadIdx.x; i < 32768; i += blockDim.x) sm[i] = 0;
  __syncthreads();
  if (threadIdx.x >= 32) return;
  const uint32_t lane = threadIdx.x, lt = (1u << lane) - 1;
  const uint32_t base = (uint32_t)__cvta_generic_to_shared(sm);
  const uint32_t sh = MODE == 0 ? 17 : 16, sz = MODE == 0 ? 4 : 2;
  uint32_t t = 1000, x = lane * 2654435761u + 7u, acc = 0;
  const long long c0 = clock64();
  for (int it = 0; it < iters; ++it) {
    x = x * 1664525u + 1013904223u;
    const uint32_t y = x + 12345u;
    uint32_t a[6] = {base + sz * ((x * 0x9E3779B1u) >> sh), base + sz * ((x * 0x85EBCA77u) >> sh), base + sz * ((x * 0xC2B2AE3Du) >> sh),
                     base + sz * ((y * 0x9E3779B1u) >> sh), base + sz * ((y * 0x85EBCA77u) >> sh), base + sz * ((y * 0xC2B2AE3Du) >> sh)};
    const uint32_t e_pre = t - 200;
    bool ovf;
    if (MODE == 0) {
      uint32_t v[6];
#pragma unroll
      for (int i = 0; i < 6; ++i) v[i] = lds32(a[i]);
      ovf = max(min(v[0], min(v[1], v[2])), min(v[3], min(v[4], v[5]))) > e_pre;
    } else if (MODE == 1) {
      uint32_t v[6];
#pragma unroll
      for (int i = 0; i < 6; ++i) v[i] = lds16(a[i]);
      const uint32_t aa = max((t - v[0]) & 0xFFFFu, max((t - v[1]) & 0xFFFFu, (t - v[2]) & 0xFFFFu));
      const uint32_t ab = max((t - v[3]) & 0xFFFFu, max((t - v[4]) & 0xFFFFu, (t - v[5]) & 0xFFFFu));
      const uint32_t win = t - e_pre;
      ovf = win > 0xFFFFu || min(aa, ab) < win;
    } else if (MODE == 2) {
      uint32_t v[6];
#pragma unroll
      for (int i = 0; i < 6; ++i) v[i] = lds16(a[i]);
      const uint32_t win = t - e_pre, e1 = e_pre + 1;
      bool r[6];
#pragma unroll
      for (int i = 0; i < 6; ++i) r[i] = ((v[i] - e1) & 0xFFFFu) < win;
      ovf = (r[0] && r[1] && r[2]) || (r[3] && r[4] && r[5]);
    } else {
      uint32_t v[6];
#pragma unroll
      for (int i = 0; i < 6; ++i) v[i] = lds16(a[i]);
      // ages of (v0,v1), (v2,v3), (v4,v5) as 16x2
      const uint32_t t2 = (t & 0xFFFFu) * 0x10001u;
      const uint32_t g01 = __vsub2(t2, v[0] | (v[1] << 16)), g23 = __vsub2(t2, v[2] | (v[3] << 16)),
                     g45 = __vsub2(t2, v[4] | (v[5] << 16));
      const uint32_t aa = max(max(g01 & 0xFFFFu, g01 >> 16), g23 & 0xFFFFu);
      const uint32_t ab = max(max(g23 >> 16, g45 & 0xFFFFu), g45 >> 16);
      const uint32_t win = t - e_pre;
      ovf = win > 0xFFFFu || min(aa, ab) < win;
    }
    const bool commit = lane < 29 && !ovf;
    const uint32_t cm = __ballot_sync(~0u, commit);
    acc += __popc(cm & lt);
    t += __popc(cm);
    if (commit) {
#pragma unroll
      for (int i = 0; i < 6; ++i) { if (MODE == 0) sts32(a[i], t); else sts16(a[i], t); }
    }
    __syncwarp();
  }
  const long long c1 = clock64();
  if (lane == 0) out[MODE] = (unsigned long long)(c1 - c0) / iters + 0 * acc;
}

// Grouped requests (csmv_workload.client_group, server_worker<G>): G
// sub-batches of 32 transfers, KH hashes per item; all G x 2 x KH probes of a
// request are issued together, G ballots, one CTS prefix, G x 2 x KH stores.
template <int G, int KH>
__global__ void kg(unsigned long long* out, int iters, int slot) {
  extern __shared__ uint32_t sm[];
  for (uint32_t i = threadIdx.x; i < 32768; i += blockDim.x) sm[i] = 0;
  __syncthreads();
  if (threadIdx.x >= 32) return;
  const uint32_t lane = threadIdx.x, lt = (1u << lane) - 1;
  const uint32_t base = (uint32_t)__cvta_generic_to_shared(sm);
  const uint32_t C[3] = {0x9E3779B1u, 0x85EBCA77u, 0xC2B2AE3Du};
  uint32_t t = 1000, x = lane * 2654435761u + 7u, acc = 0;
  const long long c0 = clock64();
  for (int it = 0; it < iters; ++it) {
    uint32_t a[G][2 * KH];
#pragma unroll
    for (int g = 0; g < G; ++g) {
      x = x * 1664525u + 1013904223u;
      const uint32_t y = x + 12345u;
#pragma unroll
      for (int k = 0; k < KH; ++k) {
        a[g][k] = base + 2 * ((x * C[k]) >> 16);
        a[g][KH + k] = base + 2 * ((y * C[k]) >> 16);
      }
    }
    const uint32_t e_pre = t - 200, win = t - e_pre, e1 = e_pre + 1;
    uint32_t v[G][2 * KH];
#pragma unroll
    for (int g = 0; g < G; ++g)
#pragma unroll
      for (int i = 0; i < 2 * KH; ++i) v[g][i] = lds16(a[g][i]);
    bool cm[G];
#pragma unroll
    for (int g = 0; g < G; ++g) {
      bool ra = true, rb = true;
#pragma unroll
      for (int k = 0; k < KH; ++k) {
        ra = ra && ((v[g][k] - e1) & 0xFFFFu) < win;
        rb = rb && ((v[g][KH + k] - e1) & 0xFFFFu) < win;
      }
      cm[g] = lane < 27 && !(ra || rb);
      const uint32_t m = __ballot_sync(~0u, cm[g]);
      acc += __popc(m & lt);
      t += __popc(m);
    }
#pragma unroll
    for (int g = 0; g < G; ++g)
      if (cm[g]) {
#pragma unroll
        for (int i = 0; i < 2 * KH; ++i) sts16(a[g][i], t);
      }
    __syncwarp();
  }
  const long long c1 = clock64();
  if (lane == 0) out[slot] = (unsigned long long)(c1 - c0) / iters + 0 * acc;
}

int main() {
  unsigned long long* out; cudaMalloc(&out, 128);
  const size_t sm = 32768 * 4;
  cudaFuncSetAttribute(k<0>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)sm);
  cudaFuncSetAttribute(k<1>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)sm);
  cudaFuncSetAttribute(k<2>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)sm);
  cudaFuncSetAttribute(k<3>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)sm);
  k<0><<<1, 256, sm>>>(out, 100000); k<1><<<1, 256, sm>>>(out, 100000);
  k<2><<<1, 256, sm>>>(out, 100000); k<3><<<1, 256, sm>>>(out, 100000);
  cudaFuncSetAttribute(kg<1, 2>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)sm);
  cudaFuncSetAttribute(kg<1, 3>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)sm);
  cudaFuncSetAttribute(kg<2, 2>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)sm);
  cudaFuncSetAttribute(kg<4, 2>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)sm);
  cudaFuncSetAttribute(kg<8, 2>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)sm);
  kg<1, 2><<<1, 256, sm>>>(out, 100000, 4); kg<1, 3><<<1, 256, sm>>>(out, 100000, 5);
  kg<2, 2><<<1, 256, sm>>>(out, 100000, 6); kg<4, 2><<<1, 256, sm>>>(out, 100000, 7);
  kg<8, 2><<<1, 256, sm>>>(out, 100000, 8);
  unsigned long long h[9]; cudaMemcpy(h, out, 72, cudaMemcpyDeviceToHost);
  const char* n[] = {"u32 min/max", "u16 age max/min", "u16 recent predicates", "u16 vsub2 ages"};
  for (int i = 0; i < 4; ++i) printf("mode %d %-22s %llu cycles/batch\n", i, n[i], h[i]);
  const char* g[] = {"g1k2", "g1k3", "g2k2", "g4k2", "g8k2"};
  for (int i = 0; i < 5; ++i) printf("grouped %s %llu cycles/request\n", g[i], h[4 + i]);
  printf("%s\n", cudaGetErrorString(cudaDeviceSynchronize()));
}
