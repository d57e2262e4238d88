// Micro-benchmark: latency of the server critical-section building blocks on
// one SM, with and without background global-load traffic from other warps.
#include <cstdio>
#include <cstdint>
#include <cuda_runtime.h>

__device__ __forceinline__ uint32_t ld_relaxed(const uint32_t* p) {
  uint32_t v; asm volatile("ld.relaxed.gpu.global.u32 %0, [%1];" : "=r"(v) : "l"(p) : "memory"); return v;
}

__global__ void bench(uint32_t* g, unsigned long long* out, int bg_warps, int bg_sleep) {
  extern __shared__ uint64_t tab[];
  __shared__ volatile int stop;
  const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
  for (int i = threadIdx.x; i < 2048 * 8; i += blockDim.x) tab[i] = 0xFFFFFFFFull;
  if (threadIdx.x == 0) stop = 0;
  __syncthreads();
  if (warp > 0) {
    if (warp <= bg_warps) {
      uint32_t acc = 0;
      while (!stop) {
        for (int k = 0; k < 8; ++k) acc += ld_relaxed(g + ((warp * 8 + k) * 32 + lane) % (1 << 20));
        if (bg_sleep) __nanosleep(bg_sleep);
      }
      if (acc == 12345) g[0] = acc;
    }
    return;
  }
  unsigned long long t[8] = {0};
  uint32_t key = (lane * 2654435761u) ^ 0x1234567u;
  uint32_t dummy = 0;
  for (int it = 0; it < 1000; ++it) {
    key = key * 1664525u + 1013904223u;
    const uint32_t set = key >> 21;                   // 2048 sets
    const bool act = lane < 16;
    long long a = clock64();
    long long b = clock64();
    t[0] += b - a;                                    // clock64 overhead
    // one dependent LDS
    a = clock64();
    uint32_t v = ((volatile uint32_t*)tab)[set];
    dummy += v;
    b = clock64();
    t[1] += b - a;
    // atr_conflict-like: 4 x LDS.128 of a random set
    a = clock64();
    const ulonglong2* e = reinterpret_cast<const ulonglong2*>(tab + set * 8);
    bool c = false;
    if (act) {
#pragma unroll
      for (int j = 0; j < 4; ++j) { ulonglong2 q = e[(j + set) & 3]; c |= (uint32_t)q.x == key || (uint32_t)q.y == key; }
    }
    uint32_t m = __ballot_sync(0xFFFFFFFFu, c);
    b = clock64();
    t[2] += b - a;
    dummy += m;
    // match_any
    a = clock64();
    uint32_t peers = __match_any_sync(0xFFFFFFFFu, set & 7);
    b = clock64();
    t[3] += b - a;
    dummy += peers;
    // STS + syncwarp + verify
    a = clock64();
    if (act) tab[set * 8 + (lane & 7)] = ((uint64_t)it << 32) | key;
    __syncwarp();
    bool ok = act && tab[set * 8 + (lane & 7)] == (((uint64_t)it << 32) | key);
    m = __ballot_sync(0xFFFFFFFFu, ok);
    b = clock64();
    t[4] += b - a;
    dummy += m;
    // fence.acq_rel.cta
    a = clock64();
    asm volatile("fence.acq_rel.cta;" ::: "memory");
    b = clock64();
    t[5] += b - a;
    // atomicMax smem
    a = clock64();
    if (lane == 0) atomicMax((unsigned*)&tab[0], (unsigned)it);
    __syncwarp();
    b = clock64();
    t[6] += b - a;
  }
  if (lane == 0) {
    stop = 1;
    for (int i = 0; i < 7; ++i) out[i] = t[i] / 1000;
    out[7] = dummy;
  }
}

int main() {
  uint32_t* g; unsigned long long* o;
  cudaMalloc(&g, 4 << 20); cudaMemset(g, 0, 4 << 20);
  cudaMallocManaged(&o, 64);
  cudaFuncSetAttribute(bench, cudaFuncAttributeMaxDynamicSharedMemorySize, 2048 * 8 * 8);
  const char* names[] = {"clock64", "LDS dep", "conflict4xLDS128+ballot", "match_any", "STS+sync+verify", "fence.cta", "atomicMax+sync"};
  int cfg[][2] = {{0, 0}, {1, 0}, {4, 0}, {15, 0}, {15, 64}};
  for (auto& c : cfg) {
    bench<<<1, 512, 2048 * 8 * 8>>>(g, o, c[0], c[1]);
    cudaDeviceSynchronize();
    printf("bg_warps=%2d sleep=%3d:", c[0], c[1]);
    for (int i = 0; i < 7; ++i) printf("  %s=%llu", names[i], o[i]);
    printf("\n");
  }
  printf("err=%s\n", cudaGetErrorString(cudaGetLastError()));
}
