// Micro-benchmark of the commit critical section's building blocks, using
// the real device code (server.cuh): random item ids, a 16K-bucket
// recent-commit table, 29 of 32 lanes committing 2 items each.
//  modes 0-3: one warp, no lock: ballot / +probe / +record / +lastw stores
//  mode 4   : W warps contending through the real ticket lock (cs_enter /
//             cs_leave), full probe+record+lastw body -> cycles per batch
//             of the whole serial chain (handoff included)
#include <cstdio>
#include <cuda_runtime.h>
#include "../../paper_conf_ipps_nunesc022_b200/csrc/kernel.cuh"
#include "../../paper_conf_ipps_nunesc022_b200/csrc/ptx.cuh"
namespace csmvd {
__device__ __forceinline__ bool watchdog(const KParams&, uint64_t, uint32_t) { return false; }
template <int NS>
__device__ void write_back(uint64_t*, const Ring<NS>&, uint32_t, uint32_t, uint32_t) {}
}
#include "../../paper_conf_ipps_nunesc022_b200/csrc/server.cuh"
using namespace csmvd;

__global__ void bench(uint32_t* lastw, unsigned long long* out, int mode, int iters, int nw) {
  extern __shared__ uint8_t smem[];
  __shared__ SrvShared sh;
  SrvCtx c;
  c.clog2 = 0;
  c.rt = reinterpret_cast<uint64_t*>(smem);
  c.evmax = reinterpret_cast<uint32_t*>(c.rt + 4 * 4096);
  c.sh = c.sh0 = &sh;
  for (int i = threadIdx.x; i < 4 * 4096; i += blockDim.x) c.rt[i] = 0xFFFFFFFFull;
  for (int i = threadIdx.x; i < 4096; i += blockDim.x) c.evmax[i] = 0;
  if (threadIdx.x == 0) sh.tail = sh.next_ticket = sh.now_serving = 0;
  __syncthreads();
  const uint32_t warp = threadIdx.x / 32;
  if (warp >= (uint32_t)nw) return;
  const uint32_t lane = threadIdx.x & 31, lt = lanemask_lt();
  uint32_t key = (warp * 32 + lane) * 2654435761u + 12345u, t = 100;
  uint32_t sink = 0;
  const long long a0 = clock64();
  long long acc = 0;
  for (int it = 0; it < iters; ++it) {
    key = key * 1664525u + 1013904223u;
    const uint32_t id0 = key >> 12, id1 = (key * 747796405u) >> 12;
    const uint32_t b0 = rt_bucket(id0, 12), b1 = rt_bucket(id1, 12);
    const bool mine = lane < 29;
    uint32_t ticket = 0;
    const bool locked = mode >= 4;
    if (locked) {
      ticket = cs_enter<false>(c);
      t = *(volatile uint32_t*)&sh.tail;
    }
    const long long a = clock64();
    const uint32_t s = t > 50 ? t - 50 : 0, e_pre = t;
    RtProbe q0{0, false, false}, q1{0, false, false};
    if (mode >= 1 && mine) {
      q0 = rt_probe<false>(c, b0, id0, s, e_pre, 0);
      q1 = rt_probe<false>(c, b1, id1, s, e_pre, 0);
      if (b1 == b0 && q1.way == q0.way) q1.way = (q1.way + 1) & 3;
    }
    const bool commit = mine && !q0.conflict && !q1.conflict && !q0.unknown && !q1.unknown;
    const uint32_t cm = __ballot_sync(0xFFFFFFFFu, commit);
    const uint32_t cts = t + 1 + __popc(cm & lt);
    t += __popc(cm);
    if (commit && mode >= 3 && mode != 5) {
      lastw[id0 & 0xFFFFF] = cts;
      lastw[id1 & 0xFFFFF] = cts;
    }
    if (commit && mode >= 2) {
      rt_record<false>(c, b0, q0.way, id0, cts);
      rt_record<false>(c, b1, q1.way, id1, cts);
    }
    __syncwarp();
    acc += clock64() - a;
    if (locked) cs_leave<false>(c, ticket, t);
    sink += cm;
  }
  const long long a1 = clock64();
  if (lane == 0 && warp == 0) {
    out[0] = mode >= 4 ? (a1 - a0) / ((long long)iters * nw) : acc / iters;
    out[1] = acc / iters;
    out[2] = sink;
  }
}

int main() {
  uint32_t* lw;
  unsigned long long* o;
  cudaMalloc(&lw, 4 << 20);
  cudaMallocManaged(&o, 64);
  const int smem = 4 * 4096 * 8 + 4096 * 4;
  cudaFuncSetAttribute(bench, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
  const char* names[] = {"ballot only", "probe", "probe+record", "probe+record+lastw"};
  for (int m = 0; m < 4; ++m) {
    bench<<<1, 256, smem>>>(lw, o, m, 20000, 1);
    cudaDeviceSynchronize();
    printf("%-22s %llu cycles/batch\n", names[m], o[0]);
  }
  for (int nw = 1; nw <= 8; nw *= 2) {
    bench<<<1, 256, smem>>>(lw, o, 4, 20000, nw);
    cudaDeviceSynchronize();
    printf("locked chain, %d warps: %llu cycles/batch (body %llu)\n", nw, o[0], o[1]);
    bench<<<1, 256, smem>>>(lw, o, 5, 20000, nw);
    cudaDeviceSynchronize();
    printf("locked chain, no lastw stores, %d warps: %llu cycles/batch (body %llu)\n", nw, o[0], o[1]);
  }
  printf("err=%s\n", cudaGetErrorString(cudaGetLastError()));
}
