// Floor of the committer's per-batch serial chain on one warp (no other
// warps): filter loads -> commit mask -> CTS -> filter stores, then adding
// the lastw stores, the response stores and the payload loads from a ring.
// Prints cycles per batch for each mode.
#include <cstdio>
#include <cstdint>
#include <cuda_runtime.h>
__device__ __forceinline__ uint32_t lds(uint32_t a) { uint32_t v; asm volatile("ld.shared.u32 %0, [%1];" : "=r"(v) : "r"(a) : "memory"); return v; }
__device__ __forceinline__ void sts(uint32_t a, uint32_t v) { asm volatile("st.shared.u32 [%0], %1;" ::"r"(a), "r"(v) : "memory"); }
__global__ void k(uint32_t* lastw, unsigned long long* resp, unsigned long long* out, int mode, int iters) {
  extern __shared__ uint32_t sm[];
  const uint32_t slots = 1u << 15;
  for (uint32_t i = threadIdx.x; i < slots + 32 * 8 * 32; i += blockDim.x) sm[i] = 0;
  __syncthreads();
  if (threadIdx.x >= 32) return;
  const uint32_t lane = threadIdx.x, lt = (1u << lane) - 1;
  const uint32_t base = (uint32_t)__cvta_generic_to_shared(sm);
  uint4* ring = reinterpret_cast<uint4*>(sm + slots);
  // ring payloads: random slot offsets
  for (int i = 0; i < 32; ++i) {
    uint32_t x = (i * 32 + lane) * 2654435761u + 7u;
    ring[(i * 2) * 32 + lane] = make_uint4(4 * ((x * 0x9E3779B1u) >> 17), 4 * ((x * 0x85EBCA77u) >> 17), 4 * ((x * 0xC2B2AE3Du) >> 17), 4 * (((x + 1) * 0x9E3779B1u) >> 17));
    ring[(i * 2 + 1) * 32 + lane] = make_uint4(4 * (((x + 1) * 0x85EBCA77u) >> 17), 4 * (((x + 1) * 0xC2B2AE3Du) >> 17), x >> 12, (x + 1) >> 12);
  }
  __syncwarp();
  uint32_t t = 0;
  uint4 w0 = ring[lane], w1 = ring[32 + lane];
  const long long c0 = clock64();
  for (int it = 0; it < iters; ++it) {
    if (mode >= 3) {
      const int j = (it + 1) & 31;
      w0 = ring[(2 * j) * 32 + lane];
      w1 = ring[(2 * j + 1) * 32 + lane];
    } else {
      w0.x ^= 4u * (it & 1); 
    }
    const uint32_t v0 = lds(base + w0.x), v1 = lds(base + w0.y), v2 = lds(base + w0.z);
    const uint32_t v3 = lds(base + w0.w), v4 = lds(base + w1.x), v5 = lds(base + w1.y);
    const uint32_t lo = max(min(v0, min(v1, v2)), min(v3, min(v4, v5)));
    const bool ovf = lo > t + 100000u;
    const bool commit = lane < 29 && !ovf;
    const uint32_t cm = __ballot_sync(~0u, commit), om = __ballot_sync(~0u, ovf);
    const uint32_t cts = t + 1 + __popc(cm & lt);
    t += __popc(cm);
    if (commit) {
      sts(base + w0.x, t); sts(base + w0.y, t); sts(base + w0.z, t);
      sts(base + w0.w, t); sts(base + w1.x, t); sts(base + w1.y, t);
      if (mode >= 1) { lastw[w1.z & 0xFFFFF] = cts; lastw[w1.w & 0xFFFFF] = cts; }
    }
    if (mode >= 2 && lane == 0) {
      resp[(it & 255) * 4] = cm; resp[(it & 255) * 4 + 1] = om; resp[(it & 255) * 4 + 2] = t;
    }
    __syncwarp();
  }
  const long long c1 = clock64();
  if (lane == 0) out[mode] = (unsigned long long)(c1 - c0) / iters + 0 * t;
}
int main() {
  uint32_t* lastw; unsigned long long *resp, *out;
  cudaMalloc(&lastw, 4 << 20); cudaMalloc(&resp, 8 * 4 * 256); cudaMalloc(&out, 64);
  const size_t sm = (32768 + 32 * 8 * 32) * 4;
  cudaFuncSetAttribute(k, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)sm);
  const char* names[] = {"filter chain", "+ lastw stores", "+ response stores", "+ ring payload loads"};
  for (int mode = 0; mode < 4; ++mode) {
    k<<<1, 256, sm>>>(lastw, resp, out, mode, 100000);
    unsigned long long h = 0;
    cudaMemcpy(&h, out + mode, 8, cudaMemcpyDeviceToHost);
    printf("mode %d %-22s %llu cycles/batch (%s)\n", mode, names[mode], h, cudaGetErrorString(cudaGetLastError()));
  }
}
