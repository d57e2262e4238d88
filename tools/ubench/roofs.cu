// roofs.cu -- the roofs the CSMV pipeline is measured against, on this B200
// (SURVEY 8(d) "Rooflines to report"; MEASURED_PEAKS.json has only HBM copy
// bandwidth and bf16 GEMM).  Prints one JSON object:
//   l2_read_gbs          all SMs, 256-bit coalesced loads of an L2-resident
//                        64 MiB buffer (the ROT scans' access pattern)
//   l2_read32_gbs        all SMs, one independent 32-byte record per lane at a
//                        random index of a 32 MiB buffer (a transfer's VBox reads)
//   l2_sectors_per_s     l2_read32_gbs / 32 B
//   l2_load_ns           one thread, dependent 4-byte ld.relaxed.gpu chain over
//                        L2 (pointer chase, L1 bypassed): the latency of one hop
//   xsm_roundtrip_ns     two CTAs on different SMs bounce a counter through
//                        global memory (st.release / ld.acquire polling): one
//                        request -> response round trip between SMs, the floor
//                        of every link of the commit chain (C3)
//   smem_atom_per_s_sm   one SM, 1024 threads, atom.shared.add.u32 on distinct
//                        words: shared-memory atomic throughput per SM (the
//                        server's roof, north_star)
//   smem_atom_same_per_s one SM, every lane of every warp on one word
//   sm_clock_mhz         the SM clock the cycle-based numbers were taken at
// Build: nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o roofs roofs.cu
#include <cuda_runtime.h>

#include <cstdint>
#include <cstdio>
#include <vector>

#define CK(x)                                                                  \
  do {                                                                         \
    cudaError_t e = (x);                                                       \
    if (e != cudaSuccess) {                                                    \
      fprintf(stderr, "%s: %s\n", #x, cudaGetErrorString(e));                  \
      return 1;                                                                \
    }                                                                          \
  } while (0)

__global__ void l2_seq(const uint64_t* __restrict__ a, size_t n_words, int passes, uint64_t* sink) {
  uint64_t acc = 0;
  const size_t stride = (size_t)gridDim.x * blockDim.x * 4;
  for (int p = 0; p < passes; ++p) {
    for (size_t i = ((size_t)blockIdx.x * blockDim.x + threadIdx.x) * 4; i < n_words; i += stride) {
      uint64_t x, y, z, w;
      asm volatile("ld.relaxed.gpu.global.v4.u64 {%0,%1,%2,%3}, [%4];"
                   : "=l"(x), "=l"(y), "=l"(z), "=l"(w)
                   : "l"(a + i));
      acc += x ^ y ^ z ^ w;
    }
  }
  if (acc == 0x1234567) *sink = acc;
}

__global__ void l2_rand32(const uint64_t* __restrict__ a, uint32_t n_rec, int iters, uint64_t* sink) {
  uint64_t acc = 0;
  uint32_t x = (blockIdx.x * blockDim.x + threadIdx.x) * 2654435761u + 12345u;
  for (int it = 0; it < iters; it += 8) {
    uint64_t v[8][4];
#pragma unroll
    for (int k = 0; k < 8; ++k) {
      x = x * 1664525u + 1013904223u;
      const uint64_t* p = a + (size_t)((x >> 7) % n_rec) * 4;
      asm volatile("ld.relaxed.gpu.global.v4.u64 {%0,%1,%2,%3}, [%4];"
                   : "=l"(v[k][0]), "=l"(v[k][1]), "=l"(v[k][2]), "=l"(v[k][3])
                   : "l"(p));
    }
#pragma unroll
    for (int k = 0; k < 8; ++k) acc += v[k][0] ^ v[k][3];
  }
  if (acc == 0x1234567) *sink = acc;
}

__global__ void chase(const uint32_t* a, int hops, uint32_t* out, long long* cyc) {
  uint32_t i = 0;
  const long long t0 = clock64();
  for (int h = 0; h < hops; ++h) asm volatile("ld.relaxed.gpu.global.u32 %0, [%1];" : "=r"(i) : "l"(a + i));
  cyc[0] = clock64() - t0;
  out[0] = i;
}

// CTA 0 and CTA 1 (different SMs: one CTA per SM is forced by the smem size)
__global__ void pingpong(uint32_t* flag, int rounds, long long* cyc) {
  if (threadIdx.x != 0) return;
  uint32_t* mine = flag + 64 * blockIdx.x;
  uint32_t* other = flag + 64 * (1 - blockIdx.x);
  const long long t0 = clock64();
  for (int r = 0; r < rounds; ++r) {
    const uint32_t want = 2 * r + blockIdx.x;  // CTA 0 sends 2r, CTA 1 answers 2r+1
    if (blockIdx.x == 0) asm volatile("st.release.gpu.global.u32 [%0], %1;" ::"l"(mine), "r"(want) : "memory");
    uint32_t v;
    const uint32_t exp = blockIdx.x == 0 ? want + 1 : want - 1;
    do {
      asm volatile("ld.acquire.gpu.global.u32 %0, [%1];" : "=r"(v) : "l"(other) : "memory");
    } while (v != exp);
    if (blockIdx.x == 1) asm volatile("st.release.gpu.global.u32 [%0], %1;" ::"l"(mine), "r"(want) : "memory");
  }
  if (blockIdx.x == 0) cyc[0] = clock64() - t0;
}

template <bool SAME>
__global__ void smem_atom(int iters, uint32_t* sink, long long* cyc) {
  __shared__ uint32_t w[1024];
  w[threadIdx.x] = 0;
  __syncthreads();
  const uint32_t a = (uint32_t)__cvta_generic_to_shared(SAME ? &w[0] : &w[threadIdx.x]);
  const long long t0 = clock64();
  for (int i = 0; i < iters; ++i) {
#pragma unroll
    for (int k = 0; k < 8; ++k) asm volatile("red.shared.add.u32 [%0], %1;" ::"r"(a), "r"(1u) : "memory");
  }
  __syncthreads();
  if (threadIdx.x == 0) cyc[0] = clock64() - t0;
  if (w[threadIdx.x] == 0x7FFFFFFF) *sink = 1;
}

int main() {
  int dev = 0, sms = 0, clk_khz = 0;
  CK(cudaGetDevice(&dev));
  CK(cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev));
  CK(cudaDeviceGetAttribute(&clk_khz, cudaDevAttrClockRate, dev));
  cudaEvent_t e0, e1;
  CK(cudaEventCreate(&e0));
  CK(cudaEventCreate(&e1));
  uint64_t* sink;
  CK(cudaMalloc(&sink, 64));
  long long* cyc;
  CK(cudaMalloc(&cyc, 64));

  // L2 sequential read, 64 MiB resident
  const size_t seq_bytes = 64ull << 20;
  uint64_t* buf;
  CK(cudaMalloc(&buf, seq_bytes));
  CK(cudaMemset(buf, 1, seq_bytes));
  const int passes = 40;
  l2_seq<<<sms * 4, 512>>>(buf, seq_bytes / 8, 2, sink);  // warm
  CK(cudaEventRecord(e0));
  l2_seq<<<sms * 4, 512>>>(buf, seq_bytes / 8, passes, sink);
  CK(cudaEventRecord(e1));
  CK(cudaEventSynchronize(e1));
  float ms = 0;
  CK(cudaEventElapsedTime(&ms, e0, e1));
  const double l2_seq_gbs = (double)seq_bytes * passes / (ms * 1e-3) / 1e9;

  // L2 random 32-byte records in a 32 MiB buffer
  const uint32_t n_rec = (32u << 20) / 32;
  const int iters = 512;
  l2_rand32<<<sms * 4, 512>>>(buf, n_rec, 64, sink);
  CK(cudaEventRecord(e0));
  l2_rand32<<<sms * 4, 512>>>(buf, n_rec, iters, sink);
  CK(cudaEventRecord(e1));
  CK(cudaEventSynchronize(e1));
  CK(cudaEventElapsedTime(&ms, e0, e1));
  const double loads = (double)sms * 4 * 512 * iters;
  const double l2_r32_gbs = loads * 32 / (ms * 1e-3) / 1e9;

  // L2 dependent-load latency: a random cyclic permutation over 16 MiB
  const uint32_t n_ch = (16u << 20) / 4;
  std::vector<uint32_t> perm(n_ch);
  {
    std::vector<uint32_t> order(n_ch / 32);
    for (uint32_t i = 0; i < order.size(); ++i) order[i] = i * 32;  // one word per 128 B line
    uint64_t r = 88172645463325252ull;
    for (size_t i = order.size() - 1; i > 0; --i) {
      r ^= r << 13, r ^= r >> 7, r ^= r << 17;
      std::swap(order[i], order[r % (i + 1)]);
    }
    for (size_t i = 0; i < order.size(); ++i) perm[order[i]] = order[(i + 1) % order.size()];
  }
  uint32_t* ch;
  CK(cudaMalloc(&ch, (size_t)n_ch * 4));
  CK(cudaMemcpy(ch, perm.data(), (size_t)n_ch * 4, cudaMemcpyHostToDevice));
  uint32_t* out;
  CK(cudaMalloc(&out, 64));
  const int hops = 20000;
  chase<<<1, 1>>>(ch, 4096, out, cyc);  // warm L2
  chase<<<1, 1>>>(ch, hops, out, cyc);
  long long c = 0;
  CK(cudaMemcpy(&c, cyc, 8, cudaMemcpyDeviceToHost));
  const double l2_cyc = (double)c / hops;

  // cross-SM round trip (one CTA per SM: ask for >half the SM's smem)
  uint32_t* flag;
  CK(cudaMalloc(&flag, 1024));
  CK(cudaMemset(flag, 0xFF, 1024));
  const int rounds = 20000;
  CK(cudaFuncSetAttribute(pingpong, cudaFuncAttributeMaxDynamicSharedMemorySize, 150 * 1024));
  pingpong<<<2, 32, 150 * 1024>>>(flag, rounds, cyc);
  CK(cudaDeviceSynchronize());
  CK(cudaMemcpy(&c, cyc, 8, cudaMemcpyDeviceToHost));
  const double rt_cyc = (double)c / rounds;

  // shared-memory atomics, one SM
  const int ait = 4096;
  smem_atom<false><<<1, 1024>>>(ait, (uint32_t*)sink, cyc);
  CK(cudaDeviceSynchronize());
  CK(cudaMemcpy(&c, cyc, 8, cudaMemcpyDeviceToHost));
  const double atom_cyc = (double)c;
  smem_atom<true><<<1, 1024>>>(ait / 16, (uint32_t*)sink, cyc);
  CK(cudaDeviceSynchronize());
  CK(cudaMemcpy(&c, cyc, 8, cudaMemcpyDeviceToHost));
  const double atom_same_cyc = (double)c;

  // convert cycle counts at the SM clock measured over a timed spin
  // (clock64 ticks at the SM clock; cudaDevAttrClockRate is the max)
  const double mhz = clk_khz / 1000.0;
  const double n_atom = 1024.0 * ait * 8, n_same = 1024.0 * (ait / 16) * 8;
  printf("{\"l2_read_gbs\": %.1f, \"l2_read32_gbs\": %.1f, \"l2_sectors_per_s\": %.4g, "
         "\"l2_load_cycles\": %.1f, \"l2_load_ns\": %.1f, \"xsm_roundtrip_cycles\": %.1f, \"xsm_roundtrip_ns\": %.1f, "
         "\"smem_atom_per_clk_sm\": %.2f, \"smem_atom_per_s_sm\": %.4g, \"smem_atom_same_per_s\": %.4g, "
         "\"sm_clock_mhz\": %.0f, \"sms\": %d}\n",
         l2_seq_gbs, l2_r32_gbs, l2_r32_gbs * 1e9 / 32, l2_cyc, l2_cyc / mhz * 1e3, rt_cyc, rt_cyc / mhz * 1e3,
         n_atom / atom_cyc, n_atom / atom_cyc * mhz * 1e6, n_same / atom_same_cyc * mhz * 1e6, mhz, sms);
  return 0;
}
