// Cycles of the KV warp-cooperative PUT read's evaluation (client_kv.cuh
// kv_put_read_eval) on an idle SM: one warp, a 16-way set of 4-version key
// rings in HBM/L2, the loads forced before the clock starts.
//   nvcc -gencode arch=compute_100a,code=sm_100a -O3 -std=c++17 -I include -o coop_ubench tools/ubench/coop_ubench.cu
#include <cstdio>
#include <vector>
#include "../../paper_conf_ipps_nunesc022_b200/csrc/fused.cuh"

using namespace csmvd;

__global__ void bench(KParams p, uint32_t t, uint32_t key, uint32_t s, int iters, unsigned long long* out) {
  uint32_t kk[4];
  kv_key16(key, kk);
  unsigned long long tot = 0, ld_tot = 0;
  uint32_t sink = 0;
  for (int it = 0; it < iters; ++it) {
    const long long a = clock64();
    KvCoopLd<4> ld;
    kv_put_read_issue<4>(p, t, ld);
    uint64_t x = ld.cr.s[0];
    for (int j = 0; j < 4; ++j) x ^= ld.kr[j].s[0] ^ ld.kr[j].s[3];
    x = __reduce_or_sync(0xFFFFFFFFu, (uint32_t)x);
    const long long b = clock64();
    int st, iv, ic;
    uint32_t seen, vic, clk;
    uint64_t dg;
    kv_put_read_eval<4>(p, s + (x == 7u), t, kk, ld, st, seen, vic, iv, ic, clk, dg);
    sink += st + seen + vic + iv + ic + clk + (uint32_t)dg;
    sink = __reduce_add_sync(0xFFFFFFFFu, sink);
    const long long c = clock64();
    ld_tot += b - a;
    tot += c - b;
  }
  if (threadIdx.x == 0) {
    out[0] = ld_tot / iters;
    out[1] = tot / iters;
    out[2] = sink;
  }
}

int main() {
  const uint32_t S = 1u << 12, A = 16, T = S / A, NS = 4;
  KParams p;
  memset(&p, 0, sizeof p);
  p.K = 4;
  p.kv_S = S;
  p.kv_A = A;
  p.kv_T = T;
  std::vector<uint64_t> key(S * NS * 4, (uint64_t)kEmptyTs << 32), clk(T * NS, (uint64_t)kEmptyTs << 32),
      lru(S * NS, (uint64_t)kEmptyTs << 32);
  // set 7 holds keys 100..115 at ts 0; the PUT's key is 108 (way 8)
  const uint32_t t = 7;
  for (uint32_t w = 0; w < A; ++w) {
    uint32_t kk[4];
    const uint64_t a = mix64((uint64_t)(100 + w)), b = mix64((uint64_t)(100 + w) ^ 0x5555555555555555ull);
    kk[0] = (uint32_t)a, kk[1] = (uint32_t)(a >> 32), kk[2] = (uint32_t)b, kk[3] = (uint32_t)(b >> 32);  // kv_key16
    for (int x = 0; x < 4; ++x) key[((size_t)(t * A + w) * NS + 0) * 4 + x] = kk[x];
    lru[(size_t)(t * A + w) * NS] = w;
  }
  clk[t * NS] = 0;
  uint64_t *dk, *dc, *dl;
  unsigned long long* dout;
  cudaMalloc(&dk, key.size() * 8);
  cudaMalloc(&dc, clk.size() * 8);
  cudaMalloc(&dl, lru.size() * 8);
  cudaMalloc(&dout, 24);
  cudaMemcpy(dk, key.data(), key.size() * 8, cudaMemcpyHostToDevice);
  cudaMemcpy(dc, clk.data(), clk.size() * 8, cudaMemcpyHostToDevice);
  cudaMemcpy(dl, lru.data(), lru.size() * 8, cudaMemcpyHostToDevice);
  p.kv_key = dk;
  p.kv_clk = dc;
  p.kv_lru = dl;
  for (uint32_t lm = 0; lm < 2; ++lm) {
    p.log_mode = lm;
    bench<<<1, 32>>>(p, t, 108, 5, 1000, dout);
    unsigned long long h[3];
    cudaMemcpy(h, dout, 24, cudaMemcpyDeviceToHost);
    printf("{\"log_mode\": %u, \"load_cycles\": %llu, \"eval_cycles\": %llu}\n", lm, h[0], h[1]);
  }
  return 0;
}
