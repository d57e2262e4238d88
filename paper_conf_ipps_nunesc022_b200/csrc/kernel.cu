// kernel.cu -- host-side launchers: the fused kernel (instantiated in
// fused_*.cu) and the small setup, dump and generator kernels.
#include <cuda_runtime.h>

#include <cub/device/device_scan.cuh>

#include "fused.cuh"
#include "kv_kernels.cuh"

namespace csmvd {

template <int NS>
__global__ void init_rings(uint64_t* rings, const int32_t* init, uint64_t n, uint32_t* gts) {
  const uint64_t i = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x;
  if (i == 0) *gts = 0;
  if (i >= n) return;
  Ring<NS> r;
#pragma unroll
  for (int j = 0; j < NS; ++j) r.s[j] = (uint64_t)kEmptyTs << 32;
  r.s[0] = (uint64_t)(uint32_t)init[i];
  *reinterpret_cast<Ring<NS>*>(rings + i * NS) = r;
}

__global__ void gen_descs_kernel(GenParams g, uint64_t tx0, uint64_t n, uint32_t* out) {
  const uint64_t i = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x;
  if (i >= n) return;
  BankTx d = gen_bank(g, tx0 + i);
  uint32_t* o = out + i * 6;
  o[0] = d.is_update;
  o[1] = d.src;
  o[2] = d.dst;
  o[3] = (uint32_t)d.amt;
  o[4] = d.start;
  o[5] = d.len;
}

static cudaError_t launch_any(const KParams& p, uint32_t nslot, uint32_t grid, size_t smem, cudaStream_t st,
                              int* occ) {
  const bool cl = p.clustered != 0;
  if (p.kind == CSMV_KIND_KV)
    return cl ? launch_fused_kv_cl(p, nslot, grid, smem, st, occ) : launch_fused_kv_cta(p, nslot, grid, smem, st, occ);
  return cl ? launch_fused_bank_cl(p, nslot, grid, smem, st, occ) : launch_fused_bank_cta(p, nslot, grid, smem, st, occ);
}

cudaError_t launch_fused(const KParams& p, uint32_t nslot, uint32_t grid, size_t smem, cudaStream_t st) {
  return launch_any(p, nslot, grid, smem, st, nullptr);
}

cudaError_t fused_capacity(const KParams& p, uint32_t nslot, size_t smem, int* ctas) {
  return launch_any(p, nslot, 0, smem, nullptr, ctas);
}

cudaError_t launch_init_kv(const KParams& p, uint32_t nslot, const uint32_t* keys, const uint32_t* vals,
                           const uint32_t* lru, const uint32_t* clocks, cudaStream_t st) {
  const uint32_t blocks = 148 * 8;
  switch (nslot) {
    case 2: init_kv_rings<2><<<blocks, 256, 0, st>>>(p, keys, vals, lru, clocks); break;
    case 4: init_kv_rings<4><<<blocks, 256, 0, st>>>(p, keys, vals, lru, clocks); break;
    case 8: init_kv_rings<8><<<blocks, 256, 0, st>>>(p, keys, vals, lru, clocks); break;
    case 16: init_kv_rings<16><<<blocks, 256, 0, st>>>(p, keys, vals, lru, clocks); break;
    default: return cudaErrorInvalidValue;
  }
  return cudaGetLastError();
}

cudaError_t launch_kv_preload(uint32_t n_keys, uint32_t T, uint32_t A, uint32_t* scratch, void* cub_tmp,
                              size_t* cub_bytes, uint32_t* keys, uint32_t* vals, uint32_t* lru, uint32_t* clocks,
                              cudaStream_t st) {
  uint32_t *cnt = scratch, *off = scratch + T, *fill = scratch + 2 * (size_t)T, *bucket = scratch + 3 * (size_t)T;
  if (!cub_tmp) return cub::DeviceScan::ExclusiveSum(nullptr, *cub_bytes, cnt, off, (int)T, st);
  if (A == 0 || A > kMaxWays) return cudaErrorInvalidValue;
  cudaError_t e = cudaMemsetAsync(cnt, 0, (size_t)T * 4, st);
  if (e == cudaSuccess) e = cudaMemsetAsync(fill, 0, (size_t)T * 4, st);
  if (e != cudaSuccess) return e;
  const uint32_t grid = 148 * 8;
  kv_preload_count<<<grid, 256, 0, st>>>(n_keys, T, cnt);
  e = cub::DeviceScan::ExclusiveSum(cub_tmp, *cub_bytes, cnt, off, (int)T, st);
  if (e != cudaSuccess) return e;
  kv_preload_scatter<<<grid, 256, 0, st>>>(n_keys, T, off, fill, bucket);
  kv_preload_place<<<(T + 127) / 128, 128, 0, st>>>(T, A, off, cnt, bucket, keys, vals, lru, clocks);
  return cudaGetLastError();
}

cudaError_t launch_kv_newest(const KParams& p, uint32_t nslot, uint32_t* keys, uint32_t* vals, uint32_t* lru,
                             uint32_t* clocks, cudaStream_t st) {
  const uint32_t blocks = (uint32_t)((p.kv_S + 255) / 256);
  switch (nslot) {
    case 2: kv_newest<2><<<blocks, 256, 0, st>>>(p, keys, vals, lru, clocks); break;
    case 4: kv_newest<4><<<blocks, 256, 0, st>>>(p, keys, vals, lru, clocks); break;
    case 8: kv_newest<8><<<blocks, 256, 0, st>>>(p, keys, vals, lru, clocks); break;
    case 16: kv_newest<16><<<blocks, 256, 0, st>>>(p, keys, vals, lru, clocks); break;
    default: return cudaErrorInvalidValue;
  }
  return cudaGetLastError();
}

cudaError_t launch_gen_kv_descs(GenParams g, uint64_t tx0, uint64_t n, uint32_t* out, cudaStream_t st) {
  if (n == 0) return cudaSuccess;
  gen_kv_descs_kernel<<<(uint32_t)((n + 255) / 256), 256, 0, st>>>(g, tx0, n, out);
  return cudaGetLastError();
}

cudaError_t launch_init_rings(uint64_t* rings, uint32_t nslot, const int32_t* init, uint64_t n,
                              uint32_t* gts, cudaStream_t st) {
  const uint32_t blocks = (uint32_t)((n + 255) / 256) + 1;
  switch (nslot) {
    case 2: init_rings<2><<<blocks, 256, 0, st>>>(rings, init, n, gts); break;
    case 4: init_rings<4><<<blocks, 256, 0, st>>>(rings, init, n, gts); break;
    case 8: init_rings<8><<<blocks, 256, 0, st>>>(rings, init, n, gts); break;
    case 16: init_rings<16><<<blocks, 256, 0, st>>>(rings, init, n, gts); break;
    default: return cudaErrorInvalidValue;
  }
  return cudaGetLastError();
}

cudaError_t launch_gen_descs(GenParams g, uint64_t tx0, uint64_t n, uint32_t* out, cudaStream_t st) {
  if (n == 0) return cudaSuccess;
  gen_descs_kernel<<<(uint32_t)((n + 255) / 256), 256, 0, st>>>(g, tx0, n, out);
  return cudaGetLastError();
}

}  // namespace csmvd
