// fused_bank_cl.cu -- instantiation of the fused kernel for the bank workload
// with the thread-block-cluster server (fused.cuh).
#include "fused.cuh"

namespace csmvd {

cudaError_t launch_fused_bank_cl(const KParams& p, uint32_t nslot, uint32_t grid, size_t smem, cudaStream_t st,
                                 int* occ) {
  return launch_kind<CSMV_KIND_BANK, true>(p, nslot, grid, smem, st, occ);
}

}  // namespace csmvd
