// Does a cooperative launch compose with cluster dimensions on this driver?
#include <cstdio>
#include <cooperative_groups.h>
namespace cg = cooperative_groups;
__global__ void k(int* out) {
  extern __shared__ int sm[];
  cg::cluster_group cl = cg::this_cluster();
  sm[0] = blockIdx.x;
  cl.sync();
  int* remote = cl.map_shared_rank(sm, (cl.block_rank() + 1) % cl.num_blocks());
  if (threadIdx.x == 0) {
    out[blockIdx.x] = remote[0];
    atomicAdd(remote + 1, 1);
  }
  cl.sync();
}
int main() {
  int* d; cudaMalloc(&d, 4096 * 4);
  for (int cs : {2, 4, 8, 16}) {
    cudaFuncSetAttribute(k, cudaFuncAttributeNonPortableClusterSizeAllowed, 1);
    cudaFuncSetAttribute(k, cudaFuncAttributeMaxDynamicSharedMemorySize, 150 * 1024);
    cudaLaunchConfig_t cfg = {};
    cudaLaunchAttribute at[2];
    at[0].id = cudaLaunchAttributeClusterDimension; at[0].val.clusterDim.x = cs; at[0].val.clusterDim.y = 1; at[0].val.clusterDim.z = 1;
    at[1].id = cudaLaunchAttributeCooperative; at[1].val.cooperative = 1;
    cfg.blockDim = dim3(256); cfg.dynamicSmemBytes = 150 * 1024; cfg.attrs = at; cfg.numAttrs = 2;
    int ncl = 0;
    cfg.gridDim = dim3(cs);
    cudaOccupancyMaxActiveClusters(&ncl, k, &cfg);
    cfg.gridDim = dim3(cs * ncl);
    cudaError_t e = cudaLaunchKernelEx(&cfg, k, d);
    cudaError_t e2 = cudaDeviceSynchronize();
    printf("cluster %2d: max active clusters %d (%d CTAs) coop launch: %s / %s\n", cs, ncl, cs * ncl,
           cudaGetErrorString(e), cudaGetErrorString(e2));
    cudaGetLastError();
  }
}
