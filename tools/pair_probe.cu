// pair_probe.cu — where does the hardware place the two CTAs of a 2-CTA cluster when two CTAs
// fit on one SM?  (Question behind a cta_group::2 prefill-attention kernel with 2 CTAs per SM:
// a CTA pair must sit on the two SMs of one TPC.)  Measurement tool, not product code.
//   nvcc -gencode arch=compute_100a,code=sm_100a -o gpurun_out/pair_probe tools/pair_probe.cu
#include <cstdio>
#include <vector>
#include <cuda_runtime.h>

__global__ void __cluster_dims__(2, 1, 1) __launch_bounds__(192, 2) probe(int* out, int spin) {
  extern __shared__ unsigned char sm[];
  unsigned smid, rank;
  asm volatile("mov.u32 %0, %%smid;" : "=r"(smid));
  asm volatile("mov.u32 %0, %%cluster_ctarank;" : "=r"(rank));
  if (threadIdx.x == 0) {
    sm[0] = 1;
    out[blockIdx.x] = int(smid);
  }
  // keep every CTA resident for a while so the scheduler must co-locate
  long long t0 = clock64();
  while (clock64() - t0 < spin) {}
}

int main() {
  int dev = 0, nsm = 0;
  cudaDeviceGetAttribute(&nsm, cudaDevAttrMultiProcessorCount, dev);
  const int smem = 97 * 1024;
  cudaFuncSetAttribute(probe, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
  int nclusters = 0;
  cudaLaunchConfig_t cfg{};
  cfg.blockDim = dim3(192);
  cfg.dynamicSmemBytes = smem;
  cudaLaunchAttribute attr[1];
  attr[0].id = cudaLaunchAttributeClusterDimension;
  attr[0].val.clusterDim.x = 2;
  attr[0].val.clusterDim.y = 1;
  attr[0].val.clusterDim.z = 1;
  cfg.attrs = attr;
  cfg.numAttrs = 1;
  cfg.gridDim = dim3(2);
  cudaOccupancyMaxActiveClusters(&nclusters, probe, &cfg);
  printf("{\"sms\": %d, \"max_active_clusters\": %d", nsm, nclusters);
  for (int grid : {2 * nclusters, 4 * nsm}) {
    int* d;
    cudaMalloc(&d, grid * sizeof(int));
    cfg.gridDim = dim3(grid);
    cudaLaunchKernelEx(&cfg, probe, d, 2000000);
    cudaError_t e = cudaDeviceSynchronize();
    std::vector<int> h(grid);
    cudaMemcpy(h.data(), d, grid * sizeof(int), cudaMemcpyDeviceToHost);
    int same = 0, tpc = 0, other = 0;
    for (int c = 0; c < grid / 2; ++c) {
      const int a = h[2 * c], b = h[2 * c + 1];
      if (a == b) ++same;
      else if ((a ^ b) == 1) ++tpc;
      else ++other;
    }
    printf(", \"grid_%d\": {\"err\": \"%s\", \"pairs_same_sm\": %d, \"pairs_tpc\": %d, \"pairs_other\": %d, \"first\": [%d, %d, %d, %d]}",
           grid, cudaGetErrorString(e), same, tpc, other, h[0], h[1], h[2], h[3]);
    cudaFree(d);
  }
  printf("}\n");
  return 0;
}
