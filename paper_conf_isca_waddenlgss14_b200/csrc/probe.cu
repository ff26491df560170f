// probe.cu -- where does the hardware place the two CTAs of an inter_cluster
// pair?  SURVEY 8(f) rank 3: if the pair always sits on two different SMs, the
// SM's L1 / LSU / scheduler are inside inter_cluster's sphere of replication
// (the paper's Inter-Group caveat P:677 is that the pair MAY share a CU).
#include "rmt_host.cuh"

namespace rmt {
namespace {

__global__ void smid_kernel(unsigned* out) {
  if (threadIdx.x == 0) {
    unsigned smid;
    asm volatile("mov.u32 %0, %%smid;" : "=r"(smid));
    out[blockIdx.x] = smid;
  }
}

}  // namespace
}  // namespace rmt

using namespace rmt;

extern "C" int rmt_probe_cluster_placement(int64_t pairs, int64_t* same_sm_pairs) {
  if (pairs <= 0 || pairs > (1 << 24) || !same_sm_pairs) {
    set_error("rmt_probe_cluster_placement: pairs in [1, 2^24], non-NULL output");
    return RMT_EINVAL;
  }
  unsigned* d = nullptr;
  int rc = cuda_check(cudaMalloc(&d, (size_t)pairs * 2 * sizeof(unsigned)), "probe malloc");
  if (rc) return rc;
  cudaLaunchConfig_t cfg = {};
  cfg.gridDim = dim3((unsigned)(2 * pairs));
  cfg.blockDim = dim3(256);
  cudaLaunchAttribute at[1];
  at[0].id = cudaLaunchAttributeClusterDimension;
  at[0].val.clusterDim.x = 2;
  at[0].val.clusterDim.y = 1;
  at[0].val.clusterDim.z = 1;
  cfg.attrs = at;
  cfg.numAttrs = 1;
  rc = cuda_check(cudaLaunchKernelEx(&cfg, smid_kernel, d), "probe launch");
  if (!rc) rc = cuda_check(cudaDeviceSynchronize(), "probe sync");
  unsigned* h = nullptr;
  if (!rc) {
    h = new unsigned[2 * pairs];
    rc = cuda_check(cudaMemcpy(h, d, (size_t)pairs * 2 * sizeof(unsigned), cudaMemcpyDeviceToHost), "probe D2H");
  }
  if (!rc) {
    int64_t same = 0;
    for (int64_t p = 0; p < pairs; ++p) same += h[2 * p] == h[2 * p + 1];
    *same_sm_pairs = same;
  }
  delete[] h;
  cudaFree(d);
  return rc;
}
