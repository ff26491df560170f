// k_dupcmp.cu -- the on-device output comparison of kernel-level duplication
// (variant dup_kernel; "entire kernel launches
// can be duplicated into primary and secondary kernels, and the resulting
// output can be compared").  The two replicas wrote shadow copies a and b; this
// kernel commits every aligned 4-word group on which they agree to `out` and
// counts the groups that differ (the same granularity as the RMT variants'
// vector commits).  Grid-stride, 16-B vectors, one atomic per warp with
// mismatches.
#include "rmt_host.cuh"

namespace rmt {
namespace {

__global__ void __launch_bounds__(256) dup_compare_kernel(const unsigned* a, const unsigned* b, unsigned* out,
                                                          unsigned long long nwords, unsigned long long* err) {
  const unsigned long long ngroups = (nwords + 3) / 4;
  const unsigned long long stride = (unsigned long long)gridDim.x * blockDim.x;
  for (unsigned long long g0 = 0; g0 < ngroups; g0 += stride) {
    const unsigned long long g = g0 + (unsigned long long)blockIdx.x * blockDim.x + threadIdx.x;
    bool mism = false;
    if (g < ngroups) {
      const unsigned long long w0 = 4 * g;
      if (w0 + 4 <= nwords) {
        const uint4 x = __ldcs(reinterpret_cast<const uint4*>(a) + g);
        const uint4 y = __ldcs(reinterpret_cast<const uint4*>(b) + g);
        mism = ((x.x ^ y.x) | (x.y ^ y.y) | (x.z ^ y.z) | (x.w ^ y.w)) != 0u;
        if (!mism) __stcs(reinterpret_cast<uint4*>(out) + g, x);
      } else {
        unsigned d = 0;
        for (unsigned long long w = w0; w < nwords; ++w) d |= a[w] ^ b[w];
        mism = d != 0u;
        if (!mism)
          for (unsigned long long w = w0; w < nwords; ++w) out[w] = a[w];
      }
    }
    const unsigned m = __ballot_sync(0xffffffffu, mism);
    if (m != 0u && (threadIdx.x & 31) == (unsigned)(__ffs(m) - 1)) atomicAdd(err, (unsigned long long)__popc(m));
  }
}

}  // namespace

int dup_compare_launch(const void* a, const void* b, void* out, unsigned long long nwords, unsigned long long* err,
                       cudaStream_t s) {
  if (nwords == 0) return RMT_OK;
  const unsigned long long groups = (nwords + 3) / 4;
  unsigned long long blocks = (groups + 255) / 256;
  if (blocks > 148ull * 16) blocks = 148ull * 16;
  dup_compare_kernel<<<(unsigned)blocks, 256, 0, s>>>((const unsigned*)a, (const unsigned*)b, (unsigned*)out, nwords,
                                                      err);
  return cuda_check(cudaGetLastError(), "dup_compare");
}

}  // namespace rmt
