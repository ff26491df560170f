// gather_probe.cu -- random-block gather microbenchmark (B200): how many DRAM
// bytes and how much time a random G-byte aligned block read costs, for
// G = 4, 16, 32, 64, 128, from a 1 GiB array (>> L2).  Informs the
// BinarySearch bottom-level block size.  Build + run:
//   nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o /tmp/gp tools/gather_probe.cu && /tmp/gp
#include <cstdio>
#include <cstdint>
#include <cuda_runtime.h>

__device__ __forceinline__ uint32_t mix(uint64_t x) {
  x += 0x9E3779B97F4A7C15ull;
  x = (x ^ (x >> 30)) * 0xBF58476D1CE4E5B9ull;
  x = (x ^ (x >> 27)) * 0x94D049BB133111EBull;
  return (uint32_t)(x ^ (x >> 31));
}

// G/16 lanes per block (G >= 16), one 16-B load each; G = 4: one 4-B load per lane
template <int G>
__global__ void gather(const uint4* __restrict__ a, size_t nblocks, unsigned nreq, unsigned* out) {
  const unsigned tid = blockIdx.x * blockDim.x + threadIdx.x;
  constexpr int LPB = G >= 16 ? G / 16 : 1;
  const unsigned req = tid / LPB, sub = tid % LPB;
  if (req >= nreq) return;
  const size_t blk = mix(req) % nblocks;
  unsigned v;
  if constexpr (G >= 16) {
    uint4 w = __ldcs(a + blk * LPB + sub);
    v = w.x ^ w.y ^ w.z ^ w.w;
  } else {
    v = __ldcs(reinterpret_cast<const unsigned*>(a) + blk);
  }
  if (v == 0x12345678u) out[0] = v;  // keep the load
}

template <int G>
void run(const uint4* a, size_t bytes, unsigned* out) {
  const size_t nblocks = bytes / G;
  const unsigned nreq = 1u << 24;
  constexpr int LPB = G >= 16 ? G / 16 : 1;
  const unsigned threads = nreq * LPB;
  cudaEvent_t e0, e1;
  cudaEventCreate(&e0);
  cudaEventCreate(&e1);
  for (int w = 0; w < 3; ++w) gather<G><<<(threads + 255) / 256, 256>>>(a, nblocks, nreq, out);
  float best = 1e9f;
  for (int r = 0; r < 10; ++r) {
    cudaEventRecord(e0);
    gather<G><<<(threads + 255) / 256, 256>>>(a, nblocks, nreq, out);
    cudaEventRecord(e1);
    cudaEventSynchronize(e1);
    float ms;
    cudaEventElapsedTime(&ms, e0, e1);
    if (ms < best) best = ms;
  }
  printf("G=%3d B: %u random blocks in %.3f ms = %.1f Mblk/s, useful %.1f GB/s\n", G, nreq, best,
         nreq / best / 1e3, (double)nreq * G / best / 1e6);
}

int main() {
  const size_t bytes = 1ull << 30;
  uint4* a;
  unsigned* out;
  cudaMalloc(&a, bytes);
  cudaMalloc(&out, 4);
  cudaMemset(a, 1, bytes);
  run<4>(a, bytes, out);
  run<16>(a, bytes, out);
  run<32>(a, bytes, out);
  run<64>(a, bytes, out);
  run<128>(a, bytes, out);
  return 0;
}
