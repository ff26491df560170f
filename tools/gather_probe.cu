// gather_probe.cu -- random-block gather microbenchmark (B200): the time and
// the DRAM traffic of 2^24 random aligned G-byte block reads from a 1 GiB array
// (>> L2), for G = 16, 32, 64, 128 and several load flavours (cache operator /
// L1 policy).  Informs the BinarySearch bottom-level block read: a random miss
// can move a whole 128-B line from DRAM whatever G is.  Build + run (ncu adds
// dram__bytes_read.sum and the L2 sector counts per launch):
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

enum { L_CS = 0, L_CG = 1, L_NC = 2, L_NA = 3, L_RLX = 4, L_CG_NA = 5 };

template <int F>
__device__ __forceinline__ uint4 ld16(const uint4* p) {
  uint4 w;
  if constexpr (F == L_CS) {
    w = __ldcs(p);
  } else if constexpr (F == L_CG) {
    w = __ldcg(p);
  } else if constexpr (F == L_NC) {
    w = __ldg(p);
  } else if constexpr (F == L_NA) {
    asm volatile("ld.global.nc.L1::no_allocate.v4.u32 {%0,%1,%2,%3}, [%4];" : "=r"(w.x), "=r"(w.y), "=r"(w.z), "=r"(w.w) : "l"(p));
  } else if constexpr (F == L_RLX) {
    asm volatile("ld.relaxed.gpu.global.v4.u32 {%0,%1,%2,%3}, [%4];" : "=r"(w.x), "=r"(w.y), "=r"(w.z), "=r"(w.w) : "l"(p));
  } else {
    asm volatile("ld.global.nc.L1::no_allocate.L2::64B.v4.u32 {%0,%1,%2,%3}, [%4];" : "=r"(w.x), "=r"(w.y), "=r"(w.z), "=r"(w.w) : "l"(p));
  }
  return w;
}

// G/16 lanes per block, one 16-B load each
template <int G, int F>
__global__ void gather(const uint4* __restrict__ a, size_t nblocks, unsigned nreq, unsigned* out) {
  const unsigned tid = blockIdx.x * blockDim.x + threadIdx.x;
  constexpr int LPB = G / 16;
  const unsigned req = tid / LPB, sub = tid % LPB;
  if (req >= nreq) return;
  const size_t blk = mix(req) % nblocks;
  uint4 w = ld16<F>(a + blk * LPB + sub);
  unsigned v = w.x ^ w.y ^ w.z ^ w.w;
  if (v == 0x12345678u) out[0] = v;  // keep the load
}

static const char* fname[] = {"ld.cs", "ld.cg", "ld.nc", "ld.nc.L1::no_allocate", "ld.relaxed.gpu", "ld.nc.L1::no_alloc.L2::64B"};

template <int G, int F>
void run(const uint4* a, size_t bytes, unsigned* out) {
  const size_t nblocks = bytes / G;
  const unsigned nreq = 1u << 24;
  constexpr int LPB = G / 16;
  const unsigned threads = nreq * LPB;
  cudaEvent_t e0, e1;
  cudaEventCreate(&e0);
  cudaEventCreate(&e1);
  for (int w = 0; w < 2; ++w) gather<G, F><<<(threads + 255) / 256, 256>>>(a, nblocks, nreq, out);
  float best = 1e9f;
  for (int r = 0; r < 5; ++r) {
    cudaEventRecord(e0);
    gather<G, F><<<(threads + 255) / 256, 256>>>(a, nblocks, nreq, out);
    cudaEventRecord(e1);
    cudaEventSynchronize(e1);
    float ms;
    cudaEventElapsedTime(&ms, e0, e1);
    if (ms < best) best = ms;
  }
  printf("G=%3d %-24s %u random blocks in %.3f ms = %.1f Mblk/s, useful %.1f GB/s\n", G, fname[F], nreq, best,
         nreq / best / 1e3, (double)nreq * G / best / 1e6);
}

template <int F>
void all(const uint4* a, size_t bytes, unsigned* out) {
  run<16, F>(a, bytes, out);
  run<32, F>(a, bytes, out);
  run<64, F>(a, bytes, out);
}

int main() {
  const size_t bytes = 1ull << 30;
  uint4* a;
  unsigned* out;
  cudaMalloc(&a, bytes);
  cudaMalloc(&out, 4);
  cudaMemset(a, 1, bytes);
  all<L_CS>(a, bytes, out);
  all<L_CG>(a, bytes, out);
  all<L_NC>(a, bytes, out);
  all<L_NA>(a, bytes, out);
  all<L_RLX>(a, bytes, out);
  all<L_CG_NA>(a, bytes, out);
  run<128, L_CS>(a, bytes, out);
  return 0;
}
