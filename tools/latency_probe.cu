// latency_probe.cu -- B200 microbenchmarks behind the Inter-Group cost analysis
// ("L2-bandwidth and atomicAdd / ld.acquire latency
// microbenchmarks").  Measures, with clock64 inside one
// warp (latency) or device events over a full grid (throughput):
//   1. dependent-load round trip of an L2-resident word: ld.relaxed.gpu (the
//      queue's polls), ld.acquire.gpu (the flag protocol's acquire), and a
//      plain cached ld (L1 hit after the first touch) for reference;
//   2. fence.sc.gpu / fence.acq_rel.gpu after a store (the flag protocol's
//      publish cost);
//   3. atomicAdd round trip on one address (the ticket / done counters), alone
//      and with every SM hammering the same address (throughput);
//   4. L2 read bandwidth of a 64 MiB buffer (L2-resident) vs a 1 GiB one (HBM).
// Build + run:  nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o /tmp/lp tools/latency_probe.cu && /tmp/lp
#include <cstdio>
#include <cstdint>
#include <cuda_runtime.h>

__device__ __forceinline__ unsigned ld_relaxed(const unsigned* p) {
  unsigned v;
  asm volatile("ld.relaxed.gpu.global.u32 %0, [%1];" : "=r"(v) : "l"(p) : "memory");
  return v;
}
__device__ __forceinline__ unsigned ld_acquire(const unsigned* p) {
  unsigned v;
  asm volatile("ld.acquire.gpu.global.u32 %0, [%1];" : "=r"(v) : "l"(p) : "memory");
  return v;
}

// pointer chase over an L2-resident ring: chain[i] = next index (stride 33 lines)
template <int KIND>
__global__ void chase(const unsigned* chain, int iters, unsigned long long* out) {
  unsigned i = 0;
  const long long t0 = clock64();
  for (int k = 0; k < iters; ++k) {
    if (KIND == 0) i = ld_relaxed(chain + i);
    else if (KIND == 1) i = ld_acquire(chain + i);
    else i = chain[i];
  }
  const long long t1 = clock64();
  if (threadIdx.x == 0) out[0] = (unsigned long long)(t1 - t0), out[1] = i;
}

template <int KIND>
__global__ void fence_cost(unsigned* buf, int iters, unsigned long long* out) {
  const long long t0 = clock64();
  for (int k = 0; k < iters; ++k) {
    buf[threadIdx.x + 32 * (k & 63)] = k;
    if (KIND == 0) asm volatile("fence.sc.gpu;" ::: "memory");
    else asm volatile("fence.acq_rel.gpu;" ::: "memory");
  }
  const long long t1 = clock64();
  if (threadIdx.x == 0) out[0] = (unsigned long long)(t1 - t0);
}

__global__ void atomic_latency(unsigned* ctr, int iters, unsigned long long* out) {
  unsigned v = 0;
  const long long t0 = clock64();
  for (int k = 0; k < iters; ++k) v += atomicAdd(ctr, 1u + (v & 0));  // dependent chain
  const long long t1 = clock64();
  if (threadIdx.x == 0) out[0] = (unsigned long long)(t1 - t0), out[1] = v;
}

__global__ void atomic_contended(unsigned* ctr, int iters) {
  if ((threadIdx.x & 31) != 0) return;  // one atomic per warp, every warp of the grid on one address
  for (int k = 0; k < iters; ++k) atomicAdd(ctr, 1u);
}

__global__ void read_bw(const uint4* p, size_t n16, unsigned* sink) {
  uint4 acc = make_uint4(0, 0, 0, 0);
  for (size_t i = blockIdx.x * (size_t)blockDim.x + threadIdx.x; i < n16; i += (size_t)gridDim.x * blockDim.x) {
    const uint4 v = __ldcg(p + i);
    acc.x ^= v.x; acc.y ^= v.y; acc.z ^= v.z; acc.w ^= v.w;
  }
  if ((acc.x ^ acc.y ^ acc.z ^ acc.w) == 0x12345u) sink[0] = 1;
}

int main() {
  int clk_khz = 0;
  cudaDeviceGetAttribute(&clk_khz, cudaDevAttrClockRate, 0);
  const double ghz = clk_khz / 1e6;
  unsigned long long* out;
  cudaMalloc(&out, 16);
  unsigned long long h[2];
  // 1. chase
  const int ring = 1 << 16;  // 64 K words x 33-line stride spread over 8 MiB (L2-resident, > L1)
  unsigned* chain;
  cudaMalloc(&chain, (size_t)ring * 33 * 32 * 4);
  {
    unsigned* hc = new unsigned[(size_t)ring * 33 * 32];
    for (int k = 0; k < ring; ++k) hc[(size_t)k * 33 * 32] = (unsigned)(((size_t)((k + 1) % ring)) * 33 * 32);
    cudaMemcpy(chain, hc, (size_t)ring * 33 * 32 * 4, cudaMemcpyHostToDevice);
    delete[] hc;
  }
  const int it = 4096;
  const char* names[3] = {"ld.relaxed.gpu", "ld.acquire.gpu", "ld (cached)"};
  for (int kind = 0; kind < 3; ++kind) {
    for (int rep = 0; rep < 2; ++rep) {
      if (kind == 0) chase<0><<<1, 1>>>(chain, it, out);
      if (kind == 1) chase<1><<<1, 1>>>(chain, it, out);
      if (kind == 2) chase<2><<<1, 1>>>(chain, it, out);
    }
    cudaMemcpy(h, out, 16, cudaMemcpyDeviceToHost);
    printf("dependent %-16s round trip: %7.1f cycles = %6.1f ns (L2-resident chain, 1 thread)\n", names[kind],
           (double)h[0] / it, (double)h[0] / it / ghz);
  }
  // 2. fences
  unsigned* buf;
  cudaMalloc(&buf, 1 << 20);
  const char* fn[2] = {"fence.sc.gpu", "fence.acq_rel.gpu"};
  for (int kind = 0; kind < 2; ++kind) {
    for (int rep = 0; rep < 2; ++rep) {
      if (kind == 0) fence_cost<0><<<1, 32>>>(buf, 1024, out);
      else fence_cost<1><<<1, 32>>>(buf, 1024, out);
    }
    cudaMemcpy(h, out, 16, cudaMemcpyDeviceToHost);
    printf("store + %-18s: %7.1f cycles = %6.1f ns per iteration (1 warp)\n", fn[kind], (double)h[0] / 1024,
           (double)h[0] / 1024 / ghz);
  }
  // 3. atomics
  unsigned* ctr;
  cudaMalloc(&ctr, 64);
  for (int rep = 0; rep < 2; ++rep) atomic_latency<<<1, 1>>>(ctr, 2048, out);
  cudaMemcpy(h, out, 16, cudaMemcpyDeviceToHost);
  printf("dependent atomicAdd round trip     : %7.1f cycles = %6.1f ns (1 thread, one address)\n", (double)h[0] / 2048,
         (double)h[0] / 2048 / ghz);
  cudaEvent_t e0, e1;
  cudaEventCreate(&e0);
  cudaEventCreate(&e1);
  const int warps = 148 * 32, per = 256;
  atomic_contended<<<148 * 4, 256>>>(ctr, per);
  cudaEventRecord(e0);
  atomic_contended<<<148 * 4, 256>>>(ctr, per);
  cudaEventRecord(e1);
  cudaEventSynchronize(e1);
  float ms;
  cudaEventElapsedTime(&ms, e0, e1);
  const double n_at = (double)warps * per;
  printf("contended atomicAdd, one address   : %.3f G atomics/s (%.2f ns each; %d warps x %d)\n", n_at / ms / 1e6,
         ms * 1e6 / n_at, warps, per);
  // 4. bandwidth: L2-resident vs HBM
  for (size_t mb : {64, 1024}) {
    const size_t bytes = mb << 20;
    uint4* p;
    cudaMalloc(&p, bytes);
    cudaMemset(p, 1, bytes);
    unsigned* sink;
    cudaMalloc(&sink, 4);
    for (int w = 0; w < 3; ++w) read_bw<<<148 * 8, 512>>>(p, bytes / 16, sink);
    cudaEventRecord(e0);
    const int reps = 10;
    for (int r = 0; r < reps; ++r) read_bw<<<148 * 8, 512>>>(p, bytes / 16, sink);
    cudaEventRecord(e1);
    cudaEventSynchronize(e1);
    cudaEventElapsedTime(&ms, e0, e1);
    printf("read bandwidth, %4zu MiB buffer     : %7.1f GB/s (%s)\n", mb, (double)bytes * reps / (ms * 1e-3) / 1e9,
           mb < 100 ? "L2-resident" : "HBM");
    cudaFree(p);
    cudaFree(sink);
  }
  printf("SM clock attribute: %.3f GHz\n", ghz);
  return 0;
}
