// rmt_host.cuh -- host-side plumbing shared by the per-kernel launchers:
// launch descriptor, variant x mode dispatch, workspace layout, error detail.
#pragma once
#include <cuda_runtime.h>
#include <stdint.h>

#include <stdlib.h>

#include <string>

#include "../../include/rmt.h"
#include "rmt_device.cuh"

namespace rmt {

#ifndef RMT_PDL
#define RMT_PDL 1  // programmatic dependent launch between the library's kernels
#endif

// Inter-group queue geometry.
constexpr int INTER_R = 1024;  // regions (> resident pairs, so a region is rarely waited for)
constexpr int INTER_S = INTER_SLOTS_MAX;  // slots allocated per (region, warp); Ctx::S <= INTER_S in use
constexpr size_t CTRL_BYTES = (size_t)(CTRL_TURN + INTER_R) * 4;

struct Launch {
  int kernel, variant, mode;
  bool inflate;               // RMT_ABL_INFLATE: run V_NONE with the RMT variant's residency
  int cl_depth;               // inter_cluster mailbox slots requested by a stress test (0: default)
  const rmt_bufs_t* bufs;
  int64_t n;
  Ctx ctx;                    // err + fault + inter queue pointers
  char* scratch;              // kernel-specific scratch (after the inter queue)
  size_t scratch_bytes;
  cudaStream_t stream;
  int launches;               // kernels launched (for rmt_last_launch_count)
};

void set_error(const std::string& msg);
int cuda_check(cudaError_t e, const char* what);

// Bytes of the inter-group queue for CTAs of `warps` physical warps.
inline size_t inter_bytes(int warps) {
  size_t slots = (size_t)INTER_R * warps * INTER_S;
  return CTRL_BYTES + slots * 4 + slots * RING_WORDS * 32 * 4;
}
inline size_t align_up(size_t x, size_t a) { return (x + a - 1) / a * a; }

template <int V_, int M_>
struct VM {
  static constexpr int V = V_;
  static constexpr int M = M_;
};

// Call f(VM<V, M>{}) for the runtime (variant, mode).  M_NOCOMM only exists for
// the RMT variants; the none variant ignores it.  M_STRESS only exists for the
// queue variants (inter_group, inter_cluster); the others run M_NORMAL.
template <class F>
int dispatch(int v, int m, F&& f) {
  switch (v) {
    case V_NONE:
      return m == M_FAULT ? f(VM<V_NONE, M_FAULT>{}) : f(VM<V_NONE, M_NORMAL>{});
    case V_INTRA_SMEM:
      return m == M_FAULT ? f(VM<V_INTRA_SMEM, M_FAULT>{})
           : m == M_NOCOMM ? f(VM<V_INTRA_SMEM, M_NOCOMM>{})
                           : f(VM<V_INTRA_SMEM, M_NORMAL>{});
    case V_INTRA_REG:
      return m == M_FAULT ? f(VM<V_INTRA_REG, M_FAULT>{})
           : m == M_NOCOMM ? f(VM<V_INTRA_REG, M_NOCOMM>{})
                           : f(VM<V_INTRA_REG, M_NORMAL>{});
    case V_INTER:
      return m == M_FAULT ? f(VM<V_INTER, M_FAULT>{})
           : m == M_NOCOMM ? f(VM<V_INTER, M_NOCOMM>{})
           : m == M_STRESS ? f(VM<V_INTER, M_STRESS>{})
                           : f(VM<V_INTER, M_NORMAL>{});
    case V_INTRA_NOLDS:
      return m == M_FAULT ? f(VM<V_INTRA_NOLDS, M_FAULT>{})
           : m == M_NOCOMM ? f(VM<V_INTRA_NOLDS, M_NOCOMM>{})
                           : f(VM<V_INTRA_NOLDS, M_NORMAL>{});
    case V_CLUSTER:
      return m == M_FAULT ? f(VM<V_CLUSTER, M_FAULT>{})
           : m == M_NOCOMM ? f(VM<V_CLUSTER, M_NOCOMM>{})
           : m == M_STRESS ? f(VM<V_CLUSTER, M_STRESS>{})
                           : f(VM<V_CLUSTER, M_NORMAL>{});
  }
  return RMT_EINVAL;
}

// Checks shared by the per-kernel validators.
inline bool buf_ok(const rmt_buf_t& b, int dtype, int64_t numel) {
  return (b.ptr != nullptr || numel == 0) && b.dtype == dtype && b.numel == numel && ((uintptr_t)b.ptr % 16) == 0;
}

// ---- per-kernel entry points (one translation unit each)
#define RMT_DECLARE_KERNEL(name)                                              \
  int name##_validate(const rmt_bufs_t* b, int64_t n);                        \
  size_t name##_scratch(int64_t n, const int64_t* dims);                      \
  int name##_inter_warps(int64_t n, const int64_t* dims);                     \
  int name##_run(Launch& L);

RMT_DECLARE_KERNEL(blackscholes)
RMT_DECLARE_KERNEL(binarysearch)
RMT_DECLARE_KERNEL(fwt)
RMT_DECLARE_KERNEL(prefixsum)
RMT_DECLARE_KERNEL(reduction)
RMT_DECLARE_KERNEL(transpose)
RMT_DECLARE_KERNEL(sobel)
RMT_DECLARE_KERNEL(floydwarshall)
RMT_DECLARE_KERNEL(dct)
RMT_DECLARE_KERNEL(matmul)
RMT_DECLARE_KERNEL(dwthaar1d)
RMT_DECLARE_KERNEL(bitonicsort)
RMT_DECLARE_KERNEL(binomialoption)

// dup_kernel: commit agreeing 4-word groups of shadows a, b to out; count the others.
int dup_compare_launch(const void* a, const void* b, void* out, unsigned long long nwords, unsigned long long* err,
                       cudaStream_t s);

}  // namespace rmt

namespace rmt {

// Smallest dynamic-smem padding that brings kernel `kn` (block bn, smem sn) to
// at most `target` CTAs per SM.
template <class K>
size_t pad_for_occupancy(K kn, int bn, size_t sn, int target) {
  cudaFuncAttributes fa;
  if (cudaFuncGetAttributes(&fa, kn) != cudaSuccess) return 0;
  const size_t cap = 227 * 1024 - fa.sharedSizeBytes;  // static + dynamic <= 227 KiB per CTA
  size_t best = 0;
  for (size_t extra = 0; sn + extra <= cap; extra += 1024) {
    if (sn + extra > 48 * 1024 &&
        cudaFuncSetAttribute(kn, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)(sn + extra)) != cudaSuccess)
      break;
    int occ = 0;
    if (cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, kn, bn, sn + extra) != cudaSuccess || occ < 1) break;
    best = extra;
    if (occ <= target) break;
  }
  cudaGetLastError();  // clear any error from probing
  return best;
}

// Standard launch of one RMT kernel instance: logical grid G of BL-thread
// logical CTAs, `smem` dynamic shared bytes.  kr = the variant's kernel,
// kn = the V_NONE kernel (used for the INFLATE ablation).
// inter_group / inter_cluster launch P = mult x (the pairs that fit on the GPU
// at once) replica pairs (<= G) and each pair walks the logical CTAs pair,
// pair + P, ... (Rep::active/advance); mult = 0 keeps one logical CTA per pair
// (and is required for kernels whose body is not the logical-CTA loop).
// Persistent replica pairs ("Persistent pairs"): the
// inter variants launch k x the pairs that fit on the GPU at once, and each pair
// walks its share of the logical CTAs.  k is chosen per kernel from the suite
// measurements (0 = one logical CTA per pair); experiment knob
// RMT_INTER_PAIRS_MULT overrides it for every kernel.
inline int inter_pairs_mult(int kernel_choice) {
  static int m = [] {
    const char* e = getenv("RMT_INTER_PAIRS_MULT");
    return e ? atoi(e) : -1;
  }();
  return m >= 0 ? m : kernel_choice;
}

template <int V, class Args>
unsigned inter_pairs(void (*kr)(Args, Ctx), int block, size_t dyn_smem, unsigned G, bool cluster, int mult) {
  mult = inter_pairs_mult(mult);
  if (mult <= 0) return G;
  int occ = 0;
  if (cluster) {
    cudaLaunchConfig_t cfg = {};
    cfg.gridDim = dim3(2);
    cfg.blockDim = dim3(block);
    cfg.dynamicSmemBytes = dyn_smem;
    cudaLaunchAttribute at[1];
    at[0].id = cudaLaunchAttributeClusterDimension;
    at[0].val.clusterDim.x = 2;
    at[0].val.clusterDim.y = 1;
    at[0].val.clusterDim.z = 1;
    cfg.attrs = at;
    cfg.numAttrs = 1;
    int ncl = 0;
    if (cudaOccupancyMaxActiveClusters(&ncl, kr, &cfg) != cudaSuccess || ncl < 1) {
      cudaGetLastError();
      ncl = 148;
    }
    occ = ncl;  // resident clusters = pairs
  } else {
    int per_sm = 0;
    if (cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, kr, block, dyn_smem) != cudaSuccess || per_sm < 1) {
      cudaGetLastError();
      per_sm = 2;
    }
    int dev = 0, nsm = 148;
    cudaGetDevice(&dev);
    cudaDeviceGetAttribute(&nsm, cudaDevAttrMultiProcessorCount, dev);
    occ = per_sm * nsm / 2;
  }
  unsigned P = (unsigned)(occ < 1 ? 1 : occ) * (unsigned)mult;
  return P < G ? P : G;
}

template <int V, class Args>
int launch_std(Launch& L, void (*kr)(Args, Ctx), void (*kn)(Args, Ctx), unsigned G, int BL, size_t smem,
               const Args& a, const char* what, int mult_inter = 0, int mult_cluster = 1, int bl_none = 0) {
  if (G == 0) return RMT_OK;
  Ctx c = L.ctx;
  c.nblocks = (int)G;
  c.pairs = (int)G;
  c.lstride = 0;
  if (L.inflate) {
    // run the original kernel with the RMT version's per-SM footprint
    // (inter: the footprint of two RMT groups).
    int occ = 0;
    if (smem > 48 * 1024) cudaFuncSetAttribute(kr, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
    cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, kr, Geom<V>::block(BL), smem);
    int target = (V == V_INTER || V == V_CLUSTER) ? (occ / 2 > 1 ? occ / 2 : 1) : (occ > 1 ? occ : 1);
    size_t pad = pad_for_occupancy(kn, bl_none ? bl_none : BL, smem, target);
    if (smem + pad > 48 * 1024)
      cudaFuncSetAttribute(kn, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)(smem + pad));
    kn<<<G, bl_none ? bl_none : BL, smem + pad, L.stream>>>(a, c);
  } else if constexpr (V == V_CLUSTER) {
    // the DSMEM mailbox (rmt_device.cuh, Rep::init) follows the kernel's own
    // dynamic shared memory
    size_t dyn = smem;
    if (L.mode != M_NOCOMM) {
      c.R = (int)align_up(smem, 16);
      c.S = BL <= 128 ? CL_S_LARGE : CL_S_SMALL;
      if (L.cl_depth > 0 && L.cl_depth < c.S) c.S = L.cl_depth;  // stress test: a shallower mailbox (power of 2)
      dyn = (size_t)c.R + (size_t)(BL / 32) * c.S * (RING_WORDS * 32 + 1) * 4;
    }
    cudaFuncSetAttribute(kr, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)dyn);
    c.pairs = (int)inter_pairs<V>(kr, Geom<V>::block(BL), dyn, G, true, mult_cluster);
    c.lstride = c.pairs < (int)G ? c.pairs : 0;
    cudaLaunchConfig_t cfg = {};
    cfg.gridDim = dim3(Geom<V>::grid((unsigned)c.pairs));
    cfg.blockDim = dim3(Geom<V>::block(BL));
    cfg.dynamicSmemBytes = dyn;
    cfg.stream = L.stream;
    cudaLaunchAttribute at[2];
    at[0].id = cudaLaunchAttributeClusterDimension;
    at[0].val.clusterDim.x = 2;  // the replica pair
    at[0].val.clusterDim.y = 1;
    at[0].val.clusterDim.z = 1;
    at[1].id = cudaLaunchAttributeProgrammaticStreamSerialization;
    at[1].val.programmaticStreamSerializationAllowed = RMT_PDL;
    cfg.attrs = at;
    cfg.numAttrs = 2;
    cudaError_t e = cudaLaunchKernelEx(&cfg, kr, a, c);
    if (e != cudaSuccess) return cuda_check(e, what);
  } else {
    if (smem > 48 * 1024) cudaFuncSetAttribute(kr, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
    if (V == V_INTER) {
      c.pairs = (int)inter_pairs<V>(kr, Geom<V>::block(BL), smem, G, false, mult_inter);
      c.lstride = c.pairs < (int)G ? c.pairs : 0;
    }
    // programmatic dependent launch: the grid is scheduled while the previous
    // kernel drains; Rep::init waits (griddepcontrol.wait) before any access
    cudaLaunchConfig_t cfg = {};
    cfg.gridDim = dim3(Geom<V>::grid(V == V_INTER ? (unsigned)c.pairs : G));
    cfg.blockDim = dim3(Geom<V>::block(BL));
    cfg.dynamicSmemBytes = smem;
    cfg.stream = L.stream;
    cudaLaunchAttribute at[1];
    at[0].id = cudaLaunchAttributeProgrammaticStreamSerialization;
    at[0].val.programmaticStreamSerializationAllowed = RMT_PDL;
    cfg.attrs = at;
    cfg.numAttrs = 1;
    cudaError_t e = cudaLaunchKernelEx(&cfg, kr, a, c);
    if (e != cudaSuccess) return cuda_check(e, what);
  }
  L.launches += 1;
  return cuda_check(cudaGetLastError(), what);
}

}  // namespace rmt
