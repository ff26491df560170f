// k_matmul.cu -- MatrixMultiplication ("MM"; high Intra
// overhead; LDS over-allocation > 1/2 of the +LDS overhead; Inter
// ~2x for compute-bound kernels).  C = A * Bt^T, bf16 operands (K-major
// both), fp32 accumulation and result (reading R-MM1).
//
// B200 design (tcgen05 + TMEM + TMA): one 128x256 output tile per logical CTA,
// K in blocks of 64 (128-B rows, SWIZZLE_128B).  Thread 0 streams A/B tiles
// into a ring of smem stages with TMA (cp.async.bulk.tensor, mbarrier
// complete_tx); thread 32 issues tcgen05.mma (M=128, N=256, K=16) into a TMEM
// accumulator and frees each stage with tcgen05.commit.  Both replicas run on
// the tensor pipe (BASELINE.json): the intra variants issue every MMA twice, into
// two TMEM accumulators (acc0 cols [0,256), acc1 cols [256,512)); INTRA_SMEM
// also keeps a private copy of every operand tile per replica (+LDS),
// INTRA_REG shares one operand copy (the load path is outside the SoR).
// Inter-group: two CTAs per tile, each with its own accumulator.
// Epilogue: warps read their replica's accumulator (tcgen05.ld 32x32b) into a
// per-replica smem staging plane (aliasing the drained operand ring), then
// every logical thread commits 16-B vectors of C through the RMT commit.
// The MMA shape and K order are identical in every variant, so outputs are
// bit-identical (determinism rule).
#include <cuda.h>
#include <string.h>

#include "rmt_host.cuh"

namespace rmt {
namespace {

constexpr int BM = 128, BN = 256, BK = 64, UK = 16;
constexpr int BL = 128;                      // logical threads per CTA (4 warps)
constexpr int TILE_A = BM * BK * 2;          // 16 KiB A tile per stage
constexpr int TILE_B = BN * BK * 2;          // 32 KiB B tile per stage
constexpr int SPITCH = 68;                   // staging row pitch (floats): conflict-free
constexpr int SPLANE = BM * SPITCH + 16;     // replica plane offset (16 banks apart)
constexpr int ECHUNK = 64;                   // epilogue columns per chunk

template <int V>
struct MmCfg {
  static constexpr int COPIES = (V == V_INTRA_SMEM) ? 2 : 1;       // operand copies in smem
  static constexpr int ACCS = (V == V_INTRA_SMEM || V == V_INTRA_REG || V == V_INTRA_NOLDS) ? 2 : 1;
  static constexpr int COPY_BYTES = TILE_A + TILE_B;
  static constexpr int STAGE_BYTES = COPY_BYTES * COPIES;
  static constexpr int NSTAGE = COPIES == 2 ? 2 : 4;               // 192 KiB of operand ring
  static constexpr int SMEM = NSTAGE * STAGE_BYTES + 1024;
  static constexpr int TMEM_COLS = BN * ACCS;                     // 256 or 512 columns
};

struct MmArgs {
  CUtensorMap tmA;  // A: M x K bf16, box 64 x 128
  CUtensorMap tmB;  // Bt: N x K bf16, box 64 x 256
  float* C;
  unsigned M, N, K;
  unsigned ntn;     // tiles along N
};

// ---------------------------------------------------------------- PTX wrappers
__device__ __forceinline__ uint32_t smem_u32(const void* p) { return (uint32_t)__cvta_generic_to_shared(p); }

__device__ __forceinline__ void mbar_init(uint32_t bar, uint32_t count) {
  asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(bar), "r"(count) : "memory");
}
__device__ __forceinline__ void mbar_expect_tx(uint32_t bar, uint32_t bytes) {
  asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(bar), "r"(bytes) : "memory");
}
__device__ __forceinline__ void mbar_wait(uint32_t bar, uint32_t parity) {
  asm volatile(
      "{\n\t.reg .pred p;\n"
      "WAIT_%=:\n\t"
      "mbarrier.try_wait.parity.shared::cta.b64 p, [%0], %1;\n\t"
      "@!p bra WAIT_%=;\n\t}" ::"r"(bar),
      "r"(parity)
      : "memory");
}
__device__ __forceinline__ void tma_load_2d(uint32_t dst, const CUtensorMap* tm, int x, int y, uint32_t bar) {
  asm volatile(
      "cp.async.bulk.tensor.2d.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1, {%2, %3}], [%4];" ::"r"(dst),
      "l"((uint64_t)tm), "r"(x), "r"(y), "r"(bar)
      : "memory");
}
__device__ __forceinline__ void tc_fence_before() { asm volatile("tcgen05.fence::before_thread_sync;" ::: "memory"); }
__device__ __forceinline__ void tc_fence_after() { asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory"); }
__device__ __forceinline__ void tc_commit(uint32_t bar) {
  asm volatile("tcgen05.commit.cta_group::1.mbarrier::arrive::one.shared::cluster.b64 [%0];" ::"r"(bar) : "memory");
}
__device__ __forceinline__ void tc_mma(uint32_t d, uint64_t a, uint64_t b, uint32_t idesc, uint32_t accum) {
  asm volatile(
      "{\n\t.reg .pred p;\n\tsetp.ne.b32 p, %4, 0;\n\t"
      "tcgen05.mma.cta_group::1.kind::f16 [%0], %1, %2, %3, p;\n\t}" ::"r"(d),
      "l"(a), "l"(b), "r"(idesc), "r"(accum)
      : "memory");
}
__device__ __forceinline__ void tc_ld16(uint32_t taddr, uint32_t (&r)[16]) {
  asm volatile(
      "tcgen05.ld.sync.aligned.32x32b.x16.b32 {%0,%1,%2,%3,%4,%5,%6,%7,%8,%9,%10,%11,%12,%13,%14,%15}, [%16];"
      : "=r"(r[0]), "=r"(r[1]), "=r"(r[2]), "=r"(r[3]), "=r"(r[4]), "=r"(r[5]), "=r"(r[6]), "=r"(r[7]), "=r"(r[8]),
        "=r"(r[9]), "=r"(r[10]), "=r"(r[11]), "=r"(r[12]), "=r"(r[13]), "=r"(r[14]), "=r"(r[15])
      : "r"(taddr)
      : "memory");
  asm volatile("tcgen05.wait::ld.sync.aligned;" ::: "memory");
}

// UMMA shared-memory descriptor, K-major SWIZZLE_128B tile (rows of 128 B,
// 8-row groups 1024 B apart): start>>4, LBO=1 (16 B, unused for swizzled
// K-major), SBO=1024>>4, version 1 (Blackwell), layout type 2 (SW128).
__device__ __forceinline__ uint64_t sdesc(uint32_t saddr) {
  uint64_t d = 0;
  d |= (uint64_t)((saddr >> 4) & 0x3FFF);
  d |= (uint64_t)1 << 16;
  d |= (uint64_t)(1024 >> 4) << 32;
  d |= (uint64_t)1 << 46;
  d |= (uint64_t)2 << 61;
  return d;
}
// Instruction descriptor: D=F32 (bit 4), A=B=BF16 (bits 7, 10), K-major both,
// N>>3 at bit 17, M>>4 at bit 24.
constexpr uint32_t IDESC = (1u << 4) | (1u << 7) | (1u << 10) | ((uint32_t)(BN >> 3) << 17) | ((uint32_t)(BM >> 4) << 24);

template <int V, int M>
__global__ void __launch_bounds__(BL * Geom<V>::DUP, 1) mm_kernel(const __grid_constant__ MmArgs a, Ctx c) {
  using Cfg = MmCfg<V>;
  extern __shared__ __align__(1024) unsigned char dsm[];
  __shared__ unsigned mb[mbox_words<V>(BL * Geom<V>::DUP)];
  constexpr int NSTAGE = Cfg::NSTAGE;
  __shared__ __align__(8) unsigned long long bar_full[NSTAGE], bar_empty[NSTAGE], bar_done;
  __shared__ uint32_t s_tmem;
  unsigned char* smem = (unsigned char*)(((uintptr_t)dsm + 1023) & ~(uintptr_t)1023);
  Rep<V, M> rep(c);
  rep.init(mb);
  const unsigned tm = (unsigned)rep.lblock / a.ntn, tn = (unsigned)rep.lblock % a.ntn;
  const int warp = threadIdx.x >> 5;
  const unsigned KB = a.K / BK;

  if (threadIdx.x == 0) {
    for (int s = 0; s < NSTAGE; ++s) {
      mbar_init(smem_u32(&bar_full[s]), 1);
      mbar_init(smem_u32(&bar_empty[s]), 1);
    }
    mbar_init(smem_u32(&bar_done), 1);
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
    asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
  }
  if (warp == 1) {  // whole warp: TMEM allocation
    asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], %1;" ::"r"(smem_u32(&s_tmem)),
                 "r"(Cfg::TMEM_COLS)
                 : "memory");
    asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;" ::: "memory");
  }
  tc_fence_before();
  __syncthreads();
  tc_fence_after();
  const uint32_t tmem = s_tmem;

  if (threadIdx.x == 0) {
    // ---- TMA producer
    for (unsigned kb = 0; kb < KB; ++kb) {
      const unsigned s = kb % NSTAGE, ph = (kb / NSTAGE) & 1u;
      mbar_wait(smem_u32(&bar_empty[s]), ph ^ 1u);
      const uint32_t fb = smem_u32(&bar_full[s]);
      mbar_expect_tx(fb, Cfg::STAGE_BYTES);
      const uint32_t st = smem_u32(smem + s * Cfg::STAGE_BYTES);
#pragma unroll
      for (int cp = 0; cp < Cfg::COPIES; ++cp) {  // INTRA_SMEM: one private copy per replica
        tma_load_2d(st + cp * Cfg::COPY_BYTES, &a.tmA, (int)(kb * BK), (int)(tm * BM), fb);
        tma_load_2d(st + cp * Cfg::COPY_BYTES + TILE_A, &a.tmB, (int)(kb * BK), (int)(tn * BN), fb);
      }
    }
  } else if (threadIdx.x == 32) {
    // ---- MMA issuer (one thread issues for the CTA)
    for (unsigned kb = 0; kb < KB; ++kb) {
      const unsigned s = kb % NSTAGE, ph = (kb / NSTAGE) & 1u;
      mbar_wait(smem_u32(&bar_full[s]), ph);
      tc_fence_after();
      const uint32_t st = smem_u32(smem + s * Cfg::STAGE_BYTES);
#pragma unroll
      for (int k = 0; k < BK / UK; ++k) {
        const uint32_t acc = (kb | (unsigned)k) != 0u;
#pragma unroll
        for (int rr = 0; rr < Cfg::ACCS; ++rr) {  // replica rr: its own accumulator (and operand copy)
          const uint32_t base = st + (Cfg::COPIES == 2 ? rr : 0) * Cfg::COPY_BYTES + k * UK * 2;
          tc_mma(tmem + rr * BN, sdesc(base), sdesc(base + TILE_A), IDESC, acc);
        }
      }
      tc_commit(smem_u32(&bar_empty[s]));  // frees the stage when these MMAs complete
    }
    tc_commit(smem_u32(&bar_done));
  }
  __syncwarp();  // reconverge the producer / issuer warps before .sync.aligned tcgen05 ops
  // ---- epilogue
  mbar_wait(smem_u32(&bar_done), 0);
  __syncwarp();
  tc_fence_after();
  float* stg = reinterpret_cast<float*>(smem);  // aliases the drained operand ring
  const int q = warp & 3;                        // TMEM lane quarter this warp may access
  const int rrep = (Cfg::ACCS == 2) ? (warp >> 2) : 0;  // which accumulator this warp stages
  const int lane = threadIdx.x & 31;
  const int row = 32 * q + lane;
  for (int ch = 0; ch < BN / ECHUNK; ++ch) {
    __syncthreads();  // previous chunk's staging fully consumed
#pragma unroll
    for (int cc = 0; cc < ECHUNK / 16; ++cc) {
      uint32_t v[16];
      tc_ld16(tmem + ((uint32_t)(32 * q) << 16) + rrep * BN + ch * ECHUNK + cc * 16, v);
      if constexpr (M == M_FAULT) {
#pragma unroll
        for (int t = 0; t < 16; ++t) {
          const long long e = (long long)(tm * BM + row) * a.N + tn * BN + ch * ECHUNK + cc * 16 + t;
          if (c.f.site == SITE_COMPUTE && c.f.elem == e && c.f.replica == (Cfg::ACCS == 2 ? rrep : rep.r))
            v[t] ^= 1u << c.f.bit;
        }
      }
      float4* dst = reinterpret_cast<float4*>(stg + rrep * SPLANE + row * SPITCH + cc * 16);
#pragma unroll
      for (int t = 0; t < 4; ++t)
        dst[t] = make_float4(__uint_as_float(v[4 * t]), __uint_as_float(v[4 * t + 1]), __uint_as_float(v[4 * t + 2]),
                             __uint_as_float(v[4 * t + 3]));
    }
    __syncthreads();
#pragma unroll 1
    for (int i = 0; i < BM * ECHUNK / 4 / BL; ++i) {
      const int vi = rep.ltid + BL * i;
      const int r = vi / (ECHUNK / 4), c4 = (vi % (ECHUNK / 4)) * 4;
      // replica r reads the staging of its own accumulator (also under -LDS: the
      // two accumulators are the replicas' state, not kernel-written shared data)
      const float4 f = *reinterpret_cast<const float4*>(stg + (Cfg::ACCS == 2 ? rep.r : 0) * SPLANE + r * SPITCH + c4);
      unsigned w[4] = {__float_as_uint(f.x), __float_as_uint(f.y), __float_as_uint(f.z), __float_as_uint(f.w)};
      const unsigned idx = (tm * BM + r) * a.N + tn * BN + ch * ECHUNK + c4;
      rep.template commit<4, 0>(0xFu, idx, w, a.M * a.N, [&](unsigned e, unsigned m, const unsigned* x) {
        if (m == 0xFu)
          __stcs(reinterpret_cast<float4*>(a.C + e), make_float4(__uint_as_float(x[0]), __uint_as_float(x[1]),
                                                                   __uint_as_float(x[2]), __uint_as_float(x[3])));
        else
          for (int k = 0; k < 4; ++k)
            if ((m >> k) & 1u) a.C[e + k] = __uint_as_float(x[k]);
      }, /*defer=*/(i & 3) != 3);
    }
  }
  tc_fence_before();
  __syncthreads();
  if (warp == 1) {
    tc_fence_after();
    asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, %1;" ::"r"(tmem), "r"(Cfg::TMEM_COLS) : "memory");
  }
  rep.finish();
}

// ---------------------------------------------------------------- host: TMA descriptors
typedef CUresult (*EncodeTiledFn)(CUtensorMap*, CUtensorMapDataType, cuuint32_t, void*, const cuuint64_t*,
                                  const cuuint64_t*, const cuuint32_t*, const cuuint32_t*, CUtensorMapInterleave,
                                  CUtensorMapSwizzle, CUtensorMapL2promotion, CUtensorMapFloatOOBfill);

EncodeTiledFn get_encode() {
  static EncodeTiledFn fn = nullptr;
  if (!fn) {
    void* p = nullptr;
    cudaDriverEntryPointQueryResult q;
    if (cudaGetDriverEntryPoint("cuTensorMapEncodeTiled", &p, cudaEnableDefault, &q) == cudaSuccess &&
        q == cudaDriverEntryPointSuccess)
      fn = (EncodeTiledFn)p;
  }
  return fn;
}

int make_tmap(CUtensorMap* tm, const void* base, unsigned rows, unsigned K, unsigned box_rows) {
  EncodeTiledFn enc = get_encode();
  if (!enc) {
    set_error("matmul: cuTensorMapEncodeTiled unavailable");
    return RMT_ECUDA;
  }
  cuuint64_t dims[2] = {K, rows};
  cuuint64_t strides[1] = {(cuuint64_t)K * 2};
  cuuint32_t box[2] = {BK, box_rows};
  cuuint32_t es[2] = {1, 1};
  CUresult r = enc(tm, CU_TENSOR_MAP_DATA_TYPE_BFLOAT16, 2, const_cast<void*>(base), dims, strides, box, es,
                   CU_TENSOR_MAP_INTERLEAVE_NONE, CU_TENSOR_MAP_SWIZZLE_128B, CU_TENSOR_MAP_L2_PROMOTION_L2_256B,
                   CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
  if (r != CUDA_SUCCESS) {
    set_error("matmul: cuTensorMapEncodeTiled failed (" + std::to_string((int)r) + ")");
    return RMT_ECUDA;
  }
  return RMT_OK;
}

}  // namespace

int matmul_validate(const rmt_bufs_t* b, int64_t n) {
  int64_t M = b->dims[0], N = b->dims[1], K = b->dims[2];
  if (b->nbuf < 3 || M <= 0 || N <= 0 || K <= 0 || M % BM || N % BN || K % BK || n != M * N ||
      M * N >= (1LL << 30) || K >= (1LL << 24) || !buf_ok(b->buf[0], RMT_BF16, M * K) ||
      !buf_ok(b->buf[1], RMT_BF16, N * K) || !buf_ok(b->buf[2], RMT_F32, M * N)) {
    set_error("matmul: expected {A:BF16[M*K], Bt:BF16[N*K], C:F32[M*N]}, dims {M,N,K}, M%128 = N%256 = 0, K%64 = 0");
    return RMT_EINVAL;
  }
  return RMT_OK;
}
size_t matmul_scratch(int64_t, const int64_t*) { return 0; }
int matmul_inter_warps(int64_t, const int64_t*) { return BL / 32; }

int matmul_run(Launch& L) {
  const unsigned M = (unsigned)L.bufs->dims[0], N = (unsigned)L.bufs->dims[1], K = (unsigned)L.bufs->dims[2];
  MmArgs a;
  memset(&a, 0, sizeof(a));
  int rc = make_tmap(&a.tmA, L.bufs->buf[0].ptr, M, K, BM);
  if (rc) return rc;
  rc = make_tmap(&a.tmB, L.bufs->buf[1].ptr, N, K, BN);
  if (rc) return rc;
  a.C = (float*)L.bufs->buf[2].ptr;
  a.M = M;
  a.N = N;
  a.K = K;
  a.ntn = N / BN;
  const unsigned G = (M / BM) * (N / BN);
  return dispatch(L.variant, L.mode, [&](auto vm) {
    constexpr int V = decltype(vm)::V, Mo = decltype(vm)::M;
    return launch_std<V>(L, mm_kernel<V, Mo>, mm_kernel<V_NONE, M_NORMAL>, G, BL, MmCfg<V>::SMEM, a, "matmul",
                         /*persistent=*/false);
  });
}

}  // namespace rmt
