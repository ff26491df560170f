// k_matmul.cu -- MatrixMultiplication ("MM"; high Intra
// overhead; LDS over-allocation > 1/2 of the +LDS overhead; Inter
// ~2x for compute-bound kernels).  C = A * Bt^T, bf16 operands (K-major
// both), fp32 accumulation and result (reading R-MM1).
//
// B200 design (tcgen05 + TMEM + TMA), warp-specialised: warp 0 streams A/B
// tiles into a ring of smem stages with TMA (cp.async.bulk.tensor, mbarrier
// complete_tx; K in blocks of 64, SWIZZLE_128B); one thread of warp 1 issues
// tcgen05.mma (M=128, K=16) into TMEM and frees each stage with tcgen05.commit;
// warps 2..9 fold.  K is cut into chunks of KC (default 1024): chunk ch
// accumulates from zero in TMEM buffer ch & 1 while the fold warps add the
// other buffer into a running fp32 total in registers with round-to-nearest
// adds (reading R-MM4: the tensor pipe's own fp32 accumulation is not RN, so
// the chunk bounds its drift; the fold order is fixed, so every variant is
// bit-identical).  Both replicas run on the tensor pipe (BASELINE.json): the
// intra variants issue every MMA twice, into two accumulators (tile 128x128,
// N=128 MMAs: 2 buffers x 2 replicas x 128 columns = the 512 TMEM columns);
// INTRA_SMEM also keeps a private copy of every operand tile per replica (+LDS,
// P:197), INTRA_REG shares one operand copy (the load path is outside the SoR,
// P:201).  Unprotected and inter-group CTAs compute 128x256 tiles (N=256).
// Epilogue: the fold warps stage their replica's totals in shared memory
// (aliasing the drained operand ring), then every logical thread commits 16-B
// vectors of C through the RMT commit.
#include <cuda.h>
#include <string.h>

#include "rmt_host.cuh"

namespace rmt {
namespace {

constexpr int BM = 128, BK = 64, UK = 16;
constexpr int NTHR = 320;                    // physical threads: warp 0 TMA, warp 1 MMA, warps 2..9 fold
constexpr int NFW = 8;                       // fold warps
constexpr int KC_DEFAULT = 1024;             // K elements per TMEM chunk (fold granularity, reading R-MM4)
constexpr int TILE_A = BM * BK * 2;          // 16 KiB A tile per stage

template <int V>
struct MmCfg {
  static constexpr int COPIES = (V == V_INTRA_SMEM) ? 2 : 1;       // operand copies in smem
  static constexpr int ACCS = (V == V_INTRA_SMEM || V == V_INTRA_REG || V == V_INTRA_NOLDS) ? 2 : 1;
  static constexpr int BN = ACCS == 2 ? 128 : 256;                 // tile width: 2 x BN x ACCS TMEM columns
  static constexpr int BL = NTHR / Geom<V>::DUP;                   // logical threads per CTA
  static constexpr int TILE_B = BN * BK * 2;
  static constexpr int COPY_BYTES = TILE_A + TILE_B;
  static constexpr int STAGE_BYTES = COPY_BYTES * COPIES;
  static constexpr int NSTAGE = (192 * 1024) / STAGE_BYTES;        // 192 KiB of operand ring
  static constexpr int SPITCH = BN + 4;                            // staging row pitch (floats)
  static constexpr int SPLANE = BM * SPITCH;                       // replica staging plane (floats)
  static constexpr int SMEM = NSTAGE * STAGE_BYTES + 1024;
  static constexpr int TMEM_COLS = 512;                            // 2 chunk buffers x BN x ACCS
  // UMMA instruction descriptor: D=F32 (bit 4), A=B=BF16 (bits 7, 10), K-major both,
  // N>>3 at bit 17, M>>4 at bit 24
  static constexpr uint32_t IDESC = (1u << 4) | (1u << 7) | (1u << 10) | ((uint32_t)(BN >> 3) << 17) |
                                    ((uint32_t)(BM >> 4) << 24);
  static_assert(ACCS * BN == 256, "a chunk buffer is 256 TMEM columns");
  static_assert(SPLANE * ACCS * 4 <= NSTAGE * STAGE_BYTES, "the staging tile fits in the drained operand ring");
};

struct MmArgs {
  CUtensorMap tmA;  // A: M x K bf16, box 64 x 128
  CUtensorMap tmB;  // Bt: N x K bf16, box 64 x BN
  float* C;
  unsigned M, N, K;
  unsigned ntn;     // tiles along N
  unsigned kpc;     // k-blocks (of BK) per TMEM chunk
};

// ---------------------------------------------------------------- PTX wrappers
__device__ __forceinline__ uint32_t smem_u32(const void* p) { return (uint32_t)__cvta_generic_to_shared(p); }

__device__ __forceinline__ void mbar_init(uint32_t bar, uint32_t count) {
  asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(bar), "r"(count) : "memory");
}
__device__ __forceinline__ void mbar_expect_tx(uint32_t bar, uint32_t bytes) {
  asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(bar), "r"(bytes) : "memory");
}
__device__ __forceinline__ void mbar_arrive(uint32_t bar) {
  asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0];" ::"r"(bar) : "memory");
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
// 16 columns of the warp's 32 TMEM lanes (no wait: the caller waits once for a batch)
__device__ __forceinline__ void tc_ld16_nowait(uint32_t taddr, uint32_t (&r)[16]) {
  asm volatile(
      "tcgen05.ld.sync.aligned.32x32b.x16.b32 {%0,%1,%2,%3,%4,%5,%6,%7,%8,%9,%10,%11,%12,%13,%14,%15}, [%16];"
      : "=r"(r[0]), "=r"(r[1]), "=r"(r[2]), "=r"(r[3]), "=r"(r[4]), "=r"(r[5]), "=r"(r[6]), "=r"(r[7]), "=r"(r[8]),
        "=r"(r[9]), "=r"(r[10]), "=r"(r[11]), "=r"(r[12]), "=r"(r[13]), "=r"(r[14]), "=r"(r[15])
      : "r"(taddr)
      : "memory");
}
__device__ __forceinline__ void tc_wait_ld() { asm volatile("tcgen05.wait::ld.sync.aligned;" ::: "memory"); }

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

// byte offset of bf16 element (row, kcol) in a TMA SWIZZLE_128B tile (1024-B
// aligned, 128-B rows): the 16-B chunk index is XORed with the row mod 8
__device__ __forceinline__ uint32_t sw128_off(uint32_t row, uint32_t kcol) {
  return row * 128u + ((((kcol * 2u) >> 4) ^ (row & 7u)) << 4) + ((kcol * 2u) & 15u);
}

// The FAULT build's operand hooks (MatMul LOAD = an A word after TMA, SMEM = a
// Bt word): flip a bit of the bf16 operand in the stage's shared-memory copy
// before the MMA reads it.  +LDS (intra_smem) keeps one operand copy per
// replica, so replica r's copy is flipped; the single-copy intra variants share
// the operand (the load path is outside their SoR): the flip reaches both
// replicas; inter CTAs flip their own copy.
template <int V, int M, class R>
__device__ __forceinline__ void operand_fault(const R& rep, const Ctx& c, const MmArgs& a, uint32_t st, unsigned kb,
                                              unsigned tm, unsigned tn) {
  using Cfg = MmCfg<V>;
  if constexpr (M == M_FAULT) {
    const bool isA = c.f.site == SITE_LOAD;
    if (!isA && c.f.site != SITE_SMEM) return;
    const long long rowg = c.f.elem / a.K, kg = c.f.elem % a.K;
    const long long row = rowg - (long long)(isA ? tm * BM : tn * Cfg::BN);
    const long long kcol = kg - (long long)kb * BK;
    if (row < 0 || row >= (isA ? BM : Cfg::BN) || kcol < 0 || kcol >= BK) return;
#pragma unroll
    for (int cp = 0; cp < Cfg::COPIES; ++cp) {
      const bool hit = Cfg::COPIES == 2 ? cp == c.f.replica : (Cfg::ACCS == 2 ? true : rep.r == c.f.replica);
      if (!hit) continue;
      const uint32_t base = st + cp * Cfg::COPY_BYTES + (isA ? 0u : (uint32_t)TILE_A);
      unsigned short* p = reinterpret_cast<unsigned short*>(
          __cvta_shared_to_generic(base + sw128_off((uint32_t)row, (uint32_t)kcol)));
      *p ^= (unsigned short)(1u << (c.f.bit & 15));
    }
    asm volatile("fence.proxy.async.shared::cta;" ::: "memory");  // generic-proxy write -> tensor core reads
  }
}

template <int V, int M>
__global__ void __launch_bounds__(NTHR, 1) mm_kernel(const __grid_constant__ MmArgs a, Ctx c) {
  using Cfg = MmCfg<V>;
  constexpr int BN = Cfg::BN;
  extern __shared__ __align__(1024) unsigned char dsm[];
  __shared__ unsigned mb[mbox_words<V>(NTHR)];
  constexpr int NSTAGE = Cfg::NSTAGE;
  __shared__ __align__(8) unsigned long long bar_full[NSTAGE], bar_empty[NSTAGE], acc_full[2], acc_empty[2];
  __shared__ uint32_t s_tmem;
  unsigned char* smem = (unsigned char*)(((uintptr_t)dsm + 1023) & ~(uintptr_t)1023);
  Rep<V, M> rep(c);
  rep.init(mb);
  const unsigned tm = (unsigned)rep.lblock / a.ntn, tn = (unsigned)rep.lblock % a.ntn;
  const int warp = threadIdx.x >> 5;
  const int lane = threadIdx.x & 31;
  const unsigned KB = a.K / BK;
  const unsigned NC = (KB + a.kpc - 1) / a.kpc;  // TMEM chunks (reading R-MM4: RN fold per chunk)

  if (threadIdx.x == 0) {
    for (int s = 0; s < NSTAGE; ++s) {
      mbar_init(smem_u32(&bar_full[s]), 1);
      mbar_init(smem_u32(&bar_empty[s]), 1);
    }
    for (int b = 0; b < 2; ++b) {
      mbar_init(smem_u32(&acc_full[b]), 1);
      mbar_init(smem_u32(&acc_empty[b]), NFW);
    }
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

  // fold warps: (TMEM lane quarter q, column group g): 32 rows x 128 columns of
  // the running fp32 total each, in registers
  const int fw = warp - 2;
  const int q = warp & 3;
  const int g = fw >> 2;
  float tot[128];

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
    // ---- MMA issuer (one thread issues for the CTA).  K chunk ch accumulates
    // from zero into TMEM buffer ch & 1; the fold warps drain the other buffer.
    for (unsigned kb = 0; kb < KB; ++kb) {
      const unsigned ch = kb / a.kpc, b = ch & 1u;
      const bool first = kb % a.kpc == 0u;
      if (first && ch >= 2u) {  // buffer b free: chunk ch - 2 folded
        mbar_wait(smem_u32(&acc_empty[b]), ((ch >> 1) - 1u) & 1u);
        tc_fence_after();
      }
      const unsigned s = kb % NSTAGE, ph = (kb / NSTAGE) & 1u;
      mbar_wait(smem_u32(&bar_full[s]), ph);
      tc_fence_after();
      const uint32_t st = smem_u32(smem + s * Cfg::STAGE_BYTES);
      operand_fault<V, M>(rep, c, a, st, kb, tm, tn);
#pragma unroll
      for (int k = 0; k < BK / UK; ++k) {
        const uint32_t acc = (first && k == 0) ? 0u : 1u;
#pragma unroll
        for (int rr = 0; rr < Cfg::ACCS; ++rr) {  // replica rr: its own accumulator (and operand copy)
          const uint32_t base = st + (Cfg::COPIES == 2 ? rr : 0) * Cfg::COPY_BYTES + k * UK * 2;
          tc_mma(tmem + 256u * b + (uint32_t)(rr * BN), sdesc(base), sdesc(base + TILE_A), Cfg::IDESC, acc);
        }
      }
      tc_commit(smem_u32(&bar_empty[s]));  // frees the stage when these MMAs complete
      if (kb % a.kpc == a.kpc - 1u || kb == KB - 1u) tc_commit(smem_u32(&acc_full[b]));  // chunk done
    }
  } else if (warp >= 2) {
    // ---- fold: total = (((c0 + c1) + c2) + ...) in fp32 round-to-nearest, the
    // same order in every variant
    for (unsigned ch = 0; ch < NC; ++ch) {
      const unsigned b = ch & 1u;
      mbar_wait(smem_u32(&acc_full[b]), (ch >> 1) & 1u);
      tc_fence_after();
      const uint32_t ta = tmem + ((uint32_t)(32 * q) << 16) + 256u * b + 128u * (uint32_t)g;
#pragma unroll
      for (int cc = 0; cc < 8; ++cc) {  // 16 columns per wait: 128 totals + 16 in flight fit the register budget
        uint32_t v[16];
        tc_ld16_nowait(ta + (uint32_t)(16 * cc), v);
        tc_wait_ld();
#pragma unroll
        for (int t = 0; t < 16; ++t) {
          const int i = 16 * cc + t;
          tot[i] = ch == 0u ? __uint_as_float(v[t]) : __fadd_rn(tot[i], __uint_as_float(v[t]));
        }
      }
      tc_fence_before();
      __syncwarp();
      if (lane == 0) mbar_arrive(smem_u32(&acc_empty[b]));
    }
  }
  __syncwarp();  // reconverge the producer / issuer warps
  __syncthreads();  // every chunk folded: the operand ring is drained, the tile is in registers
  // ---- stage the fold warps' totals: plane (replica) x 128 rows x BN columns
  float* stg = reinterpret_cast<float*>(smem);
  if (warp >= 2) {
    const int row = 32 * q + lane;
    const int rrep = Cfg::ACCS == 2 ? g : 0;              // replica of this accumulator
    const int col0 = Cfg::ACCS == 2 ? 0 : 128 * g;        // column group within the tile
#pragma unroll
    for (int t = 0; t < 128; ++t) {
      float x = tot[t];
      if constexpr (M == M_FAULT) {  // COMPUTE site: accumulator element e of one replica
        const long long e = (long long)(tm * BM + row) * a.N + tn * BN + col0 + t;
        if (c.f.site == SITE_COMPUTE && c.f.elem == e && c.f.replica == (Cfg::ACCS == 2 ? rrep : rep.r))
          x = __uint_as_float(__float_as_uint(x) ^ (1u << c.f.bit));
      }
      tot[t] = x;
    }
    float4* dst = reinterpret_cast<float4*>(stg + rrep * Cfg::SPLANE + row * Cfg::SPITCH + col0);
#pragma unroll
    for (int t = 0; t < 32; ++t) dst[t] = make_float4(tot[4 * t], tot[4 * t + 1], tot[4 * t + 2], tot[4 * t + 3]);
  }
  __syncthreads();
  // ---- RMT commits: every logical thread commits 16-B vectors of C from its
  // replica's staging plane (the accumulators are the replicas' state, also
  // under -LDS)
  constexpr int NVEC = BM * BN / 4;
  constexpr int ITERS = (NVEC + Cfg::BL - 1) / Cfg::BL;
#pragma unroll 1
  for (int i = 0; i < ITERS; ++i) {
    const int vi = rep.ltid + Cfg::BL * i;
    const bool in = vi < NVEC;
    const int r = in ? vi / (BN / 4) : 0, c4 = in ? (vi % (BN / 4)) * 4 : 0;
    const float4 f = *reinterpret_cast<const float4*>(stg + (Cfg::ACCS == 2 ? rep.r : 0) * Cfg::SPLANE +
                                                      r * Cfg::SPITCH + c4);
    unsigned w[4] = {__float_as_uint(f.x), __float_as_uint(f.y), __float_as_uint(f.z), __float_as_uint(f.w)};
    const unsigned idx = (tm * BM + r) * a.N + tn * BN + c4;
    rep.template commit<4, 0>(in ? 0xFu : 0u, idx, w, a.M * a.N, [&](unsigned e, unsigned m, const unsigned* x) {
      if (m == 0xFu)
        __stcs(reinterpret_cast<float4*>(a.C + e), make_float4(__uint_as_float(x[0]), __uint_as_float(x[1]),
                                                                 __uint_as_float(x[2]), __uint_as_float(x[3])));
      else
        for (int k = 0; k < 4; ++k)
          if ((m >> k) & 1u) a.C[e + k] = __uint_as_float(x[k]);
    }, /*defer=*/(i & 3) != 3 && i != ITERS - 1);
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
  int64_t M = b->dims[0], N = b->dims[1], K = b->dims[2], KC = b->dims[3];
  if (b->nbuf < 3 || M <= 0 || N <= 0 || K <= 0 || M % BM || N % 256 || K % BK || n != M * N ||
      M * N >= (1LL << 30) || K >= (1LL << 24) || KC < 0 || KC % BK || !buf_ok(b->buf[0], RMT_BF16, M * K) ||
      !buf_ok(b->buf[1], RMT_BF16, N * K) || !buf_ok(b->buf[2], RMT_F32, M * N)) {
    set_error("matmul: expected {A:BF16[M*K], Bt:BF16[N*K], C:F32[M*N]}, dims {M,N,K,KC}, M%128 = N%256 = 0, "
              "K%64 = 0, KC%64 = 0 (KC = 0: default TMEM chunk)");
    return RMT_EINVAL;
  }
  return RMT_OK;
}
size_t matmul_scratch(int64_t, const int64_t*) { return 0; }
int matmul_inter_warps(int64_t, const int64_t*) { return NTHR / 32; }

int matmul_run(Launch& L) {
  const unsigned M = (unsigned)L.bufs->dims[0], N = (unsigned)L.bufs->dims[1], K = (unsigned)L.bufs->dims[2];
  const unsigned KC = L.bufs->dims[3] > 0 ? (unsigned)L.bufs->dims[3] : (unsigned)KC_DEFAULT;
  return dispatch(L.variant, L.mode, [&](auto vm) {
    constexpr int V = decltype(vm)::V, Mo = decltype(vm)::M;
    using Cfg = MmCfg<V>;
    MmArgs a;
    memset(&a, 0, sizeof(a));
    int rc = make_tmap(&a.tmA, L.bufs->buf[0].ptr, M, K, BM);
    if (rc) return rc;
    rc = make_tmap(&a.tmB, L.bufs->buf[1].ptr, N, K, Cfg::BN);
    if (rc) return rc;
    a.C = (float*)L.bufs->buf[2].ptr;
    a.M = M;
    a.N = N;
    a.K = K;
    a.ntn = N / Cfg::BN;
    a.kpc = KC / BK;
    const unsigned G = (M / BM) * (N / Cfg::BN);
    return launch_std<V>(L, mm_kernel<V, Mo>, mm_kernel<V_NONE, M_NORMAL>, G, Cfg::BL, Cfg::SMEM, a, "matmul",
                         /*mult_inter=*/0, /*mult_cluster=*/0, /*bl_none=*/NTHR);
  });
}

}  // namespace rmt
