// k_fwt.cu -- FastWalshTransform ("FWT"; memory-bound, Intra
// <=10% on HD 7790; an Inter outlier >7x).
// y = H_N x, natural order, unnormalised (reading R-FWT1): log2 N radix-2
// stages h = 1, 2, ..., N/2, butterfly (a, b) -> (a + b, a - b).
//
// B200 design: the stages are fused into passes over 4096-element tiles staged
// in (duplicated, +LDS) shared memory.  Pass 1 runs stages 0..11 on contiguous
// tiles; later passes run up to 7 stages on tiles of 2^b strided rows x 2^c
// contiguous columns (c >= 5 -> 128-B coalesced rows).  Inside a pass, stages
// run as register rounds of up to 4 stages (16 elements per thread).  The
// butterfly DAG -- hence every fp32 rounding -- is fixed by the stage order
// alone, so every variant and every fusion is bit-identical to the fp32-DAG
// oracle (reading R-FWT2).  HBM traffic: 8 B/elem per pass.
// Inter-Group polls spin without back-off in this kernel (measured with the
// digest records: inter_group 3.10 -> 2.89x)
#define RMT_SPIN_NS0 0
#include "rmt_host.cuh"
#ifndef FWT_INTER_MINB
#define FWT_INTER_MINB 10  // inter_group: 10 CTAs of 128 per SM (51 registers; measured 3.05 -> 2.73x vs 72 registers)
#endif

namespace rmt {
namespace {

constexpr int BL = 256;
constexpr int TB_MAX = 12;
constexpr int TE_MAX = 1 << TB_MAX;
// Tile swizzle.  One replica per warp lane (none, inter): pad one word per 32
// ("pad32"), conflict-free for the 32-thread patterns of every round.  Two
// replicas per warp (+LDS intra variants, P16): each replica has 16 logical
// threads; pad one word per 16 makes every round's 16-thread pattern hit 16
// banks whose complement is the same set + 16, so the replica planes sit 16
// banks apart (PLANE = 16 mod 32) and a pair never conflicts.
template <bool P16>
struct Swz {
  static constexpr int WORDS = TE_MAX + TE_MAX / (P16 ? 16 : 32);
  static constexpr int PLANE = WORDS + 16;  // replica plane offset (== 16 mod 32)
  static __device__ __forceinline__ int phys(int e) { return e + (e >> (P16 ? 4 : 5)); }
  // phys(ebase | k << Q) - phys(ebase) for ebase with zeros in bits Q..Q+3
  template <int Q>
  static __device__ __forceinline__ constexpr int coff(int k) {
    if constexpr (P16) return (k << Q) + ((k << Q) >> 4);
    else return (k << Q) + ((Q >= 5) ? (k << (Q - 5)) : ((k << Q) >> 5));
  }
};

// Radix-2^NB butterfly network on registers, stages h = 1, 2, .., 2^(NB-1)
// (the normative stage order, R-FWT2).  Two butterflies of a stage share one
// packed FADD2 for the sums and one for the differences (add/sub.rn.f32x2:
// lane-wise RN(a + b), RN(a - b), bit-identical to __fadd_rn / __fsub_rn),
// halving the FP instructions of the issue-bound RMT variants.
__device__ __forceinline__ unsigned long long f2pack(float lo, float hi) {
  unsigned long long r;
  asm("mov.b64 %0, {%1, %2};" : "=l"(r) : "f"(lo), "f"(hi));
  return r;
}
__device__ __forceinline__ void f2unpack(unsigned long long v, float& lo, float& hi) {
  asm("mov.b64 {%0, %1}, %2;" : "=f"(lo), "=f"(hi) : "l"(v));
}
template <int NB>
__device__ __forceinline__ void butterflies(float (&v)[1 << NB]) {
  constexpr int G = 1 << NB;
  if constexpr (NB == 1) {
    const float x0 = v[0], x1 = v[1];
    v[0] = __fadd_rn(x0, x1);
    v[1] = __fsub_rn(x0, x1);
  } else {
    // P[j] = {v[j], v[j + G/2]}: stages h < G/2 act on both halves alike, so
    // they run on the packed pairs with the natural pairing (no register
    // shuffling between stages); the last stage (h = G/2) is lo +- hi
    constexpr int H = G / 2;
    unsigned long long P[H];
#pragma unroll
    for (int j = 0; j < H; ++j) P[j] = f2pack(v[j], v[j + H]);
#pragma unroll
    for (int s = 0; s < NB - 1; ++s) {
      const int h = 1 << s;
#pragma unroll
      for (int j = 0; j < H; ++j) {
        if (j & h) continue;
        const unsigned long long x0 = P[j], x1 = P[j + h];
        asm("add.rn.f32x2 %0, %1, %2;" : "=l"(P[j]) : "l"(x0), "l"(x1));
        asm("sub.rn.f32x2 %0, %1, %2;" : "=l"(P[j + h]) : "l"(x0), "l"(x1));
      }
    }
#pragma unroll
    for (int j = 0; j < H; ++j) {
      float lo, hi;
      f2unpack(P[j], lo, hi);
      v[j] = __fadd_rn(lo, hi);
      v[j + H] = __fsub_rn(lo, hi);
    }
  }
}

struct FwtArgs {
  const float* src;
  float* dst;
  unsigned N;
  int tb;  // tile bits (TE = 2^tb)
  int s0;  // first stage (bit position in the global index)
  int b;   // stages in this pass
  int c;   // contiguous column bits in the tile (0 for pass 1)
};

__device__ __forceinline__ unsigned gindex(const FwtArgs& a, unsigned tile, unsigned e) {
  if (a.s0 == 0) return (tile << a.tb) | e;
  const unsigned col = e & ((1u << a.c) - 1u), st = e >> a.c;
  const int midb = a.s0 - a.c;
  const unsigned mid = tile & ((1u << midb) - 1u), hi = tile >> midb;
  return (hi << (a.s0 + a.b)) | (st << a.s0) | (mid << a.c) | col;
}

// gindex with the pass shape known at compile time (KIND 1: s0 = 0, tb = 12;
// KIND 2: b = 7, c = 5)
template <int KIND>
__device__ __forceinline__ unsigned gindex_k(const FwtArgs& a, unsigned tile, unsigned e) {
  if constexpr (KIND == 1) {
    return (tile << TB_MAX) | e;
  } else if constexpr (KIND == 2) {
    const unsigned col = e & 31u, st = e >> 5;
    const int midb = a.s0 - 5;
    const unsigned mid = tile & ((1u << midb) - 1u), hi = tile >> midb;
    return (hi << (a.s0 + 7)) | (st << a.s0) | (mid << 5) | col;
  } else {
    return gindex(a, tile, e);
  }
}

// One register round: NB consecutive stages at tile-bit q on groups of 2^NB.
template <int NB, class R>
__device__ __forceinline__ void fwt_round(const R& rep, float* tp, int q, int te, const FwtArgs& a, unsigned tileid,
                                          int round_no) {
  constexpr int G = 1 << NB;
  using S = Swz<R::SMDUP>;
  const int groups = te >> NB;
  for (int gi = rep.ltid; gi < groups; gi += BL) {
    const int lowmask = (1 << q) - 1;
    const int ebase = (gi & lowmask) | ((gi >> q) << (q + NB));
    float v[G];
#pragma unroll
    for (int k = 0; k < G; ++k) {
      v[k] = tp[S::phys(ebase | (k << q))];
      if constexpr (R::FAULT) {
        if (a.s0 == 0 && round_no == 1)
          v[k] = rep.faultf(SITE_SMEM, (long long)gindex(a, tileid, ebase | (k << q)), v[k]);
      }
    }
    butterflies<NB>(v);
    unsigned vw[G];
#pragma unroll
    for (int k = 0; k < G; ++k) {
      if constexpr (R::FAULT) {
        if (a.s0 == 0 && round_no == 0)
          v[k] = rep.faultf(SITE_COMPUTE, (long long)gindex(a, tileid, ebase | (k << q)), v[k]);
      }
      vw[k] = __float_as_uint(v[k]);
    }
    if (rep.template sts_ok<G>(vw, (unsigned)ebase)) {
#pragma unroll
      for (int k = 0; k < G; ++k) tp[S::phys(ebase | (k << q))] = v[k];
    }
  }
}

// Compile-time round (full 4096-element tile): with Q known, phys(ebase | k<<Q)
// = phys(ebase) + C(k) with a constant C(k) (ebase has zeros in bits Q..Q+NB),
// so every element costs one LDS and one STS with an immediate offset.
template <int NB, int Q, class R>
__device__ __forceinline__ void fwt_round_ct(const R& rep, float* tp, const FwtArgs& a, unsigned tileid,
                                             int round_no) {
  constexpr int G = 1 << NB;
  constexpr int GPT = (TE_MAX >> NB) / BL;  // groups per thread
  using S = Swz<R::SMDUP>;
#pragma unroll
  for (int w = 0; w < GPT; ++w) {
    const int gi = rep.ltid + BL * w;
    const int ebase = (gi & ((1 << Q) - 1)) | ((gi >> Q) << (Q + NB));
    float* pb = tp + S::phys(ebase);
    float v[G];
#pragma unroll
    for (int k = 0; k < G; ++k) {
      v[k] = pb[S::template coff<Q>(k)];
      if constexpr (R::FAULT) {
        if (a.s0 == 0 && round_no == 1)
          v[k] = rep.faultf(SITE_SMEM, (long long)gindex(a, tileid, ebase | (k << Q)), v[k]);
      }
    }
    butterflies<NB>(v);
    unsigned vw[G];
#pragma unroll
    for (int k = 0; k < G; ++k) {
      if constexpr (R::FAULT) {
        if (a.s0 == 0 && round_no == 0)
          v[k] = rep.faultf(SITE_COMPUTE, (long long)gindex(a, tileid, ebase | (k << Q)), v[k]);
      }
      vw[k] = __float_as_uint(v[k]);
    }
    if (rep.template sts_ok<G>(vw, (unsigned)ebase)) {
#pragma unroll
      for (int k = 0; k < G; ++k) pb[S::template coff<Q>(k)] = v[k];
    }
  }
}

// KIND 0: generic (any tile size / stage range, runtime rounds)
// KIND 1: pass 1 on full 4096-element tiles (stages 0..11: rounds at q = 0, 4, 8)
// KIND 2: strided pass with b = 7, c = 5 (rounds at q = 5 (4 stages), q = 9 (3 stages))
template <int V, int M, int KIND>
__global__ void __launch_bounds__(BL * Geom<V>::DUP) fwt_kernel(FwtArgs a, Ctx c) {
  constexpr int DUP = Geom<V>::DUP;
  using S = Swz<Rep<V, M>::SMDUP>;
  constexpr int PLANE = S::PLANE;
  __shared__ unsigned mb[mbox_words<V>(BL * DUP)];
  __shared__ float tile[Geom<V>::SMDUP == 2 ? PLANE + S::WORDS : S::WORDS];
  Rep<V, M, true> rep(c);  // group flags: up to 8 records per warp
  rep.init(mb);
  for (; rep.active(); rep.advance()) {
    const unsigned tileid = (unsigned)rep.lblock;
    const int te = KIND != 0 ? TE_MAX : 1 << a.tb;  // full tiles in the specialised passes
    float* const tp = &rep.template smp<PLANE>(tile, 0);  // this replica's plane
    // load: 16-B vectors, contiguous in both the tile and global memory
    auto put4 = [&](int e0, unsigned g, float (&w)[4]) {
      unsigned xw[4];
#pragma unroll
      for (int k = 0; k < 4; ++k) {
        if constexpr (M == M_FAULT) {
          if (a.s0 == 0 && e0 + k < te) w[k] = rep.faultf(SITE_LOAD, (long long)g + k, w[k]);
        }
        xw[k] = __float_as_uint(w[k]);
      }
      if (rep.template sts_ok<4>(xw, (unsigned)e0)) {
#pragma unroll
        for (int k = 0; k < 4; ++k)
          if (KIND != 0 || e0 + k < te) tp[S::phys(e0 + k)] = w[k];
      }
    };
    if constexpr (KIND != 0) {
      // full tile: all of this thread's loads in flight before the first use
      constexpr int IT = TE_MAX / (4 * BL);
      float4 f[IT];
#pragma unroll
      for (int it = 0; it < IT; ++it)
        f[it] = *reinterpret_cast<const float4*>(a.src + gindex_k<KIND>(a, tileid, (unsigned)(4 * rep.ltid + it * 4 * BL)));
#pragma unroll
      for (int it = 0; it < IT; ++it) {
        const int e0 = 4 * rep.ltid + it * 4 * BL;
        float w[4] = {f[it].x, f[it].y, f[it].z, f[it].w};
        put4(e0, gindex_k<KIND>(a, tileid, (unsigned)e0), w);
      }
    } else {
      for (int e0 = 4 * rep.ltid; e0 < te; e0 += 4 * BL) {
        const unsigned g = gindex(a, tileid, (unsigned)e0);
        float w[4];
        if (te >= 4) {
          float4 f = *reinterpret_cast<const float4*>(a.src + g);
          w[0] = f.x; w[1] = f.y; w[2] = f.z; w[3] = f.w;
        } else {
#pragma unroll
          for (int k = 0; k < 4; ++k) w[k] = e0 + k < te ? a.src[g + k] : 0.0f;
        }
        put4(e0, g, w);
      }
    }
    __syncthreads();
    // stages [s0, s0 + b) live at tile bits [c, c + b); rounds of <= 4 stages
    if constexpr (KIND == 1) {
      fwt_round_ct<4, 0>(rep, tp, a, tileid, 0);
      __syncthreads();
      fwt_round_ct<4, 4>(rep, tp, a, tileid, 1);
      __syncthreads();
      fwt_round_ct<4, 8>(rep, tp, a, tileid, 2);
      __syncthreads();
    } else if constexpr (KIND == 2) {
      fwt_round_ct<4, 5>(rep, tp, a, tileid, 0);
      __syncthreads();
      fwt_round_ct<3, 9>(rep, tp, a, tileid, 1);
      __syncthreads();
    } else {
      int round_no = 0;
      for (int q = a.c; q < a.c + a.b; q += 4, ++round_no) {
        const int nb = min(4, a.c + a.b - q);
        switch (nb) {
          case 4: fwt_round<4>(rep, tp, q, te, a, tileid, round_no); break;
          case 3: fwt_round<3>(rep, tp, q, te, a, tileid, round_no); break;
          case 2: fwt_round<2>(rep, tp, q, te, a, tileid, round_no); break;
          default: fwt_round<1>(rep, tp, q, te, a, tileid, round_no); break;
        }
        __syncthreads();
      }
    }
    // store: one vector commit per 4 elements
#pragma unroll 1
    for (int it = 0; it < TE_MAX / (4 * BL); ++it) {
      const int e0 = 4 * rep.ltid + it * 4 * BL;
      unsigned w[4];
      unsigned mask = 0;
#pragma unroll
      for (int k = 0; k < 4; ++k) {
        const bool in = KIND != 0 || e0 + k < te;  // specialised passes: full tiles
        w[k] = in ? __float_as_uint(tp[S::phys(e0 + k)]) : 0u;
        mask |= (in ? 1u : 0u) << k;
      }
      const unsigned g = e0 < te ? gindex_k<KIND>(a, tileid, (unsigned)e0) : 0u;
      rep.template commit<4, 0>(mask, g, w, a.N, [&](unsigned idx, unsigned m, const unsigned* x) {
        if (m == 0xFu)
          *reinterpret_cast<float4*>(a.dst + idx) =
              make_float4(__uint_as_float(x[0]), __uint_as_float(x[1]), __uint_as_float(x[2]), __uint_as_float(x[3]));
        else
          for (int k = 0; k < 4; ++k)
            if ((m >> k) & 1u) a.dst[idx + k] = __uint_as_float(x[k]);
      }, /*defer=*/it < TE_MAX / (4 * BL) - 1);
    }
  }
  rep.finish();
}

// ---------------------------------------------------------------- specialised passes
// Tiles of 4096 elements, BLS = 128 logical threads x 32 elements.  Register
// rounds of up to 5 stages; the first round of each pass runs on the loaded
// registers and the last writes straight to global memory, so a pass touches
// shared memory only between rounds:
//   pass 1  (stages 0..11, contiguous tile):  float4 load -> stages 0,1 in
//           registers -> STS -> round A (stages 2..6, 32 elements at stride 4)
//           -> round B (stages 7..11, 32 elements at stride 128) -> STG
//           (2 STS + 2 LDS per element instead of 4 + 4);
//   strided (7 stages on the 128 rows of a 128 x 32 tile): 32 row loads per
//           thread (each warp load = one 128-B row) -> stages on row bits 0..4 in
//           registers -> STS -> stages on row bits 5, 6 (4 elements) -> STG
//           (1 STS + 1 LDS per element instead of 3 + 3).
// Stores are 4-word commits of elements at a fixed stride (each warp store
// instruction covers 128 contiguous bytes).
constexpr int BLS = 128;

// Pass-1 layouts.  Three access patterns: staging (float4 chunk t + 128 it),
// round A (e = (t & 3) + 4k + 128 (t >> 2)), round B (e = t + 128 k).
//  * none: XOR swizzle p1x(e) = e ^ ((e >> 5) & 31), a bank permutation for
//    each pattern over 32 lanes (measured 0.264 vs 0.283 ms at 2^26 against the
//    pad layout below: the address arithmetic spaces out the shared-memory
//    instructions of the unprotected kernel).
//  * RMT variants: pad layout (measured faster for every one of them)
//    p1_phys(e) = e + 4 (e >> 7) (one 16-B pad per 128 words): float4 chunks
//    stay aligned (staging is one STS.128), every pattern is conflict-free, and
//    it is additive over the disjoint bit fields of a thread's base and the
//    compile-time k (immediate offsets: fewer issued instructions, which is
//    what bounds the doubled intra kernels).  +LDS replica planes sit P1_PLANE
//    (== 16 mod 32) words apart: a warp's 16 logical lanes cover 16
//    consecutive banks in rounds A and B and 4 chunks per quarter-warp in
//    staging, so the two replicas of a pair never share a bank.
constexpr int P1_WORDS = TE_MAX + TE_MAX / 32;
constexpr int P1_PLANE = P1_WORDS + 16;
__device__ __forceinline__ constexpr int p1_phys(int e) { return e + 4 * (e >> 7); }
__device__ __forceinline__ int p1x(int e) { return e ^ ((e >> 5) & 31); }


template <int V, int M>
__global__ void __launch_bounds__(BLS * Geom<V>::DUP, V == V_INTER ? FWT_INTER_MINB : 0) fwt_p1_kernel(FwtArgs a, Ctx c) {
  using R = Rep<V, M, true>;  // group flags: 8 records per warp
  constexpr bool DUPL = R::SMDUP;
  constexpr bool PAD = V != V_NONE;  // layout choice (see p1_phys / p1x): measured per variant
  __shared__ unsigned mb[mbox_words<V>(BLS * Geom<V>::DUP)];
  __shared__ __align__(16) float tile[DUPL ? P1_PLANE + P1_WORDS : P1_WORDS];
  R rep(c);
  rep.init(mb);
  for (; rep.active(); rep.advance()) {
    const unsigned tileid = (unsigned)rep.lblock;
    const unsigned gbase = tileid << TB_MAX;
    float* const tp = tile + (DUPL ? P1_PLANE * rep.r : 0);  // this replica's plane
    const int t = rep.ltid;
    // load: 8 coalesced float4 per thread, all in flight before the first use
    float4 f[8];
#pragma unroll
    for (int it = 0; it < 8; ++it) f[it] = *reinterpret_cast<const float4*>(a.src + gbase + 4 * t + 512 * it);
    float* const ps = tp + p1_phys(4 * t);  // + p1_phys(512 it) + k: compile-time offsets
#pragma unroll
    for (int it = 0; it < 8; ++it) {
      const int e0 = 4 * t + 512 * it;
      float v[4] = {f[it].x, f[it].y, f[it].z, f[it].w};
      if constexpr (M == M_FAULT) {
#pragma unroll
        for (int k = 0; k < 4; ++k) v[k] = rep.faultf(SITE_LOAD, (long long)gbase + e0 + k, v[k]);
      }
      butterflies<2>(v);  // stages 0, 1 (element bits 0, 1)
      unsigned w[4];
#pragma unroll
      for (int k = 0; k < 4; ++k) {
        if constexpr (M == M_FAULT) v[k] = rep.faultf(SITE_COMPUTE, (long long)gbase + e0 + k, v[k]);
        w[k] = __float_as_uint(v[k]);
      }
      if (rep.template sts_ok<4>(w, (unsigned)e0)) {
        if constexpr (PAD) {
          *reinterpret_cast<float4*>(ps + p1_phys(512 * it)) = make_float4(v[0], v[1], v[2], v[3]);
        } else {
#pragma unroll
          for (int k = 0; k < 4; ++k) tp[p1x(e0 + k)] = v[k];
        }
      }
    }
    __syncthreads();
    {  // round A: stages 2..6 on elements ebase + 4k
      const int ebase = (t & 3) | ((t >> 2) << 7);
      float* const pb = tp + p1_phys(ebase);  // + p1_phys(4k): compile-time offsets
      auto at = [&](int k) -> float& { return PAD ? pb[p1_phys(4 * k)] : tp[p1x(ebase + 4 * k)]; };
      float v[32];
#pragma unroll
      for (int k = 0; k < 32; ++k) {
        v[k] = at(k);
        if constexpr (M == M_FAULT) v[k] = rep.faultf(SITE_SMEM, (long long)gbase + ebase + 4 * k, v[k]);
      }
      butterflies<5>(v);
      unsigned w[32];
#pragma unroll
      for (int k = 0; k < 32; ++k) w[k] = __float_as_uint(v[k]);
      // each thread reads and rewrites its own 32 elements: no barrier inside the round
      if (rep.template sts_ok<32>(w, (unsigned)ebase)) {
#pragma unroll
        for (int k = 0; k < 32; ++k) at(k) = v[k];
      }
    }
    __syncthreads();
    // round B: stages 7..11 on elements t + 128k, then 8 strided commits
    float* const pt = tp + p1_phys(t);
    float v[32];
#pragma unroll
    for (int k = 0; k < 32; ++k) v[k] = PAD ? pt[p1_phys(128 * k)] : tp[p1x(t + 128 * k)];
    butterflies<5>(v);
#pragma unroll
    for (int j = 0; j < 8; ++j) {
      unsigned w[4];
#pragma unroll
      for (int u = 0; u < 4; ++u) w[u] = __float_as_uint(v[4 * j + u]);
      rep.template commit<4, 0>(0xFu, gbase + t + 512 * j, w, a.N, [&](unsigned idx, unsigned m, const unsigned* x) {
#pragma unroll
        for (int u = 0; u < 4; ++u)
          if ((m >> u) & 1u) a.dst[idx + 128 * u] = __uint_as_float(x[u]);
      }, /*defer=*/j < 7, /*stride=*/128u);
    }
  }
  rep.finish();
}

// Strided pass: stages [s0, s0 + 7) on tiles of 128 rows (global stride 2^s0)
// x 32 contiguous columns.  Layout e = col | row << 5 (bank = col), replica
// planes XOR bank bit 4 (a warp's 16 logical lanes share it).
template <int V, int M>
__global__ void __launch_bounds__(BLS * Geom<V>::DUP, V == V_INTER ? FWT_INTER_MINB : 0) fwt_ps_kernel(FwtArgs a, Ctx c) {
  using R = Rep<V, M, true>;  // group flags: 8 records per warp
  constexpr bool DUPL = R::SMDUP;
  __shared__ unsigned mb[mbox_words<V>(BLS * Geom<V>::DUP)];
  __shared__ float tile[TE_MAX * Geom<V>::SMDUP];
  R rep(c);
  rep.init(mb);
  for (; rep.active(); rep.advance()) {
    const unsigned tileid = (unsigned)rep.lblock;
    const int t = rep.ltid;
    const int col = t & 31, g = t >> 5;
    // this replica's plane, column pre-applied (bank bit 4 flipped for replica 1):
    // element (col, row) is tc[row << 5], a compile-time offset from a per-thread base
    float* const tc = tile + (DUPL ? TE_MAX * rep.r : 0) + (col ^ (DUPL && rep.r ? 16 : 0));
    // global index of tile element (col, row): row bits land at s0.. (gindex_k<2>)
    const int midb = a.s0 - 5;
    const unsigned gcol = ((tileid >> midb) << (a.s0 + 7)) | ((tileid & ((1u << midb) - 1u)) << 5) | (unsigned)col;
    // rows 32 g + i, i = 0..31: one 128-B row per warp load
    float v[32];
#pragma unroll
    for (int i = 0; i < 32; ++i) v[i] = a.src[gcol + ((unsigned)(32 * g + i) << a.s0)];
    butterflies<5>(v);  // stages s0 .. s0+4 (row bits 0..4)
    unsigned w[32];
#pragma unroll
    for (int i = 0; i < 32; ++i) w[i] = __float_as_uint(v[i]);
    if (rep.template sts_ok<32>(w, (unsigned)(col | (32 * g) << 5))) {
#pragma unroll
      for (int i = 0; i < 32; ++i) tc[(32 * g + i) << 5] = v[i];
    }
    __syncthreads();
    // stages s0+5, s0+6 (row bits 5, 6): 8 groups of 4 rows {rlo + 32 k}
#pragma unroll
    for (int j = 0; j < 8; ++j) {
      const int rlo = g + 4 * j;
      float q[4];
#pragma unroll
      for (int k = 0; k < 4; ++k) q[k] = tc[(rlo + 32 * k) << 5];
      butterflies<2>(q);
      unsigned x[4];
#pragma unroll
      for (int k = 0; k < 4; ++k) x[k] = __float_as_uint(q[k]);
      const unsigned stride = 1u << (a.s0 + 5);
      rep.template commit<4, 0>(0xFu, gcol + ((unsigned)rlo << a.s0), x, a.N,
                                [&](unsigned idx, unsigned m, const unsigned* y) {
#pragma unroll
                                  for (int k = 0; k < 4; ++k)
                                    if ((m >> k) & 1u) a.dst[idx + stride * k] = __uint_as_float(y[k]);
                                }, /*defer=*/j < 7, stride);
    }
  }
  rep.finish();
}

// Cross-shard butterfly stage of a multi-GPU FWT (local FWHT of
// N/G, then log2 G stages whose pairs (i, i + h) sit on two GPUs): this rank
// holds x = its shard, p = the partner shard; the lower rank of the pair keeps
// a + b = x + p, the upper keeps a - b = p - x, the same fp32 operations (and
// operand order) as the single-GPU stage h, so the sharded result is bitwise the
// single-GPU one.  Logical thread = 4 consecutive elements, one vector commit.
struct FwtCombArgs {
  const float* x;
  const float* p;
  float* y;
  unsigned n;
  unsigned upper;
};

constexpr int BLC = 256;

template <int V, int M>
__global__ void __launch_bounds__(BLC * Geom<V>::DUP) fwt_combine_kernel(FwtCombArgs a, Ctx c) {
  __shared__ unsigned mb[mbox_words<V>(BLC * Geom<V>::DUP)];
  Rep<V, M> rep(c);
  rep.init(mb);
  for (; rep.active(); rep.advance()) {
    const unsigned i0 = ((unsigned)rep.lblock * BLC + (unsigned)rep.ltid) * 4u;
    unsigned w[4];
    unsigned mask = 0;
    if (i0 + 4 <= a.n) {  // input replication: each replica loads both operands itself
      const float4 xv = __ldcs(reinterpret_cast<const float4*>(a.x + i0));
      const float4 pv = __ldcs(reinterpret_cast<const float4*>(a.p + i0));
      const float xs[4] = {xv.x, xv.y, xv.z, xv.w}, ps[4] = {pv.x, pv.y, pv.z, pv.w};
#pragma unroll
      for (int k = 0; k < 4; ++k) {
        const float xk = rep.faultf(SITE_LOAD, (long long)i0 + k, xs[k]);
        w[k] = __float_as_uint(a.upper ? __fsub_rn(ps[k], xk) : __fadd_rn(xk, ps[k]));
      }
      mask = 0xFu;
    } else {
#pragma unroll
      for (int k = 0; k < 4; ++k) {
        const bool in = i0 + k < a.n;
        const float xk = rep.faultf(SITE_LOAD, (long long)i0 + k, in ? a.x[i0 + k] : 0.0f);
        const float pk = in ? a.p[i0 + k] : 0.0f;
        w[k] = __float_as_uint(a.upper ? __fsub_rn(pk, xk) : __fadd_rn(xk, pk));
        mask |= (in ? 1u : 0u) << k;
      }
    }
    rep.template commit<4, 0>(mask, i0, w, a.n, [&](unsigned idx, unsigned m, const unsigned* v) {
      if (m == 0xFu)
        __stcs(reinterpret_cast<float4*>(a.y + idx),
               make_float4(__uint_as_float(v[0]), __uint_as_float(v[1]), __uint_as_float(v[2]), __uint_as_float(v[3])));
      else
        for (int k = 0; k < 4; ++k)
          if ((m >> k) & 1u) a.y[idx + k] = __uint_as_float(v[k]);
    });
  }
  rep.finish();
}

int log2u(int64_t n) {
  int m = 0;
  while ((1LL << m) < n) ++m;
  return m;
}

}  // namespace

int fwt_validate(const rmt_bufs_t* b, int64_t n) {
  const int64_t mode = b->dims[0];
  if (b->nbuf < 2 || n < 1 || n > (1LL << 30) || (n & (n - 1)) || !buf_ok(b->buf[0], RMT_F32, n) ||
      !buf_ok(b->buf[1], RMT_F32, n) || (mode != 0 && mode != 1) ||
      (mode == 1 && (b->nbuf < 3 || !buf_ok(b->buf[2], RMT_F32, n) || (b->dims[1] != 0 && b->dims[1] != 1)))) {
    set_error("fwt: expected {x,y} F32[N], N a power of two in [1, 2^30] (dims[0] = 0); or the cross-shard stage "
              "{x, y, p} F32[N] with dims {1, upper}");
    return RMT_EINVAL;
  }
  return RMT_OK;
}
size_t fwt_scratch(int64_t, const int64_t*) { return 0; }
int fwt_inter_warps(int64_t, const int64_t*) { return BL / 32; }

int fwt_run(Launch& L) {
  if (L.bufs->dims[0] == 1) {  // cross-shard butterfly stage (multi-GPU)
    FwtCombArgs a{(const float*)L.bufs->buf[0].ptr, (const float*)L.bufs->buf[2].ptr, (float*)L.bufs->buf[1].ptr,
                  (unsigned)L.n, (unsigned)L.bufs->dims[1]};
    const unsigned G = (unsigned)((L.n + 4 * BLC - 1) / (4 * BLC));
    return dispatch(L.variant, L.mode, [&](auto vm) {
      constexpr int V = decltype(vm)::V, M = decltype(vm)::M;
      return launch_std<V>(L, fwt_combine_kernel<V, M>, fwt_combine_kernel<V_NONE, M_NORMAL>, G, BLC, 0, a,
                           "fwt/combine");
    });
  }
  const int m = log2u(L.n);
  const int tb = m < TB_MAX ? m : TB_MAX;
  const float* x = (const float*)L.bufs->buf[0].ptr;
  float* y = (float*)L.bufs->buf[1].ptr;
  return dispatch(L.variant, L.mode, [&](auto vm) {
    constexpr int V = decltype(vm)::V, M = decltype(vm)::M;
    const unsigned tiles = (unsigned)(L.n >> tb);
    // STORE_* fault sites target the final pass (the stored y); LOAD/COMPUTE/SMEM
    // sites target pass 1 (gated in the kernel by s0 == 0).
    const int sid = L.ctx.f.sid;
    L.ctx.f.sid = (tb < m) ? -1 : sid;
    FwtArgs a{x, y, (unsigned)L.n, tb, 0, tb, 0};
    int rc = tb == TB_MAX
                 ? launch_std<V>(L, fwt_p1_kernel<V, M>, fwt_p1_kernel<V_NONE, M_NORMAL>, tiles, BLS, 0, a, "fwt/pass1")
                 : launch_std<V>(L, fwt_kernel<V, M, 0>, fwt_kernel<V_NONE, M_NORMAL, 0>, tiles, BL, 0, a, "fwt/pass1");
    for (int s = tb; s < m && rc == RMT_OK; ) {  // strided passes, in place on y
      const int b = (m - s) < 7 ? (m - s) : 7;
      L.ctx.f.sid = (s + b < m) ? -1 : sid;
      FwtArgs p{y, y, (unsigned)L.n, TB_MAX, s, b, TB_MAX - b};
      rc = b == 7 ? launch_std<V>(L, fwt_ps_kernel<V, M>, fwt_ps_kernel<V_NONE, M_NORMAL>, tiles, BLS, 0, p, "fwt/pass")
                  : launch_std<V>(L, fwt_kernel<V, M, 0>, fwt_kernel<V_NONE, M_NORMAL, 0>, tiles, BL, 0, p, "fwt/pass");
      s += b;
    }
    L.ctx.f.sid = sid;
    return rc;
  });
}

}  // namespace rmt
