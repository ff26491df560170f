// k_blackscholes.cu -- BlackScholes (Fig. 2 "BlkSch"; P:621
// Intra <10% on HD 7790; P:809 Inter ~2x) under every RMT variant.
//
// Logical thread = 4 options (one 16-B vector): r[i..i+3] -> call, put.
// Stores leaving the SoR: 2 vector commits per logical thread (call, put).
// Arithmetic: fp32 with explicit-rounding intrinsics only, so every variant
// executes the identical operation sequence (bit-identity rule).
// Readings R-BS1 (APP-SDK input mapping) and R-BS2 (A&S CND) in DESIGN.md.
// Two input modes (dims[0]): 0 = the APP-SDK workload, one draw r per option
// mapped to (S, K, T, R, sigma) with S == K (R-BS1); 1 = independent
// parameters, five F32 planes S | K | T | R | sigma of n options each (SURVEY
// 8(c) "bs_indep": moneyness ln(S/K) != 0, negative d1/d2, deep ITM / OTM).
#include "rmt_host.cuh"
#ifndef BLKSCH_INTER_MINB
#define BLKSCH_INTER_MINB 8  // inter_group: 8 CTAs of 256 per SM (32 registers): 4.01 -> 3.75x at 2^30
#endif

namespace rmt {
namespace {

constexpr int BL = 256;  // logical threads per CTA
constexpr int VEC = 4;

struct BsArgs {
  const float* r;  // mode 0: r[n]; mode 1: params[5 n] (planes S, K, T, R, sigma)
  float* call;
  float* put;
  unsigned n;
};

// A&S 26.2.17: tail = phi(|x|) k (a1 + k(a2 + k(a3 + k(a4 + k a5)))),
// k = 1/(1 + 0.2316419|x|);  N(x) = 1 - tail (x >= 0), tail (x < 0).
// phi(x) = exp(-x^2/2 - ln sqrt(2 pi)).
__device__ __forceinline__ void cnd_pair(float x, float& nx, float& nmx) {
  const float ax = fabsf(x);
  const float k = __fdividef(1.0f, __fmaf_rn(0.2316419f, ax, 1.0f));  // one MUFU.RCP
  float poly = __fmaf_rn(k, 1.330274429f, -1.821255978f);
  poly = __fmaf_rn(k, poly, 1.781477937f);
  poly = __fmaf_rn(k, poly, -0.356563782f);
  poly = __fmaf_rn(k, poly, 0.319381530f);
  const float phi = __expf(__fmaf_rn(__fmul_rn(-0.5f, ax), ax, -0.918938533204672742f));
  const float tail = __fmul_rn(__fmul_rn(phi, k), poly);
  const float body = __fsub_rn(1.0f, tail);
  nx = x >= 0.0f ? body : tail;
  nmx = x >= 0.0f ? tail : body;
}

// Explicit fp32 operations only (fixed rounding in every variant).  The
// transcendentals are single-MUFU approximate intrinsics (rsqrt, rcp, lg2, ex2:
// ~2 ulp each, far inside the 1e-4 tolerance, and deterministic): 9 MUFU and
// ~35 FMA-pipe operations per option, balanced against 12 B of HBM traffic.
// R-BS1: S = K = 10r + 100(1-r), T = r + 10(1-r), R = .01r + .05(1-r), sigma = .01r + .1(1-r)
struct BsParams {
  float S, K, T, R, sig;
};
__device__ __forceinline__ BsParams bs_map(float r) {
  return BsParams{__fmaf_rn(-90.0f, r, 100.0f), __fmaf_rn(-90.0f, r, 100.0f), __fmaf_rn(-9.0f, r, 10.0f),
                  __fmaf_rn(-0.04f, r, 0.05f), __fmaf_rn(-0.09f, r, 0.10f)};
}

template <int V, int M>
__device__ __forceinline__ void bs_option(const Rep<V, M>& rep, const BsParams& p, long long elem, float& call,
                                          float& put) {
  const float S = p.S, K = p.K, T = p.T, R = p.R, sig = p.sig;
  const float rsT = rsqrtf(T);
  const float sT = __fmul_rn(__fmul_rn(sig, T), rsT);  // sigma sqrt(T)
  // d1 = (ln(S/K) + (R + sigma^2/2) T) / (sigma sqrt T), d2 = d1 - sigma sqrt T
  const float drift = __fmul_rn(__fmaf_rn(__fmul_rn(0.5f, sig), sig, R), T);
  float d1 = __fmul_rn(__fadd_rn(__logf(__fdividef(S, K)), drift), __fdividef(rsT, sig));
  d1 = rep.faultf(SITE_COMPUTE, elem, d1);
  const float d2 = __fsub_rn(d1, sT);
  const float disc = __fmul_rn(K, __expf(__fmul_rn(-R, T)));
  float n1, nm1, n2, nm2;
  cnd_pair(d1, n1, nm1);
  cnd_pair(d2, n2, nm2);
  call = __fmaf_rn(S, n1, -__fmul_rn(disc, n2));
  put = __fmaf_rn(disc, nm2, -__fmul_rn(S, nm1));
}

// 4 consecutive floats of plane `p` at element i0 (tail: 0.5 past n)
__device__ __forceinline__ void load4(const float* p, unsigned i0, unsigned n, float (&x)[VEC]) {
  if (i0 + VEC <= n) {
    float4 v = __ldcs(reinterpret_cast<const float4*>(p + i0));
    x[0] = v.x; x[1] = v.y; x[2] = v.z; x[3] = v.w;
  } else {
#pragma unroll
    for (int k = 0; k < VEC; ++k) x[k] = i0 + k < n ? p[i0 + k] : 0.5f;
  }
}

template <int V, int M, bool IND>
__global__ void __launch_bounds__(BL * Geom<V>::DUP, V == V_INTER ? BLKSCH_INTER_MINB : 0) bs_kernel(BsArgs a, Ctx c) {
  __shared__ unsigned mb[mbox_words<V>(BL * Geom<V>::DUP)];
  Rep<V, M> rep(c);
  rep.init(mb);
  for (; rep.active(); rep.advance()) {
    const unsigned i0 = ((unsigned)rep.lblock * BL + (unsigned)rep.ltid) * VEC;
    unsigned mask = 0;
#pragma unroll
    for (int k = 0; k < VEC; ++k) mask |= (i0 + k < a.n ? 1u : 0u) << k;
    // input replication: each replica loads its own copy
    BsParams prm[VEC];
    if constexpr (!IND) {
      float r4[VEC];
      load4(a.r, i0, a.n, r4);
#pragma unroll
      for (int k = 0; k < VEC; ++k) prm[k] = bs_map(rep.faultf(SITE_LOAD, (long long)i0 + k, r4[k]));
    } else {
      const size_t pl = a.n;  // plane pitch
      float S4[VEC], K4[VEC], T4[VEC], R4[VEC], V4[VEC];
      load4(a.r, i0, a.n, S4);
      load4(a.r + pl, i0, a.n, K4);
      load4(a.r + 2 * pl, i0, a.n, T4);
      load4(a.r + 3 * pl, i0, a.n, R4);
      load4(a.r + 4 * pl, i0, a.n, V4);
#pragma unroll
      for (int k = 0; k < VEC; ++k)
        prm[k] = BsParams{rep.faultf(SITE_LOAD, (long long)i0 + k, S4[k]), K4[k], T4[k], R4[k], V4[k]};
    }
    unsigned cv[VEC], pv[VEC];
#pragma unroll
    for (int k = 0; k < VEC; ++k) {
      float cl, pt;
      bs_option(rep, prm[k], (long long)i0 + k, cl, pt);
      cv[k] = __float_as_uint(cl);
      pv[k] = __float_as_uint(pt);
    }
    auto store_to = [](float* base) {
      return [base](unsigned idx, unsigned m, const unsigned* v) {
        if (m == 0xFu) {
          __stcs(reinterpret_cast<float4*>(base + idx),
                 make_float4(__uint_as_float(v[0]), __uint_as_float(v[1]), __uint_as_float(v[2]), __uint_as_float(v[3])));
        } else {
#pragma unroll
          for (int k = 0; k < VEC; ++k)
            if ((m >> k) & 1u) base[idx + k] = __uint_as_float(v[k]);
        }
      };
    };
    rep.template commit<VEC, 0>(mask, i0, cv, a.n, store_to(a.call), /*defer=*/true);
    rep.template commit<VEC, 1>(mask, i0, pv, a.n, store_to(a.put));
  }
  rep.finish();
}

}  // namespace

int blackscholes_validate(const rmt_bufs_t* b, int64_t n) {
  const int64_t mode = b->dims[0];
  if (b->nbuf < 3 || n < 0 || n > (1LL << 30) || (mode != 0 && mode != 1) ||
      !buf_ok(b->buf[0], RMT_F32, mode ? 5 * n : n) || !buf_ok(b->buf[1], RMT_F32, n) ||
      !buf_ok(b->buf[2], RMT_F32, n) || (mode == 1 && n % 4 != 0)) {
    set_error("blackscholes: expected {r:F32[n] (dims[0]=0) | params:F32[5n] planes S,K,T,R,sigma (dims[0]=1, "
              "n%4 = 0), call:F32[n], put:F32[n]}, n <= 2^30, 16-B aligned");
    return RMT_EINVAL;
  }
  return RMT_OK;
}
size_t blackscholes_scratch(int64_t, const int64_t*) { return 0; }
int blackscholes_inter_warps(int64_t, const int64_t*) { return BL / 32; }

int blackscholes_run(Launch& L) {
  BsArgs a{(const float*)L.bufs->buf[0].ptr, (float*)L.bufs->buf[1].ptr, (float*)L.bufs->buf[2].ptr,
           (unsigned)L.n};
  unsigned G = (unsigned)((L.n + BL * VEC - 1) / (BL * VEC));
  const bool ind = L.bufs->dims[0] == 1;
  return dispatch(L.variant, L.mode, [&](auto vm) {
    constexpr int V = decltype(vm)::V, M = decltype(vm)::M;
    return ind ? launch_std<V>(L, bs_kernel<V, M, true>, bs_kernel<V_NONE, M_NORMAL, true>, G, BL, 0, a,
                               "blackscholes/indep")
               : launch_std<V>(L, bs_kernel<V, M, false>, bs_kernel<V_NONE, M_NORMAL, false>, G, BL, 0, a,
                               "blackscholes");
  });
}

}  // namespace rmt
