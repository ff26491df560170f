// k_binomialoption.cu -- BinomialOption ("BO"; bound by local
// memory traffic on GCN, where Intra-Group-LDS trades redundant compute for an
// equally large communication cost; a FAST-swizzle beneficiary, P:853;
// ~2x when the CU's compute is saturated).
// European call on a Cox-Ross-Rubinstein lattice (readings R-BO1/2): NSTEPS =
// 254, R = 0.02, sigma = 0.30, one U[0,1) draw r per option mapped to
// S = 5(1-r) + 30r, K = (1-r) + 100r, T = 0.25(1-r) + 10r.
//
// B200 design: one option at a time per logical warp, the 256 (255 + 1 pad)
// lattice nodes in registers -- 256/LW per logical lane (8 for a 32-lane warp,
// 16 for an Intra replica's 16-lane warp) -- and each of the 254 backward steps
// is P fused multiply-adds plus ONE register shuffle (the neighbour lane's
// first node).  No shared memory at all (the GCN design's LDS traffic becomes
// register traffic).  A logical warp prices 4 consecutive options and commits
// the 4 prices as one 16-B vector.  fp32 with the risk-neutral probability in
// expm1 form, p = (expm1(R dt) - expm1(-v sqrt dt)) / (expm1(v sqrt dt) -
// expm1(-v sqrt dt)) (no cancellation), accurate expf for the leaves.
#include "rmt_host.cuh"

namespace rmt {
namespace {

constexpr int BL = 128;       // logical threads per CTA
constexpr int NSTEPS = 254;
constexpr int NODES = 256;    // 255 lattice leaves + 1 pad
constexpr float RFREE = 0.02f, VOL = 0.30f;

struct BoArgs {
  const float* r;
  float* call;
  unsigned n;
};

template <int V, int M>
__global__ void __launch_bounds__(BL * Geom<V>::DUP) bo_kernel(BoArgs a, Ctx c) {
  constexpr int DUP = Geom<V>::DUP;
  constexpr int LW = Rep<V, M>::LW;
  constexpr int P = NODES / LW;  // nodes per logical lane
  constexpr int NLW = BL / LW;   // logical warps per CTA
  __shared__ unsigned mb[mbox_words<V>(BL * DUP)];
  Rep<V, M> rep(c);
  rep.init(mb);
  for (; rep.active(); rep.advance()) {
    const unsigned lw = (unsigned)rep.ltid / LW;
    const unsigned o0 = 4u * ((unsigned)rep.lblock * NLW + lw);  // first of this warp's 4 options
    unsigned res[4] = {0u, 0u, 0u, 0u};
#pragma unroll 1
    for (int o = 0; o < 4; ++o) {
      const unsigned opt = o0 + o;
      if (opt >= a.n) break;  // uniform over the logical warp
      float r = __ldg(a.r + opt);
      if constexpr (M == M_FAULT) r = rep.faultf(SITE_LOAD, (long long)opt, r);
      const float om = __fsub_rn(1.0f, r);
      const float S = __fadd_rn(__fmul_rn(5.0f, om), __fmul_rn(30.0f, r));
      const float K = __fadd_rn(om, __fmul_rn(100.0f, r));
      const float T = __fadd_rn(__fmul_rn(0.25f, om), __fmul_rn(10.0f, r));
      const float dt = __fdiv_rn(T, (float)NSTEPS);
      const float vsdt = __fmul_rn(VOL, __fsqrt_rn(dt));
      const float rdt = __fmul_rn(RFREE, dt);
      const float em_up = expm1f(vsdt), em_dn = expm1f(-vsdt);
      float pu = __fdiv_rn(__fsub_rn(expm1f(rdt), em_dn), __fsub_rn(em_up, em_dn));
      if constexpr (M == M_FAULT) pu = rep.faultf(SITE_COMPUTE, (long long)opt, pu);
      const float disc = expf(-rdt);
      const float pur = __fmul_rn(pu, disc), pdr = __fmul_rn(__fsub_rn(1.0f, pu), disc);
      float v[P];
#pragma unroll
      for (int t = 0; t < P; ++t) {
        const int i = rep.llane * P + t;  // leaf index
        const float price = __fmul_rn(S, expf(__fmul_rn(vsdt, (float)(2 * i - NSTEPS))));
        v[t] = i <= NSTEPS ? fmaxf(__fsub_rn(price, K), 0.0f) : 0.0f;
      }
      // backward induction: V_i <- pur V_{i+1} + pdr V_i (nodes >= j are dead and never feed V_0)
#pragma unroll 2
      for (int j = NSTEPS; j > 0; --j) {
        const float nxt = __shfl_down_sync(0xffffffffu, v[0], DUP);  // logical lane + 1, same replica
#pragma unroll
        for (int t = 0; t < P - 1; ++t) v[t] = __fmaf_rn(pur, v[t + 1], __fmul_rn(pdr, v[t]));
        v[P - 1] = __fmaf_rn(pur, nxt, __fmul_rn(pdr, v[P - 1]));
      }
      res[o] = __float_as_uint(v[0]);  // meaningful in logical lane 0
    }
    const unsigned nval = a.n > o0 ? min(4u, a.n - o0) : 0u;
    const unsigned mask = (rep.llane == 0) ? ((1u << nval) - 1u) : 0u;
    rep.template commit<4, 0>(mask, mask ? o0 : 0u, res, a.n, [&](unsigned idx, unsigned m, const unsigned* w) {
      if (m == 0xFu)
        *reinterpret_cast<float4*>(a.call + idx) =
            make_float4(__uint_as_float(w[0]), __uint_as_float(w[1]), __uint_as_float(w[2]), __uint_as_float(w[3]));
      else
        for (int k = 0; k < 4; ++k)
          if ((m >> k) & 1u) a.call[idx + k] = __uint_as_float(w[k]);
    });
  }
  rep.finish();
}

}  // namespace

int binomialoption_validate(const rmt_bufs_t* b, int64_t n) {
  if (b->nbuf < 2 || n < 0 || n > (1LL << 28) || !buf_ok(b->buf[0], RMT_F32, n) || !buf_ok(b->buf[1], RMT_F32, n)) {
    set_error("binomialoption: expected {r:F32[n], call:F32[n]}, n <= 2^28");
    return RMT_EINVAL;
  }
  return RMT_OK;
}
size_t binomialoption_scratch(int64_t, const int64_t*) { return 0; }
int binomialoption_inter_warps(int64_t, const int64_t*) { return BL / 32; }

int binomialoption_run(Launch& L) {
  BoArgs a{(const float*)L.bufs->buf[0].ptr, (float*)L.bufs->buf[1].ptr, (unsigned)L.n};
  return dispatch(L.variant, L.mode, [&](auto vm) {
    constexpr int V = decltype(vm)::V, M = decltype(vm)::M;
    constexpr int LW = Rep<V, M>::LW;
    const unsigned per_cta = 4u * (BL / LW);
    const unsigned G = (unsigned)((L.n + per_cta - 1) / per_cta);
    return launch_std<V>(L, bo_kernel<V, M>, bo_kernel<V_NONE, M_NORMAL>, G, BL, 0, a, "binomialoption");
  });
}

}  // namespace rmt
