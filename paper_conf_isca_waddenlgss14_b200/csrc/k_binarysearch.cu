// k_binarysearch.cu -- BinarySearch ("BinS"; memory-bound,
// Intra <=10%).  Batched lower_bound (reading R-BIN1):
// idx[j] = #{i : A[i] < q[j]}.
//
// Logical thread = 4 queries (16-B load of q, 4 interleaved searches for
// memory-level parallelism, one 16-B vector commit of idx).  The search is
// branch-free with a trip count that depends on N only, so every lane of a warp
// runs the same number of iterations.  The top levels of the implicit tree are
// few distinct addresses and stay L1/L2-resident; the bottom levels are random
// 32-B sectors (latency-bound).
#include "rmt_host.cuh"

namespace rmt {
namespace {

constexpr int BL = 256;
constexpr int VEC = 4;

struct BsArgs {
  const unsigned* A;
  const unsigned* q;
  unsigned* idx;
  unsigned N, Q;
  int iters;  // ceil(log2 N)
};

template <int V, int M>
__global__ void __launch_bounds__(BL * Geom<V>::DUP) bins_kernel(BsArgs a, Ctx c) {
  __shared__ unsigned mb[mbox_words<V>(BL * Geom<V>::DUP)];
  Rep<V, M> rep(c);
  rep.init(mb);
  const unsigned j0 = ((unsigned)rep.lblock * BL + (unsigned)rep.ltid) * VEC;
  unsigned key[VEC];
  unsigned mask = 0;
  if (j0 + VEC <= a.Q) {
    uint4 w = __ldcs(reinterpret_cast<const uint4*>(a.q + j0));
    key[0] = w.x; key[1] = w.y; key[2] = w.z; key[3] = w.w;
    mask = 0xFu;
  } else {
#pragma unroll
    for (int k = 0; k < VEC; ++k) {
      const bool in = j0 + k < a.Q;
      key[k] = in ? a.q[j0 + k] : 0u;
      mask |= (in ? 1u : 0u) << k;
    }
  }
  if constexpr (M == M_FAULT) {
#pragma unroll
    for (int k = 0; k < VEC; ++k) key[k] = rep.fault(SITE_LOAD, (long long)j0 + k, key[k]);
  }
  unsigned lo[VEC] = {0u, 0u, 0u, 0u};
  unsigned len = a.N;
  // invariant: lower_bound(key) in [lo, lo + len]
  for (int it = 0; it < a.iters; ++it) {
    const unsigned half = len >> 1;
    unsigned probe[VEC];
#pragma unroll
    for (int k = 0; k < VEC; ++k) probe[k] = __ldg(a.A + lo[k] + half - 1);
#pragma unroll
    for (int k = 0; k < VEC; ++k) lo[k] = probe[k] < key[k] ? lo[k] + half : lo[k];
    len -= half;
    if constexpr (M == M_FAULT) {
      if (it == a.iters / 2) {  // control-flow fault: a flipped probe position, kept in bounds
#pragma unroll
        for (int k = 0; k < VEC; ++k) {
          unsigned f = rep.fault(SITE_COMPUTE, (long long)j0 + k, lo[k]);
          lo[k] = f > a.N - len ? a.N - len : f;
        }
      }
    }
  }
  unsigned out[VEC];
#pragma unroll
  for (int k = 0; k < VEC; ++k) out[k] = a.N == 0 ? 0u : lo[k] + (__ldg(a.A + lo[k]) < key[k] ? 1u : 0u);
  rep.template commit<VEC, 0>(mask, j0, out, a.Q, [&](unsigned i, unsigned m, const unsigned* w) {
    if (m == 0xFu) __stcs(reinterpret_cast<uint4*>(a.idx + i), make_uint4(w[0], w[1], w[2], w[3]));
    else
      for (int k = 0; k < VEC; ++k)
        if ((m >> k) & 1u) a.idx[i + k] = w[k];
  });
  rep.finish();
}

}  // namespace

int binarysearch_validate(const rmt_bufs_t* b, int64_t n) {
  int64_t N = b->dims[0], Q = b->dims[1];
  if (b->nbuf < 3 || N < 0 || N >= (1LL << 32) - 1 || Q < 0 || Q >= (1LL << 30) || n != Q ||
      !buf_ok(b->buf[0], RMT_U32, N) || !buf_ok(b->buf[1], RMT_U32, Q) || !buf_ok(b->buf[2], RMT_U32, Q)) {
    set_error("binarysearch: expected {A:U32[N], q:U32[Q], idx:U32[Q]}, dims {N,Q}, n = Q");
    return RMT_EINVAL;
  }
  return RMT_OK;
}
size_t binarysearch_scratch(int64_t, const int64_t*) { return 0; }
int binarysearch_inter_warps(int64_t, const int64_t*) { return BL / 32; }

int binarysearch_run(Launch& L) {
  const unsigned N = (unsigned)L.bufs->dims[0], Q = (unsigned)L.bufs->dims[1];
  int iters = 0;
  for (unsigned len = N; len > 1; len -= len >> 1) ++iters;
  BsArgs a{(const unsigned*)L.bufs->buf[0].ptr, (const unsigned*)L.bufs->buf[1].ptr, (unsigned*)L.bufs->buf[2].ptr,
           N, Q, iters};
  const unsigned G = (Q + BL * VEC - 1) / (BL * VEC);
  return dispatch(L.variant, L.mode, [&](auto vm) {
    constexpr int V = decltype(vm)::V, M = decltype(vm)::M;
    return launch_std<V>(L, bins_kernel<V, M>, bins_kernel<V_NONE, M_NORMAL>, G, BL, 0, a, "binarysearch");
  });
}

}  // namespace rmt
