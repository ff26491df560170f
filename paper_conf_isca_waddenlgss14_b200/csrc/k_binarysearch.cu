// k_binarysearch.cu -- BinarySearch ("BinS"; memory-bound,
// Intra <=10%; "many work-items never execute a global write").
// Batched lower_bound (reading R-BIN1): idx[j] = #{i : A[i] < q[j]}.
//
// B200 design.  A plain binary search over a 256 MiB array misses L2 on ~11 of
// its 26 levels (every probe is a different 32-B sector).  Instead, each launch
// first builds a 16-ary sample hierarchy L_k[j] = A[16^k j] (k = 1..T, padded
// with 0xFFFFFFFF to a multiple of 16; ~N/15 words, dense and L2-resident) --
// itself an RMT-protected kernel whose stores are committed -- then each query
// binary-searches the small top level L_T and descends with ONE 64-B block scan
// per level: if jj = lower_bound in L_{k+1}, then lower_bound in L_k =
// 16(jj-1) + #{block jj-1 of L_k < key} (jj > 0), which is exact because
// L_k[16(jj-1)] < key <= L_k[16 jj].  Logical thread = 4 interleaved queries,
// one 16-B vector commit of idx.
#include <string.h>

#include "rmt_host.cuh"

namespace rmt {
namespace {

constexpr int BL = 256;
constexpr int VEC = 4;
constexpr int FAN = 16;       // samples per block
constexpr int MAXLEV = 8;
constexpr unsigned TOP_MAX = FAN;   // sample until the top level fits in one block

struct Levels {
  int T;                         // number of sample levels (0: search A directly)
  unsigned n[MAXLEV + 1];        // entries per level (n[0] = N)
  unsigned off[MAXLEV + 1];      // word offset of level k (k >= 1) in the scratch
  unsigned padded[MAXLEV + 1];   // entries rounded up to a multiple of 16
  unsigned vecs_before[MAXLEV + 2];  // index-build vector ranges
};

struct BsArgs {
  const unsigned* A;
  const unsigned* q;
  unsigned* idx;
  unsigned* lev;  // scratch: sample levels
  unsigned N, Q;
  int top_iters;
  Levels L;
};

Levels make_levels(unsigned N) {
  Levels L;
  memset(&L, 0, sizeof(L));
  L.n[0] = N;
  unsigned off = 0;
  int k = 0;
  while (L.n[k] > TOP_MAX && k < MAXLEV) {
    ++k;
    L.n[k] = (L.n[k - 1] + FAN - 1) / FAN;
    L.padded[k] = (L.n[k] + FAN - 1) / FAN * FAN;
    L.off[k] = off;
    off += L.padded[k];
  }
  L.T = k;
  L.vecs_before[1] = 0;
  for (int i = 1; i <= L.T; ++i) L.vecs_before[i + 1] = L.vecs_before[i] + L.padded[i] / 4;
  return L;
}

// ---- index build: logical thread v writes 4 consecutive entries of one level
template <int V, int M>
__global__ void __launch_bounds__(BL * Geom<V>::DUP) bins_index_kernel(BsArgs a, Ctx c) {
  __shared__ unsigned mb[mbox_words<V>(BL * Geom<V>::DUP)];
  Rep<V, M> rep(c);
  rep.init(mb);
  const unsigned v = (unsigned)rep.lblock * BL + (unsigned)rep.ltid;
  const unsigned total = a.L.vecs_before[a.L.T + 1];
  int k = 1;
#pragma unroll 1
  while (k < a.L.T && v >= a.L.vecs_before[k + 1]) ++k;
  const bool active = v < total;
  const unsigned j0 = active ? (v - a.L.vecs_before[k]) * 4 : 0u;
  unsigned stride = 1;
#pragma unroll 1
  for (int i = 0; i < k; ++i) stride *= FAN;
  unsigned w[4];
#pragma unroll
  for (int q = 0; q < 4; ++q) {
    const unsigned j = j0 + q;
    const unsigned long long src = (unsigned long long)j * stride;
    w[q] = (active && j < a.L.n[k]) ? __ldcs(a.A + src) : 0xFFFFFFFFu;  // L_k[j] = A[16^k j] (A: evict-first)
  }
  rep.template commit<4, 1>(active ? 0xFu : 0u, active ? a.L.off[k] + j0 : 0u, w, 0xFFFFFFF0u,
                            [&](unsigned i, unsigned m, const unsigned* x) {
                              if (m == 0xFu) *reinterpret_cast<uint4*>(a.lev + i) = make_uint4(x[0], x[1], x[2], x[3]);
                            });
  rep.finish();
}

template <int V, int M>
// Intra variants: 512-thread CTAs would hold 72 registers (1 CTA/SM); cap at 40.
__global__ void __launch_bounds__(BL * Geom<V>::DUP, Geom<V>::DUP == 2 ? 3 : 4) bins_kernel(BsArgs a, Ctx c) {
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
  // Groups of 4 logical lanes descend together: for each of the group's 16
  // queries the 4 members load one 16-B quarter of the same 64-B block, so a
  // warp-wide load touches one cache line per query (1 L1 wavefront instead
  // of 4).  Each lane tracks the block base of its OWN 4 queries and fetches the
  // other members' bases by shuffle.
  const int gm = rep.llane & 3;
  const int g0 = rep.llane & ~3;
  unsigned K[4][VEC];
#pragma unroll
  for (int i = 0; i < 4; ++i)
#pragma unroll
    for (int s = 0; s < VEC; ++s) K[i][s] = rep.lshfl_idx(key[s], g0 + i);
  unsigned jj[VEC];
#pragma unroll
  for (int s = 0; s < VEC; ++s) jj[s] = a.N ? 1u : 0u;  // "block 0" of the top level
  // one level: J <- 16 (max(J,1) - 1) + #{block < key}.  When J = 0 (key <= every
  // entry) block 0 counts 0, so J stays 0 with no special case.
  auto level = [&](const unsigned* P, unsigned lim, bool tail) {
#pragma unroll
    for (int s = 0; s < VEC; ++s) {
      const unsigned mybase = (max(jj[s], 1u) - 1u) * FAN;
      unsigned packed = 0;
#pragma unroll
      for (int i = 0; i < 4; ++i) {
        const unsigned base = rep.lshfl_idx(mybase, g0 + i) + 4u * gm;
        uint4 w;
        if (!tail) {  // sample levels: keep them L2-resident (default policy)
          w = __ldg(reinterpret_cast<const uint4*>(P + base));
        } else if (base + 4u <= lim) {  // the caller's A: random 64-B blocks, evict-first
          w = __ldcs(reinterpret_cast<const uint4*>(P + base));
        } else {  // tail of the caller's A: element-wise, never past lim
          w.x = base + 0 < lim ? __ldcs(P + base + 0) : 0xFFFFFFFFu;
          w.y = base + 1 < lim ? __ldcs(P + base + 1) : 0xFFFFFFFFu;
          w.z = base + 2 < lim ? __ldcs(P + base + 2) : 0xFFFFFFFFu;
          w.w = base + 3 < lim ? __ldcs(P + base + 3) : 0xFFFFFFFFu;
        }
        const unsigned k = K[i][s];
        const unsigned bits = (w.x < k ? 1u : 0u) | (w.y < k ? 2u : 0u) | (w.z < k ? 4u : 0u) | (w.w < k ? 8u : 0u);
        packed += (unsigned)__popc(bits) << (8 * i);
      }
      packed += rep.lshfl_xor(packed, 1);  // sum the 4 quarters (bytes <= 16: no carries)
      packed += rep.lshfl_xor(packed, 2);
      jj[s] = mybase + ((packed >> (8 * gm)) & 0xFFu);
    }
  };
  for (int lv = a.L.T; lv >= 1; --lv) {  // padded sample levels: no bounds checks
    if constexpr (M == M_FAULT) {
      if (lv == a.L.T - 1) {  // control-flow fault: a flipped block index, kept in range
#pragma unroll
        for (int s = 0; s < VEC; ++s) {
          const unsigned f = rep.fault(SITE_COMPUTE, (long long)j0 + s, jj[s]);
          jj[s] = f > a.L.n[lv + 1] ? a.L.n[lv + 1] : f;
        }
      }
    }
    level(a.lev + a.L.off[lv], a.L.padded[lv], false);
  }
  if constexpr (M == M_FAULT) {
    if (a.L.T == 1) {
#pragma unroll
      for (int s = 0; s < VEC; ++s) {
        const unsigned f = rep.fault(SITE_COMPUTE, (long long)j0 + s, jj[s]);
        jj[s] = f > a.L.n[1] ? a.L.n[1] : f;
      }
    }
  }
  level(a.A, a.N, true);  // the caller's A
  rep.template commit<VEC, 0>(mask, j0, jj, a.Q, [&](unsigned i, unsigned m, const unsigned* w) {
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
  if (b->nbuf < 3 || N < 0 || N >= (1LL << 32) - 64 || Q < 0 || Q >= (1LL << 30) || n != Q ||
      !buf_ok(b->buf[0], RMT_U32, N) || !buf_ok(b->buf[1], RMT_U32, Q) || !buf_ok(b->buf[2], RMT_U32, Q)) {
    set_error("binarysearch: expected {A:U32[N], q:U32[Q], idx:U32[Q]}, dims {N,Q}, n = Q");
    return RMT_EINVAL;
  }
  return RMT_OK;
}
size_t binarysearch_scratch(int64_t, const int64_t* dims) {
  Levels L = make_levels((unsigned)dims[0]);
  size_t words = 0;
  for (int k = 1; k <= L.T; ++k) words += L.padded[k];
  return words * 4 + 64;
}
int binarysearch_inter_warps(int64_t, const int64_t*) { return BL / 32; }

int binarysearch_run(Launch& L) {
  const unsigned N = (unsigned)L.bufs->dims[0], Q = (unsigned)L.bufs->dims[1];
  BsArgs a;
  a.A = (const unsigned*)L.bufs->buf[0].ptr;
  a.q = (const unsigned*)L.bufs->buf[1].ptr;
  a.idx = (unsigned*)L.bufs->buf[2].ptr;
  a.lev = (unsigned*)L.scratch;
  a.N = N;
  a.Q = Q;
  a.L = make_levels(N);
  a.top_iters = 0;
  const unsigned Gi = (a.L.vecs_before[a.L.T + 1] + BL - 1) / BL;
  const unsigned G = (Q + BL * VEC - 1) / (BL * VEC);
  return dispatch(L.variant, L.mode, [&](auto vm) {
    constexpr int V = decltype(vm)::V, M = decltype(vm)::M;
    int rc = RMT_OK;
    if (a.L.T > 0 && Q > 0)
      rc = launch_std<V>(L, bins_index_kernel<V, M>, bins_index_kernel<V_NONE, M_NORMAL>, Gi, BL, 0, a,
                         "binarysearch/index");
    if (rc) return rc;
    return launch_std<V>(L, bins_kernel<V, M>, bins_kernel<V_NONE, M_NORMAL>, G, BL, 0, a, "binarysearch");
  });
}

}  // namespace rmt
