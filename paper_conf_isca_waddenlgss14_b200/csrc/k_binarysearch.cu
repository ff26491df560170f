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
  unsigned N16;                  // N rounded down to a multiple of 16
  unsigned tail_off;             // word offset of the padded copy of A[N16, N) (16 words)
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
  L.N16 = N & ~15u;
  L.tail_off = off;
  return L;
}

// #{w_i >= k} over the 4 words: each unsigned compare is the carry of w - k
// (sub.cc: carry = no borrow = w >= k), summed with addc -- two integer-pipe
// instructions per key instead of a compare, a select and a bit-combine.
__device__ __forceinline__ unsigned count_ge(uint4 w, unsigned k) {
  unsigned c, t;
  asm("{\n\t"
      "sub.cc.u32 %1, %2, %6;\n\t"
      "addc.u32 %0, 0, 0;\n\t"
      "sub.cc.u32 %1, %3, %6;\n\t"
      "addc.u32 %0, %0, 0;\n\t"
      "sub.cc.u32 %1, %4, %6;\n\t"
      "addc.u32 %0, %0, 0;\n\t"
      "sub.cc.u32 %1, %5, %6;\n\t"
      "addc.u32 %0, %0, 0;\n\t"
      "}"
      : "=r"(c), "=&r"(t)
      : "r"(w.x), "r"(w.y), "r"(w.z), "r"(w.w), "r"(k));
  (void)t;  // scratch register of the asm (the differences are not needed)
  return c;
}

// p + i (u32 elements) as one wide multiply-add (keeps nvcc from widening the
// index sum with carries)
__device__ __forceinline__ const unsigned* wide_addr(const unsigned* p, unsigned i) {
  const unsigned* r;
  asm("mad.wide.u32 %0, %1, 4, %2;" : "=l"(r) : "r"(i), "l"(p));
  return r;
}

// ---- index build: logical thread v writes 4 consecutive entries of one level,
// or (the last 4 vectors) 4 words of the padded tail block T[i] = A[N16 + i]
// (0xFFFFFFFF past N), so the final level's 64-B block loads need no bounds
// checks (branch-free: all of a thread's block loads are in flight together).
template <int V, int M>
__global__ void __launch_bounds__(BL * Geom<V>::DUP) bins_index_kernel(BsArgs a, Ctx c) {
  __shared__ unsigned mb[mbox_words<V>(BL * Geom<V>::DUP)];
  Rep<V, M> rep(c);
  rep.init(mb);
  for (; rep.active(); rep.advance()) {
    const unsigned v = (unsigned)rep.lblock * BL + (unsigned)rep.ltid;
    const unsigned total = a.L.vecs_before[a.L.T + 1];
    int k = 1;
#pragma unroll 1
    while (k < a.L.T && v >= a.L.vecs_before[k + 1]) ++k;
    const bool tail = v >= total && v < total + 4u;
    const bool active = v < total || tail;
    const unsigned j0 = tail ? (v - total) * 4 : active ? (v - a.L.vecs_before[k]) * 4 : 0u;
    unsigned stride = 1;
#pragma unroll 1
    for (int i = 0; i < k; ++i) stride *= FAN;
    unsigned w[4];
#pragma unroll
    for (int q = 0; q < 4; ++q) {
      const unsigned j = j0 + q;
      if (tail) {
        w[q] = a.L.N16 + j < a.N ? __ldg(a.A + a.L.N16 + j) : 0xFFFFFFFFu;
      } else {
        const unsigned long long src = (unsigned long long)j * stride;
        w[q] = (active && j < a.L.n[k]) ? __ldcs(a.A + src) : 0xFFFFFFFFu;  // L_k[j] = A[16^k j] (A: evict-first)
      }
    }
    const unsigned dst = tail ? a.L.tail_off + j0 : active ? a.L.off[k] + j0 : 0u;
    rep.template commit<4, 1>(active ? 0xFu : 0u, dst, w, 0xFFFFFFF0u,
                              [&](unsigned i, unsigned m, const unsigned* x) {
                                if (m == 0xFu) *reinterpret_cast<uint4*>(a.lev + i) = make_uint4(x[0], x[1], x[2], x[3]);
                              });
  }
  rep.finish();
}

template <int V, int M>
// Intra variants: 512-thread CTAs would hold 72 registers (1 CTA/SM); cap at 40.
__global__ void __launch_bounds__(BL * Geom<V>::DUP, Geom<V>::DUP == 2 ? 3 : 4) bins_kernel(BsArgs a, Ctx c) {
  __shared__ unsigned mb[mbox_words<V>(BL * Geom<V>::DUP)];
  Rep<V, M> rep(c);
  rep.init(mb);
  for (; rep.active(); rep.advance()) {
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
    const unsigned* tailp = a.lev + a.L.tail_off - a.L.N16;  // tailp[N16 + i] = T[i]
    // per-lane quarter pointers: element (base + 4 gm) of level P is Pq + 16 base bytes
    auto level = [&](const unsigned* P, bool last) {
      const unsigned* Pq = P + 4 * gm;
      const unsigned* Tq = tailp + 4 * gm;
#pragma unroll
      for (int s = 0; s < VEC; ++s) {
        const unsigned mybase = (max(jj[s], 1u) - 1u) * FAN;
        unsigned packed = 0;
#pragma unroll
        for (int i = 0; i < 4; ++i) {
          const unsigned base = rep.lshfl_idx(mybase, g0 + i);
          uint4 w;
          if (!last) {  // sample levels: keep them L2-resident (default policy)
            w = __ldg(reinterpret_cast<const uint4*>(wide_addr(Pq, base)));
          } else {  // the caller's A: random 64-B blocks, evict-first; the ragged
                    // last block comes from the padded copy (a block never straddles N16)
            w = __ldcs(reinterpret_cast<const uint4*>(wide_addr(base >= a.L.N16 ? Tq : Pq, base)));
          }
          packed += count_ge(w, K[i][s]) << (8 * i);
        }
        packed += rep.lshfl_xor(packed, 1);  // sum the 4 quarters (bytes <= 16: no carries)
        packed += rep.lshfl_xor(packed, 2);
        jj[s] = mybase + FAN - ((packed >> (8 * gm)) & 0xFFu);  // #{block < key} = 16 - #{block >= key}
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
      level(a.lev + a.L.off[lv], false);
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
    level(a.A, true);  // the caller's A
    rep.template commit<VEC, 0>(mask, j0, jj, a.Q, [&](unsigned i, unsigned m, const unsigned* w) {
      if (m == 0xFu) __stcs(reinterpret_cast<uint4*>(a.idx + i), make_uint4(w[0], w[1], w[2], w[3]));
      else
        for (int k = 0; k < VEC; ++k)
          if ((m >> k) & 1u) a.idx[i + k] = w[k];
    });
  }
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
  return (words + 16) * 4 + 64;  // + the padded tail block
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
  const unsigned Gi = (a.L.vecs_before[a.L.T + 1] + 4 + BL - 1) / BL;
  const unsigned G = (Q + BL * VEC - 1) / (BL * VEC);
  return dispatch(L.variant, L.mode, [&](auto vm) {
    constexpr int V = decltype(vm)::V, M = decltype(vm)::M;
    int rc = RMT_OK;
    if (Q > 0)
      rc = launch_std<V>(L, bins_index_kernel<V, M>, bins_index_kernel<V_NONE, M_NORMAL>, Gi, BL, 0, a,
                         "binarysearch/index");
    if (rc) return rc;
    return launch_std<V>(L, bins_kernel<V, M>, bins_kernel<V_NONE, M_NORMAL>, G, BL, 0, a, "binarysearch",
                         /*mult_inter=*/2);
  });
}

}  // namespace rmt
