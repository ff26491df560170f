// k_binarysearch.cu -- BinarySearch ("BinS"; memory-bound,
// Intra <=10%; "many work-items never execute a global write").
// Batched lower_bound (reading R-BIN1): idx[j] = #{i : A[i] < q[j]}.
//
// B200 design.  A plain binary search over a 256 MiB array misses L2 on ~11 of
// its 26 levels.  Instead each launch first builds a 32-ary sample hierarchy
// L_k[j] = A[32^k j] (k = 1..T, each padded with 0xFFFFFFFF to a multiple of
// 32 entries; ~N/31 words, L2-resident) -- itself an RMT-protected kernel whose
// stores are committed -- where T is the first level of at most TMAX entries.
// The query kernel copies L_T into shared memory once per CTA and finds
// lower_bound(L_T, key) by a branch-free binary search there; it then descends
// with ONE 128-B block scan per level: if jj = lower_bound in L_{k+1}, then
// lower_bound in L_k = 32(jj-1) + #{block jj-1 of L_k < key} (jj > 0), exact
// because L_k[32(jj-1)] < key <= L_k[32 jj].  For N = 2^26 that is L3 (2048
// entries) in shared memory and three 128-B global blocks per query (L2, L1
// in L2; A from DRAM).
//
// Why 128-B blocks: a random miss moves a whole 128-B line from DRAM whatever
// the request size (tools/gather_probe.cu: 117.5 B of DRAM per random 16-, 32-
// or 64-B read, ~53 G misses/s), so the A block costs the same DRAM time at
// 128 B as at 64 B, and one 128-B line per query and level is also the L1 data
// pipe's unit (the 64-B design spent a wavefront per 64 B and 7 levels).
// Group of 4 logical lanes per query, one 32-B load each (LDG.256); logical
// thread = 2 interleaved queries, one 8-B vector commit of idx; every lane of a
// group loads the group's 8 keys with one 256-bit load.
#include <string.h>

#include "rmt_host.cuh"

namespace rmt {
namespace {

constexpr int BL = 256;
constexpr int VEC = 2;
constexpr int FAN = 32;       // entries per block (128 B)
constexpr int MAXLEV = 8;
constexpr unsigned TMAX = 8192;   // shared-memory table: at most 8192 entries (32 KiB per replica)
constexpr unsigned CHUNK = BL * VEC;  // queries per logical CTA iteration

struct Levels {
  int T;                         // table level (>= 1): L_T lives in shared memory
  unsigned n[MAXLEV + 1];        // entries per level (n[0] = N)
  unsigned off[MAXLEV + 1];      // word offset of level k (k >= 1) in the scratch
  unsigned padded[MAXLEV + 1];   // entries rounded up to a multiple of 32
  unsigned vecs_before[MAXLEV + 2];  // index-build vector ranges
  unsigned N32;                  // N rounded down to a multiple of 32
  unsigned tail_off;             // word offset of the padded copy of A[N32, N) (32 words)
  unsigned P;                    // table entries in shared memory: a power of two >= n[T]
};

struct BsArgs {
  const unsigned* A;
  const unsigned* q;
  unsigned* idx;
  unsigned* lev;  // scratch: sample levels
  unsigned N, Q;
  unsigned iters;   // chunks of CHUNK queries per logical CTA
  unsigned plane;   // +LDS: replica r's table copy starts at word r * plane (P + 1: the
                    // pair's two copies of an entry sit in different banks)
  unsigned a32;     // A is 32-B aligned (256-bit block loads)
  unsigned q32;     // q is 32-B aligned (256-bit key loads)
  Levels L;
};

Levels make_levels(unsigned N) {
  Levels L;
  memset(&L, 0, sizeof(L));
  L.n[0] = N;
  unsigned off = 0;
  int k = 0;
  do {
    ++k;
    L.n[k] = (L.n[k - 1] + FAN - 1) / FAN;
    L.padded[k] = (L.n[k] + FAN - 1) / FAN * FAN;
    if (L.padded[k] == 0) L.padded[k] = FAN;  // N = 0: one all-padding block
    L.off[k] = off;
    off += L.padded[k];
  } while (L.n[k] > TMAX && k < MAXLEV);
  L.T = k;
  L.vecs_before[1] = 0;
  for (int i = 1; i <= L.T; ++i) L.vecs_before[i + 1] = L.vecs_before[i] + L.padded[i] / 4;
  L.N32 = N & ~(unsigned)(FAN - 1);
  L.tail_off = off;
  unsigned P = 32;
  while (P < L.n[L.T]) P <<= 1;
  L.P = P;
  return L;
}

// #{w_i >= k} over 8 words: each unsigned compare is the carry of w - k
// (sub.cc: carry = no borrow = w >= k), summed with addc -- two integer-pipe
// instructions per word instead of a compare, a select and a bit-combine.
__device__ __forceinline__ unsigned count_ge8(const unsigned (&w)[8], unsigned k) {
  unsigned c;
  asm("{\n\t"
      ".reg .u32 t;\n\t"  // scratch: the differences are not needed
      "sub.cc.u32 t, %1, %9;\n\t"
      "addc.u32 %0, 0, 0;\n\t"
      "sub.cc.u32 t, %2, %9;\n\t"
      "addc.u32 %0, %0, 0;\n\t"
      "sub.cc.u32 t, %3, %9;\n\t"
      "addc.u32 %0, %0, 0;\n\t"
      "sub.cc.u32 t, %4, %9;\n\t"
      "addc.u32 %0, %0, 0;\n\t"
      "sub.cc.u32 t, %5, %9;\n\t"
      "addc.u32 %0, %0, 0;\n\t"
      "sub.cc.u32 t, %6, %9;\n\t"
      "addc.u32 %0, %0, 0;\n\t"
      "sub.cc.u32 t, %7, %9;\n\t"
      "addc.u32 %0, %0, 0;\n\t"
      "sub.cc.u32 t, %8, %9;\n\t"
      "addc.u32 %0, %0, 0;\n\t"
      "}"
      : "=r"(c)
      : "r"(w[0]), "r"(w[1]), "r"(w[2]), "r"(w[3]), "r"(w[4]), "r"(w[5]), "r"(w[6]), "r"(w[7]), "r"(k));
  return c;
}

// Shared-memory table swizzle: entry i lives at word i ^ ((i >> 6) & 31).  The
// binary search's probes at step >= 32 are pos + step - 1 with pos a multiple
// of 2 step -- all in ONE bank unswizzled (a 32-way conflict at step 32); with
// the row index folded into the bank they spread over distinct banks.
__device__ __forceinline__ unsigned tsw(unsigned i) { return i ^ ((i >> 6) & 31u); }

// p + i (u32 elements) as one wide multiply-add (keeps nvcc from widening the
// index sum with carries)
__device__ __forceinline__ const unsigned* wide_addr(const unsigned* p, unsigned i) {
  const unsigned* r;
  asm("mad.wide.u32 %0, %1, 4, %2;" : "=l"(r) : "r"(i), "l"(p));
  return r;
}

// 32 B of a sample level (L2-resident: default caching, 256-bit load)
__device__ __forceinline__ void ld8(const unsigned* p, unsigned (&w)[8]) {
  asm volatile("ld.global.nc.v8.b32 {%0, %1, %2, %3, %4, %5, %6, %7}, [%8];"
               : "=r"(w[0]), "=r"(w[1]), "=r"(w[2]), "=r"(w[3]), "=r"(w[4]), "=r"(w[5]), "=r"(w[6]), "=r"(w[7])
               : "l"(p));
}

// ---- index build: logical thread v writes 4 consecutive entries of one level,
// or (the last 8 vectors) 4 words of the padded tail block T[i] = A[N32 + i]
// (0xFFFFFFFF past N), so the final level's 128-B block loads need no bounds
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
    const bool tail = v >= total && v < total + FAN / 4;
    const bool active = v < total || tail;
    const unsigned j0 = tail ? (v - total) * 4 : active ? (v - a.L.vecs_before[k]) * 4 : 0u;
    unsigned long long stride = 1;
#pragma unroll 1
    for (int i = 0; i < k; ++i) stride *= FAN;
    unsigned w[4];
#pragma unroll
    for (int q = 0; q < 4; ++q) {
      const unsigned j = j0 + q;
      if (tail) {
        w[q] = a.L.N32 + j < a.N ? __ldg(a.A + a.L.N32 + j) : 0xFFFFFFFFu;
      } else {
        const unsigned long long src = (unsigned long long)j * stride;
        w[q] = (active && j < a.L.n[k]) ? __ldcs(a.A + src) : 0xFFFFFFFFu;  // L_k[j] = A[32^k j] (A: evict-first)
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

#ifndef BINS_MINB
#define BINS_MINB 4
#endif
#ifndef BINS_INTER_MINB
#define BINS_INTER_MINB BINS_MINB
#endif
#ifndef BINS_WAVES
#define BINS_WAVES 8u  // logical CTAs per SM (the table copy is amortised over the rest)
#endif
#ifndef BINS_GROUP
#define BINS_GROUP 1
#endif
template <int V, int M>
// Registers capped at 64 (4 CTAs of 256 / 2 of 512 threads per SM).
__global__ void __launch_bounds__(BL * Geom<V>::DUP, Geom<V>::DUP == 2 ? BINS_MINB / 2 : V == V_INTER ? BINS_INTER_MINB : BINS_MINB) bins_kernel(BsArgs a, Ctx c) {
  __shared__ unsigned mb[mbox_words<V>(BL * Geom<V>::DUP)];
  extern __shared__ __align__(16) unsigned char bins_dyn[];
  // inter: group flags, the commits of BINS_GROUP consecutive chunks published
  // behind one fence (deferred commits; the last chunk of a logical CTA closes)
  Rep<V, M, (BINS_GROUP > 1)> rep(c);
  rep.init(mb);
  using R = Rep<V, M, (BINS_GROUP > 1)>;
  // ---- the table L_T in shared memory, once per physical CTA (every logical
  // CTA of a persistent pair reuses it).  +LDS: each replica writes and reads
  // its own copy; -LDS: one copy, every store compared.
  unsigned* S = reinterpret_cast<unsigned*>(bins_dyn) + (R::SMDUP ? (unsigned)rep.r * a.plane : 0u);
  {
    const unsigned* LT = a.lev + a.L.off[a.L.T];
    const unsigned nT = a.L.n[a.L.T];
    const int nthr = BL;
#pragma unroll 1
    for (unsigned i = (unsigned)rep.ltid; i < a.L.P; i += nthr) {
      const unsigned w = i < nT ? __ldg(LT + i) : 0xFFFFFFFFu;
      if (rep.sts_ok1(w, i)) S[tsw(i)] = w;
    }
  }
  __syncthreads();
  const unsigned P = a.L.P;
  const int T = a.L.T;
  for (; rep.active(); rep.advance()) {
#pragma unroll 1
    for (unsigned it = 0; it < a.iters; ++it) {
      const unsigned chunk = (unsigned)rep.lblock * a.iters + it;
      if ((unsigned long long)chunk * CHUNK >= a.Q) break;  // CTA-uniform
      const unsigned j0 = (chunk * BL + (unsigned)rep.ltid) * VEC;
      // Groups of 4 logical lanes descend together (below); every lane loads the
      // group's 8 keys (4 members x VEC, contiguous and 32-B aligned: one 256-bit
      // load, the 4 lanes' identical requests served by the same lines) --
      // K[i][s] = key s of member i, no shuffles.
      const int gm = rep.llane & 3;
      const int g0 = rep.llane & ~3;
      const unsigned jg = j0 - (unsigned)gm * VEC;  // the group's first query
      unsigned K[4][VEC];
      {
        unsigned w[8];
        if (jg + 4 * VEC <= a.Q && a.q32) {
          ldcs8(a.q + jg, w);
        } else {
#pragma unroll
          for (int k = 0; k < 8; ++k) w[k] = jg + k < a.Q ? __ldcs(a.q + jg + k) : 0u;
        }
#pragma unroll
        for (int i = 0; i < 4; ++i)
#pragma unroll
          for (int s = 0; s < VEC; ++s) K[i][s] = w[i * VEC + s];
      }
      if constexpr (M == M_FAULT) {
#pragma unroll
        for (int i = 0; i < 4; ++i)
#pragma unroll
          for (int s = 0; s < VEC; ++s) K[i][s] = rep.fault(SITE_LOAD, (long long)jg + i * VEC + s, K[i][s]);
      }
      unsigned key[VEC];
      unsigned mask = 0;
#pragma unroll
      for (int s = 0; s < VEC; ++s) {
        key[s] = gm == 0 ? K[0][s] : gm == 1 ? K[1][s] : gm == 2 ? K[2][s] : K[3][s];
        mask |= (j0 + s < a.Q ? 1u : 0u) << s;
      }
      // ---- lower_bound in L_T: pos = #{S[i] < key} over the P (padded, sorted)
      // entries, branch-free; the padding (0xFFFFFFFF) is never < key.  The
      // halving steps leave pos in [0, P-1] with S[0, pos) < key <= S[pos + 1]
      // (when that exists); one last compare of S[pos] decides pos vs pos + 1
      // (pos = P when every entry is < key: n_T = P, no padding).
      unsigned jj[VEC];
#pragma unroll
      for (int s = 0; s < VEC; ++s) jj[s] = 0u;
#pragma unroll 1
      for (unsigned step = P >> 1; step >= 1u; step >>= 1) {
#pragma unroll
        for (int s = 0; s < VEC; ++s) {
          unsigned w = S[tsw(jj[s] + step - 1u)];
          if constexpr (M == M_FAULT) w = rep.fault(SITE_SMEM, (long long)(jj[s] + step - 1u), w);
          jj[s] += w < key[s] ? step : 0u;
        }
      }
#pragma unroll
      for (int s = 0; s < VEC; ++s) {
        unsigned w = S[tsw(jj[s])];
        if constexpr (M == M_FAULT) w = rep.fault(SITE_SMEM, (long long)jj[s], w);
        jj[s] += w < key[s] ? 1u : 0u;
      }
      if constexpr (M == M_FAULT) {  // control-flow fault: a flipped block index, kept in range
#pragma unroll
        for (int s = 0; s < VEC; ++s) {
          const unsigned f = rep.fault(SITE_COMPUTE, (long long)j0 + s, jj[s]);
          jj[s] = f > a.L.n[T] ? a.L.n[T] : f;
        }
      }
      // ---- descent: for each of the group's 8 queries the 4 members load one
      // 32-B quarter of the same 128-B block (one L1 wavefront per query and
      // level).  Each lane tracks the block base of its OWN 2 queries and
      // fetches the other members' bases by shuffle.  (Tracking all 8 positions
      // in every lane instead saves the base shuffles but costs more
      // instructions: measured 0.452 -> 0.498 ms at Q = 2^24, latency-bound.)
      const unsigned* tailp = a.lev + a.L.tail_off - a.L.N32;  // tailp[N32 + i] = T[i]
      // one level: J <- 32 (max(J,1) - 1) + #{block < key}.  When J = 0 (key <=
      // every entry) block 0 counts 0, so J stays 0 with no special case.
      auto level = [&](const unsigned* Pl, bool last) {
        const unsigned* Pq = Pl + 8 * gm;
        const unsigned* Tq = tailp + 8 * gm;
#pragma unroll
        for (int s = 0; s < VEC; ++s) {
          const unsigned mybase = (max(jj[s], 1u) - 1u) * FAN;
          unsigned packed = 0;
#pragma unroll
          for (int i = 0; i < 4; ++i) {
            const unsigned base = rep.lshfl_idx(mybase, g0 + i);
            unsigned w[8];
            if (!last) {  // sample levels: keep them L2-resident (default policy)
              ld8(wide_addr(Pq, base), w);
            } else {      // the caller's A: random 128-B blocks, evict-first; the ragged
                          // last block comes from the padded copy (a block never straddles N32)
              const unsigned* p = wide_addr(base >= a.L.N32 ? Tq : Pq, base);
              if (a.a32 || base >= a.L.N32) {
                ldcs8(p, w);
              } else {
                const uint4 u0 = ldcs4(p), u1 = ldcs4(p + 4);
                w[0] = u0.x; w[1] = u0.y; w[2] = u0.z; w[3] = u0.w;
                w[4] = u1.x; w[5] = u1.y; w[6] = u1.z; w[7] = u1.w;
              }
            }
            packed += count_ge8(w, K[i][s]) << (8 * i);
          }
          packed += rep.lshfl_xor(packed, 1);  // sum the 4 quarters (bytes <= 32: no carries)
          packed += rep.lshfl_xor(packed, 2);
          jj[s] = mybase + FAN - ((packed >> (8 * gm)) & 0xFFu);  // #{block < key} = 32 - #{block >= key}
        }
      };
#pragma unroll 1
      for (int lv = T - 1; lv >= 1; --lv) level(a.lev + a.L.off[lv], false);  // padded: no bounds checks
      level(a.A, true);  // the caller's A
      const bool close = (it + 1u) % BINS_GROUP == 0u || it + 1u == a.iters ||
                         (unsigned long long)(chunk + 1u) * CHUNK >= a.Q;  // CTA-uniform
      rep.template commit<VEC, 0>(mask, j0, jj, a.Q, [&](unsigned i, unsigned m, const unsigned* w) {
        if (m == 0x3u) __stcs(reinterpret_cast<uint2*>(a.idx + i), make_uint2(w[0], w[1]));
        else
          for (int k = 0; k < VEC; ++k)
            if ((m >> k) & 1u) a.idx[i + k] = w[k];
      }, /*defer=*/!close);
    }
  }
  rep.finish();
}

// ---- ghost mode (dims[2] = 1; SURVEY 8(c) BinarySearch reading (1)): the APP
// SDK's single-key segment search, where "many work-items never execute a
// global write".  Logical CTA j searches key q[j]: logical thread t owns
// the segment [lo_t, hi_t) of A (256 near-equal segments) and checks whether
// lower_bound(A, q[j]) falls in it -- (lo_t == 0 or A[lo_t - 1] < key) and
// (hi_t == N or key <= A[hi_t - 1]), so exactly one thread (the last non-empty
// segment for lower_bound = N; thread 0 when N = 0) qualifies -- and only that
// thread binary-searches its segment and stores idx[j].  Every warp commits once
// (warp-collective), all lanes but the writer with an empty predicate.
template <int V, int M>
__global__ void __launch_bounds__(BL * Geom<V>::DUP) bins_ghost_kernel(BsArgs a, Ctx c) {
  __shared__ unsigned mb[mbox_words<V>(BL * Geom<V>::DUP)];
  Rep<V, M> rep(c);
  rep.init(mb);
  for (; rep.active(); rep.advance()) {
    const unsigned jq = (unsigned)rep.lblock;
    unsigned key = a.q[jq];
    if constexpr (M == M_FAULT) key = rep.fault(SITE_LOAD, (long long)jq, key);
    const unsigned t = (unsigned)rep.ltid;
    const unsigned seg = (unsigned)(((unsigned long long)a.N + BL - 1) / BL);  // N may be near 2^32
    const unsigned lo = min(a.N, t * seg), hi = min(a.N, lo + seg);
    bool writer;
    if (a.N == 0u) {
      writer = t == 0u;
    } else {
      const bool ge_lo = lo == 0u || (lo < a.N && a.A[lo - 1] < key) || (lo == a.N && a.A[a.N - 1] < key);
      const bool lt_hi = hi > lo && (hi == a.N || key <= a.A[hi - 1]);
      writer = ge_lo && lt_hi;
    }
    unsigned pos = lo;
    if (writer) {  // lower_bound inside [lo, hi]: binary search of the segment
      unsigned l = lo, h = hi;
      while (l < h) {
        const unsigned m = l + (h - l) / 2;
        if (a.A[m] < key) l = m + 1;
        else h = m;
      }
      pos = l;
    }
    if constexpr (M == M_FAULT) pos = rep.fault(SITE_COMPUTE, (long long)jq, pos);
    unsigned w[1] = {pos};
    rep.template commit<1, 0, false, true>(writer ? 1u : 0u, jq, w, a.Q,
                                           [&](unsigned i, unsigned, const unsigned* x) { a.idx[i] = x[0]; });
  }
  rep.finish();
}

}  // namespace

int binarysearch_validate(const rmt_bufs_t* b, int64_t n) {
  int64_t N = b->dims[0], Q = b->dims[1];
  if (b->nbuf < 3 || N < 0 || N >= (1LL << 32) - 64 || Q < 0 || Q >= (1LL << 30) || n != Q ||
      (b->dims[2] != 0 && b->dims[2] != 1) ||
      !buf_ok(b->buf[0], RMT_U32, N) || !buf_ok(b->buf[1], RMT_U32, Q) || !buf_ok(b->buf[2], RMT_U32, Q)) {
    set_error("binarysearch: expected {A:U32[N], q:U32[Q], idx:U32[Q]}, dims {N, Q, mode}, n = Q, mode 0 batched | 1 ghost");
    return RMT_EINVAL;
  }
  return RMT_OK;
}
size_t binarysearch_scratch(int64_t, const int64_t* dims) {
  Levels L = make_levels((unsigned)dims[0]);
  size_t words = 0;
  for (int k = 1; k <= L.T; ++k) words += L.padded[k];
  return (words + FAN) * 4 + 128;  // + the padded tail block
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
  a.plane = a.L.P + 1u;
  a.a32 = ((uintptr_t)a.A % 32) == 0 ? 1u : 0u;
  a.q32 = ((uintptr_t)a.q % 32) == 0 ? 1u : 0u;
  const unsigned Gi = (a.L.vecs_before[a.L.T + 1] + FAN / 4 + BL - 1) / BL;
  const unsigned chunks = (Q + CHUNK - 1) / CHUNK;
  // about 8 waves of logical CTAs: the table copy is amortised over a.iters chunks
  a.iters = (chunks + 148u * BINS_WAVES - 1u) / (148u * BINS_WAVES);
  if (a.iters == 0) a.iters = 1;
  const unsigned G = (chunks + a.iters - 1) / a.iters;
  if (L.bufs->dims[2] == 1)  // ghost mode: one logical CTA per key, no index
    return dispatch(L.variant, L.mode, [&](auto vm) {
      constexpr int V = decltype(vm)::V, M = decltype(vm)::M;
      return launch_std<V>(L, bins_ghost_kernel<V, M>, bins_ghost_kernel<V_NONE, M_NORMAL>, Q, BL, 0, a,
                           "binarysearch/ghost");
    });
  return dispatch(L.variant, L.mode, [&](auto vm) {
    constexpr int V = decltype(vm)::V, M = decltype(vm)::M;
    int rc = RMT_OK;
    if (Q > 0)
      rc = launch_std<V>(L, bins_index_kernel<V, M>, bins_index_kernel<V_NONE, M_NORMAL>, Gi, BL, 0, a,
                         "binarysearch/index");
    if (rc) return rc;
    const size_t smem = (size_t)(Rep<V, M>::SMDUP ? 2u * a.plane : a.L.P) * 4u;
    return launch_std<V>(L, bins_kernel<V, M>, bins_kernel<V_NONE, M_NORMAL>, G, BL, smem, a, "binarysearch",
                         /*mult_inter=*/2);
  });
}

}  // namespace rmt
