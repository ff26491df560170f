// k_prefixsum.cu -- PrefixSum ("PS"; Intra comm >1/2 of the
// overhead; FAST helps).  Inclusive scan of u32 mod 2^32
// (readings R-PS1, R-PS2).
//
// B200 design: reduce-then-scan over NCH = 1184 contiguous chunks (a multiple
// of 4096-element tiles each).  A single-pass decoupled look-back was measured
// (globaltimer trace of every tile) to serialise behind straggler tiles: one
// slow tile's aggregate stalls every later tile's look-back while the waiting
// CTAs hold all SM slots, so HBM idles.  Here no CTA waits on another:
//   pass 1: each logical CTA sums its chunk and commits ONE partial (u32);
//   pass 2: each logical CTA sums the partials of the chunks before it (its
//           carry-in; <= 1183 L2-resident words), then scans its chunk tile by
//           tile with a running carry and commits y.  Pass 2 visits chunks in
//           the REVERSE order of pass 1, so the chunks pass 1 read last are
//           still L2-resident.
// Integer addition is associative: every variant produces the identical result.
#include "rmt_host.cuh"
#ifndef PS_INTER_MINB
#define PS_INTER_MINB 0  // inter_group: minimum resident CTAs per SM (0: unspecified)
#endif

namespace rmt {
namespace {

constexpr int BL = 256;
constexpr int ITEMS = 16;
constexpr unsigned TILE = BL * ITEMS;   // 4096 elements
constexpr unsigned NCH = 148u * 8u;     // chunks (logical CTAs per pass)

struct PsArgs {
  const unsigned* x;
  unsigned* y;
  unsigned* partial;   // [NCH]
  unsigned n;
  unsigned chunk;      // elements per chunk (multiple of TILE)
  unsigned nch;        // chunks actually used
  unsigned carry_in;   // added to every output (multi-GPU shard offset)
  unsigned v8;         // x is 32-B aligned: 256-bit loads where a thread's run allows
  const unsigned long long* totals;  // multi-GPU: every rank's total (all-gathered on the device), or null
  unsigned rank;       // totals[0 .. rank) are added to the carry (mod 2^32)
  unsigned excl;       // exclusive scan (y_i = sum_{j<i} x_j)
};

// u32 sum over the logical CTA (logical warps + duplicated smem)
template <class R>
__device__ __forceinline__ unsigned block_sum_u32(const R& rep, unsigned s, unsigned* sw) {
  constexpr int LW = R::LW;
  constexpr int NLW = BL / LW;
#pragma unroll
  for (int m = LW / 2; m >= 1; m >>= 1) s += rep.lshfl_xor(s, m);
  if (rep.llane == 0 && rep.sts_ok1(s, rep.ltid / LW)) rep.sm(sw, rep.ltid / LW) = s;
  __syncthreads();
  unsigned t = rep.llane < NLW ? rep.sm(sw, rep.llane) : 0u;
#pragma unroll
  for (int m = LW / 2; m >= 1; m >>= 1) t += rep.lshfl_xor(t, m);
  __syncthreads();
  return t;
}

template <int V, int M>
__global__ void __launch_bounds__(BL * Geom<V>::DUP) ps_reduce_kernel(PsArgs a, Ctx c) {
  constexpr int DUP = Geom<V>::DUP;
  __shared__ unsigned mb[mbox_words<V>(BL * DUP)];
  __shared__ unsigned sw[(BL / (32 / DUP)) * Geom<V>::SMDUP];
  Rep<V, M> rep(c);
  rep.init(mb);
  for (; rep.active(); rep.advance()) {
    const unsigned ch = (unsigned)rep.lblock;
    const unsigned lo = ch * a.chunk, hi = min(a.n, lo + a.chunk);
    unsigned s = 0;
    // 16-B coalesced loads, 4 in flight per thread (chunk starts are 16-B aligned)
    // blocks of 16 BL elements visited from the END of the chunk: the scan pass
    // reads each chunk from its start, which is then what L2 still holds
    const unsigned nblk = hi > lo ? (hi - lo + 16 * BL - 1) / (16 * BL) : 0u;
#pragma unroll 1
    for (unsigned b = nblk; b-- > 0;) {
      const unsigned e = lo + b * 16 * BL + 4 * rep.ltid;
      uint4 v[4];
#pragma unroll
      for (int u = 0; u < 4; ++u) {
        const unsigned f = e + u * 4 * BL;
        if (f + 4 <= hi) {
          v[u] = __ldg(reinterpret_cast<const uint4*>(a.x + f));
        } else {  // ragged tail of the array
          v[u].x = f < hi ? a.x[f] : 0u;
          v[u].y = f + 1 < hi ? a.x[f + 1] : 0u;
          v[u].z = f + 2 < hi ? a.x[f + 2] : 0u;
          v[u].w = 0u;
        }
      }
#pragma unroll
      for (int u = 0; u < 4; ++u) {
        if constexpr (M == M_FAULT) {
          const unsigned f = e + u * 4 * BL;
          v[u].x = rep.fault(SITE_LOAD, (long long)f, v[u].x);
          v[u].y = rep.fault(SITE_LOAD, (long long)f + 1, v[u].y);
          v[u].z = rep.fault(SITE_LOAD, (long long)f + 2, v[u].z);
          v[u].w = rep.fault(SITE_LOAD, (long long)f + 3, v[u].w);
        }
        s += v[u].x + v[u].y + v[u].z + v[u].w;
      }
    }
    s = rep.fault(SITE_COMPUTE, (long long)ch * BL + rep.ltid, s);
    const unsigned t = block_sum_u32(rep, s, sw);
    if (rep.warp == 0) {  // one store per CTA leaves the SoR ("ghost" warps)
      unsigned w[1] = {t};
      rep.template commit<1, 2>(rep.llane == 0 ? 1u : 0u, ch, w, a.nch,
                                [&](unsigned i, unsigned, const unsigned* x) { a.partial[i] = x[0]; });
    }
  }
  rep.finish();
}

template <int V, int M>
__global__ void __launch_bounds__(BL * Geom<V>::DUP, V == V_INTER && PS_INTER_MINB ? PS_INTER_MINB : 4 / Geom<V>::DUP) ps_scan_kernel(PsArgs a, Ctx c) {
  constexpr int DUP = Geom<V>::DUP;
  constexpr int LW = 32 / DUP;
  constexpr int NLW = BL / LW;
  // none / inter (32-lane logical warps): NQ = 4 sub-tiles of 4 BL elements, a
  // thread owning 4 consecutive elements of each (coalesced 16-B accesses, one
  // 512-B line per warp instruction; with 16 consecutive elements per thread
  // every access touched twice the sectors and L1 ran at 80%: 0.168 -> 0.135 ms
  // at 2^26).  Intra (16-lane logical warps): one run of 16 per thread -- its
  // accesses are 256 B per instruction either way, and 4 scan chains cost more
  // shuffles than they save (measured: intra_reg 0.18 -> 0.195 ms).
  constexpr int NQ = DUP == 1 ? ITEMS / 4 : 1;  // sub-tiles per tile
  constexpr int RUN = ITEMS / NQ;                // consecutive elements per thread and sub-tile
  constexpr unsigned SUB = RUN * BL;             // elements per sub-tile
  constexpr bool FLAT = NQ * NLW == LW;          // every (sub-tile, warp) total on its own lane
  __shared__ unsigned mb[mbox_words<V>(BL * DUP)];
  __shared__ unsigned sw[NQ * NLW * Geom<V>::SMDUP];
  Rep<V, M, true> rep(c);  // group flags: many records per warp
  rep.init(mb);
  for (; rep.active(); rep.advance()) {
    const unsigned ch = a.nch - 1u - (unsigned)rep.lblock;  // reverse order: L2-hot chunks first
    // carry-in: sum of the partials of all earlier chunks (L2-resident)
    unsigned cs = 0;
    for (unsigned i = rep.ltid; i < ch; i += BL) cs += __ldcg(a.partial + i);
    if (a.totals)  // exclusive prefix of the lower ranks' totals: no host round trip
      for (unsigned i = rep.ltid; i < a.rank; i += BL) cs += (unsigned)__ldcg(a.totals + i);
    unsigned carry = a.carry_in + block_sum_u32(rep, cs, sw);
    const unsigned lo = ch * a.chunk, hi = min(a.n, lo + a.chunk);
    const int lw = rep.ltid / LW;
    // Register double buffer: the next tile's loads are in flight while this
    // tile is scanned and stored.  v[q * RUN + k] = x[t0 + q SUB + ltid RUN + k].
    auto load_tile = [&](unsigned t0, unsigned (&v)[ITEMS]) {
#pragma unroll
      for (int q = 0; q < NQ; ++q) {
        const unsigned e = t0 + q * SUB + RUN * (unsigned)rep.ltid;
        if (e + RUN <= hi) {
          if (RUN % 8 == 0 && a.v8) {  // 256-bit loads: 32 B per lane, whole lines per instruction
#pragma unroll
            for (int j = 0; j < RUN / 8; ++j) {
              unsigned w[8];
              ldcs8(a.x + e + 8 * j, w);
#pragma unroll
              for (int k = 0; k < 8; ++k) v[q * RUN + 8 * j + k] = w[k];
            }
          } else {
#pragma unroll
            for (int j = 0; j < RUN / 4; ++j) {
              uint4 w = __ldcs(reinterpret_cast<const uint4*>(a.x + e) + j);
              v[q * RUN + 4 * j] = w.x; v[q * RUN + 4 * j + 1] = w.y;
              v[q * RUN + 4 * j + 2] = w.z; v[q * RUN + 4 * j + 3] = w.w;
            }
          }
        } else {
#pragma unroll
          for (int k = 0; k < RUN; ++k) v[q * RUN + k] = e + k < hi ? a.x[e + k] : 0u;
        }
      }
    };
    unsigned nxt[ITEMS];
    if (lo < hi) load_tile(lo, nxt);
#pragma unroll 1
    for (unsigned t0 = lo; t0 < hi; t0 += TILE) {  // uniform trip count per CTA
      unsigned v[ITEMS];
#pragma unroll
      for (int i = 0; i < ITEMS; ++i) v[i] = nxt[i];
      if (t0 + TILE < hi) load_tile(t0 + TILE, nxt);
      if constexpr (M == M_FAULT) {
#pragma unroll
        for (int i = 0; i < ITEMS; ++i)
          v[i] = rep.fault(SITE_LOAD, (long long)t0 + (i / RUN) * SUB + RUN * rep.ltid + (i % RUN), v[i]);
      }
      unsigned tsum[NQ], ws[NQ];
#pragma unroll
      for (int q = 0; q < NQ; ++q) {  // thread-local inclusive scans
#pragma unroll
        for (int k = 1; k < RUN; ++k) v[q * RUN + k] += v[q * RUN + k - 1];
        tsum[q] = ws[q] = v[q * RUN + RUN - 1];
      }
#pragma unroll
      for (int d = 1; d < LW; d <<= 1) {  // logical-warp scans, NQ independent chains
#pragma unroll
        for (int q = 0; q < NQ; ++q) {
          const unsigned u = rep.lshfl_up(ws[q], d);
          if (rep.llane >= d) ws[q] += u;
        }
      }
#pragma unroll
      for (int q = 0; q < NQ; ++q)  // warp totals, sub-tile-major
        if (rep.llane == LW - 1 && rep.sts_ok1(ws[q], q * NLW + lw)) rep.sm(sw, q * NLW + lw) = ws[q];
      __syncthreads();
      unsigned pre[NQ];  // exclusive prefix of this thread's sub-tile-q run within the tile
      unsigned total;
      if constexpr (FLAT) {
        // lane l holds total l = (sub-tile l / NLW, warp l % NLW): one scan over the lanes
        unsigned wt = rep.sm(sw, rep.llane);
        if constexpr (M == M_FAULT) wt = rep.fault(SITE_SMEM, (long long)ch * BL + rep.llane, wt);
        unsigned winc = wt;
#pragma unroll
        for (int d = 1; d < LW; d <<= 1) {
          const unsigned u = rep.lshfl_up(winc, d);
          if (rep.llane >= d) winc += u;
        }
        const unsigned wex = winc - wt;
#pragma unroll
        for (int q = 0; q < NQ; ++q) pre[q] = rep.lshfl_idx(wex, q * NLW + lw);
        total = rep.lshfl_idx(winc, LW - 1);
      } else {
        unsigned wt[NQ], winc[NQ];
#pragma unroll
        for (int q = 0; q < NQ; ++q) {
          wt[q] = rep.llane < NLW ? rep.sm(sw, q * NLW + rep.llane) : 0u;
          if constexpr (M == M_FAULT) wt[q] = rep.fault(SITE_SMEM, (long long)ch * BL + q * NLW + rep.llane, wt[q]);
          winc[q] = wt[q];
        }
#pragma unroll
        for (int d = 1; d < NLW; d <<= 1) {
#pragma unroll
          for (int q = 0; q < NQ; ++q) {
            const unsigned u = rep.lshfl_up(winc[q], d);
            if (rep.llane >= d) winc[q] += u;
          }
        }
        total = 0;
#pragma unroll
        for (int q = 0; q < NQ; ++q) {
          pre[q] = total + rep.lshfl_idx(winc[q] - wt[q], lw);
          total += rep.lshfl_idx(winc[q], NLW - 1);
        }
      }
      __syncthreads();  // sw is reused by the next tile
#pragma unroll
      for (int i = 0; i < ITEMS / 4; ++i) {
        const int q = (4 * i) / RUN;
        const unsigned e0 = t0 + q * SUB + RUN * (unsigned)rep.ltid + (4 * i) % RUN;
        const unsigned prefix = carry + pre[q] + (ws[q] - tsum[q]);
        unsigned w[4];
        unsigned mask = 0;
#pragma unroll
        for (int k = 0; k < 4; ++k) {
          // exclusive: the run's inclusive value one element back (0 at a run start)
          const int ii = 4 * i + k;
          const unsigned vx = (ii % RUN == 0) ? 0u : v[ii > 0 ? ii - 1 : 0];
          w[k] = prefix + (a.excl ? vx : v[ii]);
          mask |= (e0 + k < hi ? 1u : 0u) << k;
        }
        rep.template commit<4, 0>(mask, mask ? e0 : 0u, w, a.n, [&](unsigned idx, unsigned m, const unsigned* x) {
          if (m == 0xFu) __stcs(reinterpret_cast<uint4*>(a.y + idx), make_uint4(x[0], x[1], x[2], x[3]));
          else
            for (int k = 0; k < 4; ++k)
              if ((m >> k) & 1u) a.y[idx + k] = x[k];
        }, /*defer=*/i < ITEMS / 4 - 1);
      }
      carry += total;
    }
  }
  rep.finish();
}

// ---------------------------------------------------------------- fp32 scan
// The fp32 secondary (reading R-PS3): one FIXED association order, identical in
// every variant, so the replicas (and none) are bitwise equal and the result is
// deterministic -- a thread scans its RUN = 16 consecutive elements sequentially,
// segments of 16 logical lanes scan the thread totals Kogge-Stone (d = 1, 2, 4,
// 8), the 16 segment totals of a tile are scanned the same way, tiles chain
// sequentially inside a chunk, and a chunk's carry-in is the sum of the earlier
// chunks' partials (lane l of a segment sums partials l, l + 16, ... in order,
// then a 16-lane xor tree -- IEEE addition commutes, so every lane holds the
// same bits).  A 32-lane (none / inter) warp is two 16-lane segments doing the
// same work as a 16-lane intra logical warp.  No look-back: its order would
// depend on timing.
constexpr int FSEG = 16;

template <class R>
__device__ __forceinline__ float fadd_seg_scan(const R& rep, float x) {  // inclusive, 16-lane segments
#pragma unroll
  for (int d = 1; d < FSEG; d <<= 1) {
    const float u = __uint_as_float(rep.lshfl_up(__float_as_uint(x), d));
    if ((rep.llane & (FSEG - 1)) >= d) x = __fadd_rn(u, x);
  }
  return x;
}
template <class R>
__device__ __forceinline__ float fadd_seg_all(const R& rep, float x) {  // the same total in every lane
#pragma unroll
  for (int m = FSEG / 2; m >= 1; m >>= 1) x = __fadd_rn(x, __uint_as_float(rep.lshfl_xor(__float_as_uint(x), m)));
  return x;
}
// Fixed-order fp32 sum over the logical CTA's 256 logical threads: segment xor
// trees, then the 16 segment totals (shared memory) by the same tree.
template <class R>
__device__ __forceinline__ float block_sum_f32(const R& rep, float s, unsigned* sw) {
  s = fadd_seg_all(rep, s);
  const unsigned seg = (unsigned)rep.ltid / FSEG;
  if ((rep.llane & (FSEG - 1)) == 0 && rep.sts_ok1(__float_as_uint(s), seg)) rep.sm(sw, seg) = __float_as_uint(s);
  __syncthreads();
  float t = __uint_as_float(rep.sm(sw, rep.llane & (FSEG - 1)));
  t = fadd_seg_all(rep, t);
  __syncthreads();
  return t;
}

template <int V, int M>
__global__ void __launch_bounds__(BL * Geom<V>::DUP) ps_reduce_f32_kernel(PsArgs a, Ctx c) {
  __shared__ unsigned mb[mbox_words<V>(BL * Geom<V>::DUP)];
  __shared__ unsigned sw[FSEG * Geom<V>::SMDUP];
  Rep<V, M> rep(c);
  rep.init(mb);
  const float* x = reinterpret_cast<const float*>(a.x);
  for (; rep.active(); rep.advance()) {
    const unsigned ch = (unsigned)rep.lblock;
    const unsigned lo = ch * a.chunk, hi = min(a.n, lo + a.chunk);
    float s = 0.0f;
    // thread t sums elements lo + TILE b + 16 t .. + 15 of every tile b, in order
#pragma unroll 1
    for (unsigned t0 = lo; t0 < hi; t0 += TILE) {
      const unsigned e = t0 + ITEMS * (unsigned)rep.ltid;
      float v[ITEMS];
      if (e + ITEMS <= hi) {
#pragma unroll
        for (int j = 0; j < ITEMS / 4; ++j) {
          const float4 w = __ldg(reinterpret_cast<const float4*>(x + e) + j);
          v[4 * j] = w.x; v[4 * j + 1] = w.y; v[4 * j + 2] = w.z; v[4 * j + 3] = w.w;
        }
      } else {
#pragma unroll
        for (int k = 0; k < ITEMS; ++k) v[k] = e + k < hi ? x[e + k] : 0.0f;
      }
#pragma unroll
      for (int k = 0; k < ITEMS; ++k) {
        if constexpr (M == M_FAULT) v[k] = rep.faultf(SITE_LOAD, (long long)e + k, v[k]);
        s = __fadd_rn(s, v[k]);
      }
    }
    s = rep.faultf(SITE_COMPUTE, (long long)ch * BL + rep.ltid, s);
    const float t = block_sum_f32(rep, s, sw);
    if (rep.warp == 0) {  // one store per CTA leaves the SoR ("ghost" warps)
      unsigned w[1] = {__float_as_uint(t)};
      rep.template commit<1, 2>(rep.llane == 0 ? 1u : 0u, ch, w, a.nch,
                                [&](unsigned i, unsigned, const unsigned* xx) { a.partial[i] = xx[0]; });
    }
  }
  rep.finish();
}

template <int V, int M>
__global__ void __launch_bounds__(BL * Geom<V>::DUP) ps_scan_f32_kernel(PsArgs a, Ctx c) {
  __shared__ unsigned mb[mbox_words<V>(BL * Geom<V>::DUP)];
  __shared__ unsigned sw[FSEG * Geom<V>::SMDUP];
  Rep<V, M> rep(c);
  rep.init(mb);
  const float* x = reinterpret_cast<const float*>(a.x);
  for (; rep.active(); rep.advance()) {
    const unsigned ch = a.nch - 1u - (unsigned)rep.lblock;  // reverse order: L2-hot chunks first
    // carry-in: the earlier chunks' partials, lane l of every segment summing
    // partials l, l + 16, ... in order, then the segment's xor tree
    float cs = 0.0f;
    for (unsigned i = rep.llane & (FSEG - 1); i < ch; i += FSEG) cs = __fadd_rn(cs, __uint_as_float(__ldcg(a.partial + i)));
    float carry = fadd_seg_all(rep, cs);
    const unsigned lo = ch * a.chunk, hi = min(a.n, lo + a.chunk);
    const unsigned seg = (unsigned)rep.ltid / FSEG;
#pragma unroll 1
    for (unsigned t0 = lo; t0 < hi; t0 += TILE) {  // uniform trip count per CTA
      const unsigned e = t0 + ITEMS * (unsigned)rep.ltid;
      float v[ITEMS];
      if (e + ITEMS <= hi) {
#pragma unroll
        for (int j = 0; j < ITEMS / 4; ++j) {
          const float4 w = __ldcs(reinterpret_cast<const float4*>(x + e) + j);
          v[4 * j] = w.x; v[4 * j + 1] = w.y; v[4 * j + 2] = w.z; v[4 * j + 3] = w.w;
        }
      } else {
#pragma unroll
        for (int k = 0; k < ITEMS; ++k) v[k] = e + k < hi ? x[e + k] : 0.0f;
      }
      if constexpr (M == M_FAULT) {
#pragma unroll
        for (int k = 0; k < ITEMS; ++k) v[k] = rep.faultf(SITE_LOAD, (long long)e + k, v[k]);
      }
#pragma unroll
      for (int k = 1; k < ITEMS; ++k) v[k] = __fadd_rn(v[k - 1], v[k]);  // the thread's run, in order
      const float ws = fadd_seg_scan(rep, v[ITEMS - 1]);               // segment-inclusive thread totals
      float ex = __uint_as_float(rep.lshfl_up(__float_as_uint(ws), 1));
      if ((rep.llane & (FSEG - 1)) == 0) ex = 0.0f;                    // segment-exclusive
      if ((rep.llane & (FSEG - 1)) == FSEG - 1 && rep.sts_ok1(__float_as_uint(ws), seg))
        rep.sm(sw, seg) = __float_as_uint(ws);
      __syncthreads();
      float wt = __uint_as_float(rep.sm(sw, rep.llane & (FSEG - 1)));  // the tile's 16 segment totals
      if constexpr (M == M_FAULT) wt = rep.faultf(SITE_SMEM, (long long)ch * BL + (rep.llane & (FSEG - 1)), wt);
      const float winc = fadd_seg_scan(rep, wt);
      const int g0 = rep.llane & ~(FSEG - 1);
      // (the shuffle runs in every lane -- warp-collective -- and segment 0 discards it)
      const unsigned segw = rep.lshfl_idx(__float_as_uint(winc), g0 + (seg == 0u ? 0 : (int)seg - 1));
      const float segpre = seg == 0u ? 0.0f : __uint_as_float(segw);
      const float total = __uint_as_float(rep.lshfl_idx(__float_as_uint(winc), g0 + FSEG - 1));
      __syncthreads();  // sw is reused by the next tile
      const float base = __fadd_rn(__fadd_rn(carry, segpre), ex);
#pragma unroll
      for (int i = 0; i < ITEMS / 4; ++i) {
        const unsigned e0 = e + 4 * i;
        unsigned w[4];
        unsigned mask = 0;
#pragma unroll
        for (int k = 0; k < 4; ++k) {
          const int ii = 4 * i + k;
          const float yi = a.excl ? (ii == 0 ? base : __fadd_rn(base, v[ii > 0 ? ii - 1 : 0])) : __fadd_rn(base, v[ii]);
          w[k] = __float_as_uint(yi);
          mask |= (e0 + k < hi ? 1u : 0u) << k;
        }
        rep.template commit<4, 0>(mask, mask ? e0 : 0u, w, a.n, [&](unsigned idx, unsigned m, const unsigned* xx) {
          if (m == 0xFu) __stcs(reinterpret_cast<uint4*>(a.y + idx), make_uint4(xx[0], xx[1], xx[2], xx[3]));
          else
            for (int k = 0; k < 4; ++k)
              if ((m >> k) & 1u) a.y[idx + k] = xx[k];
        }, /*defer=*/i < ITEMS / 4 - 1);
      }
      carry = __fadd_rn(carry, total);
    }
  }
  rep.finish();
}

}  // namespace

int prefixsum_validate(const rmt_bufs_t* b, int64_t n) {
  const bool tot = b->nbuf >= 3 && b->buf[2].ptr != nullptr;
  const int64_t flags = b->dims[2];
  const int dt = (flags & 2) ? RMT_F32 : RMT_U32;
  if ((flags & ~3LL) != 0 || ((flags & 2) && (tot || b->dims[0] != 0))) {
    set_error("prefixsum: dims[2] flags are bit 0 exclusive, bit 1 fp32 (fp32: no carry_in, no totals)");
    return RMT_EINVAL;
  }
  if (b->nbuf < 2 || n < 0 || n >= (1LL << 30) || !buf_ok(b->buf[0], dt, n) || !buf_ok(b->buf[1], dt, n) ||
      (tot && (b->buf[2].dtype != RMT_U64 || ((uintptr_t)b->buf[2].ptr % 16) != 0 || b->dims[1] < 0 ||
               b->dims[1] > b->buf[2].numel))) {
    set_error("prefixsum: expected {x,y} U32[n], n < 2^30, dims {carry_in}; optionally totals:U64[G] with dims "
              "{carry_in, rank}");
    return RMT_EINVAL;
  }
  return RMT_OK;
}
size_t prefixsum_scratch(int64_t, const int64_t*) { return NCH * 4; }
int prefixsum_inter_warps(int64_t, const int64_t*) { return BL / 32; }

int prefixsum_run(Launch& L) {
  const unsigned n = (unsigned)L.n;
  if (n == 0) return RMT_OK;
  const unsigned tiles = (n + TILE - 1) / TILE;
  const unsigned tiles_per_chunk = (tiles + NCH - 1) / NCH;
  const unsigned chunk = tiles_per_chunk * TILE;
  const unsigned nch = (n + chunk - 1) / chunk;
  PsArgs a{(const unsigned*)L.bufs->buf[0].ptr, (unsigned*)L.bufs->buf[1].ptr, (unsigned*)L.scratch, n, chunk, nch,
           (unsigned)(L.bufs->dims[0] & 0xFFFFFFFFu), ((uintptr_t)L.bufs->buf[0].ptr % 32) == 0 ? 1u : 0u,
           L.bufs->nbuf >= 3 ? (const unsigned long long*)L.bufs->buf[2].ptr : nullptr, (unsigned)L.bufs->dims[1],
           (unsigned)(L.bufs->dims[2] & 1)};
  const bool f32 = (L.bufs->dims[2] & 2) != 0;
  return dispatch(L.variant, L.mode, [&](auto vm) {
    constexpr int V = decltype(vm)::V, M = decltype(vm)::M;
    if (f32) {
      int rc = launch_std<V>(L, ps_reduce_f32_kernel<V, M>, ps_reduce_f32_kernel<V_NONE, M_NORMAL>, nch, BL, 0, a,
                             "prefixsum/reduce_f32");
      if (rc) return rc;
      return launch_std<V>(L, ps_scan_f32_kernel<V, M>, ps_scan_f32_kernel<V_NONE, M_NORMAL>, nch, BL, 0, a,
                           "prefixsum/scan_f32");
    }
    int rc = launch_std<V>(L, ps_reduce_kernel<V, M>, ps_reduce_kernel<V_NONE, M_NORMAL>, nch, BL, 0, a,
                           "prefixsum/reduce");
    if (rc) return rc;
    return launch_std<V>(L, ps_scan_kernel<V, M>, ps_scan_kernel<V_NONE, M_NORMAL>, nch, BL, 0, a, "prefixsum/scan");
  });
}

}  // namespace rmt
