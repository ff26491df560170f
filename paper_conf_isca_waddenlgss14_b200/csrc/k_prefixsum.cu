// k_prefixsum.cu -- PrefixSum ("PS"; Intra comm >1/2 of the
// overhead; FAST helps).  Inclusive scan of u32 mod 2^32
// (readings R-PS1, R-PS2), single pass with decoupled look-back: 8 B/elem.
//
// Tile = 256 logical threads x 16 items.  Tile ids are taken in start order
// (none/intra: a tile counter; inter: the RMT pair id, itself start-ordered,
// P:679), so look-back never waits on an unstarted tile.  Integer addition is
// associative, so every variant -- and every look-back timing -- produces the
// identical result (determinism rule: look-back only on integers).
// Tile status words are liveness-critical stores (other CTAs spin on them):
// they are committed with LIVE=true (reading R-RMT5).
#include "rmt_host.cuh"

namespace rmt {
namespace {

constexpr int BL = 256;
constexpr int ITEMS = 16;
constexpr unsigned TILE = BL * ITEMS;
constexpr unsigned long long FLAG_AGG = 1ull << 32, FLAG_INC = 2ull << 32;

struct PsArgs {
  const unsigned* x;
  unsigned* y;
  unsigned long long* status;  // [ntiles]: (flag << 32) | value
  unsigned* tile_counter;
  unsigned n;
};

template <int V, int M>
__global__ void __launch_bounds__(BL * Geom<V>::DUP) ps_kernel(PsArgs a, Ctx c) {
  constexpr int DUP = Geom<V>::DUP;
  constexpr int LW = 32 / DUP;
  constexpr int NLW = BL / LW;  // logical warps per CTA
  __shared__ unsigned mb[mbox_words<V>(BL * DUP)];
  __shared__ unsigned s_wtot[NLW * DUP];
  __shared__ unsigned s_bcast[2 * DUP];
  __shared__ unsigned s_tile;
  Rep<V, M> rep(c);
  rep.init(mb);
  unsigned tile;
  if constexpr (V == V_INTER) {
    tile = (unsigned)rep.lblock;
  } else {
    if (threadIdx.x == 0) s_tile = atomicAdd(a.tile_counter, 1u);
    __syncthreads();
    tile = s_tile;
  }
  const unsigned base = tile * TILE + (unsigned)rep.ltid * ITEMS;
  unsigned v[ITEMS];
  if (base + ITEMS <= a.n) {
#pragma unroll
    for (int q = 0; q < ITEMS / 4; ++q) {
      uint4 w = __ldg(reinterpret_cast<const uint4*>(a.x + base) + q);
      v[4 * q] = w.x; v[4 * q + 1] = w.y; v[4 * q + 2] = w.z; v[4 * q + 3] = w.w;
    }
  } else {
#pragma unroll
    for (int i = 0; i < ITEMS; ++i) v[i] = base + i < a.n ? a.x[base + i] : 0u;
  }
  if constexpr (M == M_FAULT) {
#pragma unroll
    for (int i = 0; i < ITEMS; ++i) v[i] = rep.fault(SITE_LOAD, (long long)base + i, v[i]);
  }
  // thread-local inclusive scan
#pragma unroll
  for (int i = 1; i < ITEMS; ++i) v[i] += v[i - 1];
  unsigned tsum = rep.fault(SITE_COMPUTE, (long long)tile * BL + rep.ltid, v[ITEMS - 1]);
  // logical-warp inclusive scan of thread totals
  unsigned ws = tsum;
#pragma unroll
  for (int d = 1; d < LW; d <<= 1) {
    unsigned u = rep.lshfl_up(ws, d);
    if (rep.llane >= d) ws += u;
  }
  const int lw = rep.ltid / LW;
  if (rep.llane == LW - 1) rep.sm(s_wtot, lw) = ws;
  __syncthreads();
  // warp 0: scan warp totals, then look-back
  if (rep.warp == 0) {
    unsigned t = rep.llane < NLW ? rep.sm(s_wtot, rep.llane) : 0u;
    if constexpr (M == M_FAULT) t = rep.fault(SITE_SMEM, (long long)tile * BL + rep.llane * LW, t);
    unsigned inc = t;
#pragma unroll
    for (int d = 1; d < LW; d <<= 1) {
      unsigned u = rep.lshfl_up(inc, d);
      if (rep.llane >= d) inc += u;
    }
    const unsigned agg = rep.lshfl_idx(inc, NLW - 1);
    if (rep.llane < NLW) rep.sm(s_wtot, rep.llane) = inc - t;  // exclusive per logical warp
    auto publish = [&](unsigned long long st, bool live_word) {
      unsigned w2[2] = {(unsigned)st, (unsigned)(st >> 32)};
      unsigned mask = (rep.llane == 0 && live_word) ? 3u : 0u;
      rep.template commit<2, 2, true>(mask, 2u * tile, w2, 2u * (unsigned)((a.n + TILE - 1) / TILE),
                                      [&](unsigned idx, unsigned m, const unsigned* w) {
                                        if (m == 3u)
                                          st_relaxed64(a.status + idx / 2,
                                                       (unsigned long long)w[0] | ((unsigned long long)w[1] << 32));
                                      });
    };
    unsigned excl = 0;
    if (tile == 0) {
      publish(FLAG_INC | agg, true);
    } else {
      publish(FLAG_AGG | agg, true);
      // decoupled look-back over a window of LW predecessors
      int p = (int)tile - 1;
      while (true) {
        const int idx = p - rep.llane;
        unsigned long long st;
        while (true) {  // warp-uniform spin until the whole window is valid
          st = idx >= 0 ? ld_relaxed64(a.status + idx) : FLAG_INC;
          // Intra: the pair shares one status load (replicated input, load path
          // outside the SoR) so both replicas take identical control flow.
          if constexpr (Rep<V, M>::INTRA) st = __shfl_sync(FULL, st, rep.lane & ~1);
          if (__ballot_sync(FULL, (st >> 32) == 0ull) == 0u) break;
        }
        const unsigned incmask = rep.lballot((st >> 32) == 2ull);
        const int stop = incmask ? __ffs(incmask) - 1 : LW - 1;  // closest inclusive predecessor
        unsigned contrib = rep.llane <= stop ? (unsigned)st : 0u;
#pragma unroll
        for (int m = LW / 2; m >= 1; m >>= 1) contrib += rep.lshfl_xor(contrib, m);
        excl += contrib;
        if (incmask) break;
        p -= LW;
      }
      publish(FLAG_INC | (excl + agg), true);
    }
    if (rep.llane == 0) rep.sm(s_bcast, 0) = excl;
  }
  __syncthreads();
  const unsigned prefix = rep.sm(s_bcast, 0) + rep.sm(s_wtot, lw) + (ws - tsum);
#pragma unroll
  for (int q = 0; q < ITEMS / 4; ++q) {
    const unsigned e0 = base + 4 * q;
    unsigned w[4];
    unsigned mask = 0;
#pragma unroll
    for (int k = 0; k < 4; ++k) {
      w[k] = prefix + v[4 * q + k];
      mask |= (e0 + k < a.n ? 1u : 0u) << k;
    }
    rep.template commit<4, 0>(mask, e0, w, a.n, [&](unsigned idx, unsigned m, const unsigned* x) {
      if (m == 0xFu) __stcs(reinterpret_cast<uint4*>(a.y + idx), make_uint4(x[0], x[1], x[2], x[3]));
      else
        for (int k = 0; k < 4; ++k)
          if ((m >> k) & 1u) a.y[idx + k] = x[k];
    });
  }
  rep.finish();
}

}  // namespace

int prefixsum_validate(const rmt_bufs_t* b, int64_t n) {
  if (b->nbuf < 2 || n < 0 || n >= (1LL << 30) || !buf_ok(b->buf[0], RMT_U32, n) || !buf_ok(b->buf[1], RMT_U32, n)) {
    set_error("prefixsum: expected {x,y} U32[n], n < 2^30");
    return RMT_EINVAL;
  }
  return RMT_OK;
}
size_t prefixsum_scratch(int64_t n, const int64_t*) {
  size_t tiles = (size_t)((n + TILE - 1) / TILE);
  return 256 + tiles * 8;
}
int prefixsum_inter_warps(int64_t, const int64_t*) { return BL / 32; }

int prefixsum_run(Launch& L) {
  unsigned n = (unsigned)L.n;
  unsigned G = (n + TILE - 1) / TILE;
  if (G == 0) return RMT_OK;
  int rc = cuda_check(cudaMemsetAsync(L.scratch, 0, L.scratch_bytes, L.stream), "prefixsum: reset status");
  if (rc) return rc;
  PsArgs a{(const unsigned*)L.bufs->buf[0].ptr, (unsigned*)L.bufs->buf[1].ptr,
           (unsigned long long*)(L.scratch + 256), (unsigned*)L.scratch, n};
  return dispatch(L.variant, L.mode, [&](auto vm) {
    constexpr int V = decltype(vm)::V, M = decltype(vm)::M;
    return launch_std<V>(L, ps_kernel<V, M>, ps_kernel<V_NONE, M_NORMAL>, G, BL, 0, a, "prefixsum");
  });
}

}  // namespace rmt
