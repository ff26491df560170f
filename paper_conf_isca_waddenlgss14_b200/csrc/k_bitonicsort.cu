// k_bitonicsort.cu -- BitonicSort ("BitS"; memory-bound, Intra
// <=10% on HD 7790; the worst Inter-Group case, 9.48x).
// Ascending sort of N = 2^n u32 keys with the bitonic network (reading R-BIT1):
// stage s = 0..n-1 (blocks of 2^(s+1)), pass p = s..0: the pair (i, i ^ 2^p),
// bit p of i clear, is put in ascending order iff bit s+1 of i is clear.
//
// B200 design (the FWT's pass structure, compare-exchange instead of
// butterfly): a launch owns 4096-key tiles staged in (duplicated, +LDS) shared
// memory and runs a list of passes whose pair bit lies inside the tile.  Tiles
// are either contiguous (global bits 0..11) or strided (global bits 0..c-1 as
// 2^c contiguous columns, c >= 5, plus b = 12 - c pass bits [s0, s0+b) as rows).
// Schedule: one contiguous launch sorts every tile (stages 0..11, 78 passes);
// then per stage s >= 12, strided launches cover pass bits s..12 (<= 7 per
// launch) and one contiguous launch the passes 11..0.  Inside a launch, passes
// run as register rounds: each thread takes the 16 keys that differ only in a
// window of 4 consecutive tile bits [q, q+4) and applies every consecutive
// pass on those bits (up to 10) before writing back -- one LDS + one STS per
// key per round (compile-time window: immediate smem offsets), min/max per pair.
// HBM: 8 B/key per launch.  The result is the unique sorted sequence, so every
// variant is bitwise equal to `none` and to the oracle.
#include "rmt_host.cuh"

namespace rmt {
namespace {

constexpr int BL = 256;
constexpr int TB_MAX = 12;
constexpr int TE_MAX = 1 << TB_MAX;
constexpr int SM_WORDS = TE_MAX + TE_MAX / 32;  // pad32 swizzle
constexpr int PLANE = SM_WORDS + 16;            // +LDS replica plane, 16 banks apart
constexpr int MAXR = 40, MAXP = 96;

__device__ __forceinline__ int phys(int e) { return e + (e >> 5); }

struct BitRound {
  unsigned char q;          // the round's tile bits are [q, q+4)
  unsigned char np, first;  // passes [first, first + np) of `ops`
  unsigned char run;        // 1: passes are local bits l0, l0-1, .. of ONE stage with a uniform direction
  unsigned char l0, g;      // run: first local bit, direction bit (global)
};
struct BitArgs {
  const unsigned* src;
  unsigned* dst;
  unsigned N;       // keys (real); the tile may be padded with 0xFFFFFFFF
  int tb;           // tile bits
  int s0, b, c;     // strided tile: pass bits [s0, s0+b) as rows, c column bits (b == 0: contiguous)
  int first;        // first launch (LOAD / COMPUTE / SMEM fault sites)
  int nr;
  BitRound r[MAXR];
  unsigned short ops[MAXP];  // l (2 bits) | ld (3 bits, 4 = uniform) << 2 | g (5 bits) << 5
};

__device__ __forceinline__ unsigned gidx(const BitArgs& a, unsigned tile, unsigned e) {
  if (a.b == 0) return (tile << a.tb) | e;
  const unsigned col = e & ((1u << a.c) - 1u), st = e >> a.c;
  const int midb = a.s0 - a.c;
  const unsigned mid = tile & ((1u << midb) - 1u), hi = tile >> midb;
  return (hi << (a.s0 + a.b)) | (st << a.s0) | (mid << a.c) | col;
}

// One pass on local bit L of the 16-key group; direction from local bit LD of
// the key's group index (LD >= 0) or uniform `asc` (LD < 0).
template <int L, int LD>
__device__ __forceinline__ void cmpx(unsigned (&v)[16], bool asc) {
#pragma unroll
  for (int k = 0; k < 16; ++k) {
    if (k & (1 << L)) continue;
    const unsigned x = v[k], y = v[k | (1 << L)];
    const unsigned lo = min(x, y), hi = max(x, y);
    bool up;
    if constexpr (LD >= 0) up = ((k >> LD) & 1) == 0;
    else up = asc;
    v[k] = up ? lo : hi;
    v[k | (1 << L)] = up ? hi : lo;
  }
}

// Ascending compare-exchange on local bits L0, L0-1, ..., L0-NP+1.
template <int L0, int NP>
__device__ __forceinline__ void cmpx_run(unsigned (&v)[16]) {
#pragma unroll
  for (int i = 0; i < NP; ++i) {
    const int L = L0 - i;
#pragma unroll
    for (int k = 0; k < 16; ++k) {
      if (k & (1 << L)) continue;
      const unsigned x = v[k], y = v[k | (1 << L)];
      v[k] = min(x, y);
      v[k | (1 << L)] = max(x, y);
    }
  }
}

template <int L>
__device__ __forceinline__ void cmpx_l(unsigned (&v)[16], int ld, bool asc) {
  switch (ld) {
    case 0: if constexpr (L != 0) cmpx<L, 0>(v, asc); break;
    case 1: if constexpr (L != 1) cmpx<L, 1>(v, asc); break;
    case 2: if constexpr (L != 2) cmpx<L, 2>(v, asc); break;
    case 3: if constexpr (L != 3) cmpx<L, 3>(v, asc); break;
    default: cmpx<L, -1>(v, asc); break;
  }
}

// phys(ebase | k << Q-window) - phys(ebase), for ebase with zeros in bits Q..Q+3
template <int Q>
__device__ __forceinline__ constexpr int coff(int k) {
  return (k << Q) + ((Q >= 5) ? (k << (Q - 5)) : ((k << Q) >> 5));
}

// One round on the 4-bit window [Q, Q+4): thread = one 16-key group.
template <int Q, class R_>
__device__ __forceinline__ void bit_round(const R_& rep, const BitArgs& a, unsigned* tp, unsigned tile,
                                          const BitRound& R, int ri) {
  const int groups = (1 << a.tb) >> 4;
  if (rep.ltid >= groups) return;
  const unsigned gi = (unsigned)rep.ltid;
  const unsigned ebase = (gi & ((1u << Q) - 1u)) | ((gi >> Q) << (Q + 4));
  unsigned* pb = tp + phys((int)ebase);
  unsigned v[16];
#pragma unroll
  for (int k = 0; k < 16; ++k) v[k] = pb[coff<Q>(k)];
  if constexpr (R_::FAULT) {
    if (a.first && ri == 1) {
#pragma unroll
      for (int k = 0; k < 16; ++k) v[k] = rep.fault(SITE_SMEM, (long long)gidx(a, tile, ebase | (k << Q)), v[k]);
    }
  }
  const unsigned gbase = gidx(a, tile, ebase);
  if (R.run) {
    // one stage, uniform direction: a descending pass sorts the complemented
    // keys ascending, so flip once and run pure min/max
    const unsigned flip = ((gbase >> R.g) & 1u) ? 0xFFFFFFFFu : 0u;
#pragma unroll
    for (int k = 0; k < 16; ++k) v[k] ^= flip;
    switch (R.l0 * 4 + R.np - 1) {
      case 0: cmpx_run<0, 1>(v); break;
      case 4: cmpx_run<1, 1>(v); break;
      case 5: cmpx_run<1, 2>(v); break;
      case 8: cmpx_run<2, 1>(v); break;
      case 9: cmpx_run<2, 2>(v); break;
      case 10: cmpx_run<2, 3>(v); break;
      case 12: cmpx_run<3, 1>(v); break;
      case 13: cmpx_run<3, 2>(v); break;
      case 14: cmpx_run<3, 3>(v); break;
      default: cmpx_run<3, 4>(v); break;
    }
#pragma unroll
    for (int k = 0; k < 16; ++k) v[k] ^= flip;
  } else {
    for (int pi = 0; pi < R.np; ++pi) {
      const unsigned op = a.ops[R.first + pi];
      const int l = op & 3, ld = (op >> 2) & 7, g = (op >> 5) & 31;
      const bool asc = ((gbase >> g) & 1u) == 0u;
      switch (l) {
        case 0: cmpx_l<0>(v, ld, asc); break;
        case 1: cmpx_l<1>(v, ld, asc); break;
        case 2: cmpx_l<2>(v, ld, asc); break;
        default: cmpx_l<3>(v, ld, asc); break;
      }
    }
  }
  if constexpr (R_::FAULT) {
    if (a.first && ri == 0) {
#pragma unroll
      for (int k = 0; k < 16; ++k) v[k] = rep.fault(SITE_COMPUTE, (long long)gidx(a, tile, ebase | (k << Q)), v[k]);
    }
  }
  // -LDS: the group's keys are compared as four 4-word records
#pragma unroll
  for (int q = 0; q < 4; ++q) {
    const unsigned w4[4] = {v[4 * q], v[4 * q + 1], v[4 * q + 2], v[4 * q + 3]};
    if (rep.template sts_ok<4>(w4, ebase + (unsigned)q)) {
#pragma unroll
      for (int k = 0; k < 4; ++k) pb[coff<Q>(4 * q + k)] = v[4 * q + k];
    }
  }
}

template <int V, int M>
__global__ void __launch_bounds__(BL * Geom<V>::DUP) bitonic_kernel(BitArgs a, Ctx c) {
  constexpr int DUP = Geom<V>::DUP;
  __shared__ unsigned mb[mbox_words<V>(BL * DUP)];
  __shared__ unsigned tilebuf[Geom<V>::SMDUP == 2 ? PLANE + SM_WORDS : SM_WORDS];
  Rep<V, M> rep(c);
  rep.init(mb);
  for (; rep.active(); rep.advance()) {
    const unsigned tile = (unsigned)rep.lblock;
    const int te = 1 << a.tb;
    unsigned* const tp = &rep.template smp<PLANE>(tilebuf, 0);

    // ---- load (16-B vectors; padding keys beyond N are +inf)
    {
      constexpr int IT = TE_MAX / (4 * BL);
      uint4 f[IT];
#pragma unroll
      for (int it = 0; it < IT; ++it) {
        const int e0 = 4 * (rep.ltid + it * BL);
        const unsigned g = gidx(a, tile, (unsigned)e0);
        if (e0 < te && g + 3 < a.N) {
          f[it] = __ldcs(reinterpret_cast<const uint4*>(a.src + g));
        } else {
          unsigned w[4];
#pragma unroll
          for (int k = 0; k < 4; ++k) w[k] = (e0 + k < te && g + k < a.N) ? a.src[g + k] : 0xFFFFFFFFu;
          f[it] = make_uint4(w[0], w[1], w[2], w[3]);
        }
      }
#pragma unroll
      for (int it = 0; it < IT; ++it) {
        const int e0 = 4 * (rep.ltid + it * BL);
        if (e0 < te) {
          unsigned w[4] = {f[it].x, f[it].y, f[it].z, f[it].w};
          if constexpr (M == M_FAULT) {
            if (a.first) {
              const unsigned g = gidx(a, tile, (unsigned)e0);
#pragma unroll
              for (int k = 0; k < 4; ++k) w[k] = rep.fault(SITE_LOAD, (long long)g + k, w[k]);
            }
          }
          if (rep.template sts_ok<4>(w, (unsigned)e0)) {
#pragma unroll
            for (int k = 0; k < 4; ++k) tp[phys(e0 + k)] = w[k];
          }
        }
      }
    }
    __syncthreads();

    // ---- register rounds
    for (int ri = 0; ri < a.nr; ++ri) {
      const BitRound R = a.r[ri];
      switch (R.q) {
        case 0: bit_round<0>(rep, a, tp, tile, R, ri); break;
        case 1: bit_round<1>(rep, a, tp, tile, R, ri); break;
        case 2: bit_round<2>(rep, a, tp, tile, R, ri); break;
        case 3: bit_round<3>(rep, a, tp, tile, R, ri); break;
        case 4: bit_round<4>(rep, a, tp, tile, R, ri); break;
        case 5: bit_round<5>(rep, a, tp, tile, R, ri); break;
        case 6: bit_round<6>(rep, a, tp, tile, R, ri); break;
        case 7: bit_round<7>(rep, a, tp, tile, R, ri); break;
        default: bit_round<8>(rep, a, tp, tile, R, ri); break;
      }
      __syncthreads();
    }

    // ---- store: one vector commit per 4 keys
#pragma unroll 1
    for (int it = 0; it < TE_MAX / (4 * BL); ++it) {
      const int e0 = 4 * rep.ltid + it * 4 * BL;
      const unsigned g = e0 < te ? gidx(a, tile, (unsigned)e0) : 0u;
      unsigned w[4];
      unsigned mask = 0;
#pragma unroll
      for (int k = 0; k < 4; ++k) {
        const bool in = e0 + k < te && g + k < a.N;
        w[k] = in ? tp[phys(e0 + k)] : 0u;
        mask |= (in ? 1u : 0u) << k;
      }
      rep.template commit<4, 0>(mask, mask ? g : 0u, w, a.N, [&](unsigned idx, unsigned m, const unsigned* x) {
        if (m == 0xFu)
          __stcs(reinterpret_cast<uint4*>(a.dst + idx), make_uint4(x[0], x[1], x[2], x[3]));
        else
          for (int k = 0; k < 4; ++k)
            if ((m >> k) & 1u) a.dst[idx + k] = x[k];
      }, /*defer=*/it < TE_MAX / (4 * BL) - 1);
    }
  }
  rep.finish();
}

int log2u(int64_t n) {
  int m = 0;
  while ((1LL << m) < n) ++m;
  return m;
}

struct Op {
  int s, p;
};

// Tile bit of global bit g (-1: outside the tile).
int tile_bit(const BitArgs& a, int g) {
  if (a.b == 0) return g < a.tb ? g : -1;
  if (g < a.c) return g;
  if (g >= a.s0 && g < a.s0 + a.b) return a.c + (g - a.s0);
  return -1;
}

// Group consecutive passes into rounds on 4-bit windows [q, q+4): a round
// starts at the next pass (tile bit t, window q = clamp(t - 3, 0, tb - 4)) and
// takes every following pass whose bit stays inside the window.
bool build_rounds(BitArgs& a, const Op* ops, int nops) {
  a.nr = 0;
  int np = 0, i = 0;
  while (i < nops) {
    if (a.nr >= MAXR) return false;
    const int t0 = tile_bit(a, ops[i].p);
    int q = t0 - 3;
    if (q > a.tb - 4) q = a.tb - 4;
    if (q < 0) q = 0;
    BitRound& R = a.r[a.nr++];
    R.q = (unsigned char)q;
    R.first = (unsigned char)np;
    int j = i;
    while (j < nops) {
      const int t = tile_bit(a, ops[j].p);
      if (t < q || t >= q + 4) break;
      if (np >= MAXP) return false;
      const int g = ops[j].s + 1;
      const int tg = tile_bit(a, g);
      const int ld = (tg >= q && tg < q + 4) ? tg - q : 4;
      a.ops[np++] = (unsigned short)((t - q) | (ld << 2) | ((g & 31) << 5));
      ++j;
    }
    R.np = (unsigned char)(j - i);
    // a run: one stage, uniform direction, local bits l0, l0-1, ...
    bool run = R.np >= 1 && R.np <= 4;
    const int l0 = a.ops[R.first] & 3;
    for (int k = 0; run && k < R.np; ++k) {
      const unsigned op = a.ops[R.first + k];
      run = ((op >> 2) & 7) == 4 && (int)(op & 3) == l0 - k && ops[i + k].s == ops[i].s;
    }
    R.run = run ? 1 : 0;
    R.l0 = (unsigned char)l0;
    R.g = (unsigned char)(ops[i].s + 1);
    i = j;
  }
  return true;
}

}  // namespace

int bitonicsort_validate(const rmt_bufs_t* b, int64_t n) {
  if (b->nbuf < 2 || n < 1 || n > (1LL << 30) || (n & (n - 1)) || !buf_ok(b->buf[0], RMT_U32, n) ||
      !buf_ok(b->buf[1], RMT_U32, n)) {
    set_error("bitonicsort: expected {keys:U32[N], sorted:U32[N]}, N a power of two in [1, 2^30]");
    return RMT_EINVAL;
  }
  return RMT_OK;
}
size_t bitonicsort_scratch(int64_t, const int64_t*) { return 0; }
int bitonicsort_inter_warps(int64_t, const int64_t*) { return BL / 32; }

int bitonicsort_run(Launch& L) {
  const int n = log2u(L.n);
  const unsigned* in = (const unsigned*)L.bufs->buf[0].ptr;
  unsigned* out = (unsigned*)L.bufs->buf[1].ptr;
  return dispatch(L.variant, L.mode, [&](auto vm) {
    constexpr int V = decltype(vm)::V, M = decltype(vm)::M;
    const int sid = L.ctx.f.sid;
    Op ops[MAXP];
    // launch list: (tile shape, pass list)
    auto launch = [&](const unsigned* src, int tb, int s0, int b, int c, const Op* o, int no, int first,
                      bool final) -> int {
      BitArgs a{};
      a.src = src;
      a.dst = out;
      a.N = (unsigned)L.n;
      a.tb = tb;
      a.s0 = s0;
      a.b = b;
      a.c = c;
      a.first = first;
      if (!build_rounds(a, o, no)) {
        set_error("bitonicsort: round schedule overflow");
        return RMT_EINVAL;
      }
      L.ctx.f.sid = final ? sid : -1;  // STORE_* faults target the final launch
      const unsigned tiles = (unsigned)((L.n + (1 << tb) - 1) >> tb);
      return launch_std<V>(L, bitonic_kernel<V, M>, bitonic_kernel<V_NONE, M_NORMAL>, tiles ? tiles : 1u, BL, 0, a,
                           "bitonicsort");
    };
    int rc;
    const int tb0 = n < 4 ? 4 : (n < TB_MAX ? n : TB_MAX);
    {  // stages 0 .. min(n, tb0) - 1 on contiguous tiles (padded to >= 16 keys)
      int no = 0;
      const int st = n < TB_MAX ? tb0 : TB_MAX;
      for (int s = 0; s < st; ++s)
        for (int p = s; p >= 0; --p) ops[no++] = Op{s, p};
      rc = launch(in, tb0, 0, 0, tb0, ops, no, 1, n <= TB_MAX);
    }
    for (int s = TB_MAX; s < n && rc == RMT_OK; ++s) {
      for (int hi = s; hi >= TB_MAX && rc == RMT_OK;) {  // strided launches, <= 7 pass bits each
        const int lo = hi - 6 > TB_MAX ? hi - 6 : TB_MAX;
        const int b = hi - lo + 1;
        int no = 0;
        for (int p = hi; p >= lo; --p) ops[no++] = Op{s, p};
        rc = launch(out, TB_MAX, lo, b, TB_MAX - b, ops, no, 0, false);
        hi = lo - 1;
      }
      if (rc) break;
      int no = 0;
      for (int p = TB_MAX - 1; p >= 0; --p) ops[no++] = Op{s, p};
      rc = launch(out, TB_MAX, 0, 0, TB_MAX, ops, no, 0, s == n - 1);
    }
    L.ctx.f.sid = sid;
    return rc;
  });
}

}  // namespace rmt
