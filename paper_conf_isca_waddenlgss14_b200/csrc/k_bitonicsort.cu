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
// run as register rounds: each thread takes the 16 keys that differ only in 4
// tile bits and applies every consecutive pass on those bits (up to 10) before
// writing back -- one LDS + one STS per key per round, min/max per pair.
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
  unsigned char bits[4];  // tile bits of the 16-key group, ascending
  unsigned char np, first;  // passes [first, first + np) of `ops`
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

template <int V, int M>
__global__ void __launch_bounds__(BL * Geom<V>::DUP) bitonic_kernel(BitArgs a, Ctx c) {
  constexpr int DUP = Geom<V>::DUP;
  __shared__ unsigned mb[mbox_words<V>(BL * DUP)];
  __shared__ unsigned tilebuf[Geom<V>::SMDUP == 2 ? PLANE + SM_WORDS : SM_WORDS];
  Rep<V, M> rep(c);
  rep.init(mb);
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
  const int groups = te >> 4;
  for (int ri = 0; ri < a.nr; ++ri) {
    const BitRound R = a.r[ri];
    if (rep.ltid < groups) {
      // deposit the thread's group id into the tile bits outside the round
      unsigned ebase = 0, gid = (unsigned)rep.ltid;
      const unsigned inb = (1u << R.bits[0]) | (1u << R.bits[1]) | (1u << R.bits[2]) | (1u << R.bits[3]);
      for (int t = 0; t < a.tb; ++t) {
        if (inb & (1u << t)) continue;
        ebase |= (gid & 1u) << t;
        gid >>= 1;
      }
      auto elem = [&](int k) -> unsigned {  // tile index of group key k
        return ebase | ((k & 1) << R.bits[0]) | (((k >> 1) & 1) << R.bits[1]) | (((k >> 2) & 1) << R.bits[2]) |
               (((k >> 3) & 1) << R.bits[3]);
      };
      int off[16];
      unsigned v[16];
#pragma unroll
      for (int k = 0; k < 16; ++k) {
        off[k] = phys((int)elem(k));
        v[k] = tp[off[k]];
      }
      if constexpr (M == M_FAULT) {
        if (a.first && ri == 1) {
#pragma unroll
          for (int k = 0; k < 16; ++k) v[k] = rep.fault(SITE_SMEM, (long long)gidx(a, tile, elem(k)), v[k]);
        }
      }
      const unsigned gbase = gidx(a, tile, ebase);
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
      if constexpr (M == M_FAULT) {
        if (a.first && ri == 0) {
#pragma unroll
          for (int k = 0; k < 16; ++k) v[k] = rep.fault(SITE_COMPUTE, (long long)gidx(a, tile, elem(k)), v[k]);
        }
      }
      // -LDS: the whole group's keys are compared as four 4-word records
#pragma unroll
      for (int q = 0; q < 4; ++q) {
        const unsigned w4[4] = {v[4 * q], v[4 * q + 1], v[4 * q + 2], v[4 * q + 3]};
        if (rep.template sts_ok<4>(w4, ebase + (unsigned)q)) {
#pragma unroll
          for (int k = 0; k < 4; ++k) tp[off[4 * q + k]] = v[4 * q + k];
        }
      }
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

// Group consecutive passes into register rounds of <= 4 distinct tile bits.
bool build_rounds(BitArgs& a, const Op* ops, int nops) {
  a.nr = 0;
  int np = 0, i = 0;
  while (i < nops) {
    if (a.nr >= MAXR) return false;
    unsigned set = 0;
    int cnt = 0, j = i;
    while (j < nops) {
      const int t = tile_bit(a, ops[j].p);
      if (!(set & (1u << t))) {
        if (cnt == 4) break;
        set |= 1u << t;
        ++cnt;
      }
      ++j;
    }
    for (int t = 0; cnt < 4 && t < a.tb; ++t)  // pad the group to 4 bits
      if (!(set & (1u << t))) { set |= 1u << t; ++cnt; }
    BitRound& R = a.r[a.nr++];
    int q = 0;
    for (int t = 0; t < a.tb; ++t)
      if (set & (1u << t)) R.bits[q++] = (unsigned char)t;
    R.first = (unsigned char)np;
    R.np = (unsigned char)(j - i);
    for (int k = i; k < j; ++k) {
      if (np >= MAXP) return false;
      const int t = tile_bit(a, ops[k].p);
      int l = 0;
      while (R.bits[l] != t) ++l;
      const int g = ops[k].s + 1;
      const int tg = tile_bit(a, g);
      int ld = 4;
      for (int z = 0; z < 4; ++z)
        if (tg >= 0 && R.bits[z] == tg) ld = z;
      a.ops[np++] = (unsigned short)(l | (ld << 2) | ((g & 31) << 5));
    }
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
