// k_sobel.cu -- SobelFilter ("SF"; memory-bound, Intra <=10%,
// P:567; Inter slipstreaming).  uchar4 pixels, per channel
//   Gx = i(-1,-1) + 2 i(0,-1) + i(1,-1) - i(-1,1) - 2 i(0,1) - i(1,1)
//   Gy = i(-1,-1) - i(1,-1) + 2 i(-1,0) - 2 i(1,0) + i(-1,1) - i(1,1)
//   O  = min(255, floor(isqrt(Gx^2 + Gy^2) / 2)), borders 0 (readings R-SOB1..5).
//
// Logical thread = 4 horizontally adjacent pixels (16 B) x a vertical strip of
// RY rows with a rolling 3-row register window (each input row is read once
// per thread; the two halo pixels come from L1).  Interior threads (all but the
// image's outer frame) run a copy of the body without bounds checks or border
// selects.  Arithmetic is SIMD within a
// register: two channels per 32-bit word in biased 16-bit lanes (no borrows),
// separable Sobel (vertical smooth / difference per column, then horizontal).
// isqrt: floor(sqrt(s)/2) = isqrt(s/4); computed as floor(sqrt_approx(s/4 + 1/8))
// which is exact for every s whose result is < 256 (margin >= 9.6e-7 relative
// vs approx error < 2^-22); larger results saturate to 255 anyway.  floor is
// one FADD2 with the magic 2^23 - 1/2; saturation one VIMNMX.U16x2 per two
// channels.
#include "rmt_host.cuh"

namespace rmt {
namespace {

constexpr int BL = 256;
// inter_group: the records of SOBEL_GROUP consecutive rows are published as one
// group behind one fence (group flags).  Measured at 8192^2 (x none): 1 row
// 3.89x, 2 3.62x, 3 3.36x, 5 3.41x, 6 3.57x, 8 4.08x; inter_cluster publishes
// every row (deferral there: 2.99 -> 3.04-3.49x); persistent pairs lose (4.0-4.2x).
#ifndef SOBEL_GROUP
#define SOBEL_GROUP 3
#endif
#ifndef SOBEL_INTER_MINB
#define SOBEL_INTER_MINB 4
#endif
#ifndef SOBEL_MULT_INTER
#define SOBEL_MULT_INTER 0
#endif
constexpr int RY = 30;  // output rows per thread (measured: 32 rows 0.174 ms, 30 rows 0.162 ms at 8192^2)

struct SobArgs {
  const unsigned* I;
  unsigned* O;
  unsigned H, W;
  unsigned nbx;  // logical CTAs across a row
};

__device__ __forceinline__ float sqrt_approx(float x) {
  float r;
  asm("sqrt.approx.ftz.f32 %0, %1;" : "=f"(r) : "f"(x));
  return r;
}

// Packed fp32x2 helpers (Blackwell FADD2/FFMA2/FMUL2).
typedef unsigned long long f2_t;
__device__ __forceinline__ f2_t f2(unsigned lo, unsigned hi) {
  f2_t r;
  asm("mov.b64 %0, {%1, %2};" : "=l"(r) : "r"(lo), "r"(hi));
  return r;
}
__device__ __forceinline__ void f2_split(f2_t v, unsigned& lo, unsigned& hi) {
  asm("mov.b64 {%0, %1}, %2;" : "=r"(lo), "=r"(hi) : "l"(v));
}
__device__ __forceinline__ f2_t add2(f2_t a, f2_t b) {
  f2_t r;
  asm("add.rn.f32x2 %0, %1, %2;" : "=l"(r) : "l"(a), "l"(b));
  return r;
}
__device__ __forceinline__ f2_t mul2(f2_t a, f2_t b) {
  f2_t r;
  asm("mul.rn.f32x2 %0, %1, %2;" : "=l"(r) : "l"(a), "l"(b));
  return r;
}
__device__ __forceinline__ f2_t fma2(f2_t a, f2_t b, f2_t c) {
  f2_t r;
  asm("fma.rn.f32x2 %0, %1, %2, %3;" : "=l"(r) : "l"(a), "l"(b), "l"(c));
  return r;
}

// Two channels at once: gw, yw hold two biased 16-bit lanes (value + 1024) of
// Gx and Gy.  Returns two words 2^23 + floor(sqrt_approx(s/4 + 1/8)) (as fp32
// bits; the low 10 bits hold the unsaturated output of the low / high lane
// channel).  The 16-bit lanes become floats F = 2^23 + v through the magic
// exponent (one PRMT each, no conversion pipe); d = F/2 - (2^22 + 512) = Gx/2
// is one exact FFMA2, and s/4 + 1/8 = d^2 + (e^2 + 1/8) two more (every
// intermediate is a multiple of 1/8 below 2^19: exact in fp32).
__device__ __forceinline__ void sobel_mag2(unsigned gw, unsigned yw, unsigned& out_lo, unsigned& out_hi) {
  const unsigned MAG = 0x4B000000u;
  const f2_t half = f2(__float_as_uint(0.5f), __float_as_uint(0.5f));
  const f2_t nb = f2(__float_as_uint(-4194816.0f), __float_as_uint(-4194816.0f));  // -(2^23 + 1024) / 2
  const f2_t d = fma2(f2(__byte_perm(gw, MAG, 0x7610), __byte_perm(gw, MAG, 0x7632)), half, nb);  // Gx / 2
  const f2_t e = fma2(f2(__byte_perm(yw, MAG, 0x7610), __byte_perm(yw, MAG, 0x7632)), half, nb);  // Gy / 2
  const f2_t f = fma2(d, d, fma2(e, e, f2(__float_as_uint(0.125f), __float_as_uint(0.125f))));   // s/4 + 1/8
  unsigned f0, f1;
  f2_split(f, f0, f1);
  const float r0 = sqrt_approx(__uint_as_float(f0));
  const float r1 = sqrt_approx(__uint_as_float(f1));
  // RN(r + 2^23 - 1/2) = 2^23 + floor(r) for r >= sqrt(1/8): r is never a
  // half-integer (2 (2k+1)^2 != 2 s + 1); the caller saturates at 255
  const f2_t r = add2(f2(__float_as_uint(r0), __float_as_uint(r1)), f2(__float_as_uint(8388607.5f), __float_as_uint(8388607.5f)));
  f2_split(r, out_lo, out_hi);
}

struct Row {
  unsigned lo[6], hi[6];  // columns x0-1 .. x0+4, channels (0,2) and (1,3)
};

// Raw words of one input row (columns x0-1 .. x0+4).  IN (interior thread):
// the row and both halo columns are inside the image, no checks; otherwise
// zeros outside the image.
template <bool IN>
__device__ __forceinline__ void load_raw(const SobArgs& a, int y, unsigned x0, bool active, unsigned (&p)[6]) {
  if constexpr (IN) {
    const unsigned* row = a.I + (size_t)y * a.W + x0;
    uint4 c = __ldg(reinterpret_cast<const uint4*>(row));
    p[0] = __ldg(row - 1);
    p[1] = c.x; p[2] = c.y; p[3] = c.z; p[4] = c.w;
    p[5] = __ldg(row + 4);
  } else {
#pragma unroll
    for (int k = 0; k < 6; ++k) p[k] = 0u;
    if (active && y >= 0 && y < (int)a.H) {
      const unsigned* row = a.I + (size_t)y * a.W;
      uint4 c = __ldg(reinterpret_cast<const uint4*>(row + x0));
      p[1] = c.x; p[2] = c.y; p[3] = c.z; p[4] = c.w;
      if (x0 >= 1) p[0] = __ldg(row + x0 - 1);
      if (x0 + 4 < a.W) p[5] = __ldg(row + x0 + 4);
    }
  }
}

// Apply the LOAD-site fault hook and split into 16-bit channel lanes.
template <int V, int M, bool G>
__device__ __forceinline__ void unpack_row(const Rep<V, M, G>& rep, const SobArgs& a, int y, unsigned x0,
                                           unsigned (&p)[6], Row& R) {
  if constexpr (M == M_FAULT) {
    if (y >= 0 && y < (int)a.H) {
#pragma unroll
      for (int k = 0; k < 6; ++k) {
        long long e = (long long)y * a.W + x0 + k - 1;
        if (k == 0 && x0 == 0) continue;
        p[k] = rep.fault(SITE_LOAD, e, p[k]);
      }
    }
  }
#pragma unroll
  for (int k = 0; k < 6; ++k) {
    R.lo[k] = __byte_perm(p[k], 0u, 0x4240);  // channels 0, 2 -> 16-bit lanes
    R.hi[k] = __byte_perm(p[k], 0u, 0x4341);  // channels 1, 3
  }
}

template <bool B>
struct BoolC {
  static constexpr bool value = B;
};

template <int V, int M>
__global__ void __launch_bounds__(BL * Geom<V>::DUP, Geom<V>::DUP == 2 ? 2 : V == V_INTER ? SOBEL_INTER_MINB : 4) sobel_kernel(SobArgs a, Ctx c) {
  __shared__ unsigned mb[mbox_words<V>(BL * Geom<V>::DUP)];
  Rep<V, M, (SOBEL_GROUP > 1 && V == V_INTER)> rep(c);
  rep.init(mb);
  for (; rep.active(); rep.advance()) {
    const unsigned by = (unsigned)rep.lblock / a.nbx, bx = (unsigned)rep.lblock % a.nbx;
    const unsigned x0 = (bx * BL + (unsigned)rep.ltid) * 4;
    const bool active = x0 < a.W;
    const int y0 = (int)(by * RY);
    // Interior thread: its 4 pixels and both halo columns are interior columns,
    // and every row it reads (y0-1 .. y0+RY, plus the last prefetch y0+RY+1) is
    // inside the image: no bounds checks, no border selects.  Most warps.
    // Warp-uniform (commits are warp-collective: a warp never splits between
    // the two bodies).
    const bool interior =
        __all_sync(0xFFFFFFFFu, x0 >= 4u && x0 + 8u <= a.W && y0 >= 1 && (unsigned)y0 + RY + 2u <= a.H);
    auto body = [&](auto in_tag) {
      constexpr bool IN = decltype(in_tag)::value;
      unsigned xin = 0xFu;  // interior columns among this thread's 4 pixels
      if constexpr (!IN) {
        xin = 0u;
#pragma unroll
        for (int p = 0; p < 4; ++p) xin |= ((x0 + p >= 1 && x0 + p < a.W - 1) ? 1u : 0u) << p;
      }
      // one output row from the window (t = y-1, m = y, b = y+1)
      auto row_out = [&](int y, const Row& t, const Row& m, const Row& b) {
        unsigned vs_lo[6], vs_hi[6], vd_lo[6], vd_hi[6];
#pragma unroll
        for (int k = 0; k < 6; ++k) {
          vs_lo[k] = t.lo[k] + 2u * m.lo[k] + b.lo[k];   // <= 1020 per lane
          vs_hi[k] = t.hi[k] + 2u * m.hi[k] + b.hi[k];
          vd_lo[k] = t.lo[k] + 0x01000100u - b.lo[k];    // 256 + (top - bot)
          vd_hi[k] = t.hi[k] + 0x01000100u - b.hi[k];
        }
        bool yin = true;
        if constexpr (!IN) yin = y >= 1 && y < (int)a.H - 1;
        unsigned out[4];
#pragma unroll
        for (int p = 0; p < 4; ++p) {
          const int w = p + 1;
          // biased by 1024 per 16-bit lane
          unsigned gx_lo = vd_lo[w - 1] + 2u * vd_lo[w] + vd_lo[w + 1];
          const unsigned gx_hi = vd_hi[w - 1] + 2u * vd_hi[w] + vd_hi[w + 1];
          const unsigned gy_lo = vs_lo[w - 1] + 0x04000400u - vs_lo[w + 1];
          const unsigned gy_hi = vs_hi[w - 1] + 0x04000400u - vs_hi[w + 1];
          if constexpr (M == M_FAULT) gx_lo = rep.fault(SITE_COMPUTE, (long long)y * a.W + x0 + p, gx_lo);
          unsigned m0, m2, m1, m3;
          sobel_mag2(gx_lo, gy_lo, m0, m2);  // channels 0, 2
          sobel_mag2(gx_hi, gy_hi, m1, m3);  // channels 1, 3
          // two channels per 16-bit lane pair, saturated with one VIMNMX.U16x2 each
          const unsigned h01 = __vminu2(__byte_perm(m0, m1, 0x5410), 0x00FF00FFu);
          const unsigned h23 = __vminu2(__byte_perm(m2, m3, 0x5410), 0x00FF00FFu);
          const unsigned px = __byte_perm(h01, h23, 0x6420);
          if constexpr (IN) out[p] = px;
          else out[p] = (yin && ((xin >> p) & 1u)) ? px : 0u;
        }
        unsigned mask = 0xFu;
        if constexpr (!IN) mask = (active && y < (int)a.H) ? 0xFu : 0u;
        rep.template commit<4, 0>(mask, (unsigned)y * a.W + x0, out, a.H * a.W,
                                  [&](unsigned idx, unsigned mm, const unsigned* w) {
                                    if (mm == 0xFu)
                                      __stcs(reinterpret_cast<uint4*>(a.O + idx), make_uint4(w[0], w[1], w[2], w[3]));
                                    else
                                      for (int k = 0; k < 4; ++k)
                                        if ((mm >> k) & 1u) a.O[idx + k] = w[k];
                                  }, /*defer=*/V == V_INTER && SOBEL_GROUP > 1 && (y - y0) % SOBEL_GROUP != SOBEL_GROUP - 1 && y + 1 < y0 + RY);
      };
      // rolling 3-row window; the raw words of the row after next are in flight
      // while the current row is filtered (one row of prefetch distance)
      Row top, mid, bot;
      unsigned raw[6], nxt[6];
      load_raw<IN>(a, y0 - 1, x0, active, raw);
      unpack_row(rep, a, y0 - 1, x0, raw, top);
      load_raw<IN>(a, y0, x0, active, raw);
      load_raw<IN>(a, y0 + 1, x0, active, nxt);
      unpack_row(rep, a, y0, x0, raw, mid);
#pragma unroll 1
      for (int y = y0; y < y0 + RY; ++y) {
#pragma unroll
        for (int k = 0; k < 6; ++k) raw[k] = nxt[k];
        load_raw<IN>(a, y + 2, x0, active, nxt);
        unpack_row(rep, a, y + 1, x0, raw, bot);
        row_out(y, top, mid, bot);
        top = mid;
        mid = bot;
      }
    };
    if (interior) body(BoolC<true>{});
    else body(BoolC<false>{});
  }
  rep.finish();
}

}  // namespace

int sobel_validate(const rmt_bufs_t* b, int64_t n) {
  int64_t H = b->dims[0], W = b->dims[1];
  if (b->nbuf < 2 || H < 0 || W < 0 || n != H * W || W % 4 || n >= (1LL << 30) || !buf_ok(b->buf[0], RMT_U8X4, n) ||
      !buf_ok(b->buf[1], RMT_U8X4, n)) {
    set_error("sobel: expected {I,O} U8X4[H*W], dims {H,W}, W%4 = 0, H*W < 2^30");
    return RMT_EINVAL;
  }
  return RMT_OK;
}
size_t sobel_scratch(int64_t, const int64_t*) { return 0; }
int sobel_inter_warps(int64_t, const int64_t*) { return BL / 32; }

int sobel_run(Launch& L) {
  const unsigned H = (unsigned)L.bufs->dims[0], W = (unsigned)L.bufs->dims[1];
  const unsigned nbx = (W + 4 * BL - 1) / (4 * BL), nby = (H + RY - 1) / RY;
  SobArgs a{(const unsigned*)L.bufs->buf[0].ptr, (unsigned*)L.bufs->buf[1].ptr, H, W, nbx};
  return dispatch(L.variant, L.mode, [&](auto vm) {
    constexpr int V = decltype(vm)::V, M = decltype(vm)::M;
    return launch_std<V>(L, sobel_kernel<V, M>, sobel_kernel<V_NONE, M_NORMAL>, nbx * nby, BL, 0, a, "sobel", /*mult_inter=*/SOBEL_MULT_INTER,
                         /*mult_cluster=*/0);
  });
}

}  // namespace rmt
