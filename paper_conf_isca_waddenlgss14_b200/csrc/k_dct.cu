// k_dct.cu -- DCT ("DCT"; high Intra overhead despite being
// memory-bound; Inter ~2x and the only kernel hurt by doubling groups,
// P:809).  Forward orthonormal 8x8 DCT-II per block (reading R-DCT1):
//   Y = C X C^T,  C[u][x] = alpha(u) cos((2x+1) u pi / 16).
//
// Logical CTA = NS = 4 vertically consecutive strips of 8 image rows x 256
// columns (32 blocks each), walked with the next strip's loads in flight; logical
// thread (row r, block b) does the row pass Z[r][.] = X[r][.] C^T (8 FMA-chains
// of length 8), Z goes through (duplicated, +LDS) shared memory, then logical
// thread (b, u) does the column pass Y[u][.] = C[u][.] Z and commits its output
// row as two 16-B vector stores.  Fixed FMA order with explicit rounding, so
// every variant is bit-identical.  The C table (fp64 -> fp32, computed here on
// the host, independently of the oracle) travels in the kernel arguments.
#include <math.h>

#include "rmt_host.cuh"
#ifndef DCT_INTER_MINB
#define DCT_INTER_MINB 0  // inter_group: minimum resident CTAs per SM (0: unspecified)
#endif

namespace rmt {
namespace {

constexpr int BL = 256;
constexpr int BLOCKS = 32;       // 8x8 blocks per logical CTA
constexpr int BSTRIDE = 68;      // words per block in smem (64 + 4: conflict-free column pass)
constexpr int ZWORDS = BLOCKS * BSTRIDE;
constexpr int PLANE = ZWORDS + 16;  // replica plane offset (16 banks apart)
#ifndef DCT_NS
#define DCT_NS 4
#endif
constexpr unsigned NS = DCT_NS;     // 8-row strips per logical CTA

struct DctArgs {
  const float* X;
  float* Y;
  unsigned H, W;
  unsigned nbx;  // logical CTAs across a row strip
  unsigned nby;  // 8-row strips
  unsigned v8;   // X is 32-B aligned: 256-bit row loads
  float C[8][8];
};

template <int V, int M>
__global__ void __launch_bounds__(BL * Geom<V>::DUP, V == V_INTER ? DCT_INTER_MINB : 0) dct_kernel(DctArgs a, Ctx c) {
  constexpr int DUP = Geom<V>::DUP;
  __shared__ unsigned mb[mbox_words<V>(BL * DUP)];
  __shared__ __align__(16) float Zs[Geom<V>::SMDUP == 2 ? PLANE + ZWORDS : ZWORDS];
  Rep<V, M> rep(c);
  rep.init(mb);
  for (; rep.active(); rep.advance()) {
    const unsigned bg = (unsigned)rep.lblock / a.nbx, bx = (unsigned)rep.lblock % a.nbx;
    // row pass: logical warp w = image row r of the strip, lane = block b, so a
    // warp's loads are one contiguous 1 KiB row segment (coalesced; with the
    // block-major mapping of the column pass below the loads touched 8 rows per
    // instruction and L1 ran at 98%: 0.203 -> 0.154 ms at 8192^2)
    const int b0 = rep.ltid % BLOCKS, r = rep.ltid / BLOCKS;
    const unsigned col00 = (bx * BLOCKS + b0) * 8;
    const bool active0 = col00 < a.W;
    auto load_x = [&](unsigned by, float (&x)[8]) {
      const unsigned row = by * 8 + r;
      if (active0) {
        if (a.v8) {  // one 256-bit load: the warp's 1 KiB row segment in whole lines
          unsigned w[8];
          ldcs8(a.X + (size_t)row * a.W + col00, w);
#pragma unroll
          for (int y = 0; y < 8; ++y) x[y] = __uint_as_float(w[y]);
        } else {  // X only 16-B aligned (the ABI minimum)
          const float4* src = reinterpret_cast<const float4*>(a.X + (size_t)row * a.W + col00);
          float4 p = __ldcs(src), q = __ldcs(src + 1);
          x[0] = p.x; x[1] = p.y; x[2] = p.z; x[3] = p.w; x[4] = q.x; x[5] = q.y; x[6] = q.z; x[7] = q.w;
        }
      } else {
#pragma unroll
        for (int y = 0; y < 8; ++y) x[y] = 0.0f;
      }
    };
    // A logical CTA walks NS vertically consecutive strips; the next strip's
    // row segment is in flight while this one is transformed (register double
    // buffer: twice the bytes in flight per SM)
    float xn[8];
    load_x(bg * NS, xn);
#pragma unroll 1
    for (unsigned by = bg * NS; by < bg * NS + NS && by < a.nby; ++by) {  // CTA-uniform
    int b = b0;
    unsigned col0 = col00;
    bool active = active0;
    const unsigned row = by * 8 + r;
    float x[8];
#pragma unroll
    for (int y = 0; y < 8; ++y) x[y] = xn[y];
    if (by + 1 < bg * NS + NS && by + 1 < a.nby) load_x(by + 1, xn);
    if constexpr (M == M_FAULT) {
#pragma unroll
      for (int y = 0; y < 8; ++y) x[y] = rep.faultf(SITE_LOAD, (long long)row * a.W + col0 + y, x[y]);
    }
    float z[8];
#pragma unroll
    for (int v = 0; v < 8; ++v) {
      float s = __fmul_rn(x[0], a.C[v][0]);
#pragma unroll
      for (int y = 1; y < 8; ++y) s = __fmaf_rn(x[y], a.C[v][y], s);
      if constexpr (M == M_FAULT) s = rep.faultf(SITE_COMPUTE, (long long)row * a.W + col0 + v, s);
      z[v] = s;
    }
    float* zrow = &rep.template smp<PLANE>(Zs, b * BSTRIDE + r * 8);
    const unsigned zw[8] = {__float_as_uint(z[0]), __float_as_uint(z[1]), __float_as_uint(z[2]), __float_as_uint(z[3]),
                            __float_as_uint(z[4]), __float_as_uint(z[5]), __float_as_uint(z[6]), __float_as_uint(z[7])};
    if (rep.template sts_ok<8>(zw, b * BSTRIDE + r * 8)) {
      reinterpret_cast<float4*>(zrow)[0] = make_float4(z[0], z[1], z[2], z[3]);
      reinterpret_cast<float4*>(zrow)[1] = make_float4(z[4], z[5], z[6], z[7]);
    }
    __syncthreads();
    // column pass: thread (b, u) produces output row u of block b (8 lanes per
    // block: the smem reads of a warp broadcast over 4 blocks, one wavefront;
    // routing the output back through smem for row-major stores was slower)
    b = rep.ltid / 8;
    const int u = rep.ltid % 8;
    col0 = (bx * BLOCKS + b) * 8;
    active = col0 < a.W;
    float y[8];
#pragma unroll
    for (int v = 0; v < 8; ++v) y[v] = 0.0f;
    const float* zb = &rep.template smp<PLANE>(Zs, b * BSTRIDE);
#pragma unroll
    for (int xr = 0; xr < 8; ++xr) {
      float4 p = reinterpret_cast<const float4*>(zb + xr * 8)[0];
      float4 q = reinterpret_cast<const float4*>(zb + xr * 8)[1];
      float zz[8] = {p.x, p.y, p.z, p.w, q.x, q.y, q.z, q.w};
      if constexpr (M == M_FAULT) {
#pragma unroll
        for (int v = 0; v < 8; ++v)
          zz[v] = rep.faultf(SITE_SMEM, (long long)(by * 8 + xr) * a.W + col0 + v, zz[v]);
      }
      const float cu = a.C[u][xr];
#pragma unroll
      for (int v = 0; v < 8; ++v) y[v] = xr == 0 ? __fmul_rn(cu, zz[v]) : __fmaf_rn(cu, zz[v], y[v]);
    }
    // Stores (measured per variant at 8192^2): none, intra_reg and intra_nolds
    // first swap one 16-B half between output rows u and u^4 of a block through
    // a shuffle, so that store h writes rows 4h..4h+3 of the warp's blocks as
    // whole 128-B lines (lanes u < 4: half 0 of row 4h + u; lanes u >= 4: half 1
    // of row 4h + u - 4) -- none 0.155 -> 0.145 ms, intra_reg 0.272 -> 0.253 ms;
    // intra_smem and the inter variants were slower with it and store their own
    // row u directly (8 rows of half-sectors per store).
    constexpr bool XS = (V == V_NONE || V == V_INTRA_REG || V == V_INTRA_NOLDS);
    const bool lowu = u < 4;
    unsigned got[4];
    if constexpr (XS) {
#pragma unroll
      for (int q = 0; q < 4; ++q) got[q] = rep.lshfl_xor(__float_as_uint(lowu ? y[4 + q] : y[q]), 4);
    }
#pragma unroll
    for (int h = 0; h < 2; ++h) {
      unsigned w[4];
      unsigned orow, idx;
      if constexpr (XS) {
#pragma unroll
        for (int q = 0; q < 4; ++q)
          w[q] = lowu ? (h == 0 ? __float_as_uint(y[q]) : got[q]) : (h == 0 ? got[q] : __float_as_uint(y[4 + q]));
        orow = by * 8 + (lowu ? (unsigned)u + 4u * h : (unsigned)u - 4u + 4u * h);
        idx = orow * a.W + col0 + (lowu ? 0u : 4u);
      } else {
#pragma unroll
        for (int q = 0; q < 4; ++q) w[q] = __float_as_uint(y[4 * h + q]);
        orow = by * 8 + u;
        idx = orow * a.W + col0 + 4 * h;
      }
      rep.template commit<4, 0>(active ? 0xFu : 0u, active ? idx : 0u, w, a.H * a.W,
                                [&](unsigned i, unsigned m, const unsigned* v) {
                                  if (m == 0xFu)
                                    __stcs(reinterpret_cast<float4*>(a.Y + i),
                                           make_float4(__uint_as_float(v[0]), __uint_as_float(v[1]),
                                                       __uint_as_float(v[2]), __uint_as_float(v[3])));
                                  else
                                    for (int k = 0; k < 4; ++k)
                                      if ((m >> k) & 1u) a.Y[i + k] = __uint_as_float(v[k]);
                                },
                                /*defer=*/h == 0);
    }
    __syncthreads();  // the column pass has read Zs before the next strip's row pass writes it
    }
  }
  rep.finish();
}

}  // namespace

int dct_validate(const rmt_bufs_t* b, int64_t n) {
  int64_t H = b->dims[0], W = b->dims[1];
  if (b->nbuf < 2 || H < 0 || W < 0 || n != H * W || H % 8 || W % 8 || n >= (1LL << 30) ||
      !buf_ok(b->buf[0], RMT_F32, n) || !buf_ok(b->buf[1], RMT_F32, n)) {
    set_error("dct: expected {X,Y} F32[H*W], dims {H,W}, H%8 = W%8 = 0");
    return RMT_EINVAL;
  }
  return RMT_OK;
}
size_t dct_scratch(int64_t, const int64_t*) { return 0; }
int dct_inter_warps(int64_t, const int64_t*) { return BL / 32; }

int dct_run(Launch& L) {
  const unsigned H = (unsigned)L.bufs->dims[0], W = (unsigned)L.bufs->dims[1];
  const unsigned nbx = (W / 8 + BLOCKS - 1) / BLOCKS, nby = H / 8;
  DctArgs a;
  a.X = (const float*)L.bufs->buf[0].ptr;
  a.Y = (float*)L.bufs->buf[1].ptr;
  a.H = H;
  a.W = W;
  a.nbx = nbx;
  a.nby = nby;
  a.v8 = ((uintptr_t)a.X % 32) == 0 ? 1u : 0u;
  for (int u = 0; u < 8; ++u)  // C[u][x] = alpha(u) cos((2x+1) u pi / 16), in fp64 then rounded
    for (int x = 0; x < 8; ++x)
      a.C[u][x] = (float)((u == 0 ? sqrt(0.125) : 0.5) * cos((2.0 * x + 1.0) * u * 3.14159265358979323846 / 16.0));
  return dispatch(L.variant, L.mode, [&](auto vm) {
    constexpr int V = decltype(vm)::V, M = decltype(vm)::M;
    return launch_std<V>(L, dct_kernel<V, M>, dct_kernel<V_NONE, M_NORMAL>, nbx * ((nby + NS - 1) / NS), BL, 0, a,
                         "dct");
  });
}

}  // namespace rmt
