// k_transpose.cu -- MatrixTranspose (BASELINE.json configs[1]; not one of the
// paper's 16 kernels).  B[j][i] = A[i][j], 32-bit words.
//
// A logical CTA moves a 32-row x 128-column strip of A as four 32x32 tiles
// through (duplicated, +LDS P:197) shared memory: 16-B coalesced loads of A
// rows, scalar smem stores into a 33-word-pitch tile, scalar smem loads down
// tile columns, 16-B coalesced stores of B rows -- one vector commit per 4
// output words.  Bank mapping (per warp): load phase r + 4l' + k, store phase
// 4l'' + k + c, both 32 distinct banks; for the intra variants the replica
// planes are 2 words apart mod 4, so the two replicas of every pair also land
// in disjoint banks (conflict-free in every variant).
#include "rmt_host.cuh"

namespace rmt {
namespace {

constexpr int BL = 256;
constexpr int TS = 32;          // tile side
constexpr int NT = 4;           // tiles per logical CTA (along A's columns)
constexpr int PITCH = TS + 1;
constexpr int TWORDS = TS * PITCH;
constexpr int SWORDS = NT * TWORDS;
constexpr int PLANE = SWORDS + 2;  // replica plane offset: == 2 (mod 4)

struct TrArgs {
  const unsigned* A;
  unsigned* B;
  unsigned H, W;     // A is H x W
  unsigned nsx;      // strips along W
};

template <int V, int M>
__global__ void __launch_bounds__(BL * Geom<V>::DUP) tr_kernel(TrArgs a, Ctx c) {
  constexpr int DUP = Geom<V>::DUP;
  __shared__ unsigned mb[mbox_words<V>(BL * DUP)];
  __shared__ unsigned tile[Geom<V>::SMDUP == 2 ? PLANE + SWORDS : SWORDS];
  Rep<V, M, true> rep(c);  // group flags: 4 records per warp
  rep.init(mb);
  for (; rep.active(); rep.advance()) {
    const unsigned ty = (unsigned)rep.lblock / a.nsx, sx = (unsigned)rep.lblock % a.nsx;
    const unsigned r = rep.ltid / 8, l4 = (rep.ltid % 8) * 4;
    // load phase: A row ty*32 + r, columns sx*128 + 32t + l4 .. +3
    uint4 v[NT];
    const unsigned gi = ty * TS + r;
#pragma unroll
    for (int t = 0; t < NT; ++t) {
      const unsigned gj = sx * (NT * TS) + t * TS + l4;
      v[t] = (gi < a.H && gj < a.W) ? __ldcs(reinterpret_cast<const uint4*>(a.A + (size_t)gi * a.W + gj))
                                    : make_uint4(0, 0, 0, 0);
    }
#pragma unroll
    for (int t = 0; t < NT; ++t) {
      unsigned w[4] = {v[t].x, v[t].y, v[t].z, v[t].w};
      const unsigned gj = sx * (NT * TS) + t * TS + l4;
      if constexpr (M == M_FAULT) {
#pragma unroll
        for (int k = 0; k < 4; ++k) w[k] = rep.fault(SITE_LOAD, (long long)gi * a.W + gj + k, w[k]);
      }
      if (rep.template sts_ok<4>(w, t * TWORDS + r * PITCH + l4)) {
#pragma unroll
        for (int k = 0; k < 4; ++k) rep.template smp<PLANE>(tile, t * TWORDS + r * PITCH + l4 + k) = w[k];
      }
    }
    __syncthreads();
    // store phase: B row sx*128 + 32t + c (= a column of A), columns ty*32 + l4 .. +3
    const unsigned cc = rep.ltid / 8;
#pragma unroll
    for (int t = 0; t < NT; ++t) {
      const unsigned bi = sx * (NT * TS) + t * TS + cc, bj = ty * TS + l4;
      unsigned w[4];
#pragma unroll
      for (int k = 0; k < 4; ++k) {
        w[k] = rep.template smp<PLANE>(tile, t * TWORDS + (l4 + k) * PITCH + cc);
        if constexpr (M == M_FAULT) w[k] = rep.fault(SITE_SMEM, (long long)bi * a.H + bj + k, w[k]);
      }
      const unsigned mask = (bi < a.W && bj < a.H) ? 0xFu : 0u;
      rep.template commit<4, 0>(mask, mask ? bi * a.H + bj : 0u, w, a.H * a.W,
                                [&](unsigned idx, unsigned m, const unsigned* x) {
                                  if (m == 0xFu) __stcs(reinterpret_cast<uint4*>(a.B + idx), make_uint4(x[0], x[1], x[2], x[3]));
                                  else
                                    for (int k = 0; k < 4; ++k)
                                      if ((m >> k) & 1u) a.B[idx + k] = x[k];
                                },
                                /*defer=*/t < NT - 1);
    }
  }
  rep.finish();
}

}  // namespace

int transpose_validate(const rmt_bufs_t* b, int64_t n) {
  int64_t H = b->dims[0], W = b->dims[1];
  int dt = b->buf[0].dtype;
  if (b->nbuf < 2 || H < 0 || W < 0 || n != H * W || H % 4 || W % 4 || n >= (1LL << 30) ||
      (dt != RMT_U32 && dt != RMT_F32) || !buf_ok(b->buf[0], dt, n) || !buf_ok(b->buf[1], dt, n)) {
    set_error("transpose: expected {A,B} U32|F32[H*W], dims {H,W}, H%4=W%4=0, H*W < 2^30");
    return RMT_EINVAL;
  }
  return RMT_OK;
}
size_t transpose_scratch(int64_t, const int64_t*) { return 0; }
int transpose_inter_warps(int64_t, const int64_t*) { return BL / 32; }

int transpose_run(Launch& L) {
  unsigned H = (unsigned)L.bufs->dims[0], W = (unsigned)L.bufs->dims[1];
  unsigned nsx = (W + NT * TS - 1) / (NT * TS), nty = (H + TS - 1) / TS;
  TrArgs a{(const unsigned*)L.bufs->buf[0].ptr, (unsigned*)L.bufs->buf[1].ptr, H, W, nsx};
  return dispatch(L.variant, L.mode, [&](auto vm) {
    constexpr int V = decltype(vm)::V, M = decltype(vm)::M;
    return launch_std<V>(L, tr_kernel<V, M>, tr_kernel<V_NONE, M_NORMAL>, nsx * nty, BL, 0, a, "transpose",
                         /*mult_inter=*/4);  // digest records: 4x the resident pairs 2.21 -> 2.10x
  });
}

}  // namespace rmt
