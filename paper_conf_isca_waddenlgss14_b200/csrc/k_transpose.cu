// k_transpose.cu -- MatrixTranspose (BASELINE.json configs[1]; not one of the
// paper's 16 kernels).  B[j][i] = A[i][j], 32-bit words.
// 64x64 tile staged in (duplicated, +LDS P:197) shared memory; 16-B coalesced
// loads and stores; one vector commit per 4 output words.
#include "rmt_host.cuh"

namespace rmt {
namespace {

constexpr int BL = 256;
constexpr int TILE = 64;
constexpr int PITCH = TILE + 1;

struct TrArgs {
  const unsigned* A;
  unsigned* B;
  unsigned H, W;     // A is H x W
  unsigned ntx;      // tiles along W
};

template <int V, int M>
__global__ void __launch_bounds__(BL * Geom<V>::DUP) tr_kernel(TrArgs a, Ctx c) {
  constexpr int DUP = Geom<V>::DUP;
  __shared__ unsigned mb[mbox_words<V>(BL * DUP)];
  __shared__ unsigned tile[TILE * PITCH * DUP];
  Rep<V, M> rep(c);
  rep.init(mb);
  const unsigned ty = (unsigned)rep.lblock / a.ntx, tx = (unsigned)rep.lblock % a.ntx;
  const unsigned c4 = (rep.ltid % 16) * 4;
  const unsigned r0 = rep.ltid / 16;
  // load A tile: rows ty*64 + r, cols tx*64 + c4..c4+3
#pragma unroll
  for (int q = 0; q < 4; ++q) {
    unsigned r = r0 + 16 * q;
    unsigned gi = ty * TILE + r, gj = tx * TILE + c4;
    uint4 v = make_uint4(0, 0, 0, 0);
    if (gi < a.H && gj < a.W) v = __ldcs(reinterpret_cast<const uint4*>(a.A + (size_t)gi * a.W + gj));
    unsigned w[4] = {v.x, v.y, v.z, v.w};
#pragma unroll
    for (int k = 0; k < 4; ++k) {
      if constexpr (M == M_FAULT) w[k] = rep.fault(SITE_LOAD, (long long)gi * a.W + gj + k, w[k]);
      rep.sm(tile, r * PITCH + c4 + k) = w[k];
    }
  }
  __syncthreads();
  // store B tile: B row = tx*64 + r (a column of A), cols ty*64 + c4..c4+3
#pragma unroll
  for (int q = 0; q < 4; ++q) {
    unsigned r = r0 + 16 * q;
    unsigned bi = tx * TILE + r, bj = ty * TILE + c4;
    unsigned v[4];
#pragma unroll
    for (int k = 0; k < 4; ++k) {
      v[k] = rep.sm(tile, (c4 + k) * PITCH + r);
      if constexpr (M == M_FAULT) v[k] = rep.fault(SITE_SMEM, (long long)bi * a.H + bj + k, v[k]);
    }
    unsigned mask = (bi < a.W && bj < a.H) ? 0xFu : 0u;
    rep.template commit<4, 0>(mask, bi * a.H + bj, v, a.H * a.W, [&](unsigned idx, unsigned m, const unsigned* w) {
      if (m == 0xFu) __stcs(reinterpret_cast<uint4*>(a.B + idx), make_uint4(w[0], w[1], w[2], w[3]));
      else
        for (int k = 0; k < 4; ++k)
          if ((m >> k) & 1u) a.B[idx + k] = w[k];
    });
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
  unsigned ntx = (W + TILE - 1) / TILE, nty = (H + TILE - 1) / TILE;
  TrArgs a{(const unsigned*)L.bufs->buf[0].ptr, (unsigned*)L.bufs->buf[1].ptr, H, W, ntx};
  return dispatch(L.variant, L.mode, [&](auto vm) {
    constexpr int V = decltype(vm)::V, M = decltype(vm)::M;
    return launch_std<V>(L, tr_kernel<V, M>, tr_kernel<V_NONE, M_NORMAL>, ntx * nty, BL, 0, a, "transpose");
  });
}

}  // namespace rmt
