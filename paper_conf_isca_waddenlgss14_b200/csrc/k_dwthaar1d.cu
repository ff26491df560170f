// k_dwthaar1d.cu -- DwtHaar1D ("DWT"; memory-bound yet with a
// high communication and doubled-group cost under Intra-Group RMT, P:571-575;
// an Inter-Group outlier; a FAST-swizzle beneficiary).
// Full orthonormal Haar decomposition of N = 2^L samples (readings R-DWT1/2):
// per level a_i = RN(RN(c_2i + c_2i+1) * s), d_i = RN(RN(c_2i - c_2i+1) * s),
// s = RN32(1/sqrt 2); y[0] = a_L, y[N>>k + i] = level-k detail i.
//
// B200 design: Haar levels are local, so a pass over 4096-sample tiles
// computes levels 1..10 of every tile in (duplicated, +LDS) shared memory and
// stores each level's details straight to their final place in y (one 16-B
// vector commit per 4 details).  The 4 remaining approximations per tile go to
// scratch, and the next pass treats them as a signal of length N/1024 whose
// output layout is exactly y[0 .. N/1024).  The last pass (signal <= 4096)
// finishes every level and commits [a_L, d_L, d_{L-1,0}, d_{L-1,1}] as one
// vector.  HBM traffic: 8 B/sample (read x once, write y once) + N/256 B.
// The level order is the DAG of R-DWT2, so the fp32 result is unique: every
// variant and every tiling is bit-identical to the fp32-DAG oracle.
#include "rmt_host.cuh"

namespace rmt {
namespace {

constexpr int BL = 256;
constexpr int TB_MAX = 12;
constexpr int TE_MAX = 1 << TB_MAX;
constexpr int PLANE = TE_MAX + 16;  // +LDS replica plane (64 B apart, 16-B aligned)
constexpr unsigned S_BITS = 0x3F3504F3u;  // RN32(1/sqrt 2)

struct DwtArgs {
  const float* src;  // signal of this pass (x, or the previous pass's approximations)
  float* y;          // output; this pass's sub-problem occupies y[0 .. M)
  float* approx;     // !last: 4 approximations per tile
  unsigned M;        // signal length of this pass
  int tb;            // tile bits (tile = 2^tb samples)
  int K;             // levels computed in the loop (half >= 4)
  int last;          // this pass finishes the transform
  int first;         // pass 1 (LOAD / COMPUTE / SMEM fault sites)
};

__device__ __forceinline__ void st_y(float* y, unsigned idx, unsigned m, const unsigned* w) {
  if (m == 0xFu)
    *reinterpret_cast<float4*>(y + idx) =
        make_float4(__uint_as_float(w[0]), __uint_as_float(w[1]), __uint_as_float(w[2]), __uint_as_float(w[3]));
  else
    for (int k = 0; k < 4; ++k)
      if ((m >> k) & 1u) y[idx + k] = __uint_as_float(w[k]);
}

template <int V, int M>
__global__ void __launch_bounds__(BL * Geom<V>::DUP) dwt_kernel(DwtArgs a, Ctx c) {
  constexpr int DUP = Geom<V>::DUP;
  __shared__ unsigned mb[mbox_words<V>(BL * DUP)];
  __shared__ __align__(16) float cbuf[Geom<V>::SMDUP == 2 ? PLANE + TE_MAX : TE_MAX];
  Rep<V, M> rep(c);
  rep.init(mb);
  for (; rep.active(); rep.advance()) {
    const unsigned tile = (unsigned)rep.lblock;
    const int te = 1 << a.tb;
    const float s = __uint_as_float(S_BITS);
    float* const cp = &rep.template smp<PLANE>(cbuf, 0);  // this replica's copy
    const float* src = a.src + (size_t)tile * te;

    // ---- load the tile (all of a thread's 16-B loads in flight first)
    if (te >= 4) {
      constexpr int IT = TE_MAX / (4 * BL);
      const int nv = te >> 2;
      float4 f[IT];
#pragma unroll
      for (int it = 0; it < IT; ++it) {
        const int vi = rep.ltid + it * BL;
        f[it] = vi < nv ? __ldcs(reinterpret_cast<const float4*>(src) + vi) : make_float4(0.f, 0.f, 0.f, 0.f);
      }
#pragma unroll
      for (int it = 0; it < IT; ++it) {
        const int vi = rep.ltid + it * BL;
        if (vi < nv) {  // same predicate in both replicas (a function of ltid)
          unsigned w[4] = {__float_as_uint(f[it].x), __float_as_uint(f[it].y), __float_as_uint(f[it].z),
                           __float_as_uint(f[it].w)};
          if constexpr (M == M_FAULT) {
            if (a.first) {
#pragma unroll
              for (int k = 0; k < 4; ++k) w[k] = rep.fault(SITE_LOAD, (long long)tile * te + 4 * vi + k, w[k]);
            }
          }
          if (rep.template sts_ok<4>(w, (unsigned)(4 * vi)))
            reinterpret_cast<float4*>(cp)[vi] =
                make_float4(__uint_as_float(w[0]), __uint_as_float(w[1]), __uint_as_float(w[2]), __uint_as_float(w[3]));
        }
      }
    } else if (rep.ltid < te) {
      unsigned w = __float_as_uint(src[rep.ltid]);
      if constexpr (M == M_FAULT) {
        if (a.first) w = rep.fault(SITE_LOAD, (long long)tile * te + rep.ltid, w);
      }
      if (rep.sts_ok1(w, (unsigned)rep.ltid)) cp[rep.ltid] = __uint_as_float(w);
    }
    __syncthreads();

    // ---- levels 1..K: thread group g turns c[8g .. 8g+8) into 4 approximations
    // (written back to c[4g .. 4g+4)) and 4 details (one vector commit)
    for (int k = 1; k <= a.K; ++k) {
      const int half = te >> k, ng = half >> 2;
      const int nu = (ng + BL - 1) / BL;  // 1 or 2 (uniform over the CTA)
      float av[2][4], dv[2][4];
#pragma unroll
      for (int u = 0; u < 2; ++u) {
        const int g = rep.ltid + u * BL;
        if (u < nu && g < ng) {
          const float4 p = reinterpret_cast<const float4*>(cp)[2 * g];
          const float4 q = reinterpret_cast<const float4*>(cp)[2 * g + 1];
          float x[8] = {p.x, p.y, p.z, p.w, q.x, q.y, q.z, q.w};
          if constexpr (M == M_FAULT) {
            if (a.first && k == 2) {  // level-1 approximations read back from smem
#pragma unroll
              for (int t = 0; t < 8; ++t) x[t] = rep.faultf(SITE_SMEM, (long long)tile * (te >> 1) + 8 * g + t, x[t]);
            }
          }
#pragma unroll
          for (int i = 0; i < 4; ++i) {
            av[u][i] = __fmul_rn(__fadd_rn(x[2 * i], x[2 * i + 1]), s);
            dv[u][i] = __fmul_rn(__fsub_rn(x[2 * i], x[2 * i + 1]), s);
            if constexpr (M == M_FAULT) {
              if (a.first && k == 1) av[u][i] = rep.faultf(SITE_COMPUTE, (long long)tile * (te >> 1) + 4 * g + i, av[u][i]);
            }
          }
        }
      }
      __syncthreads();  // every read of this level precedes the first write-back
      // a warp none of whose logical threads has a group this level skips the
      // commit: the decision is the same in both replicas (a function of ltid, k)
      const int lw0 = rep.ltid - rep.llane;  // first logical thread of this warp
#pragma unroll
      for (int u = 0; u < 2; ++u) {
        if (u < nu && lw0 + u * BL < ng) {
          const int g = rep.ltid + u * BL;
          const bool act = g < ng;
          if (act) {
            const unsigned aw[4] = {__float_as_uint(av[u][0]), __float_as_uint(av[u][1]), __float_as_uint(av[u][2]),
                                    __float_as_uint(av[u][3])};
            if (rep.template sts_ok<4>(aw, (unsigned)(4 * g)))
              reinterpret_cast<float4*>(cp)[g] = make_float4(av[u][0], av[u][1], av[u][2], av[u][3]);
          }
          unsigned dw[4] = {__float_as_uint(dv[u][0]), __float_as_uint(dv[u][1]), __float_as_uint(dv[u][2]),
                            __float_as_uint(dv[u][3])};
          const unsigned idx = (a.M >> k) + tile * (unsigned)half + 4u * (unsigned)g;
          rep.template commit<4, 0>(act ? 0xFu : 0u, act ? idx : 0u, dw, a.M,
                                    [&](unsigned i, unsigned m, const unsigned* w) { st_y(a.y, i, m, w); },
                                    /*defer=*/u + 1 < nu && lw0 + (u + 1) * BL < ng);
        }
      }
      __syncthreads();
    }

    // ---- the remaining m = min(te, 4) approximations of the tile
    if (rep.warp == 0) {
      const int m = te >> a.K;
      const bool me = rep.ltid == 0;
      unsigned w[4] = {0u, 0u, 0u, 0u};
      if (me) {
        float c0 = cp[0], c1 = m > 1 ? cp[1] : 0.f, c2 = m > 2 ? cp[2] : 0.f, c3 = m > 3 ? cp[3] : 0.f;
        if (!a.last) {
          w[0] = __float_as_uint(c0); w[1] = __float_as_uint(c1); w[2] = __float_as_uint(c2); w[3] = __float_as_uint(c3);
        } else if (m == 4) {
          const float a0 = __fmul_rn(__fadd_rn(c0, c1), s), d0 = __fmul_rn(__fsub_rn(c0, c1), s);
          const float a1 = __fmul_rn(__fadd_rn(c2, c3), s), d1 = __fmul_rn(__fsub_rn(c2, c3), s);
          w[0] = __float_as_uint(__fmul_rn(__fadd_rn(a0, a1), s));
          w[1] = __float_as_uint(__fmul_rn(__fsub_rn(a0, a1), s));
          w[2] = __float_as_uint(d0);
          w[3] = __float_as_uint(d1);
        } else if (m == 2) {
          w[0] = __float_as_uint(__fmul_rn(__fadd_rn(c0, c1), s));
          w[1] = __float_as_uint(__fmul_rn(__fsub_rn(c0, c1), s));
        } else {
          w[0] = __float_as_uint(c0);
        }
      }
      if (a.last) {
        const unsigned mask = me ? ((1u << m) - 1u) : 0u;
        rep.template commit<4, 0>(mask, 0u, w, a.M, [&](unsigned i, unsigned mm, const unsigned* x) { st_y(a.y, i, mm, x); });
      } else {
        rep.template commit<4, 1>(me ? 0xFu : 0u, me ? 4u * tile : 0u, w, a.M >> a.K,
                                  [&](unsigned i, unsigned mm, const unsigned* x) { st_y(a.approx, i, mm, x); });
      }
    }
  }
  rep.finish();
}

int log2u(int64_t n) {
  int m = 0;
  while ((1LL << m) < n) ++m;
  return m;
}

}  // namespace

int dwthaar1d_validate(const rmt_bufs_t* b, int64_t n) {
  if (b->nbuf < 2 || n < 1 || n > (1LL << 30) || (n & (n - 1)) || !buf_ok(b->buf[0], RMT_F32, n) ||
      !buf_ok(b->buf[1], RMT_F32, n)) {
    set_error("dwthaar1d: expected {x,y} F32[N], N a power of two in [1, 2^30]");
    return RMT_EINVAL;
  }
  return RMT_OK;
}
// two ping-pong approximation buffers: N/1024 and N/2^20 floats
size_t dwthaar1d_scratch(int64_t n, const int64_t*) {
  return align_up((size_t)(n / 1024 + 4) * 4, 256) + align_up((size_t)(n / (1 << 20) + 4) * 4, 256);
}
int dwthaar1d_inter_warps(int64_t, const int64_t*) { return BL / 32; }

int dwthaar1d_run(Launch& L) {
  const int64_t N = L.n;
  float* y = (float*)L.bufs->buf[1].ptr;
  float* bufA = (float*)L.scratch;
  float* bufB = (float*)((char*)L.scratch + align_up((size_t)(N / 1024 + 4) * 4, 256));
  return dispatch(L.variant, L.mode, [&](auto vm) {
    constexpr int V = decltype(vm)::V, M = decltype(vm)::M;
    const float* src = (const float*)L.bufs->buf[0].ptr;
    int64_t Mlen = N;
    int first = 1, rc = RMT_OK;
    while (rc == RMT_OK) {
      if (Mlen <= TE_MAX) {
        const int tb = log2u(Mlen);
        DwtArgs a{src, y, nullptr, (unsigned)Mlen, tb, tb > 2 ? tb - 2 : 0, 1, first};
        rc = launch_std<V>(L, dwt_kernel<V, M>, dwt_kernel<V_NONE, M_NORMAL>, 1, BL, 0, a, "dwthaar1d/last");
        break;
      }
      float* out = (src == bufA) ? bufB : bufA;
      DwtArgs a{src, y, out, (unsigned)Mlen, TB_MAX, TB_MAX - 2, 0, first};
      rc = launch_std<V>(L, dwt_kernel<V, M>, dwt_kernel<V_NONE, M_NORMAL>, (unsigned)(Mlen >> TB_MAX), BL, 0, a,
                         "dwthaar1d/pass");
      src = out;
      Mlen >>= (TB_MAX - 2);
      first = 0;
    }
    return rc;
  });
}

}  // namespace rmt
