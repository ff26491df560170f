// k_floydwarshall.cu -- FloydWarshall ("FW"; memory-bound with
// minimal Intra overhead at large sizes; Inter ~2x; FAST
// slower).  All-pairs shortest paths, canonical k order (readings
// R-FW1..4): for k: if D[i][k] + D[k][j] < D[i][j]: D[i][j] = that, P[i][j] = k.
//
// One launch per k (naive schedule, the faithful primary: row k and column k
// do not change during step k, so the in-place update is race-free and P is
// unique).  Logical thread = 4 consecutive j of one row i: 16-B loads of
// D[i][j..], D[k][j..], one broadcast D[i][k]; the stores are CONDITIONAL (only
// improving relaxations write) and are committed with a per-word
// predicate mask: (mask, address, D words) and (mask, address, P words).
// D (n^2 u32 = 64 MiB at n = 4096) stays L2-resident across passes.
#include <list>
#include <mutex>
#include <string>
#include <utility>

#include "rmt_host.cuh"

namespace rmt {
namespace {

constexpr int BL = 256;

struct FwArgs {
  unsigned* D;
  unsigned* P;
  unsigned n;
  unsigned k;
};

__device__ __forceinline__ void store4(unsigned* base, unsigned idx, unsigned m, const unsigned* v) {
  if (m == 0xFu) *reinterpret_cast<uint4*>(base + idx) = make_uint4(v[0], v[1], v[2], v[3]);
  else
    for (int q = 0; q < 4; ++q)
      if ((m >> q) & 1u) base[idx + q] = v[q];
}

// P[i][j] = i for all (i, j) (reading R-FW2).
template <int V, int M>
__global__ void __launch_bounds__(BL * Geom<V>::DUP) fw_init_kernel(FwArgs a, Ctx c) {
  __shared__ unsigned mb[mbox_words<V>(BL * Geom<V>::DUP)];
  Rep<V, M> rep(c);
  rep.init(mb);
  for (; rep.active(); rep.advance()) {
    const unsigned e0 = ((unsigned)rep.lblock * BL + (unsigned)rep.ltid) * 4;
    const unsigned nn = a.n * a.n;
    unsigned w[4];
    unsigned i = e0 / a.n;
#pragma unroll
    for (int q = 0; q < 4; ++q) w[q] = i;
    rep.template commit<4, 2>(e0 < nn ? 0xFu : 0u, e0 < nn ? e0 : 0u, w, nn,
                              [&](unsigned idx, unsigned m, const unsigned* v) { store4(a.P, idx, m, v); });
  }
  rep.finish();
}

// One pass k.  Each logical thread handles VPT 16-B vectors strided by the CTA
// width (coalesced), all loads in flight before the first use.  VPT per
// variant, measured at n = 4096 (B200): none 4 (52 -> 40 ms), intra 2 (an
// intra warp carries half the distinct bytes, so more vectors per thread),
// inter 2 with group flags (one published group of 4 records per warp and
// logical CTA: 703 -> 497 ms at n = 4096 as n launches; 4 was slower, 799 ms;
// the cooperative single launch below then gives 456 ms).
#ifndef FW_VPT_INTER
#define FW_VPT_INTER 2
#endif
#ifndef FW_VPT_INTRA
#define FW_VPT_INTRA 2
#endif
#ifndef FW_VPT_NONE
#define FW_VPT_NONE 4
#endif
template <int V>
constexpr int fw_vpt() {
  return (V == V_INTER || V == V_CLUSTER) ? FW_VPT_INTER : V == V_NONE ? FW_VPT_NONE : FW_VPT_INTRA;
}

// Logical CTA lb of pass k: (row i, column chunk of BL*4*VPT words), so the row
// and chunk are CTA-uniform (no per-thread division).  `kf` is the pass index
// the fault hooks see (the global fault element is k * n^2 + e).
template <int VPT, class R>
__device__ __forceinline__ void fw_block(R& rep, const FwArgs& a, unsigned k, unsigned lb) {
  constexpr int M = R::FAULT ? M_FAULT : M_NORMAL;
  const unsigned nn = a.n * a.n;
  const unsigned cpr = (a.n + BL * 4 * VPT - 1) / (BL * 4 * VPT);
  const unsigned i = lb / cpr;
  const unsigned jc = (lb - i * cpr) * (BL * 4 * VPT);
  const unsigned dik0 = a.D[(size_t)i * a.n + k];  // one broadcast word per CTA row
  // all VPT vector pairs in flight before the first use (L2 latency-bound:
  // an intra warp carries half the distinct bytes of an unprotected warp)
  uint4 dkj[VPT], dij[VPT];
#pragma unroll
  for (int it = 0; it < VPT; ++it) {
    const unsigned j = jc + ((unsigned)it * BL + (unsigned)rep.ltid) * 4;
    dkj[it] = make_uint4(0, 0, 0, 0);
    dij[it] = make_uint4(0, 0, 0, 0);
    if (j < a.n) {
      dkj[it] = *reinterpret_cast<const uint4*>(a.D + (size_t)k * a.n + j);
      dij[it] = *reinterpret_cast<const uint4*>(a.D + i * a.n + j);
    }
  }
#pragma unroll
  for (int it = 0; it < VPT; ++it) {
    const unsigned j = jc + ((unsigned)it * BL + (unsigned)rep.ltid) * 4;
    const bool active = j < a.n;
    const unsigned e0 = i * a.n + j;
    unsigned dik = dik0;
    unsigned kj[4] = {dkj[it].x, dkj[it].y, dkj[it].z, dkj[it].w};
    unsigned ij[4] = {dij[it].x, dij[it].y, dij[it].z, dij[it].w};
    if constexpr (M == M_FAULT) {
      dik = rep.fault(SITE_LOAD, (long long)i * a.n + k, dik);
#pragma unroll
      for (int q = 0; q < 4; ++q) ij[q] = rep.fault(SITE_LOAD, (long long)e0 + q, ij[q]);
    }
    unsigned nd[4], np[4], mask = 0;
#pragma unroll
    for (int q = 0; q < 4; ++q) {
      unsigned cand = dik + kj[q];
      if constexpr (M == M_FAULT) cand = rep.fault(SITE_COMPUTE, (long long)e0 + q, cand);
      const bool better = active && cand < ij[q];
      mask |= (better ? 1u : 0u) << q;
      nd[q] = cand;
      np[q] = k;
    }
    rep.template commit<4, 0, false, true>(mask, active ? e0 : 0u, nd, nn,
                                           [&](unsigned idx, unsigned m, const unsigned* v) { store4(a.D, idx, m, v); },
                                           /*defer=*/true);
    // one published group per logical CTA: every commit but the last is
    // deferred (2 VPT <= the ring depth)
    rep.template commit<4, 1, false, true>(mask, active ? e0 : 0u, np, nn,
                                           [&](unsigned idx, unsigned m, const unsigned* v) { store4(a.P, idx, m, v); },
                                           /*defer=*/it < VPT - 1);
  }
}

template <int V, int M>
__global__ void __launch_bounds__(BL * Geom<V>::DUP) fw_pass_kernel(FwArgs a, Ctx c) {
  __shared__ unsigned mb[mbox_words<V>(BL * Geom<V>::DUP)];
  Rep<V, M, V == V_INTER> rep(c);
  rep.init(mb);
  for (; rep.active(); rep.advance()) fw_block<fw_vpt<V>()>(rep, a, a.k, (unsigned)rep.lblock);
  rep.finish();
}

// Inter-Group FloydWarshall as ONE cooperative launch: 2P resident CTAs (P
// replica pairs, one ticket and one queue region per pair for the whole run)
// walk the logical CTAs of pass k, meet at a grid barrier, and go on to pass
// k + 1 -- instead of n launches that each take tickets, regions and an exit
// count for thousands of short-lived CTA pairs.  The
// barrier orders every consumer's committed D stores of pass k before any
// replica's loads of pass k + 1.  Fault builds see per-pass fault descriptors
// (the host encodes the pass: elem = k0 n^2 + e).
#ifndef FW_BAR_NS
#define FW_BAR_NS 32  // grid-barrier poll back-off (ns)
#endif
__device__ __forceinline__ void grid_barrier(unsigned* bar, unsigned nctas) {
  __syncthreads();
  if (threadIdx.x == 0) {
    const unsigned gen = ld_acquire(bar + 1);
    __threadfence();
    if (atomicAdd(bar, 1u) == nctas - 1u) {
      bar[0] = 0u;
      st_release(bar + 1, gen + 1u);
    } else {
      while (ld_acquire(bar + 1) == gen)
        if (FW_BAR_NS) __nanosleep(FW_BAR_NS);
    }
  }
  __syncthreads();
}

template <int V, int M>
__global__ void __launch_bounds__(BL * Geom<V>::DUP) fw_coop_kernel(FwArgs a, Ctx c, unsigned* bar) {
  __shared__ unsigned mb[mbox_words<V>(BL * Geom<V>::DUP)];
  Ctx cf = c;  // fault builds: the descriptor is re-aimed at each pass
  Rep<V, M, true> rep(cf);
  rep.init(mb);
  const int first = rep.lblock;
  const long long nn = (long long)a.n * a.n;
  for (unsigned k = 0; k < a.n; ++k) {
    if constexpr (M == M_FAULT) {
      cf.f = c.f;
      if ((long long)k == c.f.elem / nn) cf.f.elem = c.f.elem - (long long)k * nn;
      else cf.f.site = -1;
    }
    for (int lb = first; lb < c.nblocks; lb += rep.lstride) {
      rep.lblock = lb;
      fw_block<fw_vpt<V>()>(rep, a, k, (unsigned)lb);
    }
    grid_barrier(bar, 2u * (unsigned)c.pairs);
  }
  rep.finish();
}

}  // namespace

int floydwarshall_validate(const rmt_bufs_t* b, int64_t n) {
  if (b->nbuf < 2 || n < 0 || n % 4 || n * n >= (1LL << 30) || !buf_ok(b->buf[0], RMT_U32, n * n) ||
      !buf_ok(b->buf[1], RMT_U32, n * n)) {
    set_error("floydwarshall: expected {D (in/out), P} U32[n*n], n%4 = 0, n*n < 2^30");
    return RMT_EINVAL;
  }
  return RMT_OK;
}
size_t floydwarshall_scratch(int64_t, const int64_t*) { return 64; }  // inter_group grid barrier
int floydwarshall_inter_warps(int64_t, const int64_t*) { return BL / 32; }

namespace {

// inter_group: the whole pass sequence as one cooperative launch (fw_coop_kernel).
template <int V, int M>
int fw_coop_launch(Launch& L, const FwArgs& a, unsigned Gp) {
  int per_sm = 0, dev = 0, nsm = 148;
  cudaGetDevice(&dev);
  cudaDeviceGetAttribute(&nsm, cudaDevAttrMultiProcessorCount, dev);
  if (cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, fw_coop_kernel<V, M>, Geom<V>::block(BL), 0) !=
          cudaSuccess ||
      per_sm < 2)
    return cuda_check(cudaErrorInvalidConfiguration, "fw/coop occupancy");
  Ctx c = L.ctx;
  unsigned P = (unsigned)(per_sm * nsm / 2);
  if (P > (unsigned)c.R) P = (unsigned)c.R;  // one queue region per pair, no hand-over
  if (P > Gp) P = Gp;
  c.nblocks = (int)Gp;
  c.pairs = (int)P;
  c.lstride = (int)P;
  unsigned* bar = (unsigned*)L.scratch;
  cudaLaunchConfig_t cfg = {};
  cfg.gridDim = dim3(2 * P);
  cfg.blockDim = dim3(Geom<V>::block(BL));
  cfg.dynamicSmemBytes = 0;
  cfg.stream = L.stream;
  cudaLaunchAttribute at[1];
  at[0].id = cudaLaunchAttributeCooperative;  // every CTA co-resident: the grid barrier cannot deadlock
  at[0].val.cooperative = 1;
  cfg.attrs = at;
  cfg.numAttrs = 1;
  int rc = cuda_check(cudaLaunchKernelEx(&cfg, fw_coop_kernel<V, M>, a, c, bar), "fw/coop");
  if (!rc) L.launches += 1;
  return rc;
}

// The n + 1 launches of one FloydWarshall call, issued on L.stream.
int fw_issue(Launch& L) {
  const unsigned n = (unsigned)L.n;
  const unsigned nn = n * n;
  const unsigned G = (nn / 4 + BL - 1) / BL;  // init: one vector per thread
  FwArgs a{(unsigned*)L.bufs->buf[0].ptr, (unsigned*)L.bufs->buf[1].ptr, n, 0};
  // Fault element = k0 * n^2 + e: the pass k0 and the element e.
  const FaultDesc f = L.ctx.f;
  const unsigned k0 = (unsigned)(f.elem / nn);
  return dispatch(L.variant, L.mode, [&](auto vm) {
    constexpr int V = decltype(vm)::V, M = decltype(vm)::M;
    // passes: VPT vectors per thread (INFLATE runs the V_NONE kernel: its VPT)
    const unsigned vpt = L.inflate ? (unsigned)fw_vpt<V_NONE>() : (unsigned)fw_vpt<V>();
    const unsigned Gp = n * ((n + BL * 4 * vpt - 1) / (BL * 4 * vpt));  // rows x column chunks
    L.ctx.f.site = -1;  // the init pass carries no fault
    int rc = launch_std<V>(L, fw_init_kernel<V, M>, fw_init_kernel<V_NONE, M_NORMAL>, G, BL, 0, a, "fw/init");
    L.ctx.f = f;
    if constexpr (V == V_INTER) {
      if (!L.inflate && M != M_NOCOMM) return rc ? rc : fw_coop_launch<V, M>(L, a, Gp);
    }
    for (unsigned k = 0; k < n && rc == RMT_OK; ++k) {
      a.k = k;
      L.ctx.f = f;
      if (k == k0) L.ctx.f.elem = f.elem - (long long)k0 * nn;
      else L.ctx.f.site = -1;
      rc = launch_std<V>(L, fw_pass_kernel<V, M>, fw_pass_kernel<V_NONE, M_NORMAL>, Gp, BL, 0, a, "fw/pass",
                          /*mult_inter=*/2);
    }
    L.ctx.f = f;
    return rc;
  });
}

// Host launch overhead (~n launches per call) would starve the GPU: the pass
// sequence is captured once into a CUDA graph (keyed by every launch parameter:
// variant, mode, buffers, n and the whole Ctx -- error counter, queue pointers
// and geometry, watchdog/stress settings, fault descriptor) and replayed on the
// caller's stream.  The cache is a bounded LRU (evicted graphs are destroyed)
// guarded by a mutex.  Inside a caller's capture the launches are simply
// recorded into the caller's graph.
constexpr size_t FW_GRAPH_CACHE = 16;
std::mutex g_fw_mu;
std::list<std::pair<std::string, cudaGraphExec_t>> g_fw_graphs;  // front = most recently used
cudaStream_t g_fw_capture_stream = nullptr;

std::string fw_key(const Launch& L) {
  std::string k;
  auto put = [&k](const void* p, size_t n) { k.append((const char*)p, n); };
  put(&L.variant, sizeof L.variant);
  put(&L.mode, sizeof L.mode);
  put(&L.inflate, sizeof L.inflate);
  put(&L.bufs->buf[0].ptr, sizeof(void*));
  put(&L.bufs->buf[1].ptr, sizeof(void*));
  put(&L.n, sizeof L.n);
  const Ctx& c = L.ctx;
  put(&c.err, sizeof c.err);
  put(&c.ctrl, sizeof c.ctrl);
  put(&c.flags, sizeof c.flags);
  put(&c.payload, sizeof c.payload);
  put(&c.R, sizeof c.R);
  put(&c.W, sizeof c.W);
  put(&c.S, sizeof c.S);
  put(&c.wd, sizeof c.wd);
  put(&c.stress, sizeof c.stress);
  put(&c.skew_ns, sizeof c.skew_ns);
  put(&c.f.replica, sizeof c.f.replica);
  put(&c.f.site, sizeof c.f.site);
  put(&c.f.bit, sizeof c.f.bit);
  put(&c.f.sid, sizeof c.f.sid);
  put(&c.f.elem, sizeof c.f.elem);
  return k;
}

}  // namespace

int floydwarshall_run(Launch& L) {
  const unsigned n = (unsigned)L.n;
  if (n == 0) return RMT_OK;
  cudaStreamCaptureStatus cs = cudaStreamCaptureStatusNone;
  if (cudaStreamIsCapturing(L.stream, &cs) != cudaSuccess) {
    cudaGetLastError();
    cs = cudaStreamCaptureStatusNone;
  }
  if (cs != cudaStreamCaptureStatusNone || n < 64 ||
      (L.variant == RMT_INTER_GROUP && !L.inflate && L.mode != M_NOCOMM))  // inter: 2 launches, no graph
    return fw_issue(L);
  const std::string key = fw_key(L);
  std::lock_guard<std::mutex> lock(g_fw_mu);
  auto it = g_fw_graphs.begin();
  while (it != g_fw_graphs.end() && it->first != key) ++it;
  if (it != g_fw_graphs.end()) {
    g_fw_graphs.splice(g_fw_graphs.begin(), g_fw_graphs, it);  // most recently used
  } else {
    int rc;
    if (!g_fw_capture_stream &&
        (rc = cuda_check(cudaStreamCreateWithFlags(&g_fw_capture_stream, cudaStreamNonBlocking), "fw: stream")))
      return rc;
    Launch C = L;
    C.stream = g_fw_capture_stream;
    C.launches = 0;
    if ((rc = cuda_check(cudaStreamBeginCapture(C.stream, cudaStreamCaptureModeThreadLocal), "fw: begin capture")))
      return rc;
    rc = fw_issue(C);
    cudaGraph_t g = nullptr;
    cudaError_t ec = cudaStreamEndCapture(C.stream, &g);
    if (rc) return rc;
    if ((rc = cuda_check(ec, "fw: end capture"))) return rc;
    cudaGraphExec_t ge = nullptr;
    rc = cuda_check(cudaGraphInstantiate(&ge, g, 0), "fw: instantiate");
    cudaGraphDestroy(g);
    if (rc) return rc;
    g_fw_graphs.emplace_front(key, ge);
    while (g_fw_graphs.size() > FW_GRAPH_CACHE) {  // evict the least recently used graph
      cudaGraphExecDestroy(g_fw_graphs.back().second);
      g_fw_graphs.pop_back();
    }
  }
  L.launches += (int)n + 1;
  return cuda_check(cudaGraphLaunch(g_fw_graphs.front().second, L.stream), "fw: graph launch");
}

}  // namespace rmt
