// rmt_abi.cu -- the extern "C" boundary declared in include/rmt.h.
// Validation, workspace layout, fault/ablation state, dispatch to the
// per-kernel launchers, and the host-buffer end-to-end call.
#include <cuda_runtime.h>
#include <stdio.h>

#include <string>

#include "rmt_host.cuh"

namespace rmt {

namespace {
thread_local std::string g_err;
FaultDesc g_fault = {0, 0, 0, 0, 0};
bool g_armed = false;
int g_ablation = RMT_ABL_FULL;
struct StressCfg {
  int depth;                 // queue slots in use (0: default)
  int flags;                 // STRESS_* bits
  unsigned skew_ns;
  unsigned long long wd;     // watchdog cycles (0: WATCHDOG_CYCLES)
} g_stress = {0, 0, 0, 0};
thread_local int g_last_launches = 0;

struct KEntry {
  const char* name;
  int (*validate)(const rmt_bufs_t*, int64_t);
  size_t (*scratch)(int64_t, const int64_t*);
  int (*inter_warps)(int64_t, const int64_t*);
  int (*run)(Launch&);
  int nin, in[2], nout, out[2];  // buffer roles for rmt_run_host
};

#define KE(name, nin, i0, i1, nout, o0, o1) \
  {#name, name##_validate, name##_scratch, name##_inter_warps, name##_run, nin, {i0, i1}, nout, {o0, o1}}

const KEntry kTable[RMT_K_COUNT] = {
    KE(blackscholes, 1, 0, 0, 2, 1, 2),
    KE(binarysearch, 2, 0, 1, 1, 2, 0),
    KE(fwt, 1, 0, 0, 1, 1, 0),
    KE(prefixsum, 1, 0, 0, 1, 1, 0),
    KE(reduction, 1, 0, 0, 1, 1, 0),
    KE(transpose, 1, 0, 0, 1, 1, 0),
    KE(sobel, 1, 0, 0, 1, 1, 0),
    KE(floydwarshall, 1, 0, 0, 2, 0, 1),
    KE(dct, 1, 0, 0, 1, 1, 0),
    KE(matmul, 2, 0, 1, 1, 2, 0),
    KE(dwthaar1d, 1, 0, 0, 1, 1, 0),
    KE(bitonicsort, 1, 0, 0, 1, 1, 0),
    KE(binomialoption, 1, 0, 0, 1, 1, 0),
};

const char* kVariantNames[7] = {"none",        "intra_smem",  "intra_reg", "inter_group",
                                "inter_cluster", "intra_nolds", "dup_kernel"};

int check_device() {
  static int ok_dev = -1;
  int dev = 0;
  if (cudaGetDevice(&dev) != cudaSuccess) {
    set_error("cudaGetDevice failed (no CUDA device?)");
    return RMT_ENODEV;
  }
  if (ok_dev == dev) return RMT_OK;
  int major = 0;
  cudaDeviceGetAttribute(&major, cudaDevAttrComputeCapabilityMajor, dev);
  if (major != 10) {
    set_error("librmt is built for sm_100a only; device major=" + std::to_string(major));
    return RMT_ENODEV;
  }
  ok_dev = dev;
  return RMT_OK;
}

size_t dtype_bytes(int dt) { return dt == RMT_U64 ? 8 : dt == RMT_BF16 ? 2 : 4; }

// 32-bit words of output buffer `which` (in kTable order) as a function of n:
// every schema's outputs hold n elements, except FloydWarshall (n*n) and
// Reduction (one u64).
size_t out_words(int kernel, int64_t n) {
  if (kernel == RMT_K_FLOYDWARSHALL) return (size_t)n * (size_t)n;
  if (kernel == RMT_K_REDUCTION) return 2;
  return (size_t)n;
}

// dup_kernel workspace: [scratch A][scratch B] then, per output buffer, the
// two replicas' shadows.
size_t dup_bytes(int kernel, int64_t n, const int64_t* dims, size_t* scr) {
  const KEntry& e = kTable[kernel];
  const size_t s = align_up(e.scratch(n, dims), 256);
  if (scr) *scr = s;
  return 2 * s + (size_t)e.nout * 2 * align_up(out_words(kernel, n) * 4, 256);
}

size_t ws_size(int kernel, int variant, int64_t n, const int64_t* dims, size_t* inter_part) {
  const KEntry& e = kTable[kernel];
  size_t ip = 0;
  if (variant == RMT_DUP_KERNEL) {
    if (inter_part) *inter_part = 0;
    return dup_bytes(kernel, n, dims, nullptr);
  }
  if (variant == RMT_INTER_GROUP) ip = align_up(inter_bytes(e.inter_warps(n, dims)), 256);
  if (inter_part) *inter_part = ip;
  return ip + align_up(e.scratch(n, dims), 256);
}

// Kernel-level duplication: two runs of the unprotected kernel into
// shadows, then the on-device compare-and-commit.
int run_dup(Launch& L0, const KEntry& e, char* ws, bool armed, const FaultDesc& f) {
  const rmt_bufs_t* bufs = L0.bufs;
  size_t scr = 0;
  dup_bytes(L0.kernel, L0.n, bufs->dims, &scr);
  const size_t ow = out_words(L0.kernel, L0.n);
  const size_t sh = align_up(ow * 4, 256);
  char* shadows = ws + 2 * scr;
  rmt_bufs_t rb[2] = {*bufs, *bufs};
  for (int r = 0; r < 2; ++r) {
    for (int i = 0; i < e.nout; ++i) {
      void* p = shadows + ((size_t)i * 2 + r) * sh;
      const int bi = e.out[i];
      bool inout = false;
      for (int k = 0; k < e.nin; ++k) inout = inout || e.in[k] == bi;
      // an in/out buffer: the replica starts from its own copy of the input;
      // otherwise the shadows are poisoned differently (0xA5.. / 0x5A..) so that
      // a word one replica failed to write (e.g. a flipped store address) differs
      // from the other replica's value unless that value is the poison itself
      int rc = inout ? cuda_check(cudaMemcpyAsync(p, bufs->buf[bi].ptr, ow * 4, cudaMemcpyDeviceToDevice, L0.stream),
                                  "dup: copy in/out input")
                     : cuda_check(cudaMemsetAsync(p, r ? 0x5A : 0xA5, ow * 4, L0.stream), "dup: poison shadow");
      if (rc) return rc;
      rb[r].buf[bi].ptr = p;
    }
  }
  for (int r = 0; r < 2; ++r) {
    Launch L = L0;
    L.variant = RMT_NONE;
    L.bufs = &rb[r];
    L.scratch = ws + (size_t)r * scr;
    L.scratch_bytes = scr;
    L.launches = 0;
    const bool hit = armed && f.replica == r;
    L.mode = hit ? M_FAULT : M_NORMAL;
    L.ctx.f = f;
    L.ctx.f.replica = 0;  // the unprotected kernel is replica 0 of itself
    int rc = e.run(L);
    L0.launches += L.launches;
    if (rc) return rc;
  }
  for (int i = 0; i < e.nout; ++i) {
    const int bi = e.out[i];
    int rc = dup_compare_launch(rb[0].buf[bi].ptr, rb[1].buf[bi].ptr, bufs->buf[bi].ptr, ow, L0.ctx.err, L0.stream);
    if (rc) return rc;
    L0.launches += 1;
  }
  return RMT_OK;
}
}  // namespace

void set_error(const std::string& msg) { g_err = msg; }

#ifdef RMT_TRACE
// experiment builds: a device buffer of 2^17 x 8 u64 milestones (Rep RMT_TR)
unsigned long long* trace_buf() {
  static unsigned long long* p = nullptr;
  if (!p && cudaMalloc(&p, (size_t)(1u << 17) * 8 * 8) == cudaSuccess) cudaMemset(p, 0, (size_t)(1u << 17) * 64);
  return p;
}
#endif

int cuda_check(cudaError_t e, const char* what) {
  if (e == cudaSuccess) return RMT_OK;
  set_error(std::string(what) + ": " + cudaGetErrorString(e));
  return RMT_ECUDA;
}

}  // namespace rmt

using namespace rmt;

extern "C" {

int rmt_launch(int kernel, int variant, const rmt_bufs_t* bufs, int64_t n, unsigned long long* err_count,
               void* workspace, size_t ws_bytes, void* stream) {
  g_last_launches = 0;
  if (kernel < 0 || kernel >= RMT_K_COUNT) { set_error("bad kernel id"); return RMT_EINVAL; }
  if (variant < 0 || variant > RMT_DUP_KERNEL) { set_error("bad variant id"); return RMT_EINVAL; }
  if (!bufs || !err_count) { set_error("bufs and err_count must be non-NULL"); return RMT_EINVAL; }
  int rc = check_device();
  if (rc) return rc;
  const KEntry& e = kTable[kernel];
  rc = e.validate(bufs, n);
  if (rc) return rc;
  size_t inter_part = 0;
  size_t need = ws_size(kernel, variant, n, bufs->dims, &inter_part);
  if (need > 0 && (workspace == nullptr || ws_bytes < need)) {
    set_error("workspace too small: need " + std::to_string(need) + " bytes");
    return RMT_EWORKSPACE;
  }
  if (variant == RMT_DUP_KERNEL) {
    if (g_ablation != RMT_ABL_FULL && !g_armed) {
      set_error("dup_kernel has no ablation modes");
      return RMT_EUNSUPPORTED;
    }
    Launch L{};
    L.kernel = kernel;
    L.variant = variant;
    L.bufs = bufs;
    L.n = n;
    L.stream = (cudaStream_t)stream;
    L.ctx.err = err_count;
    L.ctx.wd = WATCHDOG_CYCLES;
    rc = run_dup(L, e, (char*)workspace, g_armed, g_fault);
    g_last_launches = L.launches;
    if (rc == RMT_OK) rc = cuda_check(cudaGetLastError(), "kernel launch");
    return rc;
  }
  if (g_armed && variant == RMT_NONE && g_fault.replica != 0) {
    set_error("variant none has a single replica: fault replica must be 0");
    return RMT_EINVAL;
  }
  Launch L{};
  L.kernel = kernel;
  L.variant = variant;
  const bool queue_variant = variant == RMT_INTER_GROUP || variant == RMT_INTER_CLUSTER;
  const bool stress = queue_variant && (g_stress.depth > 0 || g_stress.flags != 0);
  L.mode = g_armed ? M_FAULT
         : (g_ablation == RMT_ABL_NOCOMM && variant != RMT_NONE) ? M_NOCOMM
         : stress ? M_STRESS
                  : M_NORMAL;
  L.inflate = !g_armed && g_ablation == RMT_ABL_INFLATE && variant != RMT_NONE;
  L.bufs = bufs;
  L.n = n;
  L.stream = (cudaStream_t)stream;
  L.ctx.err = err_count;
  L.ctx.f = g_fault;
  L.ctx.wd = g_stress.wd ? g_stress.wd : WATCHDOG_CYCLES;
  L.ctx.stress = g_stress.flags;
  L.ctx.skew_ns = g_stress.skew_ns;
#ifdef RMT_TRACE
  L.ctx.trace = trace_buf();
#endif
  L.cl_depth = (variant == RMT_INTER_CLUSTER) ? g_stress.depth : 0;
  char* ws = (char*)workspace;
  if (variant == RMT_INTER_GROUP) {
    int W = e.inter_warps(n, bufs->dims);
    size_t slots = (size_t)INTER_R * W * INTER_S;
    L.ctx.ctrl = (unsigned*)ws;
    L.ctx.flags = (unsigned*)(ws + CTRL_BYTES);
    L.ctx.payload = (unsigned*)(ws + CTRL_BYTES + slots * 4);
    L.ctx.R = INTER_R;
    L.ctx.W = W;
    L.ctx.S = g_stress.depth > 0 ? g_stress.depth : INTER_S;
  }
  L.scratch = ws ? ws + inter_part : nullptr;
  L.scratch_bytes = need - inter_part;
  rc = e.run(L);
  g_last_launches = L.launches;
  if (rc == RMT_OK) rc = cuda_check(cudaGetLastError(), "kernel launch");
  return rc;
}

size_t rmt_workspace_size(int kernel, int variant, int64_t n, const int64_t* dims) {
  if (kernel < 0 || kernel >= RMT_K_COUNT || variant < 0 || variant > RMT_DUP_KERNEL) return 0;
  int64_t zero[4] = {0, 0, 0, 0};
  return ws_size(kernel, variant, n, dims ? dims : zero, nullptr);
}

int rmt_run_host(int kernel, int variant, const rmt_bufs_t* host, const rmt_bufs_t* dev, int64_t n,
                 unsigned long long* err_host, unsigned long long* err_dev, void* workspace, size_t ws_bytes,
                 void* stream, int64_t* h2d_bytes, int64_t* d2h_bytes) {
  if (kernel < 0 || kernel >= RMT_K_COUNT || !host || !dev || !err_host || !err_dev) {
    set_error("rmt_run_host: bad arguments");
    return RMT_EINVAL;
  }
  const KEntry& e = kTable[kernel];
  cudaStream_t s = (cudaStream_t)stream;
  int64_t hb = 0, db = 0;
  int rc;
  for (int i = 0; i < e.nin; ++i) {
    const rmt_buf_t& h = host->buf[e.in[i]];
    const rmt_buf_t& d = dev->buf[e.in[i]];
    if (!h.ptr || h.numel != d.numel || h.dtype != d.dtype) { set_error("host/dev schema mismatch"); return RMT_EINVAL; }
    size_t bytes = (size_t)h.numel * dtype_bytes(h.dtype);
    if ((rc = cuda_check(cudaMemcpyAsync(d.ptr, h.ptr, bytes, cudaMemcpyHostToDevice, s), "H2D"))) return rc;
    hb += (int64_t)bytes;
  }
  if ((rc = cuda_check(cudaMemsetAsync(err_dev, 0, sizeof(unsigned long long), s), "memset err"))) return rc;
  rc = rmt_launch(kernel, variant, dev, n, err_dev, workspace, ws_bytes, stream);
  if (rc) return rc;
  for (int i = 0; i < e.nout; ++i) {
    const rmt_buf_t& h = host->buf[e.out[i]];
    const rmt_buf_t& d = dev->buf[e.out[i]];
    if (!h.ptr || h.numel != d.numel) { set_error("host/dev schema mismatch"); return RMT_EINVAL; }
    size_t bytes = (size_t)h.numel * dtype_bytes(h.dtype);
    if ((rc = cuda_check(cudaMemcpyAsync(h.ptr, d.ptr, bytes, cudaMemcpyDeviceToHost, s), "D2H"))) return rc;
    db += (int64_t)bytes;
  }
  if ((rc = cuda_check(cudaMemcpyAsync(err_host, err_dev, 8, cudaMemcpyDeviceToHost, s), "D2H err"))) return rc;
  db += 8;
  if ((rc = cuda_check(cudaStreamSynchronize(s), "stream sync"))) return rc;
  if (h2d_bytes) *h2d_bytes = hb;
  if (d2h_bytes) *d2h_bytes = db;
  return RMT_OK;
}

int rmt_run_host_variants(int kernel, int nvar, const int* variants, const rmt_bufs_t* host, const rmt_bufs_t* dev,
                          int64_t n, unsigned long long* err_host, unsigned long long* err_dev,
                          void* const* workspaces, const size_t* ws_bytes, void* stream, int64_t* h2d_bytes,
                          int64_t* d2h_bytes) {
  if (kernel < 0 || kernel >= RMT_K_COUNT || nvar < 1 || !variants || !host || !dev || !err_host || !err_dev ||
      !workspaces || !ws_bytes) {
    set_error("rmt_run_host_variants: bad arguments");
    return RMT_EINVAL;
  }
  const KEntry& e = kTable[kernel];
  cudaStream_t s = (cudaStream_t)stream;
  int64_t hb = 0, db = 0;
  int rc;
  auto is_out = [&](int bi) {
    for (int k = 0; k < e.nout; ++k)
      if (e.out[k] == bi) return true;
    return false;
  };
  for (int v = 0; v < nvar; ++v) {
    // inputs: once; an in/out buffer (FloydWarshall's D) again before every variant
    for (int i = 0; i < e.nin; ++i) {
      const int bi = e.in[i];
      if (v > 0 && !is_out(bi)) continue;
      const rmt_buf_t& h = host->buf[bi];
      const rmt_buf_t& d = dev->buf[bi];
      if (!h.ptr || h.numel != d.numel || h.dtype != d.dtype) { set_error("host/dev schema mismatch"); return RMT_EINVAL; }
      size_t bytes = (size_t)h.numel * dtype_bytes(h.dtype);
      if ((rc = cuda_check(cudaMemcpyAsync(d.ptr, h.ptr, bytes, cudaMemcpyHostToDevice, s), "H2D"))) return rc;
      hb += (int64_t)bytes;
    }
    if ((rc = cuda_check(cudaMemsetAsync(err_dev + v, 0, sizeof(unsigned long long), s), "memset err"))) return rc;
    rc = rmt_launch(kernel, variants[v], dev, n, err_dev + v, workspaces[v], ws_bytes[v], stream);
    if (rc) return rc;
  }
  // the committed outputs (every variant writes the same bits) and every error count
  for (int i = 0; i < e.nout; ++i) {
    const rmt_buf_t& h = host->buf[e.out[i]];
    const rmt_buf_t& d = dev->buf[e.out[i]];
    if (!h.ptr || h.numel != d.numel) { set_error("host/dev schema mismatch"); return RMT_EINVAL; }
    size_t bytes = (size_t)h.numel * dtype_bytes(h.dtype);
    if ((rc = cuda_check(cudaMemcpyAsync(h.ptr, d.ptr, bytes, cudaMemcpyDeviceToHost, s), "D2H"))) return rc;
    db += (int64_t)bytes;
  }
  if ((rc = cuda_check(cudaMemcpyAsync(err_host, err_dev, 8 * (size_t)nvar, cudaMemcpyDeviceToHost, s), "D2H err")))
    return rc;
  db += 8 * nvar;
  if ((rc = cuda_check(cudaStreamSynchronize(s), "stream sync"))) return rc;
  if (h2d_bytes) *h2d_bytes = hb;
  if (d2h_bytes) *d2h_bytes = db;
  return RMT_OK;
}

int rmt_run_host_variants_pipelined(int kernel, int nvar, const int* variants, const rmt_bufs_t* host,
                                    const rmt_bufs_t* dev, int64_t n, unsigned long long* err_host,
                                    unsigned long long* err_dev, void* const* workspaces, const size_t* ws_bytes,
                                    void* stream_h2d, void* stream_compute, void* stream_d2h, int64_t* h2d_bytes,
                                    int64_t* d2h_bytes) {
  if (kernel < 0 || kernel >= RMT_K_COUNT || nvar < 1 || !variants || !host || !dev || !err_host || !err_dev ||
      !workspaces || !ws_bytes) {
    set_error("rmt_run_host_variants_pipelined: bad arguments");
    return RMT_EINVAL;
  }
  const KEntry& e = kTable[kernel];
  cudaStream_t s1 = (cudaStream_t)stream_h2d, sc = (cudaStream_t)stream_compute, s3 = (cudaStream_t)stream_d2h;
  int64_t hb = 0, db = 0;
  int rc;
  auto is_out = [&](int bi) {
    for (int k = 0; k < e.nout; ++k)
      if (e.out[k] == bi) return true;
    return false;
  };
  struct Events {  // destroyed on every return (released once the recorded work completes)
    cudaEvent_t in = nullptr, done = nullptr;
    ~Events() {
      if (in) cudaEventDestroy(in);
      if (done) cudaEventDestroy(done);
    }
  } ev;
  if ((rc = cuda_check(cudaEventCreateWithFlags(&ev.in, cudaEventDisableTiming), "event"))) return rc;
  if ((rc = cuda_check(cudaEventCreateWithFlags(&ev.done, cudaEventDisableTiming), "event"))) return rc;
  cudaEvent_t ev_in = ev.in, ev_done = ev.done;
  // inputs on the H2D stream (they overlap the previous call's compute and D2H)
  for (int i = 0; i < e.nin; ++i) {
    const int bi = e.in[i];
    const rmt_buf_t& h = host->buf[bi];
    const rmt_buf_t& d = dev->buf[bi];
    if (!h.ptr || h.numel != d.numel || h.dtype != d.dtype) { set_error("host/dev schema mismatch"); return RMT_EINVAL; }
    size_t bytes = (size_t)h.numel * dtype_bytes(h.dtype);
    if ((rc = cuda_check(cudaMemcpyAsync(d.ptr, h.ptr, bytes, cudaMemcpyHostToDevice, s1), "H2D"))) return rc;
    hb += (int64_t)bytes;
  }
  cudaEventRecord(ev_in, s1);
  cudaStreamWaitEvent(sc, ev_in, 0);
  for (int v = 0; v < nvar; ++v) {
    // an in/out buffer (FloydWarshall's D) again before every later variant, in compute order
    for (int i = 0; v > 0 && i < e.nin; ++i) {
      const int bi = e.in[i];
      if (!is_out(bi)) continue;
      const rmt_buf_t& h = host->buf[bi];
      const rmt_buf_t& d = dev->buf[bi];
      size_t bytes = (size_t)h.numel * dtype_bytes(h.dtype);
      if ((rc = cuda_check(cudaMemcpyAsync(d.ptr, h.ptr, bytes, cudaMemcpyHostToDevice, sc), "H2D"))) return rc;
      hb += (int64_t)bytes;
    }
    if ((rc = cuda_check(cudaMemsetAsync(err_dev + v, 0, sizeof(unsigned long long), sc), "memset err"))) return rc;
    rc = rmt_launch(kernel, variants[v], dev, n, err_dev + v, workspaces[v], ws_bytes[v], stream_compute);
    if (rc) return rc;
  }
  cudaEventRecord(ev_done, sc);
  cudaStreamWaitEvent(s3, ev_done, 0);
  for (int i = 0; i < e.nout; ++i) {
    const rmt_buf_t& h = host->buf[e.out[i]];
    const rmt_buf_t& d = dev->buf[e.out[i]];
    if (!h.ptr || h.numel != d.numel) { set_error("host/dev schema mismatch"); return RMT_EINVAL; }
    size_t bytes = (size_t)h.numel * dtype_bytes(h.dtype);
    if ((rc = cuda_check(cudaMemcpyAsync(h.ptr, d.ptr, bytes, cudaMemcpyDeviceToHost, s3), "D2H"))) return rc;
    db += (int64_t)bytes;
  }
  if ((rc = cuda_check(cudaMemcpyAsync(err_host, err_dev, 8 * (size_t)nvar, cudaMemcpyDeviceToHost, s3), "D2H err")))
    return rc;
  db += 8 * nvar;
  if (h2d_bytes) *h2d_bytes = hb;
  if (d2h_bytes) *d2h_bytes = db;
  return cuda_check(cudaGetLastError(), "pipelined launch");
}

int rmt_inject_fault(int replica, int site, int bit, int64_t elem) {
  if (replica < 0 || replica > 1 || site < RMT_SITE_LOAD || site > RMT_SITE_STORE_ADDR || bit < 0 || bit > 31 ||
      elem < 0) {
    set_error("rmt_inject_fault: bad arguments");
    return RMT_EINVAL;
  }
  g_fault.replica = replica;
  g_fault.site = site;
  g_fault.bit = bit;
  g_fault.sid = 0;
  g_fault.elem = elem;
  g_armed = true;
  return RMT_OK;
}

int rmt_clear_faults(void) {
  g_armed = false;
  g_fault = FaultDesc{0, 0, 0, 0, 0};
  return RMT_OK;
}

int rmt_set_ablation(int mode) {
  if (mode < RMT_ABL_FULL || mode > RMT_ABL_INFLATE) { set_error("bad ablation mode"); return RMT_EINVAL; }
  g_ablation = mode;
  return RMT_OK;
}

int rmt_last_launch_count(void) { return g_last_launches; }

#ifdef RMT_TRACE
int rmt_trace_copy(void* host, size_t bytes) {  // experiment builds only
  cudaDeviceSynchronize();
  return cuda_check(cudaMemcpy(host, trace_buf(), bytes, cudaMemcpyDeviceToHost), "trace copy");
}
#endif

int rmt_set_stress(int depth, int flags, int skew_ns, long long watchdog_cycles) {
  if (depth < 0 || depth > INTER_S || (depth & (depth - 1)) != 0 || flags < 0 ||
      flags > (STRESS_TAGS | STRESS_SKEW | STRESS_DROP) || skew_ns < 0 || watchdog_cycles < 0) {
    set_error("rmt_set_stress: depth in {0,1,2,4,8}, flags in 0..7, skew_ns >= 0, watchdog_cycles >= 0");
    return RMT_EINVAL;
  }
  g_stress.depth = depth;
  g_stress.flags = flags;
  g_stress.skew_ns = (unsigned)skew_ns;
  g_stress.wd = (unsigned long long)watchdog_cycles;
  return RMT_OK;
}

int rmt_workspace_status(int variant, void* workspace, void* stream) {
  if (variant != RMT_INTER_GROUP || workspace == nullptr) return RMT_OK;  // only the L2 queue has sticky state
  cudaStream_t s = (cudaStream_t)stream;
  unsigned flag = 0;
  unsigned* ctrl = (unsigned*)workspace;
  int rc = cuda_check(cudaMemcpyAsync(&flag, ctrl + CTRL_WATCHDOG, 4, cudaMemcpyDeviceToHost, s), "status: read");
  if (!rc) rc = cuda_check(cudaStreamSynchronize(s), "status: sync");
  if (rc) return rc;
  if (flag == 0u) return RMT_OK;
  // the last CTA of the aborted launch already cleared the slot flags; clear the
  // sticky flag so the workspace is reusable
  rc = cuda_check(cudaMemsetAsync(ctrl + CTRL_WATCHDOG, 0, 4, s), "status: clear");
  if (!rc) rc = cuda_check(cudaStreamSynchronize(s), "status: sync");
  if (rc) return rc;
  set_error("inter_group watchdog fired: a replica waited longer than the watchdog bound for its partner "
            "(each timeout was counted in *err_count, the affected stores were not committed); the queue was reset");
  return RMT_EWATCHDOG;
}

const char* rmt_strerror(int code) {
  switch (code) {
    case RMT_OK: return "ok";
    case RMT_EINVAL: return "invalid argument";
    case RMT_EUNSUPPORTED: return "unsupported kernel/variant";
    case RMT_EWORKSPACE: return "workspace too small";
    case RMT_ECUDA: return "CUDA error";
    case RMT_ENODEV: return "no sm_100 device";
    case RMT_EWATCHDOG: return "inter-group watchdog fired (a replica pair timed out)";
  }
  return "unknown error";
}

const char* rmt_last_error(void) { return g_err.c_str(); }

const char* rmt_kernel_name(int kernel) {
  return (kernel >= 0 && kernel < RMT_K_COUNT) ? kTable[kernel].name : "?";
}

const char* rmt_variant_name(int variant) {
  return (variant >= 0 && variant <= RMT_DUP_KERNEL) ? kVariantNames[variant] : "?";
}

}  // extern "C"
