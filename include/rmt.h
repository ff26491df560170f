/*
 * rmt.h -- C ABI of librmt.so: compiler-style software Redundant
 * MultiThreading (RMT) for GPGPU kernels on B200 (sm_100a).
 *
 * Method: Wadden et al., "Real-World Design and Evaluation of Compiler-Managed
 * GPU Redundant Multithreading", ISCA 2014.  "P:NNN" = line NNN of the paper
 * text (/root/reference/PAPER.md, not shipped).
 *
 *   - Each work-item is replicated; replicas run on replicated input
 *     ("input replication", "producer and consumer").
 *   - Every value that leaves the sphere of replication (SoR) -- a global store
 *     -- is sent by the producer to the consumer, which compares the store's
 *     address and value with its private copy and executes the store only if
 *     they agree ("communicate both the address and value operands
 *     of the store ... If the values differ, we have detected an error").
 *   - Detection only; recovery is orthogonal.  A mismatch suppresses the
 *     store and adds 1 to a device error counter (reading R-RMT1).
 *
 * Variants (rmt_variant_t):
 *   RMT_NONE        the unprotected kernel (the baseline every slowdown is
 *                   normalised to, "normalized to the runtime of the
 *                   original kernel").
 *   RMT_INTRA_SMEM  Intra-Group RMT +LDS: each CTA
 *                   has twice the threads; redundant pairs are lanes (2i, 2i+1)
 *                   of one warp (low bit of the thread id = replica);
 *                   kernel-written shared memory is duplicated per replica; the
 *                   producer (odd lane) passes (address, value) through a
 *                   shared-memory mailbox, the consumer (even lane, Fig. 8
 *                   P:845) compares and stores.
 *   RMT_INTRA_REG   as INTRA_SMEM, but the exchange is register-level
 *                   __shfl_xor_sync(.., 1) -- the B200 form of the paper's
 *                   "FAST" swizzle communication (Fig. 8).
 *   RMT_INTER_GROUP Inter-Group RMT: twice the CTAs; each CTA takes
 *                   a ticket from a global counter, pair = ticket>>1,
 *                   even ticket = producer; the producer passes store records
 *                   through a bounded global-memory queue with release/acquire
 *                   flags ("two-tiered locking system"; L2-coherent
 *                   reads); the consumer compares and stores.
 *   RMT_INTER_CLUSTER Inter-Group RMT, Blackwell-native:
 *                   the pair is a 2-CTA thread-block cluster (hardware
 *                   co-scheduling replaces the ticket); the producer CTA writes
 *                   its store records into the consumer CTA's shared memory
 *                   through distributed shared memory (DSMEM) with cluster-scope
 *                   release/acquire flags, instead of an L2/HBM queue.
 *   RMT_INTRA_NOLDS Intra-Group RMT -LDS:
 *                   pairs as in INTRA_REG, but the kernel's shared memory is NOT
 *                   duplicated: both replicas read one copy, and every kernel
 *                   shared-memory store is exchanged (registers), compared and
 *                   performed once by the consumer.  Shared memory is outside
 *                   this variant's sphere of replication (a fault in the copy
 *                   is read by both replicas and is not detected).
 *   RMT_DUP_KERNEL  naive kernel-level duplication (SURVEY 8(f) rank
 *                   4): the unprotected kernel runs twice, each replica into its
 *                   own shadow outputs (and scratch) in the workspace, then one
 *                   compare kernel commits every aligned 4-word output group the
 *                   two agree on and counts the others in *err_count (the paper
 *                   compares on the host and re-executes; here the comparison
 *                   stays on the device and the library only detects).
 *
 * Thread-safety: launches on different streams must use different workspaces.
 * The fault-injection and ablation state is process-global (test/bench use).
 */
#ifndef RMT_H
#define RMT_H

#include <stddef.h>
#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

typedef enum {
    RMT_NONE = 0,
    RMT_INTRA_SMEM = 1,
    RMT_INTRA_REG = 2,
    RMT_INTER_GROUP = 3,
    RMT_INTER_CLUSTER = 4,
    RMT_INTRA_NOLDS = 5,
    RMT_DUP_KERNEL = 6
} rmt_variant_t;

/* The AMD APP SDK-style kernels the paper evaluates (Fig. 2 axis
 * P:237-255) plus MatrixTranspose (BASELINE.json configs[1]); ids >= 10 are
 * the paper's communication-stress kernels. */
typedef enum {
    RMT_K_BLACKSCHOLES = 0,
    RMT_K_BINARYSEARCH = 1,
    RMT_K_FWT = 2,
    RMT_K_PREFIXSUM = 3,
    RMT_K_REDUCTION = 4,
    RMT_K_TRANSPOSE = 5,
    RMT_K_SOBEL = 6,
    RMT_K_FLOYDWARSHALL = 7,
    RMT_K_DCT = 8,
    RMT_K_MATMUL = 9,
    RMT_K_DWTHAAR1D = 10,
    RMT_K_BITONICSORT = 11,
    RMT_K_BINOMIALOPTION = 12,
    RMT_K_COUNT = 13
} rmt_kernel_t;

typedef enum { RMT_F32 = 0, RMT_U32 = 1, RMT_U64 = 2, RMT_U8X4 = 3, RMT_BF16 = 4 } rmt_dtype_t;

/* One caller-owned buffer.  ptr: device pointer for rmt_launch, host pointer
 * (ideally pinned) for the host side of rmt_run_host.  numel counts elements of
 * `dtype` (RMT_U8X4: one element = one 4-channel pixel = 4 bytes).  ptr must be
 * 16-byte aligned. */
typedef struct {
    void* ptr;
    int32_t dtype;
    int64_t numel;
} rmt_buf_t;

/* Buffer schema per kernel (n = logical units; dims as listed, others 0):
 *   BLACKSCHOLES  buf {r:F32[n], call:F32[n], put:F32[n]}           n = options, dims {mode}
 *                 mode 0: one draw r per option, (S,K,T,R,sigma) from r with S == K (DESIGN.md R-BS1)
 *                 mode 1: buf[0] = params:F32[5n], planes S | K | T | R | sigma, n%4 = 0 (R-BS4)
 *   BINARYSEARCH  buf {A:U32[N] sorted, q:U32[Q], idx:U32[Q]}       n = Q, dims {N, Q, mode}
 *                 idx[j] = lower_bound(A, q[j]) = #{i : A[i] < q[j]}; mode 0 = batched (every
 *                 query stores), mode 1 = ghost: the APP SDK single-key segment search, one
 *                 logical CTA per key and one writing work-item per key
 *   FWT           buf {x:F32[N], y:F32[N]}                          n = N = 2^m, dims {0}
 *                 dims {1, upper}: one cross-shard butterfly stage of a multi-GPU FWT,
 *                 buf {x: this shard, y: out, p: the partner shard} F32[N]; y = x + p (lower
 *                 rank of the pair) or p - x (upper) -- the single-GPU stage's fp32 operations
 *   PREFIXSUM     buf {x:U32[n], y:U32[n]}  inclusive, mod 2^32     n, dims {carry_in} (u32 added
 *                 to every y: the exclusive prefix of earlier shards in a multi-GPU scan; 0 = none);
 *                 optional buf[2] totals:U64[G] (every rank's total, all-gathered on the device)
 *                 with dims {carry_in, rank}: totals[0 .. rank) are added too (no host round trip);
 *                 dims[2] flags: bit 0 EXCLUSIVE (y_i = sum_{j<i} x_j), bit 1 FP32 (x, y F32; a
 *                 fixed association order identical in every variant: 16-element thread runs,
 *                 16-lane Kogge-Stone segments, sequential tiles, reduce-then-scan chunks;
 *                 SURVEY 8(c) PrefixSum readings (1)-(2); FP32 takes no carry_in / totals)
 *   REDUCTION     buf {x:U32[n], s:U64[1]}                          n
 *   TRANSPOSE     buf {A:U32|F32[H*W], B:same[W*H]}                 n = H*W, dims {H, W}, H%4 = W%4 = 0
 *   SOBEL         buf {I:U8X4[H*W], O:U8X4[H*W]}                    n = H*W, dims {H, W}, W%4 = 0
 *   FLOYDWARSHALL buf {D:U32[n*n] in/out, P:U32[n*n] out}           n = nodes, n%4 = 0
 *   DCT           buf {X:F32[H*W], Y:F32[H*W]}                      n = H*W, dims {H, W}, H%8 = W%8 = 0
 *   MATMUL        buf {A:BF16[M*K], Bt:BF16[N*K], C:F32[M*N]}       n = M*N, dims {M, N, K}
 *                 C = A * Bt^T (both operands K-major); M%128 = N%256 = 0, K%64 = 0
 *   DWTHAAR1D     buf {x:F32[N], y:F32[N]}                          n = N = 2^L <= 2^30
 *                 full orthonormal Haar decomposition: y[0] = a_L, y[N>>k + i] = level-k
 *                 detail i (DESIGN.md R-DWT1/2)
 *   BITONICSORT   buf {keys:U32[N], sorted:U32[N]}                  n = N = 2^n <= 2^30, ascending
 *                 (DESIGN.md R-BIT1)
 *   BINOMIALOPTION buf {r:F32[n], call:F32[n]}                      n = options <= 2^28
 *                 CRR European call, 254 steps, R = 0.02, sigma = 0.30, (S, K, T) from r
 *                 (DESIGN.md R-BO1/2)
 * Commit key: every storing commit compares the FULL
 * 32-bit element index and the store predicate of both replicas, key = idx ^
 * (mask << 28) for vector commits (idx for scalar ones); vector-committed
 * buffers must have < 2^30 elements (so that no storing key equals the
 * non-storing key 0xFFFFFFFF under a one-bit predicate fault).
 */
typedef struct {
    rmt_buf_t buf[6];
    int32_t nbuf;
    int64_t dims[4];
} rmt_bufs_t;

/* Return codes (0 = success).  A detected mismatch is NOT an error code: it is
 * counted in *err_count and the store is not committed. */
#define RMT_OK 0
#define RMT_EINVAL (-1)       /* bad kernel/variant id, dtype, numel, alignment or dims */
#define RMT_EUNSUPPORTED (-2) /* kernel x variant x mode combination not built */
#define RMT_EWORKSPACE (-3)   /* workspace NULL or smaller than rmt_workspace_size() */
#define RMT_ECUDA (-4)        /* CUDA launch/copy error; detail in rmt_last_error() */
#define RMT_ENODEV (-5)       /* no sm_100 device */
#define RMT_EWATCHDOG (-6)    /* rmt_workspace_status: an inter-group launch hit the watchdog */

/*
 * rmt_launch -- run kernel `kernel` under RMT variant `variant`, asynchronously
 * on `stream` (a cudaStream_t, passed as void*; NULL = legacy default stream).
 *   bufs       device buffers per the schema above (caller-owned, not freed).
 *   n          logical units (see schema).
 *   err_count  device pointer to one u64; the library ADDS the number of
 *              mismatching commits (caller zeroes it).  Never NULL.
 *   workspace  device scratch of >= rmt_workspace_size(...) bytes, ZERO-FILLED
 *              once at allocation; the library leaves it zero-equivalent after
 *              every successful launch (self-resetting inter-group tickets and
 *              queue; per-launch scratch is cleared with cudaMemsetAsync).
 *              May be NULL iff rmt_workspace_size() returned 0.
 * Graph-capturable (no host synchronisation, no allocation).
 * Returns RMT_OK or a negative code; never throws across the ABI.
 */
int rmt_launch(int kernel, int variant, const rmt_bufs_t* bufs, int64_t n,
               unsigned long long* err_count, void* workspace, size_t ws_bytes, void* stream);

/* Bytes of workspace rmt_launch needs for this kernel/variant/size (dims as in
 * the schema; may be NULL for 1-D kernels).  0 = none needed. */
size_t rmt_workspace_size(int kernel, int variant, int64_t n, const int64_t* dims);

/*
 * rmt_run_host -- the end-to-end call: copy the kernel's INPUT buffers from
 * `host` to `dev` (host->device), rmt_launch, copy the OUTPUT buffers back
 * (device->host) and the error count into *err_host, then synchronise
 * `stream`.  host/dev follow the same schema; dev buffers, err_dev and
 * workspace are caller-owned device memory.  Returns as rmt_launch, or
 * RMT_ECUDA on a copy/sync failure.  *h2d_bytes / *d2h_bytes (nullable)
 * receive the bytes copied.
 */
int rmt_run_host(int kernel, int variant, const rmt_bufs_t* host, const rmt_bufs_t* dev, int64_t n,
                 unsigned long long* err_host, unsigned long long* err_dev, void* workspace,
                 size_t ws_bytes, void* stream, int64_t* h2d_bytes, int64_t* d2h_bytes);

/*
 * rmt_run_host_variants -- the end-to-end call for one kernel under several
 * variants (e.g. the unprotected baseline and each RMT variant, as bench.py's
 * e2e leg runs them): copy the INPUT buffers host->device once (an in/out
 * buffer, FloydWarshall's D, again before every variant), launch variant
 * variants[v] with its own error counter err_dev[v] (device u64[nvar], zeroed
 * here) and workspace workspaces[v] (ws_bytes[v] bytes), copy the OUTPUT buffers
 * back once after the last launch (every variant commits the same bits) and the
 * nvar error counts into err_host[nvar], then synchronise `stream`.  Returns as
 * rmt_launch; *h2d_bytes / *d2h_bytes (nullable) receive the bytes copied.
 */
int rmt_run_host_variants(int kernel, int nvar, const int* variants, const rmt_bufs_t* host, const rmt_bufs_t* dev,
                          int64_t n, unsigned long long* err_host, unsigned long long* err_dev,
                          void* const* workspaces, const size_t* ws_bytes, void* stream, int64_t* h2d_bytes,
                          int64_t* d2h_bytes);

/*
 * rmt_run_host_variants_pipelined -- rmt_run_host_variants without the host
 * synchronisation, on three caller-owned streams so that consecutive calls
 * overlap: the INPUT copies go on stream_h2d, the launches (and FloydWarshall's
 * per-variant D re-copy) on stream_compute after the inputs landed, the OUTPUT
 * and error-count copies on stream_d2h after the last launch.  Keep every call's
 * launches on ONE compute stream (inter-group pairs assume their kernel is not
 * co-scheduled with another queue kernel).  err_host (u64[nvar]) and the host
 * output buffers must be pinned and are valid only after the caller
 * synchronises stream_d2h; host inputs must stay untouched until stream_h2d
 * completes.  Returns RMT_OK if everything was enqueued (errors of the
 * asynchronous work surface at the caller's synchronisation).
 */
int rmt_run_host_variants_pipelined(int kernel, int nvar, const int* variants, const rmt_bufs_t* host,
                                    const rmt_bufs_t* dev, int64_t n, unsigned long long* err_host,
                                    unsigned long long* err_dev, void* const* workspaces, const size_t* ws_bytes,
                                    void* stream_h2d, void* stream_compute, void* stream_d2h, int64_t* h2d_bytes,
                                    int64_t* d2h_bytes);

/* Fault injection (BASELINE.json north_star item (4)): arm ONE single-bit flip
 * for subsequent launches until rmt_clear_faults().
 *   replica  0|1 (intra: 0 = even lane = consumer, 1 = odd lane = producer;
 *            inter: 0 = even ticket = producer, 1 = odd ticket = consumer;
 *            none: must be 0)
 *   site     RMT_SITE_* below
 *   bit      0..31, flipped in the 32-bit word at that site
 *   elem     kernel-specific logical element; >= 0
 * Launches while armed run the FAULT instantiation of the kernel (the timed
 * path never contains fault code). */
#define RMT_SITE_LOAD 0       /* first loaded input word of elem */
#define RMT_SITE_COMPUTE 1    /* a kernel-specific intermediate of elem */
#define RMT_SITE_SMEM 2       /* a value read back from kernel-written shared memory */
#define RMT_SITE_STORE_VAL 3  /* the stored value (first output buffer) of elem */
#define RMT_SITE_STORE_ADDR 4 /* the store address: bit of the (vector) index */
int rmt_inject_fault(int replica, int site, int bit, int64_t elem);
int rmt_clear_faults(void);

/* Cost attribution "as the paper does": 0 = full RMT,
 * 1 = NOCOMM (both replicas run, no exchange/compare; the consumer stores its
 * own value), 2 = INFLATE (run RMT_NONE with its per-SM residency reduced to
 * that of the RMT variant by padding dynamic shared memory). */
#define RMT_ABL_FULL 0
#define RMT_ABL_NOCOMM 1
#define RMT_ABL_INFLATE 2
int rmt_set_ablation(int mode);

/*
 * rmt_workspace_status -- report (and clear) the inter-group queue's sticky
 * watchdog flag.  The queue waits are bounded: a replica that waits longer than
 * the watchdog bound for its partner (a fault that desynchronised the pair, or a
 * lost producer) gives up, adds 1 to *err_count, suppresses the affected stores
 * and sets a sticky flag in the workspace ("a watchdog-aborted
 * inter-group pair adds to err_count and sets a sticky flag that rmt_last_error
 * reports"); the launch's last CTA then clears every queue slot so the
 * workspace stays reusable.  This call reads the flag (synchronising `stream`):
 * RMT_OK if clear (or for any variant other than RMT_INTER_GROUP, whose queue
 * lives in the workspace); RMT_EWATCHDOG if it was set -- the flag is then
 * cleared and rmt_last_error() describes the event.
 */
int rmt_workspace_status(int variant, void* workspace, void* stream);

/*
 * rmt_set_stress -- queue-protocol stress configuration for the inter variants
 * (test use; SURVEY 8(c) "C-Q inter-group ring" pins).  While depth > 0 or
 * flags != 0, RMT_INTER_GROUP / RMT_INTER_CLUSTER launches run the STRESS
 * instantiation:
 *   depth           queue slots per (pair, warp) in use: 1, 2, 4 or 8 (0 = default 8;
 *                   inter_cluster: capped at its default mailbox depth)
 *   flags           1 TAGS: a (pair, warp, sequence) tag is folded into every record's
 *                   compared key, so a record consumed out of order, twice or from
 *                   another ring is counted in *err_count;
 *                   2 SKEW: random __nanosleep (0..skew_ns) at every CTA start and
 *                   before one commit in eight, per role;
 *                   4 DROP: the producer of pair 0 never publishes (a lost replica):
 *                   its consumer must time out through the watchdog
 *   skew_ns         maximum sleep for SKEW
 *   watchdog_cycles watchdog bound in SM clock cycles (0 = default 2^32) -- applies to
 *                   every launch, stress or not
 * All zero restores the timed configuration.  Process-global, like the fault state.
 */
int rmt_set_stress(int depth, int flags, int skew_ns, long long watchdog_cycles);

/* Kernel launches the last rmt_launch issued (for the bench's launch count). */
int rmt_last_launch_count(void);

/* Diagnostic: launch `pairs` 2-CTA clusters and
 * report in *same_sm_pairs how many had both CTAs on the same SM (read from
 * %smid).  0 means every inter_cluster pair spans two SMs, so the SM-private
 * structures (L1, LSU, schedulers) are inside that variant's sphere of
 * replication.  Synchronous; allocates and frees its own device buffer. */
int rmt_probe_cluster_placement(int64_t pairs, int64_t* same_sm_pairs);

/*
 * Peer device memory for the fused multi-GPU exchange (DESIGN.md
 * section 9): rmt_ipc_export writes the CUDA IPC handle (RMT_IPC_HANDLE_BYTES
 * bytes, caller-owned) of the allocation holding dev_ptr and dev_ptr's offset
 * in it; the partner rank passes both to rmt_ipc_open, which returns a device
 * pointer valid in the calling process (NVLink peer-to-peer access is enabled
 * lazily when the memory lives on another GPU; two processes on one GPU share
 * the memory).  That pointer may be passed as any rmt_launch input buffer: the
 * FWT cross-shard stage (dims {1, upper}) then reads the partner's shard
 * directly, with no staged copy.  rmt_ipc_close(ptr, offset) unmaps it.
 * Synchronous; not graph-capturable; RMT_ECUDA on failure.
 */
#define RMT_IPC_HANDLE_BYTES 64
int rmt_ipc_export(const void* dev_ptr, void* handle, int64_t* offset);
int rmt_ipc_open(const void* handle, int64_t offset, void** dev_ptr);
int rmt_ipc_close(void* dev_ptr, int64_t offset);

const char* rmt_strerror(int code);
const char* rmt_last_error(void); /* thread-local detail of the last failure */
const char* rmt_kernel_name(int kernel);
const char* rmt_variant_name(int variant);

#ifdef __cplusplus
}
#endif

#endif /* RMT_H */
