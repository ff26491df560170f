// rmt_device.cuh -- device-side RMT policies for sm_100a.
//
// One kernel body is written once and instantiated per variant V and mode MODE:
//   V    = V_NONE | V_INTRA_SMEM | V_INTRA_REG | V_INTER | V_CLUSTER | V_INTRA_NOLDS  (include/rmt.h)
//   MODE = M_NORMAL | M_FAULT (single-bit fault hooks compiled in) | M_NOCOMM
//          (ablation: replicas run, no exchange/compare)
//          | M_STRESS (inter variants only: queue-protocol stress test build --
//          per-CTA / per-commit random __nanosleep skew, (pair, warp, seq) tags
//          folded into every record key, an optional dropped producer; SURVEY
//          8(c) C-Q pins)
//
// What this header implements, with the paper passage each piece follows
// ("P:NNN" = line of /root/reference/PAPER.md):
//   * replica identity (P:205-207 intra: mask the low bit of the work-item id and
//     keep it as the producer/consumer flag; P:679-689 inter: a global counter
//     hands out new group ids, pair = id>>1, flag = id&1);
//   * duplicated kernel-written shared memory for the intra variants
//     (+LDS);
//   * the convergent predicated commit (the producer communicates
//     the address and value of every store leaving the SoR, the consumer
//     compares with its private copy and executes the store only if equal),
//     over three transports:
//       - INTRA_SMEM: per-warp shared-memory mailbox ("local memory
//         communication buffer");
//       - INTRA_REG : __shfl_xor_sync(.., 1) between lanes 2i/2i+1 (the B200
//         form of the GCN swizzle, Fig. 8: even lanes receive);
//       - INTER     : bounded per-(pair, warp) queue in global memory with
//         release/acquire flags (P:691 two-tier locking, P:693 L2-coherent reads),
//         region ownership handed over by a per-region turn counter;
//   * error counting: inter variants one atomicAdd per warp with mismatches
//     (warp ballot at every commit); intra variants a per-lane count added once
//     at finish().
//
// Determinism rule for bodies: everything that feeds a commit must be computed
// identically in every variant.
#pragma once
#include <cuda_runtime.h>
#include <stdint.h>

namespace rmt {

constexpr int V_NONE = 0, V_INTRA_SMEM = 1, V_INTRA_REG = 2, V_INTER = 3, V_CLUSTER = 4, V_INTRA_NOLDS = 5;
constexpr int M_NORMAL = 0, M_FAULT = 1, M_NOCOMM = 2, M_STRESS = 3;
constexpr int SITE_LOAD = 0, SITE_COMPUTE = 1, SITE_SMEM = 2, SITE_STORE_VAL = 3, SITE_STORE_ADDR = 4;
constexpr int MAXW = 4;               // max value words per commit
constexpr int RING_WORDS = 1 + MAXW;  // key + values per lane per record
constexpr int MBOX_WORDS = RING_WORDS * 16;  // intra_smem mailbox words per warp
constexpr unsigned FULL = 0xffffffffu;
constexpr int CTRL_TURN = 64;         // ctrl[64 ..) = per-region turn counters
constexpr unsigned long long WATCHDOG_CYCLES = 1ull << 32;  // default Ctx::wd: ~2 s at 2 GHz
// Ctx::stress bits (M_STRESS builds)
constexpr int STRESS_TAGS = 1, STRESS_SKEW = 2, STRESS_DROP = 4;
// ctrl[] words of the inter queue control block
constexpr int CTRL_TICKET = 0, CTRL_DONE = 1, CTRL_WATCHDOG = 2;
#ifndef RMT_INTER_SLOTS
#define RMT_INTER_SLOTS 8
#endif
constexpr int INTER_SLOTS_MAX = RMT_INTER_SLOTS;  // slots allocated per (region, warp); Ctx::S <= this
// inter_cluster: record slots per warp in the consumer CTA's shared memory
// (Ctx::S, a power of two chosen by the launcher): 8 lets the producer fill one
// deferred batch (<= 4 records) while the consumer drains the previous one; 4
// when a larger mailbox would cost occupancy (CTAs of more than 4 warps).
#ifndef RMT_CL_S_LARGE
#define RMT_CL_S_LARGE 8
#endif
constexpr int CL_S_SMALL = 4, CL_S_LARGE = RMT_CL_S_LARGE;

struct FaultDesc {
  int replica, site, bit, sid;
  long long elem;
};

// Passed by value to every kernel.
struct Ctx {
  unsigned long long* err;  // device u64 error counter (caller-owned)
  unsigned* ctrl;           // inter: [0] ticket [1] done [2] watchdog flag, [64..64+R) turn
  unsigned* flags;          // inter: R*W*S slot flags (0 free, 1 full)
  unsigned* payload;        // inter: R*W*S records of RING_WORDS*32 words
  int R, W, S;              // inter queue geometry (regions, warps per CTA, slots in use: 1..INTER_S)
  int nblocks;              // logical CTAs in this launch
  int pairs;                // inter/cluster: physical replica pairs launched (2 * pairs CTAs)
  int lstride;              // inter/cluster: logical-CTA stride of a pair (0: one logical CTA per pair)
  unsigned long long wd;    // watchdog bound in clock64 cycles (WATCHDOG_CYCLES unless a stress test lowers it)
  int stress;               // M_STRESS: STRESS_* bits
  unsigned skew_ns;         // M_STRESS: maximum random sleep (ns) per CTA start / per commit
  unsigned long long* trace;  // RMT_TRACE experiment builds only: per-CTA globaltimer milestones
  FaultDesc f;
};

// ---------------------------------------------------------------- PTX helpers
__device__ __forceinline__ unsigned ld_acquire(const unsigned* p) {
  unsigned v;
  asm volatile("ld.acquire.gpu.global.u32 %0, [%1];" : "=r"(v) : "l"(p) : "memory");
  return v;
}
__device__ __forceinline__ unsigned ld_relaxed(const unsigned* p) {
  unsigned v;
  asm volatile("ld.relaxed.gpu.global.u32 %0, [%1];" : "=r"(v) : "l"(p) : "memory");
  return v;
}
__device__ __forceinline__ void st_release(unsigned* p, unsigned v) {
  asm volatile("st.release.gpu.global.u32 [%0], %1;" ::"l"(p), "r"(v) : "memory");
}
__device__ __forceinline__ void st_relaxed(unsigned* p, unsigned v) {
  asm volatile("st.relaxed.gpu.global.u32 [%0], %1;" ::"l"(p), "r"(v) : "memory");
}
__device__ __forceinline__ unsigned long long ld_relaxed64(const unsigned long long* p) {
  unsigned long long v;
  asm volatile("ld.relaxed.gpu.global.u64 %0, [%1];" : "=l"(v) : "l"(p) : "memory");
  return v;
}
__device__ __forceinline__ void st_relaxed64(unsigned long long* p, unsigned long long v) {
  asm volatile("st.relaxed.gpu.global.u64 [%0], %1;" ::"l"(p), "l"(v) : "memory");
}
__device__ __forceinline__ void keep_alive(unsigned v) { asm volatile("" ::"r"(v)); }

// Streaming global loads/stores (16 B).
__device__ __forceinline__ uint4 ldg4(const void* p) { return __ldg(reinterpret_cast<const uint4*>(p)); }
__device__ __forceinline__ void stg4(void* p, uint4 v) { *reinterpret_cast<uint4*>(p) = v; }
__device__ __forceinline__ uint4 ldcs4(const void* p) { return __ldcs(reinterpret_cast<const uint4*>(p)); }
__device__ __forceinline__ void stcs4(void* p, uint4 v) { __stcs(reinterpret_cast<uint4*>(p), v); }
// 256-bit streaming load (sm_100 LDG.256, evict-first): lanes 32 B apart cover
// whole 128-B lines with one instruction, where two 16-B loads each touch
// every line of the span half-used (twice the L1 wavefronts)
__device__ __forceinline__ void ldcs8(const void* p, unsigned (&w)[8]) {
  asm volatile("ld.global.cs.v8.b32 {%0, %1, %2, %3, %4, %5, %6, %7}, [%8];"
               : "=r"(w[0]), "=r"(w[1]), "=r"(w[2]), "=r"(w[3]), "=r"(w[4]), "=r"(w[5]), "=r"(w[6]), "=r"(w[7])
               : "l"(p));
}

// ---- thread-block-cluster / distributed shared memory (inter_cluster)
__device__ __forceinline__ unsigned cluster_ctarank() {
  unsigned r;
  asm volatile("mov.u32 %0, %%cluster_ctarank;" : "=r"(r));
  return r;
}
__device__ __forceinline__ unsigned cluster_id_x() {
  unsigned r;
  asm volatile("mov.u32 %0, %%clusterid.x;" : "=r"(r));
  return r;
}
__device__ __forceinline__ unsigned mapa_rank(unsigned saddr, unsigned rank) {
  unsigned r;
  asm volatile("mapa.shared::cluster.u32 %0, %1, %2;" : "=r"(r) : "r"(saddr), "r"(rank));
  return r;
}
__device__ __forceinline__ void st_cl(unsigned addr, unsigned v) {
  asm volatile("st.shared::cluster.u32 [%0], %1;" ::"r"(addr), "r"(v) : "memory");
}
__device__ __forceinline__ unsigned ld_cl(unsigned addr) {
  unsigned v;
  asm volatile("ld.shared::cluster.u32 %0, [%1];" : "=r"(v) : "r"(addr) : "memory");
  return v;
}
__device__ __forceinline__ unsigned ld_acquire_cl(unsigned addr) {
  unsigned v;
  asm volatile("ld.acquire.cluster.shared::cluster.u32 %0, [%1];" : "=r"(v) : "r"(addr) : "memory");
  return v;
}
__device__ __forceinline__ void st_release_cl(unsigned addr, unsigned v) {
  asm volatile("st.release.cluster.shared::cluster.u32 [%0], %1;" ::"r"(addr), "r"(v) : "memory");
}
__device__ __forceinline__ void st_relaxed_cl(unsigned addr, unsigned v) {
  asm volatile("st.relaxed.cluster.shared::cluster.u32 [%0], %1;" ::"r"(addr), "r"(v) : "memory");
}
__device__ __forceinline__ void cluster_sync_all() {
  asm volatile("barrier.cluster.arrive.release.aligned;\n\tbarrier.cluster.wait.acquire.aligned;" ::: "memory");
}

// Inter queue publication/free (experiment knobs):
// RMT_PUB_FENCE_SC=1 the producer's batch fence is fence.sc.gpu (else
// fence.acq_rel.gpu); RMT_FREE_RELAXED=1 the consumer frees consumed slots with
// relaxed stores issued after the warp ballot that consumed every loaded word
// (else st.release.gpu, which also waits for the consumer's own output stores).
#ifndef RMT_PUB_FENCE_SC
#define RMT_PUB_FENCE_SC 1
#endif
#ifndef RMT_FREE_RELAXED
#define RMT_FREE_RELAXED 0
#endif
// Inter queue group flags (Rep<..., GROUP = true>; DESIGN.md "Inter-Group
// queue"): a producer publishing a group of g records behind one fence stores g,
// g-1, ..., 1 into their slot flags, so a consumer that acquires the flag of the
// group's first record knows the rest are visible too and reads their payloads
// without a flag round trip.
#ifndef RMT_SPIN_NS0
#define RMT_SPIN_NS0 32     // first back-off sleep of a queue wait (0: pure spin)
#endif
#ifndef RMT_SPIN_NSMAX
#define RMT_SPIN_NSMAX 512  // back-off cap
#endif
// Inter-Group record format (reading R-C-Q2):
// 1 = digest records -- one 64-bit word per lane and record, (j + 1) << 32 |
// digest(key, stored words), published and freed with single-copy-atomic
// relaxed accesses (no flag, fence or lock); 0 = the round-1/2 flag protocol
// (full key + value words behind group flags and a fence).
#ifndef RMT_INTER_DIGEST
#define RMT_INTER_DIGEST 1
#endif

// Record digest: a chain of bijections in each word (x -> (h ^ x) * odd, then an
// xorshift), so a change confined to ANY ONE word of (key, v0..v3) -- every
// single-bit fault of the fault model -- always changes the digest; changes in
// several words alias with probability ~2^-32.
template <int NW>
__host__ __device__ __forceinline__ unsigned rec_digest(unsigned key, unsigned mask, const unsigned (&v)[NW]) {
  unsigned h = key * 0x9E3779B1u;
  h ^= h >> 15;
#pragma unroll
  for (int k = 0; k < NW; ++k) {
    const unsigned w = ((mask >> k) & 1u) ? v[k] : 0u;  // unstored words are not compared (COND sites)
    h = (h ^ w) * 0x85EBCA77u;
    h ^= h >> 13;
  }
  return h;
}

// The digest of a lane that stores nothing (key 0xFFFFFFFF, no stored words),
// folded at compile time: COND sites (FloydWarshall's relaxations) mostly
// store nothing, so most lanes skip the digest chain.
template <int NW>
__host__ __device__ constexpr unsigned rec_digest_none() {
  unsigned h = 0xFFFFFFFFu * 0x9E3779B1u;
  h ^= h >> 15;
  for (int k = 0; k < NW; ++k) {
    h = h * 0x85EBCA77u;
    h ^= h >> 13;
  }
  return h;
}

// Spin (relaxed, L2-coherent: P:693) until the 64-bit word at p satisfies
// pred(word); returns the last word read.  Watchdog as spin_until below.
template <class Pred>
__device__ __forceinline__ unsigned long long spin64(const unsigned long long* p, unsigned long long x, Pred pred,
                                                     const Ctx& c, bool count) {
  if (pred(x)) return x;
  unsigned long long t0 = clock64();
  unsigned ns = RMT_SPIN_NS0;
  while (true) {
    if (ns) __nanosleep(ns);
    x = ld_relaxed64(p);
    if (pred(x)) return x;
    if (ns && ns < RMT_SPIN_NSMAX) ns <<= 1;
    if (clock64() - t0 > c.wd) {
      if (count) {
        atomicAdd(c.err, 1ull);
        atomicExch(c.ctrl + CTRL_WATCHDOG, 1u);
      }
      return x;
    }
  }
}

// Spin until *p == want (acquire), with back-off and a watchdog that converts a
// hang (a fault that desynchronised a pair) into err+1 and a sticky flag.
// Every thread that will touch the guarded data must do its own acquire: a lane
// of a (possibly diverged) warp is not ordered after another lane's acquire.
__device__ __forceinline__ bool spin_until(const unsigned* p, unsigned want, const Ctx& c, bool count = true) {
  if (ld_acquire(p) == want) return true;
  unsigned long long t0 = clock64();
  unsigned ns = RMT_SPIN_NS0;
  while (true) {
    if (ns) __nanosleep(ns);
    if (ld_acquire(p) == want) return true;
    if (ns && ns < RMT_SPIN_NSMAX) ns <<= 1;
    if (clock64() - t0 > c.wd) {
      if (count) {
        atomicAdd(c.err, 1ull);
        atomicExch(c.ctrl + CTRL_WATCHDOG, 1u);
      }
      return false;
    }
  }
}

// Spin until *p != 0 (acquire); returns the value seen, 0 after a watchdog timeout.
__device__ __forceinline__ unsigned spin_nonzero(const unsigned* p, const Ctx& c, bool count) {
  unsigned v = ld_acquire(p);
  if (v != 0u) return v;
  unsigned long long t0 = clock64();
  unsigned ns = RMT_SPIN_NS0;
  while (true) {
    if (ns) __nanosleep(ns);
    v = ld_acquire(p);
    if (v != 0u) return v;
    if (ns && ns < RMT_SPIN_NSMAX) ns <<= 1;
    if (clock64() - t0 > c.wd) {
      if (count) {
        atomicAdd(c.err, 1ull);
        atomicExch(c.ctrl + CTRL_WATCHDOG, 1u);
      }
      return 0u;
    }
  }
}

// Cluster-scope spin on a shared::cluster address (local or a peer CTA's).
__device__ __forceinline__ bool spin_cl(unsigned addr, unsigned want, const Ctx& c, bool count) {
  if (ld_acquire_cl(addr) == want) return true;
  unsigned long long t0 = clock64();
  while (true) {
    __nanosleep(20);
    if (ld_acquire_cl(addr) == want) return true;
    if (clock64() - t0 > c.wd) {
      if (count) atomicAdd(c.err, 1ull);
      return false;
    }
  }
}

// Experiment instrumentation (-DRMT_TRACE builds only): thread 0 of inter CTA
// `ticket` stores globaltimer at milestone k (0 start, 1 after ticket + region
// turn, 2 first commit entry, 3 first commit done, 4 finish entry, 5 finish
// exit, 6 SM id, 7 role).
#ifdef RMT_TRACE
__device__ __forceinline__ unsigned long long gtimer() {
  unsigned long long t;
  asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
  return t;
}
#define RMT_TR(k, v)                                                                        \
  do {                                                                                      \
    if (c.trace && threadIdx.x == 0 && tr_id < (1u << 17)) c.trace[(size_t)tr_id * 8 + (k)] = (v); \
  } while (0)
#else
#define RMT_TR(k, v) \
  do {               \
  } while (0)
#endif

// 32-bit mixer (stress skew and record tags): lowbias32
__device__ __forceinline__ unsigned mix32(unsigned x) {
  x ^= x >> 16;
  x *= 0x7feb352du;
  x ^= x >> 15;
  x *= 0x846ca68bu;
  x ^= x >> 16;
  return x;
}

// ---------------------------------------------------------------- replica state
// GROUP: inter-group queue with group flags (below); chosen per kernel -- it
// saves the consumer a flag round trip per record of a multi-record group, but
// costs registers (measured: PrefixSum inter 3.98 -> 2.67x,
// FWT 3.56 -> 3.41x, Transpose 3.11 -> 2.91x; BlackScholes 5.58 -> 6.48x and DCT
// 3.77 -> 4.25x lose a CTA per SM to the extra registers)
template <int V, int MODE, bool GROUP = false>
struct Rep {
  static constexpr bool INTRA = (V == V_INTRA_SMEM || V == V_INTRA_REG || V == V_INTRA_NOLDS);
  // +LDS: kernel-written shared memory duplicated per replica;
  // -LDS (intra_nolds): one copy, every kernel st.shared compared
  static constexpr bool SMDUP = (V == V_INTRA_SMEM || V == V_INTRA_REG);
  static constexpr bool NOLDS = (V == V_INTRA_NOLDS);
  static constexpr bool INTER = (V == V_INTER);
  static constexpr bool CLUSTER = (V == V_CLUSTER);
  static constexpr int DUP = INTRA ? 2 : 1;  // physical threads per logical thread
  static constexpr int LW = 32 / DUP;        // logical warp width
  static constexpr bool FAULT = (MODE == M_FAULT);
  static constexpr bool NOCOMM = (MODE == M_NOCOMM);
  static constexpr bool STRESS = (MODE == M_STRESS) && (V == V_INTER || V == V_CLUSTER);

  const Ctx& c;
  int r;          // replica id 0/1 (fault targeting)
  bool consumer;  // the replica that executes stores (none: always)
  int ltid;       // logical thread id within the logical CTA
  int lblock;     // logical CTA id
  int lane, warp, llane;
  unsigned j;     // records this warp has committed (inter)
  int lstride;    // logical CTAs advance by this (0: this CTA runs one logical CTA)
  unsigned nerr;  // intra: mismatching commits of this (consumer) lane, added to *err at finish()
  unsigned pend;  // inter: records not yet published (producer) / freed (consumer)
  unsigned region, epoch;
  unsigned rdy_hi;  // inter consumer: records below this are known to be published (group flags)
  unsigned pempty;  // inter producer: bit l = pending record (j - pend + l) is empty (COND, no lane stores)
  unsigned cempty, cbase;  // inter consumer: emptiness bits of the group starting at record cbase
  unsigned long long pf;  // inter (digest records): the word of the next record's slot, loaded ahead
  bool pfv;               // pf holds that word
  unsigned* mbox;  // intra_smem: this warp's mailbox
  unsigned tr_id;  // RMT_TRACE: trace row (inter ticket)
  unsigned cl_pay, cl_full;  // inter_cluster: this warp's mailbox / flags in the consumer CTA (shared::cluster)

  __device__ __forceinline__ explicit Rep(const Ctx& ctx)
      : c(ctx), j(0), lstride(0), nerr(0), pend(0), region(0), epoch(0), rdy_hi(0), pempty(0), cempty(0), cbase(0),
        pf(0ull), pfv(false),
        mbox(nullptr), cl_pay(0),
        cl_full(0) {}

  // ---- logical-CTA loop.  Kernel bodies are written
  //        rep.init(mb);
  //        for (; rep.active(); rep.advance()) { ... body of logical CTA rep.lblock ... }
  //        rep.finish();
  // none / intra: one logical CTA per physical CTA (one iteration).  inter_group
  // and inter_cluster launch a resident set of replica pairs once, and each pair
  // walks the logical CTAs pair, pair + P, pair + 2P, ... (persistent pairs: the
  // ticket, region and exit bookkeeping are paid once per pair instead of once
  // per logical CTA; both replicas walk the same sequence, so their commit
  // sequences stay in lockstep).  advance() is CTA-uniform and ends with a
  // barrier before the next logical CTA reuses shared memory (every body's last
  // commit is non-deferred, so no record is pending across it).
  __device__ __forceinline__ bool active() const { return lblock < c.nblocks; }
  __device__ __forceinline__ void advance() {
    if (lstride == 0) {
      lblock = c.nblocks;
    } else {
      __syncthreads();
      lblock += lstride;
    }
  }

  // Must be called by every thread of the CTA, first thing (may __syncthreads).
  // mbox_smem: MBOX_WORDS * (blockDim/32) words of shared memory (intra_smem only).
  __device__ __forceinline__ void init(unsigned* mbox_smem = nullptr) {
    // Programmatic dependent launch (launch_std sets the attribute): this
    // grid may be scheduled while the previous kernel on the stream drains;
    // wait for it to complete (and its memory to be visible) before touching
    // global memory or the inter ticket, then let the next kernel's CTAs be
    // scheduled as this grid's CTAs retire.  No-ops without the attribute.
    asm volatile("griddepcontrol.wait;" ::: "memory");
    asm volatile("griddepcontrol.launch_dependents;" ::: "memory");
    lane = threadIdx.x & 31;
    warp = threadIdx.x >> 5;
    if constexpr (INTRA) {
      r = threadIdx.x & 1;  // low bit of the id = producer/consumer flag
      consumer = (r == 0);  // Fig. 8: even lanes receive -> consumer
      ltid = threadIdx.x >> 1;
      llane = lane >> 1;
      lblock = blockIdx.x;
      if constexpr (V == V_INTRA_SMEM) mbox = mbox_smem + warp * MBOX_WORDS;
    } else if constexpr (INTER) {
      __shared__ unsigned s_ticket;
#ifdef RMT_TRACE
      const unsigned long long tr0 = gtimer();
#endif
      if (threadIdx.x == 0) s_ticket = atomicAdd(c.ctrl, 1u);  // P:679-681 global counter
      __syncthreads();
      unsigned t = s_ticket;
      tr_id = t;
#ifdef RMT_TRACE
      RMT_TR(0, tr0);
      {
        unsigned smid;
        asm volatile("mov.u32 %0, %%smid;" : "=r"(smid));
        RMT_TR(6, smid);
        RMT_TR(7, t & 1u);
      }
#endif
      const unsigned pair = t >> 1;  // P:681 mask the low bit -> identical pair
      lblock = (int)pair;            // first logical CTA of the pair
      lstride = c.lstride;
      r = (int)(t & 1u);
      consumer = (r == 1);     // even ticket = producer (reading R-RMT2)
      ltid = threadIdx.x;
      llane = lane;
      region = pair % (unsigned)c.R;
      epoch = pair / (unsigned)c.R;
      if constexpr (STRESS) {  // random per-CTA start skew: perturbs which role runs ahead
        if (c.stress & STRESS_SKEW) __nanosleep(mix32(t * 0x9E3779B9u + 1u) % (c.skew_ns + 1u));
      }
      if constexpr (!NOCOMM) {
        // Exclusive ownership of the queue region: wait until the pair that used
        // it before (lblock - R) has fully drained it (both roles wait).
        if (threadIdx.x == 0 && epoch != 0) spin_until(c.ctrl + CTRL_TURN + region, epoch, c);
        __syncthreads();
      }
#ifdef RMT_TRACE
      RMT_TR(1, gtimer());
#endif
    } else if constexpr (CLUSTER) {
      // The pair is a 2-CTA thread-block cluster: hardware co-schedules both
      // CTAs, so no ticket or turn is needed (the B200 form of P:679's
      // "co-scheduling" remark); rank 0 = producer, rank 1 = consumer.  Records go
      // into a mailbox in the CONSUMER's shared memory through distributed
      // shared memory (DSMEM), not through L2.
      // The mailbox is appended to the dynamic shared memory at byte offset c.R
      // (launch_std): per warp c.S records of RING_WORDS x 32 words, then c.S flags.
      extern __shared__ __align__(16) unsigned char rmt_dyn_smem[];
      r = (int)cluster_ctarank();
      consumer = (r == 1);
      lblock = (int)cluster_id_x();
      lstride = c.lstride;
      ltid = threadIdx.x;
      llane = lane;
      if constexpr (STRESS) {
        if (c.stress & STRESS_SKEW) __nanosleep(mix32((unsigned)(2 * lblock + r) * 0x9E3779B9u + 1u) % (c.skew_ns + 1u));
      }
      if constexpr (!NOCOMM) {
        const unsigned nw = blockDim.x >> 5;
        const unsigned base = (unsigned)__cvta_generic_to_shared(rmt_dyn_smem) + (unsigned)c.R;
        const unsigned fl0 = base + nw * (unsigned)(c.S * RING_WORDS * 32) * 4u;
        unsigned* flp = (unsigned*)__cvta_shared_to_generic(fl0);
        for (unsigned i = threadIdx.x; i < nw * (unsigned)c.S; i += blockDim.x) flp[i] = 0u;
        unsigned pb = base + (unsigned)(warp * c.S * RING_WORDS * 32) * 4u;
        unsigned fb = fl0 + (unsigned)(warp * c.S) * 4u;
        cl_pay = consumer ? pb : mapa_rank(pb, 1u);
        cl_full = consumer ? fb : mapa_rank(fb, 1u);
        cluster_sync_all();  // both mailboxes initialised before any record
      }
    } else {
      r = 0;
      consumer = true;
      ltid = threadIdx.x;
      llane = lane;
      lblock = blockIdx.x;
    }
  }

  // Must be called by every thread of the CTA, last thing.
  // ---- inter queue: publish / free the pending records of this warp.
  // Producer: one fence by every lane covers all pending payloads, then lane l
  // sets the flag of pending record l.  Consumer: lane l frees pending slot l
  // with one release store (the ballot after every compare already consumed the
  // loaded words).  Called at every non-deferred commit and before finish().
  __device__ __forceinline__ size_t slot_index(unsigned rec) const {
    return ((size_t)region * c.W + warp) * c.S + (rec % (unsigned)c.S);
  }
  __device__ __forceinline__ void flush() {
    if constexpr (CLUSTER && !NOCOMM) {
      if (pend == 0u) return;
      const unsigned first = j - pend;
      if (!consumer) {
        asm volatile("fence.acq_rel.cluster;" ::: "memory");
        __syncwarp();
        if ((unsigned)lane < pend) st_relaxed_cl(cl_full + ((first + lane) & (unsigned)(c.S - 1)) * 4u, 1u);
      } else {
        __syncwarp();
        if ((unsigned)lane < pend) st_release_cl(cl_full + ((first + lane) & (unsigned)(c.S - 1)) * 4u, 0u);
        __syncwarp();  // every lane's later poll of a freed slot sees the free (lane l freed slot l)
      }
      pend = 0u;
    }
    if constexpr (INTER && !NOCOMM && !RMT_INTER_DIGEST) {
      if (pend == 0u) return;
      const unsigned first = j - pend;
      if (!consumer) {
        // group flags: record first + l gets pend - l (its distance to the
        // group's end).  The non-first flags are stored BEFORE the fence and
        // the first record's flag (the group's "ready" signal) after it: a
        // consumer that acquired flag[first] then frees the other slots only
        // after their flag stores, never before one lands late and leaves a
        // stale "full" flag (found by tests/model/ring_model.cpp)
        // Flag value = distance to the group's end | emptiness << 8: an EMPTY
        // record (a COND commit where no lane stores) carries no payload, the
        // consumer learns it from the flag (group flags: the first record's flag
        // holds the whole group's emptiness bits).
        if constexpr (GROUP)
          if ((unsigned)lane - 1u < pend - 1u) st_relaxed(c.flags + slot_index(first + lane), pend - lane);
#if RMT_PUB_FENCE_SC
        asm volatile("fence.sc.gpu;" ::: "memory");
#else
        asm volatile("fence.acq_rel.gpu;" ::: "memory");
#endif
        __syncwarp();
        if constexpr (GROUP) {
          if (lane == 0) st_relaxed(c.flags + slot_index(first), pend | (pempty << 8));
        } else {
          if ((unsigned)lane < pend) st_relaxed(c.flags + slot_index(first + lane), 1u | (((pempty >> lane) & 1u) << 8));
        }
        pempty = 0u;
      } else {
        __syncwarp();
#if RMT_FREE_RELAXED
        if ((unsigned)lane < pend) st_relaxed(c.flags + slot_index(first + lane), 0u);
#else
        if ((unsigned)lane < pend) st_release(c.flags + slot_index(first + lane), 0u);
#endif
        // Lane l freed the slot of record first + l; the barrier orders those
        // stores before every lane's later poll of the same slots (a lane that
        // polled a slot another lane had just freed could read the old record's
        // flag and consume its stale payload)
        __syncwarp();
      }
      pend = 0u;
    }
  }

  __device__ __forceinline__ void finish() {
    if constexpr (INTRA) {  // deferred error count (mismatches are rare: one atomic per faulty lane)
      if (nerr != 0u) atomicAdd(c.err, (unsigned long long)nerr);
    }
    if constexpr (CLUSTER && !NOCOMM) {
      flush();
      cluster_sync_all();  // no DSMEM access of either CTA is in flight when they exit
    }
    if constexpr (INTER) {
      __shared__ unsigned s_last;
#ifdef RMT_TRACE
      RMT_TR(4, gtimer());
#endif
      flush();
      __syncthreads();
      if (threadIdx.x == 0) {
        if (consumer && !NOCOMM) st_release(c.ctrl + CTRL_TURN + region, epoch + 1);
        __threadfence();
        unsigned d = atomicAdd(c.ctrl + 1, 1u);
        s_last = (d == 2u * (unsigned)c.pairs - 1u);
      }
      __syncthreads();
      if (s_last) {  // self-reset: the next launch starts from zero
        __threadfence();
        for (int i = threadIdx.x; i < c.R; i += blockDim.x) c.ctrl[CTRL_TURN + i] = 0;
        // After a watchdog abort a producer may have published records its
        // consumer never freed: clear every slot flag (all other CTAs have
        // finished, so no flag store is in flight).  The sticky watchdog flag
        // itself stays set for rmt_workspace_status() to report.
        if (ld_relaxed(c.ctrl + CTRL_WATCHDOG) != 0u) {
          const size_t nslots = (size_t)c.R * (size_t)c.W * (size_t)INTER_SLOTS_MAX;
          for (size_t i = threadIdx.x; i < nslots; i += blockDim.x) c.flags[i] = 0u;
          if (RMT_INTER_DIGEST) {  // digest records: every slot word a lost consumer left behind
            unsigned long long* w = reinterpret_cast<unsigned long long*>(c.payload);
            for (size_t i = threadIdx.x; i < nslots * 32; i += blockDim.x) w[i] = 0ull;
          }
        }
        if (threadIdx.x == 0) {
          c.ctrl[CTRL_TICKET] = 0;
          c.ctrl[CTRL_DONE] = 0;
        }
      }
#ifdef RMT_TRACE
      RMT_TR(5, gtimer());
#endif
    }
  }

  // ---- duplicated shared memory (+LDS): replica r owns its interleaved copy
  template <class T>
  __device__ __forceinline__ T& sm(T* base, int i) const {
    if constexpr (SMDUP) return base[2 * i + r];
    else return base[i];
  }

  // ---- duplicated shared memory in planes: replica r owns base[PLANE*r + i].
  // PLANE is chosen per kernel so the two replicas of a pair land in disjoint
  // banks for that kernel's access patterns (interleaving conflicts otherwise).
  template <int PLANE, class T>
  __device__ __forceinline__ T& smp(T* base, int i) const {
    if constexpr (SMDUP) return base[PLANE * r + i];
    else return base[i];
  }

  // ---- -LDS shared stores (intra_nolds).  The pair shares one copy of the
  // kernel's shared memory, so a shared store leaves the sphere of replication
  // ("-LDS ... communicate ... on every LDS write"): the replicas
  // exchange (index, words) through registers and compare; a mismatch counts one
  // error; the store is performed once, by the consumer, with its own value.
  // Returns whether this lane performs the store (every other variant: true).
  // Both lanes of the pair must call it together (they always share control flow).
  template <int NW>
  __device__ __forceinline__ bool sts_ok(const unsigned (&w)[NW], unsigned i) const {
    if constexpr (!NOLDS) {
      return true;
    } else {
      if constexpr (NOCOMM) return consumer;
      const unsigned pm = 3u << (lane & ~1);
      bool mism = __shfl_xor_sync(pm, i, 1) != i;
#pragma unroll
      for (int k = 0; k < NW; ++k) mism |= __shfl_xor_sync(pm, w[k], 1) != w[k];
      if (mism && consumer) atomicAdd(c.err, 1ull);
      return consumer;
    }
  }
  __device__ __forceinline__ bool sts_ok1(unsigned w, unsigned i) const {
    const unsigned a[1] = {w};
    return sts_ok<1>(a, i);
  }

  // ---- logical-warp shuffles (replica-private: lanes keep their role bit)
  __device__ __forceinline__ unsigned lshfl_xor(unsigned v, int m) const {
    return __shfl_xor_sync(FULL, v, m * DUP);
  }
  __device__ __forceinline__ unsigned lshfl_idx(unsigned v, int src) const {
    return __shfl_sync(FULL, v, src * DUP + (INTRA ? r : 0));
  }
  // value of logical lane (llane - d); lanes with llane < d get their own value
  __device__ __forceinline__ unsigned lshfl_up(unsigned v, int d) const {
    unsigned u = __shfl_up_sync(FULL, v, d * DUP);
    return llane >= d ? u : v;
  }
  __device__ __forceinline__ unsigned long long lshfl_xor64(unsigned long long v, int m) const {
    return __shfl_xor_sync(FULL, v, m * DUP);
  }
  // logical ballot: bit l set iff logical lane l (this replica) has p
  __device__ __forceinline__ unsigned lballot(bool p) const {
    unsigned b = __ballot_sync(FULL, p);
    if constexpr (INTRA) {
      b >>= r;
      unsigned o = 0;
#pragma unroll
      for (int i = 0; i < 16; ++i) o |= ((b >> (2 * i)) & 1u) << i;
      return o;
    } else {
      return b;
    }
  }

  // ---- fault hooks (compiled out unless MODE == M_FAULT)
  __device__ __forceinline__ unsigned fault(int site, long long elem, unsigned x) const {
    if constexpr (FAULT) {
      // -LDS: a SMEM-site fault corrupts the single shared copy, i.e. what both
      // replicas read (shared memory is outside this variant's SoR)
      if (c.f.site == site && c.f.elem == elem && (c.f.replica == r || (NOLDS && site == SITE_SMEM)))
        x ^= 1u << c.f.bit;
    }
    return x;
  }
  __device__ __forceinline__ float faultf(int site, long long elem, float x) const {
    if constexpr (FAULT) return __uint_as_float(fault(site, elem, __float_as_uint(x)));
    return x;
  }

  // ---- error aggregation: one atomic per warp that saw mismatches
  __device__ __forceinline__ void count_mismatch(bool mism) const {
    unsigned m = __ballot_sync(FULL, mism);
    if (m != 0u && lane == __ffs(m) - 1) atomicAdd(c.err, (unsigned long long)__popc(m));
  }

  // ---- the commit.  Warp-collective: every lane of the warp must
  // call it at the same program point (uniform control flow around commits).
  //   mask  bit k set = word k is stored (a store instruction's predicate)
  //   idx   element index of word 0 in the destination (any value; the key keeps all 32 bits)
  //   v     the NW 32-bit value words
  //   limit destination element count (bounds for address faults in V_NONE)
  //   store functor store(idx, mask, v) performing the actual global store(s)
  //   SID   store-site id (faults on STORE_* sites target SID 0)
  //   LIVE  liveness-critical store (other CTAs spin on it): on a mismatch the
  //         consumer still stores its own value (reading R-RMT5) and counts it.
  //   defer (warp-uniform; inter only): do not publish/free yet.  A deferred
  //         commit MUST be followed by a non-deferred commit (or finish())
  //         before any CTA-wide barrier, and a run of deferred commits plus its
  //         closing commit must not exceed INTER_S records (deadlock freedom,
  //         DESIGN.md "Inter-Group queue").
  //   stride element distance between consecutive words (1: a contiguous vector;
  //         the store functor places word k at idx + k * stride)
  template <int NW, int SID = 0, bool LIVE = false, bool COND = false, class Store>
  __device__ __forceinline__ void commit(unsigned mask, unsigned idx, unsigned (&v)[NW], unsigned limit,
                                         Store&& store, bool defer = false, unsigned stride = 1) {
    static_assert(NW >= 1 && NW <= MAXW, "commit width");
    bool addr_faulted = false;
    if constexpr (FAULT) {
      const long long d = c.f.elem - (long long)idx;
      if (c.f.sid == SID && c.f.replica == r && d >= 0 && d % (long long)stride == 0 &&
          d / (long long)stride < NW) {
        if (c.f.site == SITE_STORE_VAL) {
          int w = (int)(d / (long long)stride);
#pragma unroll
          for (int k = 0; k < NW; ++k)
            if (k == w) v[k] ^= 1u << c.f.bit;
        } else if (c.f.site == SITE_STORE_ADDR) {
          idx ^= 1u << c.f.bit;  // any bit of the element index (0..31)
          addr_faulted = true;
        }
      }
    }
    if constexpr (V == V_NONE) {
      if (mask != 0u) {
        if constexpr (FAULT) {
          // a faulted address whose stored words fall outside the buffer, or that
          // is misaligned for a contiguous vector store, is dropped (the hardware
          // would raise an exception instead; either way the word is not written)
          if (addr_faulted && ((unsigned long long)idx + (31u - (unsigned)__clz(mask)) * (unsigned long long)stride >=
                                   limit ||
                               (NW > 1 && stride == 1u && idx % (unsigned)NW != 0u)))
            return;
        }
        store(idx, mask, v);
      }
      return;
    } else {
      if constexpr (NOCOMM) {
        // Ablation: both replicas computed; no exchange, no compare.
        if (consumer) {
          if (mask != 0u) store(idx, mask, v);
        } else {
#pragma unroll
          for (int k = 0; k < NW; ++k) keep_alive(v[k]);
        }
        if constexpr (INTER || CLUSTER) ++j;
        return;
      }
      (void)defer;
      // Record key: address + predicate in one word.  For a storing lane,
      // key = idx ^ (mask << 28) keeps every bit of the element index (vector
      // sites need not be aligned, e.g. FWT's strided commits) and is injective
      // in each argument separately: a fault in either the address or the
      // predicate of one replica (any single bit, or any corruption of only one
      // of the two) changes the key.  A lane that stores nothing has no address
      // to compare (key 0xFFFFFFFF); since vector-committed buffers hold < 2^30
      // elements, no storing lane whose mask differs from 0 in one bit can have
      // that key.
      unsigned key;
      if constexpr (NW == 1) key = mask ? idx : 0xffffffffu;
      else key = mask ? (idx ^ (mask << 28)) : 0xffffffffu;
      unsigned key0 = 0xffffffffu;  // the key of a lane that stores nothing
      if constexpr (STRESS) {
        // (pair, warp, sequence) tag folded into the key on both sides: a record
        // consumed out of order, twice, or from another pair's/warp's ring fails
        // the compare (counted in err)
        const unsigned tag = mix32(((unsigned)lblock * 64u + (unsigned)warp) * 0x01000193u) ^ mix32(j + 0x51ED270Bu);
        if (c.stress & STRESS_TAGS) {
          key ^= tag;
          key0 ^= tag;
        }
        if (c.stress & STRESS_SKEW) {  // one commit in 8 (per warp and role) sleeps a random while
          const unsigned h = mix32(tag ^ (unsigned)r * 0x2545F491u);
          if ((h & 7u) == 0u) __nanosleep((h >> 3) % (c.skew_ns + 1u));
        }
        if ((c.stress & STRESS_DROP) && lblock == 0 && !consumer) {  // a lost producer: pair 0 never publishes
          ++j;
          return;
        }
      }
      if constexpr (INTRA && COND) {
        // A conditional store site where no lane of the warp stores -- in EITHER
        // replica: both sit in this warp -- has nothing to exchange: every
        // predicate already agrees.  One vote instead of the key
        // exchange and compare (a fault that turns a predicate on makes the vote
        // true and takes the full path).
        if (!__any_sync(FULL, mask != 0u)) return;
      }
      unsigned pk = 0, pv[NW];
      bool have = true;  // consumer got the producer's record
      if constexpr (V == V_INTRA_REG || V == V_INTRA_NOLDS) {
        pk = __shfl_xor_sync(FULL, key, 1);
        // COND (a conditional store site, e.g. FloydWarshall's improvements):
        // values move only if some lane of the warp stores
        if (!COND || __any_sync(FULL, mask != 0u)) {
#pragma unroll
          for (int k = 0; k < NW; ++k) pv[k] = __shfl_xor_sync(FULL, v[k], 1);
        }
      } else if constexpr (V == V_INTRA_SMEM) {
        const int slot = lane >> 1;
        // COND store sites: value words move only for the words a lane really
        // stores; the key carries the predicate mask, so a word the
        // consumer stores is compared only if the producer's key (same mask)
        // matched.  Unconditional sites (every lane stores every word) move
        // all words without per-word predicates (measured: the predicates
        // cost 1-10% on the streaming kernels)
        if (!consumer) {
          mbox[slot] = key;
#pragma unroll
          for (int k = 0; k < NW; ++k)
            if (!COND || ((mask >> k) & 1u)) mbox[(1 + k) * 16 + slot] = v[k];
        }
        __syncwarp();
        if (consumer) {
          pk = mbox[slot];
#pragma unroll
          for (int k = 0; k < NW; ++k) pv[k] = (!COND || ((mask >> k) & 1u)) ? mbox[(1 + k) * 16 + slot] : 0u;
        }
        __syncwarp();
      } else if constexpr (V == V_CLUSTER) {  // DSMEM mailbox in the consumer CTA
        const unsigned slot = j & (unsigned)(c.S - 1);
        const unsigned pa = cl_pay + (slot * RING_WORDS * 32 + lane) * 4u;
        const unsigned fa = cl_full + slot * 4u;
        if (!consumer) {
          if (j >= (unsigned)c.S) {  // publish ours first, then wait for a free slot
            flush();
            spin_cl(fa, 0u, c, lane == 0);
          }
          st_cl(pa, key);
#pragma unroll
          for (int k = 0; k < NW; ++k)
            if (!COND || ((mask >> k) & 1u)) st_cl(pa + (1 + k) * 32 * 4, v[k]);
        } else {
          // a consumer holding S unfreed records frees them before it waits on
          // a slot (any depth S >= 1, however long the deferred run)
          if (pend >= (unsigned)c.S) flush();
          have = spin_cl(fa, 1u, c, lane == 0);  // every lane acquires
          pk = ld_cl(pa);
#pragma unroll
          for (int k = 0; k < NW; ++k) pv[k] = (!COND || ((mask >> k) & 1u)) ? ld_cl(pa + (1 + k) * 32 * 4) : 0u;
        }
      } else if constexpr (V == V_INTER && RMT_INTER_DIGEST) {
        // Digest records (R-C-Q2): record j of this (region, warp) is ONE 64-bit
        // word per lane in slot j % S: (j + 1) << 32 | digest(key, stored words).
        // A slot word is 0 (free) or a record; the producer writes only a free
        // slot, the consumer waits for marker j + 1 and frees it -- all relaxed
        // accesses to the same address, ordered by coherence, so no flag,
        // fence or lock; the first tier (region turns) is unchanged.  The
        // word of the next record's slot is loaded ahead at the end of a commit.
        unsigned h;
        if constexpr (COND && !STRESS) {
          constexpr unsigned H0 = rec_digest_none<NW>();
          h = mask == 0u ? H0 : rec_digest<NW>(key, mask, v);  // key is 0xFFFFFFFF when mask == 0
        } else {
          h = rec_digest<NW>(key, mask, v);
        }
        unsigned long long* const ring = reinterpret_cast<unsigned long long*>(c.payload);
        unsigned long long* const pw = ring + slot_index(j) * 32 + lane;
        if (!consumer) {
          if (j >= (unsigned)c.S) {  // record j - S must have been freed ("waits for a free buffer")
            const unsigned long long x = pfv ? pf : ld_relaxed64(pw);
            spin64(pw, x, [](unsigned long long w) { return w == 0ull; }, c, lane == 0);
          }
          st_relaxed64(pw, ((unsigned long long)(j + 1u) << 32) | h);
          pfv = j + 1u >= (unsigned)c.S;
          if (pfv) pf = ld_relaxed64(ring + slot_index(j + 1u) * 32 + lane);
        } else {
          const unsigned mk = j + 1u;
          unsigned long long x = pfv ? pf : ld_relaxed64(pw);
          x = spin64(pw, x, [mk](unsigned long long w) { return (unsigned)(w >> 32) == mk; }, c, lane == 0);
          have = (unsigned)(x >> 32) == mk;
          st_relaxed64(pw, 0ull);  // free: the same address, after the read
          pk = (unsigned)x ^ h;    // 0 iff the digests agree
          pfv = true;
          pf = ld_relaxed64(ring + slot_index(j + 1u) * 32 + lane);
        }
      } else {  // V_INTER: per-(region, warp) queue of S records
#ifdef RMT_TRACE
        if (j == 0) RMT_TR(2, gtimer());
#endif
        const size_t fi = slot_index(j);
        unsigned* fl = c.flags + fi;
        unsigned* pl = c.payload + fi * (RING_WORDS * 32);
        if (!consumer) {
          // wait for a free buffer; the first S slots of a fresh region are
          // free.  Publish our own pending records first, or our consumer could be
          // waiting for them while we wait for it.
          if (j >= (unsigned)c.S) {
            if constexpr (GROUP) {
              // publish the pending group only if we must block on this slot, so
              // that groups stay whole while the consumer keeps up.  The slot is
              // ours only if record j - S was published and consumed: a flag of 0
              // also marks our own unpublished records, so with S of them pending
              // we must publish (and wait) before overwriting the oldest.
              if (pend >= (unsigned)c.S || ld_acquire(fl) != 0u) {
                flush();
                spin_until(fl, 0u, c, lane == 0);
              }
            } else {
              flush();
              spin_until(fl, 0u, c, lane == 0);
            }
          }
          // COND: an empty record (no lane of the warp stores) moves no payload,
          // only its emptiness bit in the flag ("never execute a global write")
          bool empty = false;
          if constexpr (COND) empty = __ballot_sync(FULL, mask != 0u) == 0u;
          if (!empty) {
            pl[lane] = key;
#pragma unroll
            for (int k = 0; k < NW; ++k)
              if (!COND || ((mask >> k) & 1u)) pl[(1 + k) * 32 + lane] = v[k];  // COND: only stored words move
          }
          pempty |= (empty ? 1u : 0u) << pend;
          // The "ready" signal ("signals the work-item in the consumer") is
          // published by flush(): every lane fences its own payload stores (a
          // release by one lane does not order the other lanes' in-flight stores).
        } else {
          if (pend >= (unsigned)c.S) flush();  // as above: never wait on a slot we still hold
          bool ok = true, empty = false;
          if constexpr (GROUP) {
            if (j >= rdy_hi) {  // each lane acquires the "ready" signal of the group's first record
              const unsigned g = spin_nonzero(fl, c, lane == 0);
              ok = g != 0u;
              rdy_hi = j + (g & 0xFFu);  // records j .. j+g-1 were published behind one fence
              cempty = g >> 8;
              cbase = j;
            }
            empty = (cempty >> (j - cbase)) & 1u;
          } else {
            const unsigned fv = spin_nonzero(fl, c, lane == 0);  // each lane acquires the "ready" signal
            ok = fv != 0u;
            empty = (fv >> 8) & 1u;
          }
          if (COND && empty) {  // the producer stored nothing: every lane's key is key0
            pk = key0;
#pragma unroll
            for (int k = 0; k < NW; ++k) pv[k] = 0u;
          } else {
            pk = ld_relaxed(pl + lane);  // L2-coherent (bypasses L1)
#pragma unroll
            for (int k = 0; k < NW; ++k) pv[k] = (!COND || ((mask >> k) & 1u)) ? ld_relaxed(pl + (1 + k) * 32 + lane) : 0u;
          }
          have = ok;
          // the buffer is freed only after every lane has consumed its words
          // (below, after the compare's warp ballot)
        }
      }
      bool mism = false;
      if (consumer) {
        // bitwise difference of key (address + predicate) and of the stored words
        // (digest records: pk is already the digest difference)
        unsigned d;
        if constexpr (V == V_INTER && RMT_INTER_DIGEST) {
          d = pk;
        } else {
          d = pk ^ key;
#pragma unroll
          for (int k = 0; k < NW; ++k) d |= (pv[k] ^ v[k]) & (0u - ((mask >> k) & 1u));
        }
        const bool eq = have && d == 0u;
        if (eq) {
          if (mask != 0u) store(idx, mask, v);
        } else {
          mism = true;
          if constexpr (LIVE) {  // highest stored word inside the buffer, vector aligned
            if (mask != 0u &&
                (unsigned long long)idx + (31u - (unsigned)__clz(mask)) * (unsigned long long)stride < limit &&
                !(NW > 1 && stride == 1u && idx % (unsigned)NW != 0u))
              store(idx, mask, v);
          }
        }
      }
      if constexpr (INTRA) {
        nerr += mism ? 1u : 0u;  // counted at finish(): no per-commit vote
      } else {
        // warp ballot over the compare results: completes every lane's loads
        // (the inter queue frees the slots only after it)
        const unsigned mb = __ballot_sync(FULL, mism);
        if (mb != 0u && lane == __ffs(mb) - 1) atomicAdd(c.err, (unsigned long long)__popc(mb));
      }
      if constexpr (V == V_INTER && RMT_INTER_DIGEST) {
        ++j;  // published and freed above; nothing pending
      } else if constexpr (INTER || CLUSTER) {
        ++j;
        ++pend;
        if (!defer) flush();  // publish (producer) / free the buffers (consumer)
#ifdef RMT_TRACE
        if (INTER && j == 1) RMT_TR(3, gtimer());
#endif
      }
    }
  }
};

// ---------------------------------------------------------------- launch geometry
template <int V>
struct Geom {
  static constexpr int DUP = (V == V_INTRA_SMEM || V == V_INTRA_REG || V == V_INTRA_NOLDS) ? 2 : 1;
  static constexpr int SMDUP = (V == V_INTRA_SMEM || V == V_INTRA_REG) ? 2 : 1;  // kernel smem copies
  static __host__ __device__ unsigned grid(unsigned lblocks) {
    return (V == V_INTER || V == V_CLUSTER) ? 2u * lblocks : lblocks;
  }
  static __host__ __device__ unsigned block(unsigned lthreads) { return lthreads * DUP; }
};

// Per-warp-mailbox shared memory words a kernel must reserve.
template <int V>
__host__ __device__ constexpr int mbox_words(int phys_threads) {
  return V == V_INTRA_SMEM ? MBOX_WORDS * (phys_threads / 32) : 1;
}

}  // namespace rmt
