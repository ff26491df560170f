// ring_model.cpp -- CPU model of the inter-group queue protocol (TEST
// INFRASTRUCTURE; SURVEY.md 8(c) row "C-Q inter-group ring"
// "two-tiered locking system", P:693 coherent reads).
//
// Restates, with std::atomic and C++ memory orders, the protocol that
// paper_conf_isca_waddenlgss14_b200/csrc/rmt_device.cuh implements for
// V_INTER (Rep::init / commit / flush / finish), one thread per CTA role:
//   * tickets from a global counter in start order; pair = t >> 1, even ticket =
//     producer, odd = consumer;
//   * region = pair % R; both roles wait for turn[region] == pair / R, the
//     consumer advances it at exit;
//   * per (region) a ring of S slots with 0/1 flags; record j lives in slot j % S;
//   * producer: records are published in groups at every non-deferred commit:
//     record first + l (l >= 1) gets flag value g - l (g = group size), then
//     one fence, then record first gets g | emptiness bits << 8 (the group's
//     "ready" signal; an empty record -- no lane stores -- has no payload);
//     before writing record j >= S it publishes its pending group and waits
//     for slot j % S, but only if it must block: S records of its own pending,
//     or the slot's flag still set (record j - S published, not yet freed);
//   * consumer: before waiting on record j it frees its pending records if it
//     holds S of them; for the first record of a group it waits for a nonzero
//     flag (acquire) -- the value g says records j .. j+g-1 are visible, so
//     those need no flag check of their own; it reads, compares, and frees in
//     batches at every non-deferred commit (release store of 0);
//   * the last finisher resets tickets and turns.
// Workers (the resident CTA slots) take tickets until 2P are gone.  Checks: every
// record is consumed exactly once, in order, with the payload its producer wrote
// (tagged (pair, seq)); every launch finishes (no deadlock) for any S >= 1, any
// R >= 1 and any number of workers >= 2; the control block is zero afterwards.
//
//   ring_model S R WORKERS PAIRS RECORDS SEED LAUNCHES
#include <atomic>
#include <cstdint>
#include <cstdio>
#include <cstdlib>
#include <random>
#include <thread>
#include <vector>

struct Queue {
  int S, R;
  std::atomic<unsigned> ticket{0}, done{0};
  std::vector<std::atomic<unsigned>> turn;     // R
  std::vector<std::atomic<unsigned>> flag;     // R * S
  std::vector<std::atomic<uint64_t>> payload;  // R * S (relaxed: ordered by the flags)
  Queue(int S_, int R_) : S(S_), R(R_), turn(R_), flag((size_t)R_ * S_), payload((size_t)R_ * S_) {
    for (auto& t : turn) t.store(0);
    for (auto& f : flag) f.store(0);
    for (auto& p : payload) p.store(0);
  }
};

static std::atomic<long> g_errors{0};

static void jitter(std::mt19937& rng) {
  unsigned r = rng() % 16;
  if (r == 0) std::this_thread::yield();
  else if (r == 1) for (volatile int i = 0; i < (int)(rng() % 2000); ++i) {}
}

static uint64_t tag(unsigned pair, unsigned seq) { return ((uint64_t)pair << 32) ^ (seq * 0x9E3779B97F4A7C15ull); }
// an EMPTY record (a COND commit where no lane stores) carries no payload: the
// producer sets its emptiness bit in the group's first flag (bits 8..15)
static bool is_empty(unsigned pair, unsigned seq) { return ((pair * 0x9E3779B9u) ^ (seq * 0x85EBCA6Bu)) % 3u == 0u; }

// one CTA role: the commit sequence of a warp (deferral pattern = program order,
// identical in both roles: `defer[j]`)
static void run_role(Queue& q, unsigned t, unsigned nblocks, const std::vector<bool>& defer, std::mt19937& rng) {
  const unsigned pair = t >> 1;
  const bool consumer = t & 1u;
  const unsigned region = pair % (unsigned)q.R, epoch = pair / (unsigned)q.R;
  while (q.turn[region].load(std::memory_order_acquire) != epoch) std::this_thread::yield();  // region ownership
  auto slot = [&](unsigned rec) { return (size_t)region * q.S + rec % (unsigned)q.S; };
  unsigned j = 0, pend = 0, rdy_hi = 0, pempty = 0, cempty = 0, cbase = 0;
  auto flush = [&]() {
    if (pend == 0) return;
    const unsigned first = j - pend;
    if (!consumer) {
      // the group's non-first flags go out BEFORE the fence and the first
      // record's flag after it: a consumer that acquires flag[first] then sees
      // every other flag of the group already stored, so its later frees of
      // those slots cannot be overtaken by a late producer flag store (which
      // would leave a stale "full" flag: a stale read or a deadlock)
      // (jitter between the stores: lanes' stores land in any order)
      for (unsigned l = 1; l < pend; ++l) {
        q.flag[slot(first + l)].store(pend - l, std::memory_order_relaxed);
        jitter(rng);
      }
      std::atomic_thread_fence(std::memory_order_seq_cst);  // fence.sc.gpu
      q.flag[slot(first)].store(pend | (pempty << 8), std::memory_order_relaxed);
      pempty = 0;
    } else {
      for (unsigned l = 0; l < pend; ++l) q.flag[slot(first + l)].store(0, std::memory_order_release);
    }
    pend = 0;
  };
  for (size_t k = 0; k < defer.size(); ++k) {
    jitter(rng);
    const size_t s = slot(j);
    if (!consumer) {
      if (j >= (unsigned)q.S && (pend >= (unsigned)q.S || q.flag[s].load(std::memory_order_acquire) != 0)) {
        flush();
        while (q.flag[s].load(std::memory_order_acquire) != 0) std::this_thread::yield();
      }
      if (is_empty(pair, j)) pempty |= 1u << pend;
      else q.payload[s].store(tag(pair, j), std::memory_order_relaxed);
    } else {
      if (pend >= (unsigned)q.S) flush();
      if (j >= rdy_hi) {
        unsigned g;
        while ((g = q.flag[s].load(std::memory_order_acquire)) == 0) std::this_thread::yield();
        rdy_hi = j + (g & 0xFFu);
        cempty = g >> 8;
        cbase = j;
      }
      const bool empty = (cempty >> (j - cbase)) & 1u;
      if (empty != is_empty(pair, j)) {
        g_errors.fetch_add(1);
        std::fprintf(stderr, "pair %u record %u: emptiness bit %d\n", pair, j, (int)empty);
      }
      const uint64_t got = empty ? tag(pair, j) : q.payload[s].load(std::memory_order_relaxed);
      if (got != tag(pair, j)) {
        g_errors.fetch_add(1);
        std::fprintf(stderr, "pair %u record %u: got tag %llx\n", pair, j, (unsigned long long)got);
      }
    }
    ++j;
    ++pend;
    if (!defer[k]) flush();
  }
  flush();
  if (consumer) q.turn[region].store(epoch + 1, std::memory_order_release);
  std::atomic_thread_fence(std::memory_order_seq_cst);
  const unsigned d = q.done.fetch_add(1);
  if (d == 2 * nblocks - 1) {  // last CTA: self-reset
    for (auto& tr : q.turn) tr.store(0, std::memory_order_relaxed);
    q.ticket.store(0);
    q.done.store(0);
  }
}

int main(int argc, char** argv) {
  if (argc < 8) {
    std::fprintf(stderr, "usage: ring_model S R WORKERS PAIRS RECORDS SEED LAUNCHES\n");
    return 2;
  }
  const int S = atoi(argv[1]), R = atoi(argv[2]), W = atoi(argv[3]);
  const unsigned P = (unsigned)atoi(argv[4]);
  const int NREC = atoi(argv[5]);
  const unsigned seed = (unsigned)atoi(argv[6]);
  const int launches = atoi(argv[7]);
  Queue q(S, R);
  std::mt19937 g(seed);
  for (int L = 0; L < launches; ++L) {
    // the warp's commit sequence: runs of 0..5 deferred commits closed by a non-deferred one
    std::vector<bool> defer;
    while ((int)defer.size() < NREC) {
      int run = (int)(g() % 6);
      for (int i = 0; i < run && (int)defer.size() < NREC - 1; ++i) defer.push_back(true);
      defer.push_back(false);
    }
    std::atomic<unsigned> next{0};
    std::vector<std::thread> th;
    for (int w = 0; w < W; ++w) {
      th.emplace_back([&, w]() {
        std::mt19937 rng(seed * 7919u + (unsigned)w * 104729u + (unsigned)L);
        while (true) {
          // a worker (resident CTA slot) starts the next CTA: it takes a ticket first
          if (next.fetch_add(1) >= 2 * P) break;
          const unsigned t = q.ticket.fetch_add(1);
          run_role(q, t, P, defer, rng);
        }
      });
    }
    for (auto& t : th) t.join();
    bool clean = q.ticket.load() == 0 && q.done.load() == 0;
    for (auto& tr : q.turn) clean = clean && tr.load() == 0;
    for (auto& f : q.flag) clean = clean && f.load() == 0;
    if (!clean) {
      std::fprintf(stderr, "launch %d: control block not reset\n", L);
      return 1;
    }
  }
  if (g_errors.load()) {
    std::fprintf(stderr, "%ld out-of-order / foreign records\n", g_errors.load());
    return 1;
  }
  std::printf("ok S=%d R=%d workers=%d pairs=%u records=%d launches=%d\n", S, R, W, P, NREC, launches);
  return 0;
}
