// ring_model.cpp -- CPU model of the inter-group queue protocol (TEST
// INFRASTRUCTURE; SURVEY.md 8(c) row "C-Q inter-group ring"
// "two-tiered locking system", P:693 coherent reads).
//
// Restates, with std::atomic and C++ memory orders, the protocol that
// paper_conf_isca_waddenlgss14_b200/csrc/rmt_device.cuh implements for
// V_INTER (Rep::init / commit / finish), one thread per CTA role (a lane of a
// warp: lanes are independent, each owns one 64-bit word per slot):
//   * tickets from a global counter in start order; pair = t >> 1, even ticket =
//     producer, odd = consumer;
//   * first tier: region = pair % R; both roles wait for turn[region] ==
//     pair / R, the consumer advances it (release) at exit;
//   * second tier, per (region) a ring of S one-word slots; record j lives in
//     slot j % S as ONE 64-bit word (j + 1) << 32 | digest, so a record is
//     published and read with single-copy-atomic accesses and needs no flag,
//     fence or lock: a slot holds 0 (free) or a record;
//   * producer: record j >= S waits until its slot reads 0 (the consumer freed
//     record j - S), then stores the word (relaxed);
//   * consumer: waits until its slot holds marker j + 1, reads the digest,
//     then stores 0 (relaxed; the same address, so coherence orders the free
//     after the read and the producer's next write after the free);
//   * every consumed slot is freed, so a pair leaves its region all-zero; the
//     last finisher resets tickets and turns.
// Workers (the resident CTA slots) take tickets until 2P are gone.  Checks: every
// record is consumed exactly once, in order, with the digest its producer wrote
// (tagged (pair, seq)); every launch finishes (no deadlock) for any S >= 1, any
// R >= 1 and any number of workers >= 2; the control block and every slot are
// zero afterwards.
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
  std::vector<std::atomic<unsigned>> turn;  // R
  std::vector<std::atomic<uint64_t>> slot;  // R * S
  Queue(int S_, int R_) : S(S_), R(R_), turn(R_), slot((size_t)R_ * S_) {
    for (auto& t : turn) t.store(0);
    for (auto& w : slot) w.store(0);
  }
};

static std::atomic<long> g_errors{0};

static void jitter(std::mt19937& rng) {
  unsigned r = rng() % 16;
  if (r == 0) std::this_thread::yield();
  else if (r == 1) for (volatile int i = 0; i < (int)(rng() % 2000); ++i) {}
}

static uint32_t tag(unsigned pair, unsigned seq) { return (pair * 0x9E3779B9u) ^ (seq * 0x85EBCA6Bu) ^ 0x5bd1e995u; }

static void run_role(Queue& q, unsigned t, unsigned nblocks, unsigned nrec, std::mt19937& rng) {
  const unsigned pair = t >> 1;
  const bool consumer = t & 1u;
  const unsigned region = pair % (unsigned)q.R, epoch = pair / (unsigned)q.R;
  while (q.turn[region].load(std::memory_order_acquire) != epoch) std::this_thread::yield();  // region ownership
  for (unsigned j = 0; j < nrec; ++j) {
    jitter(rng);
    std::atomic<uint64_t>& w = q.slot[(size_t)region * q.S + j % (unsigned)q.S];
    if (!consumer) {
      if (j >= (unsigned)q.S)
        while (w.load(std::memory_order_relaxed) != 0) std::this_thread::yield();  // record j - S freed
      w.store((uint64_t)(j + 1) << 32 | tag(pair, j), std::memory_order_relaxed);
    } else {
      uint64_t v;
      while (((v = w.load(std::memory_order_relaxed)) >> 32) != j + 1) std::this_thread::yield();
      if ((uint32_t)v != tag(pair, j)) {
        g_errors.fetch_add(1);
        std::fprintf(stderr, "pair %u record %u: got digest %x\n", pair, j, (unsigned)v);
      }
      w.store(0, std::memory_order_relaxed);  // free (same address: after the read)
    }
  }
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
  const unsigned NREC = (unsigned)atoi(argv[5]);
  const unsigned seed = (unsigned)atoi(argv[6]);
  const int launches = atoi(argv[7]);
  Queue q(S, R);
  for (int L = 0; L < launches; ++L) {
    std::atomic<unsigned> next{0};
    std::vector<std::thread> th;
    for (int w = 0; w < W; ++w) {
      th.emplace_back([&, w]() {
        std::mt19937 rng(seed * 7919u + (unsigned)w * 104729u + (unsigned)L);
        while (true) {
          // a worker (resident CTA slot) starts the next CTA: it takes a ticket first
          if (next.fetch_add(1) >= 2 * P) break;
          const unsigned t = q.ticket.fetch_add(1);
          run_role(q, t, P, NREC, rng);
        }
      });
    }
    for (auto& t : th) t.join();
    bool clean = q.ticket.load() == 0 && q.done.load() == 0;
    for (auto& tr : q.turn) clean = clean && tr.load() == 0;
    for (auto& s : q.slot) clean = clean && s.load() == 0;
    if (!clean) {
      std::fprintf(stderr, "launch %d: control block or a slot not reset\n", L);
      return 1;
    }
  }
  if (g_errors.load()) {
    std::fprintf(stderr, "%ld out-of-order / foreign records\n", g_errors.load());
    return 1;
  }
  std::printf("ok S=%d R=%d workers=%d pairs=%u records=%u launches=%d\n", S, R, W, P, NREC, launches);
  return 0;
}
