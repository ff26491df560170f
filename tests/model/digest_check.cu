// digest_check.cu -- host-side check of the Inter-Group record digest (TEST
// INFRASTRUCTURE; reading R-C-Q2): rec_digest from
// rmt_device.cuh must change whenever ANY ONE word of (key, stored words)
// changes -- in particular every single-bit flip -- and a lane that stores
// nothing must get the compile-time constant rec_digest_none.  Exhaustive over
// the 32 bits of every word for random records, plus random multi-bit changes
// confined to one word.
//   nvcc -std=c++17 -I include -I <csrc> digest_check.cu -o digest_check && ./digest_check
#include <cstdio>
#include <random>

#include "rmt_device.cuh"

template <int NW>
static int check(std::mt19937& g, int records) {
  int bad = 0;
  for (int r = 0; r < records; ++r) {
    unsigned key = g(), mask = (g() & ((1u << NW) - 1u)) | 1u;
    unsigned v[NW];
    for (int k = 0; k < NW; ++k) v[k] = g();
    const unsigned h = rmt::rec_digest<NW>(key, mask, v);
    for (int b = 0; b < 32; ++b) {  // the key
      if (rmt::rec_digest<NW>(key ^ (1u << b), mask, v) == h) ++bad;
    }
    for (int k = 0; k < NW; ++k) {
      if (!((mask >> k) & 1u)) {  // an unstored word is not compared
        unsigned w[NW];
        for (int q = 0; q < NW; ++q) w[q] = v[q];
        w[k] ^= g() | 1u;
        if (rmt::rec_digest<NW>(key, mask, w) != h) ++bad;
        continue;
      }
      for (int b = 0; b < 32; ++b) {  // every single-bit flip of a stored word
        unsigned w[NW];
        for (int q = 0; q < NW; ++q) w[q] = v[q];
        w[k] ^= 1u << b;
        if (rmt::rec_digest<NW>(key, mask, w) == h) ++bad;
      }
      for (int t = 0; t < 64; ++t) {  // any change confined to that word
        unsigned w[NW];
        for (int q = 0; q < NW; ++q) w[q] = v[q];
        const unsigned d = g();
        if (d == 0u) continue;
        w[k] ^= d;
        if (rmt::rec_digest<NW>(key, mask, w) == h) ++bad;
      }
    }
    unsigned z[NW] = {};
    if (rmt::rec_digest<NW>(0xFFFFFFFFu, 0u, v) != rmt::rec_digest_none<NW>() ||
        rmt::rec_digest<NW>(0xFFFFFFFFu, 0u, z) != rmt::rec_digest_none<NW>())
      ++bad;
  }
  return bad;
}

int main() {
  std::mt19937 g(12345);
  const int bad = check<1>(g, 3000) + check<2>(g, 3000) + check<4>(g, 3000);
  if (bad) {
    std::printf("digest_check: %d undetected single-word changes\n", bad);
    return 1;
  }
  std::printf("ok\n");
  return 0;
}
