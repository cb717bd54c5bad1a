// oracle/metrics.cpp — TEST INFRASTRUCTURE ONLY (see pem.hpp).
// O7 latency histogram and O12 percentiles (reading Q30), O11 VM draws (reading Q28).
#include "pem.hpp"

namespace pem {

// Log-linear bucket: x < 128 -> x; else with k = floor(log2 x),
// bucket = 128 + (k-7)*128 + ((x >> (k-7)) & 127).  x saturates at 2^32-1 -> last bucket 3327.
int bucket_of(uint64_t x) {
  if (x > kSat32) x = kSat32;
  if (x < 128) return (int)x;
  int k = 0;
  while ((x >> (k + 1)) != 0) ++k;  // floor(log2 x), written out
  return 128 + (k - 7) * 128 + (int)((x >> (k - 7)) & 127);
}

uint64_t bucket_lower(int b) {
  if (b < 128) return (uint64_t)b;
  int k = 7 + (b - 128) / 128;
  return (uint64_t)(128 + (b - 128) % 128) << (k - 7);
}

// Nearest rank: rank = ceil(q*n/100); report the lower edge of the first bucket whose
// cumulative count reaches rank; 0 when the histogram is empty.
uint64_t percentile(const uint32_t* hist, int q_percent) {
  uint64_t n = 0;
  for (int b = 0; b < kBuckets; ++b) n += hist[b];
  if (n == 0) return 0;
  uint64_t rank = (q_percent * n + 99) / 100;
  uint64_t cum = 0;
  for (int b = 0; b < kBuckets; ++b) {
    cum += hist[b];
    if (cum >= rank) return bucket_lower(b);
  }
  return bucket_lower(kBuckets - 1);
}

uint64_t splitmix64(uint64_t x) {
  x += 0x9E3779B97F4A7C15ull;
  x = (x ^ (x >> 30)) * 0xBF58476D1CE4E5B9ull;
  x = (x ^ (x >> 27)) * 0x94D049BB133111EBull;
  return x ^ (x >> 31);
}

// draw(d) = splitmix64(seed ^ splitmix64((replica<<32) ^ (node<<20) ^ (k<<2) ^ d)) >> 11
uint64_t vm_draw(uint64_t seed, uint64_t replica, uint64_t node, uint64_t k, uint64_t d) {
  return splitmix64(seed ^ splitmix64((replica << 32) ^ (node << 20) ^ (k << 2) ^ d)) >> 11;
}

int64_t make_key(int64_t misses, int64_t tail, int tag) {
  const int64_t mmax = (1LL << 23) - 1;
  if (misses > mmax) misses = mmax;
  if (tail > (int64_t)kSat32) tail = (int64_t)kSat32;
  return (misses << 40) | (tail << 8) | (int64_t)tag;
}

}  // namespace pem
