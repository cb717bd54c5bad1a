// pem_device.cuh — device-side building blocks of the B200 PROTEAN epoch engine (sm_100a).
//
// The lane-level Place() is Alg 1 under the slowdown model Eq 1 / Eq 2 (P:L191,
// P:L208) in exact integers; every reading it relies on is listed in DESIGN.md §3.  One lane
// owns one resident list (the actual GPU state, or one candidate geometry replayed from idle)
// and walks the GPU-epoch's batches; lanes of the same simulated GPU walk the same batch list in
// lock-step, so batch descriptors are warp-broadcast loads.
#pragma once
#include <stdint.h>
#include "../../include/protean.h"

namespace pemgpu {

constexpr int kNProf = 5;
constexpr int kMaxSl = 7;
constexpr int64_t kPpm = 1000000;
constexpr uint32_t kNoGeom = 0xFF;
constexpr int kNB = PROTEAN_NBUCKETS;

constexpr uint32_t kMemMask = 0xFFFFFFu;  // packed resident words: footprint in the low 24 bits

// T2 — memory eighths and compute sevenths per profile (1g,2g,3g,4g,7g); a slice's
// memory is gpu_mem * eighths / 8 (A100-40GB: 5120/10240/20480/20480/40960 MiB; N4c: the same
// structure over the H100 / H200 / B200 memories), staged per handle in Tab::cap.
__host__ __device__ __forceinline__ int32_t prof_eighths(int p) {
  return p == 0 ? 1 : p == 1 ? 2 : p == 4 ? 8 : 4;
}
__host__ __device__ __forceinline__ int32_t prof_compute(int p) {
  return p == 0 ? 1 : p == 1 ? 2 : p == 2 ? 3 : p == 3 ? 4 : 7;
}

// Table block layout (int32 words), identical on host and device; staged into smem per CTA.
struct TabLayout {
  int M, G;
  int o_solo, o_fbr, o_mem, o_bsz, o_slo, o_tmo;  // [M*5],[M*5],[M],[M],[M],[M]
  int o_gprof;   // G*8 bytes packed into G*2 words: profile ids ascending, 0xFF padded
  int o_gn;      // G words: slice count
  int o_gpref;   // G*8 words: prefix capacity including slice s (tag walk, Alg 1 lines 1-8)
  int o_cap;     // 5 words: slice memory per profile (MiB), N4c
  int words;
  __host__ __device__ void init(int m, int g) {
    M = m; G = g;
    o_solo = 0; o_fbr = o_solo + 5 * M; o_mem = o_fbr + 5 * M; o_bsz = o_mem + M;
    o_slo = o_bsz + M; o_tmo = o_slo + M; o_gprof = o_tmo + M; o_gn = o_gprof + 2 * G;
    o_gpref = o_gn + G; o_cap = o_gpref + 8 * G; words = o_cap + 8;
  }
};

struct Tab {  // smem views
  int M, G;
  const int32_t *solo, *fbr, *mem, *bsz, *slo, *tmo, *gn, *gpref, *cap;
  const uint8_t *gprof;
  __device__ void bind(const int32_t* w, const TabLayout& L) {
    M = L.M; G = L.G;
    solo = w + L.o_solo; fbr = w + L.o_fbr; mem = w + L.o_mem; bsz = w + L.o_bsz;
    slo = w + L.o_slo; tmo = w + L.o_tmo; gn = w + L.o_gn; gpref = w + L.o_gpref; cap = w + L.o_cap;
    gprof = reinterpret_cast<const uint8_t*>(w + L.o_gprof);
  }
};

// A resident list: protean_resident rows (24 B), contiguous per lane.
// meta word at byte 20 = slice | model << 8 | strict << 16.
struct Rows {
  protean_resident* r;
  __device__ __forceinline__ int64_t st(int i) const { return r[i].start_us; }
  __device__ __forceinline__ int64_t en(int i) const { return r[i].end_us; }
  __device__ __forceinline__ int32_t mem(int i) const { return r[i].mem_mib; }
  __device__ __forceinline__ uint32_t meta(int i) const {
    return *reinterpret_cast<const uint32_t*>(&r[i].slice);
  }
};

struct PlaceRes {
  int64_t start, end;
  int slice;
  int dropped;  // 0 placed, 2 no slice holds the footprint, 3 max_live overflow
};

// Eq 1 in integers: exec = floor(solo * max(F, 10^6) / 10^6) (reading Q10).  Both
// factors are non-negative and F <= (max_live + 1) * 10^6 < 2^32 (every FBR <= 10^6), so the
// product fits an unsigned 64-bit word and the division by the constant is the unsigned
// multiply-high sequence (8 SASS instructions instead of 15 for the signed one).
__device__ __forceinline__ int64_t exec_time(int32_t solo, int64_t F) {
  const uint32_t f = F < kPpm ? (uint32_t)kPpm : (uint32_t)F;
  return (int64_t)(((uint64_t)(uint32_t)solo * (uint64_t)f) / 1000000ull);
}

// Rare path of Place for one slice (memory wait, or a resident starting after t0): the plain
// definition of O6(a)/(b) by explicit scans.  Kept out of line to keep the hot loop small.
static __device__ __noinline__ void place_slow_slice(const Tab& T, const uint8_t* gp, Rows L, int n, int s,
                                              int p, int64_t t0, int32_t q, int m, int64_t* start_out,
                                              int64_t* F_out) {
  const int32_t Ms = T.cap[p];
  int64_t used = 0, e = INT64_MAX;
  for (int i = 0; i < n; ++i)
    if ((int)(L.meta(i) & 0xFF) == s && L.en(i) > t0) {
      used += L.mem(i);
      e = L.en(i) < e ? L.en(i) : e;
    }
  int64_t start = t0;
  if (used + q > Ms) {  // earliest release that makes the batch fit, releases in ascending order
    for (;;) {
      int64_t rem = 0, nxt = INT64_MAX;
      for (int j = 0; j < n; ++j)
        if ((int)(L.meta(j) & 0xFF) == s && L.en(j) > e) {
          rem += L.mem(j);
          nxt = L.en(j) < nxt ? L.en(j) : nxt;
        }
      if (rem + q <= Ms) break;
      e = nxt;
    }
    start = e;
  }
  int64_t F = T.fbr[m * kNProf + p];
  for (int i = 0; i < n; ++i) {
    const uint32_t mt = L.meta(i);
    if ((int)(mt & 0xFF) == s && L.st(i) <= start && start < L.en(i))
      F += T.fbr[((mt >> 8) & 0xFF) * kNProf + gp[s]];
  }
  *start_out = start;
  *F_out = F;
}

// Place one batch (model m, class strict, ready t) on geometry `geom` over list L (n rows).
// ls[] = last start per slice position (FIFO).  One pass over the residents accumulates, per
// slice, the memory still held after t0_s = max(t, last_start_s) and the FBR of those residents;
// since every resident of a slice started at or before its last start (FIFO), they are exactly
// Eq 1's co-runners at t0_s.  The rare memory-wait case takes place_slow_slice().
// depth (N4b, reading R28): -1 = Alg 1's BE tags; d >= 0 = the d smallest slices reserved for BE.
__device__ __forceinline__ PlaceRes place_lane(const Tab& T, int geom, Rows L, int& n,
                                               int64_t (&ls)[kMaxSl], int64_t t, int m,
                                               bool strict, int max_live, int depth = -1) {
  PlaceRes o;
  o.dropped = 0;
  o.slice = -1;
  o.start = o.end = 0;
  const uint8_t* gp = T.gprof + geom * 8;
  int64_t t0[kMaxSl];
  int32_t used[kMaxSl], fs[kMaxSl];
  uint32_t fut = 0;
#pragma unroll
  for (int x = 0; x < kMaxSl; ++x) {
    t0[x] = t > ls[x] ? t : ls[x];
    used[x] = 0;
    fs[x] = 0;
  }
  int32_t be_mem = 0;
  int k = 0;
  for (int i = 0; i < n; ++i) {
    const protean_resident r = L.r[i];
    if (r.end_us <= t) continue;  // ended: can never matter again (stable compaction)
    if (k != i) L.r[k] = r;
    ++k;
    const int s = r.slice;
    if (!r.strict) be_mem += r.mem_mib;
    const int32_t f = T.fbr[r.model * kNProf + gp[s]];
#pragma unroll
    for (int x = 0; x < kMaxSl; ++x) {
      if (x == s && r.end_us > t0[x]) {
        used[x] += r.mem_mib;
        fs[x] += f;
        if (r.start_us > t0[x]) fut |= 1u << x;
      }
    }
  }
  n = k;
  if (n >= max_live) {  // reading Q39
    o.dropped = 3;
    return o;
  }
  const int32_t q = T.mem[m];
  const int ns = T.gn[geom];
  uint64_t best = ~0ull;
  int64_t bstart = 0, bend = 0;
#pragma unroll
  for (int x = 0; x < kMaxSl; ++x) {
    if (x < ns) {
      const int p = gp[x];
      const int32_t Ms = T.cap[p];
      if (q <= Ms) {
        int64_t start, F;
        if (used[x] + q <= Ms && !((fut >> x) & 1)) {
          start = t0[x];
          F = (int64_t)T.fbr[m * kNProf + p] + fs[x];
        } else {
          place_slow_slice(T, gp, L, n, x, p, t0[x], q, m, &start, &F);
        }
        const int64_t c = start + exec_time(T.solo[m * kNProf + p], F);
        uint64_t key;
        if (strict) {  // choose_strict_slice: tag < 1, least eta == least completion (Q11)
          const bool full = depth >= 0 ? x < depth : be_mem >= T.gpref[geom * 8 + x];
          const uint64_t inelig = full ? (1ull << 62) : 0ull;
          key = inelig | ((uint64_t)c << 6) | ((uint64_t)(4 - p) << 3) | (uint64_t)x;
        } else {       // choose_best_effort_slice: first fit, else earliest start (Q12)
          key = ((uint64_t)start << 3) | (uint64_t)x;
        }
        if (key < best) {
          best = key;
          bstart = start;
          bend = c;
        }
      }
    }
  }
  if (best == ~0ull) {
    o.dropped = 2;
    return o;
  }
  const int s = (int)(best & 7);
  protean_resident nr;
  nr.start_us = bstart;
  nr.end_us = bend;
  nr.mem_mib = q;
  nr.slice = (uint8_t)s;
  nr.model = (uint8_t)m;
  nr.strict = strict ? 1 : 0;
  nr.pad = 0;
  L.r[n] = nr;
  ++n;
#pragma unroll
  for (int x = 0; x < kMaxSl; ++x)
    if (x == s) ls[x] = bstart;
  o.slice = s;
  o.start = bstart;
  o.end = bend;
  return o;
}

// O7 log-linear latency bucket (reading Q30).
__device__ __forceinline__ int lat_bucket(int64_t x) {
  uint64_t v = x < 0 ? 0 : (uint64_t)x;
  if (v > 0xFFFFFFFFull) v = 0xFFFFFFFFull;
  if (v < 128) return (int)v;
  const int k = 31 - __clz((unsigned)v);
  return 128 + (k - 7) * 128 + (int)((v >> (k - 7)) & 127);
}

__host__ __device__ __forceinline__ uint64_t bucket_lower_edge(int b) {
  if (b < 128) return (uint64_t)b;
  const int k = 7 + (b - 128) / 128;
  return (uint64_t)(128 + (b - 128) % 128) << (k - 7);
}

// O8 key (reading Q20)
__device__ __forceinline__ int64_t make_key(int64_t misses, int64_t tail, int tag) {
  const int64_t mm = (1LL << 23) - 1;
  if (misses > mm) misses = mm;
  if (tail > 0xFFFFFFFFLL) tail = 0xFFFFFFFFLL;
  return (misses << 40) | (tail << 8) | (int64_t)tag;
}

__device__ __forceinline__ uint64_t smix(uint64_t x) {
  x += 0x9E3779B97F4A7C15ull;
  x = (x ^ (x >> 30)) * 0xBF58476D1CE4E5B9ull;
  x = (x ^ (x >> 27)) * 0x94D049BB133111EBull;
  return x ^ (x >> 31);
}

// #{members a with c - a <= slo} over a sorted ascending member list (binary search).
__device__ __forceinline__ int hits_sorted(const uint32_t* a, int n, int64_t c, int64_t slo) {
  const int64_t lo_a = c - slo;  // need a >= c - slo
  int lo = 0, hi = n;
  while (lo < hi) {
    int mid = (lo + hi) >> 1;
    if ((int64_t)a[mid] >= lo_a) hi = mid; else lo = mid + 1;
  }
  return n - lo;
}

}  // namespace pemgpu
