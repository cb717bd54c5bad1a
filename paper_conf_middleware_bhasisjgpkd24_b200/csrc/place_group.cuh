// place_group.cuh — the lane-per-slice Place() of the epoch engine (Alg 1, under
// Eq 1 / Eq 2, P:L191 / P:L208; readings Q4-Q13, Q39 of DESIGN.md), shared by the fused replay
// (replay.cu) and protean_score_epoch (score.cu).  A placement unit is a lane group of Z lanes (a
// power of two >= the geometry's slice count); lane s of the group owns slice position s and its
// resident list; group shuffles give the GPU-wide live count, the BE memory of the tag walk and the
// min-loc of the slice keys.
#pragma once
#include <stdint.h>
#include "pem_device.cuh"

namespace pemgpu {
namespace pg {

// Per-lane resident list, interleaved across lanes (entry i of lane l at i*stride + l) so that a
// warp walking its lists in lock-step issues coalesced loads.  mm = mem | model << 24 | strict << 30
// (footprints < 2^24 MiB: every MIG table of N4c fits).
struct LaneList {
  int64_t* st;
  int64_t* en;
  uint32_t* mm;
  int stride;
  __device__ __forceinline__ int64_t S(int i) const { return st[i * stride]; }
  __device__ __forceinline__ int64_t E(int i) const { return en[i * stride]; }
  __device__ __forceinline__ uint32_t M(int i) const { return mm[i * stride]; }
  __device__ __forceinline__ void put(int i, int64_t s, int64_t e, uint32_t m) const {
    st[i * stride] = s;
    en[i * stride] = e;
    mm[i * stride] = m;
  }
};

__device__ __forceinline__ int hits_in(const uint32_t* a, int n, int64_t end, int64_t slo) {
  const int64_t need = end - slo;  // c - a <= slo  <=>  a >= c - slo
  int lo = 0, hi = n;
#pragma unroll 1
  while (lo < hi) {
    const int mid = (lo + hi) >> 1;
    if ((int64_t)a[mid] >= need) hi = mid; else lo = mid + 1;
  }
  return n - lo;
}

// Sum / min over the aligned lane group of size Z (1..8) containing this lane.
__device__ __forceinline__ int group_sum32(int v, int Z) {
#pragma unroll
  for (int d = 1; d < 8; d <<= 1) {
    const int o = __shfl_xor_sync(0xffffffffu, v, d);
    if (d < Z) v += o;
  }
  return v;
}
__device__ __forceinline__ int64_t group_sum(int64_t v, int Z) {
#pragma unroll
  for (int d = 1; d < 8; d <<= 1) {
    const int64_t o = __shfl_xor_sync(0xffffffffu, v, d);
    if (d < Z) v += o;
  }
  return v;
}
__device__ __forceinline__ uint64_t group_min(uint64_t v, int Z) {
#pragma unroll
  for (int d = 1; d < 8; d <<= 1) {
    const uint64_t o = __shfl_xor_sync(0xffffffffu, v, d);
    if (d < Z && o < v) v = o;
  }
  return v;
}

// The slice lane's own list: memory wait and Eq 1 co-runner sum by their plain definitions
// (rare: only when the batch does not fit the slice at t0, or a resident starts after t0).
static __device__ __noinline__ void slice_slow(const LaneList& L, int n, int64_t t0, int32_t q, int32_t Ms,
                                        const int32_t* fbr_p, int64_t own_f, int64_t* start_out,
                                        int64_t* F_out) {
  // one pass per tried start time: memory still held, the next release, and Eq 1's co-runner sum
  // at that time (residents with S <= start < E), so the accepted pass already holds F
  int64_t used = 0, e = INT64_MAX, F = own_f;  // at t0: memory held after t0, earliest release
#pragma unroll 1
  for (int i = 0; i < n; ++i) {
    const int64_t ei = L.E(i);
    if (ei > t0) {
      const uint32_t mi = L.M(i);
      used += mi & kMemMask;
      e = ei < e ? ei : e;
      if (L.S(i) <= t0) F += fbr_p[((mi >> 24) & 63) * kNProf];
    }
  }
  int64_t start = t0;
  if (used + q > Ms) {
    // the earliest release e after which the footprints still held (ends > e) leave room: the
    // held memory only shrinks as e grows, so releases are tried in ascending order and the first
    // that fits is the minimum of the plain definition (each pass also finds the next release)
#pragma unroll 1
    for (;;) {
      int64_t rem = 0, nxt = INT64_MAX, Fe = own_f;
#pragma unroll 1
      for (int k = 0; k < n; ++k) {
        const int64_t ek = L.E(k);
        if (ek > e) {
          const uint32_t mk = L.M(k);
          rem += mk & kMemMask;
          nxt = ek < nxt ? ek : nxt;
          if (L.S(k) <= e) Fe += fbr_p[((mk >> 24) & 63) * kNProf];
        }
      }
      if (rem + q <= Ms) {  // always by the last release (q <= Ms)
        F = Fe;
        break;
      }
      e = nxt;
    }
    start = e;
  }
  *start_out = start;
  *F_out = F;
}

struct SliceOut {
  uint64_t kmin;     // group min key (~0 = no feasible slice or overflow)
  bool drop_overflow;
};

// One Place() (Alg 1) of a batch on one lane group: each lane is one slice position s of
// geometry j; the lane keeps its own slice's resident list.  Returns the group outcome; this
// lane's own [start, end) candidate in *my_start / *my_end.
struct SliceLane {        // per-lane constants of one placement unit
  const int32_t* fbr_p;   // fbr[model][p] = fbr_p[model * 5]
  const int32_t* solo_p;  // solo[model][p] = solo_p[model * 5]
  int32_t Ms, pref;       // slice memory; capacity of slices 0..s (tag walk, Alg 1 lines 1-8)
  int s, p, Z;
};

template <int kPL>
__device__ __forceinline__ SliceOut place_group(const Tab& T, bool active, const SliceLane& K,
                                                const LaneList& L, int& n, int64_t& ls,
                                                int64_t t, int m, bool strict, int max_live,
                                                int64_t* my_start, int64_t* my_end) {
  const int64_t t0 = t > ls ? t : ls;
  const int32_t* fbr_p = K.fbr_p;
  const int Z = K.Z, s = K.s, p = K.p;
  int32_t used = 0, be = 0;
  int64_t fs = 0;
  bool fut = false;
  if (active) {
    // residents in groups of kPL: the group's loads are issued together (the compaction only
    // writes indices below the group, so no store can clobber an element not yet loaded)
    // kPL = 1 for the many-replica launch (its lists are short, and a wider group costs it
    // registers: measured 181 -> 191 ms); 4 for few-replica launches of long-list workloads
    // (Mix-B-shaped 1 h replay: 485 -> 418 ms per 600 s)
    int k = 0;
#pragma unroll 1
    for (int i0 = 0; i0 < n; i0 += kPL) {
      int64_t e_[kPL], s_[kPL];
      uint32_t m_[kPL];
#pragma unroll
      for (int u = 0; u < kPL; ++u) {
        const int i = i0 + u < n ? i0 + u : i0;
        e_[u] = L.E(i);
        s_[u] = L.S(i);
        m_[u] = L.M(i);
      }
#pragma unroll
      for (int u = 0; u < kPL; ++u) {
        const int i = i0 + u;
        const int64_t ei = e_[u];
        if (i >= n || ei <= t) continue;  // ended: can never matter again (stable compaction)
        const int64_t si = s_[u];
        const uint32_t mi = m_[u];
        if (k != i) L.put(k, si, ei, mi);
        ++k;
        if (!((mi >> 30) & 1)) be += mi & kMemMask;
        if (ei > t0) {
          used += mi & kMemMask;
          fs += fbr_p[((mi >> 24) & 63) * kNProf];
          fut |= si > t0;
        }
      }
    }
    n = k;
  }
  const int live = group_sum32(active ? n : 0, Z);
  const int be_mem = group_sum32(be, Z);
  SliceOut o;
  o.drop_overflow = live >= max_live;
  uint64_t key = ~0ull;
  int64_t start = 0, c = 0;
  const int32_t q = T.mem[m];
  const int32_t Ms = K.Ms;
  if (active && !o.drop_overflow && q <= Ms) {
    int64_t F;
    const int64_t own_f = fbr_p[m * kNProf];
    if (used + q <= Ms && !fut) {
      start = t0;
      F = own_f + fs;
    } else {
      slice_slow(L, n, t0, q, Ms, fbr_p, own_f, &start, &F);
    }
    c = start + exec_time(K.solo_p[m * kNProf], F);
    if (strict) {  // choose_strict_slice: tag < 1 (Alg 1 lines 1-8), least eta == least completion
      const uint64_t inelig = (be_mem >= K.pref) ? (1ull << 62) : 0ull;
      key = inelig | ((uint64_t)c << 6) | ((uint64_t)(4 - p) << 3) | (uint64_t)s;
    } else {       // choose_best_effort_slice: first fit, else earliest start (reading Q12)
      key = ((uint64_t)start << 3) | (uint64_t)s;
    }
  }
  o.kmin = group_min(key, Z);
  *my_start = start;
  *my_end = c;
  if (o.kmin != ~0ull && key == o.kmin) {  // schedule(batch, chosen_slice)
    L.put(n, start, c, (uint32_t)q | ((uint32_t)m << 24) | ((uint32_t)(strict ? 1 : 0) << 30));
    ++n;
    ls = start;
  }
  return o;
}


// ---- Sub-lanes: one warp per simulated GPU, lane = sub * 8 + s; the 4 lanes (s, sub = 0..3) share
// slice position s and each keeps a quarter of its resident list (a new resident goes to the
// shortest).  Long lists (overloaded single-replica workloads) are pruned and summed 4 lanes wide;
// the per-slice quantities are reduced over the 4 sub-lanes (xor 8, 16), the GPU-wide live count
// and BE memory over the warp, and the slice min-loc runs within each group of 8 as in
// place_group.  Same results as place_group: every rule of O6 depends on the resident set only.
__device__ __forceinline__ int64_t sub_sum(int64_t v) {
  v += __shfl_xor_sync(0xffffffffu, v, 8);
  return v + __shfl_xor_sync(0xffffffffu, v, 16);
}
__device__ __forceinline__ int64_t sub_min(int64_t v) {
  int64_t o = __shfl_xor_sync(0xffffffffu, v, 8);
  v = o < v ? o : v;
  o = __shfl_xor_sync(0xffffffffu, v, 16);
  return o < v ? o : v;
}
__device__ __forceinline__ int warp_sum32(int v) {
#pragma unroll
  for (int d = 1; d < 32; d <<= 1) v += __shfl_xor_sync(0xffffffffu, v, d);
  return v;
}

template <int kPL>
__device__ __forceinline__ SliceOut place_group_sub(const Tab& T, bool active, const SliceLane& K,
                                                    const LaneList& L, int& n, int64_t& ls,
                                                    int64_t t, int m, bool strict, int max_live,
                                                    int64_t* my_start, int64_t* my_end) {
  const int lane = threadIdx.x & 31, sub = lane >> 3;
  const int64_t t0 = t > ls ? t : ls;
  const int32_t* fbr_p = K.fbr_p;
  const int s = K.s, p = K.p;
  int64_t used = 0, fs = 0;
  int32_t be = 0;
  bool fut = false;
  if (active) {  // prune this lane's quarter of the list (as place_group)
    int k = 0;
#pragma unroll 1
    for (int i0 = 0; i0 < n; i0 += kPL) {
      int64_t e_[kPL], s_[kPL];
      uint32_t m_[kPL];
#pragma unroll
      for (int u = 0; u < kPL; ++u) {
        const int i = i0 + u < n ? i0 + u : i0;
        e_[u] = L.E(i);
        s_[u] = L.S(i);
        m_[u] = L.M(i);
      }
#pragma unroll
      for (int u = 0; u < kPL; ++u) {
        const int i = i0 + u;
        const int64_t ei = e_[u];
        if (i >= n || ei <= t) continue;
        const int64_t si = s_[u];
        const uint32_t mi = m_[u];
        if (k != i) L.put(k, si, ei, mi);
        ++k;
        if (!((mi >> 30) & 1)) be += mi & kMemMask;
        if (ei > t0) {
          used += mi & kMemMask;
          fs += fbr_p[((mi >> 24) & 63) * kNProf];
          fut |= si > t0;
        }
      }
    }
    n = k;
  }
  const int live = warp_sum32(active ? n : 0);
  const int be_mem = warp_sum32(be);
  used = sub_sum(used);
  fs = sub_sum(fs);
  fut = sub_sum(fut ? 1 : 0) != 0;
  SliceOut o;
  o.drop_overflow = live >= max_live;
  uint64_t key = ~0ull;
  int64_t start = 0, c = 0;
  const int32_t q = T.mem[m];
  const int32_t Ms = K.Ms;
  const bool doit = active && !o.drop_overflow && q <= Ms;  // uniform over a slice's 4 lanes
  const int64_t own_f = fbr_p[m * kNProf];
  int64_t F = own_f + fs;
  start = t0;
  bool slow = doit && !(used + q <= Ms && !fut);
  if (__any_sync(0xffffffffu, slow)) {
    // the plain definition over the slice's whole list, 4 lanes wide: the held memory, the next
    // release and Eq 1's co-runner sum at a tried start (first t0, then releases ascending)
    int64_t e = t0;
    bool first = true;
#pragma unroll 1
    for (;;) {
      int64_t rem = 0, nxt = INT64_MAX, Fe = 0;
      if (slow) {
#pragma unroll 1
        for (int k = 0; k < n; ++k) {
          const int64_t ek = L.E(k);
          if (ek > e) {
            const uint32_t mk = L.M(k);
            rem += mk & kMemMask;
            nxt = ek < nxt ? ek : nxt;
            if (L.S(k) <= e) Fe += fbr_p[((mk >> 24) & 63) * kNProf];
          }
        }
      }
      rem = sub_sum(rem);
      nxt = sub_min(nxt);
      Fe = sub_sum(Fe);
      if (slow) {
        if (rem + q <= Ms) {  // always by the last release (q <= Ms)
          start = e;
          F = own_f + Fe;
          slow = false;
        } else {
          e = nxt;
        }
      }
      first = false;
      if (!__any_sync(0xffffffffu, slow)) break;
    }
    (void)first;
  }
  if (doit) {
    c = start + exec_time(K.solo_p[m * kNProf], F);
    if (strict) {  // choose_strict_slice: tag < 1 (Alg 1 lines 1-8), least eta == least completion
      const uint64_t inelig = (be_mem >= K.pref) ? (1ull << 62) : 0ull;
      key = inelig | ((uint64_t)c << 6) | ((uint64_t)(4 - p) << 3) | (uint64_t)s;
    } else {       // choose_best_effort_slice: first fit, else earliest start (reading Q12)
      key = ((uint64_t)start << 3) | (uint64_t)s;
    }
  }
  o.kmin = group_min(key, 8);
  *my_start = start;
  *my_end = c;
  // schedule(batch, chosen_slice): the chosen slice's shortest quarter list (lowest sub on ties)
  const int64_t pick = sub_min(((int64_t)n << 2) | sub);
  const bool chosen = o.kmin != ~0ull && key == o.kmin;
  if (chosen && pick == (((int64_t)n << 2) | sub)) {
    L.put(n, start, c, (uint32_t)q | ((uint32_t)m << 24) | ((uint32_t)(strict ? 1 : 0) << 30));
    ++n;
  }
  if (chosen) ls = start;
  return o;
}

}  // namespace pg
}  // namespace pemgpu
