// oracle/sweep.cpp — TEST INFRASTRUCTURE ONLY (see pem.hpp).
// N4a: the exhaustive assignment sweep of the paper's "Oracle" scheme ("ideal GPU configurations
// ... multiple offline ... scheduling sweeps").  For one GPU-epoch's batches and every
// candidate geometry j, every assignment of the b batches to the S_j slices (S_j^b of them) is
// scheduled from idle with the slice FORCED (readings R18-R21 of DESIGN.md), scored like a
// candidate of O8 (strict misses, BE tail) and the minimum kept.  Alg 1's greedy choice is one of
// these assignments, so the sweep's key never exceeds the greedy candidate key.
#include "pem.hpp"
#include <algorithm>
#include <climits>

namespace pem {

// One batch scheduled on a GIVEN slice of `geom` (O6 steps (a)-(b) restricted to that slice,
// reading R19): prune, live bound (Q39), footprint fit, FIFO after the slice's last start, memory
// wait (Q13), Eq 1 at the start instant over the slice's co-runners (Q8, Q9, Q10).
PlaceOut place_forced(const Tables& tb, const std::vector<int>& geom, GpuState& S, int64_t t, int m,
                      bool strict, int max_live, int slice) {
  PlaceOut o;
  std::vector<Resident> kept;
  for (const Resident& r : S.res)
    if (r.end > t) kept.push_back(r);
  S.res = kept;
  if ((int)S.res.size() >= max_live) {
    o.dropped = 3;
    return o;
  }
  const int p = geom[slice];
  const int32_t Ms = tb.cap(p);
  const int32_t q = tb.mem[m];
  if (q > Ms) {
    o.dropped = 2;
    return o;
  }
  const int64_t t0 = std::max(t, S.last_start[slice]);
  int64_t used = 0;
  for (const Resident& r : S.res)
    if (r.slice == slice && r.end > t0) used += r.mem;
  int64_t start = t0;
  if (used + q > Ms) {
    start = LLONG_MAX;
    for (const Resident& rj : S.res) {
      if (rj.slice != slice || rj.end <= t0) continue;
      int64_t remaining = 0;
      for (const Resident& ri : S.res)
        if (ri.slice == slice && ri.end > rj.end) remaining += ri.mem;
      if (remaining + q <= Ms && rj.end < start) start = rj.end;
    }
  }
  int64_t F = tb.fbr_at(m, p);
  for (const Resident& r : S.res)
    if (r.slice == slice && r.start <= start && start < r.end) F += tb.fbr_at(r.model, p);
  o.slice = slice;
  o.start = start;
  o.end = start + exec_us(tb.solo_at(m, p), F);
  Resident nr;
  nr.start = o.start;
  nr.end = o.end;
  nr.mem = q;
  nr.slice = slice;
  nr.model = m;
  nr.strict = strict;
  S.res.push_back(nr);
  S.last_start[slice] = o.start;
  return o;
}

// The sweep of one GPU-epoch on geometry j: returns the min key (R20) and its assignment index
// idx = sum_x slice_x * S^x (batch 0 = least significant digit; lowest index among equal keys).
void sweep_gpu(const Tables& tb, int j, int tag, const std::vector<SweepBatch>& bs, int max_live,
               int64_t* key_out, uint64_t* idx_out, uint64_t* n_assign) {
  const std::vector<int>& geom = tb.geoms[j];
  const int S = (int)geom.size();
  const int b = (int)bs.size();
  uint64_t total = 1;
  for (int x = 0; x < b; ++x) total *= (uint64_t)S;
  int64_t best = -1;
  uint64_t best_idx = 0;
  std::vector<int> slice(b);
  for (uint64_t idx = 0; idx < total; ++idx) {
    uint64_t rem = idx;
    for (int x = 0; x < b; ++x) {
      slice[x] = (int)(rem % (uint64_t)S);
      rem /= (uint64_t)S;
    }
    GpuState C;  // idle GPU in geometry j (reading Q19)
    C.geom = j;
    int64_t misses = 0, tail = 0;
    for (int x = 0; x < b; ++x) {
      const SweepBatch& bt = bs[x];
      PlaceOut po = place_forced(tb, geom, C, bt.ready, bt.model, bt.strict, max_live, slice[x]);
      if (bt.strict) {
        if (po.dropped) {
          misses += (int64_t)bt.arr.size();
        } else {
          int64_t hits = 0;
          for (uint32_t a : bt.arr)
            if (po.end - (int64_t)a <= tb.slo[bt.model]) hits++;
          misses += (int64_t)bt.arr.size() - hits;
        }
      } else {
        const int64_t t_b = po.dropped ? (int64_t)kSat32 : po.end - (int64_t)bt.arr[0];
        tail = std::max(tail, t_b);
      }
    }
    const int64_t key = make_key(misses, tail, tag);
    if (best < 0 || key < best) {
      best = key;
      best_idx = idx;
    }
  }
  *key_out = best;
  *idx_out = best_idx;
  *n_assign += total;
}

// N4b: the BE-reserve depth as an enumerated dimension (reading R28).  For geometry j with S_j
// slices, depth d in {auto, 0, 1, ..., S_j - 1} replays the GPU-epoch's batches from idle with
// Alg 1's greedy choice (O6) whose strict eligibility is "position >= d" (auto = the BE tag walk of
// Alg 1 lines 1-8).  keys[1 + d] (keys[0] = auto) is the O8 key; the minimum over (key, auto < 0 <
// 1 < ...) is returned with its depth code (0 = auto, 1 + d).
void sweep_depths(const Tables& tb, int j, int tag, const std::vector<SweepBatch>& bs, int max_live,
                  int64_t* keys /* [8] */, int64_t* best_key, int* best_code, uint64_t* n_eval) {
  const std::vector<int>& geom = tb.geoms[j];
  const int S = (int)geom.size();
  *best_key = -1;
  *best_code = 0;
  for (int code = 0; code < 8; ++code) keys[code] = -1;
  for (int code = 0; code <= S; ++code) {
    GpuState C;  // idle GPU in geometry j (reading Q19)
    C.geom = j;
    int64_t misses = 0, tail = 0;
    for (const SweepBatch& bt : bs) {
      PlaceOut po = place(tb, geom, C, bt.ready, bt.model, bt.strict, max_live, nullptr, INT64_MAX, code - 1);
      if (bt.strict) {
        if (po.dropped) {
          misses += (int64_t)bt.arr.size();
        } else {
          int64_t hits = 0;
          for (uint32_t a : bt.arr)
            if (po.end - (int64_t)a <= tb.slo[bt.model]) hits++;
          misses += (int64_t)bt.arr.size() - hits;
        }
      } else {
        const int64_t t_b = po.dropped ? (int64_t)kSat32 : po.end - (int64_t)bt.arr[0];
        tail = std::max(tail, t_b);
      }
    }
    keys[code] = make_key(misses, tail, tag);
    if (*best_key < 0 || keys[code] < *best_key) {
      *best_key = keys[code];
      *best_code = code;
    }
    *n_eval += 1;
  }
}

}  // namespace pem
