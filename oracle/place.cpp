// oracle/place.cpp — TEST INFRASTRUCTURE ONLY (see pem.hpp).
// O6: event-driven Place(b, S, geometry) = Alg 1 under Eq 1 / Eq 2.
#include "pem.hpp"
#include <algorithm>
#include <climits>

namespace pem {

// Eq 1:  T_k = Solo_k * max{ FBR_k + sum_i FBR_i , 1 }.
// Integers (reading Q10): F in ppm, exec = floor(solo * max(F, 10^6) / 10^6), int64.
int64_t exec_us(int64_t solo, int64_t F_ppm) {
  int64_t f = F_ppm < kPpm ? kPpm : F_ppm;
  return solo * f / kPpm;
}

PlaceOut place(const Tables& tb, const std::vector<int>& geom, GpuState& S, int64_t t, int m,
               bool strict, int max_live, Accum* acc, int64_t H, int depth) {
  PlaceOut o;

  // Residents that ended at or before t can never be co-runners or memory holders again.
  std::vector<Resident> kept;
  for (const Resident& r : S.res)
    if (r.end > t) kept.push_back(r);
  S.res = kept;

  // Live bound (reading Q39): max_live batches with end > t already -> overflow drop.
  if ((int)S.res.size() >= max_live) {
    o.dropped = 3;
    return o;
  }

  const int k = (int)geom.size();
  const int32_t q = tb.mem[m];

  // (a) earliest start on each slice: FIFO after the slice's last start, then the first
  //     instant at which concurrent footprints + q fit the slice memory (reading Q13).
  // (b) completion with Eq 1 evaluated at that start instant (reading Q8, Q9).
  for (int s = 0; s < k; ++s) {
    const int p = geom[s];
    const int32_t Ms = tb.cap(p);
    if (q > Ms) continue;  // the batch can never fit this slice
    o.feasible[s] = true;

    const int64_t t0 = std::max(t, S.last_start[s]);
    std::vector<const Resident*> L;  // residents of slice s still holding memory after t0
    for (const Resident& r : S.res)
      if (r.slice == s && r.end > t0) L.push_back(&r);

    int64_t used = 0;
    for (const Resident* r : L) used += r->mem;

    int64_t start;
    if (used + q <= Ms) {
      start = t0;
    } else {
      // smallest release time end_j after which the batch fits
      start = LLONG_MAX;
      for (const Resident* rj : L) {
        int64_t remaining = 0;
        for (const Resident* ri : L)
          if (ri->end > rj->end) remaining += ri->mem;
        if (remaining + q <= Ms && rj->end < start) start = rj->end;
      }
    }

    // Eq 1's sum over the jobs co-located on the slice at the start instant.
    int64_t F = tb.fbr_at(m, p);
    for (const Resident& r : S.res)
      if (r.slice == s && r.start <= start && start < r.end) F += tb.fbr_at(r.model, p);

    o.s_start[s] = start;
    o.s_F[s] = F;
    o.s_end[s] = start + exec_us(tb.solo_at(m, p), F);
  }

  int chosen = -1;
  if (strict) {
    // Alg 1 lines 1-8: BE memory from the reordering module (reading Q5) tags the
    // slices in ascending order; tag = min(1, BE_mem/avail) and BE_mem -= avail (reading Q4:
    // avail = slice capacity).  choose_strict_slice keeps slices with tag < 1.
    int64_t be_mem = 0;
    for (const Resident& r : S.res)
      if (!r.strict) be_mem += r.mem;
    int64_t R = be_mem;
    for (int s = 0; s < k; ++s) {
      const int32_t Ms = tb.cap(geom[s]);
      if (depth >= 0) {  // N4b (R28): an enumerated BE-reserve depth replaces the tags
        o.eligible[s] = s >= depth;
      } else if (R >= Ms) {  // tag_value == 1: completely occupied by BE
        o.eligible[s] = false;
        R -= Ms;
      } else {        // tag_value < 1
        o.eligible[s] = true;
        R = 0;
      }
    }
    // least slowdown factor eta (Eq 2) == least predicted completion (reading Q11);
    // ties -> larger profile (strict gets the large slice), then lower position.
    for (int pass = 0; pass < 2 && chosen < 0; ++pass) {
      for (int s = 0; s < k; ++s) {
        if (!o.feasible[s]) continue;
        if (pass == 0 && !o.eligible[s]) continue;  // pass 1 = fallback to every fitting slice (Q6)
        if (chosen < 0) { chosen = s; continue; }
        const int p = geom[s], pc = geom[chosen];
        if (o.s_end[s] < o.s_end[chosen] ||
            (o.s_end[s] == o.s_end[chosen] && p > pc))
          chosen = s;  // equal (c, p) keeps the lower position
      }
    }
  } else {
    // choose_best_effort_slice: first-fit bin packing in ascending slice order —
    // the first slice where the batch starts now; otherwise the earliest start (reading Q12).
    for (int s = 0; s < k; ++s)
      if (o.feasible[s] && o.s_start[s] == t) { chosen = s; break; }
    if (chosen < 0)
      for (int s = 0; s < k; ++s)
        if (o.feasible[s] && (chosen < 0 || o.s_start[s] < o.s_start[chosen])) chosen = s;
  }

  if (chosen < 0) {  // no slice can ever hold the footprint: placement drop (reading Q32)
    o.dropped = 2;
    return o;
  }

  // schedule(batch, chosen_slice) (Alg 1 line 15, both branches, reading Q7)
  o.slice = chosen;
  o.start = o.s_start[chosen];
  o.end = o.s_end[chosen];
  Resident nr;
  nr.start = o.start;
  nr.end = o.end;
  nr.mem = q;
  nr.slice = chosen;
  nr.model = m;
  nr.strict = strict;
  S.res.push_back(nr);
  S.last_start[chosen] = o.start;

  if (acc) {
    // busy time of the slice instance as a union of intervals (starts are non-decreasing per
    // slice), clipped to [0, H); memory-time of the batch clipped to [0, H) (reading Q29).
    const int p = geom[chosen];
    int64_t lo = std::max(o.start, S.busy_until[chosen]);
    int64_t hi = std::min(o.end, H);
    if (hi > lo) {
      acc->busy_w += (int64_t)kCompute[p] * (hi - lo);
      S.busy_us[chosen] += hi - lo;
    }
    int64_t mhi = std::min(o.end, H);
    if (mhi > o.start) acc->mem_num += (int64_t)q * (mhi - o.start);
  }
  S.busy_until[chosen] = std::max(S.busy_until[chosen], o.end);
  return o;
}

}  // namespace pem
