// oracle/geom.cpp — TEST INFRASTRUCTURE ONLY (see pem.hpp).
// O2: the candidate geometry set.  The paper defines a geometry as "any configuration with a
// combination of profiles" and gives T2 but no list (reading Q2).  The
// oracle enumerates by NVIDIA's A100-40GB MIG *placement* rules (memory-slice intervals, from the
// MIG user guide the paper cites as [24], P:L542 — not in the paper's text): a geometry is a set
// of pairwise disjoint placements.  The CUDA library enumerates by T2 sum constraints instead;
// tests check the two agree.
#include "pem.hpp"
#include <algorithm>
#include <set>

namespace pem {

namespace {
struct Placement { int profile, first, size; };  // occupies memory slices [first, first+size)

std::vector<Placement> a100_placements() {
  std::vector<Placement> v;
  for (int s = 0; s <= 6; ++s) v.push_back({0, s, 1});            // 1g.5gb  at 0..6
  for (int s : {0, 2, 4}) v.push_back({1, s, 2});                 // 2g.10gb at 0,2,4
  for (int s : {0, 4}) v.push_back({2, s, 4});                    // 3g.20gb at 0,4
  v.push_back({3, 0, 4});                                         // 4g.20gb at 0
  v.push_back({4, 0, 8});                                         // 7g.40gb at 0
  return v;
}

using Counts = std::vector<int>;  // count per profile 1g..7g

bool contains_strictly(const Counts& big, const Counts& small) {
  bool ge = true, ne = false;
  for (int p = 0; p < kProfiles; ++p) {
    if (big[p] < small[p]) ge = false;
    if (big[p] != small[p]) ne = true;
  }
  return ge && ne;
}
}  // namespace

std::vector<std::vector<int>> enumerate_geometries(bool all37, GeomStats* stats) {
  const std::vector<Placement> P = a100_placements();
  const int n = (int)P.size();
  std::set<Counts> feasible, placement_maximal;
  int maximal_placements = 0;
  for (int mask = 1; mask < (1 << n); ++mask) {
    unsigned occupied = 0;
    bool ok = true;
    for (int i = 0; i < n && ok; ++i) {
      if (!(mask >> i & 1)) continue;
      unsigned bits = ((1u << P[i].size) - 1u) << P[i].first;
      if (occupied & bits) ok = false;
      occupied |= bits;
    }
    if (!ok) continue;
    Counts c(kProfiles, 0);
    for (int i = 0; i < n; ++i)
      if (mask >> i & 1) c[P[i].profile]++;
    feasible.insert(c);
    bool maximal = true;  // no further placement fits the free memory slices
    for (int i = 0; i < n && maximal; ++i) {
      if (mask >> i & 1) continue;
      unsigned bits = ((1u << P[i].size) - 1u) << P[i].first;
      if (!(occupied & bits)) maximal = false;
    }
    if (maximal) {
      maximal_placements++;
      placement_maximal.insert(c);
    }
  }
  std::vector<Counts> chosen;
  int multiset_maximal = 0;
  for (const Counts& a : feasible) {
    bool maximal = true;
    for (const Counts& b : feasible)
      if (contains_strictly(b, a)) maximal = false;
    if (maximal) multiset_maximal++;
    if (all37 || maximal) chosen.push_back(a);
  }
  if (stats) {
    stats->feasible = (int)feasible.size();
    stats->maximal_placements = maximal_placements;
    stats->placement_maximal_multisets = (int)placement_maximal.size();
    stats->multiset_maximal = multiset_maximal;
  }
  // canonical order: (c7g, c4g, c3g, c2g, c1g) descending lexicographically
  std::sort(chosen.begin(), chosen.end(), [](const Counts& a, const Counts& b) {
    for (int p = kProfiles - 1; p >= 0; --p)
      if (a[p] != b[p]) return a[p] > b[p];
    return false;
  });
  std::vector<std::vector<int>> out;
  for (const Counts& c : chosen) {
    std::vector<int> g;  // slice positions list profiles ascending
    for (int p = 0; p < kProfiles; ++p)
      for (int i = 0; i < c[p]; ++i) g.push_back(p);
    out.push_back(g);
  }
  return out;
}

}  // namespace pem
