// oracle/tick.cpp — TEST INFRASTRUCTURE ONLY (see pem.hpp).
// A second, independent formulation of O6(a)/(b): advance time one microsecond at a time, keep
// one FIFO queue per slice, retire batches at their end, admit the queue head whenever the
// slice's memory (T2) has room, and freeze Eq 1's execution time from the
// batches running at the admission instant.  The slice of every batch is given (it comes from
// the event-driven Place); this simulator only re-derives start and end times.
#include "pem.hpp"
#include <deque>

namespace pem {

void tick_simulate(const Tables& tb, const std::vector<int>& geom, std::vector<TickBatch>& bs) {
  const int k = (int)geom.size();
  std::vector<std::deque<int>> queue(k);
  std::vector<std::vector<int>> running(k);
  size_t next = 0, admitted = 0;
  int64_t tau = bs.empty() ? 0 : bs[0].t;
  while (admitted < bs.size()) {
    while (next < bs.size() && bs[next].t == tau) {
      queue[bs[next].slice].push_back((int)next);
      ++next;
    }
    for (int s = 0; s < k; ++s) {
      const int p = geom[s];
      std::vector<int> still;
      for (int i : running[s])
        if (bs[i].end > tau) still.push_back(i);
      running[s] = still;
      while (!queue[s].empty()) {
        int h = queue[s].front();
        int64_t used = 0;
        for (int i : running[s]) used += tb.mem[bs[i].m];
        if (used + tb.mem[bs[h].m] > tb.cap(p)) break;
        int64_t F = tb.fbr_at(bs[h].m, p);
        for (int i : running[s]) F += tb.fbr_at(bs[i].m, p);
        int64_t f = F < kPpm ? kPpm : F;
        bs[h].start = tau;
        bs[h].end = tau + (int64_t)tb.solo_at(bs[h].m, p) * f / kPpm;
        running[s].push_back(h);
        queue[s].pop_front();
        ++admitted;
      }
    }
    ++tau;
  }
}

}  // namespace pem
