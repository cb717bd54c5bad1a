// oracle/batch.cpp — TEST INFRASTRUCTURE ONLY (see pem.hpp).
// O3 batch formation.  Requests are batch-served after strict-first reordering
// (P:L233); one container per batch.  The paper gives no batch-closing rule; reading
// Q14: a batch of model m closes at B_m requests or at first arrival + T_m.
#include "pem.hpp"
#include <algorithm>
#include <tuple>

namespace pem {

std::vector<Batch> form_batches(const Tables& tb, const uint32_t* arrival, const uint8_t* meta,
                                int64_t n) {
  // one stream per (model, class); each stream in (arrival, request index) order — the trace is
  // already sorted by arrival, so a stable partition keeps that order.
  std::vector<std::vector<int64_t>> stream(2 * tb.M);
  for (int64_t i = 0; i < n; ++i) {
    int m = meta[i] & 63;
    bool strict = (meta[i] >> 7) & 1;
    stream[2 * m + (strict ? 0 : 1)].push_back(i);
  }
  std::vector<Batch> out;
  for (int m = 0; m < tb.M; ++m) {
    for (int cls = 0; cls < 2; ++cls) {
      const std::vector<int64_t>& idx = stream[2 * m + cls];
      const int64_t B = tb.bsz[m], T = tb.tmo[m];
      size_t i = 0;
      while (i < idx.size()) {
        const int64_t a0 = arrival[idx[i]];
        size_t j = i;
        while (j < idx.size() && (int64_t)(j - i) < B && (int64_t)arrival[idx[j]] <= a0 + T) ++j;
        Batch b;
        b.n = (int)(j - i);
        b.model = m;
        b.strict = (cls == 0);
        b.first_raw = idx[i];
        b.ready = (b.n == B) ? (int64_t)arrival[idx[j - 1]] : a0 + T;  // full, else timeout
        for (size_t r = i; r < j; ++r) b.arr.push_back(arrival[idx[r]]);
        out.push_back(std::move(b));
        i = j;
      }
    }
  }
  // batch id order: (ready, class strict=0 < BE=1, model, first request index)
  std::sort(out.begin(), out.end(), [](const Batch& a, const Batch& b) {
    return std::make_tuple(a.ready, a.strict ? 0 : 1, a.model, a.first_raw) <
           std::make_tuple(b.ready, b.strict ? 0 : 1, b.model, b.first_raw);
  });
  return out;
}

}  // namespace pem
