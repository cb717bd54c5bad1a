// form.cu — protean_form_batches (SURVEY §8(b) helper): O3 batch formation (P:L229, P:L239,
// reading Q14) and O5.2 round-robin dispatch (reading Q18) for an epoch range, on the
// stream-sorted copy the partition passes build (partition.cu).  One thread per replica: the
// replica's 2M streams are formed lazily (each stream's next batch: close at B requests or at
// first arrival + T, a binary search over the sorted stream) and merged in batch-id order
// (ready, strict first, model — distinct streams never tie on these), so the round-robin cursor
// sees the batches exactly in id order from epoch 0.  Pass 0 counts rows per (replica, epoch,
// GPU); pass 1 writes them at the host-scanned offsets.  A helper, not the bench path.
#include <cuda_runtime.h>
#include <stdint.h>

#include "replay.cuh"

namespace pemgpu {

namespace {

constexpr int kFormThreads = 64;

__global__ void __launch_bounds__(kFormThreads) form_kernel(FormParams P) {
  const int r = blockIdx.x * blockDim.x + threadIdx.x;
  if (r >= P.R) return;
  const int S = P.S, N = P.N, Ew = P.e_hi - P.e_lo;
  const uint32_t* sa = P.sa + P.saoff[r];
  const uint32_t* s0 = P.sidx + (size_t)r * (P.E + 1) * S;            // stream starts (epoch 0)
  const uint32_t* s1 = P.sidx + ((size_t)r * (P.E + 1) + P.E) * S;    // stream ends
  int cur[kMaxStreams] = {}, nn[kMaxStreams] = {};
  int64_t rd[kMaxStreams];  // the stream's next batch: ready time (INT64_MAX: exhausted), size
  auto next = [&](int k) {
    const int i = cur[k], end = (int)s1[k];
    if (i >= end) { rd[k] = INT64_MAX; nn[k] = 0; return; }
    const int m = k >> 1;
    const int B = P.bsz[m];
    const int64_t a0 = sa[i], T = P.tmo[m];
    int lo = i + 1, hi = end - i > B ? i + B : end;  // first member beyond the timeout, else hi
    while (lo < hi) {
      const int mid = (lo + hi) >> 1;
      if ((int64_t)sa[mid] > a0 + T) hi = mid; else lo = mid + 1;
    }
    nn[k] = lo - i;
    rd[k] = nn[k] == B ? (int64_t)sa[lo - 1] : a0 + T;  // full, else timeout (Q14)
  };
  for (int k = 0; k < S; ++k) {
    cur[k] = (int)s0[k];
    next(k);
  }
  int cursor = 0;
  for (;;) {
    int best = -1;  // batch id order: (ready, class strict = even stream first, model)
    for (int k = 0; k < S; ++k) {
      if (rd[k] == INT64_MAX) continue;
      if (best < 0 || rd[k] < rd[best] ||
          (rd[k] == rd[best] && ((k & 1) < (best & 1) || ((k & 1) == (best & 1) && k < best))))
        best = k;
    }
    if (best < 0) break;
    const int64_t ready = rd[best], e = ready / P.W;
    if (e >= P.e_hi) break;  // ids are in ready order: nothing later lands in range
    int g = -1;
    for (int i = 0; i < N; ++i) {
      const int n = (cursor + i) % N;
      const bool ok = !P.avail || (P.avail[((size_t)r * N + n) * 2] <= ready &&
                                   ready < P.avail[((size_t)r * N + n) * 2 + 1]);
      if (ok) { g = n; break; }
    }
    if (g >= 0) {
      cursor = (g + 1) % N;
      if (e >= P.e_lo) {
        const size_t cell = ((size_t)r * Ew + (e - P.e_lo)) * N + g;
        if (P.pass == 0) {
          P.cnt[cell] += 1;
        } else {
          const int64_t row = (int64_t)P.off[cell] + P.cnt[cell]++;
          protean_batch b;
          b.ready_us = (uint32_t)ready;
          b.req_off = (uint32_t)(P.saoff[r] + cur[best]);
          b.n_req = (uint16_t)nn[best];
          b.model = (uint8_t)(best >> 1);
          b.strict = (best & 1) ? 0 : 1;
          b.gpu = (uint32_t)g;
          P.rows[row] = b;
        }
      }
    }
    cur[best] += nn[best];
    next(best);
  }
}

}  // namespace

cudaError_t launch_form(const FormParams& P, cudaStream_t st) {
  form_kernel<<<(P.R + kFormThreads - 1) / kFormThreads, kFormThreads, 0, st>>>(P);
  return cudaGetLastError();
}

cudaError_t preload_form_kernel() {
  cudaFuncAttributes a;
  return cudaFuncGetAttributes(&a, form_kernel);
}

}  // namespace pemgpu
