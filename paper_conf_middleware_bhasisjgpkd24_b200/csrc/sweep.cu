// sweep.cu — N4a: the exhaustive assignment sweep of the paper's "Oracle" scheme ("ideal GPU
// configurations ... multiple offline ... scheduling sweeps"; readings R18-R21).
//
// One CTA per (replica, sim-GPU) unit (grid-stride).  For each geometry j in range the CTA's
// threads split the S_j^b assignments of the unit's b <= 8 batches; a thread evaluates its
// assignments one by one with the whole schedule in registers (the batch loop is unrolled for
// b = kB, so start/end/drop per batch never leave registers): live bound, footprint, FIFO +
// memory wait on the forced slice, Eq 1 at the start instant over the slice's co-runners, then
// the O8 key (strict misses via both-ends tests + binary search over the sorted members, BE tail).
// Per-(batch, slice) constants (FBR on the slice's profile, Solo, capacity) are staged in shared
// memory per geometry; the min (key, index) is a warp-shuffle + shared-memory reduction.
// Integer-only: bound by the ALU/issue rate, not by HBM (a unit reads <= 8 batch rows + members).
#include <cuda_runtime.h>
#include <stdint.h>

#include "replay.cuh"

namespace pemgpu {

namespace {

constexpr int kSwMax = 8;      // batches per unit (max_batches cap)
constexpr int kSwThreads = 256;

struct SwBatch {
  int64_t ready;
  int32_t q;         // footprint MiB
  int32_t n;         // members
  int32_t strict;
  int32_t slo;
  uint32_t moff;     // first member in the arrival array
};

struct SwShared {
  SwBatch b[kSwMax];
  int32_t fx[kSwMax][8];   // fbr of batch x's model on slice s's profile (ppm)
  int32_t sx[kSwMax][8];   // solo of batch x's model on slice s's profile (us)
  int32_t cap[8];          // slice capacity MiB
  int64_t wkey[kSwThreads / 32];
  uint32_t widx[kSwThreads / 32];
  int nb;
};

// members of a placed strict batch that miss the SLO: #{a : end - a > slo} over sorted arrivals
__device__ __forceinline__ int strict_misses(const uint32_t* arr, int n, int64_t end, int64_t slo) {
  if (end - (int64_t)__ldg(arr) <= slo) return 0;             // the earliest member meets it
  if (end - (int64_t)__ldg(arr + n - 1) > slo) return n;      // even the latest misses
  int lo = 0, hi = n;  // first index with end - a <= slo  <=>  a >= end - slo
  const int64_t need = end - slo;
  while (lo < hi) {
    const int mid = (lo + hi) >> 1;
    if ((int64_t)__ldg(arr + mid) >= need) hi = mid; else lo = mid + 1;
  }
  return lo;
}

__device__ __forceinline__ bool key_less(int64_t k1, uint32_t i1, int64_t k2, uint32_t i2) {
  return k1 < k2 || (k1 == k2 && i1 < i2);
}

// Every assignment idx in [first, total) step `step` of a unit with exactly kB batches on a
// geometry with S slices; returns the thread's best (key without tag, idx).
template <int kB>
__device__ __forceinline__ void sweep_range(const SwShared& sh, const uint32_t* arrival, int S, uint32_t total,
                                            uint32_t first, uint32_t step, int max_live, int64_t* bk,
                                            uint32_t* bi) {
  int64_t best = INT64_MAX;
  uint32_t bidx = 0;
#pragma unroll 1
  for (uint32_t idx = first; idx < total; idx += step) {
    int sl[kB];
    {
      uint32_t rem = idx;
#pragma unroll
      for (int x = 0; x < kB; ++x) {
        const uint32_t qd = rem / (uint32_t)S;
        sl[x] = (int)(rem - qd * (uint32_t)S);
        rem = qd;
      }
    }
    int64_t st[kB], en[kB];
    bool ok[kB];
    int64_t misses = 0, tail = 0;
#pragma unroll
    for (int x = 0; x < kB; ++x) {
      const SwBatch& b = sh.b[x];
      const int s = sl[x];
      const int64_t t = b.ready;
      int live = 0;
      int64_t ls = 0;
#pragma unroll
      for (int y = 0; y < x; ++y) {
        live += (ok[y] && en[y] > t) ? 1 : 0;
        if (ok[y] && sl[y] == s && st[y] > ls) ls = st[y];  // FIFO: the slice's last start
      }
      const int32_t Ms = sh.cap[s];
      ok[x] = live < max_live && b.q <= Ms;
      st[x] = en[x] = 0;
      if (ok[x]) {
        const int64_t t0 = t > ls ? t : ls;
        int64_t used = b.q;
#pragma unroll
        for (int y = 0; y < x; ++y)
          if (ok[y] && sl[y] == s && en[y] > t0) used += sh.b[y].q;
        int64_t start = t0;
        if (used > Ms) {  // memory wait: the earliest release after which the batch fits
          start = INT64_MAX;
#pragma unroll
          for (int y = 0; y < x; ++y) {
            if (!(ok[y] && sl[y] == s && en[y] > t0)) continue;
            int64_t rem = b.q;
#pragma unroll
            for (int z = 0; z < x; ++z)
              if (ok[z] && sl[z] == s && en[z] > en[y]) rem += sh.b[z].q;
            if (rem <= Ms && en[y] < start) start = en[y];
          }
        }
        int64_t F = sh.fx[x][s];
#pragma unroll
        for (int y = 0; y < x; ++y)
          if (ok[y] && sl[y] == s && st[y] <= start && start < en[y]) F += sh.fx[y][s];
        st[x] = start;
        en[x] = start + exec_time(sh.sx[x][s], F);
      }
      if (b.strict) {
        misses += ok[x] ? strict_misses(arrival + b.moff, b.n, en[x], b.slo) : b.n;
      } else {
        const int64_t tb = ok[x] ? en[x] - (int64_t)__ldg(arrival + b.moff) : (int64_t)0xFFFFFFFFLL;
        tail = tb > tail ? tb : tail;
      }
    }
    const int64_t key = make_key(misses, tail, 0);
    if (key < best) {  // idx ascending per thread: keep the first minimiser
      best = key;
      bidx = idx;
    }
  }
  *bk = best;
  *bi = bidx;
}

__global__ void __launch_bounds__(kSwThreads) sweep_kernel(SweepParams P) {
  extern __shared__ __align__(16) unsigned char smem[];
  __shared__ SwShared sh;
  const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
  int32_t* tabw = reinterpret_cast<int32_t*>(smem);
  for (int i = tid; i < P.tl.words; i += blockDim.x) tabw[i] = P.tab[i];
  Tab T;
  T.bind(tabw, P.tl);
  __syncthreads();
  const int units = P.R * P.N;
  const int Gc = P.geom_hi - P.geom_lo;
#pragma unroll 1
  for (int u = blockIdx.x; u < units; u += gridDim.x) {
    const int32_t b0 = P.batch_off[u], b1 = P.batch_off[u + 1];
    const int nb = b1 - b0;
    const int cur = P.cur_geom[u];
    bool bad = nb < 0 || (cur != 0xFF && cur >= T.G);
    if (!bad && nb > P.max_batches) {
      if (tid == 0) atomicOr(&P.err[1], 1);
      continue;  // uniform
    }
    if (tid == 0) sh.nb = nb;
    if (!bad && tid < nb) {
      const protean_batch& pb = P.batches[b0 + tid];
      SwBatch& b = sh.b[tid];
      const int m = pb.model;
      bad = m >= T.M || pb.n_req < 1 || (tid > 0 && P.batches[b0 + tid - 1].ready_us > pb.ready_us);
      if (!bad) {
        b.ready = pb.ready_us;
        b.q = T.mem[m];
        b.n = pb.n_req;
        b.strict = pb.strict ? 1 : 0;
        b.slo = T.slo[m];
        b.moff = pb.req_off;
        for (int i = 0; i < pb.n_req; ++i) {  // members sorted and not after ready
          const uint32_t a = P.arrival[pb.req_off + i];
          if (a > pb.ready_us || (i > 0 && a < P.arrival[pb.req_off + i - 1])) { bad = true; break; }
        }
      }
    }
    if (__syncthreads_or(bad)) {
      if (tid == 0) atomicOr(&P.err[0], 1);
      continue;
    }
    int64_t kbest = INT64_MAX;
    unsigned long long n_assign = 0;
#pragma unroll 1
    for (int j = P.geom_lo; j < P.geom_hi; ++j) {
      const int S = T.gn[j];
      for (int i = tid; i < kSwMax * 8; i += blockDim.x) {
        const int x = i >> 3, s = i & 7;
        if (x < nb && s < S) {
          const int p = T.gprof[j * 8 + s];
          const int m = P.batches[b0 + x].model;
          sh.fx[x][s] = T.fbr[m * kNProf + p];
          sh.sx[x][s] = T.solo[m * kNProf + p];
        }
      }
      if (tid < S) sh.cap[tid] = prof_cap(T.gprof[j * 8 + tid]);
      __syncthreads();
      uint32_t total = 1;
      for (int x = 0; x < nb; ++x) total *= (uint32_t)S;
      n_assign += total;
      int64_t k = INT64_MAX;
      uint32_t ix = 0;
      switch (nb) {
        case 0: if (tid == 0) { k = make_key(0, 0, 0); ix = 0; } break;
        case 1: sweep_range<1>(sh, P.arrival, S, total, tid, blockDim.x, P.max_live, &k, &ix); break;
        case 2: sweep_range<2>(sh, P.arrival, S, total, tid, blockDim.x, P.max_live, &k, &ix); break;
        case 3: sweep_range<3>(sh, P.arrival, S, total, tid, blockDim.x, P.max_live, &k, &ix); break;
        case 4: sweep_range<4>(sh, P.arrival, S, total, tid, blockDim.x, P.max_live, &k, &ix); break;
        case 5: sweep_range<5>(sh, P.arrival, S, total, tid, blockDim.x, P.max_live, &k, &ix); break;
        case 6: sweep_range<6>(sh, P.arrival, S, total, tid, blockDim.x, P.max_live, &k, &ix); break;
        case 7: sweep_range<7>(sh, P.arrival, S, total, tid, blockDim.x, P.max_live, &k, &ix); break;
        default: sweep_range<8>(sh, P.arrival, S, total, tid, blockDim.x, P.max_live, &k, &ix); break;
      }
      // min (key, idx) over the CTA: lowest index among equal keys (R20)
#pragma unroll
      for (int d = 16; d > 0; d >>= 1) {
        const int64_t ok = __shfl_xor_sync(0xffffffffu, k, d);
        const uint32_t oi = __shfl_xor_sync(0xffffffffu, ix, d);
        if (key_less(ok, oi, k, ix)) { k = ok; ix = oi; }
      }
      if (lane == 0) { sh.wkey[warp] = k; sh.widx[warp] = ix; }
      __syncthreads();
      if (tid == 0) {
        k = sh.wkey[0];
        ix = sh.widx[0];
        for (int w = 1; w < (int)(blockDim.x >> 5); ++w)
          if (key_less(sh.wkey[w], sh.widx[w], k, ix)) { k = sh.wkey[w]; ix = sh.widx[w]; }
        const int64_t key = k | (int64_t)(j == cur ? 0 : j + 1);  // tag (O8)
        uint32_t code = 0, rem = ix;
        for (int x = 0; x < nb; ++x) {
          code |= (rem % (uint32_t)S) << (3 * x);
          rem /= (uint32_t)S;
        }
        const size_t o = (size_t)u * Gc + (j - P.geom_lo);
        if (P.sweep_key) P.sweep_key[o] = key;
        if (P.assign) P.assign[o] = code;
        kbest = key < kbest ? key : kbest;
      }
      __syncthreads();  // sh.fx / sh.cap / sh.wkey reused by the next geometry
    }
    if (tid == 0) {
      P.best_key[u] = kbest;
      atomicAdd(reinterpret_cast<unsigned long long*>(P.n_assign), n_assign);
    }
  }
}

}  // namespace

cudaError_t launch_sweep(const SweepParams& P, int grid, cudaStream_t st) {
  const size_t smem = (size_t)P.tl.words * 4;
  sweep_kernel<<<grid, kSwThreads, smem, st>>>(P);
  return cudaGetLastError();
}

cudaError_t preload_sweep_kernel() {
  cudaFuncAttributes a;
  return cudaFuncGetAttributes(&a, sweep_kernel);
}

}  // namespace pemgpu
