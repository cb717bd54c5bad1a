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
#ifndef PROTEAN_SWEEP_MINB
#define PROTEAN_SWEEP_MINB 3  // resident CTAs per SM the register budget is sized for
#endif

struct SwBatch {
  int64_t ready;
  int32_t q;         // footprint MiB
  int32_t n;         // members
  int32_t strict;
  int32_t slo;
  uint32_t moff;     // first member in the arrival array
  int64_t a_first, a_last;  // first and last member arrivals (the both-ends SLO tests)
};

struct SwShared {
  SwBatch b[kSwMax];
  int32_t fx[kSwMax][8];   // fbr of batch x's model on slice s's profile (ppm)
  int32_t sx[kSwMax][8];   // solo of batch x's model on slice s's profile (us)
  int32_t cap[8];          // slice capacity MiB
  int64_t wkey[kSwThreads / 32];
  uint32_t widx[kSwThreads / 32];
  int64_t tb;    // first ready time of the unit: schedule times are relative to it
  bool narrow;   // every relative time of any assignment fits int32 (bound below)
  int nb;
};

// members of a placed strict batch that miss the SLO: #{a : end - a > slo} over sorted arrivals
__device__ __forceinline__ int strict_misses(const SwBatch& b, const uint32_t* arr, int n, int64_t end,
                                             int64_t slo) {
  if (end - b.a_first <= slo) return 0;  // the earliest member meets it
  if (end - b.a_last > slo) return n;    // even the latest misses
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

// Batch X of a unit placed on its forced slice sl[X] after batches 0..X-1 (R19): live bound,
// footprint, FIFO after the slice's last start, memory wait, Eq 1 at the start instant over the
// slice's co-runners; then its share of the key (strict misses / BE tail).  Times are relative to
// the unit's first ready time tb, in TT (int32_t when the unit's bound fits, else int64_t).  X is a
// constant after unrolling, so the schedule arrays stay in registers.
template <int kB, typename TT>
__device__ __forceinline__ void place_at(const int X, const SwShared& sh, const int32_t (&qv)[kB], int (&sl)[kB],
                                         TT (&st)[kB], TT (&en)[kB], int max_live, int64_t tb,
                                         const uint32_t* arrival, int64_t& misses, int64_t& tail,
                                         int live_in = -1) {
  // sl[y] of an earlier batch is its slice if it was placed, else kOff (matches no slice), and
  // en[y] = 0 if it was not placed (never > t >= 0): one compare per test instead of two.
  constexpr int kOff = 15;
  const SwBatch& b = sh.b[X];
  const int s = sl[X];
  const TT t = (TT)(b.ready - tb);
  int live = live_in;  // residents live at t, GPU-wide: the same for every slice of batch X
  TT ls = 0;
  if (live < 0) {
    live = 0;
#pragma unroll
    for (int y = 0; y < kB; ++y) {
      if (y >= X) break;
      live += en[y] > t ? 1 : 0;
    }
  }
#pragma unroll
  for (int y = 0; y < kB; ++y) {
    if (y >= X) break;
    if (sl[y] == s && st[y] > ls) ls = st[y];  // FIFO: the slice's last start
  }
  const int32_t Ms = sh.cap[s];
  const bool ok = live < max_live && qv[X] <= Ms;
  st[X] = en[X] = 0;
  if (ok) {
    const TT t0 = t > ls ? t : ls;
    int32_t used = qv[X];  // only batches that fit a slice are held: sums stay far below 2^31
#pragma unroll
    for (int y = 0; y < kB; ++y) {
      if (y >= X) break;
      if (sl[y] == s && en[y] > t0) used += qv[y];
    }
    TT start = t0;
    if (used > Ms) {  // memory wait: the earliest release after which the batch fits
      start = (TT)(sizeof(TT) == 4 ? INT32_MAX : INT64_MAX);
#pragma unroll
      for (int y = 0; y < kB; ++y) {
        if (y >= X) break;
        if (!(sl[y] == s && en[y] > t0)) continue;
        int32_t rem = qv[X];
#pragma unroll
        for (int z = 0; z < kB; ++z) {
          if (z >= X) break;
          if (sl[z] == s && en[z] > en[y]) rem += qv[z];
        }
        if (rem <= Ms && en[y] < start) start = en[y];
      }
    }
    int64_t F = sh.fx[X][s];
#pragma unroll
    for (int y = 0; y < kB; ++y) {
      if (y >= X) break;
      if (sl[y] == s && st[y] <= start && start < en[y]) F += sh.fx[y][s];
    }
    st[X] = start;
    en[X] = start + (TT)exec_time(sh.sx[X][s], F);
  } else {
    sl[X] = kOff;
  }
  if (b.strict) {
    misses += ok ? strict_misses(b, arrival + b.moff, b.n, tb + (int64_t)en[X], b.slo) : b.n;
  } else {
    const int64_t tv = ok ? tb + (int64_t)en[X] - b.a_first : (int64_t)0xFFFFFFFFLL;
    tail = tv > tail ? tv : tail;
  }
}

// The assignments of a unit with exactly kB batches on a geometry with S slices, shared-prefix
// enumeration: a thread owns prefixes (slices of batches 0..kB-D-1, index p = sum s_x S^x), places
// them once, then loops over the last D batches' slices re-placing only what changed -- about
// S/(S-1) placements per assignment instead of kB.  Keeps the thread's min (key, index).
template <int kB, int D, typename TT>
__device__ __forceinline__ void sweep_range(const SwShared& sh, const uint32_t* arrival, int S, uint32_t first,
                                            uint32_t step, int max_live, int64_t tb, int64_t* bk, uint32_t* bi) {
  constexpr int K = kB - D;
  uint32_t npre = 1;
  for (int x = 0; x < K; ++x) npre *= (uint32_t)S;
  const uint32_t wK = npre, wK1 = npre * (uint32_t)S;  // index weights of batches K and K+1
  int64_t best = INT64_MAX;
  uint32_t bidx = 0;
  int32_t qv[kB];  // footprints, loop-invariant
#pragma unroll
  for (int x = 0; x < kB; ++x) qv[x] = sh.b[x].q;
#pragma unroll 1
  for (uint32_t p = first; p < npre; p += step) {
    int sl[kB];
    TT st[kB], en[kB];
    int64_t m0 = 0, t0 = 0;
    {
      uint32_t rem = p;
#pragma unroll
      for (int x = 0; x < K; ++x) {
        const uint32_t qd = rem / (uint32_t)S;
        sl[x] = (int)(rem - qd * (uint32_t)S);
        rem = qd;
      }
    }
#pragma unroll
    for (int x = 0; x < K; ++x) place_at<kB, TT>(x, sh, qv, sl, st, en, max_live, tb, arrival, m0, t0);
#pragma unroll 1
    for (int s1 = 0; s1 < S; ++s1) {
      sl[K] = s1;
      int64_t m1 = m0, t1 = t0;
      place_at<kB, TT>(K, sh, qv, sl, st, en, max_live, tb, arrival, m1, t1);
      if constexpr (D == 1) {
        const int64_t key = make_key(m1, t1, 0);
        const uint32_t idx = p + (uint32_t)s1 * wK;
        if (key_less(key, idx, best, bidx)) { best = key; bidx = idx; }
      } else {
        int live2 = 0;  // the last batch's live count does not depend on its own slice
        {
          const TT t2r = (TT)(sh.b[K + 1].ready - tb);
#pragma unroll
          for (int y = 0; y < kB; ++y) {
            if (y > K) break;
            live2 += en[y] > t2r ? 1 : 0;
          }
        }
#pragma unroll 1
        for (int s2 = 0; s2 < S; ++s2) {
          sl[K + 1] = s2;
          int64_t m2 = m1, t2 = t1;
          place_at<kB, TT>(K + 1, sh, qv, sl, st, en, max_live, tb, arrival, m2, t2, live2);
          const int64_t key = make_key(m2, t2, 0);
          const uint32_t idx = p + (uint32_t)s1 * wK + (uint32_t)s2 * wK1;
          if (key_less(key, idx, best, bidx)) { best = key; bidx = idx; }
        }
      }
    }
  }
  *bk = best;
  *bi = bidx;
}

template <int kB>
__device__ __forceinline__ void sweep_unit_geom(const SwShared& sh, const uint32_t* arrival, int S, uint32_t first,
                                                uint32_t step, int max_live, int64_t tb, bool narrow,
                                                int64_t* bk, uint32_t* bi) {
  constexpr int D = kB >= 4 ? 2 : 1;
  if (narrow) sweep_range<kB, D, int32_t>(sh, arrival, S, first, step, max_live, tb, bk, bi);
  else sweep_range<kB, D, int64_t>(sh, arrival, S, first, step, max_live, tb, bk, bi);
}

__global__ void __launch_bounds__(kSwThreads, PROTEAN_SWEEP_MINB) sweep_kernel(SweepParams P) {
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
        b.a_first = P.arrival[pb.req_off];
        b.a_last = P.arrival[pb.req_off + pb.n_req - 1];
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
    if (tid == 0) {  // relative-time bound: ends <= last ready + sum of the largest execution times
      int64_t tb = nb ? sh.b[0].ready : 0, fsum = 0, span = 0;
      for (int x = 0; x < nb; ++x) {
        const int m = P.batches[b0 + x].model;
        int32_t fm = 0;
        for (int q = 0; q < kNProf; ++q) fm = max(fm, T.fbr[m * kNProf + q]);
        fsum += fm;
      }
      for (int x = 0; x < nb; ++x) {
        const int m = P.batches[b0 + x].model;
        int32_t sm = 0;
        for (int q = 0; q < kNProf; ++q) sm = max(sm, T.solo[m * kNProf + q]);
        span += exec_time(sm, fsum);
      }
      if (nb) span += sh.b[nb - 1].ready - tb;
      sh.tb = tb;
      sh.narrow = span < (int64_t)INT32_MAX;
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
      if (tid < S) sh.cap[tid] = T.cap[T.gprof[j * 8 + tid]];
      __syncthreads();
      uint32_t total = 1;
      for (int x = 0; x < nb; ++x) total *= (uint32_t)S;
      n_assign += total;  // (sh.tb / sh.narrow are published by the barrier above)
      int64_t k = INT64_MAX;
      uint32_t ix = 0;
      switch (nb) {
        case 0: if (tid == 0) { k = make_key(0, 0, 0); ix = 0; } break;
        case 1: sweep_unit_geom<1>(sh, P.arrival, S, tid, blockDim.x, P.max_live, sh.tb, sh.narrow, &k, &ix); break;
        case 2: sweep_unit_geom<2>(sh, P.arrival, S, tid, blockDim.x, P.max_live, sh.tb, sh.narrow, &k, &ix); break;
        case 3: sweep_unit_geom<3>(sh, P.arrival, S, tid, blockDim.x, P.max_live, sh.tb, sh.narrow, &k, &ix); break;
        case 4: sweep_unit_geom<4>(sh, P.arrival, S, tid, blockDim.x, P.max_live, sh.tb, sh.narrow, &k, &ix); break;
        case 5: sweep_unit_geom<5>(sh, P.arrival, S, tid, blockDim.x, P.max_live, sh.tb, sh.narrow, &k, &ix); break;
        case 6: sweep_unit_geom<6>(sh, P.arrival, S, tid, blockDim.x, P.max_live, sh.tb, sh.narrow, &k, &ix); break;
        case 7: sweep_unit_geom<7>(sh, P.arrival, S, tid, blockDim.x, P.max_live, sh.tb, sh.narrow, &k, &ix); break;
        default: sweep_unit_geom<8>(sh, P.arrival, S, tid, blockDim.x, P.max_live, sh.tb, sh.narrow, &k, &ix); break;
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
