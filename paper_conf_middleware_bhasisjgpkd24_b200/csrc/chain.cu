// chain.cu — the lean per-replica epoch chain and the per-request accounting pass (sm_100a).
//
// With the candidate search (cand.cu) taken out of the chain, what remains sequential per replica
// is small: per epoch, the VM events and installs (O11, O5.3), the round-robin dispatch of the
// epoch's id-ordered batches (Q18), the actual Alg 1 placement on the carried GPU state
// (P:L251-277 under Eq 1 / Eq 2, P:L191 / P:L208), and the decision step (argmin over the
// candidate keys, hysteresis and the ~30% cap).  One WARP carries one replica
// (no CTA barriers; a few KB of shared memory per replica), so every replica of config 5 is
// resident at once instead of three per SM:
//
//   chain_kernel  warp per replica.  Per epoch: A (lane = GPU), the epoch's batch rows (cand.cu,
//                 prefetched one epoch ahead with cp.async), D (closed form when every GPU is
//                 available, else a ballot over availability per batch), E (lane = GPU: Alg 1 over
//                 the GPU's 64 resident slots -- alive and per-slice masks; the per-slice FIFO keeps
//                 every resident's start <= t0, so only ends, footprints and co-runner FBRs are
//                 stored), G (lane = GPU).  The candidate keys come from cand.cu for closed-form
//                 epochs (rotated by the cursor); other epochs are scored here, one lane per (GPU,
//                 geometry), Alg 1 from idle (32-bit time, 64-bit fallback).  Each batch's outcome
//                 goes to HBM for the accounting pass.
//   acct_kernel   CTA per replica: per-request latencies end - arrival of every placed batch (O7),
//                 log-linear histograms in shared memory, SLO hits, arrival / drop counters, then
//                 the nearest-rank P50 / P99 (O12) -- the fused engine's phase F and finalize.
//
// Both produce exactly the fused engine's outputs (replay.cu); the host takes this path for mode R,
// policy 0 (keys from cand.cu) or 2 (Alg 2's heuristic in G; cand.cu forms rows only), no container
// pools, N <= 32, N * G even, max_live <= 64 (api.cu).
#include <cuda_runtime.h>
#include <stdint.h>

#include "replay.cuh"
#include "place_group.cuh"
#include "chain_state.cuh"

namespace pemgpu {

namespace {

using namespace pg;
constexpr int kChainWarps = 4;  // warps (replicas) per chain CTA
#ifndef PROTEAN_CHAIN_MINB
#define PROTEAN_CHAIN_MINB 7  // 7 x 4 warps per SM: all 4096 replicas of config 5 resident at once
#endif
constexpr int kAcctWarps = 8;  // warps per accounting CTA
constexpr int kUB = kUnitBats;

__device__ __forceinline__ void cp_async16(const void* dst_smem, const void* src) {
  const uint32_t d = (uint32_t)__cvta_generic_to_shared(dst_smem);
  asm volatile("cp.async.cg.shared.global [%0], [%1], 16;" ::"r"(d), "l"(src) : "memory");
}
__device__ __forceinline__ void cp_async_commit() { asm volatile("cp.async.commit_group;" ::: "memory"); }
__device__ __forceinline__ void cp_async_wait_all() { asm volatile("cp.async.wait_all;" ::: "memory"); }

// Alg 1 from idle of GPU-epoch batches gl[0..cnt) on geometry j (O8), one lane, 64-bit times: the
// plain definitions (live residents, BE memory for the tag walk, FIFO start, memory wait, Eq 1
// co-runners) by scans over the batches placed so far.  Per-lane arrays in global scratch,
// interleaved by lane.  For the epochs cand.cu did not hold (a GPU unavailable inside the epoch).
__device__ int64_t score_idle(const Tab& T, int j, int cur, const UnitBats& U, const uint8_t* gl, int cnt,
                              const uint32_t* sa_r, int max_live, int64_t* en, uint32_t* pk, int32_t* fb) {
  constexpr int L = 32;  // lane stride of the per-lane arrays
  const int ns = T.gn[j];
  int64_t ls[kMaxSl];
#pragma unroll
  for (int s = 0; s < kMaxSl; ++s) ls[s] = 0;
  int64_t misses = 0, tail = 0;
#pragma unroll 1
  for (int x = 0; x < cnt; ++x) {
    const int b = gl[x];
    const uint32_t info = U.info[b];
    const int m = (info >> 16) & 0xFF, nreq = info & 0xFFFF;
    const bool strict = (info >> 24) & 1;
    const int64_t t = U.ready[b];
    int live = 0;
    int32_t be = 0;
#pragma unroll 1
    for (int i = 0; i < x; ++i) {
      if (en[i * L] > t) {
        ++live;
        if (pk[i * L] >> 27) be += (int32_t)(pk[i * L] & kMemMask);
      }
    }
    const int32_t q = T.mem[m];
    uint64_t best = ~0ull;
    int64_t bst = 0, bend = 0;
    if (live < max_live) {
#pragma unroll 1
      for (int s = 0; s < ns; ++s) {
        const int p = T.gprof[j * 8 + s];
        const int32_t Ms = T.cap[p];
        if (q > Ms) continue;
        int64_t lss = 0;
#pragma unroll
        for (int z = 0; z < kMaxSl; ++z)
          if (z == s) lss = ls[z];
        const int64_t t0 = t > lss ? t : lss;
        int32_t used = 0;
        int64_t F = T.fbr[m * kNProf + p];
#pragma unroll 1
        for (int i = 0; i < x; ++i)
          if ((int)((pk[i * L] >> 24) & 7) == s && en[i * L] > t0) {
            used += (int32_t)(pk[i * L] & kMemMask);
            F += fb[i * L];
          }
        int64_t start = t0;
        if (used + q > Ms) {  // releases after t0 ascending; the first that fits (q <= Ms)
          int64_t ev = t0;
#pragma unroll 1
          for (;;) {
            int64_t nxt = INT64_MAX;
            int32_t rem = 0;
#pragma unroll 1
            for (int i = 0; i < x; ++i)
              if ((int)((pk[i * L] >> 24) & 7) == s && en[i * L] > ev && en[i * L] < nxt) nxt = en[i * L];
            ev = nxt;
#pragma unroll 1
            for (int i = 0; i < x; ++i)
              if ((int)((pk[i * L] >> 24) & 7) == s && en[i * L] > ev) rem += (int32_t)(pk[i * L] & kMemMask);
            if (rem + q <= Ms) break;
          }
          start = ev;
          F = T.fbr[m * kNProf + p];
#pragma unroll 1
          for (int i = 0; i < x; ++i)
            if ((int)((pk[i * L] >> 24) & 7) == s && en[i * L] > start) F += fb[i * L];
        }
        const int64_t c = start + exec_time(T.solo[m * kNProf + p], F);
        uint64_t key;
        if (strict) {  // choose_strict_slice (Q11)
          const uint64_t inelig = (be >= T.gpref[j * 8 + s]) ? (1ull << 62) : 0ull;
          key = inelig | ((uint64_t)c << 6) | ((uint64_t)(4 - p) << 3) | (uint64_t)s;
        } else {       // choose_best_effort_slice (Q12)
          key = ((uint64_t)start << 3) | (uint64_t)s;
        }
        if (key < best) {
          best = key;
          bst = start;
          bend = c;
        }
      }
    }
    const bool placed = best != ~0ull;
    const int bsl = (int)(best & 7);
    en[x * L] = placed ? bend : 0;
    pk[x * L] = (uint32_t)q | ((uint32_t)bsl << 24) | (strict ? 0u : (1u << 27));
    fb[x * L] = placed ? T.fbr[m * kNProf + T.gprof[j * 8 + bsl]] : 0;
    if (placed) {
#pragma unroll
      for (int z = 0; z < kMaxSl; ++z)
        if (z == bsl) ls[z] = bst;
    }
    const uint32_t* ma = sa_r + U.pos[b];
    if (strict) {
      if (!placed) {
        misses += nreq;
      } else {
        const int64_t slo = T.slo[m];
        if (bend - (int64_t)ma[0] > slo)
          misses += (bend - (int64_t)ma[nreq - 1] > slo) ? nreq : nreq - hits_in(ma, nreq, bend, slo);
      }
    } else {
      const int64_t tb = placed ? bend - (int64_t)ma[0] : (int64_t)0xFFFFFFFFLL;
      tail = tb > tail ? tb : tail;
    }
  }
  return make_key(misses, tail, j == cur ? 0 : j + 1);
}

// The same Alg 1 from idle in 32-bit time relative to eW with per-slice bit masks of the batches
// placed so far (cand.cu's lane, its state in global scratch instead of shared memory).  Returns
// false when a completion is 2^25 us past eW or the GPU holds more than 32 batches: the caller
// then takes score_idle.
__device__ bool score_idle32(const Tab& T, int j, int cur, const UnitBats& U, const uint8_t* gl, int cnt,
                             const uint32_t* sa_r, int max_live, uint32_t eW32, int64_t eW, uint32_t* en,
                             uint32_t* pk, int32_t* fb, uint32_t* lsm, const uint8_t* fitm, int M,
                             int64_t* key_out) {
  constexpr int L = 32;
  if (cnt > 32) return false;
  const int ns = T.gn[j];
  const uint8_t* gp = T.gprof + j * 8;
  const int32_t* gpref = T.gpref + j * 8;
#pragma unroll 1
  for (int s = 0; s < ns; ++s) {
    lsm[(2 * s) * L] = 0;      // last start
    lsm[(2 * s + 1) * L] = 0;  // batches placed on the slice
  }
  uint32_t alive = 0;
  int be = 0;
  bool wide = false;
  int64_t misses = 0, tail = 0;
#pragma unroll 1
  for (int x = 0; x < cnt; ++x) {
    const int b = gl[x];
    const uint32_t info = U.info[b];
    const int m = (info >> 16) & 0xFF, nreq = info & 0xFFFF;
    const bool strict = (info >> 24) & 1;
    const uint32_t rt = U.ready[b] - eW32;
#pragma unroll 1
    for (uint32_t a = alive; a; a &= a - 1) {
      const int i = __ffs(a) - 1;
      if (en[i * L] <= rt) {
        alive &= ~(1u << i);
        if (pk[i * L] >> 27) be -= (int)(pk[i * L] & kMemMask);
      }
    }
    const int32_t q = T.mem[m];
    const int32_t* fbr_m = T.fbr + m * kNProf;
    const int32_t* solo_m = T.solo + m * kNProf;
    uint32_t best = 0xFFFFFFFFu, bst = 0, bc = 0;
    const uint32_t sflag = strict ? 0xFFFFFFFFu : 0u;
#pragma unroll 1
    for (uint32_t fit = __popc(alive) < max_live ? (uint32_t)fitm[j * M + m] : 0u; fit; fit &= fit - 1) {
      const int s = __ffs(fit) - 1;
      const int p = gp[s];
      const int32_t Ms = T.cap[p];
      const uint32_t lss = lsm[(2 * s) * L];
      const uint32_t t0 = rt > lss ? rt : lss;
      const uint32_t set = lsm[(2 * s + 1) * L] & alive;
      int32_t used = 0;
      uint32_t F = (uint32_t)fbr_m[p];
#pragma unroll 1
      for (uint32_t a = set; a; a &= a - 1) {
        const int i = __ffs(a) - 1;
        if (en[i * L] > t0) {
          used += (int32_t)(pk[i * L] & kMemMask);
          F += (uint32_t)fb[i * L];
        }
      }
      uint32_t start = t0;
      if (used + q > Ms) {  // releases after t0 ascending; the first that fits
        uint32_t ev = t0;
#pragma unroll 1
        for (;;) {
          uint32_t nxt = 0xFFFFFFFFu;
          for (uint32_t a = set; a; a &= a - 1) {
            const uint32_t e = en[(__ffs(a) - 1) * L];
            if (e > ev && e < nxt) nxt = e;
          }
          ev = nxt;
          int32_t rem = 0;
          for (uint32_t a = set; a; a &= a - 1) {
            const int i = __ffs(a) - 1;
            if (en[i * L] > ev) rem += (int32_t)(pk[i * L] & kMemMask);
          }
          if (rem + q <= Ms) break;
        }
        start = ev;
        F = (uint32_t)fbr_m[p];
        for (uint32_t a = set; a; a &= a - 1) {
          const int i = __ffs(a) - 1;
          if (en[i * L] > start) F += (uint32_t)fb[i * L];
        }
      }
      // completions clamp to 2^25 - 1 in the key; a clamped winner sends the GPU to score_idle
      const int32_t so = solo_m[p];
      const int64_t ex = F <= (uint32_t)kPpm ? (int64_t)so : exec_time(so, F);
      const uint32_t cc = ex >= (1 << 25) ? (1u << 25) : min(start + (uint32_t)ex, 1u << 25);
      const uint32_t ks = ((be >= gpref[s]) ? 0x80000000u : 0u) | (min(cc, (1u << 25) - 1u) << 6) |
                          ((uint32_t)(4 - p) << 3) | (uint32_t)s;
      const uint32_t kb = (start << 3) | (uint32_t)s;
      const uint32_t key = (ks & sflag) | (kb & ~sflag);
      if (key < best) {
        best = key;
        bst = start;
        bc = cc;
      }
    }
    wide |= best != 0xFFFFFFFFu && bc >= (1u << 25) - 1u;
    if (wide) return false;
    const bool placed = best != 0xFFFFFFFFu;
    const int bsl = best & 7;
    en[x * L] = placed ? bc : 0u;
    pk[x * L] = (uint32_t)q | (strict ? 0u : (1u << 27));
    fb[x * L] = fbr_m[gp[bsl]];
    if (placed) {
      lsm[(2 * bsl) * L] = bst;
      lsm[(2 * bsl + 1) * L] |= 1u << x;
      alive |= 1u << x;
      if (!strict) be += q;
    }
    const int64_t cw = eW + (int64_t)bc;
    const uint32_t* ma = sa_r + U.pos[b];
    if (strict) {
      if (!placed) {
        misses += nreq;
      } else {
        const int64_t slo = T.slo[m];
        if (cw - (int64_t)ma[0] > slo)
          misses += (cw - (int64_t)ma[nreq - 1] > slo) ? nreq : nreq - hits_in(ma, nreq, cw, slo);
      }
    } else {
      const int64_t tb = placed ? cw - (int64_t)ma[0] : (int64_t)0xFFFFFFFFLL;
      tail = tb > tail ? tb : tail;
    }
  }
  *key_out = make_key(misses, tail, j == cur ? 0 : j + 1);
  return true;
}

// ---- N3 container pools on the lean chain (readings R22-R27), lane = sim-GPU:
// per (GPU, model) busy-until [kPoolCap] int64, size and surplus counter int32, in the warp's slot.
struct LanePools {
  int64_t* bu;
  int32_t* sz;
  int32_t* ctr;
  int M;
  __device__ __forceinline__ size_t pm(int g, int m) const { return (size_t)g * M + m; }
};
__device__ __forceinline__ void lane_pool_reset(const ReplayParams& P, const LanePools& pl, int g) {  // R22
  for (int m = 0; m < pl.M; ++m) {
    for (int i = 0; i < P.prewarm; ++i) pl.bu[pl.pm(g, m) * kPoolCap + i] = 0;
    pl.sz[pl.pm(g, m)] = P.prewarm;
    pl.ctr[pl.pm(g, m)] = 0;
  }
}
// R23: the first container of (g, m) idle at t, else a new one after a cold start (t + cold_us).
__device__ __forceinline__ int lane_pool_acquire(const ReplayParams& P, const LanePools& pl, int g, int m,
                                                 int64_t t, int64_t* t_eff, unsigned long long* cold) {
  const size_t k = pl.pm(g, m);
  const int64_t* b = pl.bu + k * kPoolCap;
  const int n = pl.sz[k];
  *t_eff = t;
#pragma unroll 1
  for (int i = 0; i < n; ++i)
    if (b[i] <= t) return i;
  *t_eff = t + P.cold_us;  // reactive scale-up
  *cold += 1;
  if (n >= kPoolCap) {
    atomicOr(&P.err[2], 1);
    return -1;
  }
  pl.bu[k * kPoolCap + n] = t;
  pl.sz[k] = n + 1;
  return n;
}
// R26: pools larger than the epoch's batch count for keepalive epochs in a row terminate their
// surplus containers idle at T (stable compaction).
__device__ __forceinline__ void lane_pool_terminate(const ReplayParams& P, const LanePools& pl, int g, int m,
                                                    int need, int64_t T) {
  const size_t k = pl.pm(g, m);
  const int n = pl.sz[k];
  int surplus = n - need;
  if (surplus <= 0) {
    pl.ctr[k] = 0;
    return;
  }
  if (++pl.ctr[k] < P.keepalive) return;
  int64_t* b = pl.bu + k * kPoolCap;
  int w = 0;
  for (int i = 0; i < n; ++i) {
    if (surplus > 0 && b[i] <= T) { --surplus; continue; }
    b[w++] = b[i];
  }
  pl.sz[k] = w;
  pl.ctr[k] = 0;
}

// kN3: container pools (cold_us > 0).  A template argument so that the pool-free instantiation
// carries none of the pool code (the runtime flag alone cost config 5's chain 13.4 -> 16.2 ms).
template <bool kN3>
__global__ void __launch_bounds__(32 * kChainWarps, PROTEAN_CHAIN_MINB) chain_kernel(ReplayParams P) {
  extern __shared__ __align__(16) unsigned char smem[];
  if (*(volatile const int*)P.ovf) return;  // the host replays the call on the fused engine
  const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
  int32_t* tabw = reinterpret_cast<int32_t*>(smem);
#pragma unroll 1
  for (int i = tid; i < P.tl.words; i += blockDim.x) tabw[i] = P.tab[i];
  __syncthreads();
  const ChainLayout& CL = P.cl;
  {
    uint8_t* fw = smem + (((size_t)P.tl.words * 4 + 15) & ~(size_t)15) + (size_t)kChainWarps * CL.total;
    Tab T0;
    T0.bind(tabw, P.tl);
#pragma unroll 1
    for (int i = tid; i < P.tl.G * P.tl.M; i += blockDim.x) {
      const int j = i / P.tl.M, m = i % P.tl.M;
      uint32_t f = 0;
      for (int s = 0; s < T0.gn[j]; ++s)
        if (T0.mem[m] <= T0.cap[T0.gprof[j * 8 + s]]) f |= 1u << s;
      fw[i] = (uint8_t)f;
    }
    __syncthreads();
  }
  unsigned char* wb = smem + (((size_t)P.tl.words * 4 + 15) & ~(size_t)15) + (size_t)warp * CL.total;
  const int N = P.N, G = P.tl.G, KS = CL.KS;
  const int64_t E = P.E, W = P.W;
  Ctx c;
  c.T.bind(tabw, P.tl);
  c.N = N;
  c.gu8 = wb + CL.gu8;
  c.gi = reinterpret_cast<int64_t*>(wb + CL.gi);
  c.g_cnt = reinterpret_cast<int*>(wb + CL.gcnt);
  c.g_off = reinterpret_cast<int*>(wb + CL.goff);
  c.a_n = reinterpret_cast<int*>(wb + CL.a_n);
  c.a_ls = reinterpret_cast<int64_t*>(wb + CL.a_ls);
  c.a_bu = reinterpret_cast<int64_t*>(wb + CL.a_bu);
  const Tab& T = c.T;
  UnitBats* ubs = reinterpret_cast<UnitBats*>(wb + CL.ub);
  int64_t* kst = reinterpret_cast<int64_t*>(wb + CL.kst);
  uint8_t* gl = wb + CL.gl;
  uint8_t* gpu_of = wb + CL.gpu;
  int sum_slots = 0;  // slot-evals per batch per decidable GPU (counter 8)
#pragma unroll 1
  for (int j = 0; j < G; ++j) sum_slots += T.gn[j];
  const int gw = blockIdx.x * kChainWarps + warp;  // this warp's scratch slot
  char* slot = P.scratch + (size_t)gw * P.slot_bytes;
  // the actual residents of GPU lane: 64 slots, lane-interleaved (slot i of lane l at i * 32 + l)
  // ga[i * 32]: end; ga[(64 + i) * 32]: packed word | co-runner FBR << 32 (one live base pointer)
  int64_t* ga = reinterpret_cast<int64_t*>(slot + P.o_alist) + lane;
  constexpr bool n3 = kN3;  // N3: container pools ahead of each actual placement
  LanePools pl;
  pl.M = P.tl.M;
  pl.bu = reinterpret_cast<int64_t*>(slot + P.o_pool);
  pl.sz = reinterpret_cast<int32_t*>(slot + P.o_pool + (size_t)N * pl.M * kPoolCap * 8);
  pl.ctr = pl.sz + (size_t)N * pl.M;
  // fitm[j][m]: the slice positions of geometry j that hold model m's footprint (CTA-wide table)
  const uint8_t* fitm = smem + (((size_t)P.tl.words * 4 + 15) & ~(size_t)15) + (size_t)kChainWarps * CL.total;
  int64_t* sc_en = reinterpret_cast<int64_t*>(slot + P.o_clist) + lane;  // score_idle arrays
  uint32_t* sc_pk = reinterpret_cast<uint32_t*>(slot + P.o_clist + (size_t)kUB * 32 * 8) + lane;
  int32_t* sc_fb = reinterpret_cast<int32_t*>(slot + P.o_clist + (size_t)kUB * 32 * 12) + lane;
  uint32_t* sc_ls = reinterpret_cast<uint32_t*>(slot + P.o_clist + (size_t)kUB * 32 * 16) + lane;
  uint32_t* sc_en32 = reinterpret_cast<uint32_t*>(slot + P.o_clist) + lane;  // score_idle32's ends
  constexpr int kUBChunks = (int)(sizeof(UnitBats) / 16);

#pragma unroll 1
  for (int r = gw; r < P.R; r += gridDim.x * kChainWarps) {
    const uint64_t replica = (uint64_t)(P.base + r);
    const UnitBats* ubr = P.ub + (size_t)r * E;
    const int64_t* kfr = P.kfc ? P.kfc + (size_t)r * E * KS : nullptr;
    int64_t* bres = P.bres + (size_t)r * E * kUB;
    const uint32_t* sa_r = P.sa + P.saoff[r];
    // ---- replica init (as replay.cu)
#pragma unroll 1
    for (int i = lane; i < N * kZA; i += 32) reinterpret_cast<uint64_t*>(wb + CL.msk)[i] = 0;
#pragma unroll 1
    for (int i = lane; i < 64; i += 32)  // every slot's packed word names slice 0 (no stale bits)
      for (int g = 0; g < N; ++g)
        reinterpret_cast<int64_t*>(slot + P.o_alist)[(64 + i) * 32 + g] = 0;
#pragma unroll 1
    for (int g = lane; g < N; g += 32) {
      reset_gpu_state(c, g, P.init_geom);
      c.gu8[3 * N + g] = c.gu8[4 * N + g] = (P.vm_policy == 0) ? VM_OD : VM_SPOT;
      c.gi[0 * N + g] = c.gi[1 * N + g] = 0;
      c.gi[2 * N + g] = 0;
      c.gi[3 * N + g] = kForever;
      c.gi[4 * N + g] = 0;
      c.gi[8 * N + g] = c.gi[9 * N + g] = c.gi[10 * N + g] = c.gi[11 * N + g] = 0;
      c.gi[12 * N + g] = c.gi[13 * N + g] = 0;
      if (n3) lane_pool_reset(P, pl, g);
    }
    int cursor = 0;
    unsigned long long n_cold = 0;  // this lane's GPU's cold starts (N3)
    int64_t nlog = 0;
    unsigned long long n_recfg = 0, n_slot = 0, n_cand = 0;
#pragma unroll 1
    for (int i = lane; i < kUBChunks; i += 32)
      cp_async16(reinterpret_cast<const char*>(&ubs[0]) + 16 * i, reinterpret_cast<const char*>(ubr) + 16 * i);
    cp_async_commit();
    cp_async_wait_all();
    __syncwarp();

#pragma unroll 1
    for (int64_t e = 0; e < E; ++e) {
      const int64_t eW = e * W, Tend = eW + W;
      const UnitBats& U = ubs[e & 1];
      // the candidate keys of this epoch and the batch rows of the next one, in flight during A-E
      if (kfr) {
#pragma unroll 1
        for (int i = lane; i < KS / 2; i += 32) cp_async16(kst + 2 * i, kfr + (size_t)e * KS + 2 * i);
      }
      if (e + 1 < E) {
#pragma unroll 1
        for (int i = lane; i < kUBChunks; i += 32)
          cp_async16(reinterpret_cast<const char*>(&ubs[(e + 1) & 1]) + 16 * i,
                     reinterpret_cast<const char*>(ubr + e + 1) + 16 * i);
      }
      cp_async_commit();
      // ---- A: VM events, installs, decidability (lane = simulated GPU)
      bool whole = true;
#pragma unroll 1
      for (int g = lane; g < N; g += 32) {
        if (P.vm_policy != 0) {
#pragma unroll 1
          for (int64_t k = (eW + P.rev - 1) / P.rev; k * P.rev < Tend; ++k) {
            const int64_t tau = k * P.rev;
            if (k < 1 || tau >= P.H) continue;
            if (c.gu8[1 * N + g] != kNoGeom && c.gi[1 * N + g] <= tau) reset_gpu_state(c, g, c.gu8[1 * N + g]);
            const bool lost = vm_event(P, c, replica, g, k, tau);
            if (n3 && lost) lane_pool_reset(P, pl, g);  // its containers go with the VM (R27)
          }
        }
        if (c.gu8[1 * N + g] != kNoGeom && c.gi[1 * N + g] <= Tend) reset_gpu_state(c, g, c.gu8[1 * N + g]);
        c.gu8[5 * N + g] = (has_vm(c, g, Tend) && c.gi[1 * N + g] <= Tend) ? 1 : 0;
        c.gu8[7 * N + g] = 0;
        c.gu8[6 * N + g] = kNoGeom;
        c.gi[7 * N + g] = -1;
        whole &= c.gi[2 * N + g] <= eW && c.gi[3 * N + g] >= Tend &&
                 !(c.gi[0 * N + g] < Tend && c.gi[1 * N + g] > eW);
      }
      const bool avail_all = __all_sync(0xffffffffu, whole);
      __syncwarp();
      const int nb = (int)U.nb;
      const int cur0 = cursor;
      // ---- D: dispatch (id order = row order)
      if (avail_all) {  // closed form (Q18): rank b -> GPU (cursor + b) mod N, position b div N
        const int dq = nb / N, drem = nb - dq * N;
        auto goff = [&](int g) {
          const int wrap = cursor + drem - N;
          int x = g - cursor;
          x = x < 0 ? 0 : (x > drem ? drem : x);
          if (wrap > 0) x = min(max(g - cursor, 0), N - cursor) + min(g, wrap);
          return g * dq + x;
        };
#pragma unroll 1
        for (int b = lane; b < nb; b += 32) {
          const int q = b / N, g = cursor + (b - q * N);
          const int gg = g >= N ? g - N : g;
          gpu_of[b] = (uint8_t)gg;
          gl[goff(gg) + q] = (uint8_t)b;
        }
        for (int g = lane; g <= N; g += 32) c.g_off[g] = goff(g);
        cursor = (int)((cursor + nb) % N);
      } else {
        // round robin over the GPUs available at each batch's ready time (lane = GPU): a ballot
        // of availability, the first available GPU at or after the cursor
        const unsigned nmask = N == 32 ? 0xffffffffu : ((1u << N) - 1u);
        int cu = cursor;
#pragma unroll 1
        for (int b = 0; b < nb; ++b) {
          const unsigned av = __ballot_sync(0xffffffffu, lane < N && available(c, lane, U.ready[b])) & nmask;
          int chosen = -1;
          if (av) {
            const unsigned hi = av & ~((1u << cu) - 1u);  // GPUs cu..N-1
            chosen = hi ? __ffs(hi) - 1 : __ffs(av) - 1;
            cu = chosen + 1 == N ? 0 : chosen + 1;
          }
          if (lane == 0) gpu_of[b] = chosen < 0 ? 0xFF : (uint8_t)chosen;
        }
        cursor = cu;
        __syncwarp();
        {  // per-GPU lists in id order: counts, exclusive scan over lanes, fill
          int cntg = 0;
          if (lane < N)
            for (int b = 0; b < nb; ++b) cntg += gpu_of[b] == lane ? 1 : 0;
          int x = cntg;
#pragma unroll
          for (int d = 1; d < 32; d <<= 1) {
            const int y = __shfl_up_sync(0xffffffffu, x, d);
            if (lane >= d) x += y;
          }
          if (lane < N) {
            int o = x - cntg;
            c.g_off[lane] = o;
            for (int b = 0; b < nb; ++b)
              if (gpu_of[b] == lane) gl[o++] = (uint8_t)b;
          }
          if (lane == N - 1) c.g_off[N] = x;
        }
        __syncwarp();
#pragma unroll 1
        for (int b = lane; b < nb; b += 32) {  // no GPU available: dropped (drop code 1)
          if (gpu_of[b] != 0xFF) continue;
          bres[(size_t)e * kUB + b] = -1;
          if (P.log && nlog + b < P.log_cap) {
            protean_batch_rec rec;
            const uint32_t info = U.info[b];
            rec.ready_us = U.ready[b];
            rec.epoch = (uint32_t)e;
            rec.n_req = (uint16_t)(info & 0xFFFF);
            rec.model = (uint8_t)((info >> 16) & 0xFF);
            rec.strict = (uint8_t)((info >> 24) & 1);
            rec.gpu = 0xFF;
            rec.slice = 0xFF;
            rec.dropped = 1;
            rec.pad = 0;
            rec.start_us = rec.end_us = 0;
            P.log[(size_t)r * P.log_cap + nlog + b] = rec;
          }
        }
      }
      __syncwarp();
      // ---- E: actual placement (O6, Alg 1), lane = simulated GPU, its batches in id order.
      // The carried residents of a GPU live in 64 slots (max_live <= 64): an alive mask, per-slice
      // masks, and per slot the end, footprint | best-effort flag and the FBR on its slice's
      // profile.  Per-slice FIFO keeps every resident's start <= the slice's last start <= t0, so
      // Eq 1's co-runners at any tried start are the slice's residents that end after it.
      if (lane < N) {
        const int g = lane, j = c.gu8[0 * N + g];
        uint64_t* alive_p = reinterpret_cast<uint64_t*>(c.a_n + g * kZA);
        uint64_t alive = *alive_p;
        uint64_t* msk = reinterpret_cast<uint64_t*>(wb + CL.msk) + g * kZA;
        int64_t* lsg = c.a_ls + g * kZA;
        int64_t* bug = c.a_bu + g * kZA;
        const uint8_t* gp = T.gprof + j * 8;
        const int32_t* gpref = T.gpref + j * 8;
        int64_t acc0 = 0, acc1 = 0;  // busy, memory-time of the placed batches
        const int x0 = c.g_off[g], cnt = c.g_off[g + 1] - x0;
#pragma unroll 1
        for (int xi = 0; xi < cnt; ++xi) {
          const int b = gl[x0 + xi];
          const uint32_t info = U.info[b];
          const int m = (info >> 16) & 0xFF;
          const bool strict = (info >> 24) & 1;
          int64_t t = (int64_t)U.ready[b];
          int ci = -1;  // N3: the batch's container (R23; acquisition on the actual placement, R25)
          if (n3) {
            int64_t te;
            ci = lane_pool_acquire(P, pl, g, m, t, &te, &n_cold);
            t = te;
          }
          const int32_t q = T.mem[m];
          int be = 0;  // best-effort footprint still running at t (Alg 1's tag walk)
#pragma unroll 1
          for (uint64_t a = alive; a; a &= a - 1) {  // residents ended by t never matter again
            const int i = __ffsll((long long)a) - 1;
            if (ga[i * 32] <= t) {
              alive &= ~(1ull << i);
            } else {
              const uint32_t pki = (uint32_t)ga[(64 + i) * 32];
              if (pki >> 27) be += (int)(pki & kMemMask);
            }
          }
          const bool overflow = __popcll(alive) >= P.max_live;  // reading Q39
          uint64_t best = ~0ull;
          int64_t bst = 0, bend = 0;
          uint32_t fit = overflow ? 0u : (uint32_t)fitm[j * CL.M + m];
#pragma unroll 1
          for (; fit; fit &= fit - 1) {
            const int s = __ffs(fit) - 1;
            const int p = gp[s];
            const int32_t Ms = T.cap[p];
            const int64_t t0 = t > lsg[s] ? t : lsg[s];
            const uint64_t set = msk[s] & alive;
            int32_t used = 0;
            int64_t F = T.fbr[m * kNProf + p];
#pragma unroll 1
            for (uint64_t a = set; a; a &= a - 1) {
              const int i = __ffsll((long long)a) - 1;
              if (ga[i * 32] > t0) {
                const uint64_t pf = (uint64_t)ga[(64 + i) * 32];
                used += (int32_t)((uint32_t)pf & kMemMask);
                F += (int32_t)(pf >> 32);
              }
            }
            int64_t start = t0;
            if (used + q > Ms) {  // the earliest release after which the batch fits (q <= Ms)
              int64_t ev = t0;
#pragma unroll 1
              for (;;) {
                int64_t nxt = INT64_MAX;
                int32_t rem = 0;
                for (uint64_t a = set; a; a &= a - 1) {
                  const int64_t ei = ga[(__ffsll((long long)a) - 1) * 32];
                  if (ei > ev && ei < nxt) nxt = ei;
                }
                ev = nxt;
                for (uint64_t a = set; a; a &= a - 1) {
                  const int i = __ffsll((long long)a) - 1;
                  if (ga[i * 32] > ev) rem += (int32_t)((uint32_t)ga[(64 + i) * 32] & kMemMask);
                }
                if (rem + q <= Ms) break;
              }
              start = ev;
              F = T.fbr[m * kNProf + p];
              for (uint64_t a = set; a; a &= a - 1) {
                const int i = __ffsll((long long)a) - 1;
                if (ga[i * 32] > start) F += (int32_t)((uint64_t)ga[(64 + i) * 32] >> 32);
              }
            }
            const int64_t cc = start + exec_time(T.solo[m * kNProf + p], F);
            const uint64_t key = strict  // choose_strict_slice (Q11) / choose_best_effort_slice (Q12)
                ? ((be >= gpref[s]) ? (1ull << 62) : 0ull) | ((uint64_t)cc << 6) | ((uint64_t)(4 - p) << 3) | (uint64_t)s
                : ((uint64_t)start << 3) | (uint64_t)s;
            if (key < best) {
              best = key;
              bst = start;
              bend = cc;
            }
          }
          const bool placed = best != ~0ull;
          const int s = (int)(best & 7);
          if (placed) {  // schedule(batch, slice): a free slot, the slice's FIFO, the busy union
            const int i = __ffsll((long long)~alive) - 1;
            const int p = gp[s];
            // a slot's bit sits only in the mask of the slice its packed word names (masks are
            // zeroed at replica start; a reset clears alive, not the masks)
            msk[((uint32_t)ga[(64 + i) * 32] >> 24) & 7] &= ~(1ull << i);
            ga[i * 32] = bend;
            ga[(64 + i) * 32] = (int64_t)((uint64_t)((uint32_t)q | ((uint32_t)s << 24) | (strict ? 0u : (1u << 27))) |
                                          ((uint64_t)(uint32_t)T.fbr[m * kNProf + p] << 32));
            alive |= 1ull << i;
            msk[s] |= 1ull << i;
            lsg[s] = bst;
            const int64_t bu = bug[s];
            const int64_t lo = bst > bu ? bst : bu;
            const int64_t hi = bend < P.H ? bend : P.H;
            if (hi > lo) acc0 += (int64_t)prof_compute(p) * (hi - lo);
            if (hi > bst) acc1 += (int64_t)q * (hi - bst);
            if (bend > bu) bug[s] = bend;
          }
          if (n3 && ci >= 0) pl.bu[pl.pm(g, m) * kPoolCap + ci] = placed ? bend : t;  // R24
          const int drop = placed ? 0 : (overflow ? 3 : 2);
          bres[(size_t)e * kUB + b] = placed ? bend : -(int64_t)drop;
          if (P.log && nlog + b < P.log_cap) {
            protean_batch_rec rec;
            rec.ready_us = U.ready[b];
            rec.epoch = (uint32_t)e;
            rec.n_req = (uint16_t)(info & 0xFFFF);
            rec.model = (uint8_t)m;
            rec.strict = strict ? 1 : 0;
            rec.gpu = (uint8_t)g;
            rec.slice = placed ? (uint8_t)s : 0xFF;
            rec.dropped = (uint8_t)drop;
            rec.pad = 0;
            rec.start_us = placed ? bst : 0;
            rec.end_us = placed ? bend : 0;
            P.log[(size_t)r * P.log_cap + nlog + b] = rec;
          }
        }
        *alive_p = alive;
        int64_t mx = 0;  // the latest end among the GPU's residents (drain end of a reconfiguration)
        for (uint64_t a = alive; a; a &= a - 1) {
          const int64_t ei = ga[(__ffsll((long long)a) - 1) * 32];
          mx = ei > mx ? ei : mx;
        }
        c.gi[5 * N + g] = mx;
        c.gi[10 * N + g] += acc0;
        c.gi[11 * N + g] += acc1;
      }
      if (n3) {  // R26: delayed termination, every (GPU, model) of the epoch
#pragma unroll 1
        for (int g = lane; g < N; g += 32) {
          const int x0 = c.g_off[g], cnt = c.g_off[g + 1] - x0;
#pragma unroll 1
          for (int m = 0; m < pl.M; ++m) {
            int need = 0;
            for (int x = 0; x < cnt; ++x) need += ((U.info[gl[x0 + x]] >> 16) & 0xFF) == (uint32_t)m ? 1 : 0;
            lane_pool_terminate(P, pl, g, m, need, Tend);
          }
        }
      }
      __syncwarp();
      cp_async_wait_all();
      __syncwarp();
      // ---- candidate keys: cand.cu's (closed form) or scored here.  The sentinel is read by
      // lane 0 and broadcast: when it is set, the scoring below overwrites kst[0], and a lane
      // still behind (ITS gives no lockstep after a __syncwarp) would otherwise read the key.
      const bool pre = P.policy == 0 && kfr && avail_all &&
                       __shfl_sync(0xffffffffu, (int)(kst[0] != INT64_MIN), 0) != 0;
      if (P.policy == 0 && !pre) {
#pragma unroll 1
        for (int pi = lane; pi < N * G; pi += 32) {
          const int g = pi / G, j = pi - g * G;
          int64_t key = -1;
          if (c.gu8[5 * N + g]) {
            const int cur = c.gu8[0 * N + g], x0 = c.g_off[g], cnt = c.g_off[g + 1] - x0;
            if (!score_idle32(T, j, cur, U, gl + x0, cnt, sa_r, P.max_live, (uint32_t)eW, eW,
                              sc_en32, sc_pk, sc_fb, sc_ls, fitm, CL.M, &key))
              key = score_idle(T, j, cur, U, gl + x0, cnt, sa_r, P.max_live, sc_en, sc_pk, sc_fb);
          }
          kst[pi] = key;  // by GPU
        }
        __syncwarp();
      }
      // ---- G: decisions (O9, O10), lane = simulated GPU (replay.cu's one-warp path)
      {
        const int g = lane;
        const bool gv = g < N;
        bool want = false;
        int64_t kb = kForever, kc = -1;
        uint32_t scored_b = 0;
        bool scored = false;
        if (gv) {
          uint8_t dec_out = kNoGeom;
          if (P.policy != 1 && c.gu8[5 * N + g]) {
            const int cur = c.gu8[0 * N + g];
            int best;
            if (P.policy == 0) {  // S8: argmin over the candidate keys
              int cl = g;  // keys by GPU (scored here) or by residue class (cand.cu)
              if (pre) {
                cl = g - cur0;
                cl = cl < 0 ? cl + N : cl;
              }
              const int64_t* kr = kst + cl * G;
#pragma unroll 1
              for (int v = 0; v < G; ++v) {
                int64_t kv = kr[v];
                if (v == cur) {
                  if (pre) kv &= ~(int64_t)255;  // tag 0: the current geometry (O8, Q20)
                  kc = kv;
                }
                kb = kv < kb ? kv : kb;
                if (P.cand_keys) P.cand_keys[(((size_t)r * E + e) * N + g) * (size_t)G + v] = kv;
              }
              c.gi[6 * N + g] = kb;
              c.gi[7 * N + g] = kc;
              const int tag = (int)(kb & 255);
              best = tag == 0 ? cur : tag - 1;
              scored_b = (uint32_t)(c.g_off[g + 1] - c.g_off[g]);
              scored = true;
            } else {  // policy 2: Alg 2's own heuristic (N1, readings R10-R15)
              int64_t be_num = 0, be_mem = 0;  // line 2: the BE batches dispatched to g (R10)
#pragma unroll 1
              for (int x = c.g_off[g]; x < c.g_off[g + 1]; ++x) {
                const uint32_t info = U.info[gl[x]];
                if ((info >> 24) & 1u) continue;
                be_num += 1;
                be_mem += T.mem[(info >> 16) & 0xFFu];  // footprint per batch (Q36)
              }
              const int64_t a = P.ewma_a;  // lines 8-9: EWMA in milli-units (R11)
              const int64_t X = (a * 1000 * be_num + (1000 - a) * c.gi[12 * N + g]) / 1000;
              const int64_t Y = (a * 1000 * be_mem + (1000 - a) * c.gi[13 * N + g]) / 1000;
              c.gi[12 * N + g] = X;
              c.gi[13 * N + g] = Y;
              // lines 10-18: the first of [[1g,2g],[3g]] whose summed capacity holds pred_BE_mem
              const bool fits12 = (int64_t)(T.cap[0] + T.cap[1]) * 1000 >= Y;
              const bool found = fits12 || (int64_t)T.cap[2] * 1000 >= Y;
              // lines 19-23: thresholds on pred_BE_num (R13, R14), (4g,3g) fallback, + 4g (R15)
              best = (!found || X < P.t_low || X > P.t_high) ? P.g43 : (fits12 ? P.g421 : P.g43);
            }
            dec_out = (uint8_t)best;
            c.gu8[6 * N + g] = (uint8_t)best;
            if (best != cur) {  // Alg 2 lines 24-30 (Q22)
              if (c.gu8[2 * N + g] >= P.wait_limit) want = true;
              else c.gu8[2 * N + g]++;
            } else {
              c.gu8[2 * N + g] = 0;
            }
          } else if (P.policy == 0) {
            c.gi[6 * N + g] = kForever;
          }
          if (P.decisions) P.decisions[((size_t)r * E + e) * N + g] = dec_out;
          if (P.cand_keys && (P.policy != 0 || !c.gu8[5 * N + g])) {
#pragma unroll 1
            for (int j = 0; j < G; ++j) P.cand_keys[(((size_t)r * E + e) * N + g) * (size_t)G + j] = -1;
          }
        }
        {  // counters 8, 9: slot-evals = scored GPUs' batches x the slots of the geometry set
          const uint32_t tb = __reduce_add_sync(0xffffffffu, scored_b);
          const int nsc = __popc(__ballot_sync(0xffffffffu, scored));
          n_slot += (unsigned long long)tb * (unsigned long long)sum_slots;
          n_cand += (unsigned long long)nsc * (unsigned long long)G;
        }
        if (P.policy != 1) {  // the ~30% cap: picks by (delta misses desc, GPU asc)
          const unsigned alive = __ballot_sync(0xffffffffu, gv && has_vm(c, g, Tend));
          const unsigned open = __ballot_sync(0xffffffffu, gv && c.gi[1 * N + g] > Tend);
          int cap = P.cap_pct * __popc(alive) / 100;
          if (cap < 1) cap = 1;
          int free_slots = cap - __popc(open);
          const int64_t d = (want && P.policy == 0) ? (kc >> 40) - (kb >> 40) : 0;
#pragma unroll 1
          while (free_slots > 0) {
            const unsigned wm = __ballot_sync(0xffffffffu, want);
            if (!wm) break;
            int64_t best_d = want ? d : INT64_MIN;
#pragma unroll
            for (int o = 16; o > 0; o >>= 1) {
              const int64_t od = __shfl_xor_sync(0xffffffffu, best_d, o);
              best_d = od > best_d ? od : best_d;
            }
            const unsigned tie = __ballot_sync(0xffffffffu, want && d == best_d);
            const int pick = __ffs(tie) - 1;
            if (lane == pick) {
              want = false;
              const int64_t drain_end = c.gi[5 * N + g] > Tend ? c.gi[5 * N + g] : Tend;
              c.gi[0 * N + g] = Tend;
              c.gi[1 * N + g] = drain_end + P.reconfig_us;
              c.gu8[1 * N + g] = c.gu8[6 * N + g];
              ++n_recfg;
            }
            --free_slots;
          }
        }
      }
      nlog += nb;
      __syncwarp();
    }
    // ---- finalize (O12): VM bills to H, cost, utilisation, counters 7-9 (0-6: acct_kernel)
#pragma unroll 1
    for (int g = lane; g < N; g += 32) bill_switch(c, g, VM_NONE, P.H, P.H);
    __syncwarp();
    n_recfg = __reduce_add_sync(0xffffffffu, (unsigned)n_recfg);
    n_cold = __reduce_add_sync(0xffffffffu, (unsigned)n_cold);
    if (lane == 0) {
      int64_t od = 0, spot = 0, busy = 0, memt = 0;
#pragma unroll 1
      for (int g = 0; g < N; ++g) {
        od += c.gi[8 * N + g];
        spot += c.gi[9 * N + g];
        busy += c.gi[10 * N + g];
        memt += c.gi[11 * N + g];
      }
      P.counters[(size_t)r * 10 + 7] = (int64_t)n_recfg;
      P.counters[(size_t)r * 10 + 8] = (int64_t)n_slot;
      P.counters[(size_t)r * 10 + 9] = (int64_t)n_cand;
      P.accum[(size_t)r * 4 + 0] = busy;
      P.accum[(size_t)r * 4 + 1] = memt;
      P.accum[(size_t)r * 4 + 2] = od;
      P.accum[(size_t)r * 4 + 3] = spot;
      P.cost[r] = __ddiv_rn(__dadd_rn(__dmul_rn((double)od, P.price_od),
                                      __dmul_rn((double)spot, P.price_spot)), 3.6e9);
      const double dN = (double)N, dH = (double)P.H;
      P.util[2 * (size_t)r] = __ddiv_rn((double)busy, __dmul_rn(__dmul_rn(7.0, dN), dH));
      P.util[2 * (size_t)r + 1] = __ddiv_rn((double)memt, __dmul_rn(__dmul_rn((double)T.cap[4], dN), dH));
      if (P.n_batches) P.n_batches[r] = nlog;
      if (P.cold_starts) P.cold_starts[r] = (int64_t)n_cold;
    }
    __syncwarp();
  }
}

// ---------------------------------------------------------------- accounting (O7, O12)
#ifndef PROTEAN_ACCT_MINB
#define PROTEAN_ACCT_MINB 4  // measured (4096 x 120 s): 4 -> 4.08, 6 -> 4.13, 8 -> 4.27 ms (issue-bound)
#endif
__global__ void __launch_bounds__(32 * kAcctWarps, PROTEAN_ACCT_MINB) acct_kernel(ReplayParams P) {
  if (*(volatile const int*)P.ovf) return;
  __shared__ uint32_t s_hist[2 * kNB];
  __shared__ uint32_t s_sink;
  __shared__ unsigned long long s_cnt[kAcctWarps][5];
  const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
  const uint32_t sink = (uint32_t)__cvta_generic_to_shared(&s_sink);
  const int64_t E = P.E;
  const int32_t* tabw = P.tab;
  const int32_t* slo_t = tabw + P.tl.o_slo;
#pragma unroll 1
  for (int r = blockIdx.x; r < P.R; r += gridDim.x) {
#pragma unroll 1
    for (int i = tid; i < 2 * kNB; i += blockDim.x) s_hist[i] = 0;
    __syncthreads();
    const UnitBats* ubr = P.ub + (size_t)r * E;
    const int64_t* bres = P.bres + (size_t)r * E * kUB;
    const uint32_t* sa_r = P.sa + P.saoff[r];
    unsigned long long c_sarr = 0, c_met = 0, c_sdrop = 0, c_barr = 0, c_bdrop = 0;  // warp-uniform
#pragma unroll 1
    for (int64_t e = warp; e < E; e += kAcctWarps) {  // warp per epoch
      const UnitBats& U = ubr[e];
      const int nb = (int)U.nb;
      // the epoch's rows and outcomes, one batch per lane, then the members batch by batch
#pragma unroll 1
      for (int b0 = 0; b0 < nb; b0 += 32) {
        const int bl = b0 + lane;
        uint32_t info_l = 0, pos_l = 0;
        int64_t end_l = 0;
        if (bl < nb) {
          info_l = U.info[bl];
          pos_l = U.pos[bl];
          end_l = bres[(size_t)e * kUB + bl];
        }
        const int nbl = min(32, nb - b0);
        // batch by batch, the next batch's first 128 members in flight while this one is counted
        uint32_t nxt[4];
        auto load128 = [&](int k, uint32_t* a) {
          const uint32_t pos = __shfl_sync(0xffffffffu, pos_l, k);
          const int nreq = (int)(__shfl_sync(0xffffffffu, info_l, k) & 0xFFFF);
          const uint32_t* ma = sa_r + pos;
#pragma unroll
          for (int q = 0; q < 4; ++q) {
            const int i = q * 32 + lane;
            a[q] = i < nreq ? __ldcs(ma + i) : 0u;
          }
        };
        if (nbl > 0) load128(0, nxt);
#pragma unroll 1
        for (int k = 0; k < nbl; ++k) {
          uint32_t cur[4];
#pragma unroll
          for (int q = 0; q < 4; ++q) cur[q] = nxt[q];
          if (k + 1 < nbl) load128(k + 1, nxt);
          const uint32_t info = __shfl_sync(0xffffffffu, info_l, k);
          const uint32_t pos = __shfl_sync(0xffffffffu, pos_l, k);
          const int64_t bend = __shfl_sync(0xffffffffu, end_l, k);
          const int nreq = info & 0xFFFF, m = (info >> 16) & 0xFF;
          const bool strict = (info >> 24) & 1;
          uint32_t met = 0;
          const bool drop = bend < 0;
          if (!drop) {
            const int64_t slo = slo_t[m];
            const uint32_t* ma = sa_r + pos;
            const uint32_t hb = (uint32_t)__cvta_generic_to_shared(s_hist + (strict ? 0 : kNB));
            if (bend - (int64_t)__shfl_sync(0xffffffffu, cur[0], 0) <= (int64_t)0xFFFFFFFFLL) {
              // latencies fit 32 bits: bucket = 128 s + (lat >> s), s = max(0, floor(log2 lat) - 7)
              const uint32_t e32 = (uint32_t)bend;
              const uint32_t slo32 = slo > (int64_t)0xFFFFFFFFLL ? 0xFFFFFFFFu : (uint32_t)slo;
#pragma unroll
              for (int q = 0; q < 4; ++q) {
                const int i = q * 32 + lane;
                const bool valid = i < nreq;
                const uint32_t lat = e32 - cur[q];
                const int sh = max(24 - __clz(lat), 0);
                inc_shared(valid ? hb + 4u * (uint32_t)((sh << 7) + (int)(lat >> sh)) : sink);
                met += __popc(__ballot_sync(0xffffffffu, valid && lat <= slo32));
              }
#pragma unroll 1
              for (int i0 = 128; i0 < nreq; i0 += 32) {  // batches above 128 requests
                const int i = i0 + lane;
                const bool valid = i < nreq;
                const uint32_t lat = e32 - ma[valid ? i : 0];
                const int sh = max(24 - __clz(lat), 0);
                inc_shared(valid ? hb + 4u * (uint32_t)((sh << 7) + (int)(lat >> sh)) : sink);
                met += __popc(__ballot_sync(0xffffffffu, valid && lat <= slo32));
              }
            } else {  // some latency >= 2^32 us: the saturating 64-bit bucket
#pragma unroll 1
              for (int i0 = 0; i0 < nreq; i0 += 32) {
                const int i = i0 + lane;
                const bool valid = i < nreq;
                const int64_t lat = bend - (int64_t)ma[valid ? i : 0];
                inc_shared(valid ? hb + 4u * (uint32_t)lat_bucket(lat) : sink);
                met += __popc(__ballot_sync(0xffffffffu, valid && lat <= slo));
              }
            }
          }
          if (strict) {
            c_sarr += nreq;
            if (drop) c_sdrop += nreq; else c_met += met;
          } else {
            c_barr += nreq;
            if (drop) c_bdrop += nreq;
          }
        }
      }
    }
    if (lane == 0) {
      s_cnt[warp][0] = c_sarr;
      s_cnt[warp][1] = c_met;
      s_cnt[warp][2] = c_sdrop;
      s_cnt[warp][3] = c_barr;
      s_cnt[warp][4] = c_bdrop;
    }
    __syncthreads();
    uint32_t* ghist = P.hist + (size_t)r * 2 * kNB;
#pragma unroll 1
    for (int w = tid; w < 2 * kNB; w += blockDim.x) ghist[w] = s_hist[w];
    if (tid == 0) {  // counters 0-6 (fold_wcnt's formulas)
      unsigned long long v[5] = {0, 0, 0, 0, 0};
#pragma unroll 1
      for (int w = 0; w < kAcctWarps; ++w)
        for (int i = 0; i < 5; ++i) v[i] += s_cnt[w][i];
      int64_t* cn = P.counters + (size_t)r * 10;
      cn[0] = (int64_t)v[0];
      cn[1] = (int64_t)v[1];
      cn[2] = (int64_t)(v[0] - v[1] - v[2]);
      cn[3] = (int64_t)v[2];
      cn[4] = (int64_t)v[3];
      cn[5] = (int64_t)(v[3] - v[4]);
      cn[6] = (int64_t)v[4];
    }
    if (warp < 2) {  // nearest-rank P50 / P99 per class (O12), from the shared histogram
      const uint32_t* h = s_hist + warp * kNB;
      uint32_t n = 0;
#pragma unroll 1
      for (int b = lane; b < kNB; b += 32) n += h[b];
#pragma unroll
      for (int d = 16; d > 0; d >>= 1) n += __shfl_xor_sync(0xffffffffu, n, d);
      int64_t p50 = 0, p99 = 0;
      if (n) {
        const uint64_t r50 = (50 * (uint64_t)n + 99) / 100, r99 = (99 * (uint64_t)n + 99) / 100;
        uint64_t cum = 0;
        int f50 = -1, f99 = -1;
#pragma unroll 1
        for (int b0 = 0; b0 < kNB && f99 < 0; b0 += 32) {
          uint32_t x = h[b0 + lane];
#pragma unroll
          for (int d = 1; d < 32; d <<= 1) {
            const uint32_t y = __shfl_up_sync(0xffffffffu, x, d);
            if (lane >= d) x += y;
          }
          const unsigned m50 = __ballot_sync(0xffffffffu, cum + x >= r50);
          const unsigned m99 = __ballot_sync(0xffffffffu, cum + x >= r99);
          if (f50 < 0 && m50) f50 = b0 + __ffs(m50) - 1;
          if (f99 < 0 && m99) f99 = b0 + __ffs(m99) - 1;
          cum += __shfl_sync(0xffffffffu, x, 31);
        }
        p50 = (int64_t)bucket_lower_edge(f50);
        p99 = (int64_t)bucket_lower_edge(f99);
      }
      if (lane == 0) {
        P.pct[(size_t)r * 4 + warp * 2] = p50;
        P.pct[(size_t)r * 4 + warp * 2 + 1] = p99;
      }
    }
    __syncthreads();
  }
}

}  // namespace

size_t chain_smem_bytes(const ReplayParams& P) {
  return (((size_t)P.tl.words * 4 + 15) & ~(size_t)15) + P.cl.total * kChainWarps + P.cl.fitm;
}

cudaError_t chain_occupancy(const ReplayParams& P, int* per_sm) {
  const size_t smem = chain_smem_bytes(P);
  auto k = P.cold_us > 0 ? chain_kernel<true> : chain_kernel<false>;
  cudaError_t e = cudaFuncSetAttribute(k, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
  if (e != cudaSuccess) return e;
  return cudaOccupancyMaxActiveBlocksPerMultiprocessor(per_sm, k, 32 * kChainWarps, smem);
}

cudaError_t launch_chain(const ReplayParams& P, int grid, cudaStream_t st) {
  if (P.cold_us > 0)
    chain_kernel<true><<<grid, 32 * kChainWarps, chain_smem_bytes(P), st>>>(P);
  else
    chain_kernel<false><<<grid, 32 * kChainWarps, chain_smem_bytes(P), st>>>(P);
  return cudaGetLastError();
}

cudaError_t launch_acct(const ReplayParams& P, cudaStream_t st) {
  acct_kernel<<<P.R, 32 * kAcctWarps, 0, st>>>(P);
  return cudaGetLastError();
}

cudaError_t preload_chain_kernels() {
  cudaFuncAttributes a;
  cudaError_t e = cudaFuncGetAttributes(&a, chain_kernel<false>);
  if (e == cudaSuccess) e = cudaFuncGetAttributes(&a, chain_kernel<true>);
  if (e != cudaSuccess) return e;
  return cudaFuncGetAttributes(&a, acct_kernel);
}

}  // namespace pemgpu
