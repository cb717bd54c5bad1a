// replay.cu — the fused B200 epoch engine (sm_100a): one CTA per trace replica (or k CTAs per
// replica, "virtual ranks", when replicas are fewer than SMs), persistent over its E epochs.  Per
// epoch (O5):
//   A  VM events + pending installs (thread per simulated GPU)            O11, O5.3
//   B  the epoch's stream runs TMA-copied (cp.async.bulk) from the        O3
//      stream-sorted trace copy (partition.cu) into shared memory
//   C  batch formation, warp per (model, class) stream; id-order ranks   O3
//   D  round-robin dispatch (closed form when every GPU is available)    Q18
//   E  placement units, lane per MIG slice: a lane group = one geometry  O6 + O8 (Alg 1, Eq 1/2,
//      (actual state, or a candidate replayed from idle); group shuffles  the "Oracle" P:L485)
//      give BE memory, live count and the min-loc of the slice keys;
//      N3 container pools ahead of each actual placement                 R22-R27
//   F  per-request accounting: SLO hits, log-linear histogram updates    O7
//   G  argmin (or Alg 2's heuristic, policy 2) + hysteresis + ~30% cap   O9, O10
//      with the mode-G / virtual-rank min-loc exchange when ranks > 1    S8
// The caller's trace (5 B/request) is read from HBM once by the partition passes and the
// stream-sorted copy (4 B/request) once by this kernel; everything else lives in shared memory,
// registers and L1-resident scratch.
#include <cuda_runtime.h>
#include <mutex>

#include "replay.cuh"
#include "place_group.cuh"
#include "chain_state.cuh"
#ifndef PROTEAN_D_BARRIER
#define PROTEAN_D_BARRIER 1
#endif
#ifndef PROTEAN_ACCT_UNROLL
#define PROTEAN_ACCT_UNROLL 1  // measured (4096 x 120 s): 4 -> 38.2, 2 -> 38.7, 1 -> 37.1 ms (code size)
#endif
#ifndef PROTEAN_RANK_UNROLL
#define PROTEAN_RANK_UNROLL 4  // 1 -> 38.9 ms
#endif
#ifndef PROTEAN_WARP_G
#define PROTEAN_WARP_G 1
#endif
#ifndef PROTEAN_FEW_WARPS
#define PROTEAN_FEW_WARPS 16  // warps per CTA in the few-replica instances
#endif
#ifndef PROTEAN_FEW_AG
#define PROTEAN_FEW_AG 1  // GPUs per actual-placement warp in the few-replica instances
#endif
#ifndef PROTEAN_FEW_NMAX
#define PROTEAN_FEW_NMAX 16  // up to this many sim-GPUs the few-replica instances use PROTEAN_FEW_AG
#endif
#ifndef PROTEAN_MINB
#define PROTEAN_MINB 3
#endif
#ifdef PROTEAN_PHASE_TIMING  // debug build only: per-phase wall cycles between CTA barriers
__device__ unsigned long long g_phase_cycles[16];
#define PH(k)                                   \
  do {                                          \
    if (threadIdx.x == 0) {                     \
      const long long t_ = clock64();           \
      ph_acc[k] += (unsigned long long)(t_ - ph_last); \
      ph_last = t_;                             \
    }                                           \
  } while (0)
#else
#define PH(k) do {} while (0)
#endif

namespace pemgpu {

namespace {

using namespace pg;
constexpr int kMaxWarps = 32;

struct CtaState {
  int64_t nlog;
  int nb, cursor, all_avail, bad;
  int task, adone;
  int task_r[2];            // PROTEAN_ACCT_BARRIER debug build: the two rounds' task counters
  int glo, ghi, cw, xrank;  // this CTA's candidate geometry range, its candidate warps per GPU and
                            // its rank in the key exchange (virtual ranks: several CTAs per replica)
  int wtot;
  int nact;                 // active streams of the epoch (s_act)
  unsigned long long cold;  // N3 cold starts of the replica          // window entries copied this epoch (incl. alignment padding)
  unsigned long long cnt[10];
};

// ------------------------------------------------------------------ mode G exchange (S8, §8(e))
__device__ __forceinline__ uint64_t global_ns() {
  uint64_t t;
  asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
  return t;
}

// Per (replica r, sequence seq): publish this rank's {best, current} key pairs of every sim-GPU
// into every rank's buffer (peer stores over NVLink), release a flag per destination, acquire
// every source's flag, then take the min of each pair over sources into gi rows 6 (best) and 7
// (current geometry's key).  Called by the whole CTA (contains barriers).
static __device__ __noinline__ void exchange_keys(XLayout X, char* const* xpeer, int xrank,
                                                   int* err, uint64_t timeout_ns, int64_t* gi,
                                                   int N, int r, uint32_t seq, int tid, int NT) {
  const int par = (int)(seq & 1u);
  __syncthreads();  // gi row 6 of every sim-GPU is final
  for (int i = tid; i < N * X.n; i += NT) {  // (gpu, destination) pairs
    const int g = i % N, dst = i / N;
    const int64_t kb = gi[6 * N + g], kc0 = gi[7 * N + g];
    const int64_t kc = kc0 >= 0 ? kc0 : kForever;
    longlong2* d = reinterpret_cast<longlong2*>(xpeer[dst] + X.key_off(par, xrank, r, g));
    *d = make_longlong2(kb, kc);
  }
  __threadfence_system();
  __syncthreads();
  if (tid < X.n) {  // release: the pairs above are visible before the flag
    uint32_t* f = reinterpret_cast<uint32_t*>(xpeer[tid] + X.flag_off(xrank, r));
    asm volatile("st.release.sys.global.u32 [%0], %1;" ::"l"(f), "r"(seq + 1u) : "memory");
  }
  if (tid < X.n && *(volatile int*)(err + 1) == 0) {  // acquire every source's flag (fail fast
    // once any wait of this call timed out)
    const uint32_t* f = reinterpret_cast<const uint32_t*>(xpeer[xrank] + X.flag_off(tid, r));
    const uint64_t t0 = global_ns();
    for (;;) {
      uint32_t v;
      asm volatile("ld.acquire.sys.global.u32 %0, [%1];" : "=r"(v) : "l"(f) : "memory");
      if ((int32_t)(v - (seq + 1u)) >= 0) break;
      if (global_ns() - t0 > timeout_ns) {
        atomicOr(err + 1, 1);
        break;
      }
      __nanosleep(256);
    }
  }
  __syncthreads();
  const char* mine = xpeer[xrank];
  for (int g = tid; g < N; g += NT) {
    int64_t kb = kForever, kc = kForever;
    for (int src = 0; src < X.n; ++src) {
      const longlong2 v = __ldcv(reinterpret_cast<const longlong2*>(mine + X.key_off(par, src, r, g)));
      kb = v.x < kb ? v.x : kb;
      kc = v.y < kc ? v.y : kc;
    }
    gi[6 * N + g] = kb;
    gi[7 * N + g] = kc;
  }
  __syncthreads();
}

// ---- N3: the Autoscaler's container pools (readings R22-R27).  Per CTA slot
// in global scratch: busy-until [N][M][kPoolCap] int64, size [N][M] and surplus counter [N][M] int32.
struct Pools {
  int64_t* bu;
  int32_t* sz;
  int32_t* ctr;
  int M;
  __device__ __forceinline__ size_t pm(int g, int m) const { return (size_t)g * M + m; }
};

__device__ __forceinline__ void pool_reset(const ReplayParams& P, const Pools& pl, int g) {  // R22
  for (int m = 0; m < pl.M; ++m) {
    for (int i = 0; i < P.prewarm; ++i) pl.bu[pl.pm(g, m) * kPoolCap + i] = 0;
    pl.sz[pl.pm(g, m)] = P.prewarm;
    pl.ctr[pl.pm(g, m)] = 0;
  }
}

// R23: the first container of (g, m) idle at t, else a new one after a cold start.  Called by every
// lane of an actual-placement warp; the 8 lanes of a GPU's group scan its pool 8 entries at a time
// (one coalesced 64-byte load), a ballot finds the first idle one.  `part`: this lane's group
// places a batch now.  Returns the container index (-1: pool full, err[2]) and *t_eff = t or
// t + cold_us, identical on every lane of the group; the group leader counts the cold start.
__device__ __forceinline__ int pool_acquire(const ReplayParams& P, const Pools& pl, bool part, int g, int m,
                                            int64_t t, int lane, int gbase, int64_t* t_eff,
                                            unsigned long long* cold) {
  const size_t k = part ? pl.pm(g, m) : 0;
  const int64_t* b = pl.bu + k * kPoolCap;
  const int n = part ? pl.sz[k] : 0;
  int found = -1;
#pragma unroll 1
  for (int base = 0;; base += 8) {
    const bool left = part && found < 0 && base < n;
    if (!__any_sync(0xffffffffu, left)) break;
    const int i = base + (lane & 7);
    const bool hit = left && i < n && b[i] <= t;
    const unsigned gm = (__ballot_sync(0xffffffffu, hit) >> gbase) & 0xFFu;
    if (left && gm) found = base + __ffs(gm) - 1;
  }
  *t_eff = t;
  if (!part || found >= 0) return found;
  *t_eff = t + P.cold_us;  // a new container (reactive scale-up)
  if (lane == gbase) *cold += 1;
  if (n >= kPoolCap) {
    if (lane == gbase) atomicOr(&P.err[2], 1);
    return -1;
  }
  if (lane == gbase) {
    pl.bu[k * kPoolCap + n] = t;
    pl.sz[k] = n + 1;
  }
  return n;
}

// R26: at the epoch end, pools larger than the epoch's batch count n_c for keepalive_epochs
// consecutive epochs terminate their surplus containers idle at T (stable compaction).
__device__ __forceinline__ void pool_terminate(const ReplayParams& P, const Pools& pl, const Ctx& c, int g, int m,
                                               const Bat* bats, const uint32_t* gl, int64_t T) {
  int need = 0;
  for (int x = c.g_off[g]; x < c.g_off[g + 1]; ++x) need += (((bats[gl[x]].info >> 16) & 0xFF) == (uint32_t)m) ? 1 : 0;
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

// Bulk L2 prefetch (TMA engine, sm_90+): [p, p + bytes) rounded out to 16-byte boundaries.
__device__ __forceinline__ void prefetch_l2(const void* p, int64_t bytes) {
  if (bytes <= 0) return;
  uintptr_t a = reinterpret_cast<uintptr_t>(p) & ~(uintptr_t)15;
  uintptr_t e = (reinterpret_cast<uintptr_t>(p) + (uintptr_t)bytes + 15) & ~(uintptr_t)15;
  while (a < e) {
    const uint32_t n = (uint32_t)((e - a) > (1u << 20) ? (1u << 20) : (e - a));
    asm volatile("cp.async.bulk.prefetch.L2.global [%0], %1;" ::"l"(a), "r"(n) : "memory");
    a += n;
  }
}

#ifndef PROTEAN_KKR
#define PROTEAN_KKR 7  // measured: 5 -> 41.2, 6 -> 39.8, 7 -> 39.5, 8 -> 40.1 ms (4096 x 120 s)
#endif
constexpr int kKR = PROTEAN_KKR;
constexpr int kAcctUnroll = PROTEAN_ACCT_UNROLL, kRankUnroll = PROTEAN_RANK_UNROLL;  // batches per GPU-epoch handled by the register fast path
constexpr int kAK = 4;  // batch ranks per accounting task (phase F)
constexpr int kBW = 1;  // the warp that lays out the next epoch's windows (phase B) during G

// Candidate unit, fast path: the GPU-epoch's <= kKR batches fully unrolled, times 32-bit relative to
// the first batch's ready time tb.  Every lane of a geometry's group keeps the whole placement so
// far (end en[x], footprint / BE flag mm[x], FBR on the lane's own profile fb[x], and the mask of
// batches on its own slice), so the GPU-wide quantities of Alg 1 -- live residents (reading Q39)
// and BE memory for the tag walk (lines 1-8) -- need no shuffles; only the slice min-loc does.
// Returns false (warp-uniform) if a completion does not fit 25 bits; the caller then re-runs the
// unit on the 64-bit path.  Same arithmetic as candidate_unit_regs (Eq 1 exact integers, Q10-Q12).
__device__ __forceinline__ uint32_t group_min32(uint32_t v, int Z) {
#pragma unroll
  for (int d = 1; d < 8; d <<= 1) {
    const uint32_t o = __shfl_xor_sync(0xffffffffu, v, d);
    if (d < Z && o < v) v = o;
  }
  return v;
}

__device__ __forceinline__ bool candidate_unit_fast(const Tab& T, const SliceLane& K, bool active,
                                                    bool leader, const Bat* bats, const uint32_t* gl,
                                                    int x0, int len, const uint32_t* sarr, int max_live,
                                                    int64_t* misses_out, int64_t* tail_out) {
  uint32_t en[kKR], mm[kKR];
  int32_t fb[kKR];
  uint32_t mine = 0, rls = 0;
  bool ok = true;
  int64_t misses = 0, tail = 0;
  const int lane = threadIdx.x & 31;
  const int gbase = lane & ~(K.Z - 1);
  const uint32_t tb = len > 0 ? bats[gl[x0]].ready : 0u;
#pragma unroll
  for (int x = 0; x < kKR; ++x) {
    if (x >= len) break;
    const Bat& bt = bats[gl[x0 + x]];
    const uint32_t info = bt.info;
    const int m = (info >> 16) & 0xFF, nreq = info & 0xFFFF;
    const bool strict = (info >> 24) & 1;
    const uint32_t rt = bt.ready - tb;
    const uint32_t rt0 = rt > rls ? rt : rls;
    int32_t used = 0, be = 0, live = 0, fs = 0;
#pragma unroll
    for (int i = 0; i < x; ++i) {
      const bool alive = en[i] > rt;
      live += alive ? 1 : 0;
      if (alive && (mm[i] >> 24)) be += (int32_t)(mm[i] & kMemMask);
      if (((mine >> i) & 1u) && en[i] > rt0) {
        used += (int32_t)(mm[i] & kMemMask);
        fs += fb[i];
      }
    }
    const int32_t q = T.mem[m];
    const int32_t fbm = K.fbr_p[m * kNProf];
    const bool overflow = live >= max_live;
    uint32_t key = 0xFFFFFFFFu, start = 0, c = 0;
    if (active && !overflow && q <= K.Ms) {
      int64_t F = fbm;
      if (used + q <= K.Ms) {
        start = rt0;
        F += fs;
      } else {  // memory wait: the earliest release on this slice after which the batch fits --
                // releases after rt0 in ascending order, the held footprint only shrinks, so the
                // first that fits is the minimum (ends at the last release: q <= Ms).  A rolled
                // walk (O(x) code per batch, not O(x^2)): the unrolled form cost i-cache space.
        uint32_t e = rt0;
#pragma unroll 1
        for (;;) {
          uint32_t nxt = 0xFFFFFFFFu;
#pragma unroll
          for (int i = 0; i < x; ++i)
            if (((mine >> i) & 1u) && en[i] > e && en[i] < nxt) nxt = en[i];
          e = nxt;
          int32_t rem = 0;
#pragma unroll
          for (int i = 0; i < x; ++i)
            if (((mine >> i) & 1u) && en[i] > e) rem += (int32_t)(mm[i] & kMemMask);
          if (rem + q <= K.Ms) break;
        }
        start = e;
#pragma unroll
        for (int i = 0; i < x; ++i)
          if (((mine >> i) & 1u) && en[i] > start) F += fb[i];
      }
      const int64_t c64 = (int64_t)start + exec_time(K.solo_p[m * kNProf], F);
      ok &= c64 < (int64_t)(1 << 25);
      c = (uint32_t)c64;
      key = strict ? (((be >= K.pref) ? 0x80000000u : 0u) | (c << 6) | ((uint32_t)(4 - K.p) << 3) | (uint32_t)K.s)
                   : ((start << 3) | (uint32_t)K.s);
    }
    const uint32_t kmin = group_min32(key, K.Z);
    const bool placed = !overflow && kmin != 0xFFFFFFFFu;
    const uint32_t cwin = __shfl_sync(0xffffffffu, c, (gbase + (int)(kmin & 7)) & 31);
    en[x] = placed ? cwin : 0u;
    mm[x] = (uint32_t)q | (strict ? 0u : 0x1000000u);
    fb[x] = fbm;
    if (placed && key == kmin) {  // schedule(batch, chosen_slice)
      mine |= 1u << x;
      rls = start;
    }
    if (leader) {
      const int64_t cw = (int64_t)tb + (int64_t)cwin;
      if (strict) {
        if (!placed) {
          misses += nreq;
        } else {  // latencies fall along the sorted members: test the ends first
          const uint32_t* ma = sarr + bt.pos;
          const int64_t slo = T.slo[m];
          if (cw - (int64_t)ma[0] > slo)
            misses += (cw - (int64_t)ma[nreq - 1] > slo) ? nreq : nreq - hits_in(ma, nreq, cw, slo);
        }
      } else {
        const int64_t tbv = placed ? cw - (int64_t)sarr[bt.pos] : (int64_t)0xFFFFFFFFLL;
        tail = tbv > tail ? tbv : tail;
      }
    }
  }
  *misses_out = misses;
  *tail_out = tail;
  return __all_sync(0xffffffffu, ok);
}

}  // namespace

// The n-th (0-based) set bit of m (n < popcount(m)).
__device__ __forceinline__ int nth_bit64(uint64_t m, int n) {
  const uint32_t lo = (uint32_t)m;
  const int pl = __popc(lo);
  return n < pl ? (int)__fns(lo, 0, n + 1) : 32 + (int)__fns((uint32_t)(m >> 32), 0, n - pl + 1);
}

// Fold the per-warp request counters of the epoch (phase F) into the replica's 64-bit counters
// 0..6 (O7) and clear them; called by all lanes of warp 0 after the phase-E barrier.
__device__ __forceinline__ void fold_wcnt(CtaState& cs, uint32_t (*wcnt)[5], int NW, int lane) {
  uint32_t v = 0;
  if (lane < 5) {
#pragma unroll 1
    for (int w = 0; w < NW; ++w) {
      v += wcnt[w][lane];
      wcnt[w][lane] = 0;
    }
  }
  const uint32_t sarr = __shfl_sync(0xffffffffu, v, 0), met = __shfl_sync(0xffffffffu, v, 1);
  const uint32_t sdrop = __shfl_sync(0xffffffffu, v, 2), barr = __shfl_sync(0xffffffffu, v, 3);
  const uint32_t bdrop = __shfl_sync(0xffffffffu, v, 4);
  if (lane == 0) {
    cs.cnt[0] += sarr;
    cs.cnt[1] += met;
    cs.cnt[2] += sarr - met - sdrop;
    cs.cnt[3] += sdrop;
    cs.cnt[4] += barr;
    cs.cnt[5] += barr - bdrop;
    cs.cnt[6] += bdrop;
  }
}

// Policy 2 (N1): Alg 2 GPU_Reconfigurator lines 1-23 for decidable GPU g, readings
// R10-R15 of DESIGN.md.  Returns final_geometry; advances the GPU's EWMA history (gi rows 12, 13).
__device__ __forceinline__ int alg2_final_geometry(const ReplayParams& P, const Ctx& c, int g,
                                                const Bat* bats, const uint32_t* gl) {
  int64_t be_num = 0, be_mem = 0;  // line 2: the BE batches dispatched to g this epoch (R10)
#pragma unroll 1
  for (int x = c.g_off[g]; x < c.g_off[g + 1]; ++x) {
    const uint32_t info = bats[gl[x]].info;
    if ((info >> 24) & 1u) continue;
    be_num += 1;
    be_mem += c.T.mem[(info >> 16) & 0xFFu];  // footprint per batch (Q36)
  }
  // lines 8-9: EWMA in milli-units (R11)
  const int64_t a = P.ewma_a;
  const int64_t X = (a * 1000 * be_num + (1000 - a) * c.gi[12 * c.N + g]) / 1000;
  const int64_t Y = (a * 1000 * be_mem + (1000 - a) * c.gi[13 * c.N + g]) / 1000;
  c.gi[12 * c.N + g] = X;
  c.gi[13 * c.N + g] = Y;
  // lines 10-18: the first of [[1g,2g],[3g]] whose summed T2 capacity holds pred_BE_mem (R12)
  const bool fits12 = (int64_t)(c.T.cap[0] + c.T.cap[1]) * 1000 >= Y;
  const bool found = fits12 || (int64_t)c.T.cap[2] * 1000 >= Y;
  // lines 19-23: thresholds on pot_occupancy = pred_BE_num (R13, R14), (4g,3g) fallback, + 4g (R15)
  if (!found || X < P.t_low || X > P.t_high) return P.g43;
  return fits12 ? P.g421 : P.g43;
}

// kAlg2: the policy-2 instance (N1).  A separate instance keeps Alg 2's code out of the search
// kernel's register allocation (measured: a shared instance costs the search path 1.5%).
// kPL = 4 marks the few-replica instances: 16 warps, one CTA per SM (actual-placement chains and
// candidate chains of a replica run side by side); kPL = 1: 8 warps, 3 CTAs per SM.
template <bool kAlg2, bool kN3, int kPL>
__global__ void __launch_bounds__(kPL == 4 ? 32 * PROTEAN_FEW_WARPS : 32 * PROTEAN_WARPS,
                                  kPL == 4 ? 1 : PROTEAN_MINB) replay_kernel(ReplayParams P) {
  extern __shared__ __align__(16) unsigned char smem[];
  __shared__ CtaState cs;
  __shared__ uint32_t s_hist[2 * kNB];  // 2 classes x 3328 buckets (u32 < 2^32 per replica)
  __shared__ uint32_t s_sink;           // target of increments with nothing to count
  // per-warp request counters of the current epoch (O7): strict arrivals, strict met, strict
  // dropped, BE arrivals, BE dropped; each warp adds only to its own row (no atomics), warp 0 folds
  // them into the 64-bit replica counters once per epoch (an epoch holds < 2^25 requests)
  __shared__ uint32_t s_wcnt[kMaxWarps][5];
  const uint32_t sink = (uint32_t)__cvta_generic_to_shared(&s_sink);
  __shared__ __align__(8) uint64_t s_mbar;  // TMA bulk-copy completion of the epoch's window
  __shared__ int s_base[kMaxStreams], s_tot[kMaxStreams], s_cur[kMaxStreams], s_pend[kMaxStreams];
  __shared__ int s_dst[kMaxStreams], s_alo[kMaxStreams], s_asz[kMaxStreams];
  __shared__ uint8_t s_act[kMaxStreams];  // streams with requests in this epoch's window (phase C)
#ifdef PROTEAN_PHASE_TIMING
  unsigned long long ph_acc[10] = {0, 0, 0, 0, 0, 0, 0, 0, 0, 0};
  long long ph_last = clock64();
#endif
  const SmemLayout& SL = P.sl;
  const int tid = threadIdx.x, NT = blockDim.x, lane = tid & 31, warp = tid >> 5, NW = NT >> 5;
  const int N = P.N, S = SL.S, Gc = SL.Gc;  // Gc: key stride (the largest range of any CTA)
  // virtual ranks (P.vr_n > 1): CTA b serves replica b / vr_n and scores geometry range b % vr_n,
  // exchanging min-loc keys with the replica's other CTAs exactly as mode G ranks do
  const int vrn = P.vr_n > 1 ? P.vr_n : 1;
  const int vr = (int)(blockIdx.x % (unsigned)vrn);
  const int glo = vrn > 1 ? P.vr_lo[vr] : P.geom_lo, ghi = vrn > 1 ? P.vr_hi[vr] : P.geom_hi;
  const int cwr = vrn > 1 ? P.vr_cw[vr] : SL.CW;
  // the few-replica instances split the replica's accounting over its virtual ranks (the
  // many-replica instance, where virtual ranks are an explicit request, replicates it)
  const bool vsplit = kPL == 4 && vrn > 1;
  const uint32_t* pack_src = vrn > 1 ? P.vr_pack[vr] : P.pack;
  if (tid == 0) {
    cs.glo = glo;
    cs.ghi = ghi;
    cs.cw = cwr;
    cs.xrank = vrn > 1 ? vr : P.xrank;
  }

  Ctx c;
  int32_t* tabw = reinterpret_cast<int32_t*>(smem + SL.tab);
#pragma unroll 1
  for (int i = tid; i < P.tl.words; i += NT) tabw[i] = P.tab[i];
  uint32_t* packs = reinterpret_cast<uint32_t*>(smem + SL.pack);
#pragma unroll 1
  for (int i = tid; i < cwr * 32; i += NT) packs[i] = pack_src[i];
  const uint32_t mbar = (uint32_t)__cvta_generic_to_shared(&s_mbar);
  if (tid == 0) {
    asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" ::"r"(mbar) : "memory");
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
  }
  uint32_t mphase = 0;  // parity of the window barrier's next phase (uniform)
  c.T.bind(tabw, P.tl);
  c.pack = packs;
  c.N = N;
  c.gu8 = smem + SL.g_u8;
  c.gi = reinterpret_cast<int64_t*>(smem + SL.g_i64);
  c.g_cnt = reinterpret_cast<int*>(smem + SL.g_i32);
  c.g_off = c.g_cnt + N;
  c.a_n = reinterpret_cast<int*>(smem + SL.a_n);
  c.a_ls = reinterpret_cast<int64_t*>(smem + SL.a_ls);
  c.a_bu = reinterpret_cast<int64_t*>(smem + SL.a_bu);
  c.keys = reinterpret_cast<int64_t*>(smem + SL.keys);
  c.BS = SL.BS;
  c.sb = reinterpret_cast<Bat*>(smem + SL.bats);
  c.sord = reinterpret_cast<uint32_t*>(smem + SL.ord);
  c.sgl = reinterpret_cast<uint32_t*>(smem + SL.glist);
  char* slot = P.scratch + (size_t)blockIdx.x * P.slot_bytes;
  Pools pl;  // N3 container pools (kN3 instance only)
  pl.bu = reinterpret_cast<int64_t*>(slot + P.o_pool);
  pl.sz = reinterpret_cast<int32_t*>(slot + P.o_pool + (size_t)N * P.tl.M * kPoolCap * 8);
  pl.ctr = pl.sz + (size_t)N * P.tl.M;
  pl.M = P.tl.M;
  c.gb = reinterpret_cast<Bat*>(slot + P.o_gbat);
  c.gord = reinterpret_cast<uint32_t*>(slot + P.o_gord);
  c.ggl = reinterpret_cast<uint32_t*>(slot + P.o_gglist);
  const bool win_smem = SL.WS > 0;  // the epoch window in shared memory (else global scratch)
  c.sarr = win_smem ? reinterpret_cast<uint32_t*>(smem + SL.sarr) : reinterpret_cast<uint32_t*>(slot + P.o_gsarr);
  // resident lists: actual lanes [N*8 lanes][max_live] (x 4 sub-lanes in the few-replica instances
  // with one GPU per warp), candidate lanes [NT lanes][max_live]
  const bool subm = kPL == 4 && !kN3 && N <= PROTEAN_FEW_NMAX && PROTEAN_FEW_AG == 1;
  const int NA = N * kZA * (subm ? 4 : 1);
  LaneList AL;
  AL.stride = NA;
  AL.st = reinterpret_cast<int64_t*>(slot + P.o_alist);
  AL.en = AL.st + (size_t)NA * P.max_live;
  AL.mm = reinterpret_cast<uint32_t*>(AL.en + (size_t)NA * P.max_live);
  LaneList CL;
  CL.stride = NT;
  CL.st = reinterpret_cast<int64_t*>(slot + P.o_clist) + tid;
  CL.en = CL.st + (size_t)NT * P.max_live;
  CL.mm = reinterpret_cast<uint32_t*>(reinterpret_cast<int64_t*>(slot + P.o_clist) + 2 * (size_t)NT * P.max_live) + tid;
  const Tab& T = c.T;
  __syncthreads();
  int sum_slots = 0;  // slot-evals per batch per decidable GPU
#pragma unroll 1
  for (int j = glo; j < ghi; ++j) sum_slots += T.gn[j];
  // actual-placement warp units: AG GPUs x 8 slice lanes.  Few-replica launches (long lists, slow
  // paths common) give each GPU its own warp, so one GPU's slow path never serialises another's
  // (up to 16 sim-GPUs; beyond, 64-GPU configs keep 4 per warp: more units than warps cost more)
  const int AG = (kPL == 4 && N <= PROTEAN_FEW_NMAX) ? PROTEAN_FEW_AG : kAG;
  const int n_aunits = (N + AG - 1) / AG;
  const uint32_t* sarr = c.sarr;

#pragma unroll 1
  for (int r = (int)(blockIdx.x / (unsigned)vrn); r < P.R; r += (int)(gridDim.x / (unsigned)vrn)) {
    const uint64_t replica = (uint64_t)(P.base + r);
    uint32_t* ghist = P.hist + (size_t)r * 2 * kNB;

    // ---------------------------------------------------------------- replica init
#pragma unroll 1
    for (int i = tid; i < 2 * kNB; i += NT) s_hist[i] = 0;
#pragma unroll 1
    for (int i = tid; i < kMaxWarps * 5; i += NT) (&s_wcnt[0][0])[i] = 0;
#pragma unroll 1
    for (int k = tid; k < S; k += NT) s_cur[k] = (int)P.sidx[(size_t)r * (P.E + 1) * S + k];
#pragma unroll 1
    for (int g = tid; g < N; g += NT) {
      reset_gpu_state(c, g, P.init_geom);
      c.gu8[3 * c.N + g] = c.gu8[4 * c.N + g] = (P.vm_policy == 0) ? VM_OD : VM_SPOT;
      c.gi[0 * c.N + g] = c.gi[1 * c.N + g] = 0;
      c.gi[2 * c.N + g] = 0;
      c.gi[3 * c.N + g] = kForever;
      c.gi[4 * c.N + g] = 0;
      c.gi[8 * c.N + g] = c.gi[9 * c.N + g] = c.gi[10 * c.N + g] = c.gi[11 * c.N + g] = 0;
      c.gi[12 * c.N + g] = c.gi[13 * c.N + g] = 0;  // Alg 2 EWMA history (policy 2)
      if constexpr (kN3) pool_reset(P, pl, g);
    }
    if (tid == 0) {
      cs.nlog = 0;
      cs.cursor = 0;
      cs.bad = 0;
      cs.task = 0;  // per-epoch scratch, re-armed at the end of every epoch
      cs.task_r[0] = cs.task_r[1] = 0;
      cs.adone = 0;
      cs.nb = 0;
      cs.all_avail = 1;
      cs.cold = 0;
#pragma unroll
      for (int i = 0; i < 10; ++i) cs.cnt[i] = 0;
    }
    __syncthreads();

    // ---------------------------------------------------------------- A: VM events, installs
    // (warp 0, lane = simulated GPU), for epoch ee; runs right after G of epoch ee - 1 in the same
    // warp (program order: the windows G opened are visible), overlapping B of epoch ee in warp kBW
    auto phase_a = [&](int64_t ee) {
      const int64_t eW = ee * P.W, Tend = eW + P.W;
#pragma unroll 1
      for (int g = lane; g < N; g += 32) {
        if (P.vm_policy != 0) {
#pragma unroll 1
          for (int64_t k = (eW + P.rev - 1) / P.rev; k * P.rev < Tend; ++k) {
            const int64_t tau = k * P.rev;
            if (k < 1 || tau >= P.H) continue;
            if (c.gu8[1 * c.N + g] != kNoGeom && c.gi[1 * c.N + g] <= tau) reset_gpu_state(c, g, c.gu8[1 * c.N + g]);
            const bool lost = vm_event(P, c, replica, g, k, tau);
            if constexpr (kN3) {
              if (lost) pool_reset(P, pl, g);
            }
          }
        }
        if (c.gu8[1 * c.N + g] != kNoGeom && c.gi[1 * c.N + g] <= Tend) reset_gpu_state(c, g, c.gu8[1 * c.N + g]);
        c.gu8[5 * c.N + g] = (has_vm(c, g, Tend) && c.gi[1 * c.N + g] <= Tend) ? 1 : 0;
        c.gu8[7 * c.N + g] = 0;
        c.gu8[6 * c.N + g] = kNoGeom;
        c.gi[7 * c.N + g] = -1;
        const bool whole = c.gi[2 * c.N + g] <= eW && c.gi[3 * c.N + g] >= Tend &&
                           !(c.gi[0 * c.N + g] < Tend && c.gi[1 * c.N + g] > eW);
        if (!whole) cs.all_avail = 0;  // set to 1 before the previous epoch's last barrier
      }
    };
    // ---------------------------------------------------------------- B: stream windows
    // Stream k's unbatched requests are [s_cur[k], sidx[r][e+1][k]) of the stream-sorted copy
    // (partition.cu).  Warp kBW lays the streams out contiguously in the window (each as its
    // 16-byte aligned superset) and, for a shared-memory window, every lane issues its streams'
    // TMA bulk copies (cp.async.bulk global -> shared, completion on one mbarrier); the next
    // epoch's new requests are prefetched into L2 meanwhile.  A global-scratch window (too large
    // for shared memory) is filled by a cooperative 16-byte copy after the barrier instead.
    // B of epoch e + 1 runs while warp 0 decides epoch e (G): it reads only s_cur (final after
    // epoch e's formation) and overwrites the window, which no phase after E reads.
    const uint32_t* sa_r = P.sa + P.saoff[r];
    int64_t* kst = reinterpret_cast<int64_t*>(smem + SL.kst);  // [2][N*G] precomputed keys (cand.cu)
    auto phase_b = [&](int64_t ee) {
      if (P.kfc) {  // the epoch's candidate keys by residue class; G of epoch ee - 1 reads the other half
        const int KS = SL.KS;
        const int64_t* src = P.kfc + ((size_t)r * P.E + ee) * KS;
        int64_t* dst = kst + (ee & 1) * KS;
#pragma unroll 1
        for (int i = lane; i < KS; i += 32) dst[i] = __ldg(src + i);
      }
      {
        const uint32_t* s1 = P.sidx + ((size_t)r * (P.E + 1) + ee + 1) * S;
        int carry = 0, nact = 0;
#pragma unroll 1
        for (int k0 = 0; k0 < S; k0 += 32) {
          const int k = k0 + lane;
          int cur = 0, len = 0, alo = 0, asz = 0;
          if (k < S) {
            cur = s_cur[k];
            const int hi = (int)s1[k];
            len = hi - cur;
            alo = cur & ~3;
            asz = len > 0 ? ((hi + 3) & ~3) - alo : 0;
            if (ee + 1 < P.E) {  // the next epoch's new requests: into L2 during this one
              const int h2 = (int)s1[S + k];
              if (h2 > hi) prefetch_l2(sa_r + hi, (int64_t)(h2 - hi) * 4);
            }
          }
          int x = asz;
#pragma unroll
          for (int d = 1; d < 32; d <<= 1) {
            const int y = __shfl_up_sync(0xffffffffu, x, d);
            if (lane >= d) x += y;
          }
          const int dst = carry + x - asz;
          if (k < S) {
            s_base[k] = dst + (cur - alo);
            s_tot[k] = len > 0 ? len : 0;
            s_dst[k] = dst;
            s_alo[k] = alo;
            s_asz[k] = asz;
            s_pend[k] = 0;
          }
          const unsigned am = __ballot_sync(0xffffffffu, k < S && len > 0);
          if (k < S && len > 0) s_act[nact + __popc(am & ((1u << lane) - 1u))] = (uint8_t)k;
          nact += __popc(am);
          carry += __shfl_sync(0xffffffffu, x, 31);
        }
        const bool overflow = carry > P.WCAP;  // cannot happen for a valid trace (host bound)
        if (overflow) {
          for (int k = lane; k < S; k += 32) s_tot[k] = 0;
          if (lane == 0) atomicOr(P.err, 1);
        }
        if (lane == 0) cs.nact = overflow ? 0 : nact;
        const int tot = overflow ? 0 : carry;
        if (lane == 0) cs.wtot = tot;
        if (win_smem && tot > 0) {
          asm volatile("fence.proxy.async.shared::cta;" ::: "memory");  // prior generic accesses
          __syncwarp();
#pragma unroll 1
          for (int k = lane; k < S; k += 32) {
            const int asz = s_asz[k];
            if (asz > 0) {
              const uint32_t dsts = (uint32_t)__cvta_generic_to_shared(c.sarr + s_dst[k]);
              asm volatile(
                  "cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];"
                  ::"r"(dsts), "l"(sa_r + s_alo[k]), "r"(asz * 4), "r"(mbar) : "memory");
            }
          }
          if (lane == 0)
            asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(mbar), "r"(tot * 4) : "memory");
        }
      }
    };
    // e = -1 only prepares epoch 0 (A and B below); one call site each keeps one inlined copy
#pragma unroll 1
    for (int64_t e = -1; e < P.E; ++e) {
      const int64_t eW = e * P.W, Tend = eW + P.W;
      (void)eW;
      if (e >= 0) {
      __syncthreads();
      PH(1);
      if (win_smem) {
        if (cs.wtot > 0) {  // uniform: wait for this epoch's bulk copies
          uint32_t done = 0;
          while (!done)
            asm volatile("{\n\t.reg .pred p;\n\tmbarrier.try_wait.parity.shared::cta.b64 p, [%1], %2;\n\t"
                         "selp.u32 %0, 1, 0, p;\n\t}"
                         : "=r"(done) : "r"(mbar), "r"(mphase) : "memory");
          mphase ^= 1u;
        }
      } else {
#pragma unroll 1
        for (int k = 0; k < S; ++k) {
          const int asz = s_asz[k];
          if (asz <= 0 || cs.wtot == 0) continue;
          const uint4* src = reinterpret_cast<const uint4*>(sa_r + s_alo[k]);
          uint4* dst = reinterpret_cast<uint4*>(c.sarr + s_dst[k]);
          for (int i = tid; i < asz / 4; i += NT) dst[i] = src[i];
        }
        __syncthreads();
      }
      PH(3);
      // ---------------------------------------------------------------- C: batch formation
      // warp per stream: lanes test 32 consecutive B-sized batches at once (full batches are the
      // common case); a batch closed by the timeout, or still open, is resolved by lane 0.
      const int nact = cs.nact;
#pragma unroll 1
      for (int ka = warp; ka < nact; ka += NW) {
        const int k = s_act[ka];
        const int m = k >> 1;
        const bool strict = (k & 1) == 0;
        const int B = T.bsz[m];
        const int64_t Tm = T.tmo[m];
        int i = s_base[k];
        const int end = s_base[k] + s_tot[k];
        int pend = 0;
#pragma unroll 1
        while (i < end) {
          const int64_t st = (int64_t)i + (int64_t)lane * B;
          bool full = false;
          if (st + B <= end) full = (int64_t)sarr[st + B - 1] <= (int64_t)sarr[st] + Tm;
          const unsigned fm = __ballot_sync(0xffffffffu, full);
          const int nfull = __ffs(~fm) ? __ffs(~fm) - 1 : 32;
          int slot0 = 0;
          if (lane == 0 && nfull) slot0 = atomicAdd(&cs.nb, nfull);
          slot0 = __shfl_sync(0xffffffffu, slot0, 0);
          if (lane < nfull) {
            const int ii = (int)st;
            const uint32_t ready = sarr[ii + B - 1];
            Bat& bt = c.bat_w(slot0 + lane);
            bt.key = ((uint64_t)ready << 32) | ((uint64_t)(strict ? 0 : 1) << 31) |
                     ((uint64_t)m << 25) | (uint64_t)(ii & 0x1FFFFFF);
            bt.ready = ready;
            bt.info = (uint32_t)B | ((uint32_t)m << 16) | ((uint32_t)(strict ? 1 : 0) << 24);
            bt.pos = (uint32_t)ii;
            bt.gpu = 0xFF;
            bt.slice = 0xFF;
            bt.drop = 0;
            bt.start = bt.end = 0;
          }
          i += nfull * B;
          if (nfull == 32) continue;
          if (i >= end) break;
          int j = 0, state = 0;  // state 0 emit, 1 pending
          if (lane == 0) {
            const int64_t a0 = sarr[i];
            const int64_t deadline = a0 + Tm;
            const int lim = (end - i > B) ? i + B : end;
            int lo = i + 1, hi = lim;  // first member beyond the timeout, else lim
#pragma unroll 1
            while (lo < hi) {
              const int mid = (lo + hi) >> 1;
              if ((int64_t)sarr[mid] > deadline) hi = mid; else lo = mid + 1;
            }
            j = lo;
            int64_t ready = 0;
            if (j - i == B) ready = sarr[j - 1];        // full (only at the window end)
            else if (j < end) ready = deadline;         // a later arrival missed the timeout
            else if (deadline < Tend) ready = deadline; // timed out inside this epoch
            else { state = 1; pend = end - i; }
            if (state == 0) {
              const int slot = atomicAdd(&cs.nb, 1);
              Bat& bt = c.bat_w(slot);
              bt.key = ((uint64_t)ready << 32) | ((uint64_t)(strict ? 0 : 1) << 31) |
                       ((uint64_t)m << 25) | (uint64_t)(i & 0x1FFFFFF);
              bt.ready = (uint32_t)ready;
              bt.info = (uint32_t)(j - i) | ((uint32_t)m << 16) | ((uint32_t)(strict ? 1 : 0) << 24);
              bt.pos = (uint32_t)i;
              bt.gpu = 0xFF;
              bt.slice = 0xFF;
              bt.drop = 0;
              bt.start = bt.end = 0;
            }
          }
          state = __shfl_sync(0xffffffffu, state, 0);
          j = __shfl_sync(0xffffffffu, j, 0);
          if (state) break;
          i = j;
        }
        if (lane == 0) s_pend[k] = pend;
      }
      __syncthreads();
      PH(4);
      const int nb = cs.nb;
      if (nb > c.BS) {  // rare: more batches than the smem arrays hold -> all in global scratch
#pragma unroll 1
        for (int b = tid; b < c.BS; b += NT) c.gb[b] = c.sb[b];
        c.bats = c.gb;
        c.ord = c.gord;
        c.gl = c.ggl;
        __syncthreads();
      } else {
        c.bats = c.sb;
        c.ord = c.sord;
        c.gl = c.sgl;
      }
      // the open batch's requests (if any) stay unbatched: the next epoch's window starts there
#pragma unroll 1
      for (int k = tid; k < S; k += NT) s_cur[k] += s_tot[k] - s_pend[k];
      Bat* bats = c.bats;
      uint32_t* ord = c.ord;
      uint32_t* gl = c.gl;
      // D (closed form, Q18) fused with the id-order ranking when every GPU is available all
      // epoch: rank rk goes to GPU (cursor + rk) mod N, the rk / N-th of that GPU's list; GPU h
      // receives q + [d_h < rem] batches (q, rem = nb div/mod N, d_h = (h - cursor) mod N)
      const bool avail_all = cs.all_avail;
      const int cursor = cs.cursor;
      const int dq = nb / N, drem = nb - dq * N;
      auto goff = [&](int g) {  // batches of GPUs 0..g-1
        const int wrap = cursor + drem - N;
        int x = g - cursor;
        x = x < 0 ? 0 : (x > drem ? drem : x);
        if (wrap > 0) x = min(max(g - cursor, 0), N - cursor) + min(g, wrap);
        return g * dq + x;
      };
#pragma unroll 1
      for (int b = tid; b < nb; b += NT) {  // id order (O3): rank by key
        const uint64_t kb = bats[b].key;
        int rank = 0;
#pragma unroll kRankUnroll
        for (int x = 0; x < nb; ++x) rank += (bats[x].key < kb) ? 1 : 0;
        ord[rank] = (uint32_t)b;
        if (avail_all) {
          const int q = rank / N, g = cursor + (rank - q * N);
          const int gg = g >= N ? g - N : g;
          bats[b].gpu = (uint8_t)gg;
          gl[goff(gg) + q] = (uint32_t)b;
        }
      }
      if (avail_all)
        for (int g = tid; g <= N; g += NT) c.g_off[g] = goff(g);
      __syncthreads();
      PH(5);
      if (tid == 0) {
        if (avail_all) cs.cursor = (int)((cursor + nb) % N);
      }
      // ---------------------------------------------------------------- D: dispatch
      if (avail_all) {
        // done above
      } else if (N <= 64) {
        // availability mask per batch (parallel); then runs of equal masks are dispatched in
        // closed form: inside a run the k-th batch goes to the (i0 + k) mod |A|-th available GPU
        // (i0: the first available at or after the cursor), exactly the serial round robin (O4)
        // few-replica instances (long epochs, many GPUs): masks per 32 consecutive ranks (ready
        // times ascend along the ranks): lanes hold GPUs lane and lane + 32; when no GPU's VM or
        // reconfiguration bound falls inside (t_first, t_last] the chunk shares one mask (two
        // ballots), else each rank of the chunk takes its own.  The many-replica instance keeps
        // the per-rank loop (C4: 273 -> 244 us per epoch; the larger code cost C5 1%).
        if constexpr (kPL != 4) {
#pragma unroll 1
          for (int rk = tid; rk < nb; rk += NT) {
            Bat& bt = bats[ord[rk]];
            const int64_t t = bt.ready;
            uint64_t m = 0;
#pragma unroll 1
            for (int g = 0; g < N; ++g)
              if (available(c, g, t)) m |= 1ull << g;
            bt.key = m;  // the id-order key is no longer needed
          }
        } else {
          const int g0 = lane, g1 = lane + 32;
          const int64_t v0l = g0 < N ? c.gi[2 * c.N + g0] : INT64_MAX, v0h = g0 < N ? c.gi[3 * c.N + g0] : INT64_MAX;
          const int64_t r0l = g0 < N ? c.gi[0 * c.N + g0] : 0, r0h = g0 < N ? c.gi[1 * c.N + g0] : 0;
          const int64_t v1l = g1 < N ? c.gi[2 * c.N + g1] : INT64_MAX, v1h = g1 < N ? c.gi[3 * c.N + g1] : INT64_MAX;
          const int64_t r1l = g1 < N ? c.gi[0 * c.N + g1] : 0, r1h = g1 < N ? c.gi[1 * c.N + g1] : 0;
          auto mask_at = [&](int64_t t) {  // available(c, g, t) for every g < N, as a 64-bit mask
            const bool a0 = v0l <= t && t < v0h && !(r0l <= t && t < r0h);
            const bool a1 = v1l <= t && t < v1h && !(r1l <= t && t < r1h);
            return (uint64_t)__ballot_sync(0xffffffffu, a0) | ((uint64_t)__ballot_sync(0xffffffffu, a1) << 32);
          };
#pragma unroll 1
          for (int ch = warp; ch * 32 < nb; ch += NW) {
            const int rk = ch * 32 + lane;
            const bool v = rk < nb;
            const uint32_t b = v ? ord[rk] : 0u;
            const int64_t t = v ? (int64_t)bats[b].ready : 0;
            const int last = min(32, nb - ch * 32) - 1;
            const int64_t tf = __shfl_sync(0xffffffffu, t, 0), tl = __shfl_sync(0xffffffffu, t, last);
            auto in = [&](int64_t x) { return tf < x && x <= tl; };
            const bool chg = in(v0l) || in(v0h) || in(r0l) || in(r0h) || in(v1l) || in(v1h) || in(r1l) || in(r1h);
            uint64_t m;
            if (!__any_sync(0xffffffffu, chg)) {
              m = mask_at(tf);
            } else {
              m = 0;
#pragma unroll 1
              for (int j = 0; j <= last; ++j) {
                const uint64_t mj = mask_at(__shfl_sync(0xffffffffu, t, j));
                if (lane == j) m = mj;
              }
            }
            if (v) bats[b].key = m;  // the id-order key is no longer needed
          }
        }
        __syncthreads();
        if (warp == 0) {
          int cur = cs.cursor;
#pragma unroll 1
          for (int r0 = 0; r0 < nb;) {
            const uint64_t m = bats[ord[r0]].key;
            int r1 = r0 + 1;
#pragma unroll 1
            for (;;) {  // end of the run of equal masks
              const int rk = r1 + lane;
              const unsigned dm = __ballot_sync(0xffffffffu, rk >= nb || bats[ord[rk]].key != m);
              if (dm) { r1 += __ffs(dm) - 1; break; }
              r1 += 32;
            }
            const int A = __popcll(m);
            const int i0 = A ? __popcll(m & ((1ull << cur) - 1ull)) % A : 0;  // first available >= cur
#pragma unroll 1
            for (int rk = r0 + lane; rk < r1; rk += 32) {
              Bat& bt = bats[ord[rk]];
              if (A == 0) {
                bt.gpu = 0xFF;
                bt.drop = 1;  // dispatch drop
              } else {
                bt.gpu = (uint8_t)nth_bit64(m, (i0 + (rk - r0)) % A);
              }
            }
            if (A) cur = (nth_bit64(m, (i0 + (r1 - 1 - r0)) % A) + 1) % N;
            r0 = r1;
          }
          __syncwarp();
          // per-GPU lists in id order: a warp-stable counting sort over 32 ranks at a time (peers by
          // match_any; the highest peer lane advances the GPU's running count)
          if (lane < N) c.g_cnt[lane] = 0;
          if (lane + 32 < N) c.g_cnt[lane + 32] = 0;
          __syncwarp();
#pragma unroll 1
          for (int rk0 = 0; rk0 < nb; rk0 += 32) {
            const int rk = rk0 + lane;
            const int gg = rk < nb ? bats[ord[rk]].gpu : 0xFF;
            const unsigned peers = __match_any_sync(0xffffffffu, gg);
            if (gg < N && lane == 31 - __clz(peers)) c.g_cnt[gg] += __popc(peers);
            __syncwarp();
          }
          const int c0 = lane < N ? c.g_cnt[lane] : 0, c1 = lane + 32 < N ? c.g_cnt[lane + 32] : 0;
          int x0 = c0, x1 = c1;
#pragma unroll
          for (int d = 1; d < 32; d <<= 1) {
            const int y0 = __shfl_up_sync(0xffffffffu, x0, d), y1 = __shfl_up_sync(0xffffffffu, x1, d);
            if (lane >= d) { x0 += y0; x1 += y1; }
          }
          const int t0 = __shfl_sync(0xffffffffu, x0, 31), t1 = __shfl_sync(0xffffffffu, x1, 31);
          if (lane < N) { c.g_off[lane] = x0 - c0; c.g_cnt[lane] = 0; }
          if (lane + 32 < N) { c.g_off[lane + 32] = t0 + x1 - c1; c.g_cnt[lane + 32] = 0; }
          if (lane == 0) c.g_off[N] = t0 + t1;  // dropped batches (gpu 0xFF) are in no list
          __syncwarp();
#pragma unroll 1
          for (int rk0 = 0; rk0 < nb; rk0 += 32) {
            const int rk = rk0 + lane;
            const uint32_t b = rk < nb ? ord[rk] : 0u;
            const int gg = rk < nb ? bats[b].gpu : 0xFF;
            const unsigned peers = __match_any_sync(0xffffffffu, gg);
            const int base = gg < N ? c.g_off[gg] + c.g_cnt[gg] : 0;
            __syncwarp();
            if (gg < N) {
              gl[base + __popc(peers & ((1u << lane) - 1u))] = b;
              if (lane == 31 - __clz(peers)) c.g_cnt[gg] += __popc(peers);
            }
            __syncwarp();
          }
          if (lane == 0) cs.cursor = cur;
        }
      } else if (tid == 0) {
        int cur = cs.cursor;
#pragma unroll 1
        for (int g = 0; g < N; ++g) c.g_cnt[g] = 0;
#pragma unroll 1
        for (int rk = 0; rk < nb; ++rk) {
          Bat& bt = bats[ord[rk]];
          int chosen = -1;
#pragma unroll 1
          for (int i = 0; i < N; ++i) {
            const int g = (cur + i) % N;
            if (available(c, g, bt.ready)) { chosen = g; break; }
          }
          if (chosen < 0) {
            bt.drop = 1;
            bt.gpu = 0xFF;
          } else {
            bt.gpu = (uint8_t)chosen;
            c.g_cnt[chosen]++;
            cur = (chosen + 1) % N;
          }
        }
        int off = 0;
#pragma unroll 1
        for (int g = 0; g < N; ++g) {
          c.g_off[g] = off;
          off += c.g_cnt[g];
          c.g_cnt[g] = 0;
        }
        c.g_off[N] = off;
#pragma unroll 1
        for (int rk = 0; rk < nb; ++rk) {
          const uint32_t b = ord[rk];
          const Bat& bt = bats[b];
          if (bt.drop) continue;
          gl[c.g_off[bt.gpu] + c.g_cnt[bt.gpu]++] = b;
        }
        cs.cursor = cur;
      }
      if (PROTEAN_D_BARRIER || !avail_all) __syncthreads();  // (uniform)
      PH(6);
      // ---------------------------------------------------------------- E: placement units
      // unit < n_aunits: actual placement of GPUs 4u..4u+3 (8 slice lanes each, carried state);
      // otherwise candidate warp w of GPU g: lane groups = candidate geometries from idle (O8).
      // One loop body serves both kinds (a single inlined copy of Place).
      // dynamic task queue: [actual units][candidate units][accounting of batch rank rk];
      // accounting waits (rarely) for the actual units, whose warps publish via cs.adone
      // closed-form dispatch + keys held by cand.cu: the candidate units are done (G reads kst)
      const bool pre = P.kfc && avail_all && kst[(e & 1) * SL.KS] != INT64_MIN;
      const int n_units = n_aunits + (P.policy == 0 && !pre ? N * cs.cw : 0);
      // split accounting (vsplit): CTA vr takes tasks vr, vr + vrn, ... (counters and the histogram
      // are summed in finalize); otherwise every CTA takes them all
      const int ntk = (nb + kAK - 1) / kAK;
      const int n_tasks = n_units + (vsplit ? (ntk + vrn - 1 - vr) / vrn : ntk);
#ifndef PROTEAN_ACCT_BARRIER
#define PROTEAN_ACCT_BARRIER 0  // 1: debug build for compute-sanitizer racecheck (accounting after a CTA barrier)
#endif
      constexpr int kRounds = PROTEAN_ACCT_BARRIER ? 2 : 1;
#pragma unroll 1
      for (int round = 0; round < kRounds; ++round) {
      if (PROTEAN_ACCT_BARRIER && round == 1) __syncthreads();  // every actual unit has finished
      for (;;) {
        int u = 0;
        if (lane == 0) u = PROTEAN_ACCT_BARRIER ? atomicAdd(&cs.task_r[round], 1) + (round ? n_units : 0)
                                                : atomicAdd(&cs.task, 1);
        u = __shfl_sync(0xffffffffu, u, 0);
        if (u >= (PROTEAN_ACCT_BARRIER && round == 0 ? n_units : n_tasks)) break;
#ifdef PROTEAN_PHASE_TIMING
        const long long tk0 = clock64();
        const int tkind = u >= n_units ? 2 : (u < n_aunits ? 0 : 1);
        struct TaskClock {
          long long t0; int kind; int lane; unsigned long long* acc;
          __device__ ~TaskClock() { if (lane == 0) atomicAdd(&acc[kind], (unsigned long long)(clock64() - t0)); }
        } tclock{tk0, tkind, lane, g_phase_cycles + 10};
#endif
        if (u >= n_units) {  // ---- F: accounting (O7) of batch ranks [kAK t, kAK t + kAK)
          // acquire the actual units' batch results (slice, start, end, drop): lane 0's acquire
          // load, then the warp barrier orders it before every lane's reads (PTX memory model:
          // release/acquire at CTA scope + bar.warp.sync)
          if (!PROTEAN_ACCT_BARRIER && lane == 0) {
            const uint32_t fa = (uint32_t)__cvta_generic_to_shared(&cs.adone);
            for (;;) {
              int v;
              asm volatile("ld.acquire.cta.shared::cta.s32 %0, [%1];" : "=r"(v) : "r"(fa) : "memory");
              if (v >= n_aunits) break;
              __nanosleep(64);
            }
          }
          __syncwarp();
          const int rk0 = (vsplit ? (u - n_units) * vrn + vr : u - n_units) * kAK, rk1 = min(nb, rk0 + kAK);
          uint32_t c_sarr = 0, c_met = 0, c_sdrop = 0, c_barr = 0, c_bdrop = 0;  // warp-uniform
#pragma unroll 1
          for (int rk = rk0; rk < rk1; ++rk) {
            const Bat& bt = bats[ord[rk]];
            const uint32_t info = bt.info;
            const int nreq = info & 0xFFFF, m = (info >> 16) & 0xFF;
            const bool strict = (info >> 24) & 1;
            const int drop = bt.drop;
            if (P.log && lane == 0) {
              const int64_t row = cs.nlog + rk;
              if (row < P.log_cap) {
                protean_batch_rec rec;
                rec.ready_us = bt.ready;
                rec.epoch = (uint32_t)e;
                rec.n_req = (uint16_t)nreq;
                rec.model = (uint8_t)m;
                rec.strict = strict ? 1 : 0;
                rec.gpu = bt.gpu;
                rec.slice = bt.slice;
                rec.dropped = (uint8_t)drop;
                rec.pad = 0;
                rec.start_us = bt.start;
                rec.end_us = bt.end;
                P.log[(size_t)r * P.log_cap + row] = rec;
              }
            }
            uint32_t met = 0;  // strict members within the SLO
            if (!drop) {
              const int64_t slo = T.slo[m];
              const uint32_t* ma = sarr + bt.pos;
              const int64_t bend = bt.end;
              const uint32_t hb = (uint32_t)__cvta_generic_to_shared(s_hist + (strict ? 0 : kNB));
              if (bend - (int64_t)ma[0] <= (int64_t)0xFFFFFFFFLL) {
                // every latency end - a (>= 0, <= end - a_first) fits 32 bits: lat = end - a mod 2^32;
                // bucket = 128 s + (lat >> s), s = max(0, floor(log2 lat) - 7) (O7, reading Q30)
                const uint32_t e32 = (uint32_t)bend;
                const uint32_t slo32 = slo > (int64_t)0xFFFFFFFFLL ? 0xFFFFFFFFu : (uint32_t)slo;
#pragma unroll kAcctUnroll
                for (int i0 = 0; i0 < nreq; i0 += 32) {
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
          if (lane < 5) {
            const uint32_t v = lane == 0 ? c_sarr : lane == 1 ? c_met : lane == 2 ? c_sdrop : lane == 3 ? c_barr : c_bdrop;
            s_wcnt[warp][lane] += v;
          }
          continue;
        }
        const bool actual = u < n_aunits;
        int g, s, Z, gbase, j;
        bool valid;
        if (actual) {
          g = subm ? u : u * AG + (lane >> 3);
          s = lane & 7;
          Z = kZA;
          gbase = lane & ~7;
          valid = subm ? g < N : ((lane >> 3) < AG && g < N);
          j = valid ? c.gu8[0 * c.N + g] : 0;
        } else {
          const int cw = cs.cw;
          const int cu = u - n_aunits, w = cu % cw;
          g = cu / cw;
          const uint32_t pk = c.pack[w * 32 + lane];
          const int jr = pk & 0xFF;
          s = (pk >> 8) & 0xFF;
          Z = (pk >> 16) & 0xFF;
          gbase = pk >> 24;
          valid = jr != 0xFF;
          j = valid ? jr : 0;
          if (!c.gu8[5 * c.N + g]) {  // undecidable at T: no candidates scored (O5.4)
            if (valid && lane == gbase) {
              c.keys[g * Gc + (j - cs.glo)] = -1;
              if (P.cand_keys) P.cand_keys[(((size_t)r * P.E + e) * N + g) * (size_t)T.G + j] = -1;
            }
            continue;  // warp-uniform: the whole unit belongs to g
          }
        }
        const bool active = valid && s < T.gn[j];
        const int p = active ? T.gprof[j * 8 + s] : 0;
        SliceLane K;
        K.fbr_p = T.fbr + p;
        K.solo_p = T.solo + p;
        K.Ms = T.cap[p];
        K.pref = T.gpref[j * 8 + (s & 7)];
        K.s = s;
        K.p = p;
        K.Z = Z;
        const int al = actual && valid ? g * kZA + s : 0;  // actual slice state id
        const int sub = subm ? lane >> 3 : 0;                // sub-lane of the slice (subm)
        LaneList L;
        if (actual) {
          L = AL;
          const int ll = subm ? (actual && valid ? g * 32 + lane : 0) : al;  // actual list id
          L.st += ll; L.en += ll; L.mm += ll;
        } else {
          L = CL;
        }
        int n = actual && valid ? (subm ? (c.a_n[al] >> (8 * sub)) & 0xFF : c.a_n[al]) : 0;
        int64_t ls = actual && valid ? c.a_ls[al] : 0;
        int64_t bu = actual && valid ? c.a_bu[al] : 0;
        const int x0 = valid ? c.g_off[g] : 0, x1 = valid ? c.g_off[g + 1] : 0;
        int len_max;
        if (actual) {  // up to AG GPUs per warp: the longest batch list of the warp's GPUs
          len_max = x1 - x0;
#pragma unroll
          for (int d = 1; d < 32; d <<= 1) {
            const int o = __shfl_xor_sync(0xffffffffu, len_max, d);
            len_max = o > len_max ? o : len_max;
          }
        } else {       // one GPU per candidate warp: uniform
          len_max = c.g_off[g + 1] - c.g_off[g];
        }
        int64_t misses, tail;
        // register fast path (warp-uniform batch range: idle lanes still take part in the shuffles);
        // if a completion does not fit its 32-bit frame, the unit re-runs on the generic path below
        if (!actual && len_max <= kKR &&
            candidate_unit_fast(T, K, active, lane == gbase && valid, bats, gl, c.g_off[g],
                                c.g_off[g + 1] - c.g_off[g], sarr, P.max_live, &misses, &tail)) {
          if (valid && lane == gbase) {
            const int64_t key = make_key(misses, tail, j == c.gu8[0 * c.N + g] ? 0 : j + 1);
            if (j == c.gu8[0 * c.N + g]) c.gi[7 * c.N + g] = key;
            c.keys[g * Gc + (j - cs.glo)] = key;
            if (P.cand_keys) P.cand_keys[(((size_t)r * P.E + e) * N + g) * (size_t)T.G + j] = key;
          }
          continue;
        }
        int64_t acc0 = 0, acc1 = 0;  // actual: busy, mem-time; candidate: misses, BE tail
#pragma unroll 1
        for (int xi = 0; xi < len_max; ++xi) {
          const bool has = xi < x1 - x0;
          Bat* bt = &bats[has ? gl[x0 + xi] : 0];
          const uint32_t info = has ? bt->info : 0u;
          const int m = (info >> 16) & 0xFF, nreq = info & 0xFFFF;
          const bool strict = (info >> 24) & 1;
          int64_t t = has ? (int64_t)bt->ready : 0;
          int ci = -1;  // N3: the batch's container (group leader)
          if constexpr (kN3) {  // R23: container acquisition on the actual placement only (R25)
            if (actual) {
              int64_t te = t;
              unsigned long long cold = 0;
              ci = pool_acquire(P, pl, has && valid, g, m, t, lane, gbase, &te, &cold);
              if (cold) atomicAdd(&cs.cold, cold);
              t = te;
              if (lane != gbase) ci = -1;  // the leader releases it after the placement
            }
          }
          int64_t st, en;
          const SliceOut so = (subm && actual)
              ? place_group_sub<kPL>(T, active && has, K, L, n, ls, t, m, strict, P.max_live, &st, &en)
              : place_group<kPL>(T, active && has, K, L, n, ls, t, m, strict, P.max_live, &st, &en);
          const bool placed = !so.drop_overflow && so.kmin != ~0ull;
          const int wl = (gbase + (int)(so.kmin & 7)) & 31;
          const int64_t cwin = __shfl_sync(0xffffffffu, en, wl);
          if constexpr (kN3) {  // R24: busy until the batch ends (a drop releases it at once)
            if (actual) {
              if (ci >= 0) pl.bu[pl.pm(g, m) * kPoolCap + ci] = placed ? cwin : t;
              __syncwarp();  // the group's next search reads the pool
            }
          }
          if (!has) continue;
          if (actual) {
            // winner: busy union + memory-time, clipped to [0, H) (with sub-lanes: the slice's 4
            // lanes keep busy-until replicated, sub-lane 0 accounts and records)
            if (placed && (subm ? s == (int)(so.kmin & 7) : lane == wl)) {
              const int64_t lo = st > bu ? st : bu;
              const int64_t hi = en < P.H ? en : P.H;
              if (sub == 0) {
                if (hi > lo) acc0 += (int64_t)prof_compute(p) * (hi - lo);
                if (hi > st) acc1 += (int64_t)T.mem[m] * (hi - st);
                bt->slice = (uint8_t)s;
                bt->start = st;
                bt->end = en;
                bt->drop = 0;
              }
              if (en > bu) bu = en;
            }
            if (!placed && lane == gbase && sub == 0) {
              bt->drop = so.drop_overflow ? 3 : 2;
              bt->slice = 0xFF;
              bt->start = bt->end = 0;
            }
          } else if (lane == gbase && valid) {  // group leader keeps the candidate's score
            if (strict) {
              if (!placed) {
                acc0 += nreq;
              } else {  // latencies fall along the sorted members: test the ends first
                const uint32_t* ma = sarr + bt->pos;
                const int64_t slo = T.slo[m];
                if (cwin - (int64_t)ma[0] > slo)
                  acc0 += (cwin - (int64_t)ma[nreq - 1] > slo) ? nreq : nreq - hits_in(ma, nreq, cwin, slo);
              }
            } else {
              const int64_t tb = placed ? cwin - (int64_t)sarr[bt->pos] : (int64_t)0xFFFFFFFFLL;
              acc1 = tb > acc1 ? tb : acc1;
            }
          }
        }
        if (actual) {
          int64_t mx = 0;
          if (valid) {
            if (subm) {  // one count byte per sub-list; ls / bu are replicated over the 4 sub-lanes
              reinterpret_cast<uint8_t*>(c.a_n + al)[sub] = (uint8_t)n;
            } else {
              c.a_n[al] = n;
            }
            if (sub == 0) {
              c.a_ls[al] = ls;
              c.a_bu[al] = bu;
            }
#pragma unroll 1
            for (int i = 0; i < n; ++i) mx = L.E(i) > mx ? L.E(i) : mx;
          }
#pragma unroll
          for (int d = 1; d < 32; d <<= 1) {  // AG = 1 with sub-lanes: the whole warp is one GPU
            const int64_t o = __shfl_xor_sync(0xffffffffu, mx, d);
            if (subm || d < 8) mx = o > mx ? o : mx;
          }
          const int64_t bsum = group_sum(acc0, 8), msum = group_sum(acc1, 8);
          if (valid && s == 0 && sub == 0) {
            c.gi[5 * c.N + g] = mx;
            c.gi[10 * c.N + g] += bsum;
            c.gi[11 * c.N + g] += msum;
          }
          __syncwarp();  // every lane's batch-result stores precede lane 0's release below
          if (lane == 0) {
            const uint32_t fa = (uint32_t)__cvta_generic_to_shared(&cs.adone);
            asm volatile("red.release.cta.shared::cta.add.s32 [%0], 1;" ::"r"(fa) : "memory");
          }
        } else if (valid && lane == gbase) {
          const int64_t key = make_key(acc0, acc1, j == c.gu8[0 * c.N + g] ? 0 : j + 1);
          if (j == c.gu8[0 * c.N + g]) c.gi[7 * c.N + g] = key;
          c.keys[g * Gc + (j - cs.glo)] = key;
          if (P.cand_keys) P.cand_keys[(((size_t)r * P.E + e) * N + g) * (size_t)T.G + j] = key;
        }
      }
      }  // rounds
      __syncthreads();
      PH(7);
      if constexpr (kN3) {  // R26: delayed termination (pools are next used in the next epoch's E)
#pragma unroll 1
        for (int k = tid; k < N * pl.M; k += NT) pool_terminate(P, pl, c, k / pl.M, k % pl.M, c.bats, c.gl, Tend);
        __syncthreads();  // the next epoch's A (warp 0) may reset pools on a VM change
      }
      // ---------------------------------------------------------------- G: decisions (O9, O10)
      if (PROTEAN_WARP_G && P.xl.n <= 1 && N <= 32) {
        // one warp, lane = simulated GPU: argmin over the candidate keys, Alg 2 hysteresis, then
        // the ~30% cap by (delta misses desc, GPU asc) as a warp argmax per pick; the other warps
        // go straight to the epoch's last barrier
        if (warp == 0) {
          const int g = lane;
          const bool gv = g < N;
          bool want = false;
          int64_t kb = kForever, kc = -1;
          uint32_t scored_b = 0;  // batches of this GPU scored by every candidate (counters 8, 9)
          bool scored = false;
          if (gv) {
            uint8_t dec_out = kNoGeom;
            if (P.policy != 1 && c.gu8[5 * c.N + g]) {
              const int cur = c.gu8[0 * c.N + g];
              int best;
              if (P.policy == 0 && pre) {  // S8 over the keys of g's residue class (cand.cu)
                int cl = g - cursor;
                cl = cl < 0 ? cl + N : cl;
                const int64_t* kr = kst + (e & 1) * SL.KS + cl * T.G;
#pragma unroll 1
                for (int v = 0; v < T.G; ++v) {
                  int64_t kv = kr[v];
                  if (v == cur) {
                    kv &= ~(int64_t)255;  // tag 0: the current geometry (O8, Q20)
                    kc = kv;
                  }
                  kb = kv < kb ? kv : kb;
                  if (P.cand_keys) P.cand_keys[(((size_t)r * P.E + e) * N + g) * (size_t)T.G + v] = kv;
                }
                c.gi[6 * c.N + g] = kb;
                c.gi[7 * c.N + g] = kc;
                const int tag = (int)(kb & 255);
                best = tag == 0 ? cur : tag - 1;
                scored_b = (uint32_t)(c.g_off[g + 1] - c.g_off[g]);
                scored = true;
              } else if (P.policy == 0) {  // S8: argmin over the candidate keys
#pragma unroll 1
                for (int v = 0; v < cs.ghi - cs.glo; ++v) kb = c.keys[g * Gc + v] < kb ? c.keys[g * Gc + v] : kb;
                c.gi[6 * c.N + g] = kb;
                kc = c.gi[7 * c.N + g];
                const int tag = (int)(kb & 255);
                best = tag == 0 ? cur : tag - 1;
                scored_b = (uint32_t)(c.g_off[g + 1] - c.g_off[g]);
                scored = true;
              } else {  // policy 2: Alg 2's own heuristic (N1)
                if constexpr (kAlg2) best = alg2_final_geometry(P, c, g, c.bats, c.gl);
                else best = cur;  // unreachable: policy 2 launches replay_kernel<true, *, *>
              }
              dec_out = (uint8_t)best;
              c.gu8[6 * c.N + g] = (uint8_t)best;
              if (best != cur) {  // Alg 2 lines 24-30 (Q22)
                if (c.gu8[2 * c.N + g] >= P.wait_limit) want = true;
                else c.gu8[2 * c.N + g]++;
              } else {
                c.gu8[2 * c.N + g] = 0;
              }
            } else if (P.policy == 0) {
              c.gi[6 * c.N + g] = kForever;
            }
            if (P.decisions) P.decisions[((size_t)r * P.E + e) * N + g] = dec_out;
            if ((P.policy != 0 || (pre && !c.gu8[5 * c.N + g])) && P.cand_keys) {  // nothing scored
#pragma unroll 1
              for (int j = cs.glo; j < cs.ghi; ++j)
                P.cand_keys[(((size_t)r * P.E + e) * N + g) * (size_t)T.G + j] = -1;
            }
          }
          {  // counters 8, 9 (O8): slot-evals = sum over scored GPUs of batches x slots of the range
            const uint32_t tb = __reduce_add_sync(0xffffffffu, scored_b);  // <= nb < 2^25
            const int nsc = __popc(__ballot_sync(0xffffffffu, scored));
            if (lane == 0) {
              cs.cnt[8] += (unsigned long long)tb * (unsigned long long)sum_slots;
              cs.cnt[9] += (unsigned long long)nsc * (unsigned long long)(cs.ghi - cs.glo);
            }
          }
          fold_wcnt(cs, s_wcnt, NW, lane);
          if (P.policy != 1) {
            const unsigned alive = __ballot_sync(0xffffffffu, gv && has_vm(c, g, Tend));
            const unsigned open = __ballot_sync(0xffffffffu, gv && c.gi[1 * c.N + g] > Tend);
            int cap = P.cap_pct * __popc(alive) / 100;
            if (cap < 1) cap = 1;
            int free_slots = cap - __popc(open);
            const int64_t d = (want && P.policy == 0) ? (kc >> 40) - (kb >> 40) : 0;  // policy 2: GPU order (R16)
#pragma unroll 1
            while (free_slots > 0) {
              const unsigned wm = __ballot_sync(0xffffffffu, want);
              if (!wm) break;
              int64_t best_d = want ? d : INT64_MIN;  // max d, then lowest GPU
#pragma unroll
              for (int o = 16; o > 0; o >>= 1) {
                const int64_t od = __shfl_xor_sync(0xffffffffu, best_d, o);
                best_d = od > best_d ? od : best_d;
              }
              const unsigned tie = __ballot_sync(0xffffffffu, want && d == best_d);
              const int pick = __ffs(tie) - 1;
              if (lane == pick) {
                want = false;
                const int64_t drain_end = c.gi[5 * c.N + g] > Tend ? c.gi[5 * c.N + g] : Tend;
                c.gi[0 * c.N + g] = Tend;
                c.gi[1 * c.N + g] = drain_end + P.reconfig_us;
                c.gu8[1 * c.N + g] = c.gu8[6 * c.N + g];
                cs.cnt[7] += 1;
              }
              --free_slots;
            }
          }
          if (lane == 0) {
            cs.nlog += nb;
            cs.task = 0;  // re-arm the per-epoch scratch for the next epoch
            cs.task_r[0] = cs.task_r[1] = 0;
            cs.adone = 0;
            cs.nb = 0;
            cs.all_avail = 1;
          }
        }
      } else {
      if (P.policy == 0) {  // S8: min over this rank's geometry range
#pragma unroll 1
        for (int g = tid; g < N; g += NT) {
          int64_t kb = kForever;
          if (c.gu8[5 * c.N + g]) {
#pragma unroll 1
            for (int v = 0; v < cs.ghi - cs.glo; ++v) kb = c.keys[g * Gc + v] < kb ? c.keys[g * Gc + v] : kb;
          }
          c.gi[6 * c.N + g] = kb;
        }
        if (P.xl.n > 1)
          exchange_keys(P.xl, P.xpeer, cs.xrank, P.err, P.xtimeout_ns, c.gi, N, r,
                        (uint32_t)(P.xseq + (uint32_t)e), tid, NT);
      }
#pragma unroll 1
      for (int g = tid; g < N; g += NT) {
        uint8_t dec_out = kNoGeom;
        if (P.policy != 1 && c.gu8[5 * c.N + g]) {
          const int cur = c.gu8[0 * c.N + g];
          int best;
          if (P.policy == 0) {
            const int64_t kb = c.gi[6 * c.N + g];
            const int tag = (int)(kb & 255);
            best = tag == 0 ? cur : tag - 1;
            atomicAdd(&cs.cnt[8], (unsigned long long)(c.g_off[g + 1] - c.g_off[g]) * (unsigned long long)sum_slots);
            atomicAdd(&cs.cnt[9], (unsigned long long)(cs.ghi - cs.glo));
          } else {  // policy 2: Alg 2's own heuristic (N1)
            if constexpr (kAlg2) best = alg2_final_geometry(P, c, g, c.bats, c.gl);
            else best = cur;  // unreachable: policy 2 launches replay_kernel<true, *, *>
          }
          dec_out = (uint8_t)best;
          c.gu8[6 * c.N + g] = (uint8_t)best;
          if (best != cur) {
            if (c.gu8[2 * c.N + g] >= P.wait_limit) c.gu8[7 * c.N + g] = 1;
            else c.gu8[2 * c.N + g]++;
          } else {
            c.gu8[2 * c.N + g] = 0;
          }
        }
        if (P.decisions) P.decisions[((size_t)r * P.E + e) * N + g] = dec_out;
        if (P.policy != 0 && P.cand_keys) {
#pragma unroll 1
          for (int j = cs.glo; j < cs.ghi; ++j)
            P.cand_keys[(((size_t)r * P.E + e) * N + g) * (size_t)T.G + j] = -1;
        }
      }
      __syncthreads();
      PH(8);
      if (warp == 0) fold_wcnt(cs, s_wcnt, NW, lane);
      if (tid == 0) {
        if (P.policy != 1) {
          int alive = 0, open = 0;
#pragma unroll 1
          for (int g = 0; g < N; ++g) {
            alive += has_vm(c, g, Tend) ? 1 : 0;
            open += c.gi[1 * c.N + g] > Tend ? 1 : 0;
          }
          int cap = P.cap_pct * alive / 100;
          if (cap < 1) cap = 1;
          int free_slots = cap - open;
#pragma unroll 1
          while (free_slots > 0) {  // wants by (delta misses desc, gpu asc)
            int pick = -1;
            int64_t pd = 0;
#pragma unroll 1
            for (int g = 0; g < N; ++g) {
              if (!c.gu8[7 * c.N + g]) continue;
              const int64_t d = P.policy == 0 ? (c.gi[7 * c.N + g] >> 40) - (c.gi[6 * c.N + g] >> 40) : 0;
              if (pick < 0 || d > pd) { pick = g; pd = d; }
            }
            if (pick < 0) break;
            c.gu8[7 * c.N + pick] = 0;
            const int64_t drain_end = c.gi[5 * c.N + pick] > Tend ? c.gi[5 * c.N + pick] : Tend;
            c.gi[0 * c.N + pick] = Tend;
            c.gi[1 * c.N + pick] = drain_end + P.reconfig_us;
            c.gu8[1 * c.N + pick] = c.gu8[6 * c.N + pick];
            cs.cnt[7] += 1;
            --free_slots;
          }
        }
        cs.nlog += nb;
        cs.task = 0;  // re-arm the per-epoch scratch for the next epoch
        cs.task_r[0] = cs.task_r[1] = 0;
        cs.adone = 0;
        cs.nb = 0;
        cs.all_avail = 1;
      }
      }
      PH(9);  // the next epoch's first barrier closes this one
      }  // e >= 0
      // A and B of the next epoch: A in warp 0 after its decisions (program order: the windows G
      // opened are visible to A), B in warp kBW at the same time (it reads only s_cur and writes the
      // window, which nothing after E reads)
      if (e + 1 < P.E) {
        if (warp == 0) {
          __syncwarp();
          phase_a(e + 1);
        } else if (warp == kBW) {
          phase_b(e + 1);
        }
      }
    }
    __syncthreads();  // the last epoch's decisions before finalize

    // ---------------------------------------------------------------- finalize (O12)
#pragma unroll 1
    for (int g = tid; g < N; g += NT) bill_switch(c, g, VM_NONE, P.H, P.H);
    bool pct_here = true;  // this CTA holds the replica's whole histogram
    if (vsplit) {  // partial histograms (split accounting): summed in HBM, the last CTA ranks them
#pragma unroll 1
      for (int w = tid; w < 2 * kNB; w += NT)
        if (s_hist[w]) atomicAdd(ghist + w, s_hist[w]);
      __threadfence();
      __syncthreads();
      if (tid == 0) cs.task = (int)(atomicAdd(P.vr_done + r, 1u) == (unsigned)(vrn - 1));
      __syncthreads();
      pct_here = cs.task != 0;
      __threadfence();
    } else {
#pragma unroll 1
      for (int w = tid; w < 2 * kNB; w += NT) ghist[w] = s_hist[w];  // histogram to HBM
      __syncthreads();
    }
    if (warp < 2 && pct_here) {  // nearest-rank P50 / P99 per class
      const uint32_t* h = ghist + warp * kNB;
      uint32_t n = 0;  // requests per class per replica < 2^32
#pragma unroll 1
      for (int b = lane; b < kNB; b += 32) n += __ldcg(h + b);
#pragma unroll
      for (int d = 16; d > 0; d >>= 1) n += __shfl_xor_sync(0xffffffffu, n, d);
      int64_t p50 = 0, p99 = 0;
      if (n) {
        const uint64_t r50 = (50 * (uint64_t)n + 99) / 100, r99 = (99 * (uint64_t)n + 99) / 100;
        uint64_t cum = 0;
        int f50 = -1, f99 = -1;
#pragma unroll 1
        for (int b0 = 0; b0 < kNB && f99 < 0; b0 += 32) {
          uint32_t x = __ldcg(h + b0 + lane);
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
    if (tid == 0) {
      int64_t od = 0, spot = 0, busy = 0, memt = 0;
#pragma unroll 1
      for (int g = 0; g < N; ++g) {
        od += c.gi[8 * c.N + g];
        spot += c.gi[9 * c.N + g];
        busy += c.gi[10 * c.N + g];
        memt += c.gi[11 * c.N + g];
      }
#pragma unroll 1
      for (int i = 0; i < 10; ++i) {
        // virtual ranks: slot-evals / candidates (this CTA's range) and the request counters (its
        // accounting tasks) are partial sums (zeroed by the host); reconfigurations are replicated
        if ((vsplit && i != 7) || (vrn > 1 && i >= 8))
          atomicAdd(reinterpret_cast<unsigned long long*>(&P.counters[(size_t)r * 10 + i]), cs.cnt[i]);
        else
          P.counters[(size_t)r * 10 + i] = (int64_t)cs.cnt[i];
      }
      P.accum[(size_t)r * 4 + 0] = busy;
      P.accum[(size_t)r * 4 + 1] = memt;
      P.accum[(size_t)r * 4 + 2] = od;
      P.accum[(size_t)r * 4 + 3] = spot;
      P.cost[r] = __ddiv_rn(__dadd_rn(__dmul_rn((double)od, P.price_od),
                                      __dmul_rn((double)spot, P.price_spot)), 3.6e9);
      const double dN = (double)N, dH = (double)P.H;
      P.util[2 * (size_t)r] = __ddiv_rn((double)busy, __dmul_rn(__dmul_rn(7.0, dN), dH));
      P.util[2 * (size_t)r + 1] = __ddiv_rn((double)memt, __dmul_rn(__dmul_rn((double)T.cap[4], dN), dH));
      if (P.n_batches) P.n_batches[r] = cs.nlog;
      if (P.cold_starts) P.cold_starts[r] = (int64_t)cs.cold;
    }
    __syncthreads();
  }
#ifdef PROTEAN_PHASE_TIMING
  if (threadIdx.x == 0)
    for (int k = 0; k < 10; ++k) atomicAdd(&g_phase_cycles[k], ph_acc[k]);
#endif
}

#ifdef PROTEAN_PHASE_TIMING
extern "C" int protean_debug_phase_cycles(unsigned long long* out) {
  return (int)cudaMemcpyFromSymbol(out, g_phase_cycles, sizeof(unsigned long long) * 13);
}
#endif

// replica_off on the device (no host round trip before the prepass): one CTA checks
// replica_off[0] == 0 and monotone (else err[0] |= 4, and every later pass of the call skips) and
// writes the stream-sorted copy's per-replica offsets saoff[r] = sum over r' < r of the replica's
// request count rounded up to 4 (16-byte aligned runs), saoff[R] = the copy's length.
__global__ void __launch_bounds__(1024) roff_scan_kernel(const int64_t* roff, int R, int64_t* saoff,
                                                         int* err) {
  __shared__ int64_t wsum[32];
  __shared__ int64_t carry;
  __shared__ int bad;
  const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
  if (tid == 0) {
    carry = 0;
    bad = roff[0] != 0;
    saoff[0] = 0;
  }
  __syncthreads();
#pragma unroll 1
  for (int r0 = 0; r0 < R; r0 += 1024) {
    const int r = r0 + tid;
    int64_t v = 0;
    if (r < R) {
      const int64_t n = roff[r + 1] - roff[r];
      if (n < 0) bad = 1;
      v = n < 0 ? 0 : (n + 3) & ~(int64_t)3;
    }
#pragma unroll
    for (int d = 1; d < 32; d <<= 1) {
      const int64_t y = __shfl_up_sync(0xffffffffu, v, d);
      if (lane >= d) v += y;
    }
    if (lane == 31) wsum[warp] = v;
    __syncthreads();
    if (warp == 0) {
      int64_t w = wsum[lane];
#pragma unroll
      for (int d = 1; d < 32; d <<= 1) {
        const int64_t y = __shfl_up_sync(0xffffffffu, w, d);
        if (lane >= d) w += y;
      }
      wsum[lane] = w;  // inclusive over warps
    }
    __syncthreads();
    const int64_t incl = carry + v + (warp ? wsum[warp - 1] : 0);
    if (r < R) saoff[r + 1] = incl;
    __syncthreads();
    if (tid == 1023) carry = incl;
    __syncthreads();
  }
  if (tid == 0 && bad) atomicOr(err, 4);
}

cudaError_t launch_roff_scan(const int64_t* roff, int R, int64_t* saoff, int* err, cudaStream_t st) {
  roff_scan_kernel<<<1, 1024, 0, st>>>(roff, R, saoff, err);
  return cudaGetLastError();
}

// Prepass: eoff[r][e] = first request of replica r with arrival >= e*W (e = 0..E), and the
// largest request window any epoch needs: [lower_bound(eW - maxT), eoff[e+1]).  A warp covers 32
// consecutive epochs of one replica and owns the first 31 (lane 31 only computes its lower bound
// for lane 30, and is owned again by the next warp's lane 0): eoff[e+1] comes from the next lane,
// and when maxT <= W the window start lies in [eoff[e-1], eoff[e]] (the previous lane's bound), so
// a lane runs one full-range binary search and one over about an epoch's requests.  On a sorted
// trace the bounds equal the full-range searches; an unsorted one is flagged (next < here) here or
// by the scatter pass, as before.
__global__ void prepass_kernel(const uint32_t* arr, const int64_t* roff, int R, int64_t E,
                               int64_t W, int64_t maxT, int64_t* eoff, unsigned long long* wmax,
                               int* err) {
  if (*(volatile int*)err & 4) return;  // replica_off rejected by roff_scan_kernel
  const int lane = threadIdx.x & 31;
  const int64_t gw = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5;
  const int64_t wpr = (E + 31) / 31;  // warps per replica: epochs 0..E, 31 owned per warp
  if (gw >= (int64_t)R * wpr) return;  // warp-uniform
  const int r = (int)(gw / wpr);
  const int64_t e = (gw - (int64_t)r * wpr) * 31 + lane;
  const int64_t lo0 = roff[r], hi0 = roff[r + 1];
  auto lower = [&](int64_t v, int64_t lo, int64_t hi) {
    while (lo < hi) {
      const int64_t mid = (lo + hi) >> 1;
      if ((int64_t)arr[mid] >= v) hi = mid; else lo = mid + 1;
    }
    return lo;
  };
  const bool live = e <= E;
  const int64_t here = live ? lower(e * W, lo0, hi0) : hi0;
  const int64_t next = __shfl_down_sync(0xffffffffu, here, 1);
  const int64_t prev = __shfl_up_sync(0xffffffffu, here, 1);
  if (lane == 31 || !live) return;
  eoff[(size_t)r * (E + 1) + e] = here;
  if (e < E) {  // lane + 1 <= 31 holds epoch e + 1 <= E
    const int64_t a = e * W - maxT;
    if (next < here) atomicOr(err, 1);  // arrivals not sorted
    const int64_t from = (lane > 0 && maxT <= W) ? prev : lo0;  // (e-1)W <= a <= eW
    const int64_t w = next - lower(a < 0 ? 0 : a, from, here);
    if (w > 0) atomicMax(wmax, (unsigned long long)w);
  } else if (here != hi0) {
    atomicOr(err, 1);                   // an arrival at or beyond E*W >= trace_len
  }
}

cudaError_t launch_prepass(const uint32_t* arr, const int64_t* roff, int R, int64_t E, int64_t W,
                           int64_t maxT, int64_t* eoff, unsigned long long* wmax, int* err,
                           cudaStream_t st) {
  const int64_t total = (int64_t)R * ((E + 31) / 31) * 32;  // threads: one warp per 31 epochs
  const int bs = 256;
  prepass_kernel<<<(unsigned)((total + bs - 1) / bs), bs, 0, st>>>(arr, roff, R, E, W, maxT, eoff, wmax, err);
  return cudaGetLastError();
}

// The replay kernel's dynamic shared-memory limit is raised once per device, to the opt-in
// maximum: changing a function attribute while an instance of the function runs can wait for it,
// which would serialise concurrently running mode-G ranks of one process.
static cudaError_t raise_dyn_smem_once() {
  static std::mutex mu;
  static bool done[256] = {};
  int dev = 0;
  cudaError_t e = cudaGetDevice(&dev);
  if (e != cudaSuccess) return e;
  std::lock_guard<std::mutex> lk(mu);
  if (dev < 256 && done[dev]) return cudaSuccess;
  int optin = 0;
  e = cudaDeviceGetAttribute(&optin, cudaDevAttrMaxSharedMemoryPerBlockOptin, dev);
  if (e != cudaSuccess) return e;
  for (auto k : {replay_kernel<false, false, 1>, replay_kernel<true, false, 1>, replay_kernel<false, true, 1>,
                 replay_kernel<true, true, 1>, replay_kernel<false, false, 4>, replay_kernel<true, false, 4>,
                 replay_kernel<false, true, 4>, replay_kernel<true, true, 4>}) {
    cudaFuncAttributes a;
    e = cudaFuncGetAttributes(&a, k);
    if (e != cudaSuccess) return e;
    e = cudaFuncSetAttribute(k, cudaFuncAttributeMaxDynamicSharedMemorySize, optin - (int)a.sharedSizeBytes);
    if (e != cudaSuccess) return e;
  }
  if (dev < 256) done[dev] = true;
  return e;
}

cudaError_t preload_kernels() {
  cudaFuncAttributes a;
  cudaError_t e = cudaSuccess;
  for (auto k : {replay_kernel<false, false, 1>, replay_kernel<true, false, 1>, replay_kernel<false, true, 1>,
                 replay_kernel<true, true, 1>, replay_kernel<false, false, 4>, replay_kernel<true, false, 4>,
                 replay_kernel<false, true, 4>, replay_kernel<true, true, 4>})
    if (e == cudaSuccess) e = cudaFuncGetAttributes(&a, k);
  if (e == cudaSuccess) e = cudaFuncGetAttributes(&a, prepass_kernel);
  if (e == cudaSuccess) e = preload_partition_kernels();
  if (e == cudaSuccess) e = raise_dyn_smem_once();
  return e;
}

cudaError_t launch_replay(const ReplayParams& P, int grid, int block, cudaStream_t st) {
  cudaError_t e = raise_dyn_smem_once();
  if (e != cudaSuccess) return e;
  const bool n3 = P.cold_us > 0;  // cold_us = 0: warm containers, no pool work (reading Q15)
  const bool wide = P.few;        // few replicas: long-list workloads get the 4-wide prune
  void (*k)(ReplayParams) = nullptr;
  if (P.policy == 2) {
    if (n3) k = wide ? replay_kernel<true, true, 4> : replay_kernel<true, true, 1>;
    else k = wide ? replay_kernel<true, false, 4> : replay_kernel<true, false, 1>;
  } else {
    if (n3) k = wide ? replay_kernel<false, true, 4> : replay_kernel<false, true, 1>;
    else k = wide ? replay_kernel<false, false, 4> : replay_kernel<false, false, 1>;
  }
  if (P.vr_n > 1) {
    // virtual ranks: the CTAs of a replica spin on each other's exchange flags, so the whole grid
    // must be co-resident; a cooperative launch guarantees it or fails at launch (instead of a
    // 30 s exchange timeout under MPS or concurrent work).  Mode G ranks (separate launches that
    // must run side by side) keep the plain launch and the timeout.
    cudaLaunchConfig_t lc = {};
    lc.gridDim = dim3((unsigned)grid);
    lc.blockDim = dim3((unsigned)block);
    lc.dynamicSmemBytes = P.sl.total;
    lc.stream = st;
    cudaLaunchAttribute at[1];
    at[0].id = cudaLaunchAttributeCooperative;
    at[0].val.cooperative = 1;
    lc.attrs = at;
    lc.numAttrs = 1;
    return cudaLaunchKernelEx(&lc, k, P);
  }
  k<<<grid, block, P.sl.total, st>>>(P);
  return cudaGetLastError();
}

// Occupancy of the instances a launch of this shape would use (few: the kPL = 4 instances).
cudaError_t replay_occupancy(int block, size_t smem, bool few, int* blocks_per_sm) {
  cudaError_t e = raise_dyn_smem_once();
  if (e != cudaSuccess) return e;
  int lo = 1 << 30;
  if (few) {
    for (auto k : {replay_kernel<false, false, 4>, replay_kernel<true, false, 4>, replay_kernel<false, true, 4>,
                   replay_kernel<true, true, 4>}) {
      int a = 0;
      if (e == cudaSuccess) e = cudaOccupancyMaxActiveBlocksPerMultiprocessor(&a, k, block, smem);
      lo = a < lo ? a : lo;
    }
  } else {
    for (auto k : {replay_kernel<false, false, 1>, replay_kernel<true, false, 1>, replay_kernel<false, true, 1>,
                   replay_kernel<true, true, 1>}) {
      int a = 0;
      if (e == cudaSuccess) e = cudaOccupancyMaxActiveBlocksPerMultiprocessor(&a, k, block, smem);
      lo = a < lo ? a : lo;
    }
  }
  *blocks_per_sm = lo;
  return e;
}

}  // namespace pemgpu
