// cand.cu — the candidate search taken out of the epoch chain (sm_100a).
//
// A candidate geometry is replayed from idle on the GPU-epoch's batches (O8, the "Oracle" scheme
// run online), so its key depends only on the batches that GPU receives in that epoch, not
// on the carried state.  When every simulated GPU is available the whole epoch, dispatch is the
// closed form of Q18: batch rank rk goes to GPU (cursor + rk) mod N, so GPU g receives the
// residue class (g - cursor) mod N of the epoch's id-ordered batches, and only the cursor -- known
// when the chain reaches the epoch -- decides which GPU a class lands on.  The search is therefore
// a data-parallel pass over (replica, epoch) units ahead of the chain:
//
//   walk_kernel   warp per (replica, stream): O3 batch formation (reading Q14) is a
//                 greedy chain along the stream -- close at B requests or at the first arrival + T
//                 -- whose batches have non-decreasing ready times, so the chain kernel's stream
//                 cursor at the start of epoch e is the first batch start whose ready time is
//                 >= eW (DESIGN F1).  Lanes test 32 consecutive full batches per load round.
//                 Records bstart[r][k][e] (e = 0..E).
//   cand_kernel   warp per (replica, epoch): forms the epoch's batches from bstart (the warp on one
//                 active stream at a time, 32 batches per round), ranks them into id order (ready,
//                 strict first, model, position), writes the rows (UnitBats) for the chain and the
//                 accounting pass, and scores every (residue class, geometry) pair with one lane
//                 each -- Alg 1 under Eq 1 / Eq 2 over the class's
//                 batches from idle in 32-bit time relative to eW, the lane walking its geometry's
//                 fitting slices itself (bit masks of the batches placed per slice, dominated idle
//                 slices dropped) -- then the O8 key (misses << 40 | BE tail << 8 | tag j + 1; the
//                 chain re-tags the GPU's current geometry with 0).  Writes kfc[r][e][class][j].  A
//                 unit it cannot hold (more than kBC = 64 batches: the whole call goes back to the
//                 fused engine; more than kKC = 10 in a class, or a completion 2^25 us past eW: that
//                 epoch is scored in the chain) is marked with kfc[r][e][0][0] = INT64_MIN.
//
// The chain (chain.cu, or the fused replay.cu) uses the keys for every epoch whose dispatch is the
// closed form; an epoch with a GPU unavailable inside it (reconfiguration window, VM change) is
// scored in the chain.
#include <cuda_runtime.h>
#include <stdint.h>

#include "replay.cuh"

namespace pemgpu {

namespace {

constexpr int kBC = kUnitBats;  // batches per (replica, epoch) unit held in shared memory
static_assert(kBC <= 64, "the id-order rank: two batches per lane");
constexpr int kKC = 10;        // batches per residue class held per lane (config 5: ~5)
constexpr int kCandWarps = 8;  // warps per CTA

// ---------------------------------------------------------------- walk
// Warp per (replica, stream): lanes test 32 consecutive B-sized batches at once (a batch is full
// when its B-th member arrives within the timeout; full batches are the common case), lane 0
// resolves a batch closed by the timeout with a binary search.  Lane l of a step records the
// epochs (ep_{l-1}, ep_l] as starting at its batch.
__global__ void __launch_bounds__(256) walk_kernel(CandParams P) {
  const int64_t wid = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5;
  const int lane = threadIdx.x & 31;
  const int S = P.S;
  if (wid >= (int64_t)P.R * S) return;
  const int r = (int)(wid / S), k = (int)(wid % S);
  const int64_t E = P.E, W = P.W;
  const uint32_t* sa = P.sa + P.saoff[r];
  const uint32_t* srow = P.sidx + (size_t)r * (E + 1) * S;
  uint32_t i = srow[k];
  const uint32_t end = srow[(size_t)E * S + k];
  const int m = k >> 1;
  const uint32_t B = (uint32_t)P.tab[P.tl.o_bsz + m];
  const int64_t Tm = P.tab[P.tl.o_tmo + m];
  uint32_t* out = P.bstart + ((size_t)r * S + k) * (E + 1);
  int64_t en = 0;  // next epoch whose start is not yet recorded (uniform)
#pragma unroll 1
  while (i < end) {
    const uint64_t st = (uint64_t)i + (uint64_t)lane * B;
    bool full = false;
    int64_t ready = 0;
    if (st + B <= end) {
      const int64_t a0 = sa[st], al = sa[st + B - 1];
      full = al <= a0 + Tm;
      ready = al;
    }
    const unsigned fm = __ballot_sync(0xffffffffu, full);
    const int nfull = (~fm) ? __ffs(~fm) - 1 : 32;
    if (nfull > 0) {
      const int64_t ep = lane < nfull ? ready / W : INT64_MAX;
      int64_t prev = __shfl_up_sync(0xffffffffu, ep, 1);
      if (lane == 0) prev = en - 1;
      if (lane < nfull) {
        const int64_t hi = ep < E ? ep : E;
#pragma unroll 1
        for (int64_t x = prev + 1; x <= hi; ++x) out[x] = (uint32_t)st;
      }
      const int64_t last = __shfl_sync(0xffffffffu, ep, nfull - 1);
      en = (last < E ? last : E) + 1;
      if (last >= E) return;  // a batch beyond the horizon: out[0..E] is complete
      i += (uint32_t)nfull * B;
      if (nfull == 32) continue;
      if (i >= end) break;
    }
    // the batch at i is not full: it closes at its first arrival + T (or the stream end)
    int64_t rd = 0;
    uint32_t j = 0;
    if (lane == 0) {
      const int64_t dl = (int64_t)sa[i] + Tm;
      const uint32_t lim = end - i > B ? i + B : end;
      uint32_t lo = i + 1, hi = lim;
#pragma unroll 1
      while (lo < hi) {
        const uint32_t mid = (lo + hi) >> 1;
        if ((int64_t)sa[mid] > dl) hi = mid; else lo = mid + 1;
      }
      j = lo;
      rd = (j - i == B) ? (int64_t)sa[j - 1] : dl;
    }
    rd = __shfl_sync(0xffffffffu, rd, 0);
    j = __shfl_sync(0xffffffffu, j, 0);
    const int64_t ep = rd / W;
    const int64_t hi = ep < E ? ep : E;
#pragma unroll 1
    for (int64_t x = en + lane; x <= hi; x += 32) out[x] = i;
    en = hi + 1;
    if (ep >= E) return;
    i = j;
  }
#pragma unroll 1
  for (int64_t x = en + lane; x <= E; x += 32) out[x] = i;
}

// ---------------------------------------------------------------- candidates
struct WarpSmem {
  union {                  // the rank keys are dead once the epoch is in id order
    uint64_t key[kBC];
    struct {
      uint32_t en[kKC][32];  // per lane: end of each placed batch, relative to eW (0: dropped)
      uint32_t pk[kKC][32];  //           footprint | best-effort << 27
      int32_t fb[kKC][32];   //           FBR of the batch on its slice's profile
    };
  };
  uint32_t ready[kBC], info[kBC], pos[kBC], afirst[kBC], alast[kBC];
  uint8_t ord[kBC];
  uint32_t ls[kMaxSl][32];   //       last start per slice position (FIFO), relative to eW
  uint16_t msk[kMaxSl][32];  //       batches placed on each slice position
  int nb, bad;
};
static_assert(kKC <= 16, "16-bit slice masks");

// Memory wait of Alg 1 on one slice (the batch does not fit at t0): releases after t0 in ascending
// order, the footprint still held only shrinks, so the first that fits is the minimum of the plain
// definition (always by the last release: q <= Ms); Eq 1's co-runners at that start into *F.
static __device__ __noinline__ uint32_t mem_wait(const WarpSmem& ws, int lane, uint32_t set, uint32_t t0,
                                                 int32_t q, int32_t Ms, uint32_t* F) {
  uint32_t ev = t0;
#pragma unroll 1
  for (;;) {
    uint32_t nxt = 0xFFFFFFFFu;
    for (uint32_t a = set; a; a &= a - 1) {
      const uint32_t e = ws.en[__ffs(a) - 1][lane];
      if (e > ev && e < nxt) nxt = e;
    }
    ev = nxt;
    int32_t rem = 0;
    for (uint32_t a = set; a; a &= a - 1) {
      const int i = __ffs(a) - 1;
      if (ws.en[i][lane] > ev) rem += (int32_t)(ws.pk[i][lane] & kMemMask);
    }
    if (rem + q <= Ms) break;
  }
  for (uint32_t a = set; a; a &= a - 1) {
    const int i = __ffs(a) - 1;
    if (ws.en[i][lane] > ev) *F += (uint32_t)ws.fb[i][lane];
  }
  return ev;
}

__device__ __forceinline__ void prefetch_members(const uint32_t* a, uint32_t n) {
  const char* p0 = reinterpret_cast<const char*>(a);
  const char* p1 = reinterpret_cast<const char*>(a + n);
  for (const char* p = reinterpret_cast<const char*>((uintptr_t)p0 & ~(uintptr_t)127); p < p1; p += 128)
    asm volatile("prefetch.global.L2 [%0];" ::"l"(p));
}

__device__ __forceinline__ int hits_from(const uint32_t* a, int n, int64_t c, int64_t slo) {
  const int64_t need = c - slo;  // c - a <= slo  <=>  a >= c - slo
  int lo = 0, hi = n;
#pragma unroll 1
  while (lo < hi) {
    const int mid = (lo + hi) >> 1;
    if ((int64_t)a[mid] >= need) hi = mid; else lo = mid + 1;
  }
  return n - lo;
}

__device__ __forceinline__ int64_t key_of(int64_t misses, int64_t tail, int tag) {  // O8 (Q20)
  const int64_t mm = (1LL << 23) - 1;
  if (misses > mm) misses = mm;
  if (tail > 0xFFFFFFFFLL) tail = 0xFFFFFFFFLL;
  return (misses << 40) | (tail << 8) | (int64_t)tag;
}

#ifdef PROTEAN_CAND_MINB  // experiment knob: minimum resident CTAs per SM (register cap)
__global__ void __launch_bounds__(32 * kCandWarps, PROTEAN_CAND_MINB) cand_kernel(CandParams P) {
#else
__global__ void __launch_bounds__(32 * kCandWarps) cand_kernel(CandParams P) {
#endif
  extern __shared__ __align__(16) unsigned char smem[];
  int32_t* tabw = reinterpret_cast<int32_t*>(smem);
  const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
#pragma unroll 1
  for (int i = tid; i < P.tl.words; i += blockDim.x) tabw[i] = P.tab[i];
  uint8_t* gord = smem + ((P.tl.words * 4 + 15) & ~15);  // geometry order (slice count desc)
#pragma unroll 1
  for (int i = tid; i < P.tl.G; i += blockDim.x) gord[i] = P.gorder[i];
  // fitm[j][m]: the slice positions of geometry j whose memory holds model m's footprint
  uint8_t* fitm = gord + ((P.tl.G + 15) & ~15);
  {
    Tab T0;
    T0.bind(tabw, P.tl);
    __syncthreads();  // the table is staged
#pragma unroll 1
    for (int i = tid; i < P.tl.G * P.tl.M; i += blockDim.x) {
      const int j = i / P.tl.M, m = i % P.tl.M;
      uint32_t f = 0;
      for (int s = 0; s < T0.gn[j]; ++s)
        if (T0.mem[m] <= T0.cap[T0.gprof[j * 8 + s]]) f |= 1u << s;
      fitm[i] = (uint8_t)f;
    }
#pragma unroll 1
    for (int i = tid; i < P.tl.G * kNProf; i += blockDim.x) {  // pmask[j][p]: slices of profile p
      const int j = i / kNProf, pp = i % kNProf;
      uint32_t f = 0;
      for (int s = 0; s < T0.gn[j]; ++s)
        if (T0.gprof[j * 8 + s] == pp) f |= 1u << s;
      fitm[P.tl.G * P.tl.M + i] = (uint8_t)f;
    }
  }
  const uint8_t* pmask = fitm + P.tl.G * P.tl.M;
  WarpSmem& ws = reinterpret_cast<WarpSmem*>(smem + P.ws_off)[warp];
  __syncthreads();
  Tab T;
  T.bind(tabw, P.tl);
  const int S = P.S, N = P.N, G = P.tl.G, M = P.tl.M;
  const int64_t E = P.E, W = P.W;
  const int64_t n_units = (int64_t)P.R * E;
  const int npairs = N * G;
  const int64_t gw = (int64_t)gridDim.x * kCandWarps;
#pragma unroll 1
  for (int64_t u = (int64_t)blockIdx.x * kCandWarps + warp; u < n_units; u += gw) {
    const int r = (int)(u / E);
    const int64_t e = u - (int64_t)r * E;
    const int64_t eW = e * W;
    const int64_t sbase = P.saoff[r];
    const uint32_t* sa = P.sa + sbase;
    int64_t* kout = P.kfc ? P.kfc + (size_t)u * N * G : nullptr;  // NULL: rows only (policy 2)
    if (lane == 0) {
      ws.nb = 0;
      ws.bad = 0;
    }
    __syncwarp();
    // ---- formation (O3): the epoch's batches of every stream, from the batch-aligned cursor.
    // The warp takes the active streams one at a time; lanes test 32 consecutive B-sized batches
    // at once (a batch starting before the next epoch's cursor ends by it), lane 0 resolves a
    // batch closed by the timeout.
    {
      int nbw = 0;  // uniform
#pragma unroll 1
      for (int k0 = 0; k0 < S; k0 += 32) {
        const int kl = k0 + lane;
        uint32_t i0 = 0, i1 = 0;
        if (kl < S) {
          const uint32_t* bs = P.bstart + ((size_t)r * S + kl) * (E + 1) + e;
          i0 = bs[0];
          i1 = bs[1];
        }
#pragma unroll 1
        for (unsigned act = __ballot_sync(0xffffffffu, i0 < i1); act; act &= act - 1) {
          const int src = __ffs(act) - 1;
          const int k = k0 + src;
          uint32_t i = __shfl_sync(0xffffffffu, i0, src);
          const uint32_t iend = __shfl_sync(0xffffffffu, i1, src);
          const int m = k >> 1;
          const bool strict = (k & 1) == 0;
          const uint32_t B = (uint32_t)T.bsz[m];
          const int64_t Tm = T.tmo[m];
          const uint32_t ibase = i;
          const uint32_t tag = ((strict ? 0u : 1u) << 31) | ((uint32_t)m << 25);
#pragma unroll 1
          while (i < iend) {
            const uint64_t st = (uint64_t)i + (uint64_t)lane * B;
            bool full = false;
            uint32_t a0 = 0, al = 0;
            if (st + B <= iend) {
              a0 = sa[st];
              al = sa[st + B - 1];
              full = (int64_t)al <= (int64_t)a0 + Tm;
            }
            const unsigned fm = __ballot_sync(0xffffffffu, full);
            const int nfull = (~fm) ? __ffs(~fm) - 1 : 32;
            if (lane < nfull) {
              const int slot = nbw + lane;
              if (slot < kBC) {
                ws.key[slot] = ((uint64_t)al << 32) | tag | (uint64_t)(((uint32_t)st - ibase) & 0x1FFFFFF);
                ws.ready[slot] = al;
                ws.info[slot] = B | ((uint32_t)m << 16) | ((uint32_t)(strict ? 1 : 0) << 24);
                ws.pos[slot] = (uint32_t)st;
                ws.afirst[slot] = a0;
                ws.alast[slot] = al;
              }
              if (strict) prefetch_members(sa + st, B);  // the candidates' SLO counts search them
            }
            nbw += nfull;
            i += (uint32_t)nfull * B;
            if (nfull == 32) continue;
            if (i >= iend) break;
            uint32_t j = 0;
            if (lane == 0) {  // closed by the timeout: first member beyond a0 + T (or the cursor)
              const uint32_t b0 = sa[i];
              const int64_t dl = (int64_t)b0 + Tm;
              const uint32_t lim = iend - i > B ? i + B : iend;
              uint32_t lo = i + 1, hi = lim;
#pragma unroll 1
              while (lo < hi) {
                const uint32_t mid = (lo + hi) >> 1;
                if ((int64_t)sa[mid] > dl) hi = mid; else lo = mid + 1;
              }
              j = lo;
              const uint32_t blast = sa[j - 1];
              const uint32_t ready = (j - i == B) ? blast : (uint32_t)dl;
              if (nbw < kBC) {
                ws.key[nbw] = ((uint64_t)ready << 32) | tag | (uint64_t)((i - ibase) & 0x1FFFFFF);
                ws.ready[nbw] = ready;
                ws.info[nbw] = (j - i) | ((uint32_t)m << 16) | ((uint32_t)(strict ? 1 : 0) << 24);
                ws.pos[nbw] = i;
                ws.afirst[nbw] = b0;
                ws.alast[nbw] = blast;
              }
            }
            nbw += 1;
            i = __shfl_sync(0xffffffffu, j, 0);
          }
        }
      }
      if (lane == 0) ws.nb = nbw;
    }
    __syncwarp();
    const int nb = ws.nb;
    UnitBats* ubu = P.ub ? P.ub + u : nullptr;
    if (ubu && lane == 0) ubu->nb = (uint32_t)nb;
    if (nb > kBC) {  // the chain scores this epoch itself (the lean chain cannot hold it)
      if (lane == 0) {
        if (kout) kout[0] = INT64_MIN;
        if (P.overflow) atomicOr(P.overflow, 1);
      }
      __syncwarp();
      continue;
    }
    // ---- id order (O3): rank by key
    {  // nb <= kBC = 64: lane ranks batches lane and lane + 32 in one pass over the keys
      const int b0 = lane, b1 = lane + 32;
      const uint64_t k0 = b0 < nb ? ws.key[b0] : ~0ull, k1 = b1 < nb ? ws.key[b1] : ~0ull;
      int r0 = 0, r1 = 0;
#pragma unroll 4
      for (int x = 0; x < nb; ++x) {
        const uint64_t kx = ws.key[x];
        r0 += kx < k0 ? 1 : 0;
        r1 += kx < k1 ? 1 : 0;
      }
#pragma unroll
      for (int h = 0; h < 2; ++h) {
        const int b = h ? b1 : b0, rank = h ? r1 : r0;
        if (b >= nb) continue;
        ws.ord[rank] = (uint8_t)b;
        if (ubu) {  // the epoch's batches in id order for the lean chain / accounting
          ubu->ready[rank] = ws.ready[b];
          ubu->info[rank] = ws.info[b];
          ubu->pos[rank] = ws.pos[b];
        }
      }
    }
    __syncwarp();
    if (!kout) continue;  // rows only: no candidate keys (Alg 2's heuristic decides, policy 2)
    // ---- candidates: lane per (residue class c, geometry j), Alg 1 from idle
    bool bad = false, wide = false;
#pragma unroll 1
    for (int p0 = 0; p0 < npairs; p0 += 32) {
      const int pi = p0 + lane;
      const bool act = pi < npairs;
      const int c = act ? pi % N : 0;
      const int j = act ? gord[pi / N] : 0;
      const int nbc = act && c < nb ? (nb - c + N - 1) / N : 0;
      if (nbc > kKC) bad = true;
      const int nx = nbc > kKC ? 0 : nbc;
      const int ns = act ? T.gn[j] : 0;
      const uint8_t* gp = T.gprof + j * 8;
      const int32_t* gpref = T.gpref + j * 8;
#pragma unroll
      for (int s = 0; s < kMaxSl; ++s) {
        ws.ls[s][lane] = 0;
        ws.msk[s][lane] = 0;
      }
      uint32_t alive = 0;  // placed batches still running at the current ready time
      int be = 0;          // their best-effort footprint
      int64_t misses = 0, tail = 0;
#pragma unroll 1
      for (int x = 0; x < nx; ++x) {
        const int b = ws.ord[c + x * N];
        const uint32_t info = ws.info[b];
        const int m = (info >> 16) & 0xFF, nreq = info & 0xFFFF;
        const bool strict = (info >> 24) & 1;
        const uint32_t rt = ws.ready[b] - (uint32_t)eW;  // ready - eW in [0, W); ready order
        // residents that ended by rt never matter again (ready times ascend along the class)
        uint32_t occ = 0;  // slices with a resident still running at rt
#pragma unroll 1
        for (uint32_t a = alive; a; a &= a - 1) {
          const int i = __ffs(a) - 1;
          const uint32_t pki = ws.pk[i][lane];
          if (ws.en[i][lane] <= rt) {
            alive &= ~(1u << i);
            if (pki >> 27) be -= (int)(pki & kMemMask);
          } else {
            occ |= 1u << ((pki >> 24) & 7);
          }
        }
        const int32_t q = T.mem[m];
        const int32_t* fbr_m = T.fbr + m * kNProf;
        const int32_t* solo_m = T.solo + m * kNProf;
        // slice keys in 32 bits: completions < 2^25 us past eW (else the unit goes to the chain):
        // strict = inelig << 31 | c << 6 | (4 - p) << 3 | s, best-effort = start << 3 | s
        uint32_t best = 0xFFFFFFFFu;
        uint32_t bst = 0, bc = 0;
        // the slices of j that hold the batch's footprint (q <= Ms), none without room (Q39)
        uint32_t fit = __popc(alive) < P.max_live ? (uint32_t)fitm[j * M + m] : 0u;
        // An idle slice (no resident running at rt; its last start is below rt) starts the batch
        // at rt alone: exec = solo (F = its own FBR <= 10^6), so idle slices of one profile tie on
        // completion and differ only in the tag bit and the position.  Only the lowest of them --
        // and, for a strict batch, the lowest one past the tag walk's threshold (pref[s] > be,
        // pref ascending in s) -- can hold the minimum key: the rest are dropped unevaluated.
        if (const uint32_t idle = fit & ~occ) {
          uint32_t elig = 0;
          if (strict) {
#pragma unroll 1
            for (int s = 0; s < kMaxSl && !elig; ++s)
              if (s < ns && gpref[s] > be) elig = ~((1u << s) - 1u);
          }
          uint32_t keep = 0;
#pragma unroll
          for (int pp = 0; pp < kNProf; ++pp) {
            const uint32_t ip = idle & pmask[j * kNProf + pp];
            const uint32_t ie = ip & elig;
            keep |= (ip & (0u - ip)) | (ie & (0u - ie));
          }
          fit = (fit & occ) | keep;
        }
        const uint32_t sflag = strict ? 0xFFFFFFFFu : 0u;
#pragma unroll 1
        for (; fit; fit &= fit - 1) {
          const int s = __ffs(fit) - 1;
          const int p = gp[s];
          const uint32_t lss = ws.ls[s][lane];
          const uint32_t t0 = rt > lss ? rt : lss;
          const uint32_t set = ws.msk[s][lane] & alive;
          int32_t used = 0;
          uint32_t F = (uint32_t)fbr_m[p];
#pragma unroll 1
          for (uint32_t a = set; a; a &= a - 1) {  // Eq 1's co-runners at t0
            const int i = __ffs(a) - 1;
            if (ws.en[i][lane] > t0) {
              used += (int32_t)(ws.pk[i][lane] & kMemMask);
              F += (uint32_t)ws.fb[i][lane];
            }
          }
          uint32_t start = t0;
          if (used + q > T.cap[p]) {
            F = (uint32_t)fbr_m[p];
            start = mem_wait(ws, lane, set, t0, q, T.cap[p], &F);
          }
          // Eq 1: exec = floor(solo * max(F, 10^6) / 10^6) = solo when F <= 10^6.  Completions at or
          // past 2^25 us clamp to 2^25 - 1 in the key (a clamped slice can only win when every
          // slice clamps, and then the unit goes to the chain: checked once per batch below)
          const int32_t so = solo_m[p];
          const int64_t ex = F <= (uint32_t)kPpm ? (int64_t)so : exec_time(so, F);
          const uint32_t cc = ex >= (1 << 25) ? (1u << 25) : min(start + (uint32_t)ex, 1u << 25);
          const uint32_t ks = ((be >= gpref[s]) ? 0x80000000u : 0u) | (min(cc, (1u << 25) - 1u) << 6) |
                              ((uint32_t)(4 - p) << 3) | (uint32_t)s;   // choose_strict_slice (Q11)
          const uint32_t kb = (start << 3) | (uint32_t)s;               // choose_best_effort_slice (Q12)
          const uint32_t key = (ks & sflag) | (kb & ~sflag);
          if (key < best) {
            best = key;
            bst = start;
            bc = cc;
          }
        }
        wide |= best != 0xFFFFFFFFu && bc >= (1u << 25) - 1u;  // ends and keys are held in 25 bits
        const int bsl = best & 7;
        const bool placed = best != 0xFFFFFFFFu;
        ws.en[x][lane] = placed ? bc : 0u;
        ws.pk[x][lane] = (uint32_t)q | ((uint32_t)bsl << 24) | (strict ? 0u : (1u << 27));
        ws.fb[x][lane] = fbr_m[gp[bsl]];
        if (placed) {
          ws.ls[bsl][lane] = bst;
          ws.msk[bsl][lane] |= (uint16_t)(1u << x);
          alive |= 1u << x;
          if (!strict) be += q;
        }
        const int64_t cw = eW + (int64_t)bc;  // absolute completion
        if (strict) {
          if (!placed) {
            misses += nreq;
          } else {  // latencies fall along the sorted members: test the ends first
            const int64_t slo = T.slo[m];
            if (cw - (int64_t)ws.afirst[b] > slo)
              misses += (cw - (int64_t)ws.alast[b] > slo) ? nreq : nreq - hits_from(sa + ws.pos[b], nreq, cw, slo);
          }
        } else {
          const int64_t tbv = placed ? cw - (int64_t)ws.afirst[b] : (int64_t)0xFFFFFFFFLL;
          tail = tbv > tail ? tbv : tail;
        }
      }
      if (act) kout[c * G + j] = key_of(misses, tail, j + 1);
    }
    if (__any_sync(0xffffffffu, bad || wide)) {
      __syncwarp();
      if (lane == 0) kout[0] = INT64_MIN;
    }
    __syncwarp();
  }
}

}  // namespace

size_t cand_smem_bytes(const TabLayout& tl, size_t* ws_off) {
  const size_t o = (((size_t)tl.words * 4 + 15) & ~(size_t)15) + (((size_t)tl.G + 15) & ~(size_t)15) +
                   (((size_t)tl.G * tl.M + (size_t)tl.G * kNProf + 15) & ~(size_t)15);
  *ws_off = o;
  return o + sizeof(WarpSmem) * kCandWarps;
}

cudaError_t launch_walk(const CandParams& P, cudaStream_t st) {
  const int64_t n = (int64_t)P.R * P.S * 32;  // a warp per (replica, stream)
  walk_kernel<<<(unsigned)((n + 255) / 256), 256, 0, st>>>(P);
  return cudaGetLastError();
}

cudaError_t launch_cand(const CandParams& P, int grid, cudaStream_t st) {
  size_t off = 0;
  const size_t smem = cand_smem_bytes(P.tl, &off);
  cand_kernel<<<grid, 32 * kCandWarps, smem, st>>>(P);
  return cudaGetLastError();
}

cudaError_t cand_occupancy(const TabLayout& tl, int* per_sm) {
  size_t off = 0;
  const size_t smem = cand_smem_bytes(tl, &off);
  cudaError_t e = cudaFuncSetAttribute(cand_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
  if (e != cudaSuccess) return e;
  return cudaOccupancyMaxActiveBlocksPerMultiprocessor(per_sm, cand_kernel, 32 * kCandWarps, smem);
}

cudaError_t preload_cand_kernels() {
  cudaFuncAttributes a;
  cudaError_t e = cudaFuncGetAttributes(&a, walk_kernel);
  if (e != cudaSuccess) return e;
  return cudaFuncGetAttributes(&a, cand_kernel);
}

}  // namespace pemgpu
