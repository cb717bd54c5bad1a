// replay.cu — the fused B200 epoch engine (sm_100a): one CTA per trace replica, persistent
// over its E epochs.  Per epoch (O5):
//   A  VM events + pending installs (thread per simulated GPU)            O11, O5.3
//   B  stream partition of the epoch's request window in shared memory   O3
//   C  batch formation per (model, class) stream, id-order rank sort     O3
//   D  round-robin dispatch (closed form when every GPU is available)    Q18
//   E  placement lanes: lane = (sim-GPU, actual | candidate geometry);   O6 + O8 (Alg 1, Eq 1/2,
//      candidates replay the GPU-epoch from idle and pack an int64 key    the "Oracle" P:L485)
//   F  per-request accounting: SLO hits, log-linear histogram (smem)     O7
//   G  argmin + Alg 2 hysteresis + ~30% cap                              O9, O10
// The request stream (5 B/request) is read from HBM once, with coalesced loads; everything else
// lives in shared memory, registers and L1/L2-resident per-CTA scratch.
#include <cuda_runtime.h>
#include "replay.cuh"

namespace pemgpu {

namespace {

struct Ctx {
  Tab T;
  uint32_t* hist;
  int *s_cnt, *s_run, *s_base, *s_tot, *s_skip, *s_pend;
  uint8_t *g_geom, *g_target, *g_ctr, *g_vm, *g_bill, *g_dec, *g_best, *g_want;
  int64_t *g_rs, *g_re, *g_from, *g_until, *g_since, *g_maxend, *g_kbest, *g_kcur, *g_od,
      *g_spot, *g_busy, *g_mem;
  int *g_cnt, *g_off;
  int64_t* keys;
  Bat *sb, *gb;
  uint32_t *sord, *gord, *sgl, *ggl, *ssarr, *gsarr;
  int BS, WS;
  protean_resident* lists;
  int* lane_n;
  int64_t *ls, *bu;  // [N][7]
  __device__ __forceinline__ Bat& bat(int i) const { return i < BS ? sb[i] : gb[i - BS]; }
  __device__ __forceinline__ uint32_t& ord(int i) const { return i < BS ? sord[i] : gord[i - BS]; }
  __device__ __forceinline__ uint32_t& gl(int i) const { return i < BS ? sgl[i] : ggl[i - BS]; }
  __device__ __forceinline__ uint32_t& sa(int i) const { return i < WS ? ssarr[i] : gsarr[i - WS]; }
};

struct CtaState {
  int64_t w_lo, lt_total, nlog;
  int nb, cursor, all_avail, bad;
  unsigned amin;
  unsigned long long cnt[10];
};

enum { VM_NONE = 0, VM_OD = 1, VM_SPOT = 2 };

__device__ __forceinline__ int64_t clip_h(int64_t x, int64_t H) { return x < H ? x : H; }

__device__ void bill_switch(const Ctx& c, int g, int type, int64_t at, int64_t H) {
  const int64_t d = clip_h(at, H) - clip_h(c.g_since[g], H);
  if (c.g_bill[g] == VM_OD) c.g_od[g] += d;
  if (c.g_bill[g] == VM_SPOT) c.g_spot[g] += d;
  c.g_bill[g] = (uint8_t)type;
  c.g_since[g] = at;
}

__device__ void reset_gpu_state(const Ctx& c, int g, int geom) {
  c.g_geom[g] = (uint8_t)geom;
  c.g_target[g] = kNoGeom;
  c.g_ctr[g] = 0;
  c.lane_n[g] = 0;
#pragma unroll
  for (int s = 0; s < kMaxSl; ++s) {
    c.ls[g * kMaxSl + s] = 0;
    c.bu[g * kMaxSl + s] = 0;
  }
}

__device__ __forceinline__ bool has_vm(const Ctx& c, int g, int64_t t) {
  return c.g_from[g] <= t && t < c.g_until[g];
}
__device__ __forceinline__ bool available(const Ctx& c, int g, int64_t t) {
  return has_vm(c, g, t) && !(c.g_rs[g] <= t && t < c.g_re[g]);
}

// O11: one revocation boundary tau = k * T_rev for node g (draws specified in DESIGN.md §3).
__device__ void vm_event(const ReplayParams& P, const Ctx& c, uint64_t replica, int g, int64_t k,
                         int64_t tau) {
  const uint64_t x = (replica << 32) ^ ((uint64_t)g << 20) ^ ((uint64_t)k << 2);
  const uint64_t d0 = smix(P.seed ^ smix(x ^ 0ull)) >> 11;
  const uint64_t d1 = smix(P.seed ^ smix(x ^ 1ull)) >> 11;
  const bool revoked = d0 < P.thr, spot_ok = d1 >= P.thr;
  if (P.vm_policy == 1) {
    if (c.g_vm[g] == VM_SPOT) {
      if (revoked && !spot_ok) {
        c.g_vm[g] = VM_OD;
        bill_switch(c, g, VM_OD, tau + P.notice, P.H);
      }
    } else if (c.g_vm[g] == VM_OD) {
      if (spot_ok) {
        c.g_vm[g] = VM_SPOT;
        bill_switch(c, g, VM_SPOT, tau, P.H);
      }
    }
  } else if (P.vm_policy == 2) {
    if (c.g_vm[g] == VM_SPOT) {
      if (revoked && !spot_ok) {
        c.g_vm[g] = VM_NONE;
        c.g_until[g] = tau;
        bill_switch(c, g, VM_NONE, tau + P.notice, P.H);
        c.g_target[g] = kNoGeom;
        c.g_rs[g] = c.g_re[g] = 0;
      }
    } else if (c.g_vm[g] == VM_NONE) {
      if (spot_ok) {
        c.g_vm[g] = VM_SPOT;
        c.g_from[g] = tau;
        c.g_until[g] = kForever;
        bill_switch(c, g, VM_SPOT, tau, P.H);
        reset_gpu_state(c, g, P.init_geom);
        c.g_rs[g] = c.g_re[g] = 0;
      }
    }
  }
}

__device__ __forceinline__ void install(const Ctx& c, int g) { reset_gpu_state(c, g, c.g_target[g]); }

// Packed u16 smem histogram; a half crossing 2^15 moves 2^15 counts to the HBM histogram
// (cnt <= 32 per call, so a half never exceeds 0xFFFF before the move).
__device__ __forceinline__ void hist_add(const Ctx& c, uint32_t* ghist, int idx, uint32_t cnt) {
  const int w = idx >> 1, sh = (idx & 1) * 16;
  const uint32_t old = (atomicAdd(&c.hist[w], cnt << sh) >> sh) & 0xFFFFu;
  if (old < 0x8000u && old + cnt >= 0x8000u) {
    atomicSub(&c.hist[w], 0x8000u << sh);
    atomicAdd(&ghist[idx], 0x8000u);
  }
}

__device__ __forceinline__ int hits_in(const Ctx& c, int pos, int n, int64_t end, int64_t slo) {
  const int64_t need = end - slo;  // c - a <= slo  <=>  a >= c - slo
  int lo = 0, hi = n;
  while (lo < hi) {
    const int mid = (lo + hi) >> 1;
    if ((int64_t)c.sa(pos + mid) >= need) hi = mid; else lo = mid + 1;
  }
  return n - lo;
}

}  // namespace

__global__ void __launch_bounds__(256, 2) replay_kernel(ReplayParams P) {
  extern __shared__ __align__(16) unsigned char smem[];
  __shared__ CtaState cs;
  const SmemLayout& SL = P.sl;
  const int tid = threadIdx.x, NT = blockDim.x, lane = tid & 31, warp = tid >> 5, NW = NT >> 5;
  const int N = P.N, S = SL.S, Gc = SL.Gc;

  Ctx c;
  int32_t* tabw = reinterpret_cast<int32_t*>(smem + SL.tab);
#pragma unroll 1
  for (int i = tid; i < P.tl.words; i += NT) tabw[i] = P.tab[i];
  c.T.bind(tabw, P.tl);
  c.hist = reinterpret_cast<uint32_t*>(smem + SL.hist);
  c.s_cnt = reinterpret_cast<int*>(smem + SL.s_cnt);
  c.s_run = reinterpret_cast<int*>(smem + SL.s_run);
  c.s_base = reinterpret_cast<int*>(smem + SL.s_base);
  c.s_tot = reinterpret_cast<int*>(smem + SL.s_tot);
  c.s_skip = reinterpret_cast<int*>(smem + SL.s_skip);
  c.s_pend = reinterpret_cast<int*>(smem + SL.s_pend);
  uint8_t* gu8 = smem + SL.g_u8;
  c.g_geom = gu8; c.g_target = gu8 + N; c.g_ctr = gu8 + 2 * N; c.g_vm = gu8 + 3 * N;
  c.g_bill = gu8 + 4 * N; c.g_dec = gu8 + 5 * N; c.g_best = gu8 + 6 * N; c.g_want = gu8 + 7 * N;
  int64_t* gi = reinterpret_cast<int64_t*>(smem + SL.g_i64);
  c.g_rs = gi; c.g_re = gi + N; c.g_from = gi + 2 * N; c.g_until = gi + 3 * N;
  c.g_since = gi + 4 * N; c.g_maxend = gi + 5 * N; c.g_kbest = gi + 6 * N; c.g_kcur = gi + 7 * N;
  c.g_od = gi + 8 * N; c.g_spot = gi + 9 * N; c.g_busy = gi + 10 * N; c.g_mem = gi + 11 * N;
  c.g_cnt = reinterpret_cast<int*>(smem + SL.g_i32);
  c.g_off = c.g_cnt + N;
  c.keys = reinterpret_cast<int64_t*>(smem + SL.keys);
  c.BS = SL.BS;
  c.WS = SL.WS;
  c.sb = reinterpret_cast<Bat*>(smem + SL.bats);
  c.sord = reinterpret_cast<uint32_t*>(smem + SL.ord);
  c.sgl = reinterpret_cast<uint32_t*>(smem + SL.glist);
  c.ssarr = reinterpret_cast<uint32_t*>(smem + SL.sarr);
  char* slot = P.scratch + (size_t)blockIdx.x * P.slot_bytes;
  c.lists = reinterpret_cast<protean_resident*>(slot + P.o_lists);
  c.lane_n = reinterpret_cast<int*>(slot + P.o_lane_n);
  c.ls = reinterpret_cast<int64_t*>(slot + P.o_ls);
  c.bu = reinterpret_cast<int64_t*>(slot + P.o_bu);
  c.gb = reinterpret_cast<Bat*>(slot + P.o_gbat);
  c.gord = reinterpret_cast<uint32_t*>(slot + P.o_gord);
  c.ggl = reinterpret_cast<uint32_t*>(slot + P.o_gglist);
  c.gsarr = reinterpret_cast<uint32_t*>(slot + P.o_gsarr);
  const Tab& T = c.T;
  int sum_slots = 0;  // sum of slice counts over the candidate range (slot-evals per batch)
  __syncthreads();
#pragma unroll 1
  for (int j = P.geom_lo; j < P.geom_hi; ++j) sum_slots += T.gn[j];
  const int LPG = (1 + Gc) <= 16 ? 16 : ((1 + Gc + 31) / 32) * 32;  // lanes per simulated GPU
  const int nlp = N * LPG;

#pragma unroll 1
  for (int r = blockIdx.x; r < P.R; r += gridDim.x) {
    const uint64_t replica = (uint64_t)(P.base + r);
    const int64_t r_lo = P.roff[r];
    const int64_t* eoff = P.eoff + (size_t)r * (P.E + 1);
    uint32_t* ghist = P.hist + (size_t)r * 2 * kNB;
    int64_t cnt[10];
#pragma unroll
    for (int i = 0; i < 10; ++i) cnt[i] = 0;

    // ---------------------------------------------------------------- replica init
#pragma unroll 1
    for (int i = tid; i < kNB; i += NT) c.hist[i] = 0;          // kNB words = 2*3328 halves
#pragma unroll 1
    for (int i = tid; i < 2 * kNB; i += NT) ghist[i] = 0;
#pragma unroll 1
    for (int k = tid; k < S; k += NT) c.s_skip[k] = 0;
#pragma unroll 1
    for (int g = tid; g < N; g += NT) {
      reset_gpu_state(c, g, P.init_geom);
      c.g_vm[g] = c.g_bill[g] = (P.vm_policy == 0) ? VM_OD : VM_SPOT;
      c.g_rs[g] = c.g_re[g] = 0;
      c.g_from[g] = 0;
      c.g_until[g] = kForever;
      c.g_since[g] = 0;
      c.g_od[g] = c.g_spot[g] = c.g_busy[g] = c.g_mem[g] = 0;
    }
    if (tid == 0) {
      cs.w_lo = r_lo;
      cs.nlog = 0;
      cs.cursor = 0;
      cs.bad = 0;
#pragma unroll
      for (int i = 0; i < 10; ++i) cs.cnt[i] = 0;
    }
    __syncthreads();

#pragma unroll 1
    for (int64_t e = 0; e < P.E; ++e) {
      const int64_t eW = e * P.W, Tend = eW + P.W;
      // ---------------------------------------------------------------- A: VM events, installs
#pragma unroll 1
      for (int i = tid; i < kNSeg * S; i += NT) c.s_cnt[i] = 0;
#pragma unroll 1
      for (int g = tid; g < N; g += NT) {
        if (P.vm_policy != 0) {
#pragma unroll 1
          for (int64_t k = (eW + P.rev - 1) / P.rev; k * P.rev < Tend; ++k) {
            const int64_t tau = k * P.rev;
            if (k < 1 || tau >= P.H) continue;
            if (c.g_target[g] != kNoGeom && c.g_re[g] <= tau) install(c, g);
            vm_event(P, c, replica, g, k, tau);
          }
        }
        if (c.g_target[g] != kNoGeom && c.g_re[g] <= Tend) install(c, g);
        c.g_dec[g] = (has_vm(c, g, Tend) && c.g_re[g] <= Tend) ? 1 : 0;
        c.g_want[g] = 0;
        c.g_best[g] = kNoGeom;
        c.g_kcur[g] = -1;
      }
      if (tid == 0) {
        cs.nb = 0;
        cs.amin = 0xFFFFFFFFu;
        cs.lt_total = 0;
        cs.all_avail = 1;
      }
      const int64_t w_beg = eoff[e], w_end = eoff[e + 1];
      const int64_t w_lo = cs.w_lo;
      __syncthreads();
#pragma unroll 1
      for (int g = tid; g < N; g += NT) {
        const bool whole = c.g_from[g] <= eW && c.g_until[g] >= Tend &&
                           !(c.g_rs[g] < Tend && c.g_re[g] > eW);
        if (!whole) cs.all_avail = 0;
      }
      const int64_t len = w_end - w_lo;
      const bool bad_window = len < 0 || len > P.WCAP || w_beg < w_lo;
      if (bad_window) {
        if (tid == 0) atomicOr(P.err, 1);
      }
      // ---------------------------------------------------------------- B: stream partition
      if (!bad_window && warp < kNSeg) {  // count per (segment, stream); 4 loads in flight per lane
        const int64_t a = w_lo + len * warp / kNSeg, b = w_lo + len * (warp + 1) / kNSeg;
        int* cntw = c.s_cnt + warp * S;
#pragma unroll 1
        for (int64_t i0 = a; i0 < b; i0 += 128) {
          uint8_t mt[4];
#pragma unroll
          for (int u = 0; u < 4; ++u) {
            const int64_t i = i0 + u * 32 + lane;
            mt[u] = i < b ? P.meta[i] : (uint8_t)0xFF;
          }
#pragma unroll
          for (int u = 0; u < 4; ++u) {
            const bool valid = i0 + u * 32 + lane < b;
            int m = mt[u] & 63;
            if (m >= T.M) m = 0;
            const int key = valid ? 2 * m + ((mt[u] >> 7) ? 0 : 1) : 1024 + lane;
            const unsigned peers = __match_any_sync(0xffffffffu, key);
            if (valid && (peers & ((1u << lane) - 1u)) == 0) cntw[key] += __popc(peers);
          }
        }
      }
      __syncthreads();
      if (warp == 0) {  // stream offsets: per-stream totals, exclusive scan over streams
        int carry = 0;
#pragma unroll 1
        for (int k0 = 0; k0 < S; k0 += 32) {
          const int k = k0 + lane;
          int tot = 0;
          if (k < S) {
#pragma unroll 1
            for (int w = 0; w < kNSeg; ++w) {
              const int cv = c.s_cnt[w * S + k];
              c.s_run[w * S + k] = tot;
              tot += cv;
            }
          }
          int x = tot;
#pragma unroll
          for (int d = 1; d < 32; d <<= 1) {
            const int y = __shfl_up_sync(0xffffffffu, x, d);
            if (lane >= d) x += y;
          }
          const int base = carry + x - tot;
          if (k < S) {
            c.s_base[k] = base;
            c.s_tot[k] = tot;
#pragma unroll 1
            for (int w = 0; w < kNSeg; ++w) c.s_run[w * S + k] += base;
          }
          carry += __shfl_sync(0xffffffffu, x, 31);
        }
      }
      __syncthreads();
      if (!bad_window && warp < kNSeg) {  // stable scatter into stream-sorted order + validation
        const int64_t a = w_lo + len * warp / kNSeg, b = w_lo + len * (warp + 1) / kNSeg;
        int* runw = c.s_run + warp * S;
#pragma unroll 1
        for (int64_t i0 = a; i0 < b; i0 += 128) {
          uint8_t mt[4];
          uint32_t ai[4], ap[4];
#pragma unroll
          for (int u = 0; u < 4; ++u) {
            const int64_t i = i0 + u * 32 + lane;
            const bool valid = i < b;
            mt[u] = valid ? P.meta[i] : (uint8_t)0;
            ai[u] = valid ? P.arr[i] : 0u;
            ap[u] = (valid && i >= w_beg && i > r_lo) ? P.arr[i - 1] : 0u;
          }
#pragma unroll
          for (int u = 0; u < 4; ++u) {
            const int64_t i = i0 + u * 32 + lane;
            const bool valid = i < b;
            int m = mt[u] & 63;
            if (valid && i >= w_beg &&  // validate each request once (when it is new)
                ((mt[u] & 0x40) || m >= T.M || (int64_t)ai[u] >= P.trace_len || ai[u] < ap[u]))
              atomicOr(P.err, 1);
            if (m >= T.M) m = 0;
            const int key = valid ? 2 * m + ((mt[u] >> 7) ? 0 : 1) : 1024 + lane;
            const unsigned peers = __match_any_sync(0xffffffffu, key);
            const unsigned rank = __popc(peers & ((1u << lane) - 1u));
            if (valid) c.sa(runw[key] + (int)rank) = ai[u];
            __syncwarp();
            if (valid && rank == 0) runw[key] += __popc(peers);
            __syncwarp();
          }
        }
      }
      __syncthreads();
      // ---------------------------------------------------------------- C: batch formation
      // warp per stream: lanes test 32 consecutive B-sized batches at once (full batches are the
      // common case); a batch closed by the timeout, or still open, is resolved by lane 0.
#pragma unroll 1
      for (int k = warp; k < S; k += NW) {
        if (bad_window) break;
        const int m = k >> 1;
        const bool strict = (k & 1) == 0;
        const int B = T.bsz[m];
        const int64_t Tm = T.tmo[m];
        int i = c.s_base[k] + c.s_skip[k];
        const int end = c.s_base[k] + c.s_tot[k];
        int pend = 0;
        uint32_t a0p = 0xFFFFFFFFu;
        while (i < end) {
          const int64_t st = (int64_t)i + (int64_t)lane * B;
          bool full = false;
          if (st + B <= end) full = (int64_t)c.sa((int)(st + B - 1)) <= (int64_t)c.sa((int)st) + Tm;
          const unsigned fm = __ballot_sync(0xffffffffu, full);
          const int nfull = __ffs(~fm) ? __ffs(~fm) - 1 : 32;
          int slot0 = 0;
          if (lane == 0 && nfull) slot0 = atomicAdd(&cs.nb, nfull);
          slot0 = __shfl_sync(0xffffffffu, slot0, 0);
          if (lane < nfull) {
            const int ii = (int)st;
            const uint32_t ready = c.sa(ii + B - 1);
            Bat& bt = c.bat(slot0 + lane);
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
          // batch starting at i is not full within this window: lane 0 resolves it
          int j = 0, state = 0;  // state 0 emit, 1 pending
          int64_t ready = 0;
          if (lane == 0) {
            const int64_t a0 = c.sa(i);
            const int64_t deadline = a0 + Tm;
            const int lim = (end - i > B) ? i + B : end;
            int lo = i + 1, hi = lim;  // first member beyond the timeout, else lim
            while (lo < hi) {
              const int mid = (lo + hi) >> 1;
              if ((int64_t)c.sa(mid) > deadline) hi = mid; else lo = mid + 1;
            }
            j = lo;
            if (j - i == B) ready = c.sa(j - 1);        // full (only possible at the window end)
            else if (j < end) ready = deadline;         // a later arrival missed the timeout
            else if (deadline < Tend) ready = deadline; // timed out inside this epoch
            else { state = 1; pend = end - i; a0p = (uint32_t)a0; }
            if (state == 0) {
              const int slot = atomicAdd(&cs.nb, 1);
              Bat& bt = c.bat(slot);
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
        if (lane == 0) {
          c.s_pend[k] = pend;
          if (pend) atomicMin(&cs.amin, a0p);
        }
      }
      __syncthreads();
      const int nb = cs.nb;
      const unsigned amin = cs.amin;
      // next window: stream entries at/after the earliest open batch's first arrival are re-read
#pragma unroll 1
      for (int k = tid; k < S; k += NT) {
        if (bad_window) break;
        const int b0 = c.s_base[k], tot = c.s_tot[k];
        int lo = 0, hi = tot;
        while (lo < hi) {
          const int mid = (lo + hi) >> 1;
          if (c.sa(b0 + mid) >= amin) hi = mid; else lo = mid + 1;
        }
        const int ge = tot - lo;
        if (lo) atomicAdd(reinterpret_cast<unsigned long long*>(&cs.lt_total), (unsigned long long)lo);
        c.s_skip[k] = ge - c.s_pend[k];
      }
#pragma unroll 1
      for (int b = tid; b < nb; b += NT) {  // id order (O3): rank by key
        const uint64_t kb = c.bat(b).key;
        int rank = 0;
#pragma unroll 1
        for (int x = 0; x < nb; ++x) rank += (c.bat(x).key < kb) ? 1 : 0;
        c.ord(rank) = (uint32_t)b;
      }
      __syncthreads();
      if (tid == 0) cs.w_lo = bad_window ? w_end : w_lo + cs.lt_total;
      // ---------------------------------------------------------------- D: dispatch
      if (cs.all_avail) {
        const int cursor = cs.cursor;
#pragma unroll 1
        for (int rk = tid; rk < nb; rk += NT) c.bat(c.ord(rk)).gpu = (uint8_t)((cursor + rk) % N);
#pragma unroll 1
        for (int g = tid; g < N; g += NT) {
          const int d = (g - cursor % N + N) % N;
          const int cntg = d < nb ? (nb - d + N - 1) / N : 0;
          c.g_cnt[g] = cntg;
          // offset = sum of counts of GPUs before g
          int off = 0;
#pragma unroll 1
          for (int h = 0; h < g; ++h) {
            const int dh = (h - cursor % N + N) % N;
            off += dh < nb ? (nb - dh + N - 1) / N : 0;
          }
          c.g_off[g] = off;
          if (g == N - 1) c.g_off[N] = off + cntg;
        }
        __syncthreads();
#pragma unroll 1
        for (int rk = tid; rk < nb; rk += NT) {
          const int g = (cursor + rk) % N;
          c.gl(c.g_off[g] + rk / N) = c.ord(rk);
        }
        if (tid == 0) cs.cursor = (int)((cursor + nb) % N);
      } else if (N <= 32) {
        if (warp == 0) {  // lanes = simulated GPUs; availability masks + cursor chase
          int64_t fr = 0, un = 0, rs = 0, re = 0;
          if (lane < N) { fr = c.g_from[lane]; un = c.g_until[lane]; rs = c.g_rs[lane]; re = c.g_re[lane]; }
          int cur = cs.cursor, mycnt = 0;
#pragma unroll 1
          for (int rk = 0; rk < nb; ++rk) {
            Bat& bt = c.bat(c.ord(rk));
            const int64_t t = bt.ready;
            const bool av = lane < N && fr <= t && t < un && !(rs <= t && t < re);
            const unsigned am = __ballot_sync(0xffffffffu, av);
            int chosen = -1;
            if (am) {
              const unsigned hi = am & ~((1u << cur) - 1u);
              chosen = hi ? __ffs(hi) - 1 : __ffs(am) - 1;
              cur = (chosen + 1) % N;
              if (lane == chosen) ++mycnt;
            }
            if (lane == 0) {
              bt.gpu = chosen < 0 ? (uint8_t)0xFF : (uint8_t)chosen;
              if (chosen < 0) bt.drop = 1;  // dispatch drop
            }
          }
          int x = mycnt;
#pragma unroll
          for (int d = 1; d < 32; d <<= 1) {
            const int y = __shfl_up_sync(0xffffffffu, x, d);
            if (lane >= d) x += y;
          }
          if (lane < N) c.g_off[lane] = x - mycnt;
          if (lane == N - 1) c.g_off[N] = x;
          __syncwarp();
          int fill = 0;
#pragma unroll 1
          for (int rk = 0; rk < nb; ++rk) {
            const uint32_t b = c.ord(rk);
            const int g = c.bat(b).gpu;
            if (lane == g) c.gl(c.g_off[lane] + fill++) = b;
          }
          if (lane == 0) cs.cursor = cur;
        }
      } else {
        if (tid == 0) {
          int cur = cs.cursor;
#pragma unroll 1
          for (int g = 0; g < N; ++g) c.g_cnt[g] = 0;
#pragma unroll 1
          for (int rk = 0; rk < nb; ++rk) {
            Bat& bt = c.bat(c.ord(rk));
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
            const uint32_t b = c.ord(rk);
            const Bat& bt = c.bat(b);
            if (bt.drop) continue;
            c.gl(c.g_off[bt.gpu] + c.g_cnt[bt.gpu]++) = b;
          }
          cs.cursor = cur;
        }
      }
      __syncthreads();
      // ---------------------------------------------------------------- E: placement lanes
      // lane = (GPU g, v): v = 0 the actual placement on the current geometry (carried state),
      // v = 1..Gc candidate geometry v-1 replayed from idle on the same batch list (O8).
#pragma unroll 1
      for (int L = tid; L < nlp; L += NT) {
        const int g = L / LPG, v = L - g * LPG;
        if (g >= N || v > Gc) continue;
        const bool actual = v == 0;
        const int j = actual ? (int)c.g_geom[g] : P.geom_lo + v - 1;
        if (!actual && !(P.policy == 0 && c.g_dec[g])) {
          c.keys[g * Gc + v - 1] = -1;
          if (P.cand_keys) P.cand_keys[(((size_t)r * P.E + e) * N + g) * (size_t)T.G + j] = -1;
          continue;
        }
        const int x0 = c.g_off[g], x1 = c.g_off[g + 1];
        Rows rows{c.lists + (size_t)L * P.max_live};
        int n = actual ? c.lane_n[g] : 0;
        int64_t ls[kMaxSl];
#pragma unroll
        for (int s = 0; s < kMaxSl; ++s) ls[s] = actual ? c.ls[g * kMaxSl + s] : 0;
        int64_t acc0 = 0, acc1 = 0;  // actual: busy, mem-time;  candidate: misses, BE tail
#pragma unroll 1
        for (int x = x0; x < x1; ++x) {
          Bat& bt = c.bat(c.gl(x));
          const uint32_t info = bt.info;
          const int m = (info >> 16) & 0xFF, nreq = info & 0xFFFF;
          const bool strict = (info >> 24) & 1;
          const PlaceRes pr = place_lane(T, j, rows, n, ls, bt.ready, m, strict, P.max_live);
          if (actual) {
            bt.drop = (uint8_t)pr.dropped;
            bt.slice = pr.dropped ? 0xFF : (uint8_t)pr.slice;
            bt.start = pr.dropped ? 0 : pr.start;
            bt.end = pr.dropped ? 0 : pr.end;
            if (!pr.dropped) {  // busy union + memory-time, clipped to [0, H) (reading Q29)
              int64_t& b_until = c.bu[g * kMaxSl + pr.slice];
              const int64_t b_old = b_until;
              const int p = T.gprof[j * 8 + pr.slice];
              const int64_t lo = pr.start > b_old ? pr.start : b_old;
              const int64_t hi = pr.end < P.H ? pr.end : P.H;
              if (hi > lo) acc0 += (int64_t)prof_compute(p) * (hi - lo);
              if (pr.end > b_old) b_until = pr.end;
              if (hi > pr.start) acc1 += (int64_t)T.mem[m] * (hi - pr.start);
            }
          } else if (strict) {
            acc0 += pr.dropped ? nreq : nreq - hits_in(c, bt.pos, nreq, pr.end, T.slo[m]);
          } else {
            const int64_t tb = pr.dropped ? (int64_t)0xFFFFFFFFLL : pr.end - (int64_t)c.sa(bt.pos);
            acc1 = tb > acc1 ? tb : acc1;
          }
        }
        if (actual) {
          c.lane_n[g] = n;
          int64_t mx = 0;
#pragma unroll 1
          for (int i = 0; i < n; ++i) mx = rows.en(i) > mx ? rows.en(i) : mx;
          c.g_maxend[g] = mx;
#pragma unroll
          for (int s = 0; s < kMaxSl; ++s) c.ls[g * kMaxSl + s] = ls[s];
          c.g_busy[g] += acc0;
          c.g_mem[g] += acc1;
        } else {
          const int64_t key = make_key(acc0, acc1, j == c.g_geom[g] ? 0 : j + 1);
          if (j == c.g_geom[g]) c.g_kcur[g] = key;
          c.keys[g * Gc + v - 1] = key;
          if (P.cand_keys) P.cand_keys[(((size_t)r * P.E + e) * N + g) * (size_t)T.G + j] = key;
        }
      }
      __syncthreads();
      // ---------------------------------------------------------------- F: accounting (O7)
#pragma unroll 1
      for (int rk = warp; rk < nb; rk += NW) {
        const Bat& bt = c.bat(c.ord(rk));
        const int nreq = bt.info & 0xFFFF, m = (bt.info >> 16) & 0xFF;
        const bool strict = (bt.info >> 24) & 1;
        if (lane == 0) {
          if (strict) {
            cnt[0] += nreq;
            if (bt.drop) cnt[3] += nreq;
          } else {
            cnt[4] += nreq;
            if (bt.drop) cnt[6] += nreq;
          }
          const int64_t row = cs.nlog + rk;
          if (P.log && row < P.log_cap) {
            protean_batch_rec rec;
            rec.ready_us = bt.ready;
            rec.epoch = (uint32_t)e;
            rec.n_req = (uint16_t)nreq;
            rec.model = (uint8_t)m;
            rec.strict = strict ? 1 : 0;
            rec.gpu = bt.gpu;
            rec.slice = bt.slice;
            rec.dropped = bt.drop;
            rec.pad = 0;
            rec.start_us = bt.start;
            rec.end_us = bt.end;
            P.log[(size_t)r * P.log_cap + row] = rec;
          }
        }
        if (!bt.drop) {  // latencies are non-increasing along the sorted members: runs of equal
          const int64_t slo = T.slo[m];  // buckets become one histogram update
          const int cls = strict ? 0 : kNB;
#pragma unroll 1
          for (int i0 = 0; i0 < nreq; i0 += 32) {
            const int i = i0 + lane;
            const bool valid = i < nreq;
            const int64_t lat = valid ? bt.end - (int64_t)c.sa(bt.pos + i) : 0;
            const int bk = valid ? lat_bucket(lat) : -1;
            const int prev = __shfl_up_sync(0xffffffffu, bk, 1);
            const bool head = valid && (lane == 0 || prev != bk);
            const unsigned heads = __ballot_sync(0xffffffffu, head);
            const unsigned vmask = __ballot_sync(0xffffffffu, valid);
            const unsigned met = __ballot_sync(0xffffffffu, valid && lat <= slo);
            if (head) {
              const unsigned after = heads & ~((2u << lane) - 1u);
              const int stop = after ? __ffs(after) - 1 : 32 - __clz(vmask);
              hist_add(c, ghist, cls + bk, (uint32_t)(stop - lane));
            }
            if (lane == 0) {
              if (strict) {
                cnt[1] += __popc(met);
                cnt[2] += __popc(vmask) - __popc(met);
              } else {
                cnt[5] += __popc(vmask);
              }
            }
          }
        }
      }
      // ---------------------------------------------------------------- G: decisions (O9, O10)
#pragma unroll 1
      for (int g = tid; g < N; g += NT) {
        uint8_t dec_out = kNoGeom;
        if (P.policy == 0 && c.g_dec[g]) {
          int64_t kb = c.keys[g * Gc];
#pragma unroll 1
          for (int v = 1; v < Gc; ++v) kb = c.keys[g * Gc + v] < kb ? c.keys[g * Gc + v] : kb;
          const int cur = c.g_geom[g];
          const int tag = (int)(kb & 255);
          const int best = tag == 0 ? cur : tag - 1;
          dec_out = (uint8_t)best;
          c.g_best[g] = (uint8_t)best;
          c.g_kbest[g] = kb;
          if (best != cur) {
            if (c.g_ctr[g] >= P.wait_limit) c.g_want[g] = 1;
            else c.g_ctr[g]++;
          } else {
            c.g_ctr[g] = 0;
          }
          cnt[8] += (int64_t)(c.g_off[g + 1] - c.g_off[g]) * sum_slots;
          cnt[9] += Gc;
        }
        if (P.decisions) P.decisions[((size_t)r * P.E + e) * N + g] = dec_out;
      }
      __syncthreads();
      if (tid == 0) {
        if (P.policy == 0) {
          int alive = 0, open = 0;
#pragma unroll 1
          for (int g = 0; g < N; ++g) {
            alive += has_vm(c, g, Tend) ? 1 : 0;
            open += c.g_re[g] > Tend ? 1 : 0;
          }
          int cap = P.cap_pct * alive / 100;
          if (cap < 1) cap = 1;
          int free_slots = cap - open;
          while (free_slots > 0) {  // wants by (delta misses desc, gpu asc)
            int pick = -1;
            int64_t pd = 0;
#pragma unroll 1
            for (int g = 0; g < N; ++g) {
              if (!c.g_want[g]) continue;
              const int64_t d = (c.g_kcur[g] >> 40) - (c.g_kbest[g] >> 40);
              if (pick < 0 || d > pd) { pick = g; pd = d; }
            }
            if (pick < 0) break;
            c.g_want[pick] = 0;
            const int64_t drain_end = c.g_maxend[pick] > Tend ? c.g_maxend[pick] : Tend;
            c.g_rs[pick] = Tend;
            c.g_re[pick] = drain_end + P.reconfig_us;
            c.g_target[pick] = c.g_best[pick];
            cnt[7] += 1;
            --free_slots;
          }
        }
        cs.nlog += nb;
      }
      __syncthreads();
    }

    // ---------------------------------------------------------------- finalize (O12)
#pragma unroll 1
    for (int g = tid; g < N; g += NT) bill_switch(c, g, VM_NONE, P.H, P.H);
#pragma unroll
    for (int i = 0; i < 10; ++i)
      if (cnt[i]) atomicAdd(&cs.cnt[i], (unsigned long long)cnt[i]);
#pragma unroll 1
    for (int w = tid; w < kNB; w += NT) {  // fold the packed smem halves into the HBM histogram
      const uint32_t v = c.hist[w];
      if (v & 0xFFFFu) atomicAdd(&ghist[2 * w], v & 0xFFFFu);
      if (v >> 16) atomicAdd(&ghist[2 * w + 1], v >> 16);
    }
    __syncthreads();
    if (warp < 2) {  // nearest-rank P50 / P99 per class
      const uint32_t* h = ghist + warp * kNB;
      uint64_t n = 0;
#pragma unroll 1
      for (int b = lane; b < kNB; b += 32) n += h[b];
#pragma unroll
      for (int d = 16; d > 0; d >>= 1) n += __shfl_xor_sync(0xffffffffu, n, d);
      int64_t p50 = 0, p99 = 0;
      if (n) {
        const uint64_t r50 = (50 * n + 99) / 100, r99 = (99 * n + 99) / 100;
        uint64_t cum = 0;
        int f50 = -1, f99 = -1;
#pragma unroll 1
        for (int b0 = 0; b0 < kNB && f99 < 0; b0 += 32) {
          uint64_t x = h[b0 + lane];
#pragma unroll
          for (int d = 1; d < 32; d <<= 1) {
            const uint64_t y = __shfl_up_sync(0xffffffffu, x, d);
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
        od += c.g_od[g];
        spot += c.g_spot[g];
        busy += c.g_busy[g];
        memt += c.g_mem[g];
      }
      for (int i = 0; i < 10; ++i) P.counters[(size_t)r * 10 + i] = (int64_t)cs.cnt[i];
      P.accum[(size_t)r * 4 + 0] = busy;
      P.accum[(size_t)r * 4 + 1] = memt;
      P.accum[(size_t)r * 4 + 2] = od;
      P.accum[(size_t)r * 4 + 3] = spot;
      P.cost[r] = __ddiv_rn(__dadd_rn(__dmul_rn((double)od, P.price_od),
                                      __dmul_rn((double)spot, P.price_spot)), 3.6e9);
      const double dN = (double)N, dH = (double)P.H;
      P.util[2 * (size_t)r] = __ddiv_rn((double)busy, __dmul_rn(__dmul_rn(7.0, dN), dH));
      P.util[2 * (size_t)r + 1] = __ddiv_rn((double)memt, __dmul_rn(__dmul_rn(40960.0, dN), dH));
      if (P.n_batches) P.n_batches[r] = cs.nlog;
    }
    __syncthreads();
  }
}

// Prepass: eoff[r][e] = first request of replica r with arrival >= e*W (e = 0..E), and the
// largest request window any epoch needs: [lower_bound(eW - maxT), eoff[e+1]).
__global__ void prepass_kernel(const uint32_t* arr, const int64_t* roff, int R, int64_t E,
                               int64_t W, int64_t maxT, int64_t* eoff, unsigned long long* wmax,
                               int* err) {
  const int64_t idx = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
  if (idx >= (int64_t)R * (E + 1)) return;
  const int r = (int)(idx / (E + 1));
  const int64_t e = idx - (int64_t)r * (E + 1);
  const int64_t lo0 = roff[r], hi0 = roff[r + 1];
  auto lower = [&](int64_t v) {
    int64_t lo = lo0, hi = hi0;
    while (lo < hi) {
      const int64_t mid = (lo + hi) >> 1;
      if ((int64_t)arr[mid] >= v) hi = mid; else lo = mid + 1;
    }
    return lo;
  };
  const int64_t here = lower(e * W);
  eoff[idx] = here;
  if (e < E) {
    const int64_t a = e * W - maxT;
    const int64_t next = lower((e + 1) * W);
    if (next < here) atomicOr(err, 1);  // arrivals not sorted
    const int64_t w = next - lower(a < 0 ? 0 : a);
    if (w > 0) atomicMax(wmax, (unsigned long long)w);
  } else if (here != hi0) {
    atomicOr(err, 1);                   // an arrival at or beyond E*W >= trace_len
  }
}

cudaError_t launch_prepass(const uint32_t* arr, const int64_t* roff, int R, int64_t E, int64_t W,
                           int64_t maxT, int64_t* eoff, unsigned long long* wmax, int* err,
                           cudaStream_t st) {
  const int64_t total = (int64_t)R * (E + 1);
  const int bs = 256;
  prepass_kernel<<<(unsigned)((total + bs - 1) / bs), bs, 0, st>>>(arr, roff, R, E, W, maxT, eoff, wmax, err);
  return cudaGetLastError();
}

cudaError_t launch_replay(const ReplayParams& P, int grid, int block, cudaStream_t st) {
  cudaError_t e = cudaFuncSetAttribute(replay_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize,
                                       (int)P.sl.total);
  if (e != cudaSuccess) return e;
  replay_kernel<<<grid, block, P.sl.total, st>>>(P);
  return cudaGetLastError();
}

cudaError_t replay_occupancy(int block, size_t smem, int* blocks_per_sm) {
  cudaError_t e = cudaFuncSetAttribute(replay_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize,
                                       (int)smem);
  if (e != cudaSuccess) return e;
  return cudaOccupancyMaxActiveBlocksPerMultiprocessor(blocks_per_sm, replay_kernel, block, smem);
}

}  // namespace pemgpu
