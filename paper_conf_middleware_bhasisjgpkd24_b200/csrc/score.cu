// score.cu — protean_score_epoch: one epoch of the search on caller-supplied dispatched batches
// and caller-owned GPU states.  One CTA per replica; lanes =
// (sim-GPU, actual | candidate geometry) exactly as in the fused replay engine.
#include <cuda_runtime.h>
#include "replay.cuh"
#include "place_group.cuh"

namespace pemgpu {

using namespace pg;


// One CTA per replica, 8 warps; placement units are the fused engine's lane groups (lane = MIG
// slice position, place_group.cuh): one warp per sim-GPU for the actual placement on the carried
// state (its 8 lanes hold the slices' resident lists, built from and written back to the caller's
// protean_gpu_state), and the candidate warps of the geometry range's lane packing, each group
// replaying the GPU-epoch's batches from idle (Q19).  Validation runs first; an invalid replica
// writes nothing.
__global__ void __launch_bounds__(256) score_kernel(ScoreParams P) {
  extern __shared__ __align__(16) unsigned char smem[];
  __shared__ int bad;
  __shared__ int s_task;
  __shared__ unsigned long long s_cn[10], s_busy, s_mem;
  const int tid = threadIdx.x, NT = blockDim.x, lane = tid & 31, warp = tid >> 5, NW = NT >> 5;
  const int r = blockIdx.x, N = P.N, Gc = P.geom_hi - P.geom_lo;
  int32_t* tabw = reinterpret_cast<int32_t*>(smem);
  for (int i = tid; i < P.tl.words; i += NT) tabw[i] = P.tab[i];
  int64_t* keys = reinterpret_cast<int64_t*>(smem + (((size_t)P.tl.words * 4 + 15) & ~(size_t)15));
  uint8_t* dec = reinterpret_cast<uint8_t*>(keys + (size_t)N * Gc);
  Tab T;
  T.bind(tabw, P.tl);
  if (tid == 0) {
    bad = 0;
    s_task = 0;
    s_busy = s_mem = 0;
  }
  if (tid < 10) s_cn[tid] = 0;
  __syncthreads();
  const int64_t eW = (int64_t)P.epoch * P.W, Tend = eW + P.W;

  for (int g = tid; g < N; g += NT) {  // validate, install pending reconfiguration (O5.3)
    const int x = r * N + g;
    protean_gpu_state& st = P.state[x];
    bool inval = st.geom >= T.G || (st.target != 0xFF && st.target >= T.G) ||
                 P.batch_off[x + 1] < P.batch_off[x] || P.batch_off[0] != 0 || st.vm_type > 2;
    const bool range = st.n_live > P.max_live;
    if (!inval && !range) {
      for (int i = 0; i < st.n_live; ++i)
        if (st.live[i].slice >= T.gn[st.geom] || st.live[i].model >= T.M) inval = true;
      for (int b = P.batch_off[x]; b < P.batch_off[x + 1] && !inval; ++b) {
        const protean_batch& bt = P.batches[b];
        if (bt.model >= T.M || bt.n_req < 1 || (int64_t)bt.ready_us < eW ||
            (int64_t)bt.ready_us >= Tend || bt.strict > 1)
          inval = true;
        if (b > P.batch_off[x] && bt.ready_us < P.batches[b - 1].ready_us) inval = true;
        for (int i = 0; i < bt.n_req && !inval; ++i) {
          const uint32_t a = P.arrival[bt.req_off + i];
          if (a > bt.ready_us || (i > 0 && a < P.arrival[bt.req_off + i - 1])) inval = true;
        }
      }
    }
    if (inval) { atomicOr(&P.err[0], 1); bad = 1; }
    if (range) { atomicOr(&P.err[1], 1); bad = 1; }
  }
  __syncthreads();
  if (bad) return;
  for (int g = tid; g < N; g += NT) {
    protean_gpu_state& st = P.state[r * N + g];
    if (st.target != 0xFF && st.recfg_end_us <= Tend) {
      st.geom = st.target;
      st.target = 0xFF;
      st.wait_ctr = 0;
      st.n_live = 0;
      for (int s = 0; s < kMaxSl; ++s) st.last_start_us[s] = st.busy_until_us[s] = st.busy_us[s] = 0;
    }
    dec[g] = (st.has_vm && st.recfg_end_us <= Tend) ? 1 : 0;
    if (P.cost) {  // node-epoch VM cost: price(vm_type) * W / 3.6e9 (T3 P:L173-179, Q35)
      const double price = !st.has_vm ? 0.0 : st.vm_type == 1 ? P.price_od : st.vm_type == 2 ? P.price_spot : 0.0;
      P.cost[r * N + g] = __ddiv_rn(__dmul_rn(price, (double)P.W), 3.6e9);
    }
  }
  __syncthreads();

  // lane lists in this CTA's scratch slot: actual [N * 8 lanes][max_live], candidate [NW * 32][max_live]
  const int NA = N * 8, NCL = NW * 32, ML = P.max_live;
  char* slot = reinterpret_cast<char*>(P.lists) + (size_t)r * P.list_bytes;
  LaneList AL;
  AL.stride = NA;
  AL.st = reinterpret_cast<int64_t*>(slot);
  AL.en = AL.st + (size_t)NA * ML;
  AL.mm = reinterpret_cast<uint32_t*>(AL.en + (size_t)NA * ML);
  LaneList CLb;
  CLb.stride = NCL;
  CLb.st = reinterpret_cast<int64_t*>(slot + (size_t)NA * ML * 20);
  CLb.en = CLb.st + (size_t)NCL * ML;
  CLb.mm = reinterpret_cast<uint32_t*>(CLb.en + (size_t)NCL * ML);

  const int n_units = N + N * P.cw;  // actual: one warp per GPU; candidates: cw warps per GPU
  unsigned long long cn[10] = {0, 0, 0, 0, 0, 0, 0, 0, 0, 0};
  unsigned long long busy = 0, memt = 0;
  for (;;) {
    int u = 0;
    if (lane == 0) u = atomicAdd(&s_task, 1);
    u = __shfl_sync(0xffffffffu, u, 0);
    if (u >= n_units) break;
    const bool actual = u < N;
    int g, s, Z, gbase, j;
    bool valid;
    if (actual) {
      g = u;
      s = lane & 7;
      Z = 8;
      gbase = lane & ~7;
      valid = lane < 8;
      j = P.state[r * N + g].geom;
    } else {
      const int cu = u - N, w = cu % P.cw;
      g = cu / P.cw;
      const uint32_t pk = P.pack[w * 32 + lane];
      const int jr = pk & 0xFF;
      s = (pk >> 8) & 0xFF;
      Z = (pk >> 16) & 0xFF;
      gbase = pk >> 24;
      valid = jr != 0xFF;
      j = valid ? jr : 0;
      if (!dec[g]) {  // undecidable at T: no candidates scored (O5.4)
        if (valid && lane == gbase) {
          keys[g * Gc + (j - P.geom_lo)] = -1;
          if (P.cand_key) P.cand_key[(size_t)(r * N + g) * Gc + (j - P.geom_lo)] = -1;
        }
        continue;
      }
    }
    const int x = r * N + g;
    protean_gpu_state& st = P.state[x];
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
    LaneList L;
    int n = 0;
    int64_t ls = 0, bu = 0, bsl = 0;
    if (actual) {
      L = AL;
      const int al = g * 8 + s;
      L.st += al; L.en += al; L.mm += al;
      if (active) {  // this slice's residents, in the state's order
        for (int i = 0; i < st.n_live; ++i) {
          const protean_resident& rr = st.live[i];
          if (rr.slice != s) continue;
          L.put(n++, rr.start_us, rr.end_us,
                (uint32_t)rr.mem_mib | ((uint32_t)rr.model << 24) | ((uint32_t)(rr.strict ? 1 : 0) << 30));
        }
        ls = st.last_start_us[s];
        bu = st.busy_until_us[s];
        bsl = st.busy_us[s];
      }
    } else {
      L = CLb;
      L.st += warp * 32 + lane; L.en += warp * 32 + lane; L.mm += warp * 32 + lane;
    }
    __syncwarp();
    const int b0 = P.batch_off[x], b1 = P.batch_off[x + 1];
    int64_t misses = 0, tail = 0;
    for (int b = b0; b < b1; ++b) {
      const protean_batch& bt = P.batches[b];
      const int m = bt.model, nreq = bt.n_req;
      const bool strict = bt.strict != 0;
      int64_t stt, enn;
      const SliceOut so = place_group<1>(T, active, K, L, n, ls, (int64_t)bt.ready_us, m, strict, P.max_live,
                                         &stt, &enn);
      const bool placed = !so.drop_overflow && so.kmin != ~0ull;
      const int wl = (gbase + (int)(so.kmin & 7)) & 31;
      const int64_t cwin = __shfl_sync(0xffffffffu, enn, wl);
      if (actual) {
        if (placed && lane == wl) {  // winner: placement row, busy union + memory-time clipped to [0, H)
          protean_placement pl;
          pl.start_us = stt;
          pl.end_us = enn;
          pl.slice = (uint8_t)s;
          pl.dropped = 0;
          for (int i = 0; i < 6; ++i) pl.pad[i] = 0;
          P.placement[b] = pl;
          const int64_t lo = stt > bu ? stt : bu;
          const int64_t hi = enn < P.H ? enn : P.H;
          if (hi > lo) {
            busy += (unsigned long long)((int64_t)prof_compute(p) * (hi - lo));
            bsl += hi - lo;
          }
          if (enn > bu) bu = enn;
          if (hi > stt) memt += (unsigned long long)((int64_t)T.mem[m] * (hi - stt));
        }
        if (lane == 0) {
          if (!placed) {
            protean_placement pl;
            pl.start_us = pl.end_us = 0;
            pl.slice = 0xFF;
            pl.dropped = so.drop_overflow ? 3 : 2;
            for (int i = 0; i < 6; ++i) pl.pad[i] = 0;
            P.placement[b] = pl;
          }
          if (strict) cn[0] += nreq; else cn[4] += nreq;
          if (!placed) {
            if (strict) cn[3] += nreq; else cn[6] += nreq;
          } else if (strict) {
            const int hh = hits_sorted(P.arrival + bt.req_off, nreq, cwin, T.slo[m]);
            cn[1] += hh;
            cn[2] += nreq - hh;
          } else {
            cn[5] += nreq;
          }
        }
      } else if (valid && lane == gbase) {  // group leader keeps the candidate's score (O8)
        if (strict) {
          misses += placed ? nreq - hits_sorted(P.arrival + bt.req_off, nreq, cwin, T.slo[m]) : nreq;
        } else {
          const int64_t tb = placed ? cwin - (int64_t)P.arrival[bt.req_off] : (int64_t)0xFFFFFFFFLL;
          tail = tb > tail ? tb : tail;
        }
      }
    }
    if (actual) {  // write the slices' lists back to the caller's state (slice order)
      int off = active ? n : 0;
#pragma unroll
      for (int d = 1; d < 8; d <<= 1) {
        const int y = __shfl_up_sync(0xffffffffu, off, d);
        if ((lane & 7) >= d) off += y;
      }
      const int base = off - (active ? n : 0);
      if (active) {
        for (int i = 0; i < n; ++i) {
          protean_resident rr;
          rr.start_us = L.S(i);
          rr.end_us = L.E(i);
          const uint32_t mm = L.M(i);
          rr.mem_mib = (int32_t)(mm & kMemMask);
          rr.slice = (uint8_t)s;
          rr.model = (uint8_t)((mm >> 24) & 63);
          rr.strict = (uint8_t)((mm >> 30) & 1);
          rr.pad = 0;
          st.live[base + i] = rr;
        }
        st.last_start_us[s] = ls;
        st.busy_until_us[s] = bu;
        st.busy_us[s] = bsl;
      }
      const int tot = __shfl_sync(0xffffffffu, off, 7);
      if (lane == 0) st.n_live = (uint8_t)tot;
    } else if (valid && lane == gbase) {
      const int64_t key = make_key(misses, tail, j == st.geom ? 0 : j + 1);
      keys[g * Gc + (j - P.geom_lo)] = key;
      if (P.cand_key) P.cand_key[(size_t)x * Gc + (j - P.geom_lo)] = key;
      cn[8] += (unsigned long long)(b1 - b0) * T.gn[j];
      cn[9] += 1;
    }
    __syncwarp();
  }
  for (int i = 0; i < 10; ++i)
    if (cn[i]) atomicAdd(&s_cn[i], cn[i]);
  if (busy) atomicAdd(&s_busy, busy);
  if (memt) atomicAdd(&s_mem, memt);
  __syncthreads();
  if (tid < 10 && s_cn[tid])
    atomicAdd(reinterpret_cast<unsigned long long*>(&P.counters[(size_t)r * 10 + tid]), s_cn[tid]);
  if (P.accum && tid == 0) {
    if (s_busy) atomicAdd(reinterpret_cast<unsigned long long*>(&P.accum[(size_t)r * 4]), s_busy);
    if (s_mem) atomicAdd(reinterpret_cast<unsigned long long*>(&P.accum[(size_t)r * 4 + 1]), s_mem);
  }
  for (int g = tid; g < N; g += NT) {  // S8: min over the range (warp-free: <= 254 keys per GPU)
    int64_t kb = -1;
    if (dec[g]) {
      kb = keys[g * Gc];
      for (int v = 1; v < Gc; ++v) kb = keys[g * Gc + v] < kb ? keys[g * Gc + v] : kb;
    }
    P.best_key[r * N + g] = kb;
  }
}

// N4b: the BE-reserve depth as an enumerated dimension (reading R28).  A lane is (replica r, gpu
// g, geometry j, depth code c): code 0 replays the GPU-epoch's batches from idle with Alg 1's tag
// walk, code 1 + d with "the d smallest slices reserved for BE" (strict eligible on positions >= d,
// fallback to every fitting slice), both through place_lane (O6) and scored by the O8 key.  Grid-
// stride lanes; each thread's resident list is its own scratch slot.
__global__ void __launch_bounds__(128) depth_kernel(DepthParams P) {
  extern __shared__ int32_t tabw[];
  const int tid = threadIdx.x;
  if (*(volatile int*)P.err) return;  // the validation kernel (same stream) rejected the input
  for (int i = tid; i < P.tl.words; i += blockDim.x) tabw[i] = P.tab[i];
  __syncthreads();
  Tab T;
  T.bind(tabw, P.tl);
  const int nc = P.geom_hi - P.geom_lo;
  const int64_t lanes = (int64_t)P.R * P.N * nc * 8;
  const int64_t slot = (int64_t)blockIdx.x * blockDim.x + tid;
  Rows rows{P.scratch + slot * P.max_live};
  for (int64_t L = slot; L < lanes; L += (int64_t)gridDim.x * blockDim.x) {
    const int code = (int)(L & 7);
    const int64_t xj = L >> 3;
    const int jj = (int)(xj % nc);
    const int64_t x = xj / nc;
    const int j = P.geom_lo + jj;
    int64_t key = -1;
    if (code <= T.gn[j]) {
      const int b0 = P.batch_off[x], b1 = P.batch_off[x + 1];
      int n = 0;
      int64_t ls[kMaxSl];
#pragma unroll
      for (int s = 0; s < kMaxSl; ++s) ls[s] = 0;
      int64_t misses = 0, tail = 0;
      for (int b = b0; b < b1; ++b) {
        const protean_batch& bt = P.batches[b];
        const PlaceRes pr = place_lane(T, j, rows, n, ls, bt.ready_us, bt.model, bt.strict != 0, P.max_live,
                                       code - 1);
        if (bt.strict) {
          misses += pr.dropped ? bt.n_req
                               : bt.n_req - hits_sorted(P.arrival + bt.req_off, bt.n_req, pr.end, T.slo[bt.model]);
        } else {
          const int64_t tb = pr.dropped ? (int64_t)0xFFFFFFFFLL : pr.end - (int64_t)P.arrival[bt.req_off];
          tail = tb > tail ? tb : tail;
        }
      }
      key = make_key(misses, tail, P.cur_geom[x] == j ? 0 : j + 1);
    }
    P.depth_key[L] = key;
  }
}

// Per (replica, gpu): the best code of every geometry (lowest code among equal keys) and the min key
__global__ void depth_reduce_kernel(DepthParams P) {
  const int64_t x = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
  const int nc = P.geom_hi - P.geom_lo;
  if (*(volatile int*)P.err) return;
  if (x == 0) *P.n_eval += P.n_eval_add;
  if (x >= (int64_t)P.R * P.N) return;
  int64_t best = -1;
  for (int jj = 0; jj < nc; ++jj) {
    const int64_t* k = P.depth_key + (x * nc + jj) * 8;
    int bc = 0;
    for (int c = 1; c < 8; ++c)
      if (k[c] >= 0 && k[c] < k[bc]) bc = c;
    if (P.depth_code) P.depth_code[x * nc + jj] = (uint8_t)bc;
    if (best < 0 || k[bc] < best) best = k[bc];
  }
  P.best_key[x] = best;
}

// Input validation, one thread per (replica, gpu): the sweep's rules (include/protean.h 3b).
__global__ void depth_validate_kernel(DepthParams P) {
  const int64_t x = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
  if (x >= (int64_t)P.R * P.N) return;
  const int G = P.tl.G, M = P.tl.M;
  bool bad = P.batch_off[x + 1] < P.batch_off[x] || P.batch_off[0] != 0 ||
             (P.cur_geom[x] != 0xFF && P.cur_geom[x] >= G);
  for (int b = P.batch_off[x]; b < P.batch_off[x + 1] && !bad; ++b) {
    const protean_batch& bt = P.batches[b];
    if (bt.model >= M || bt.n_req < 1 || bt.strict > 1) bad = true;
    if (b > P.batch_off[x] && bt.ready_us < P.batches[b - 1].ready_us) bad = true;
    for (int i = 0; i < bt.n_req && !bad; ++i) {
      const uint32_t a = P.arrival[bt.req_off + i];
      if (a > bt.ready_us || (i > 0 && a < P.arrival[bt.req_off + i - 1])) bad = true;
    }
  }
  if (bad) atomicOr(&P.err[0], 1);
}

cudaError_t launch_depths(const DepthParams& P, int grid, int block, cudaStream_t st) {
  const int64_t X0 = (int64_t)P.R * P.N;
  depth_validate_kernel<<<(unsigned)((X0 + 127) / 128), 128, 0, st>>>(P);
  depth_kernel<<<grid, block, (size_t)P.tl.words * 4, st>>>(P);
  cudaError_t e = cudaGetLastError();
  if (e != cudaSuccess) return e;
  const int64_t X = (int64_t)P.R * P.N;
  depth_reduce_kernel<<<(unsigned)((X + 127) / 128), 128, 0, st>>>(P);
  return cudaGetLastError();
}

size_t score_smem_bytes(const TabLayout& tl, int N, int Gc) {
  return (((size_t)tl.words * 4 + 15) & ~(size_t)15) + (size_t)N * Gc * 8 + (((size_t)N + 15) & ~(size_t)15);
}

// per-CTA lane lists (SoA start, end, packed word = 20 B per row): N * 8 actual lanes + the block's lanes
size_t score_list_bytes(int N, int block, int max_live) {
  return (((size_t)N * 8 + (size_t)block) * (size_t)max_live * 20 + 255) & ~(size_t)255;
}

cudaError_t launch_score(const ScoreParams& P, int block, cudaStream_t st) {
  const size_t sm = score_smem_bytes(P.tl, P.N, P.geom_hi - P.geom_lo);
  cudaError_t e = cudaSuccess;
  if (sm > 48 * 1024) e = cudaFuncSetAttribute(score_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)sm);
  if (e != cudaSuccess) return e;
  score_kernel<<<P.R, block, sm, st>>>(P);
  return cudaGetLastError();
}

}  // namespace pemgpu
