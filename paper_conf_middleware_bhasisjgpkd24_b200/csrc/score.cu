// score.cu — protean_score_epoch: one epoch of the search on caller-supplied dispatched batches
// and caller-owned GPU states.  One CTA per replica; lanes =
// (sim-GPU, actual | candidate geometry) exactly as in the fused replay engine.
#include <cuda_runtime.h>
#include "replay.cuh"

namespace pemgpu {


__global__ void __launch_bounds__(256) score_kernel(ScoreParams P) {
  extern __shared__ __align__(16) unsigned char smem[];
  __shared__ int bad;
  const int tid = threadIdx.x, NT = blockDim.x;
  const int r = blockIdx.x, N = P.N, Gc = P.geom_hi - P.geom_lo;
  int32_t* tabw = reinterpret_cast<int32_t*>(smem);
  for (int i = tid; i < P.tl.words; i += NT) tabw[i] = P.tab[i];
  int64_t* keys = reinterpret_cast<int64_t*>(smem + (((size_t)P.tl.words * 4 + 15) & ~(size_t)15));
  uint8_t* dec = reinterpret_cast<uint8_t*>(keys + (size_t)N * Gc);
  // every lane's resident list in shared memory when it fits (P.smem_lists), else global scratch
  protean_resident* slists = reinterpret_cast<protean_resident*>(
      reinterpret_cast<unsigned char*>(dec) + (((size_t)N + 15) & ~(size_t)15));
  Tab T;
  T.bind(tabw, P.tl);
  if (tid == 0) bad = 0;
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

  const int nl = N * (1 + Gc);
  unsigned long long cn[10] = {0, 0, 0, 0, 0, 0, 0, 0, 0, 0};
  unsigned long long busy = 0, memt = 0;
  for (int L = tid; L < nl; L += NT) {
    const int g = L / (1 + Gc), v = L - g * (1 + Gc);
    const int x = r * N + g;
    protean_gpu_state& st = P.state[x];
    const int b0 = P.batch_off[x], b1 = P.batch_off[x + 1];
    if (v == 0) {
      Rows rows{P.smem_lists ? slists + (size_t)L * P.max_live : st.live};
      const int geom = st.geom;
      int n = st.n_live;
      if (P.smem_lists)
        for (int i = 0; i < n; ++i) rows.r[i] = st.live[i];
      int64_t ls[kMaxSl], bu[kMaxSl], bs[kMaxSl];
#pragma unroll
      for (int s = 0; s < kMaxSl; ++s) {
        ls[s] = st.last_start_us[s];
        bu[s] = st.busy_until_us[s];
        bs[s] = st.busy_us[s];
      }
      for (int b = b0; b < b1; ++b) {
        const protean_batch& bt = P.batches[b];
        const PlaceRes pr = place_lane(T, geom, rows, n, ls, bt.ready_us, bt.model, bt.strict != 0,
                                       P.max_live);
        protean_placement pl;
        pl.start_us = pr.dropped ? 0 : pr.start;
        pl.end_us = pr.dropped ? 0 : pr.end;
        pl.slice = pr.dropped ? 0xFF : (uint8_t)pr.slice;
        pl.dropped = (uint8_t)pr.dropped;
        for (int i = 0; i < 6; ++i) pl.pad[i] = 0;
        P.placement[b] = pl;
        if (bt.strict) cn[0] += bt.n_req; else cn[4] += bt.n_req;
        if (pr.dropped) {
          if (bt.strict) cn[3] += bt.n_req; else cn[6] += bt.n_req;
          continue;
        }
        if (bt.strict) {
          const int h = hits_sorted(P.arrival + bt.req_off, bt.n_req, pr.end, T.slo[bt.model]);
          cn[1] += h;
          cn[2] += bt.n_req - h;
        } else {
          cn[5] += bt.n_req;
        }
        const int p = T.gprof[geom * 8 + pr.slice];
#pragma unroll
        for (int s = 0; s < kMaxSl; ++s) {
          if (s == pr.slice) {
            const int64_t lo = pr.start > bu[s] ? pr.start : bu[s];
            const int64_t hi = pr.end < P.H ? pr.end : P.H;
            if (hi > lo) {
              busy += (unsigned long long)((int64_t)prof_compute(p) * (hi - lo));
              bs[s] += hi - lo;
            }
            if (pr.end > bu[s]) bu[s] = pr.end;
          }
        }
        const int64_t mhi = pr.end < P.H ? pr.end : P.H;
        if (mhi > pr.start) memt += (unsigned long long)((int64_t)T.mem[bt.model] * (mhi - pr.start));
      }
      st.n_live = (uint8_t)n;
      if (P.smem_lists)
        for (int i = 0; i < n; ++i) st.live[i] = rows.r[i];
#pragma unroll
      for (int s = 0; s < kMaxSl; ++s) {
        st.last_start_us[s] = ls[s];
        st.busy_until_us[s] = bu[s];
        st.busy_us[s] = bs[s];
      }
    } else {
      const int j = P.geom_lo + v - 1;
      int64_t key = -1;
      if (dec[g]) {
        Rows rows{P.smem_lists ? slists + (size_t)L * P.max_live
                               : P.scratch + ((size_t)r * N * Gc + (size_t)g * Gc + (v - 1)) * P.max_live};
        int n = 0;
        int64_t ls[kMaxSl];
#pragma unroll
        for (int s = 0; s < kMaxSl; ++s) ls[s] = 0;
        int64_t misses = 0, tail = 0;
        for (int b = b0; b < b1; ++b) {
          const protean_batch& bt = P.batches[b];
          const PlaceRes pr = place_lane(T, j, rows, n, ls, bt.ready_us, bt.model, bt.strict != 0,
                                         P.max_live);
          if (bt.strict) {
            misses += pr.dropped ? bt.n_req
                                 : bt.n_req - hits_sorted(P.arrival + bt.req_off, bt.n_req, pr.end,
                                                          T.slo[bt.model]);
          } else {
            const int64_t tb = pr.dropped ? (int64_t)0xFFFFFFFFLL : pr.end - (int64_t)P.arrival[bt.req_off];
            tail = tb > tail ? tb : tail;
          }
        }
        key = make_key(misses, tail, j == st.geom ? 0 : j + 1);
        cn[8] += (unsigned long long)(b1 - b0) * T.gn[j];
        cn[9] += 1;
      }
      keys[g * Gc + v - 1] = key;
      if (P.cand_key) P.cand_key[(size_t)x * Gc + (v - 1)] = key;
    }
  }
  for (int i = 0; i < 10; ++i)
    if (cn[i]) atomicAdd(reinterpret_cast<unsigned long long*>(&P.counters[(size_t)r * 10 + i]), cn[i]);
  if (P.accum) {
    if (busy) atomicAdd(reinterpret_cast<unsigned long long*>(&P.accum[(size_t)r * 4]), busy);
    if (memt) atomicAdd(reinterpret_cast<unsigned long long*>(&P.accum[(size_t)r * 4 + 1]), memt);
  }
  __syncthreads();
  for (int g = tid; g < N; g += NT) {
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

// the lanes' resident lists in shared memory: N * (1 + Gc) lanes x max_live rows of 24 B
size_t score_list_bytes(int N, int Gc, int max_live) {
  return (size_t)N * (1 + Gc) * (size_t)max_live * sizeof(protean_resident);
}

cudaError_t launch_score(const ScoreParams& P, int block, cudaStream_t st) {
  const size_t sm = score_smem_bytes(P.tl, P.N, P.geom_hi - P.geom_lo) +
                    (P.smem_lists ? score_list_bytes(P.N, P.geom_hi - P.geom_lo, P.max_live) : 0);
  cudaError_t e = cudaFuncSetAttribute(score_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)sm);
  if (e != cudaSuccess) return e;
  score_kernel<<<P.R, block, sm, st>>>(P);
  return cudaGetLastError();
}

}  // namespace pemgpu
