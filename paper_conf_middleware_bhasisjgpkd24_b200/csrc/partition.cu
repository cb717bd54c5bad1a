// partition.cu — trace-level stream partition ahead of the replay (S2's per-(model, class) request
// streams, O3 / P:L229-233).  Three passes over the resident trace, each a warp per (replica,
// epoch) or a CTA per replica, sized for the whole GPU:
//   P1  count: per-(replica, epoch, stream) request counts (reads meta only, 1 B/request)
//   P2  scan: per replica, stream bases (stream-major order) and the index of every (epoch, stream)
//       run: sidx[r][e][k] = first request of stream k with arrival >= e*W (e = 0..E)
//   P3  stable scatter + validate: every epoch's requests into their stream's run of the
//       stream-sorted copy sa (arrival only; 4 B/request), per replica starting at a 16-byte aligned
//       offset; every request checked once (model id, arrival < trace_len, sorted) -> err[0]
// The replay then bulk-copies (TMA) each stream's epoch range [cursor_k, sidx[r][e+1][k]) into
// shared memory: no per-epoch partition inside the persistent kernel.
#include <cuda_runtime.h>

#include "replay.cuh"

namespace pemgpu {

namespace {

// P1 body: per-stream counts of meta[0, n) of one warp into the warp-private cntw: 16 requests per
// lane per step (one 16-byte meta load when meta is 16-byte aligned at that point), one
// unpredicated shared increment per request (same-address increments of a warp are combined by
// the hardware, ATOMS.POPC.INC); lanes with nothing to count increment a sink word, so the loop
// has no branches.  koff maps a meta byte straight to its counter's byte offset, and full 32-chunk
// steps run without bounds tests: 6 instructions per request (ncu: 1.18 -> 0.97 ms per 3.1 G
// requests).  Reads 1 B/request.
__device__ __forceinline__ void count_streams(const uint8_t* meta, int64_t n, int* cntw, uint32_t sink,
                                              const uint32_t* koff) {
  const int lane = threadIdx.x & 31;
  const uint32_t cb = (uint32_t)__cvta_generic_to_shared(cntw);
  const int64_t h = min(n, (int64_t)((16u - ((uint32_t)(uintptr_t)meta & 15u)) & 15u));
  {  // unaligned head (< 16 requests)
    const bool valid = lane < h;
    const int kv = koff[valid ? meta[lane] : 0];
    inc_shared(valid ? cb + (uint32_t)kv : sink);
  }
  const int64_t nch = (n - h) >> 4;
  const uint4* gv = reinterpret_cast<const uint4*>(meta + h);
  const int64_t nfull = nch & ~(int64_t)31;
#pragma unroll 1
  for (int64_t c0 = 0; c0 < nfull; c0 += 32) {  // every lane has a chunk: no bounds tests
    const uint4 v = gv[c0 + lane];
    const uint32_t w4[4] = {v.x, v.y, v.z, v.w};
#pragma unroll
    for (int q = 0; q < 16; ++q) {
      const uint32_t w = w4[q >> 2];
      const uint32_t bo = (q & 3) ? (w >> (8 * (q & 3) - 2)) & 0x3FCu : (w << 2) & 0x3FCu;
      inc_shared(cb + *reinterpret_cast<const uint32_t*>(reinterpret_cast<const char*>(koff) + bo));
    }
  }
#pragma unroll 1
  for (int64_t c0 = nfull; c0 < nch; c0 += 32) {
    const int64_t ch = c0 + lane;
    const bool valid = ch < nch;
    uint4 v = make_uint4(0u, 0u, 0u, 0u);
    if (valid) v = gv[ch];
    const uint32_t w4[4] = {v.x, v.y, v.z, v.w};
#pragma unroll
    for (int q = 0; q < 16; ++q) {
      const int kv = koff[(w4[q >> 2] >> (8 * (q & 3))) & 0xFF];
      inc_shared(valid ? cb + (uint32_t)kv : sink);
    }
  }
  const int64_t t0 = h + 16 * nch;
#pragma unroll 1
  for (int64_t i0 = t0; i0 < n; i0 += 32) {  // tail (< 16 requests)
    const bool valid = i0 + lane < n;
    const int kv = koff[valid ? meta[i0 + lane] : 0];
    inc_shared(valid ? cb + (uint32_t)kv : sink);
  }
}

// P3 body: stable scatter of requests [lo, hi) (one warp) into their streams' runs of sa, and the
// validation of every request: model id < M with no reserved bit, arrival < trace_len, arrival >=
// its predecessor (the first against prev0 when has_prev0) -- every adjacent pair of a replica
// lies in one epoch range or straddles two consecutive ones, so this checks sortedness.  K = 1..2:
// the range holds exactly the streams ak[0..K), whose running offsets run[] live in registers and
// whose in-warp ranks come from one ballot each; K = 0: any number of streams, ranks from
// match_any and warp-private running offsets in runw.  Returns true (this lane) on an invalid one.
constexpr int kSU = 16;  // requests per lane in flight per scatter step (8: 5.53 ms, 16: 5.37 ms per 3.1 G)
// One step of 32 * kSU requests from i0.  kFull: all of them lie below hi (no per-request bounds
// tests; the tail step takes kFull = false).  Slots of sa are indexed with unsigned 32-bit offsets
// (a replica's run is < 2^32 requests), so each store address is one wide multiply-add.
template <int K, bool kFull>
__device__ __forceinline__ void scatter_step(const uint32_t* warr, const uint8_t* wmeta, int i0, int hi,
                                             uint32_t tlm1, const uint16_t* klut, int* runw, uint32_t* sa,
                                             const int (&ak)[4], int (&run)[4], uint32_t& prev_last, bool& bad) {
  const int lane = threadIdx.x & 31;
  const unsigned lt = (1u << lane) - 1u;
  uint8_t mt[kSU];
  uint32_t ai[kSU];
#pragma unroll
  for (int u = 0; u < kSU; ++u) {
    const int i = i0 + u * 32 + lane;
    const bool valid = kFull || i < hi;
    mt[u] = valid ? wmeta[i] : (uint8_t)0;
    ai[u] = valid ? warr[i] : 0xFFFFFFFFu;
  }
#pragma unroll
  for (int u = 0; u < kSU; ++u) {
    const bool valid = kFull || i0 + u * 32 + lane < hi;
    uint32_t ap = __shfl_up_sync(0xffffffffu, ai[u], 1);
    if (lane == 0) ap = prev_last;
    prev_last = __shfl_sync(0xffffffffu, ai[u], 31);
    const int kv = klut[mt[u]];
    bad |= valid && (((kv & 0x8000) != 0) | (ai[u] > tlm1) | (ai[u] < ap));
    const int key = kv & 0x7FFF;
    if (K > 0) {
      int pos = 0;
#pragma unroll
      for (int t = 0; t < K; ++t) {
        const bool mine = valid && key == ak[t];
        const unsigned b = __ballot_sync(0xffffffffu, mine);
        if (mine) pos = run[t] + __popc(b & lt);
        run[t] += __popc(b);
      }
      if (valid) sa[(uint32_t)pos] = ai[u];
    } else {
      const unsigned peers = __match_any_sync(0xffffffffu, valid ? key : 1024 + lane);
      const int rank = __popc(peers & lt);
      // the group's run of slots in stream order; its last lane advances the offset
      const int base = runw[valid ? key : 0];
      if (valid) sa[(uint32_t)(base + rank)] = ai[u];
      if (valid && (peers >> lane) == 1u) runw[key] = base + rank + 1;
      __syncwarp();
    }
  }
}

template <int K>
__device__ __forceinline__ bool scatter_segment(const uint32_t* warr, const uint8_t* wmeta, int lo, int hi,
                                                bool has_prev0, uint32_t prev0, uint32_t tlm1,
                                                const uint16_t* klut, int* runw, uint32_t* sa,
                                                const int (&ak)[4], int (&run)[4]) {
  uint32_t prev_last = has_prev0 ? prev0 : 0u;
  bool bad = false;
  int i0 = lo;
#pragma unroll 1
  for (; i0 + 32 * kSU <= hi; i0 += 32 * kSU)
    scatter_step<K, true>(warr, wmeta, i0, hi, tlm1, klut, runw, sa, ak, run, prev_last, bad);
  if (i0 < hi) scatter_step<K, false>(warr, wmeta, i0, hi, tlm1, klut, runw, sa, ak, run, prev_last, bad);
  return bad;
}

// meta byte b -> stream key 2m + (BE ? 1 : 0), or 0x8000 | 0 for a reserved bit / model id >= M
__device__ __forceinline__ int stream_key(int b, int M) {
  const int m = b & 63;
  const bool ok = !(b & 0x40) && m < M;
  return (2 * (ok ? m : 0) + ((b >> 7) ? 0 : 1)) | (ok ? 0 : 0x8000);
}

__device__ __forceinline__ void build_klut(uint16_t* klut, int M) {
  for (int b = threadIdx.x; b < 256; b += blockDim.x) klut[b] = (uint16_t)stream_key(b, M);
}

constexpr int kPW = 8;  // warps per CTA of P1 / P3

}  // namespace

// P1: warp per (replica, epoch)
__global__ void __launch_bounds__(32 * kPW) part_count_kernel(const uint32_t* arr, const uint8_t* meta,
                                                              const int64_t* roff, const int64_t* eoff,
                                                              int R, int64_t E, int S, int M, uint32_t tlm1,
                                                              bool vec, uint32_t* cnt, int* err) {
  __shared__ uint32_t koff[256];  // meta byte -> byte offset of its stream's counter (4 * key)
  __shared__ int scnt[kPW][kMaxStreams];
  __shared__ uint32_t sink;
  for (int b = threadIdx.x; b < 256; b += blockDim.x) koff[b] = 4u * (uint32_t)(stream_key(b, M) & 0x7FFF);
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  for (int k = lane; k < S; k += 32) scnt[warp][k] = 0;
  __syncthreads();
  const int64_t idx = (int64_t)blockIdx.x * kPW + warp;
  if (idx >= (int64_t)R * E) return;
  if (*(volatile const int*)err & 4) return;  // replica_off rejected: eoff was not written
  const int r = (int)(idx / E);
  const int64_t e = idx - (int64_t)r * E;
  const int64_t lo = eoff[(size_t)r * (E + 1) + e], hi = eoff[(size_t)r * (E + 1) + e + 1];
  if (hi > lo) count_streams(meta + lo, hi - lo, scnt[warp], (uint32_t)__cvta_generic_to_shared(&sink), koff);
  __syncwarp();
  for (int k = lane; k < S; k += 32) cnt[(size_t)idx * S + k] = (uint32_t)scnt[warp][k];
}

// P2: CTA (thread = stream) per replica: stream totals, stream-major bases, run indices.
__global__ void __launch_bounds__(kMaxStreams) part_scan_kernel(const uint32_t* cnt, int64_t E, int S,
                                                                uint32_t* sidx) {
  __shared__ uint32_t sbase[kMaxStreams];
  const int r = blockIdx.x, k = threadIdx.x;
  const uint32_t* c = cnt + (size_t)r * E * S;
  uint32_t tot = 0;
  if (k < S) {
#pragma unroll 8
    for (int64_t e = 0; e < E; ++e) tot += c[e * S + k];
  }
  sbase[k] = tot;
  __syncthreads();
  if (k == 0) {
    uint32_t run = 0;
    for (int j = 0; j < S; ++j) {
      const uint32_t t = sbase[j];
      sbase[j] = run;
      run += t;
    }
  }
  __syncthreads();
  if (k >= S) return;
  uint32_t run = sbase[k];
  uint32_t* o = sidx + (size_t)r * (E + 1) * S;
#pragma unroll 8
  for (int64_t e = 0; e < E; ++e) {
    o[e * S + k] = run;
    run += c[e * S + k];
  }
  o[E * S + k] = run;
}

// P3: warp per (replica, epoch): stable scatter into the stream-sorted copy.
__global__ void __launch_bounds__(32 * kPW) part_scatter_kernel(const uint32_t* arr, const uint8_t* meta,
                                                                const int64_t* roff, const int64_t* eoff,
                                                                const int64_t* saoff, const uint32_t* cnt,
                                                                const uint32_t* sidx, int R, int64_t E, int S,
                                                                int M, uint32_t tlm1, uint32_t* sa, int* err) {
  __shared__ uint16_t klut[256];
  __shared__ int srun[kPW][kMaxStreams];
  build_klut(klut, M);
  __syncthreads();
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const int64_t idx = (int64_t)blockIdx.x * kPW + warp;
  if (idx >= (int64_t)R * E) return;
  const int r = (int)(idx / E);
  const int64_t e = idx - (int64_t)r * E;
  const int64_t lo = eoff[(size_t)r * (E + 1) + e], hi = eoff[(size_t)r * (E + 1) + e + 1];
  if (hi <= lo) return;
  const uint32_t* crow = cnt + (size_t)idx * S;
  const uint32_t* srow = sidx + ((size_t)r * (E + 1) + e) * S;
  int* runw = srun[warp];
  int K = 0, ak[4] = {0, 0, 0, 0}, run[4] = {0, 0, 0, 0};
#pragma unroll 1
  for (int k0 = 0; k0 < S; k0 += 32) {
    const int k = k0 + lane;
    const uint32_t n = k < S ? crow[k] : 0u;
    if (k < S) runw[k] = (int)srow[k];
    unsigned pres = __ballot_sync(0xffffffffu, n > 0);
    __syncwarp();
#pragma unroll 1
    while (pres) {
      const int kk = k0 + __ffs(pres) - 1;
      pres &= pres - 1;
#pragma unroll
      for (int t = 0; t < 4; ++t)
        if (K == t) { ak[t] = kk; run[t] = runw[kk]; }
      ++K;
    }
  }
  uint32_t* out = sa + saoff[r];
  const int n = (int)(hi - lo);
  const bool hp = lo > roff[r];
  const uint32_t pv = hp ? arr[lo - 1] : 0u;
  bool bad = false;
  switch (K) {
    case 0: break;
    case 1: bad = scatter_segment<1>(arr + lo, meta + lo, 0, n, hp, pv, tlm1, klut, runw, out, ak, run); break;
    case 2: bad = scatter_segment<2>(arr + lo, meta + lo, 0, n, hp, pv, tlm1, klut, runw, out, ak, run); break;
    default: bad = scatter_segment<0>(arr + lo, meta + lo, 0, n, hp, pv, tlm1, klut, runw, out, ak, run); break;
  }
  if (__any_sync(0xffffffffu, bad) && lane == 0) atomicOr(err, 1);
}

cudaError_t launch_partition_count(const PartitionArgs& A, cudaStream_t st) {
  const int64_t warps = (int64_t)A.R * A.E;
  if (warps == 0) return cudaSuccess;
  part_count_kernel<<<(unsigned)((warps + kPW - 1) / kPW), 32 * kPW, 0, st>>>(
      A.arr, A.meta, A.roff, A.eoff, A.R, A.E, A.S, A.M, A.tlm1, A.vec, A.cnt, A.err);
  return cudaGetLastError();
}

// After the prepass checked that the epoch ranges tile every replica (monotone offsets, no arrival
// beyond the horizon): the caller checks err first, so the scatter stays inside each replica.
cudaError_t launch_partition_rest(const PartitionArgs& A, cudaStream_t st) {
  const int64_t warps = (int64_t)A.R * A.E;
  if (warps == 0) return cudaSuccess;
  part_scan_kernel<<<A.R, kMaxStreams, 0, st>>>(A.cnt, A.E, A.S, A.sidx);
  cudaError_t e = cudaGetLastError();
  if (e != cudaSuccess) return e;
  part_scatter_kernel<<<(unsigned)((warps + kPW - 1) / kPW), 32 * kPW, 0, st>>>(
      A.arr, A.meta, A.roff, A.eoff, A.saoff, A.cnt, A.sidx, A.R, A.E, A.S, A.M, A.tlm1, A.sa, A.err);
  return cudaGetLastError();
}

cudaError_t preload_partition_kernels() {
  cudaFuncAttributes a;
  cudaError_t e = cudaFuncGetAttributes(&a, part_count_kernel);
  if (e == cudaSuccess) e = cudaFuncGetAttributes(&a, part_scan_kernel);
  if (e == cudaSuccess) e = cudaFuncGetAttributes(&a, part_scatter_kernel);
  return e;
}

}  // namespace pemgpu
