// tools/tracegen.cu — CUDA twin of protean_inputs.traces GEN-1 (input generator only; holds none
// of the method's arithmetic).  Produces the same bytes as the numpy generator for mixes A / B:
// tick i of replica r, source s emits a request iff h>>32 < thr[r][s][sec(i)] with
// h = splitmix64(seed ^ splitmix64(r<<40 ^ i<<2 ^ s)); arrival = 16 i + (h & 15); strict = bit 4;
// model from bits 5..31 (mix A: fixed strict model / per-20 s BE model; mix B: Zipf CDF).
// Two passes: count per (replica, chunk), exclusive scan (host-driven via cub-free block scan),
// then write.  Used by bench.py to build the 61 GB config-5 trace directly in HBM (untimed).
#include <cuda_runtime.h>
#include <stdint.h>

namespace {
constexpr int kTick = 16;
constexpr int64_t kTicksPerSec = 1000000 / kTick;
constexpr int kChunk = 8192;  // ticks per block (256 threads x 32 ticks)

struct Gen {
  int kind, R, seconds, nseg;
  uint64_t seed, base;
  const uint32_t* thr;       // [R][2][seconds]
  const uint8_t* strict_model;  // [R]
  const uint8_t* be_model;   // [R][nseg]
  const uint32_t* cdf;       // [R][2][16]
  int model_base1;
};

__device__ __forceinline__ uint64_t sm64(uint64_t x) {
  x += 0x9E3779B97F4A7C15ull;
  x = (x ^ (x >> 30)) * 0xBF58476D1CE4E5B9ull;
  x = (x ^ (x >> 27)) * 0x94D049BB133111EBull;
  return x ^ (x >> 31);
}

// events of one tick: up to 2 (source 0, source 1) in (time, source) order
__device__ __forceinline__ int tick_events(const Gen& g, int ri, int64_t tick, uint32_t* t_out,
                                           uint8_t* m_out) {
  const uint64_t r = g.base + (uint64_t)ri;
  const int sec = (int)(tick / kTicksPerSec);
  const int nsrc = g.kind == 0 ? 1 : 2;
  int n = 0;
  uint32_t tt[2];
  uint8_t mm[2];
  for (int s = 0; s < nsrc; ++s) {
    const uint64_t h = sm64(g.seed ^ sm64((r << 40) ^ ((uint64_t)tick << 2) ^ (uint64_t)s));
    if ((uint32_t)(h >> 32) < g.thr[((size_t)ri * 2 + s) * g.seconds + sec]) {
      const uint32_t t = (uint32_t)(tick * kTick + (int64_t)(h & 15));
      const uint32_t strict = (uint32_t)((h >> 4) & 1);
      const uint32_t u = (uint32_t)((h >> 5) & ((1u << 27) - 1));
      int model;
      if (g.kind == 0) {
        model = strict ? g.strict_model[ri] : g.be_model[(size_t)ri * g.nseg + sec / 20];
      } else {
        const uint32_t* c = g.cdf + ((size_t)ri * 2 + s) * 16;
        int k = 0;
        while (k < 15 && u >= c[k]) ++k;
        model = k + (s == 0 ? 0 : g.model_base1);
      }
      tt[n] = t;
      mm[n] = (uint8_t)((model & 63) | (strict << 7));
      ++n;
    }
  }
  if (n == 2 && tt[1] < tt[0]) {  // (time, source) order
    t_out[0] = tt[1]; m_out[0] = mm[1]; t_out[1] = tt[0]; m_out[1] = mm[0];
  } else {
    for (int i = 0; i < n; ++i) { t_out[i] = tt[i]; m_out[i] = mm[i]; }
  }
  return n;
}

__global__ void count_kernel(Gen g, int64_t ticks, int nchunk, int64_t* counts) {
  const int ri = blockIdx.y, ch = blockIdx.x;
  const int64_t t0 = (int64_t)ch * kChunk + (int64_t)threadIdx.x * 32;
  int c = 0;
  uint32_t tt[2];
  uint8_t mm[2];
  for (int i = 0; i < 32; ++i) {
    const int64_t tick = t0 + i;
    if (tick < ticks) c += tick_events(g, ri, tick, tt, mm);
  }
  for (int d = 16; d > 0; d >>= 1) c += __shfl_xor_sync(0xffffffffu, c, d);
  __shared__ int ws[8];
  if ((threadIdx.x & 31) == 0) ws[threadIdx.x >> 5] = c;
  __syncthreads();
  if (threadIdx.x == 0) {
    int s = 0;
    for (int w = 0; w < 8; ++w) s += ws[w];
    counts[(size_t)ri * nchunk + ch] = s;
  }
}

// exclusive scan of counts [R*nchunk] in one block (sequential over tiles), replica offsets
__global__ void scan_kernel(int64_t* counts, int64_t n, int nchunk, int64_t* roff) {
  __shared__ int64_t carry;
  __shared__ int64_t buf[1024];
  if (threadIdx.x == 0) carry = 0;
  __syncthreads();
  for (int64_t b = 0; b < n; b += 1024) {
    const int64_t i = b + threadIdx.x;
    const int64_t v = i < n ? counts[i] : 0;
    buf[threadIdx.x] = v;
    __syncthreads();
    for (int d = 1; d < 1024; d <<= 1) {
      int64_t y = threadIdx.x >= d ? buf[threadIdx.x - d] : 0;
      __syncthreads();
      buf[threadIdx.x] += y;
      __syncthreads();
    }
    const int64_t excl = carry + buf[threadIdx.x] - v;
    if (i < n) {
      counts[i] = excl;
      if (i % nchunk == 0) roff[i / nchunk] = excl;
    }
    __syncthreads();
    if (threadIdx.x == 1023) carry += buf[1023];
    __syncthreads();
  }
  if (threadIdx.x == 0) roff[n / nchunk] = carry;
}

__global__ void write_kernel(Gen g, int64_t ticks, int nchunk, const int64_t* offs, uint32_t* arr,
                             uint8_t* meta) {
  const int ri = blockIdx.y, ch = blockIdx.x;
  const int64_t t0 = (int64_t)ch * kChunk + (int64_t)threadIdx.x * 32;
  uint32_t tt[2];
  uint8_t mm[2];
  int c = 0;
  for (int i = 0; i < 32; ++i) {
    const int64_t tick = t0 + i;
    if (tick < ticks) c += tick_events(g, ri, tick, tt, mm);
  }
  __shared__ int sc[256];
  sc[threadIdx.x] = c;
  __syncthreads();
  for (int d = 1; d < 256; d <<= 1) {
    int y = threadIdx.x >= d ? sc[threadIdx.x - d] : 0;
    __syncthreads();
    sc[threadIdx.x] += y;
    __syncthreads();
  }
  int64_t pos = offs[(size_t)ri * nchunk + ch] + sc[threadIdx.x] - c;
  for (int i = 0; i < 32; ++i) {
    const int64_t tick = t0 + i;
    if (tick >= ticks) break;
    const int n = tick_events(g, ri, tick, tt, mm);
    for (int k = 0; k < n; ++k) {
      arr[pos] = tt[k];
      meta[pos] = mm[k];
      ++pos;
    }
  }
}
}  // namespace

extern "C" {

// Pass 1: returns total requests via *total (host), fills roff [R+1] and the chunk offsets
// (scratch counts: R * nchunk int64, caller-allocated via tracegen_scratch_elems).
int64_t tracegen_scratch_elems(int R, int seconds) {
  const int64_t ticks = (int64_t)seconds * kTicksPerSec;
  return (int64_t)R * ((ticks + kChunk - 1) / kChunk);
}

int tracegen_count(int kind, int R, int seconds, uint64_t seed, uint64_t base, const uint32_t* thr,
                   const uint8_t* strict_model, const uint8_t* be_model, int nseg, const uint32_t* cdf,
                   int model_base1, int64_t* scratch, int64_t* roff, int64_t* total, void* stream) {
  Gen g{kind, R, seconds, nseg, seed, base, thr, strict_model, be_model, cdf, model_base1};
  const int64_t ticks = (int64_t)seconds * kTicksPerSec;
  const int nchunk = (int)((ticks + kChunk - 1) / kChunk);
  cudaStream_t st = (cudaStream_t)stream;
  count_kernel<<<dim3(nchunk, R), 256, 0, st>>>(g, ticks, nchunk, scratch);
  scan_kernel<<<1, 1024, 0, st>>>(scratch, (int64_t)R * nchunk, nchunk, roff);
  if (cudaMemcpyAsync(total, roff + R, 8, cudaMemcpyDeviceToHost, st) != cudaSuccess) return -4;
  if (cudaStreamSynchronize(st) != cudaSuccess) return -4;
  return cudaGetLastError() == cudaSuccess ? 0 : -4;
}

int tracegen_write(int kind, int R, int seconds, uint64_t seed, uint64_t base, const uint32_t* thr,
                   const uint8_t* strict_model, const uint8_t* be_model, int nseg, const uint32_t* cdf,
                   int model_base1, const int64_t* scratch, uint32_t* arr, uint8_t* meta, void* stream) {
  Gen g{kind, R, seconds, nseg, seed, base, thr, strict_model, be_model, cdf, model_base1};
  const int64_t ticks = (int64_t)seconds * kTicksPerSec;
  const int nchunk = (int)((ticks + kChunk - 1) / kChunk);
  write_kernel<<<dim3(nchunk, R), 256, 0, (cudaStream_t)stream>>>(g, ticks, nchunk, scratch, arr, meta);
  if (cudaStreamSynchronize((cudaStream_t)stream) != cudaSuccess) return -4;
  return cudaGetLastError() == cudaSuccess ? 0 : -4;
}
}
