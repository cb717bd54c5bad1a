// Microbenchmark: throughput of MATCH.ANY / REDUX / VOTE / ATOMS on one SM (B200).
#include <cstdio>
#include <cuda_runtime.h>
__global__ void k_match(unsigned* out, int iters, int nkeys) {
  unsigned lane = threadIdx.x & 31, acc = 0, key = (lane * 7) & (nkeys - 1);
  for (int i = 0; i < iters; ++i) {
    unsigned p = __match_any_sync(0xffffffffu, key);
    acc += p; key = (key + (p & 1)) & (nkeys - 1);
  }
  out[blockIdx.x * blockDim.x + threadIdx.x] = acc;
}
__global__ void k_redux(unsigned* out, int iters, int nkeys) {
  unsigned lane = threadIdx.x & 31, acc = 0, key = (lane * 7) & (nkeys - 1);
  for (int i = 0; i < iters; ++i) {
    unsigned p = __reduce_add_sync(0xffffffffu, key);
    acc += p; key = (key + (p & 1)) & (nkeys - 1);
  }
  out[blockIdx.x * blockDim.x + threadIdx.x] = acc;
}
__global__ void k_vote(unsigned* out, int iters, int nkeys) {
  unsigned lane = threadIdx.x & 31, acc = 0, key = (lane * 7) & (nkeys - 1);
  for (int i = 0; i < iters; ++i) {
    unsigned p = __ballot_sync(0xffffffffu, key == 3);
    acc += p; key = (key + (p & 1)) & (nkeys - 1);
  }
  out[blockIdx.x * blockDim.x + threadIdx.x] = acc;
}
__global__ void k_atoms(unsigned* out, int iters, int nkeys) {
  __shared__ unsigned h[1024];
  for (int i = threadIdx.x; i < 1024; i += blockDim.x) h[i] = 0;
  __syncthreads();
  unsigned lane = threadIdx.x & 31, acc = 0, key = (lane * 7) & (nkeys - 1);
  for (int i = 0; i < iters; ++i) {
    atomicAdd(&h[key + (threadIdx.x >> 5) * 0], 1u);
    acc += key; key = (key + 1) & (nkeys - 1);
  }
  __syncthreads();
  out[blockIdx.x * blockDim.x + threadIdx.x] = acc + h[threadIdx.x & 1023];
}
int main() {
  unsigned* d; cudaMalloc(&d, 1 << 24);
  cudaEvent_t a, b; cudaEventCreate(&a); cudaEventCreate(&b);
  const int iters = 4096;
  typedef void (*K)(unsigned*, int, int);
  K ks[4] = {k_match, k_redux, k_vote, k_atoms};
  const char* nm[4] = {"match_any", "redux_add", "ballot", "atoms"};
  int dev; cudaGetDevice(&dev); int nsm; cudaDeviceGetAttribute(&nsm, cudaDevAttrMultiProcessorCount, dev);
  int clk; cudaDeviceGetAttribute(&clk, cudaDevAttrClockRate, dev);
  for (int kk = 0; kk < 4; ++kk)
    for (int nkeys : {1, 2, 8, 32})
      for (int warps : {1, 32}) {
        ks[kk]<<<nsm, 32 * warps>>>(d, iters, nkeys);
        cudaEventRecord(a);
        ks[kk]<<<nsm, 32 * warps>>>(d, iters, nkeys);
        cudaEventRecord(b); cudaEventSynchronize(b);
        float ms; cudaEventElapsedTime(&ms, a, b);
        double cyc = ms * 1e-3 * clk * 1e3;
        printf("%-10s keys %2d warps/SM %2d : %.2f SM-cycles per warp-op (incl loop)\n", nm[kk], nkeys, warps,
               cyc / ((double)iters * warps));
      }
  return 0;
}
