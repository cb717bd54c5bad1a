// chain_state.cuh — the simulated cluster's per-GPU state and its VM / installation events, shared
// by the fused epoch engine (replay.cu) and the lean per-replica chain (chain.cu).  Row layout of
// the per-GPU arrays (shared memory, one column per simulated GPU):
//   gu8 [8][N]  geometry, pending target, hysteresis counter, VM kind, billed kind, decidable,
//               best geometry, reconfiguration wanted
//   gi [14][N]  reconfiguration window start/end, VM from/until, billed since, latest resident end,
//               best key, current geometry's key, on-demand us, spot us, busy, memory-time,
//               Alg 2 EWMA history (policy 2)
#pragma once
#include <stdint.h>
#include "replay.cuh"

namespace pemgpu {
namespace {

struct Ctx {
  Tab T;
  const uint32_t* pack;
  int N;
  uint8_t* gu8;   // [8][N]: geom, target, ctr, vm, bill, dec, best, want
  int64_t* gi;    // [12][N]: rs, re, from, until, since, maxend, kbest, kcur, od, spot, busy, mem
  int *g_cnt, *g_off;
  int* a_n;
  int64_t *a_ls, *a_bu;
  int64_t* keys;
  Bat *sb, *gb;
  uint32_t *sord, *gord, *sgl, *ggl, *sarr;
  int BS;
  // per-epoch generic views (shared or global memory)
  Bat* bats;
  uint32_t *ord, *gl;
  __device__ __forceinline__ Bat& bat_w(int i) const { return i < BS ? sb[i] : gb[i]; }
};

enum { VM_NONE = 0, VM_OD = 1, VM_SPOT = 2 };

__device__ __forceinline__ int64_t clip_h(int64_t x, int64_t H) { return x < H ? x : H; }

__device__ void bill_switch(const Ctx& c, int g, int type, int64_t at, int64_t H) {
  const int64_t d = clip_h(at, H) - clip_h(c.gi[4 * c.N + g], H);
  if (c.gu8[4 * c.N + g] == VM_OD) c.gi[8 * c.N + g] += d;
  if (c.gu8[4 * c.N + g] == VM_SPOT) c.gi[9 * c.N + g] += d;
  c.gu8[4 * c.N + g] = (uint8_t)type;
  c.gi[4 * c.N + g] = at;
}

__device__ void reset_gpu_state(const Ctx& c, int g, int geom) {
  c.gu8[0 * c.N + g] = (uint8_t)geom;
  c.gu8[1 * c.N + g] = kNoGeom;
  c.gu8[2 * c.N + g] = 0;
#pragma unroll 1
  for (int s = 0; s < kZA; ++s) {
    c.a_n[g * kZA + s] = 0;
    c.a_ls[g * kZA + s] = 0;
    c.a_bu[g * kZA + s] = 0;
  }
}

__device__ __forceinline__ bool has_vm(const Ctx& c, int g, int64_t t) {
  return c.gi[2 * c.N + g] <= t && t < c.gi[3 * c.N + g];
}
__device__ __forceinline__ bool available(const Ctx& c, int g, int64_t t) {
  return has_vm(c, g, t) && !(c.gi[0 * c.N + g] <= t && t < c.gi[1 * c.N + g]);
}

// O11: one revocation boundary tau = k * T_rev for node g (draws specified in DESIGN.md §3).
// Returns true when the node changes VM under Spot Only (its containers go with it, reading R27).
__device__ __forceinline__ bool vm_event(const ReplayParams& P, const Ctx& c, uint64_t replica, int g,
                                      int64_t k, int64_t tau) {
  const uint64_t x = (replica << 32) ^ ((uint64_t)g << 20) ^ ((uint64_t)k << 2);
  const uint64_t d0 = smix(P.seed ^ smix(x ^ 0ull)) >> 11;
  const uint64_t d1 = smix(P.seed ^ smix(x ^ 1ull)) >> 11;
  const bool revoked = d0 < P.thr, spot_ok = d1 >= P.thr;
  if (P.vm_policy == 1) {  // PROTEAN: retry spot, else on-demand; seamless redirect
    if (c.gu8[3 * c.N + g] == VM_SPOT) {
      if (revoked && !spot_ok) {
        c.gu8[3 * c.N + g] = VM_OD;
        bill_switch(c, g, VM_OD, tau + P.notice, P.H);
      }
    } else if (c.gu8[3 * c.N + g] == VM_OD) {
      if (spot_ok) {
        c.gu8[3 * c.N + g] = VM_SPOT;
        bill_switch(c, g, VM_SPOT, tau, P.H);
      }
    }
  } else if (P.vm_policy == 2) {  // Spot Only
    if (c.gu8[3 * c.N + g] == VM_SPOT) {
      if (revoked && !spot_ok) {
        c.gu8[3 * c.N + g] = VM_NONE;
        c.gi[3 * c.N + g] = tau;
        bill_switch(c, g, VM_NONE, tau + P.notice, P.H);
        c.gu8[1 * c.N + g] = kNoGeom;
        c.gi[0 * c.N + g] = c.gi[1 * c.N + g] = 0;
        return true;
      }
    } else if (c.gu8[3 * c.N + g] == VM_NONE) {
      if (spot_ok) {
        c.gu8[3 * c.N + g] = VM_SPOT;
        c.gi[2 * c.N + g] = tau;
        c.gi[3 * c.N + g] = kForever;
        bill_switch(c, g, VM_SPOT, tau, P.H);
        reset_gpu_state(c, g, P.init_geom);
        c.gi[0 * c.N + g] = c.gi[1 * c.N + g] = 0;
        return true;
      }
    }
  }
  return false;
}

}  // namespace
}  // namespace pemgpu
