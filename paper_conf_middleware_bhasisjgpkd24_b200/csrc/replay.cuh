// replay.cuh — host/device shared launch structures of the fused epoch engine.
#pragma once
#include <stddef.h>
#include <stdint.h>
#include <cuda_runtime.h>
#include "pem_device.cuh"

namespace pemgpu {

// Shared-memory increment by exactly 1, unpredicated (ptxas aggregates a warp's same-address
// increments, ATOMS.POPC.INC); lanes with nothing to count increment a sink word instead, which
// keeps the per-element loops free of branches.
__device__ __forceinline__ void inc_shared(uint32_t saddr) {
  asm volatile("red.shared.add.u32 [%0], 1;" ::"r"(saddr) : "memory");
}

#ifndef PROTEAN_WARPS
#define PROTEAN_WARPS 8  // warps per replay CTA (many-replica launches)
#endif
#ifndef PROTEAN_FEW_WARPS
#define PROTEAN_FEW_WARPS 16  // warps per replay CTA when replicas are fewer than SMs
#endif
constexpr int kNSeg = PROTEAN_WARPS;  // warps per CTA (stream-partition segments)
constexpr int kZA = 8;            // lanes per actual-placement group (one per slice position)
#ifndef PROTEAN_AGPU
#define PROTEAN_AGPU 4
#endif
constexpr int kAG = PROTEAN_AGPU;  // simulated GPUs per actual-placement warp unit (1, 2 or 4)
constexpr int kMaxStreams = 2 * PROTEAN_MAX_MODELS;
constexpr int kPoolCap = 128;     // N3: containers per (sim-GPU, model) (reading R22)
constexpr int kMaxVR = 16;        // virtual ranks: CTAs per replica splitting the geometry range
constexpr int64_t kForever = INT64_MAX;

// One batch of the current epoch (40 B).  info = n | model << 16 | strict << 24.
struct Bat {
  uint64_t key;       // id-order key: ready(32) | class(1) | model(6) | stream position(25)
  uint32_t ready, info, pos;
  uint8_t gpu, slice, drop, pad;
  int64_t start, end;
};

constexpr int kUnitBats = 64;  // batches held per (replica, epoch) unit (config 5: ~38 per epoch)
struct UnitBats {              // 784 B, 16-byte aligned: one cp.async run
  uint32_t nb, pad[3];         // batch count (> kUnitBats: not held, the call takes the fused path)
  uint32_t ready[kUnitBats];
  uint32_t info[kUnitBats];    // n | model << 16 | strict << 24
  uint32_t pos[kUnitBats];     // first member in the replica's stream-sorted copy
};

// Candidate lane packing (host-built, P.pack): per candidate warp w of a GPU and lane l, the
// geometry (0xFF idle), the slice position, the group size Z (power of two >= slice count) and the
// lane of the group's slice 0, packed as j | s << 8 | Z << 16 | base << 24.

// Dynamic shared-memory layout (byte offsets), computed on the host.
struct SmemLayout {
  int S;            // streams = 2 * M
  int N, Gc, CW;    // simulated GPUs, candidate geometries in range, candidate warps per GPU
  int BS, WS;       // batches / window entries held in smem
  size_t tab, pack;
  int KS;           // precomputed candidate keys staged per epoch (cand.cu): N * G, 0 = off
  size_t g_u8, g_i64, g_i32, a_n, a_ls, a_bu, keys, kst, bats, ord, glist, sarr, total;
  __host__ void init(int words, int M, int n_gpus, int gc, int cw, int bs, int ws, int ks = 0) {
    S = 2 * M; N = n_gpus; Gc = gc; CW = cw; BS = bs; WS = ws; KS = ks;
    size_t o = 0;
    auto take = [&](size_t bytes) { size_t r = o; o += (bytes + 15) & ~(size_t)15; return r; };
    tab = take((size_t)words * 4);
    pack = take((size_t)CW * 32 * 4);
    g_u8 = take((size_t)N * 8);                 // geom, target, ctr, vm, bill, dec, best, want
    g_i64 = take((size_t)N * 14 * 8);           // rs, re, from, until, since, maxend, kbest, kcur, od, spot, busy, mem,
                                                // Alg 2 EWMA pred_num, pred_mem (policy 2)
    g_i32 = take((size_t)(2 * N + 2) * 4);      // gcnt[N], goff[N+1]
    a_n = take((size_t)N * kZA * 4);            // actual lanes: list length, last start, busy-until
    a_ls = take((size_t)N * kZA * 8);
    a_bu = take((size_t)N * kZA * 8);
    keys = take((size_t)N * Gc * 8);
    kst = take((size_t)2 * KS * 8);             // [epoch parity][class][geometry]
    bats = take((size_t)BS * sizeof(Bat));
    ord = take((size_t)BS * 4);
    glist = take((size_t)BS * 4);
    sarr = take((size_t)WS * 4);
    total = o;
  }
};

// Mode G exchange buffer of one rank (byte offsets): keys [2 parity][n src][Rcap][Ncap] x
// {best, current} int64, then flags [n src][Rcap] uint32 (the source's sequence number + 1).
struct XLayout {
  int n, Rcap, Ncap;  // n = 0: no exchange
  __host__ __device__ size_t key_off(int par, int src, int r, int g) const {
    return ((((size_t)par * n + src) * Rcap + r) * Ncap + g) * 16;
  }
  __host__ __device__ size_t flag_off(int src, int r) const {
    return (size_t)2 * n * Rcap * Ncap * 16 + ((size_t)src * Rcap + r) * 4;
  }
  __host__ __device__ size_t bytes() const { return flag_off(n, 0); }
};

// Per-warp shared-memory layout of the lean chain (chain.cu), byte offsets from the warp's base.
struct ChainLayout {
  int N, KS;
  int G, M;
  size_t gu8, gi, gcnt, goff, a_n, a_ls, a_bu, msk, kst, ub, gl, gpu, total, fitm;
  __host__ void init(int n, int ks, int g, int m) {
    N = n; KS = ks; G = g; M = m;
    size_t o = 0;
    auto take = [&](size_t bytes) { size_t r = o; o += (bytes + 15) & ~(size_t)15; return r; };
    ub = take(2 * sizeof(UnitBats));             // this epoch's rows and the next one's (cp.async)
    kst = take((size_t)KS * 8);                  // keys: by residue class (cand.cu) or by GPU
    gu8 = take((size_t)N * 8);
    gi = take((size_t)N * 14 * 8);
    gcnt = take((size_t)N * 4);
    goff = take((size_t)(N + 1) * 4);
    a_n = take((size_t)N * kZA * 4);
    a_ls = take((size_t)N * kZA * 8);
    a_bu = take((size_t)N * kZA * 8);
    msk = take((size_t)N * kZA * 8);             // per (GPU, slice): resident slots on the slice
    gl = take(kUnitBats);
    gpu = take(kUnitBats);
    total = o;
    fitm = ((size_t)G * M + 15) & ~(size_t)15;   // per CTA: [G][M] slices of j that hold model m
  }
};

struct ReplayParams {
  // tables
  const int32_t* tab;
  TabLayout tl;
  const uint32_t* pack;    // [CW*32] candidate lane packing
  int maxT;
  // trace (device): the stream-sorted copy built by the partition passes (partition.cu)
  const uint32_t* sa;      // arrivals, per replica stream-major, replica r at sa + saoff[r]
  const int64_t* saoff;    // [R+1] 16-byte aligned replica offsets into sa
  const uint32_t* sidx;    // [R][E+1][S] first request of stream k with arrival >= e*W (replica-relative)
  const int64_t* kfc;      // [R][E][N][G] candidate keys by residue class (cand.cu), or NULL
  // lean chain (chain.cu): the epochs' id-ordered batch rows (cand.cu) and each batch's outcome
  // for the accounting pass: end (us) if placed, else -drop (1 no GPU, 2 no slice, 3 max_live)
  const UnitBats* ub;
  int64_t* bres;           // [R][E][kUnitBats]
  ChainLayout cl;
  const int* ovf;          // set by cand.cu when an epoch outgrew kUnitBats: the chain does nothing
  int R, N;
  int64_t base, trace_len, W, E, H;
  // policy
  int policy, wait_limit, cap_pct, init_geom, max_live, vm_policy;
  int ewma_a, g421, g43;   // policy 2 (N1): EWMA weight per mille, indices of (4g,2g,1g), (4g,3g)
  int64_t t_low, t_high;   //   T_low / T_high in milli-BE-batches per epoch
  int64_t cold_us;         // N3: container cold start (0 = warm containers, no pool work)
  int keepalive, prewarm;  //   delayed termination (epochs), idle containers at t = 0
  int64_t reconfig_us, rev, notice;
  uint64_t thr, seed;
  double price_od, price_spot;
  int geom_lo, geom_hi;
  // outputs (device)
  int64_t* counters;
  int64_t* accum;
  uint32_t* hist;
  int64_t* pct;
  double* cost;
  double* util;
  uint8_t* decisions;
  int64_t* cand_keys;
  protean_batch_rec* log;
  int64_t log_cap;
  int64_t* n_batches;
  int64_t* cold_starts;    // [R] N3 cold starts, or NULL
  // scratch
  SmemLayout sl;
  int WCAP;                // max window entries of any epoch (prepass)
  char* scratch;
  size_t slot_bytes, o_alist, o_clist, o_gbat, o_gord, o_gglist, o_gsarr, o_pool;
  int* err;                // err[0]: invalid request, err[1]: exchange timeout, err[2]: pool overflow
  // mode G exchange (xl.n == 0: off)
  XLayout xl;
  char* const* xpeer;      // [n] every rank's exchange buffer, mapped in this process
  int xrank;
  uint32_t xseq;           // sequence number of epoch 0 of this call
  uint64_t xtimeout_ns;    // a source flag not seen within this time fails the call (ENCCL)
  // virtual ranks (vr_n > 1): CTA b serves replica b / vr_n, geometry range b % vr_n
  int vr_n;
  bool few;                // fewer replicas than SMs (the long-list kernel instances)
  int vr_lo[kMaxVR], vr_hi[kMaxVR], vr_cw[kMaxVR];
  const uint32_t* vr_pack[kMaxVR];
  uint32_t* vr_done;       // [R] CTAs of the replica past finalize's histogram (zeroed by the host)
};

struct ScoreParams {
  const int32_t* tab;
  TabLayout tl;
  int R, N, epoch, max_live, geom_lo, geom_hi;
  int64_t W, H;
  const protean_batch* batches;
  const int32_t* batch_off;
  const uint32_t* arrival;
  protean_gpu_state* state;
  int64_t* best_key;
  int64_t* cand_key;
  protean_placement* placement;
  int64_t* counters;
  int64_t* accum;
  double* cost;               // [R*N] node-epoch VM cost, or NULL
  double price_od, price_spot;
  const uint32_t* pack;       // [cw * 32] candidate lane packing of [geom_lo, geom_hi)
  int cw;                     // candidate warps per GPU
  void* lists;                // per-CTA lane lists, list_bytes each (score_list_bytes)
  size_t list_bytes;
  int* err;                   // err[0] EINVAL, err[1] ERANGE (latched until protean_score_epoch_status)
};

// protean_form_batches (form.cu): batch formation + round-robin dispatch on the stream-sorted copy
struct FormParams {
  const uint32_t* sa;      // stream-sorted arrivals (partition.cu), replica r at sa + saoff[r]
  const int64_t* saoff;
  const uint32_t* sidx;    // [R][E+1][S] stream run starts per epoch (row E = stream ends)
  const int32_t* bsz;      // [M] batch sizes, [M] timeouts (the staged table)
  const int32_t* tmo;
  const int64_t* avail;    // [R][N][2] {from, until} or NULL
  int R, N, S, e_lo, e_hi, pass;
  int64_t E, W;
  int32_t* cnt;            // [R][e_hi - e_lo][N] rows per cell (pass 0) / fill (pass 1, zeroed)
  const int32_t* off;      // pass 1: first row of every cell (the caller's batch_off)
  protean_batch* rows;
};
cudaError_t launch_form(const FormParams& P, cudaStream_t st);
cudaError_t preload_form_kernel();

// N4a exhaustive assignment sweep (sweep.cu)
struct SweepParams {
  const int32_t* tab;
  TabLayout tl;
  int R, N, max_live, max_batches, geom_lo, geom_hi;
  const protean_batch* batches;
  const int32_t* batch_off;
  const uint32_t* arrival;
  const uint8_t* cur_geom;
  int64_t* sweep_key;
  uint32_t* assign;
  int64_t* best_key;
  int64_t* n_assign;
  int* err;                   // err[0] EINVAL, err[1] ERANGE
};
cudaError_t launch_sweep(const SweepParams& P, int grid, cudaStream_t st);

// N4b BE-reserve depth sweep (score.cu): lanes (replica, gpu, geometry, depth code)
struct DepthParams {
  const int32_t* tab;
  TabLayout tl;
  int R, N, max_live, geom_lo, geom_hi;
  const protean_batch* batches;
  const int32_t* batch_off;
  const uint32_t* arrival;
  const uint8_t* cur_geom;
  int64_t* depth_key;         // [R*N*nc*8] (library scratch when the caller passes NULL)
  uint8_t* depth_code;        // [R*N*nc] or NULL
  int64_t* best_key;          // [R*N]
  int64_t* n_eval;            // [1] += evaluations
  int64_t n_eval_add;
  protean_resident* scratch;  // [grid*block][max_live]
  int* err;                   // err[0] EINVAL
};
cudaError_t launch_depths(const DepthParams& P, int grid, int block, cudaStream_t st);
cudaError_t preload_sweep_kernel();

// Trace-level stream partition (partition.cu): P1 count + validate, P2 scan, P3 stable scatter.
struct PartitionArgs {
  const uint32_t* arr;
  const uint8_t* meta;
  const int64_t* roff;
  const int64_t* eoff;     // [R][E+1]
  const int64_t* saoff;    // [R+1]
  int R, S, M;
  int64_t E;
  uint32_t tlm1;           // trace_len - 1 (arrivals fit 32 bits, host check)
  bool vec;                // arr and meta 16-byte aligned
  uint32_t* cnt;           // [R][E][S] scratch
  uint32_t* sidx;          // [R][E+1][S]
  uint32_t* sa;            // stream-sorted arrivals
  int* err;                // err[0] |= invalid request
};
cudaError_t launch_partition_count(const PartitionArgs& A, cudaStream_t st);
cudaError_t launch_partition_rest(const PartitionArgs& A, cudaStream_t st);
cudaError_t preload_partition_kernels();

// The candidate search ahead of the chain (cand.cu): batch-aligned stream cursors, then the keys
// of every (replica, epoch, residue class, geometry) from idle, and every epoch's id-ordered
// batch rows (UnitBats) for the lean chain and the accounting pass (chain.cu).
struct CandParams {
  const int32_t* tab;      // device table block (global)
  TabLayout tl;
  const uint32_t* sa;
  const int64_t* saoff;
  const uint32_t* sidx;    // [R][E+1][S]
  uint32_t* bstart;        // [R][S][E+1] the chain's stream cursor at the start of each epoch
  int64_t* kfc;            // [R][E][N][G]; [..][0][0] = INT64_MIN: unit not held, chain scores it
  UnitBats* ub;            // [R][E] id-ordered batch rows, or NULL (fused chain: it forms its own)
  int* overflow;           // set when some unit holds more than kUnitBats batches
  const uint8_t* gorder;   // [G] geometries by slice count, descending (lane order)
  int R, S, N, max_live;
  int64_t E, W;
  size_t ws_off;
};
cudaError_t launch_walk(const CandParams& P, cudaStream_t st);
cudaError_t launch_cand(const CandParams& P, int grid, cudaStream_t st);
cudaError_t cand_occupancy(const TabLayout& tl, int* per_sm);
size_t cand_smem_bytes(const TabLayout& tl, size_t* ws_off);
cudaError_t preload_cand_kernels();
cudaError_t launch_chain(const ReplayParams& P, int grid, cudaStream_t st);
cudaError_t launch_acct(const ReplayParams& P, cudaStream_t st);
cudaError_t chain_occupancy(const ReplayParams& P, int* per_sm);
size_t chain_smem_bytes(const ReplayParams& P);
cudaError_t preload_chain_kernels();

// launchers (replay.cu / score.cu)
cudaError_t launch_roff_scan(const int64_t* roff, int R, int64_t* saoff, int* err, cudaStream_t st);
cudaError_t launch_prepass(const uint32_t* arr, const int64_t* roff, int R, int64_t E, int64_t W,
                           int64_t maxT, int64_t* eoff, unsigned long long* wmax, int* err,
                           cudaStream_t st);
cudaError_t launch_replay(const ReplayParams& P, int grid, int block, cudaStream_t st);
cudaError_t replay_occupancy(int block, size_t smem, bool few, int* blocks_per_sm);
cudaError_t preload_kernels();
cudaError_t launch_score(const ScoreParams& P, int block, cudaStream_t st);
size_t score_smem_bytes(const TabLayout& tl, int N, int Gc);
size_t score_list_bytes(int N, int block, int max_live);

}  // namespace pemgpu
