// oracle/pem.hpp — TEST INFRASTRUCTURE ONLY.
//
// The CPU oracle of the PROTEAN epoch model (PEM): a plain, slow, step-by-step C++17 reading of
// the paper's slowdown model (Eq 1/2), Job Distribution (Alg 1), GPU
// Reconfigurator (Alg 2: decision step lines 24-30 + the ~30% cap, and its own
// heuristic, lines 1-23, as policy 2) and
// cost-aware procurement, with the readings of DESIGN.md §3.
//
// Only tests/, __graft_entry__.smoke() and bench.py's cpu_baseline / --impl reference leg may
// load this code.  It shares nothing with the CUDA product (paper_conf_middleware_bhasisjgpkd24_b200/):
// no header, no table, no helper.  Deliberately different data structures: std::vector, explicit
// std::sort / stable partition, geometry enumeration by MIG *placement intervals*.
#pragma once
#include <cstdint>
#include <vector>
#include <string>

namespace pem {

// ---- T2: profiles 1g,2g,3g,4g,7g in ascending-resource order (reading Q3) ------
constexpr int kProfiles = 5;
constexpr int kCompute[kProfiles] = {1, 2, 3, 4, 7};                  // sevenths of the SMs
constexpr int kMemEighths[kProfiles] = {1, 2, 4, 4, 8};               // memory slices of 8 (T2)
constexpr int32_t kA100Mem = 40960;                                    // A100-40GB: 5/10/20/20/40 GB
constexpr int kMaxCount[kProfiles] = {7, 3, 2, 1, 1};
constexpr int kMaxSlices = 7;
constexpr int64_t kPpm = 1000000;               // FBR 1.0 ("0.2 -> 20%")
constexpr int kBuckets = 3328;
constexpr uint64_t kSat32 = 0xFFFFFFFFull;
constexpr int kPoolCap = 128;                   // N3: containers per (sim-GPU, model) (R22)

enum Err { OK = 0, EINVAL_ = -1, ERANGE_ = -2, ENOMEM_ = -3, EUNSUP_ = -7 };

struct Tables {
  int M = 0;
  std::vector<int32_t> solo, fbr;               // [M*5]
  std::vector<int32_t> mem, bsz, slo, tmo;      // [M]
  std::vector<std::vector<int>> geoms;          // candidate geometries: profile ids ascending
  // N4c (P:L495 generalizability; NVIDIA MIG tables, not in the paper): the GPU's memory; a
  // profile holds eighths_p / 8 of it (A100-40GB 40960 MiB -> 5120/10240/20480/20480/40960)
  int32_t gpu_mem = kA100Mem;
  int32_t cap_mem[kProfiles] = {5120, 10240, 20480, 20480, 40960};
  int32_t cap(int p) const { return cap_mem[p]; }
  int32_t solo_at(int m, int p) const { return solo[m * kProfiles + p]; }
  int32_t fbr_at(int m, int p) const { return fbr[m * kProfiles + p]; }
};

// One batch resident on a simulated GPU (Eq 1's "job": jobs may be request batches).
struct Resident {
  int64_t start = 0, end = 0;
  int32_t mem = 0;
  int slice = 0, model = 0;
  bool strict = false;
};

// Carried per-GPU placement state (O6).  Residents whose end <= t can never matter again for
// a Place at a time >= t (every test below is "end > something >= t"), so they are pruned.
struct GpuState {
  int geom = 0;
  std::vector<Resident> res;
  int64_t last_start[kMaxSlices] = {0};
  int64_t busy_until[kMaxSlices] = {0};
  int64_t busy_us[kMaxSlices] = {0};  // O6e: busy union of each slice instance, clipped to [0, H)
};

struct PlaceOut {
  int dropped = 0;          // 0 placed, 2 placement drop, 3 overflow drop
  int slice = -1;
  int64_t start = 0, end = 0;
  // diagnostics for the pins (per slice position): feasible, start, completion, eligible
  bool feasible[kMaxSlices] = {false};
  bool eligible[kMaxSlices] = {false};
  int64_t s_start[kMaxSlices] = {0};
  int64_t s_end[kMaxSlices] = {0};
  int64_t s_F[kMaxSlices] = {0};   // Eq 1's F (ppm) at each feasible slice's start (diagnostic)
};

// Accounting hooks of the actual placement (O6e): busy union + memory-time, clipped to [0,H).
struct Accum {
  int64_t busy_w = 0;   // sum compute7 * busy us
  int64_t mem_num = 0;  // sum mem * |[start,end) ∩ [0,H)|
};

// Eq 1 in integers: exec = floor(solo * max(F, 10^6) / 10^6)  (reading Q10).
int64_t exec_us(int64_t solo, int64_t F_ppm);

// O6: Alg 1 Distribute_Jobs for one batch of model m at time t on geometry `geom`.
// depth (N4b, reading R28): -1 = Alg 1's BE tag walk; d >= 0 = the d smallest slices are reserved
// for BE (strict eligible on positions >= d), with the same fallback to every fitting slice.
PlaceOut place(const Tables& tb, const std::vector<int>& geom, GpuState& S, int64_t t, int m,
               bool strict, int max_live, Accum* acc, int64_t H, int depth = -1);

// ---- O2: geometries by NVIDIA A100 MIG placement intervals (reading Q2) -------------------------
struct GeomStats { int feasible, maximal_placements, placement_maximal_multisets, multiset_maximal; };
std::vector<std::vector<int>> enumerate_geometries(bool all37, GeomStats* stats);

// ---- O3: batch formation -----------------------------------------------------------------------
struct Batch {
  int64_t ready = 0;
  int n = 0;
  int model = 0;
  bool strict = false;
  int64_t first_raw = 0;          // raw index of the first member (id tie-break)
  std::vector<uint32_t> arr;      // member arrivals, ascending
};
std::vector<Batch> form_batches(const Tables& tb, const uint32_t* arrival, const uint8_t* meta,
                                int64_t n);

// ---- O7 / O12 metrics ----------------------------------------------------------------------------
int bucket_of(uint64_t x);
uint64_t bucket_lower(int b);
uint64_t percentile(const uint32_t* hist, int q_percent);

// ---- O11 VM draws ---------------------------------------------------------------------------------
uint64_t splitmix64(uint64_t x);
uint64_t vm_draw(uint64_t seed, uint64_t replica, uint64_t node, uint64_t k, uint64_t d);

// ---- O5..O12: one replica's replay --------------------------------------------------------------
struct ReplayCfg {
  int N = 8;
  int64_t trace_len = 0, W = 1000000;
  int policy = 0, wait_limit = 3, cap_pct = 30, init_geom = 2, max_live = 64, vm_policy = 0;
  int64_t reconfig_us = 2000000;
  double p_rev = 0, price_od = 4.096575, price_spot = 1.228975;
  int64_t rev_interval = 300000000, notice = 30000000;
  uint64_t seed = 0;
  int ewma_alpha_pm = 500;                 // policy 2 (N1): EWMA weight of the newest epoch, per mille
  int64_t t_low = 500, t_high = 4000;      //   T_low / T_high, milli-BE-batches per epoch (R14)
  int64_t cold_us = 0;                     // N3: container cold start t_cold (0 = warm, reading Q15)
  int keepalive_epochs = 600;              //   delayed termination (~10 min of surplus)
  int prewarm = 0;                         //   idle containers per (sim-GPU, model) at t = 0
};
struct BatchRec {
  uint32_t ready; uint32_t epoch; int n, model; bool strict;
  int gpu, slice, dropped; int64_t start, end;
};
struct ReplayOut {
  int64_t counters[10] = {0};
  int64_t cold_starts = 0;              // N3: containers spawned for a batch (cold starts)
  bool pool_overflow = false;           // N3: a pool outgrew kPoolCap containers (ERANGE)
  int64_t accum[4] = {0};
  std::vector<uint32_t> hist;           // [2][3328]
  int64_t p[2][2] = {{0, 0}, {0, 0}};
  double cost = 0, util[2] = {0, 0};
  std::vector<uint8_t> decisions;       // [E][N]
  std::vector<int64_t> cand_keys;       // [E][N][G]
  std::vector<BatchRec> log;
  int64_t n_batches = 0;
  int64_t stats[4] = {0, 0, 0, 0};      // h5 workload self-checks (oracle.h orc_replay_out.stats)
};
int64_t num_epochs(const Tables& tb, int64_t trace_len, int64_t W);
void replay_replica(const Tables& tb, const ReplayCfg& cfg, uint64_t replica_id,
                    const uint32_t* arrival, const uint8_t* meta, int64_t n, bool want_keys,
                    bool want_log, ReplayOut* out);

// second formulation of O6(a)/(b), oracle/tick.cpp
struct TickBatch { int64_t t; int m; int slice; int64_t start = -1, end = -1; };
void tick_simulate(const Tables& tb, const std::vector<int>& geom, std::vector<TickBatch>& bs);

// key of O8 (reading Q20)
int64_t make_key(int64_t misses, int64_t tail, int tag);

// ---- N4a: exhaustive assignment sweep (oracle/sweep.cpp, readings R18-R21) ---------------------
struct SweepBatch {
  int64_t ready = 0;
  int model = 0;
  bool strict = false;
  std::vector<uint32_t> arr;  // member arrivals, ascending
};
PlaceOut place_forced(const Tables& tb, const std::vector<int>& geom, GpuState& S, int64_t t, int m,
                      bool strict, int max_live, int slice);
void sweep_depths(const Tables& tb, int j, int tag, const std::vector<SweepBatch>& bs, int max_live,
                  int64_t* keys, int64_t* best_key, int* best_code, uint64_t* n_eval);
void sweep_gpu(const Tables& tb, int j, int tag, const std::vector<SweepBatch>& bs, int max_live,
               int64_t* key_out, uint64_t* idx_out, uint64_t* n_assign);

}  // namespace pem
