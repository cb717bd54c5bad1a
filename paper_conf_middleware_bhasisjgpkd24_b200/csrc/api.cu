// api.cu — host side of the C ABI (include/protean.h): validation, the geometry set by T2 sum
// constraints (reading Q2), device tables, scratch, launches.
#include <cuda_runtime.h>

#include <algorithm>
#include <array>
#include <cmath>
#include <cstdio>
#include <cstdlib>
#include <cstring>
#include <string>
#include <vector>

#include "replay.cuh"

using namespace pemgpu;

struct protean_handle {
  int device = 0;
  int M = 0, G = 0, maxT = 0;
  TabLayout tl;
  std::vector<int32_t> words;
  std::vector<uint8_t> geoms;  // [G][8]
  int32_t* d_tab = nullptr;
  std::string err;
  bool poisoned = false;
  int nsm = 148;
  void* d_scratch = nullptr;
  size_t scratch_bytes = 0;
  int64_t* d_eoff = nullptr;
  size_t eoff_bytes = 0;
  // trace-level stream partition (partition.cu): counts, run indices, stream-sorted arrivals
  void* d_cnt = nullptr;
  size_t cnt_bytes = 0;
  void* d_sidx = nullptr;
  size_t sidx_bytes = 0;
  void* d_sa = nullptr;
  size_t sa_bytes = 0;
  void* d_saoff = nullptr;
  size_t saoff_bytes = 0;
  void* d_small = nullptr;  // wmax (8 B) + err (16 B) at 64; score_epoch's latched verdict (8 B) at 256
  uint32_t* d_pack = nullptr;  // candidate lane packing for the full geometry range
  int CW = 0;
  // [0,1] prepass + partition count, [4,5] partition scan + scatter, [2,3] replay kernel
  cudaEvent_t ev[6] = {nullptr, nullptr, nullptr, nullptr, nullptr, nullptr};
  float t_prepass = 0.f, t_replay = 0.f, t_search = 0.f;
  // the candidate search ahead of the chain (cand.cu): batch-aligned cursors, keys, lane order
  void* d_cand = nullptr;
  size_t cand_bytes = 0;
  cudaEvent_t evc[4] = {nullptr, nullptr, nullptr, nullptr};
  float t_walk = 0.f, t_acct = 0.f;
  uint8_t* d_gorder = nullptr;
  int last_grid = 0, last_block = 0, last_smem = 0, last_per_sm = 0;
  std::vector<int> gn;  // slice count per geometry
  // mode G: candidate lane packing of the rank's geometry range
  uint32_t* d_pack_g = nullptr;
  int CW_g = 0, pack_lo = -1, pack_hi = -1;
  // virtual ranks (several CTAs per replica inside one launch): packs, exchange buffers
  int vr_n = 0;
  std::vector<uint32_t*> vr_pack;
  std::vector<int> vr_b, vr_cw;
  void* d_vxbuf = nullptr;
  size_t vx_bytes = 0;
  char** d_vpeer = nullptr;
  void* d_vdone = nullptr;  // [R] finalize arrival counters of the split accounting
  size_t vdone_bytes = 0;
  XLayout vxl{0, 0, 0};
  uint32_t vseq = 0;
  // mode G exchange (protean_xchg_*)
  XLayout xl{0, 0, 0};
  int xrank = 0;
  bool x_ready = false;
  uint32_t xseq = 0;
  void* d_xbuf = nullptr;                // this rank's buffer (owned)
  std::vector<char*> xpeer;              // every rank's buffer in this process
  std::vector<char> x_opened;            // 1 = opened through cudaIpcOpenMemHandle
  char** d_xpeer = nullptr;              // device copy of xpeer
  // protean_score_epoch: candidate lane packing of the last geometry range
  uint32_t* d_sc_pack = nullptr;
  int sc_lo = -1, sc_hi = -1, sc_cw = 0;
  // protean_replay_traces_host: double-buffered device staging of trace chunks and outputs
  void* d_hb[2] = {nullptr, nullptr};
  size_t hb_bytes[2] = {0, 0};
  cudaStream_t hs_copy = nullptr, hs_back = nullptr;
  cudaEvent_t hev[3][2] = {{nullptr, nullptr}, {nullptr, nullptr}, {nullptr, nullptr}};
};

namespace {

int fail(protean_handle* h, int code, const std::string& what) {
  if (h) h->err = what;
  return code;
}

int cuda_fail(protean_handle* h, cudaError_t e, const char* where) {
  if (h) {
    h->poisoned = true;
    h->err = std::string(where) + ": " + cudaGetErrorString(e);
  }
  return PROTEAN_ECUDA;
}

#define CK(h, call)                                    \
  do {                                                 \
    cudaError_t e_ = (call);                           \
    if (e_ != cudaSuccess) return cuda_fail(h, e_, #call); \
  } while (0)

const int kCompute[5] = {1, 2, 3, 4, 7};
const int kMem[5] = {5120, 10240, 20480, 20480, 40960};
const int kMaxCnt[5] = {7, 3, 2, 1, 1};

// O2 by T2 sum constraints: count vectors with at most the T2 max counts, <= 7/7 compute and
// <= 40 GB (<= 8/8 of the memory: the set is the same for every MIG table of N4c, whose profiles
// keep T2's memory eighths).  Default set = multiset-maximal ones.  Order: (c7g,c4g,c3g,c2g,c1g) descending.
std::vector<std::vector<uint8_t>> geometry_set(bool all) {
  std::vector<std::array<int, 5>> feas;
  for (int a = 0; a <= kMaxCnt[0]; ++a)
    for (int b = 0; b <= kMaxCnt[1]; ++b)
      for (int c = 0; c <= kMaxCnt[2]; ++c)
        for (int d = 0; d <= kMaxCnt[3]; ++d)
          for (int f = 0; f <= kMaxCnt[4]; ++f) {
            const int cnt[5] = {a, b, c, d, f};
            int comp = 0, mem = 0, tot = 0;
            for (int p = 0; p < 5; ++p) {
              comp += cnt[p] * kCompute[p];
              mem += cnt[p] * kMem[p];
              tot += cnt[p];
            }
            if (tot >= 1 && comp <= 7 && mem <= 40960) feas.push_back({a, b, c, d, f});
          }
  std::vector<std::array<int, 5>> keep;
  for (const auto& x : feas) {
    bool dominated = false;
    for (const auto& y : feas) {
      if (y == x) continue;
      bool ge = true;
      for (int p = 0; p < 5; ++p) ge = ge && y[p] >= x[p];
      if (ge) dominated = true;
    }
    if (all || !dominated) keep.push_back(x);
  }
  std::sort(keep.begin(), keep.end(), [](const std::array<int, 5>& x, const std::array<int, 5>& y) {
    for (int p = 4; p >= 0; --p)
      if (x[p] != y[p]) return x[p] > y[p];
    return false;
  });
  std::vector<std::vector<uint8_t>> out;
  for (const auto& x : keep) {
    std::vector<uint8_t> g;
    for (int p = 0; p < 5; ++p)
      for (int i = 0; i < x[p]; ++i) g.push_back((uint8_t)p);
    out.push_back(g);
  }
  return out;
}

int validate_row(const uint8_t* row, std::vector<uint8_t>* g) {
  int cnt[5] = {0, 0, 0, 0, 0}, comp = 0, mem = 0, k = 0;
  bool ended = false;
  for (int i = 0; i < 8; ++i) {
    if (row[i] == 0xFF) { ended = true; continue; }
    if (ended || row[i] >= 5 || i >= 7 || (k > 0 && row[i] < (*g)[k - 1])) return PROTEAN_EINVAL;
    cnt[row[i]]++;
    comp += kCompute[row[i]];
    mem += kMem[row[i]];
    g->push_back(row[i]);
    ++k;
  }
  if (k == 0) return PROTEAN_EINVAL;
  for (int p = 0; p < 5; ++p)
    if (cnt[p] > kMaxCnt[p]) return PROTEAN_EINVAL;
  if (comp > 7 || mem > 40960) return PROTEAN_EINVAL;
  return PROTEAN_OK;
}

// Grow a scratch buffer with the stream-ordered allocator: cudaMalloc / cudaFree are implicit
// device-wide synchronisation points, which would serialise (and, with the mode-G exchange,
// stall) replay kernels that other handles of this process run concurrently.
int ensure(protean_handle* h, void** p, size_t* have, size_t need, cudaStream_t st) {
  if (*have >= need && *p) return PROTEAN_OK;
  if (*p) cudaFreeAsync(*p, st);
  *p = nullptr;
  *have = 0;
  cudaError_t e = cudaMallocAsync(p, need, st);
  if (e != cudaSuccess) {  // give the device pool's idle memory back and retry once
    cudaGetLastError();
    cudaMemPool_t pool;
    if (cudaDeviceGetDefaultMemPool(&pool, h->device) == cudaSuccess) {
      cudaStreamSynchronize(st);
      cudaMemPoolTrimTo(pool, 0);
      e = cudaMallocAsync(p, need, st);
    }
  }
  if (e != cudaSuccess) {
    cudaGetLastError();
    *p = nullptr;
    return fail(h, PROTEAN_ENOMEM, "cudaMallocAsync scratch failed");
  }
  *have = need;
  return PROTEAN_OK;
}

size_t al(size_t x) { return (x + 255) & ~(size_t)255; }

// Candidate lane packing of geometries [lo, hi): power-of-two lane groups (>= the slice count),
// largest first, filled into 32-lane warps; entry = j | slice << 8 | Z << 16 | group base << 24.
std::vector<uint32_t> build_pack(const std::vector<int>& gn, int lo, int hi, int* CW) {
  std::vector<uint32_t> pack;
  std::vector<std::pair<int, int>> order;  // (Z, j)
  for (int j = lo; j < hi; ++j) {
    int Z = 1;
    while (Z < gn[j]) Z <<= 1;
    order.push_back({Z, j});
  }
  std::stable_sort(order.begin(), order.end(),
                   [](const std::pair<int, int>& a, const std::pair<int, int>& b) { return a.first > b.first; });
  int fill = 32;
  for (const auto& zj : order) {
    const int Z = zj.first, j = zj.second;
    if (fill + Z > 32) {
      pack.insert(pack.end(), 32, 0xFFu);
      fill = 0;
    }
    const size_t w0 = pack.size() - 32;
    for (int s = 0; s < Z; ++s)
      pack[w0 + fill + s] = (uint32_t)j | ((uint32_t)s << 8) | ((uint32_t)Z << 16) | ((uint32_t)fill << 24);
    fill += Z;
  }
  *CW = (int)(pack.size() / 32);
  return pack;
}

// Slot-balanced split of G geometries (slice counts gn) into nranks non-empty ranges: cut k sits
// at the geometry boundary whose running slice count is nearest k/nranks of the total (ties to
// the earlier boundary), kept strictly increasing.
void split_ranges(const std::vector<int>& gn, int nranks, int32_t* b) {
  const int G = (int)gn.size();
  std::vector<int64_t> pre(G + 1, 0);
  for (int j = 0; j < G; ++j) pre[j + 1] = pre[j] + gn[j];
  const int64_t total = pre[G];
  b[0] = 0;
  for (int k = 1; k < nranks; ++k) {
    int best = 0;
    int64_t bd = -1;
    for (int j = 0; j <= G; ++j) {
      const int64_t d = std::llabs(pre[j] * nranks - (int64_t)k * total);
      if (bd < 0 || d < bd) { bd = d; best = j; }
    }
    best = std::max(best, b[k - 1] + 1);
    best = std::min(best, G - (nranks - k));
    b[k] = best;
  }
  b[nranks] = G;
}

// Geometry lists of a profile set (protean_load_profiles' rules), host only.
int profile_geometries(const protean_profiles* p, std::vector<std::vector<uint8_t>>* gs) {
  if (!p || p->abi_version != PROTEAN_ABI_VERSION) return PROTEAN_EINVAL;
  if (p->geometry_set == 0 || p->geometry_set == 1) {
    *gs = geometry_set(p->geometry_set == 1);
    return PROTEAN_OK;
  }
  if (p->geometry_set != 2) return PROTEAN_EINVAL;
  if (p->n_geoms < 1) return PROTEAN_EINVAL;
  if (p->n_geoms > 254) return PROTEAN_ERANGE;
  if (!p->geoms) return PROTEAN_EINVAL;
  for (int j = 0; j < p->n_geoms; ++j) {
    std::vector<uint8_t> g;
    int rc = validate_row(p->geoms + 8 * j, &g);
    if (rc) return rc;
    gs->push_back(g);
  }
  return PROTEAN_OK;
}

void xchg_release(protean_handle* h) {
  for (size_t i = 0; i < h->xpeer.size(); ++i)
    if (h->x_opened[i] && h->xpeer[i]) cudaIpcCloseMemHandle(h->xpeer[i]);
  if (h->d_xbuf) cudaFree(h->d_xbuf);
  if (h->d_xpeer) cudaFree(h->d_xpeer);
  h->d_xbuf = nullptr;
  h->d_xpeer = nullptr;
  h->xpeer.clear();
  h->x_opened.clear();
  h->x_ready = false;
  h->xl = XLayout{0, 0, 0};
  h->xseq = 0;
}

int xchg_alloc(protean_handle* h, int nranks, int rank, int max_replicas, int max_gpus) {
  if (nranks < 2 || nranks > 64 || rank < 0 || rank >= nranks) return fail(h, PROTEAN_EINVAL, "nranks/rank");
  if (max_replicas < 1 || max_gpus < 1) return fail(h, PROTEAN_EINVAL, "exchange capacity");
  if (max_gpus > 255) return fail(h, PROTEAN_ERANGE, "max_gpus > 255");
  if (nranks > h->G) return fail(h, PROTEAN_EINVAL, "more ranks than geometries");
  CK(h, cudaSetDevice(h->device));
  xchg_release(h);
  h->xl = XLayout{nranks, max_replicas, max_gpus};
  h->xrank = rank;
  const size_t bytes = h->xl.bytes();
  cudaError_t e = cudaMalloc(&h->d_xbuf, bytes);
  if (e != cudaSuccess) {
    cudaGetLastError();
    h->d_xbuf = nullptr;
    h->xl = XLayout{0, 0, 0};
    return fail(h, PROTEAN_ENOMEM, "exchange buffer");
  }
  CK(h, cudaMemset(h->d_xbuf, 0, bytes));
  CK(h, cudaDeviceSynchronize());
  h->xpeer.assign(nranks, nullptr);
  h->x_opened.assign(nranks, 0);
  h->xpeer[rank] = static_cast<char*>(h->d_xbuf);
  return PROTEAN_OK;
}

int xchg_finish(protean_handle* h) {
  CK(h, cudaSetDevice(h->device));
  {  // candidate lane packing of this rank's geometry range
    std::vector<int32_t> b(h->xl.n + 1);
    split_ranges(h->gn, h->xl.n, b.data());
    int cw = 0;
    std::vector<uint32_t> pk = build_pack(h->gn, b[h->xrank], b[h->xrank + 1], &cw);
    if (h->d_pack_g) cudaFree(h->d_pack_g);
  if (h->d_sc_pack) cudaFree(h->d_sc_pack);
    h->d_pack_g = nullptr;
    CK(h, cudaMalloc(&h->d_pack_g, pk.size() * 4));
    CK(h, cudaMemcpy(h->d_pack_g, pk.data(), pk.size() * 4, cudaMemcpyHostToDevice));
    h->CW_g = cw;
    h->pack_lo = b[h->xrank];
    h->pack_hi = b[h->xrank + 1];
  }
  // load every kernel now: lazy module loading at first launch must not run while a peer rank's
  // replay kernel in this process spins on the exchange
  CK(h, preload_kernels());
  CK(h, preload_sweep_kernel());
  CK(h, preload_form_kernel());
  CK(h, preload_cand_kernels());
  CK(h, preload_chain_kernels());
  CK(h, cudaMalloc(&h->d_xpeer, sizeof(char*) * h->xpeer.size()));
  CK(h, cudaMemcpy(h->d_xpeer, h->xpeer.data(), sizeof(char*) * h->xpeer.size(), cudaMemcpyHostToDevice));
  h->x_ready = true;
  h->xseq = 0;
  return PROTEAN_OK;
}

}  // namespace

// The trace-level stream partition shared by protean_replay_traces and protean_form_batches
// (partition.cu): prepass (epoch offsets, largest window, sortedness), P1 count + validate, then
// P2 run indices and the P3 stable scatter into the stream-sorted copy (h->d_sa at h->d_saoff).
// Request-level faults found by P3 are left in err[0] for the caller to report after its kernels.
// timing: record the prepass / partition events read by protean_last_timings.
int partition_trace(protean_handle* h, const protean_replay_cfg& c, int64_t E, cudaStream_t st,
                    bool timing, unsigned long long* wmax_out) {
  const int R = c.n_replicas, S = 2 * h->M;
  const int64_t W = c.epoch_len_us;
  {
    void* p = h->d_eoff;
    int rc = ensure(h, &p, &h->eoff_bytes, sizeof(int64_t) * (size_t)R * (size_t)(E + 1), st);
    h->d_eoff = static_cast<int64_t*>(p);
    if (!rc) rc = ensure(h, &h->d_cnt, &h->cnt_bytes, std::max<size_t>(4, sizeof(uint32_t) * (size_t)R * E * S), st);
    if (!rc) rc = ensure(h, &h->d_sidx, &h->sidx_bytes, std::max<size_t>(4, sizeof(uint32_t) * (size_t)R * (E + 1) * S), st);
    if (!rc) rc = ensure(h, &h->d_saoff, &h->saoff_bytes, sizeof(int64_t) * (size_t)(R + 1), st);
    if (rc) return rc;
  }
  unsigned long long* d_wmax = static_cast<unsigned long long*>(h->d_small);
  int* d_err = reinterpret_cast<int*>(static_cast<char*>(h->d_small) + 64);
  CK(h, cudaMemsetAsync(h->d_small, 0, 256, st));
  if (timing) CK(h, cudaEventRecord(h->ev[0], st));
  // replica_off is validated and scanned on the device: the call's only host round trip before
  // the replay is the one below (the window size and the copy's length size the next launches)
  CK(h, launch_roff_scan(c.replica_off, R, static_cast<int64_t*>(h->d_saoff), d_err, st));
  CK(h, launch_prepass(c.arrival_us, c.replica_off, R, E, W, h->maxT, h->d_eoff, d_wmax, d_err, st));
  PartitionArgs PA;
  PA.arr = c.arrival_us;
  PA.meta = c.meta;
  PA.roff = c.replica_off;
  PA.eoff = h->d_eoff;
  PA.saoff = static_cast<const int64_t*>(h->d_saoff);
  PA.R = R;
  PA.S = S;
  PA.M = h->M;
  PA.E = E;
  PA.tlm1 = (uint32_t)(c.trace_len_us - 1);  // trace_len - 1 + maxT <= 2^32 - 1 (checked by callers)
  PA.vec = ((reinterpret_cast<uintptr_t>(c.arrival_us) & 15u) == 0) &&
           ((reinterpret_cast<uintptr_t>(c.meta) & 15u) == 0);
  PA.cnt = static_cast<uint32_t*>(h->d_cnt);
  PA.sidx = static_cast<uint32_t*>(h->d_sidx);
  PA.sa = nullptr;
  PA.err = d_err;
  CK(h, launch_partition_count(PA, st));
  if (timing) CK(h, cudaEventRecord(h->ev[1], st));
  unsigned long long wmax = 0;
  int herr = 0;
  int64_t sa_len = 0;
  CK(h, cudaMemcpyAsync(&wmax, d_wmax, 8, cudaMemcpyDeviceToHost, st));
  CK(h, cudaMemcpyAsync(&herr, d_err, 4, cudaMemcpyDeviceToHost, st));
  CK(h, cudaMemcpyAsync(&sa_len, static_cast<int64_t*>(h->d_saoff) + R, 8, cudaMemcpyDeviceToHost, st));
  CK(h, cudaStreamSynchronize(st));
  if (herr & 4) return fail(h, PROTEAN_EINVAL, "replica_off: first entry != 0 or not monotone");
  // the prepass guarantees that the epoch ranges tile every replica (else the scatter could leave
  // it); request-level validation happens in the scatter pass and is reported by the caller
  if (herr) return fail(h, PROTEAN_EINVAL, "arrivals not sorted or beyond the trace");
  if (wmax >= (1ull << 25)) return fail(h, PROTEAN_ERANGE, "epoch window >= 2^25 requests");
  {
    int rc = ensure(h, &h->d_sa, &h->sa_bytes, std::max<size_t>(16, sizeof(uint32_t) * (size_t)sa_len), st);
    if (rc) return rc;
  }
  PA.sa = static_cast<uint32_t*>(h->d_sa);
  // P2 + P3: run indices and the stable scatter (only on a validated trace)
  if (timing) CK(h, cudaEventRecord(h->ev[4], st));
  CK(h, launch_partition_rest(PA, st));
  if (timing) CK(h, cudaEventRecord(h->ev[5], st));
  *wmax_out = wmax;
  return PROTEAN_OK;
}

extern "C" {

const char* protean_strerror(int code) {
  switch (code) {
    case PROTEAN_OK: return "ok";
    case PROTEAN_EINVAL: return "invalid argument";
    case PROTEAN_ERANGE: return "value out of range";
    case PROTEAN_ENOMEM: return "out of memory";
    case PROTEAN_ECUDA: return "CUDA error";
    case PROTEAN_ENCCL: return "NCCL error";
    case PROTEAN_ESTATE: return "bad state (poisoned handle or call order)";
    case PROTEAN_EUNSUP: return "unsupported in this build";
    default: return "unknown error";
  }
}

const char* protean_last_error(const protean_handle* h) { return h ? h->err.c_str() : ""; }

void protean_replay_cfg_defaults(protean_replay_cfg* c) {
  std::memset(c, 0, sizeof(*c));
  c->n_gpus = 8;
  c->epoch_len_us = 1000000;
  c->policy = 0;
  c->wait_limit = 3;
  c->reconfig_cap_pct = 30;
  c->init_geom = 2;
  c->max_live = 64;
  c->vm_policy = 0;
  c->reconfig_us = 2000000;
  c->p_rev = 0.0;
  c->price_od_node_hr = 32.7726 / 8.0;
  c->price_spot_node_hr = 9.8318 / 8.0;
  c->rev_interval_us = 300000000;
  c->notice_us = 30000000;
  c->ewma_alpha_pm = 500;
  c->t_low_milli = 500;
  c->t_high_milli = 4000;
  c->cold_start_us = 0;
  c->keepalive_epochs = 600;
  c->prewarm = 0;
  c->ctas_per_replica = 0;
}

int protean_load_profiles(const protean_profiles* p, protean_handle** out) {
  if (!out) return PROTEAN_EINVAL;
  *out = nullptr;
  if (!p || p->abi_version != PROTEAN_ABI_VERSION) return PROTEAN_EINVAL;
  const int M = p->n_models;
  if (M < 1 || M > PROTEAN_MAX_MODELS) return PROTEAN_EINVAL;
  if (!p->solo_us || !p->fbr_ppm || !p->mem_mib || !p->batch_size || !p->slo_us || !p->batch_timeout_us)
    return PROTEAN_EINVAL;
  for (int i = 0; i < 5 * M; ++i) {
    if (p->solo_us[i] <= 0) return PROTEAN_EINVAL;
    if (p->fbr_ppm[i] < 0 || p->fbr_ppm[i] > 1000000) return PROTEAN_EINVAL;
  }
  // N4c: the GPU's memory (0 = A100-40GB); profile p holds gmem * eighths_p / 8
  const int32_t gmem = p->gpu_mem_mib == 0 ? 40960 : p->gpu_mem_mib;
  if (gmem < 8 || gmem % 8 != 0 || gmem > (1 << 24)) return PROTEAN_EINVAL;
  int32_t cap[5];
  for (int q = 0; q < 5; ++q) cap[q] = gmem / 8 * prof_eighths(q);
  int maxT = 0;
  for (int m = 0; m < M; ++m) {
    if (p->mem_mib[m] < 1 || p->mem_mib[m] > gmem) return PROTEAN_EINVAL;
    if (p->batch_size[m] < 1 || p->batch_size[m] > 65535) return PROTEAN_EINVAL;
    if (p->slo_us[m] <= 0 || p->batch_timeout_us[m] < 0) return PROTEAN_EINVAL;
    maxT = std::max(maxT, p->batch_timeout_us[m]);
  }
  std::vector<std::vector<uint8_t>> gs;
  {
    int rc = profile_geometries(p, &gs);
    if (rc) return rc;
  }
  protean_handle* h = new protean_handle();
  h->device = p->device;
  h->M = M;
  h->G = (int)gs.size();
  h->maxT = maxT;
  h->tl.init(M, h->G);
  h->words.assign(h->tl.words, 0);
  int32_t* w = h->words.data();
  std::memcpy(w + h->tl.o_solo, p->solo_us, sizeof(int32_t) * 5 * M);
  std::memcpy(w + h->tl.o_fbr, p->fbr_ppm, sizeof(int32_t) * 5 * M);
  std::memcpy(w + h->tl.o_mem, p->mem_mib, sizeof(int32_t) * M);
  std::memcpy(w + h->tl.o_bsz, p->batch_size, sizeof(int32_t) * M);
  std::memcpy(w + h->tl.o_slo, p->slo_us, sizeof(int32_t) * M);
  std::memcpy(w + h->tl.o_tmo, p->batch_timeout_us, sizeof(int32_t) * M);
  uint8_t* gp = reinterpret_cast<uint8_t*>(w + h->tl.o_gprof);
  h->geoms.assign((size_t)h->G * 8, 0xFF);
  for (int j = 0; j < h->G; ++j) {
    int pref = 0;
    for (int s = 0; s < 8; ++s) {
      const uint8_t v = s < (int)gs[j].size() ? gs[j][s] : 0xFF;
      gp[j * 8 + s] = v;
      h->geoms[j * 8 + s] = v;
      if (v != 0xFF) pref += cap[v];
      w[h->tl.o_gpref + j * 8 + s] = pref;  // capacity of slices 0..s (Alg 1 tag walk)
    }
    w[h->tl.o_gn + j] = (int32_t)gs[j].size();
  }
  for (int q = 0; q < 5; ++q) w[h->tl.o_cap + q] = cap[q];
  for (int j = 0; j < h->G; ++j) h->gn.push_back((int)gs[j].size());
  int cw = 0;
  std::vector<uint32_t> pack = build_pack(h->gn, 0, h->G, &cw);
  h->CW = cw;
  cudaError_t e = cudaSetDevice(h->device);
  if (e == cudaSuccess) e = cudaDeviceGetAttribute(&h->nsm, cudaDevAttrMultiProcessorCount, h->device);
  if (e == cudaSuccess) e = cudaMalloc(&h->d_tab, sizeof(int32_t) * h->words.size());
  if (e == cudaSuccess)
    e = cudaMemcpy(h->d_tab, h->words.data(), sizeof(int32_t) * h->words.size(), cudaMemcpyHostToDevice);
  if (e == cudaSuccess) e = cudaMalloc(&h->d_small, 512);
  if (e == cudaSuccess) e = cudaMemset(h->d_small, 0, 512);  // [256, 264): score_epoch's latched verdict
  for (int i = 0; i < 6 && e == cudaSuccess; ++i) e = cudaEventCreate(&h->ev[i]);
  for (int i = 0; i < 4 && e == cudaSuccess; ++i) e = cudaEventCreate(&h->evc[i]);
  if (e == cudaSuccess) {  // cand.cu lane order: geometries by slice count, descending
    std::vector<uint8_t> go(h->G);
    for (int j = 0; j < h->G; ++j) go[j] = (uint8_t)j;
    std::stable_sort(go.begin(), go.end(), [&](uint8_t a, uint8_t b) { return h->gn[a] > h->gn[b]; });
    e = cudaMalloc(&h->d_gorder, h->G);
    if (e == cudaSuccess) e = cudaMemcpy(h->d_gorder, go.data(), h->G, cudaMemcpyHostToDevice);
  }
  if (e == cudaSuccess) e = cudaMalloc(&h->d_pack, pack.size() * 4);
  if (e == cudaSuccess) e = cudaMemcpy(h->d_pack, pack.data(), pack.size() * 4, cudaMemcpyHostToDevice);
  if (e != cudaSuccess) {
    cudaGetLastError();
    protean_free(h);
    return e == cudaErrorMemoryAllocation ? PROTEAN_ENOMEM : PROTEAN_ECUDA;
  }
  *out = h;
  return PROTEAN_OK;
}

void protean_free(protean_handle* h) {
  if (!h) return;
  cudaSetDevice(h->device);
  if (h->d_tab) cudaFree(h->d_tab);
  if (h->d_scratch) cudaFree(h->d_scratch);
  if (h->d_eoff) cudaFree(h->d_eoff);
  for (void* q : {h->d_cnt, h->d_sidx, h->d_sa, h->d_saoff})
    if (q) cudaFree(q);
  if (h->d_small) cudaFree(h->d_small);
  if (h->d_pack) cudaFree(h->d_pack);
  if (h->d_gorder) cudaFree(h->d_gorder);
  if (h->d_cand) cudaFree(h->d_cand);
  for (cudaEvent_t v : h->evc)
    if (v) cudaEventDestroy(v);
  if (h->d_pack_g) cudaFree(h->d_pack_g);
  if (h->d_sc_pack) cudaFree(h->d_sc_pack);
  for (uint32_t* q : h->vr_pack) cudaFree(q);
  if (h->d_vxbuf) cudaFree(h->d_vxbuf);
  if (h->d_vdone) cudaFree(h->d_vdone);
  if (h->d_vpeer) cudaFree(h->d_vpeer);
  xchg_release(h);
  for (int i = 0; i < 6; ++i)
    if (h->ev[i]) cudaEventDestroy(h->ev[i]);
  for (int b = 0; b < 2; ++b) {
    if (h->d_hb[b]) cudaFree(h->d_hb[b]);
    for (int k = 0; k < 3; ++k)
      if (h->hev[k][b]) cudaEventDestroy(h->hev[k][b]);
  }
  if (h->hs_copy) cudaStreamDestroy(h->hs_copy);
  if (h->hs_back) cudaStreamDestroy(h->hs_back);
  {  // the stream-ordered allocations go back to the device pool: return it to the device
    cudaMemPool_t pool;
    if (cudaDeviceGetDefaultMemPool(&pool, h->device) == cudaSuccess) {
      cudaDeviceSynchronize();
      cudaMemPoolTrimTo(pool, 0);
    }
    cudaGetLastError();
  }
  delete h;
}

int protean_geometry_split(const protean_profiles* p, int32_t nranks, int32_t* bounds) {
  if (!bounds) return PROTEAN_EINVAL;
  std::vector<std::vector<uint8_t>> gs;
  int rc = profile_geometries(p, &gs);
  if (rc) return rc;
  if (nranks < 1 || nranks > (int)gs.size()) return PROTEAN_EINVAL;
  std::vector<int> gn;
  for (const auto& g : gs) gn.push_back((int)g.size());
  split_ranges(gn, nranks, bounds);
  return PROTEAN_OK;
}

int protean_xchg_export(protean_handle* h, int32_t nranks, int32_t rank, int32_t max_replicas,
                        int32_t max_gpus, void* ipc_handle) {
  if (!h) return PROTEAN_EINVAL;
  if (h->poisoned) return PROTEAN_ESTATE;
  if (!ipc_handle) return fail(h, PROTEAN_EINVAL, "null ipc_handle");
  int rc = xchg_alloc(h, nranks, rank, max_replicas, max_gpus);
  if (rc) return rc;
  cudaIpcMemHandle_t ih;
  CK(h, cudaIpcGetMemHandle(&ih, h->d_xbuf));
  static_assert(sizeof(cudaIpcMemHandle_t) == 64, "ipc handle size");
  std::memcpy(ipc_handle, &ih, 64);
  return PROTEAN_OK;
}

int protean_xchg_import(protean_handle* h, const void* ipc_handles) {
  if (!h) return PROTEAN_EINVAL;
  if (h->poisoned) return PROTEAN_ESTATE;
  if (!ipc_handles) return fail(h, PROTEAN_EINVAL, "null ipc_handles");
  if (!h->d_xbuf || h->x_ready) return fail(h, PROTEAN_ESTATE, "import needs a fresh export");
  CK(h, cudaSetDevice(h->device));
  for (int k = 0; k < h->xl.n; ++k) {
    if (k == h->xrank) continue;
    cudaIpcMemHandle_t ih;
    std::memcpy(&ih, static_cast<const char*>(ipc_handles) + 64 * k, 64);
    void* ptr = nullptr;
    CK(h, cudaIpcOpenMemHandle(&ptr, ih, cudaIpcMemLazyEnablePeerAccess));
    h->xpeer[k] = static_cast<char*>(ptr);
    h->x_opened[k] = 1;
  }
  return xchg_finish(h);
}

int protean_xchg_attach(protean_handle* const* hs, int32_t nranks, int32_t max_replicas,
                        int32_t max_gpus) {
  if (!hs || nranks < 2 || nranks > 64) return PROTEAN_EINVAL;
  for (int k = 0; k < nranks; ++k) {
    if (!hs[k]) return PROTEAN_EINVAL;
    if (hs[k]->poisoned) return PROTEAN_ESTATE;
    for (int q = 0; q < k; ++q)
      if (hs[q] == hs[k]) return fail(hs[k], PROTEAN_EINVAL, "one handle per rank");
  }
  for (int k = 0; k < nranks; ++k) {
    int rc = xchg_alloc(hs[k], nranks, k, max_replicas, max_gpus);
    if (rc) return rc;
  }
  for (int k = 0; k < nranks; ++k) {  // peer access between distinct devices
    for (int q = 0; q < nranks; ++q) {
      if (hs[q]->device == hs[k]->device) continue;
      CK(hs[k], cudaSetDevice(hs[k]->device));
      cudaError_t e = cudaDeviceEnablePeerAccess(hs[q]->device, 0);
      if (e != cudaSuccess && e != cudaErrorPeerAccessAlreadyEnabled) return cuda_fail(hs[k], e, "peer access");
      cudaGetLastError();
    }
    for (int q = 0; q < nranks; ++q) hs[k]->xpeer[q] = static_cast<char*>(hs[q]->d_xbuf);
  }
  for (int k = 0; k < nranks; ++k) {
    int rc = xchg_finish(hs[k]);
    if (rc) return rc;
  }
  return PROTEAN_OK;
}

int protean_last_timings(const protean_handle* h, float* prepass_ms, float* replay_ms,
                          int32_t* launch) {
  if (!h) return PROTEAN_EINVAL;
  if (prepass_ms) *prepass_ms = h->t_prepass;
  if (replay_ms) *replay_ms = h->t_replay;
  if (launch) {
    launch[0] = h->last_grid;
    launch[1] = h->last_block;
    launch[2] = h->last_smem;
    launch[3] = h->last_per_sm;
  }
  return PROTEAN_OK;
}

int protean_last_search_ms(const protean_handle* h, float* search_ms, float* walk_ms, float* acct_ms) {
  if (!h || !search_ms) return PROTEAN_EINVAL;
  *search_ms = h->t_search;
  if (walk_ms) *walk_ms = h->t_walk;
  if (acct_ms) *acct_ms = h->t_acct;
  return PROTEAN_OK;
}

int protean_get_geometries(const protean_handle* h, int32_t* n, uint8_t* geoms) {
  if (!h || !n) return PROTEAN_EINVAL;
  *n = h->G;
  if (geoms) std::memcpy(geoms, h->geoms.data(), h->geoms.size());
  return PROTEAN_OK;
}

int protean_num_epochs(const protean_handle* h, int64_t trace_len, int64_t W, int64_t* E) {
  if (!h || !E || W <= 0 || trace_len <= 0) return PROTEAN_EINVAL;
  *E = (trace_len + W - 1) / W + ((int64_t)h->maxT + W - 1) / W;
  return PROTEAN_OK;
}

int protean_replay_traces(protean_handle* h, const protean_replay_cfg* cfg, protean_replay_out* out,
                          void* stream) {
  if (!h) return PROTEAN_EINVAL;
  if (h->poisoned) return PROTEAN_ESTATE;
  if (!cfg || !out) return fail(h, PROTEAN_EINVAL, "null cfg/out");
  const protean_replay_cfg& c = *cfg;
  if (c.n_replicas < 1) return fail(h, PROTEAN_EINVAL, "n_replicas < 1");
  if (c.n_gpus < 1) return fail(h, PROTEAN_EINVAL, "n_gpus < 1");
  if (c.n_gpus > 255) return fail(h, PROTEAN_ERANGE, "n_gpus > 255");
  if (c.epoch_len_us <= 0 || c.trace_len_us <= 0) return fail(h, PROTEAN_EINVAL, "W / trace_len");
  if (c.trace_len_us - 1 + h->maxT > (int64_t)0xFFFFFFFFLL)
    return fail(h, PROTEAN_ERANGE, "ready times exceed uint32 us");
  if (c.policy < 0 || c.policy > 2) return fail(h, PROTEAN_EINVAL, "policy");
  int g421 = -1, g43 = -1;  // Alg 2's two outcomes (R15): (4g,2g,1g) and (4g,3g) in the loaded set
  if (c.policy == 2) {
    if (c.ewma_alpha_pm < 1 || c.ewma_alpha_pm > 1000) return fail(h, PROTEAN_EINVAL, "ewma_alpha_pm");
    if (c.t_low_milli < 0 || c.t_high_milli < c.t_low_milli) return fail(h, PROTEAN_EINVAL, "t_low / t_high");
    for (int j = 0; j < h->G; ++j) {
      const uint8_t* row = &h->geoms[(size_t)j * 8];
      if (g421 < 0 && row[0] == 0 && row[1] == 1 && row[2] == 3 && row[3] == 0xFF) g421 = j;
      if (g43 < 0 && row[0] == 2 && row[1] == 3 && row[2] == 0xFF) g43 = j;
    }
    if (g421 < 0 || g43 < 0) return fail(h, PROTEAN_EINVAL, "policy 2 needs (4g,2g,1g) and (4g,3g) in the set");
  }
  if (c.shard_mode != 0 && c.shard_mode != 1) return fail(h, PROTEAN_EINVAL, "shard_mode");
  if (c.cold_start_us < 0 || c.keepalive_epochs < 1 || c.prewarm < 0 || c.prewarm > kPoolCap)
    return fail(h, PROTEAN_EINVAL, "cold_start_us / keepalive_epochs / prewarm");
  if (c.ctas_per_replica < 0 || c.reserved2 != 0) return fail(h, PROTEAN_EINVAL, "ctas_per_replica / reserved2");
  if (c.max_ctas < 0) return fail(h, PROTEAN_EINVAL, "max_ctas");
  const bool modeG = c.shard_mode == 1;
  if (modeG) {
    if (!h->x_ready) return fail(h, PROTEAN_ESTATE, "mode G without an exchange set-up");
    if (c.nranks != h->xl.n || c.rank != h->xrank) return fail(h, PROTEAN_EINVAL, "rank/nranks vs exchange");
    if (c.n_replicas > h->xl.Rcap || c.n_gpus > h->xl.Ncap)
      return fail(h, PROTEAN_ERANGE, "replicas/gpus exceed the exchange capacity");
  }
  if (c.wait_limit < 0 || c.wait_limit > 255) return fail(h, PROTEAN_EINVAL, "wait_limit");
  if (c.reconfig_cap_pct < 0 || c.reconfig_cap_pct > 100) return fail(h, PROTEAN_EINVAL, "cap pct");
  if (c.init_geom < 0 || c.init_geom >= h->G) return fail(h, PROTEAN_EINVAL, "init_geom");
  if (c.max_live < 1 || c.max_live > PROTEAN_MAX_LIVE) return fail(h, PROTEAN_EINVAL, "max_live");
  if (c.vm_policy < 0 || c.vm_policy > 2) return fail(h, PROTEAN_EINVAL, "vm_policy");
  if (c.reconfig_us < 0) return fail(h, PROTEAN_EINVAL, "reconfig_us");
  if (!(c.price_od_node_hr >= 0) || !(c.price_spot_node_hr >= 0)) return fail(h, PROTEAN_EINVAL, "price");
  if (c.vm_policy != 0) {
    if (!(c.p_rev >= 0 && c.p_rev <= 1)) return fail(h, PROTEAN_EINVAL, "p_rev");
    if (c.rev_interval_us < c.epoch_len_us) return fail(h, PROTEAN_EINVAL, "rev_interval < W");
    if (c.notice_us < 0 || c.notice_us >= c.rev_interval_us) return fail(h, PROTEAN_EINVAL, "notice");
  }
  if (!c.arrival_us || !c.meta || !c.replica_off) return fail(h, PROTEAN_EINVAL, "null trace");
  if (!out->counters || !out->accum || !out->hist || !out->p50_p99_us || !out->cost_usd || !out->util)
    return fail(h, PROTEAN_EINVAL, "null output");
  cudaStream_t st = reinterpret_cast<cudaStream_t>(stream);
  CK(h, cudaSetDevice(h->device));
  const int R = c.n_replicas, N = c.n_gpus;
  const int64_t W = c.epoch_len_us;
  const int64_t E = (c.trace_len_us + W - 1) / W + ((int64_t)h->maxT + W - 1) / W;
  const int64_t H = E * W;

  // the trace-level stream partition: prepass, P1 count + validate, P2 runs, P3 stable scatter
  const int kWarps = PROTEAN_WARPS;  // replay CTA warps (replay.cuh)
  const int S = 2 * h->M;
  unsigned long long wmax = 0;
  int* d_err = reinterpret_cast<int*>(static_cast<char*>(h->d_small) + 64);
  {
    int rc = partition_trace(h, c, E, st, true, &wmax);
    if (rc) return rc;
  }
  int herr = 0;
  // window capacity: the largest window (requests in [eW - maxT, (e+1)W)) + per-stream alignment
  const int WCAP = (int)std::max<unsigned long long>(wmax, 1) + 8 * S;

  // candidate range: all geometries, or this rank's slot-balanced range (mode G)
  int geom_lo = 0, geom_hi = h->G;
  const uint32_t* d_pack = h->d_pack;
  int CW = h->CW;
  if (modeG) {
    std::vector<int32_t> b(h->xl.n + 1);
    split_ranges(h->gn, h->xl.n, b.data());
    geom_lo = b[h->xrank];
    geom_hi = b[h->xrank + 1];
    if (h->pack_lo != geom_lo || h->pack_hi != geom_hi) return fail(h, PROTEAN_ESTATE, "range packing");
    d_pack = h->d_pack_g;
    CW = h->CW_g;
  }
  // virtual ranks: with fewer replicas than SMs, several CTAs share one replica, each scoring a
  // slot-balanced geometry range and exchanging min-loc keys per epoch in device memory (the
  // mode G exchange inside one launch); auto = min(16, G, SMs / R)
  int vr_n = 1;
  // PROTEAN_LEAN=2 (test knob): the lean chain whenever it can hold the call (no virtual ranks,
  // no few-replica instance), so small parity cases exercise it
  const char* lean_env = std::getenv("PROTEAN_LEAN");
  const bool lean_force = lean_env && std::atoi(lean_env) == 2;
  if (!modeG && c.policy == 0 && h->G >= 2 && c.ctas_per_replica != 1 && !lean_force) {
    vr_n = c.ctas_per_replica > 1 ? c.ctas_per_replica : (R < h->nsm ? h->nsm / R : 1);
    vr_n = std::min(vr_n, std::min(kMaxVR, h->G));
    if (vr_n < 2) vr_n = 1;
  }
  if (vr_n > 1 && vr_n != h->vr_n) {  // per-range candidate packing (cached per split)
    for (uint32_t* q : h->vr_pack) cudaFree(q);
    h->vr_pack.assign(vr_n, nullptr);
    h->vr_b.assign(vr_n + 1, 0);
    h->vr_cw.assign(vr_n, 0);
    split_ranges(h->gn, vr_n, h->vr_b.data());
    for (int k = 0; k < vr_n; ++k) {
      std::vector<uint32_t> pk = build_pack(h->gn, h->vr_b[k], h->vr_b[k + 1], &h->vr_cw[k]);
      CK(h, cudaMalloc(&h->vr_pack[k], pk.size() * 4));
      CK(h, cudaMemcpy(h->vr_pack[k], pk.data(), pk.size() * 4, cudaMemcpyHostToDevice));
    }
    h->vr_n = vr_n;
  }
  if (vr_n > 1) {  // the layout holds the largest range of any virtual rank
    geom_lo = 0;
    geom_hi = 0;
    CW = 0;
    for (int k = 0; k < vr_n; ++k) {
      geom_hi = std::max(geom_hi, h->vr_b[k + 1] - h->vr_b[k]);
      CW = std::max(CW, h->vr_cw[k]);
    }
  }
  // launch geometry: 8 warps; units = actual-placement warps + candidate warps per GPU
  const int Gc = geom_hi - geom_lo;
  // warps per CTA: the placement phase runs n_units warp units; pick 4..8 warps that divide them
  // most evenly (prefer more warps on ties)
  const int n_units = (N + kAG - 1) / kAG + (c.policy == 0 ? N * CW : 0);
  (void)n_units;
  // measured on B200: 8 warps x 3 CTAs/SM beat 6 x 4 for many replicas; with fewer replicas than
  // SMs one 16-warp CTA per SM runs a replica's actual and candidate chains side by side
  bool few_r = (int64_t)R < (int64_t)h->nsm;
  if (const char* ev = std::getenv("PROTEAN_FEW"))  // experiment knob: force the instance family
    few_r = std::atoi(ev) != 0;
  const int block = 32 * (few_r ? PROTEAN_FEW_WARPS : kWarps);
  // the candidate search as a data-parallel pass ahead of the chain (cand.cu): mode R, policy 0,
  // one CTA per replica, the one-warp decision path (N <= 32)
  // (policy 2 runs the search pass for its batch rows only, and only to feed the lean chain)
  bool precand = (c.policy == 0 || c.policy == 2) && !modeG && vr_n == 1 && N <= 32;
  const bool keys = c.policy == 0;
  if (const char* ev = std::getenv("PROTEAN_PRECAND"))  // experiment knob: 0 = in-chain candidates only
    if (std::atoi(ev) == 0) precand = false;
  const int KS = precand && keys ? N * h->G : 0;
  SmemLayout sl;
  sl.init(h->tl.words, h->M, N, Gc, CW, 0, 0, KS);
  const size_t fixed = sl.total;
  int BS = std::min(WCAP, 64);
  size_t budget = 72 * 1024;
  if (const char* ev = std::getenv("PROTEAN_SMEM_BUDGET_KB")) {  // test knob: force spill paths
    budget = (size_t)std::atoi(ev) * 1024;
    BS = std::min(BS, std::max(1, std::atoi(ev)));
  }
  const size_t with_bats = fixed + (size_t)BS * (sizeof(Bat) + 8) + 64;
  int WS = (with_bats + (size_t)WCAP * 4 <= budget) ? WCAP : 0;  // window all in smem or all in HBM
  if (const char* ev = std::getenv("PROTEAN_WINDOW_SMEM"))  // experiment knob: 0 = window in global scratch
    if (std::atoi(ev) == 0) WS = 0;
  sl.init(h->tl.words, h->M, N, Gc, CW, BS, WS, KS);
  if (sl.total > 227 * 1024) return fail(h, PROTEAN_ERANGE, "shared memory layout too large");
  int per_sm = 0;
  CK(h, replay_occupancy(block, sl.total, few_r, &per_sm));
  if (per_sm < 1) return fail(h, PROTEAN_ERANGE, "replay kernel does not fit an SM");
  if (const char* ev = std::getenv("PROTEAN_PER_SM"))  // experiment knob: fewer resident CTAs per SM
    per_sm = std::max(1, std::min(per_sm, std::atoi(ev)));
  int grid = (int)std::min<int64_t>((int64_t)R * vr_n, (int64_t)h->nsm * per_sm);
  grid -= grid % vr_n;  // every replica's CTAs are resident together (exchange partners)
  if (c.max_ctas > 0) grid = std::min(grid, std::max(c.max_ctas, vr_n) / vr_n * vr_n);

  ReplayParams P;
  std::memset(&P, 0, sizeof(P));
  P.tab = h->d_tab;
  P.tl = h->tl;
  P.pack = d_pack;
  P.maxT = h->maxT;
  P.sa = static_cast<const uint32_t*>(h->d_sa);
  P.saoff = static_cast<const int64_t*>(h->d_saoff);
  P.sidx = static_cast<const uint32_t*>(h->d_sidx);
  P.R = R;
  P.N = N;
  P.base = c.replica_base;
  P.trace_len = c.trace_len_us;
  P.W = W;
  P.E = E;
  P.H = H;
  P.policy = c.policy;
  P.cold_us = c.cold_start_us;
  P.keepalive = c.keepalive_epochs;
  P.prewarm = c.prewarm;
  P.cold_starts = out->cold_starts;
  P.ewma_a = c.ewma_alpha_pm;
  P.t_low = c.t_low_milli;
  P.t_high = c.t_high_milli;
  P.g421 = g421;
  P.g43 = g43;
  P.wait_limit = c.wait_limit;
  P.cap_pct = c.reconfig_cap_pct;
  P.init_geom = c.init_geom;
  P.max_live = c.max_live;
  P.vm_policy = c.vm_policy;
  P.reconfig_us = c.reconfig_us;
  P.rev = c.vm_policy ? c.rev_interval_us : 1;
  P.notice = c.notice_us;
  P.thr = (uint64_t)(c.p_rev * 9007199254740992.0);
  P.seed = c.seed;
  P.price_od = c.price_od_node_hr;
  P.price_spot = c.price_spot_node_hr;
  P.geom_lo = vr_n > 1 ? 0 : geom_lo;
  P.geom_hi = vr_n > 1 ? h->G : geom_hi;
  P.vr_n = vr_n;
  P.few = few_r;
  if (vr_n > 1) {
    for (int k = 0; k < vr_n; ++k) {
      P.vr_lo[k] = h->vr_b[k];
      P.vr_hi[k] = h->vr_b[k + 1];
      P.vr_cw[k] = h->vr_cw[k];
      P.vr_pack[k] = h->vr_pack[k];
    }
    const XLayout X{vr_n, R, N};
    const size_t stride = al(X.bytes());  // 16-byte key pairs: every rank's buffer 256-aligned
    const size_t need = stride * (size_t)vr_n;
    if (h->vxl.n != X.n || h->vxl.Rcap != X.Rcap || h->vxl.Ncap != X.Ncap || h->vx_bytes < need) {
      int rc = ensure(h, &h->d_vxbuf, &h->vx_bytes, need, st);
      if (rc) return rc;
      CK(h, cudaMemsetAsync(h->d_vxbuf, 0, need, st));  // flags restart with the sequence
      std::vector<char*> peers(vr_n);
      for (int k = 0; k < vr_n; ++k) peers[k] = static_cast<char*>(h->d_vxbuf) + stride * k;
      void* dp = h->d_vpeer;
      size_t have = h->d_vpeer ? sizeof(char*) * kMaxVR : 0;
      rc = ensure(h, &dp, &have, sizeof(char*) * kMaxVR, st);
      if (rc) return rc;
      h->d_vpeer = static_cast<char**>(dp);
      CK(h, cudaMemcpyAsync(h->d_vpeer, peers.data(), sizeof(char*) * vr_n, cudaMemcpyHostToDevice, st));
      CK(h, cudaStreamSynchronize(st));  // peers lives on this stack frame
      h->vxl = X;
      h->vseq = 0;
    }
    P.xl = X;
    P.xpeer = h->d_vpeer;
    P.xrank = 0;
    P.xseq = h->vseq;
    P.xtimeout_ns = 30ull * 1000000000ull;
    if (const char* ev = std::getenv("PROTEAN_XCHG_TIMEOUT_S"))
      P.xtimeout_ns = (uint64_t)std::max(1, std::atoi(ev)) * 1000000000ull;
    // the CTAs of a replica split the accounting: counters, histogram and finalize's arrival
    // counter accumulate
    CK(h, cudaMemsetAsync(out->counters, 0, sizeof(int64_t) * 10 * (size_t)R, st));
    CK(h, cudaMemsetAsync(out->hist, 0, sizeof(uint32_t) * 2 * PROTEAN_NBUCKETS * (size_t)R, st));
    {
      int rc = ensure(h, &h->d_vdone, &h->vdone_bytes, sizeof(uint32_t) * (size_t)R, st);
      if (rc) return rc;
    }
    CK(h, cudaMemsetAsync(h->d_vdone, 0, sizeof(uint32_t) * (size_t)R, st));
    P.vr_done = static_cast<uint32_t*>(h->d_vdone);
  }
  if (modeG && !std::getenv("PROTEAN_XCHG_OFF")) {  // debug knob: score the range, no exchange
    P.xl = h->xl;
    P.xpeer = h->d_xpeer;
    P.xrank = h->xrank;
    P.xseq = h->xseq;
    P.xtimeout_ns = 30ull * 1000000000ull;
    if (const char* ev = std::getenv("PROTEAN_XCHG_TIMEOUT_S"))
      P.xtimeout_ns = (uint64_t)std::max(1, std::atoi(ev)) * 1000000000ull;
  }
  P.counters = out->counters;
  P.accum = out->accum;
  P.hist = out->hist;
  P.pct = out->p50_p99_us;
  P.cost = out->cost_usd;
  P.util = out->util;
  P.decisions = out->decisions;
  P.cand_keys = out->cand_keys;
  P.log = out->batch_log;
  P.log_cap = out->batch_log ? out->batch_log_cap : 0;
  P.n_batches = out->n_batches;
  P.sl = sl;
  P.WCAP = WCAP;
  size_t o = 0;
  P.o_alist = o; o += al((size_t)N * kZA * (few_r ? 4 : 1) * c.max_live * 20);  // x4: sub-lanes (few)
  P.o_clist = o; o += al((size_t)block * c.max_live * 20);
  P.o_gbat = o; o += al((size_t)WCAP * sizeof(Bat));
  P.o_gord = o; o += al((size_t)WCAP * 4);
  P.o_gglist = o; o += al((size_t)WCAP * 4);
  P.o_gsarr = o; o += al((size_t)(WS > 0 ? 0 : WCAP) * 4);
  P.o_pool = o;  // N3 pools: busy-until [N][M][kPoolCap] int64, size + counter [N][M] int32
  if (c.cold_start_us > 0) o += al((size_t)N * h->M * (kPoolCap * 8 + 8));
  P.slot_bytes = al(o);
  {
    int rc = ensure(h, &h->d_scratch, &h->scratch_bytes, P.slot_bytes * (size_t)grid, st);
    if (rc) return rc;
  }
  P.scratch = static_cast<char*>(h->d_scratch);
  P.err = d_err;
  h->t_search = 0.f;
  h->t_acct = 0.f;
  // the lean chain (chain.cu): a warp per replica on cand.cu's batch rows and keys, accounting in
  // its own pass; many-replica calls, container pools (N3) included (an epoch with more than 64
  // batches sends the call back to the fused engine below)
  bool lean = precand && (!few_r || lean_force) && (N * h->G) % 2 == 0 &&
              c.max_live <= 64;  // the chain's resident slots: 64-bit masks
  if (lean_env && std::atoi(lean_env) == 0) lean = false;  // experiment knob: 0 = the fused engine
  if (!keys && !lean) precand = false;  // Alg 2 on the fused engine forms its own batches
  size_t b_ub = 0, b_br = 0;
  if (precand) {
    const size_t b_bs = al((size_t)R * S * (E + 1) * 4), b_kf = keys ? al((size_t)R * E * N * h->G * 8) : 0;
    if (lean) {
      b_ub = al((size_t)R * E * sizeof(UnitBats));
      b_br = al((size_t)R * E * kUnitBats * 8);
    }
    int rc = ensure(h, &h->d_cand, &h->cand_bytes, b_bs + b_kf + b_ub + b_br, st);
    if (rc == PROTEAN_ENOMEM && lean && keys) {  // without the lean chain's rows: the search alone
      lean = false;
      b_ub = b_br = 0;
      rc = ensure(h, &h->d_cand, &h->cand_bytes, b_bs + b_kf, st);
    }
    if (rc == PROTEAN_ENOMEM) {  // no room for the search either: the fused engine scores in-chain
      precand = lean = false;
      h->err.clear();
    } else if (rc) {
      return rc;
    }
  }
  if (precand) {
    const size_t b_bs = al((size_t)R * S * (E + 1) * 4), b_kf = keys ? al((size_t)R * E * N * h->G * 8) : 0;
    CandParams Q;
    std::memset(&Q, 0, sizeof(Q));
    Q.tab = h->d_tab;
    Q.tl = h->tl;
    Q.sa = P.sa;
    Q.saoff = P.saoff;
    Q.sidx = P.sidx;
    Q.bstart = static_cast<uint32_t*>(h->d_cand);
    Q.kfc = keys ? reinterpret_cast<int64_t*>(static_cast<char*>(h->d_cand) + b_bs) : nullptr;
    Q.gorder = h->d_gorder;
    if (lean) {
      Q.ub = reinterpret_cast<UnitBats*>(static_cast<char*>(h->d_cand) + b_bs + b_kf);
      Q.overflow = d_err + 3;
      P.ub = Q.ub;
      P.bres = reinterpret_cast<int64_t*>(static_cast<char*>(h->d_cand) + b_bs + b_kf + b_ub);
      P.ovf = d_err + 3;
    }
    Q.R = R;
    Q.S = S;
    Q.N = N;
    Q.max_live = c.max_live;
    Q.E = E;
    Q.W = W;
    size_t ws_off = 0;
    cand_smem_bytes(h->tl, &ws_off);
    Q.ws_off = ws_off;
    int cper = 0;
    CK(h, cand_occupancy(h->tl, &cper));
    if (cper < 1) return fail(h, PROTEAN_ERANGE, "candidate kernel does not fit an SM");
    CK(h, cudaEventRecord(h->evc[0], st));
    CK(h, launch_walk(Q, st));
    CK(h, cudaEventRecord(h->evc[2], st));
    CK(h, launch_cand(Q, h->nsm * cper, st));
    CK(h, cudaEventRecord(h->evc[1], st));
    P.kfc = Q.kfc;
  }
  ReplayParams PL = P;
  int cper = 0, cgrid_l = 0;
  if (lean) {
    PL.cl.init(N, N * h->G, h->G, h->M);
    const size_t sl_a = al((size_t)64 * 32 * 16), sl_c = al((size_t)kUnitBats * 32 * 16 + 2 * kMaxSl * 32 * 4);
    PL.o_alist = 0;
    PL.o_clist = sl_a;
    PL.o_pool = sl_a + sl_c;  // N3 pools: busy-until [N][M][kPoolCap] int64, size + counter [N][M] int32
    PL.slot_bytes = sl_a + sl_c + (c.cold_start_us > 0 ? al((size_t)N * h->M * (kPoolCap * 8 + 8)) : 0);
    CK(h, chain_occupancy(PL, &cper));
    if (cper < 1) return fail(h, PROTEAN_ERANGE, "chain kernel does not fit an SM");
    const int cgrid = (int)std::min<int64_t>((int64_t)h->nsm * cper, ((int64_t)R + 3) / 4);
    cgrid_l = cgrid;
    int rc = ensure(h, &h->d_scratch, &h->scratch_bytes,
                    std::max(PL.slot_bytes * (size_t)cgrid * 4, P.slot_bytes * (size_t)grid), st);
    if (rc == PROTEAN_ENOMEM) {  // the fused engine's scratch is smaller: replay there
      h->err.clear();
      rc = ensure(h, &h->d_scratch, &h->scratch_bytes, P.slot_bytes * (size_t)grid, st);
      if (rc) return rc;
      lean = false;
    } else if (rc) {
      return rc;
    }
    P.scratch = PL.scratch = static_cast<char*>(h->d_scratch);
  }
  if (lean) {
    const int cgrid = cgrid_l;
    CK(h, cudaEventRecord(h->ev[2], st));
    CK(h, launch_chain(PL, cgrid, st));
    CK(h, cudaEventRecord(h->ev[3], st));
    CK(h, launch_acct(PL, st));
    CK(h, cudaEventRecord(h->evc[3], st));
    int herr3[4] = {0, 0, 0, 0};
    CK(h, cudaMemcpyAsync(herr3, d_err, 16, cudaMemcpyDeviceToHost, st));
    CK(h, cudaStreamSynchronize(st));
    if (!herr3[3]) {  // every epoch fitted the chain's batch rows
      if (herr3[2]) return fail(h, PROTEAN_ERANGE, "a container pool outgrew 128 containers (N3)");
      float a = 0.f, b = 0.f;
      CK(h, cudaEventElapsedTime(&a, h->ev[0], h->ev[1]));
      CK(h, cudaEventElapsedTime(&b, h->ev[4], h->ev[5]));
      h->t_prepass = a + b;
      CK(h, cudaEventElapsedTime(&h->t_replay, h->ev[2], h->ev[3]));
      CK(h, cudaEventElapsedTime(&h->t_acct, h->ev[3], h->evc[3]));
      CK(h, cudaEventElapsedTime(&h->t_search, h->evc[0], h->evc[1]));
      CK(h, cudaEventElapsedTime(&h->t_walk, h->evc[0], h->evc[2]));
      h->last_grid = cgrid;
      h->last_block = 32 * 4;
      h->last_smem = (int)chain_smem_bytes(PL);
      h->last_per_sm = cper;
      if (herr3[0]) return fail(h, PROTEAN_EINVAL, "invalid request (unsorted, model id, or arrival >= trace_len)");
      return PROTEAN_OK;
    }
    // some epoch held more than kUnitBats batches: the fused engine replays the call (its keys
    // for the epochs cand.cu held are still valid)
  }
  CK(h, cudaEventRecord(h->ev[2], st));
  CK(h, launch_replay(P, grid, block, st));
  CK(h, cudaEventRecord(h->ev[3], st));
  int herr2[3] = {0, 0, 0};
  CK(h, cudaMemcpyAsync(herr2, d_err, 12, cudaMemcpyDeviceToHost, st));
  CK(h, cudaStreamSynchronize(st));
  herr = herr2[0];
  if (modeG) h->xseq += (uint32_t)E;
  if (vr_n > 1) h->vseq += (uint32_t)E;
  if (herr2[1]) {
    h->poisoned = true;
    return fail(h, PROTEAN_ENCCL, "mode G exchange: a peer rank did not publish within 30 s");
  }
  {
    float a = 0.f, b = 0.f;
    CK(h, cudaEventElapsedTime(&a, h->ev[0], h->ev[1]));
    CK(h, cudaEventElapsedTime(&b, h->ev[4], h->ev[5]));
    h->t_prepass = a + b;  // device time of the prepass and the three partition passes
  }
  CK(h, cudaEventElapsedTime(&h->t_replay, h->ev[2], h->ev[3]));
  if (precand) {
    CK(h, cudaEventElapsedTime(&h->t_search, h->evc[0], h->evc[1]));
    CK(h, cudaEventElapsedTime(&h->t_walk, h->evc[0], h->evc[2]));
  }
  h->last_grid = grid;
  h->last_block = block;
  h->last_smem = (int)sl.total;
  h->last_per_sm = per_sm;
  if (herr) return fail(h, PROTEAN_EINVAL, "invalid request (unsorted, model id, or arrival >= trace_len)");
  if (herr2[2]) return fail(h, PROTEAN_ERANGE, "a container pool outgrew 128 containers (N3)");
  return PROTEAN_OK;
}

int protean_score_epoch(protean_handle* h, const protean_epoch_in* in, protean_epoch_out* out,
                        void* stream) {
  if (!h) return PROTEAN_EINVAL;
  if (h->poisoned) return PROTEAN_ESTATE;
  if (!in || !out) return fail(h, PROTEAN_EINVAL, "null in/out");
  if (in->n_replicas < 1 || in->n_gpus < 1 || in->epoch < 0 || in->epoch_len_us <= 0 || in->horizon_us < 0)
    return fail(h, PROTEAN_EINVAL, "sizes");
  if (in->n_gpus > 255) return fail(h, PROTEAN_ERANGE, "n_gpus > 255");
  if (in->max_live < 1 || in->max_live > PROTEAN_MAX_LIVE) return fail(h, PROTEAN_EINVAL, "max_live");
  if (in->geom_lo < 0 || in->geom_hi > h->G || in->geom_lo >= in->geom_hi)
    return fail(h, PROTEAN_EINVAL, "geometry range");
  if (!in->batch_off || !in->state || !out->best_key || !out->counters || !out->placement)
    return fail(h, PROTEAN_EINVAL, "null pointer");
  if (!(in->price_od_node_hr >= 0) || !(in->price_spot_node_hr >= 0)) return fail(h, PROTEAN_EINVAL, "price");
  cudaStream_t st = reinterpret_cast<cudaStream_t>(stream);
  CK(h, cudaSetDevice(h->device));
  const int R = in->n_replicas, N = in->n_gpus;
  // enqueue-only: batch_off[0], the states and the batches are validated in the kernel, whose
  // verdict is latched in the handle's device word (protean_score_epoch_status)
  const int block = 256;  // 8 warps: one per actual unit / candidate warp of the lane packing
  const size_t lb = score_list_bytes(N, block, in->max_live);
  {
    int rc = ensure(h, &h->d_scratch, &h->scratch_bytes, std::max<size_t>(lb * (size_t)R, 256), st);
    if (rc) return rc;
  }
  if (h->sc_lo != in->geom_lo || h->sc_hi != in->geom_hi) {  // lane packing of the range (cached)
    std::vector<uint32_t> pk = build_pack(h->gn, in->geom_lo, in->geom_hi, &h->sc_cw);
    if (h->d_sc_pack) cudaFree(h->d_sc_pack);
    h->d_sc_pack = nullptr;
    CK(h, cudaMalloc(&h->d_sc_pack, pk.size() * 4));
    CK(h, cudaMemcpy(h->d_sc_pack, pk.data(), pk.size() * 4, cudaMemcpyHostToDevice));
    h->sc_lo = in->geom_lo;
    h->sc_hi = in->geom_hi;
  }
  int* d_err = reinterpret_cast<int*>(static_cast<char*>(h->d_small) + 256);
  ScoreParams P;
  std::memset(&P, 0, sizeof(P));
  P.tab = h->d_tab;
  P.tl = h->tl;
  P.R = R;
  P.N = N;
  P.epoch = in->epoch;
  P.max_live = in->max_live;
  P.geom_lo = in->geom_lo;
  P.geom_hi = in->geom_hi;
  P.W = in->epoch_len_us;
  P.H = in->horizon_us;
  P.batches = in->batches;
  P.batch_off = in->batch_off;
  P.arrival = in->arrival_us;
  P.state = in->state;
  P.best_key = out->best_key;
  P.cand_key = out->cand_key;
  P.placement = out->placement;
  P.counters = out->counters;
  P.accum = out->accum;
  P.cost = out->cost_usd;
  P.price_od = in->price_od_node_hr;
  P.price_spot = in->price_spot_node_hr;
  P.pack = h->d_sc_pack;
  P.cw = h->sc_cw;
  P.lists = h->d_scratch;
  P.list_bytes = lb;
  P.err = d_err;
  CK(h, launch_score(P, block, st));
  return PROTEAN_OK;
}

int protean_score_epoch_status(protean_handle* h) {
  if (!h) return PROTEAN_EINVAL;
  if (h->poisoned) return PROTEAN_ESTATE;
  CK(h, cudaSetDevice(h->device));
  CK(h, cudaDeviceSynchronize());
  int errs[2] = {0, 0};
  int* d_err = reinterpret_cast<int*>(static_cast<char*>(h->d_small) + 256);
  CK(h, cudaMemcpy(errs, d_err, 8, cudaMemcpyDeviceToHost));
  CK(h, cudaMemset(d_err, 0, 8));
  if (errs[0]) return fail(h, PROTEAN_EINVAL, "score_epoch: invalid state / batch / batch_off");
  if (errs[1]) return fail(h, PROTEAN_ERANGE, "score_epoch: n_live > max_live");
  return PROTEAN_OK;
}


int protean_sweep_assignments(protean_handle* h, const protean_sweep_in* in, protean_sweep_out* out,
                              void* stream) {
  if (!h) return PROTEAN_EINVAL;
  if (h->poisoned) return PROTEAN_ESTATE;
  if (!in || !out) return fail(h, PROTEAN_EINVAL, "null in/out");
  if (in->n_replicas < 1 || in->n_gpus < 1) return fail(h, PROTEAN_EINVAL, "sizes");
  if (in->n_gpus > 255) return fail(h, PROTEAN_ERANGE, "n_gpus > 255");
  if (in->max_live < 1 || in->max_live > PROTEAN_MAX_LIVE) return fail(h, PROTEAN_EINVAL, "max_live");
  if (in->max_batches < 1 || in->max_batches > 8) return fail(h, PROTEAN_EINVAL, "max_batches");
  if (in->geom_lo < 0 || in->geom_hi > h->G || in->geom_lo >= in->geom_hi)
    return fail(h, PROTEAN_EINVAL, "geometry range");
  if (!in->batch_off || !in->cur_geom || !out->best_key || !out->n_assign)
    return fail(h, PROTEAN_EINVAL, "null pointer");
  cudaStream_t st = reinterpret_cast<cudaStream_t>(stream);
  CK(h, cudaSetDevice(h->device));
  int32_t b0 = 0;
  CK(h, cudaMemcpyAsync(&b0, in->batch_off, 4, cudaMemcpyDeviceToHost, st));
  CK(h, cudaStreamSynchronize(st));
  if (b0 != 0) return fail(h, PROTEAN_EINVAL, "batch_off[0] != 0");
  int* d_err = reinterpret_cast<int*>(static_cast<char*>(h->d_small) + 64);
  CK(h, cudaMemsetAsync(d_err, 0, 16, st));
  SweepParams P;
  std::memset(&P, 0, sizeof(P));
  P.tab = h->d_tab;
  P.tl = h->tl;
  P.R = in->n_replicas;
  P.N = in->n_gpus;
  P.max_live = in->max_live;
  P.max_batches = in->max_batches;
  P.geom_lo = in->geom_lo;
  P.geom_hi = in->geom_hi;
  P.batches = in->batches;
  P.batch_off = in->batch_off;
  P.arrival = in->arrival_us;
  P.cur_geom = in->cur_geom;
  P.sweep_key = out->sweep_key;
  P.assign = out->assign;
  P.best_key = out->best_key;
  P.n_assign = out->n_assign;
  P.err = d_err;
  const int64_t units = (int64_t)in->n_replicas * in->n_gpus;
  const int grid = (int)std::min<int64_t>(units, (int64_t)h->nsm * 8);
  CK(h, launch_sweep(P, grid, st));
  int errs[2] = {0, 0};
  CK(h, cudaMemcpyAsync(errs, d_err, 8, cudaMemcpyDeviceToHost, st));
  CK(h, cudaStreamSynchronize(st));
  if (errs[0]) return fail(h, PROTEAN_EINVAL, "invalid batch / offsets / cur_geom");
  if (errs[1]) return fail(h, PROTEAN_ERANGE, "more than max_batches batches on a GPU");
  return PROTEAN_OK;
}

int protean_sweep_depths(protean_handle* h, const protean_sweep_in* in, protean_depth_out* out, void* stream) {
  if (!h) return PROTEAN_EINVAL;
  if (h->poisoned) return PROTEAN_ESTATE;
  if (!in || !out) return fail(h, PROTEAN_EINVAL, "null in/out");
  if (in->n_replicas < 1 || in->n_gpus < 1) return fail(h, PROTEAN_EINVAL, "sizes");
  if (in->n_gpus > 255) return fail(h, PROTEAN_ERANGE, "n_gpus > 255");
  if (in->max_live < 1 || in->max_live > PROTEAN_MAX_LIVE) return fail(h, PROTEAN_EINVAL, "max_live");
  if (in->geom_lo < 0 || in->geom_hi > h->G || in->geom_lo >= in->geom_hi)
    return fail(h, PROTEAN_EINVAL, "geometry range");
  if (!in->batch_off || !in->cur_geom || !out->best_key || !out->n_eval)
    return fail(h, PROTEAN_EINVAL, "null pointer");
  cudaStream_t st = reinterpret_cast<cudaStream_t>(stream);
  CK(h, cudaSetDevice(h->device));
  const int R = in->n_replicas, N = in->n_gpus, nc = in->geom_hi - in->geom_lo;
  const int block = 128;
  const int64_t lanes = (int64_t)R * N * nc * 8;
  const int grid = (int)std::max<int64_t>(1, std::min<int64_t>((lanes + block - 1) / block, (int64_t)h->nsm * 8));
  // scratch: one resident list per thread of the grid, then (if the caller passes no depth_key) the keys
  const size_t lists = al((size_t)grid * block * in->max_live * sizeof(protean_resident));
  const size_t keys = out->depth_key ? 0 : al((size_t)lanes * 8);
  {
    int rc = ensure(h, &h->d_scratch, &h->scratch_bytes, lists + keys, st);
    if (rc) return rc;
  }
  int* d_err = reinterpret_cast<int*>(static_cast<char*>(h->d_small) + 64);
  CK(h, cudaMemsetAsync(d_err, 0, 16, st));
  DepthParams P;
  std::memset(&P, 0, sizeof(P));
  P.tab = h->d_tab;
  P.tl = h->tl;
  P.R = R;
  P.N = N;
  P.max_live = in->max_live;
  P.geom_lo = in->geom_lo;
  P.geom_hi = in->geom_hi;
  P.batches = in->batches;
  P.batch_off = in->batch_off;
  P.arrival = in->arrival_us;
  P.cur_geom = in->cur_geom;
  P.scratch = static_cast<protean_resident*>(h->d_scratch);
  P.depth_key = out->depth_key ? out->depth_key
                               : reinterpret_cast<int64_t*>(static_cast<char*>(h->d_scratch) + lists);
  P.depth_code = out->depth_code;
  P.best_key = out->best_key;
  P.n_eval = out->n_eval;
  int64_t per_x = 0;  // depth codes per (replica, gpu): sum over the range of (slices + 1)
  for (int j = in->geom_lo; j < in->geom_hi; ++j) per_x += h->gn[j] + 1;
  P.n_eval_add = per_x * (int64_t)R * N;
  P.err = d_err;
  CK(h, launch_depths(P, grid, block, st));
  int err0 = 0;
  CK(h, cudaMemcpyAsync(&err0, d_err, 4, cudaMemcpyDeviceToHost, st));
  CK(h, cudaStreamSynchronize(st));
  if (err0) return fail(h, PROTEAN_EINVAL, "invalid batch / offsets / cur_geom");
  return PROTEAN_OK;
}

int protean_form_batches(protean_handle* h, const protean_replay_cfg* cfg, int32_t e_lo, int32_t e_hi,
                         const int64_t* avail_windows, protean_batch* batches, int32_t* batch_off,
                         int64_t* n_batches, uint32_t* members, int64_t members_cap, void* stream) {
  if (!h) return PROTEAN_EINVAL;
  if (h->poisoned) return PROTEAN_ESTATE;
  if (!cfg || !n_batches || !batch_off || !members) return fail(h, PROTEAN_EINVAL, "null pointer");
  const protean_replay_cfg& c = *cfg;
  if (c.n_replicas < 1 || c.n_gpus < 1) return fail(h, PROTEAN_EINVAL, "sizes");
  if (c.n_gpus > 255) return fail(h, PROTEAN_ERANGE, "n_gpus > 255");
  if (c.epoch_len_us <= 0 || c.trace_len_us <= 0) return fail(h, PROTEAN_EINVAL, "W / trace_len");
  if (c.trace_len_us - 1 + h->maxT > (int64_t)0xFFFFFFFFLL)
    return fail(h, PROTEAN_ERANGE, "ready times exceed uint32 us");
  if (!c.arrival_us || !c.meta || !c.replica_off) return fail(h, PROTEAN_EINVAL, "null trace");
  const int64_t W = c.epoch_len_us;
  const int64_t E = (c.trace_len_us + W - 1) / W + ((int64_t)h->maxT + W - 1) / W;
  if (e_lo < 0 || e_hi > E || e_lo > e_hi) return fail(h, PROTEAN_EINVAL, "epoch range");
  cudaStream_t st = reinterpret_cast<cudaStream_t>(stream);
  CK(h, cudaSetDevice(h->device));
  const int R = c.n_replicas, N = c.n_gpus, S = 2 * h->M, Ew = e_hi - e_lo;
  std::vector<int64_t> roff(R + 1);
  CK(h, cudaMemcpyAsync(roff.data(), c.replica_off, sizeof(int64_t) * (R + 1), cudaMemcpyDeviceToHost, st));
  CK(h, cudaStreamSynchronize(st));
  if (roff[0] != 0) return fail(h, PROTEAN_EINVAL, "replica_off[0] != 0");
  for (int r = 0; r < R; ++r)
    if (roff[r + 1] < roff[r]) return fail(h, PROTEAN_EINVAL, "replica_off not monotone");
  // the trace-level stream partition of protean_replay_traces: the stream-sorted copy is the
  // members array
  int64_t sa_len = 0;
  for (int r = 0; r < R; ++r) sa_len += (roff[r + 1] - roff[r] + 3) & ~(int64_t)3;
  if (members_cap < sa_len) return fail(h, PROTEAN_ERANGE, "members capacity < requests + 4 per replica");
  int* d_err = reinterpret_cast<int*>(static_cast<char*>(h->d_small) + 64);
  {
    unsigned long long wmax = 0;
    int rc = partition_trace(h, c, E, st, false, &wmax);
    if (rc) return rc;
  }
  int herr = 0;
  // pass 0: rows per (replica, epoch, GPU) cell
  const size_t cells = (size_t)R * Ew * N;
  void* dc = nullptr;
  size_t dc_have = 0;
  {
    int rc = ensure(h, &dc, &dc_have, std::max<size_t>(4, sizeof(int32_t) * cells), st);
    if (rc) return rc;
  }
  CK(h, cudaMemsetAsync(dc, 0, std::max<size_t>(4, sizeof(int32_t) * cells), st));
  FormParams F;
  std::memset(&F, 0, sizeof(F));
  F.sa = static_cast<const uint32_t*>(h->d_sa);
  F.saoff = static_cast<const int64_t*>(h->d_saoff);
  F.sidx = static_cast<const uint32_t*>(h->d_sidx);
  F.bsz = h->d_tab + h->tl.o_bsz;
  F.tmo = h->d_tab + h->tl.o_tmo;
  F.avail = avail_windows;
  F.R = R;
  F.N = N;
  F.S = S;
  F.e_lo = e_lo;
  F.e_hi = e_hi;
  F.E = E;
  F.W = W;
  F.cnt = static_cast<int32_t*>(dc);
  F.pass = 0;
  CK(h, launch_form(F, st));
  std::vector<int32_t> cnt(cells);
  if (cells) CK(h, cudaMemcpyAsync(cnt.data(), dc, sizeof(int32_t) * cells, cudaMemcpyDeviceToHost, st));
  CK(h, cudaMemcpyAsync(&herr, d_err, 4, cudaMemcpyDeviceToHost, st));
  CK(h, cudaStreamSynchronize(st));
  if (herr) {
    cudaFreeAsync(dc, st);
    return fail(h, PROTEAN_EINVAL, "invalid request (model id or arrival >= trace_len)");
  }
  std::vector<int32_t> off(cells + 1);
  off[0] = 0;
  int64_t total = 0;
  for (size_t i = 0; i < cells; ++i) {
    total += cnt[i];
    if (total > INT32_MAX) {
      cudaFreeAsync(dc, st);
      return fail(h, PROTEAN_ERANGE, "more than 2^31 rows");
    }
    off[i + 1] = (int32_t)total;
  }
  const int64_t cap = *n_batches;
  *n_batches = total;
  if (total > cap || (total > 0 && !batches)) {
    cudaFreeAsync(dc, st);
    return fail(h, PROTEAN_ERANGE, "batches capacity too small (n_batches holds the rows needed)");
  }
  CK(h, cudaMemcpyAsync(batch_off, off.data(), sizeof(int32_t) * (cells + 1), cudaMemcpyHostToDevice, st));
  CK(h, cudaMemsetAsync(dc, 0, std::max<size_t>(4, sizeof(int32_t) * cells), st));
  // pass 1: the rows, in (replica, epoch, GPU, batch id) order
  F.pass = 1;
  F.off = batch_off;
  F.rows = batches;
  CK(h, launch_form(F, st));
  if (sa_len) CK(h, cudaMemcpyAsync(members, h->d_sa, sizeof(uint32_t) * (size_t)sa_len, cudaMemcpyDeviceToDevice, st));
  CK(h, cudaStreamSynchronize(st));  // off lives on this stack frame
  cudaFreeAsync(dc, st);
  return PROTEAN_OK;
}


// End-to-end replay from HOST buffers (include/protean.h section 3c).  Chunk k's trace bytes go
// host -> device on the handle's copy stream while chunk k-1 replays on `stream`; chunk k's outputs
// go device -> host on the handle's return stream while chunk k+1 replays.  Two staging slots,
// each [trace arrivals | meta | relative offsets | per-replica outputs], alternate between chunks.
int protean_replay_traces_host(protean_handle* h, const protean_replay_cfg* cfg, protean_replay_out* out,
                               int32_t chunks, void* stream) {
  if (!h) return PROTEAN_EINVAL;
  if (h->poisoned) return PROTEAN_ESTATE;
  if (!cfg || !out) return fail(h, PROTEAN_EINVAL, "null cfg/out");
  const protean_replay_cfg& c = *cfg;
  if (c.n_replicas < 1 || c.n_gpus < 1 || c.epoch_len_us <= 0 || c.trace_len_us <= 0)
    return fail(h, PROTEAN_EINVAL, "sizes");
  if (c.shard_mode != 0) return fail(h, PROTEAN_EINVAL, "host replay is mode R only");
  if (!c.arrival_us || !c.meta || !c.replica_off) return fail(h, PROTEAN_EINVAL, "null trace");
  if (!out->counters || !out->accum || !out->hist || !out->p50_p99_us || !out->cost_usd || !out->util)
    return fail(h, PROTEAN_EINVAL, "null output");
  if (out->cand_keys || out->batch_log) return fail(h, PROTEAN_EINVAL, "host replay: cand_keys / batch_log unsupported");
  const int R = c.n_replicas, N = c.n_gpus;
  const int64_t* roff = c.replica_off;  // host
  if (roff[0] != 0) return fail(h, PROTEAN_EINVAL, "replica_off[0] != 0");
  for (int r = 0; r < R; ++r)
    if (roff[r + 1] < roff[r]) return fail(h, PROTEAN_EINVAL, "replica_off not monotone");
  const int64_t W = c.epoch_len_us;
  const int64_t E = (c.trace_len_us + W - 1) / W + ((int64_t)h->maxT + W - 1) / W;
  const int K = std::max(1, std::min<int>(chunks < 1 ? 1 : chunks, R));
  std::vector<int> bnd(K + 1);
  for (int k = 0; k <= K; ++k) bnd[k] = (int)(((int64_t)k * R) / K);
  int64_t cap = 1;
  int rcap = 1;
  for (int k = 0; k < K; ++k) {
    cap = std::max<int64_t>(cap, roff[bnd[k + 1]] - roff[bnd[k]]);
    rcap = std::max(rcap, bnd[k + 1] - bnd[k]);
  }
  // staging slot layout (256-byte aligned pieces)
  size_t o = 0;
  const size_t o_arr = o; o += al((size_t)cap * 4);
  const size_t o_meta = o; o += al((size_t)cap);
  const size_t o_off = o; o += al((size_t)(rcap + 1) * 8);
  const size_t o_cnt = o; o += al((size_t)rcap * 10 * 8);
  const size_t o_acc = o; o += al((size_t)rcap * 4 * 8);
  const size_t o_hist = o; o += al((size_t)rcap * 2 * PROTEAN_NBUCKETS * 4);
  const size_t o_pct = o; o += al((size_t)rcap * 4 * 8);
  const size_t o_cost = o; o += al((size_t)rcap * 8);
  const size_t o_util = o; o += al((size_t)rcap * 2 * 8);
  const size_t o_dec = o; o += al(out->decisions ? (size_t)rcap * E * N : 0);
  const size_t o_nb = o; o += al((size_t)rcap * 8);
  const size_t o_cold = o; o += al((size_t)rcap * 8);
  const size_t slot = o;
  cudaStream_t st = reinterpret_cast<cudaStream_t>(stream);
  CK(h, cudaSetDevice(h->device));
  if (!h->hs_copy) CK(h, cudaStreamCreateWithFlags(&h->hs_copy, cudaStreamNonBlocking));
  if (!h->hs_back) CK(h, cudaStreamCreateWithFlags(&h->hs_back, cudaStreamNonBlocking));
  for (int k = 0; k < 3; ++k)
    for (int b = 0; b < 2; ++b)
      if (!h->hev[k][b]) CK(h, cudaEventCreateWithFlags(&h->hev[k][b], cudaEventDisableTiming));
  for (int b = 0; b < 2; ++b) {
    int rc = ensure(h, &h->d_hb[b], &h->hb_bytes[b], slot, st);
    if (rc) return rc;
  }
  CK(h, cudaStreamSynchronize(st));  // the staging slots are allocated before the copy stream uses them
  // hev[0][b]: slot b's trace is on the device; hev[1][b]: slot b's replay finished;
  // hev[2][b]: slot b's outputs are back on the host (the slot may be refilled)
  std::vector<std::vector<int64_t>> rel(K);
  auto h2d = [&](int k) -> int {
    const int b = k & 1;
    char* d = static_cast<char*>(h->d_hb[b]);
    if (k >= 2) CK(h, cudaStreamWaitEvent(h->hs_copy, h->hev[2][b], 0));
    const int64_t lo = roff[bnd[k]], n = roff[bnd[k + 1]] - lo;
    rel[k].resize(bnd[k + 1] - bnd[k] + 1);
    for (int r = bnd[k]; r <= bnd[k + 1]; ++r) rel[k][r - bnd[k]] = roff[r] - lo;
    if (n > 0) {
      CK(h, cudaMemcpyAsync(d + o_arr, c.arrival_us + lo, (size_t)n * 4, cudaMemcpyHostToDevice, h->hs_copy));
      CK(h, cudaMemcpyAsync(d + o_meta, c.meta + lo, (size_t)n, cudaMemcpyHostToDevice, h->hs_copy));
    }
    CK(h, cudaMemcpyAsync(d + o_off, rel[k].data(), rel[k].size() * 8, cudaMemcpyHostToDevice, h->hs_copy));
    CK(h, cudaEventRecord(h->hev[0][b], h->hs_copy));
    return PROTEAN_OK;
  };
  int rc = h2d(0);
  if (rc) return rc;
  float t_pre = 0.f, t_rep = 0.f;
  for (int k = 0; k < K; ++k) {
    const int b = k & 1;
    if (k + 1 < K) {
      rc = h2d(k + 1);  // overlaps chunk k's replay
      if (rc) return rc;
    }
    char* d = static_cast<char*>(h->d_hb[b]);
    const int r0 = bnd[k], rn = bnd[k + 1] - bnd[k];
    protean_replay_cfg cc = c;
    cc.n_replicas = rn;
    cc.replica_base = c.replica_base + r0;
    cc.arrival_us = reinterpret_cast<const uint32_t*>(d + o_arr);
    cc.meta = reinterpret_cast<const uint8_t*>(d + o_meta);
    cc.replica_off = reinterpret_cast<const int64_t*>(d + o_off);
    protean_replay_out oo;
    std::memset(&oo, 0, sizeof(oo));
    oo.counters = reinterpret_cast<int64_t*>(d + o_cnt);
    oo.accum = reinterpret_cast<int64_t*>(d + o_acc);
    oo.hist = reinterpret_cast<uint32_t*>(d + o_hist);
    oo.p50_p99_us = reinterpret_cast<int64_t*>(d + o_pct);
    oo.cost_usd = reinterpret_cast<double*>(d + o_cost);
    oo.util = reinterpret_cast<double*>(d + o_util);
    oo.decisions = out->decisions ? reinterpret_cast<uint8_t*>(d + o_dec) : nullptr;
    oo.n_batches = reinterpret_cast<int64_t*>(d + o_nb);
    oo.cold_starts = reinterpret_cast<int64_t*>(d + o_cold);
    CK(h, cudaStreamWaitEvent(st, h->hev[0][b], 0));
    rc = protean_replay_traces(h, &cc, &oo, stream);
    if (rc) return rc;
    t_pre += h->t_prepass;
    t_rep += h->t_replay;
    CK(h, cudaEventRecord(h->hev[1][b], st));
    CK(h, cudaStreamWaitEvent(h->hs_back, h->hev[1][b], 0));
    auto back = [&](void* dst, size_t off, size_t bytes) -> int {
      if (dst && bytes) CK(h, cudaMemcpyAsync(dst, d + off, bytes, cudaMemcpyDeviceToHost, h->hs_back));
      return PROTEAN_OK;
    };
    const size_t n = (size_t)rn;
    if ((rc = back(out->counters + (size_t)r0 * 10, o_cnt, n * 80))) return rc;
    if ((rc = back(out->accum + (size_t)r0 * 4, o_acc, n * 32))) return rc;
    if ((rc = back(out->hist + (size_t)r0 * 2 * PROTEAN_NBUCKETS, o_hist, n * 2 * PROTEAN_NBUCKETS * 4))) return rc;
    if ((rc = back(out->p50_p99_us + (size_t)r0 * 4, o_pct, n * 32))) return rc;
    if ((rc = back(out->cost_usd + r0, o_cost, n * 8))) return rc;
    if ((rc = back(out->util + (size_t)r0 * 2, o_util, n * 16))) return rc;
    if (out->decisions && (rc = back(out->decisions + (size_t)r0 * E * N, o_dec, n * E * N))) return rc;
    if (out->n_batches && (rc = back(out->n_batches + r0, o_nb, n * 8))) return rc;
    if (out->cold_starts && (rc = back(out->cold_starts + r0, o_cold, n * 8))) return rc;
    CK(h, cudaEventRecord(h->hev[2][b], h->hs_back));
  }
  CK(h, cudaStreamSynchronize(h->hs_back));
  CK(h, cudaStreamSynchronize(h->hs_copy));
  h->t_prepass = t_pre;
  h->t_replay = t_rep;
  return PROTEAN_OK;
}

}  // extern "C"
