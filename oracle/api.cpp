// oracle/api.cpp — TEST INFRASTRUCTURE ONLY (see pem.hpp).
// C interface (oracle/oracle.h): input validation with the same numeric error codes the product
// documents in include/protean.h (defined independently here), conversions, a std::thread pool
// over replicas.
#include "oracle.h"
#include "pem.hpp"
#include <algorithm>
#include <atomic>
#include <cmath>
#include <thread>

using namespace pem;

namespace {

int check_geometry_row(const uint8_t* row, std::vector<int>* g) {
  int cnt[kProfiles] = {0}, compute = 0, last = -1, k = 0;
  int32_t mem = 0;
  for (int i = 0; i < 8; ++i) {
    if (row[i] == 0xFF) {
      for (int j = i; j < 8; ++j)
        if (row[j] != 0xFF) return ORC_EINVAL;
      break;
    }
    if (row[i] >= kProfiles || (int)row[i] < last || i >= kMaxSlices) return ORC_EINVAL;
    last = row[i];
    cnt[row[i]]++;
    compute += kCompute[row[i]];
    mem += kMemEighths[row[i]];
    g->push_back(row[i]);
    ++k;
  }
  if (k == 0) return ORC_EINVAL;
  for (int p = 0; p < kProfiles; ++p)
    if (cnt[p] > kMaxCount[p]) return ORC_EINVAL;
  if (compute > 7 || mem > 8) return ORC_EINVAL;  // <= 7/7 of the SMs, <= 8/8 of the memory (T2)
  return ORC_OK;
}

int build_tables(const orc_tables* t, Tables* tb) {
  if (!t) return ORC_EINVAL;
  if (t->M < 1 || t->M > 64) return ORC_EINVAL;
  if (!t->solo || !t->fbr || !t->mem || !t->bsz || !t->slo || !t->tmo) return ORC_EINVAL;
  const int M = t->M;
  const int32_t gmem = t->gpu_mem_mib == 0 ? kA100Mem : t->gpu_mem_mib;
  if (gmem < 8 || gmem % 8 != 0 || gmem > (1 << 24)) return ORC_EINVAL;
  tb->gpu_mem = gmem;
  for (int p = 0; p < kProfiles; ++p) tb->cap_mem[p] = gmem / 8 * kMemEighths[p];
  for (int i = 0; i < M * kProfiles; ++i) {
    if (t->solo[i] <= 0) return ORC_EINVAL;
    if (t->fbr[i] < 0 || t->fbr[i] > 1000000) return ORC_EINVAL;
  }
  for (int m = 0; m < M; ++m) {
    if (t->mem[m] < 1 || t->mem[m] > gmem) return ORC_EINVAL;
    if (t->bsz[m] < 1 || t->bsz[m] > 65535) return ORC_EINVAL;
    if (t->slo[m] <= 0 || t->tmo[m] < 0) return ORC_EINVAL;
  }
  tb->M = M;
  tb->solo.assign(t->solo, t->solo + M * kProfiles);
  tb->fbr.assign(t->fbr, t->fbr + M * kProfiles);
  tb->mem.assign(t->mem, t->mem + M);
  tb->bsz.assign(t->bsz, t->bsz + M);
  tb->slo.assign(t->slo, t->slo + M);
  tb->tmo.assign(t->tmo, t->tmo + M);
  if (t->geometry_set == 0 || t->geometry_set == 1) {
    tb->geoms = enumerate_geometries(t->geometry_set == 1, nullptr);
  } else if (t->geometry_set == 2) {
    if (t->n_geoms < 1) return ORC_EINVAL;
    if (t->n_geoms > 254) return ORC_ERANGE;
    if (!t->geoms) return ORC_EINVAL;
    for (int j = 0; j < t->n_geoms; ++j) {
      std::vector<int> g;
      int rc = check_geometry_row(t->geoms + 8 * j, &g);
      if (rc) return rc;
      tb->geoms.push_back(g);
    }
  } else {
    return ORC_EINVAL;
  }
  return ORC_OK;
}

void geoms_to_bytes(const std::vector<std::vector<int>>& gs, uint8_t* out) {
  for (size_t j = 0; j < gs.size(); ++j) {
    for (int i = 0; i < 8; ++i) out[8 * j + i] = 0xFF;
    for (size_t i = 0; i < gs[j].size(); ++i) out[8 * j + i] = (uint8_t)gs[j][i];
  }
}

void state_in(const orc_state* s, GpuState* S) {
  S->geom = s->geom;
  for (int i = 0; i < kMaxSlices; ++i) {
    S->last_start[i] = s->last_start[i];
    S->busy_until[i] = s->busy_until[i];
    S->busy_us[i] = s->busy_us[i];
  }
  S->res.clear();
  for (int i = 0; i < s->n_res; ++i) {
    Resident r;
    r.start = s->res[i].start;
    r.end = s->res[i].end;
    r.mem = s->res[i].mem;
    r.slice = s->res[i].slice;
    r.model = s->res[i].model;
    r.strict = s->res[i].strict != 0;
    S->res.push_back(r);
  }
}

void state_out(const GpuState& S, orc_state* s) {
  s->geom = S.geom;
  for (int i = 0; i < kMaxSlices; ++i) {
    s->last_start[i] = S.last_start[i];
    s->busy_until[i] = S.busy_until[i];
    s->busy_us[i] = S.busy_us[i];
  }
  s->n_res = (int32_t)S.res.size();
  for (size_t i = 0; i < S.res.size() && i < 64; ++i) {
    s->res[i].start = S.res[i].start;
    s->res[i].end = S.res[i].end;
    s->res[i].mem = S.res[i].mem;
    s->res[i].slice = S.res[i].slice;
    s->res[i].model = S.res[i].model;
    s->res[i].strict = S.res[i].strict ? 1 : 0;
  }
}

}  // namespace

extern "C" {

int orc_enumerate(int32_t set, int32_t* n, uint8_t* out, int32_t* stats) {
  if (set != 0 && set != 1) return ORC_EINVAL;
  GeomStats st;
  std::vector<std::vector<int>> gs = enumerate_geometries(set == 1, &st);
  if (n) *n = (int32_t)gs.size();
  if (out) geoms_to_bytes(gs, out);
  if (stats) {
    stats[0] = st.feasible;
    stats[1] = st.maximal_placements;
    stats[2] = st.placement_maximal_multisets;
    stats[3] = st.multiset_maximal;
  }
  return ORC_OK;
}

int orc_table_geometries(const orc_tables* t, int32_t* n, uint8_t* out) {
  Tables tb;
  int rc = build_tables(t, &tb);
  if (rc) return rc;
  if (n) *n = (int32_t)tb.geoms.size();
  if (out) geoms_to_bytes(tb.geoms, out);
  return ORC_OK;
}

int64_t orc_exec_us(int64_t solo, int64_t F) { return exec_us(solo, F); }

int orc_place(const orc_tables* t, orc_state* st, int64_t t_ready, int32_t model, int32_t strict,
              int32_t max_live, int64_t H, int32_t* slice, int64_t* start, int64_t* end,
              int32_t* dropped, int64_t* s_start, int64_t* s_end, int32_t* feasible,
              int32_t* eligible, int64_t* accum) {
  Tables tb;
  int rc = build_tables(t, &tb);
  if (rc) return rc;
  if (!st || st->geom < 0 || st->geom >= (int)tb.geoms.size() || model < 0 || model >= tb.M)
    return ORC_EINVAL;
  GpuState S;
  state_in(st, &S);
  Accum acc;
  PlaceOut o = place(tb, tb.geoms[st->geom], S, t_ready, model, strict != 0, max_live, &acc, H);
  state_out(S, st);
  if (slice) *slice = o.slice;
  if (start) *start = o.start;
  if (end) *end = o.end;
  if (dropped) *dropped = o.dropped;
  for (int s = 0; s < kMaxSlices; ++s) {
    if (s_start) s_start[s] = o.s_start[s];
    if (s_end) s_end[s] = o.s_end[s];
    if (feasible) feasible[s] = o.feasible[s];
    if (eligible) eligible[s] = o.eligible[s];
  }
  if (accum) {
    accum[0] += acc.busy_w;
    accum[1] += acc.mem_num;
  }
  return ORC_OK;
}

int64_t orc_form_batches(const orc_tables* t, const uint32_t* arrival, const uint8_t* meta,
                         int64_t n, uint32_t* ready, int32_t* nreq, int32_t* model,
                         int32_t* strict, int64_t* first_raw, int64_t cap) {
  Tables tb;
  int rc = build_tables(t, &tb);
  if (rc) return rc;
  for (int64_t i = 0; i < n; ++i)
    if ((meta[i] & 63) >= tb.M || (meta[i] & 0x40)) return ORC_EINVAL;
  std::vector<Batch> bs = form_batches(tb, arrival, meta, n);
  for (size_t i = 0; i < bs.size() && (int64_t)i < cap; ++i) {
    ready[i] = (uint32_t)bs[i].ready;
    nreq[i] = bs[i].n;
    model[i] = bs[i].model;
    strict[i] = bs[i].strict;
    first_raw[i] = bs[i].first_raw;
  }
  return (int64_t)bs.size();
}

int orc_tick_simulate(const orc_tables* t, int32_t geom, int32_t nb, const int64_t* t_ready,
                      const int32_t* model, const int32_t* slice, int64_t* start, int64_t* end) {
  Tables tb;
  int rc = build_tables(t, &tb);
  if (rc) return rc;
  if (geom < 0 || geom >= (int)tb.geoms.size()) return ORC_EINVAL;
  const std::vector<int>& g = tb.geoms[geom];
  std::vector<TickBatch> bs(nb);
  for (int i = 0; i < nb; ++i) {
    if (slice[i] < 0 || slice[i] >= (int)g.size()) return ORC_EINVAL;
    if (tb.mem[model[i]] > tb.cap(g[slice[i]])) return ORC_EINVAL;
    if (i > 0 && t_ready[i] < t_ready[i - 1]) return ORC_EINVAL;
    bs[i].t = t_ready[i];
    bs[i].m = model[i];
    bs[i].slice = slice[i];
  }
  tick_simulate(tb, g, bs);
  for (int i = 0; i < nb; ++i) {
    start[i] = bs[i].start;
    end[i] = bs[i].end;
  }
  return ORC_OK;
}

int32_t orc_bucket(uint64_t x) { return bucket_of(x); }
uint64_t orc_bucket_lower(int32_t b) { return bucket_lower(b); }
uint64_t orc_percentile(const uint32_t* hist, int32_t q) { return percentile(hist, q); }
uint64_t orc_vm_draw(uint64_t seed, uint64_t replica, uint64_t node, uint64_t k, uint64_t d) {
  return vm_draw(seed, replica, node, k, d);
}
int64_t orc_key(int64_t misses, int64_t tail, int32_t tag) { return make_key(misses, tail, tag); }

int64_t orc_num_epochs(const orc_tables* t, int64_t trace_len, int64_t W) {
  Tables tb;
  int rc = build_tables(t, &tb);
  if (rc) return rc;
  if (W <= 0 || trace_len <= 0) return ORC_EINVAL;
  return num_epochs(tb, trace_len, W);
}

int orc_replay(const orc_tables* t, const orc_replay_in* in, orc_replay_out* out) {
  Tables tb;
  int rc = build_tables(t, &tb);
  if (rc) return rc;
  if (!in || !out) return ORC_EINVAL;
  if (in->R < 1) return ORC_EINVAL;
  if (in->N < 1) return ORC_EINVAL;
  if (in->N > 255) return ORC_ERANGE;
  if (in->W <= 0 || in->trace_len <= 0) return ORC_EINVAL;
  int64_t maxT = 0;
  for (int m = 0; m < tb.M; ++m) maxT = std::max<int64_t>(maxT, tb.tmo[m]);
  if (in->trace_len - 1 + maxT > (int64_t)0xFFFFFFFFLL) return ORC_ERANGE;
  if (in->policy < 0 || in->policy > 2) return ORC_EINVAL;
  if (in->cold_us < 0 || in->keepalive_epochs < 1 || in->prewarm < 0 || in->prewarm > kPoolCap)
    return ORC_EINVAL;
  if (in->policy == 2) {  // Alg 2 heuristic (N1): its knobs, and both of its geometries in the set
    if (in->ewma_alpha_pm < 1 || in->ewma_alpha_pm > 1000) return ORC_EINVAL;
    if (in->t_low < 0 || in->t_high < in->t_low) return ORC_EINVAL;
    const std::vector<int> g421 = {0, 1, 3}, g43 = {2, 3};  // (4g,2g,1g), (4g,3g)
    bool h421 = false, h43 = false;
    for (const std::vector<int>& g : tb.geoms) {
      h421 = h421 || g == g421;
      h43 = h43 || g == g43;
    }
    if (!h421 || !h43) return ORC_EINVAL;
  }
  if (in->shard_mode != 0 && in->shard_mode != 1) return ORC_EINVAL;
  if (in->wait_limit < 0 || in->wait_limit > 255) return ORC_EINVAL;
  if (in->cap_pct < 0 || in->cap_pct > 100) return ORC_EINVAL;
  if (in->init_geom < 0 || in->init_geom >= (int)tb.geoms.size()) return ORC_EINVAL;
  if (in->max_live < 1 || in->max_live > 64) return ORC_EINVAL;
  if (in->vm_policy < 0 || in->vm_policy > 2) return ORC_EINVAL;
  if (in->reconfig_us < 0) return ORC_EINVAL;
  if (!(in->price_od >= 0) || !(in->price_spot >= 0)) return ORC_EINVAL;
  if (in->vm_policy != 0) {
    if (!(in->p_rev >= 0 && in->p_rev <= 1)) return ORC_EINVAL;
    if (in->rev_interval < in->W) return ORC_EINVAL;
    if (in->notice < 0 || in->notice >= in->rev_interval) return ORC_EINVAL;
  }
  if (!in->arrival || !in->meta || !in->replica_off) return ORC_EINVAL;
  if (in->replica_off[0] != 0) return ORC_EINVAL;
  for (int r = 0; r < in->R; ++r)
    if (in->replica_off[r + 1] < in->replica_off[r]) return ORC_EINVAL;
  for (int r = 0; r < in->R; ++r) {
    for (int64_t i = in->replica_off[r]; i < in->replica_off[r + 1]; ++i) {
      if (i > in->replica_off[r] && in->arrival[i] < in->arrival[i - 1]) return ORC_EINVAL;
      if ((int64_t)in->arrival[i] >= in->trace_len) return ORC_EINVAL;
      if ((in->meta[i] & 63) >= tb.M || (in->meta[i] & 0x40)) return ORC_EINVAL;
    }
  }

  ReplayCfg cfg;
  cfg.N = in->N;
  cfg.trace_len = in->trace_len;
  cfg.W = in->W;
  cfg.policy = in->policy;
  cfg.wait_limit = in->wait_limit;
  cfg.cap_pct = in->cap_pct;
  cfg.init_geom = in->init_geom;
  cfg.max_live = in->max_live;
  cfg.vm_policy = in->vm_policy;
  cfg.reconfig_us = in->reconfig_us;
  cfg.p_rev = in->p_rev;
  cfg.price_od = in->price_od;
  cfg.price_spot = in->price_spot;
  cfg.rev_interval = in->rev_interval;
  cfg.notice = in->notice;
  cfg.seed = in->seed;
  cfg.cold_us = in->cold_us;
  cfg.keepalive_epochs = in->keepalive_epochs;
  cfg.prewarm = in->prewarm;
  cfg.ewma_alpha_pm = in->ewma_alpha_pm;
  cfg.t_low = in->t_low;
  cfg.t_high = in->t_high;
  const int64_t E = num_epochs(tb, in->trace_len, in->W);
  const int G = (int)tb.geoms.size();
  const int N = in->N;

  std::atomic<int> next(0);
  std::atomic<bool> overflow(false);
  auto worker = [&]() {
    for (;;) {
      int r = next.fetch_add(1);
      if (r >= in->R) break;
      ReplayOut ro;
      const int64_t off = in->replica_off[r];
      replay_replica(tb, cfg, (uint64_t)(in->replica_base + r), in->arrival + off, in->meta + off,
                     in->replica_off[r + 1] - off, out->cand_keys != nullptr, out->log != nullptr,
                     &ro);
      for (int i = 0; i < 10; ++i) out->counters[r * 10 + i] = ro.counters[i];
      for (int i = 0; i < 4; ++i) out->accum[r * 4 + i] = ro.accum[i];
      for (int i = 0; i < 2 * kBuckets; ++i) out->hist[(int64_t)r * 2 * kBuckets + i] = ro.hist[i];
      for (int c = 0; c < 2; ++c)
        for (int q = 0; q < 2; ++q) out->p50_p99[r * 4 + c * 2 + q] = ro.p[c][q];
      out->cost[r] = ro.cost;
      out->util[2 * r] = ro.util[0];
      out->util[2 * r + 1] = ro.util[1];
      if (out->decisions)
        std::copy(ro.decisions.begin(), ro.decisions.end(), out->decisions + (int64_t)r * E * N);
      if (out->cand_keys)
        std::copy(ro.cand_keys.begin(), ro.cand_keys.end(), out->cand_keys + (int64_t)r * E * N * G);
      if (out->n_batches) out->n_batches[r] = ro.n_batches;
      if (out->cold_starts) out->cold_starts[r] = ro.cold_starts;
      if (out->stats)
        for (int i = 0; i < 4; ++i) out->stats[r * 4 + i] = ro.stats[i];
      if (ro.pool_overflow) overflow = true;
      if (out->log) {
        for (size_t i = 0; i < ro.log.size() && (int64_t)i < out->log_cap; ++i) {
          const BatchRec& b = ro.log[i];
          orc_batch_rec& o = out->log[(int64_t)r * out->log_cap + i];
          o.ready = b.ready;
          o.epoch = b.epoch;
          o.n = b.n;
          o.model = b.model;
          o.strict = b.strict;
          o.gpu = b.gpu;
          o.slice = b.slice;
          o.dropped = b.dropped;
          o.start = b.start;
          o.end = b.end;
        }
      }
    }
  };
  int nt = std::max(1, std::min(in->nthreads, in->R));
  std::vector<std::thread> th;
  for (int i = 1; i < nt; ++i) th.emplace_back(worker);
  worker();
  for (auto& x : th) x.join();
  if (overflow) return ORC_ERANGE;  // a container pool outgrew kPoolCap (N3, R22)
  return ORC_OK;
}

int orc_score_epoch(const orc_tables* t, int32_t R, int32_t N, int32_t epoch, int32_t max_live,
                    int64_t W, int64_t H, const uint32_t* b_ready, const uint32_t* b_req_off,
                    const int32_t* b_n, const int32_t* b_model, const int32_t* b_strict,
                    const int32_t* batch_off, const uint32_t* arrival, orc_state* state,
                    int32_t geom_lo, int32_t geom_hi, int64_t* best_key, int64_t* cand_key,
                    int64_t* p_start, int64_t* p_end, int32_t* p_slice, int32_t* p_dropped,
                    int64_t* counters, int64_t* accum, double price_od, double price_spot,
                    double* cost) {
  Tables tb;
  int rc = build_tables(t, &tb);
  if (rc) return rc;
  const int G = (int)tb.geoms.size();
  if (R < 1 || N < 1 || epoch < 0 || W <= 0 || H < 0) return ORC_EINVAL;
  if (N > 255) return ORC_ERANGE;
  if (max_live < 1 || max_live > 64) return ORC_EINVAL;
  if (geom_lo < 0 || geom_hi > G || geom_lo >= geom_hi) return ORC_EINVAL;
  if (!batch_off || !state || !best_key || !counters) return ORC_EINVAL;
  if (batch_off[0] != 0) return ORC_EINVAL;
  if (!(price_od >= 0) || !(price_spot >= 0)) return ORC_EINVAL;
  const int64_t eW = (int64_t)epoch * W, T = eW + W;
  for (int x = 0; x < R * N; ++x) {
    if (batch_off[x + 1] < batch_off[x]) return ORC_EINVAL;
    const orc_state& s = state[x];
    if (s.geom < 0 || s.geom >= G) return ORC_EINVAL;
    if (s.target != -1 && (s.target < 0 || s.target >= G)) return ORC_EINVAL;
    if (s.n_res < 0) return ORC_EINVAL;
    if (s.vm_type < 0 || s.vm_type > 2) return ORC_EINVAL;
    if (s.n_res > max_live) return ORC_ERANGE;
    for (int i = 0; i < s.n_res; ++i)
      if (s.res[i].slice < 0 || s.res[i].slice >= (int)tb.geoms[s.geom].size() ||
          s.res[i].model < 0 || s.res[i].model >= tb.M)
        return ORC_EINVAL;
    for (int32_t b = batch_off[x]; b < batch_off[x + 1]; ++b) {
      if (b_model[b] < 0 || b_model[b] >= tb.M || b_n[b] < 1) return ORC_EINVAL;
      if ((int64_t)b_ready[b] < eW || (int64_t)b_ready[b] >= T) return ORC_EINVAL;
      if (b > batch_off[x] && b_ready[b] < b_ready[b - 1]) return ORC_EINVAL;
      for (int i = 0; i < b_n[b]; ++i) {
        uint32_t a = arrival[b_req_off[b] + i];
        if (a > b_ready[b] || (i > 0 && a < arrival[b_req_off[b] + i - 1])) return ORC_EINVAL;
      }
    }
  }
  const int nc = geom_hi - geom_lo;
  for (int r = 0; r < R; ++r) {
    for (int g = 0; g < N; ++g) {
      const int x = r * N + g;
      orc_state& st = state[x];
      if (st.target >= 0 && st.recfg_end <= T) {  // install (O5.3)
        GpuState fresh;
        fresh.geom = st.target;
        state_out(fresh, &st);
        st.target = -1;
        st.wait_ctr = 0;
      }
      GpuState S;
      state_in(&st, &S);
      Accum acc;
      int64_t* c = counters + 10 * r;
      for (int32_t b = batch_off[x]; b < batch_off[x + 1]; ++b) {
        PlaceOut po = place(tb, tb.geoms[S.geom], S, b_ready[b], b_model[b], b_strict[b] != 0,
                            max_live, &acc, H);
        if (p_start) {
          p_start[b] = po.dropped ? 0 : po.start;
          p_end[b] = po.dropped ? 0 : po.end;
          p_slice[b] = po.dropped ? 0xFF : po.slice;
          p_dropped[b] = po.dropped;
        }
        const bool strict = b_strict[b] != 0;
        if (strict) c[0] += b_n[b]; else c[4] += b_n[b];
        if (po.dropped) {
          if (strict) c[3] += b_n[b]; else c[6] += b_n[b];
          continue;
        }
        for (int i = 0; i < b_n[b]; ++i) {
          int64_t lat = po.end - (int64_t)arrival[b_req_off[b] + i];
          if (strict) { if (lat <= tb.slo[b_model[b]]) c[1]++; else c[2]++; }
          else c[5]++;
        }
      }
      state_out(S, &st);
      if (accum) {
        accum[4 * r] += acc.busy_w;
        accum[4 * r + 1] += acc.mem_num;
      }
      const bool decidable = st.has_vm && st.recfg_end <= T;
      // node-epoch VM cost (T3 P:L173-179, cost projection P:L333, reading Q35): the node's
      // price for its billing type over the epoch, price [$/h] * W [us] / 3.6e9 [us/h]
      if (cost) {
        const double price = !st.has_vm ? 0.0 : st.vm_type == 1 ? price_od : st.vm_type == 2 ? price_spot : 0.0;
        cost[x] = (price * (double)W) / 3.6e9;
      }
      best_key[x] = -1;
      for (int j = geom_lo; j < geom_hi; ++j) {
        int64_t key = -1;
        if (decidable) {
          GpuState C;
          C.geom = j;
          int64_t misses = 0, tail = 0;
          for (int32_t b = batch_off[x]; b < batch_off[x + 1]; ++b) {
            PlaceOut po = place(tb, tb.geoms[j], C, b_ready[b], b_model[b], b_strict[b] != 0,
                                max_live, nullptr, H);
            if (b_strict[b]) {
              if (po.dropped) {
                misses += b_n[b];
              } else {
                int64_t hits = 0;
                for (int i = 0; i < b_n[b]; ++i)
                  if (po.end - (int64_t)arrival[b_req_off[b] + i] <= tb.slo[b_model[b]]) hits++;
                misses += b_n[b] - hits;
              }
            } else {
              tail = std::max(tail, po.dropped ? (int64_t)kSat32
                                               : po.end - (int64_t)arrival[b_req_off[b]]);
            }
          }
          key = make_key(misses, tail, j == S.geom ? 0 : j + 1);
          c[8] += (int64_t)(batch_off[x + 1] - batch_off[x]) * (int64_t)tb.geoms[j].size();
          c[9] += 1;
          if (best_key[x] < 0 || key < best_key[x]) best_key[x] = key;
        }
        if (cand_key) cand_key[(int64_t)x * nc + (j - geom_lo)] = key;
      }
    }
  }
  return ORC_OK;
}

int orc_sweep_depths(const orc_tables* t, int32_t R, int32_t N, int32_t max_live,
              const uint32_t* b_ready, const uint32_t* b_req_off, const int32_t* b_n,
              const int32_t* b_model, const int32_t* b_strict, const int32_t* batch_off,
              const uint32_t* arrival, const uint8_t* cur_geom, int32_t geom_lo, int32_t geom_hi,
              int64_t* depth_key, uint8_t* depth_code, int64_t* best_key, int64_t* n_eval) {
  Tables tb;
  int rc = build_tables(t, &tb);
  if (rc) return rc;
  const int G = (int)tb.geoms.size();
  if (R < 1 || N < 1) return ORC_EINVAL;
  if (N > 255) return ORC_ERANGE;
  if (max_live < 1 || max_live > 64) return ORC_EINVAL;
  if (geom_lo < 0 || geom_hi > G || geom_lo >= geom_hi) return ORC_EINVAL;
  if (!batch_off || !cur_geom || !best_key || !n_eval) return ORC_EINVAL;
  if (batch_off[0] != 0) return ORC_EINVAL;
  for (int x = 0; x < R * N; ++x) {
    if (batch_off[x + 1] < batch_off[x]) return ORC_EINVAL;
    if (cur_geom[x] != 0xFF && cur_geom[x] >= G) return ORC_EINVAL;
    for (int32_t b = batch_off[x]; b < batch_off[x + 1]; ++b) {
      if (b_model[b] < 0 || b_model[b] >= tb.M || b_n[b] < 1) return ORC_EINVAL;
      if (b > batch_off[x] && b_ready[b] < b_ready[b - 1]) return ORC_EINVAL;
      for (int i = 0; i < b_n[b]; ++i) {
        uint32_t a = arrival[b_req_off[b] + i];
        if (a > b_ready[b] || (i > 0 && a < arrival[b_req_off[b] + i - 1])) return ORC_EINVAL;
      }
    }
  }
  const int nc = geom_hi - geom_lo;
  uint64_t total = 0;
  for (int x = 0; x < R * N; ++x) {
    std::vector<SweepBatch> bs;
    for (int32_t b = batch_off[x]; b < batch_off[x + 1]; ++b) {
      SweepBatch sb;
      sb.ready = b_ready[b];
      sb.model = b_model[b];
      sb.strict = b_strict[b] != 0;
      sb.arr.assign(arrival + b_req_off[b], arrival + b_req_off[b] + b_n[b]);
      bs.push_back(sb);
    }
    best_key[x] = -1;
    for (int j = geom_lo; j < geom_hi; ++j) {
      int64_t keys[8], key;
      int code;
      sweep_depths(tb, j, cur_geom[x] == j ? 0 : j + 1, bs, max_live, keys, &key, &code, &total);
      if (depth_key)
        for (int c = 0; c < 8; ++c) depth_key[((int64_t)x * nc + (j - geom_lo)) * 8 + c] = keys[c];
      if (depth_code) depth_code[(int64_t)x * nc + (j - geom_lo)] = (uint8_t)code;
      if (best_key[x] < 0 || key < best_key[x]) best_key[x] = key;
    }
  }
  *n_eval += (int64_t)total;
  return ORC_OK;
}

int orc_sweep(const orc_tables* t, int32_t R, int32_t N, int32_t max_live, int32_t max_batches,
              const uint32_t* b_ready, const uint32_t* b_req_off, const int32_t* b_n,
              const int32_t* b_model, const int32_t* b_strict, const int32_t* batch_off,
              const uint32_t* arrival, const uint8_t* cur_geom, int32_t geom_lo, int32_t geom_hi,
              int64_t* sweep_key, uint32_t* assign, int64_t* best_key, int64_t* n_assign) {
  Tables tb;
  int rc = build_tables(t, &tb);
  if (rc) return rc;
  const int G = (int)tb.geoms.size();
  if (R < 1 || N < 1) return ORC_EINVAL;
  if (N > 255) return ORC_ERANGE;
  if (max_live < 1 || max_live > 64) return ORC_EINVAL;
  if (max_batches < 1 || max_batches > 8) return ORC_EINVAL;
  if (geom_lo < 0 || geom_hi > G || geom_lo >= geom_hi) return ORC_EINVAL;
  if (!batch_off || !cur_geom || !best_key || !n_assign) return ORC_EINVAL;
  if (batch_off[0] != 0) return ORC_EINVAL;
  for (int x = 0; x < R * N; ++x) {
    if (batch_off[x + 1] < batch_off[x]) return ORC_EINVAL;
    if (cur_geom[x] != 0xFF && cur_geom[x] >= G) return ORC_EINVAL;
    for (int32_t b = batch_off[x]; b < batch_off[x + 1]; ++b) {
      if (b_model[b] < 0 || b_model[b] >= tb.M || b_n[b] < 1) return ORC_EINVAL;
      if (b > batch_off[x] && b_ready[b] < b_ready[b - 1]) return ORC_EINVAL;
      for (int i = 0; i < b_n[b]; ++i) {
        uint32_t a = arrival[b_req_off[b] + i];
        if (a > b_ready[b] || (i > 0 && a < arrival[b_req_off[b] + i - 1])) return ORC_EINVAL;
      }
    }
    if (batch_off[x + 1] - batch_off[x] > max_batches) return ORC_ERANGE;
  }
  const int nc = geom_hi - geom_lo;
  uint64_t total = 0;
  for (int x = 0; x < R * N; ++x) {
    std::vector<SweepBatch> bs;
    for (int32_t b = batch_off[x]; b < batch_off[x + 1]; ++b) {
      SweepBatch sb;
      sb.ready = b_ready[b];
      sb.model = b_model[b];
      sb.strict = b_strict[b] != 0;
      sb.arr.assign(arrival + b_req_off[b], arrival + b_req_off[b] + b_n[b]);
      bs.push_back(sb);
    }
    best_key[x] = -1;
    for (int j = geom_lo; j < geom_hi; ++j) {
      int64_t key;
      uint64_t idx;
      sweep_gpu(tb, j, cur_geom[x] == j ? 0 : j + 1, bs, max_live, &key, &idx, &total);
      const int S = (int)tb.geoms[j].size();
      uint32_t code = 0;
      for (size_t k = 0; k < bs.size(); ++k) {  // base-S digits -> 3-bit slice fields
        code |= (uint32_t)(idx % (uint64_t)S) << (3 * k);
        idx /= (uint64_t)S;
      }
      if (sweep_key) sweep_key[(int64_t)x * nc + (j - geom_lo)] = key;
      if (assign) assign[(int64_t)x * nc + (j - geom_lo)] = code;
      if (best_key[x] < 0 || key < best_key[x]) best_key[x] = key;
    }
  }
  *n_assign += (int64_t)total;
  return ORC_OK;
}

int orc_form_dispatch(const orc_tables* t, int32_t R, int32_t N, int64_t W, int64_t trace_len,
                     const uint32_t* arrival, const uint8_t* meta, const int64_t* replica_off,
                     int32_t e_lo, int32_t e_hi, const int64_t* avail, uint32_t* b_ready,
                     uint32_t* b_req_off, int32_t* b_n, int32_t* b_model, int32_t* b_strict,
                     int32_t* b_gpu, int32_t* batch_off, int64_t* n_rows, uint32_t* members,
                     int64_t members_cap) {
  Tables tb;
  int rc = build_tables(t, &tb);
  if (rc) return rc;
  if (R < 1 || N < 1 || W <= 0 || trace_len <= 0 || !n_rows || !batch_off) return ORC_EINVAL;
  if (N > 255) return ORC_ERANGE;
  const int64_t E = num_epochs(tb, trace_len, W);
  if (e_lo < 0 || e_hi > E || e_lo > e_hi) return ORC_EINVAL;
  if (!arrival || !meta || !replica_off || replica_off[0] != 0) return ORC_EINVAL;
  for (int r = 0; r < R; ++r) {
    if (replica_off[r + 1] < replica_off[r]) return ORC_EINVAL;
    for (int64_t i = replica_off[r]; i < replica_off[r + 1]; ++i) {
      if (i > replica_off[r] && arrival[i] < arrival[i - 1]) return ORC_EINVAL;
      if ((int64_t)arrival[i] >= trace_len) return ORC_EINVAL;
      if ((meta[i] & 63) >= tb.M || (meta[i] & 0x40)) return ORC_EINVAL;
    }
  }
  if (trace_len - 1 + [&] { int64_t m = 0; for (int q = 0; q < tb.M; ++q) m = std::max<int64_t>(m, tb.tmo[q]); return m; }() >
      (int64_t)0xFFFFFFFFLL)
    return ORC_ERANGE;
  const int Ew = e_hi - e_lo;
  // per replica: batches in id order (O3), then dispatch from epoch 0 (O5.2, reading Q18)
  struct Row { int e, gpu; const Batch* b; };
  std::vector<std::vector<Batch>> all(R);
  std::vector<std::vector<Row>> rows(R);
  for (int r = 0; r < R; ++r) {
    const int64_t off = replica_off[r];
    all[r] = form_batches(tb, arrival + off, meta + off, replica_off[r + 1] - off);
    int cursor = 0;
    for (const Batch& b : all[r]) {
      const int64_t e = b.ready / W;  // half-open epochs (Q31)
      if (e >= e_hi) break;
      int chosen = -1;
      for (int i = 0; i < N; ++i) {
        const int n = (cursor + i) % N;
        const bool ok = !avail || (avail[((int64_t)r * N + n) * 2] <= b.ready &&
                                   b.ready < avail[((int64_t)r * N + n) * 2 + 1]);
        if (ok) { chosen = n; break; }
      }
      if (chosen < 0) continue;  // dispatch drop: not emitted
      cursor = (chosen + 1) % N;
      if (e >= e_lo) rows[r].push_back({(int)(e - e_lo), chosen, &b});
    }
    std::stable_sort(rows[r].begin(), rows[r].end(), [](const Row& a, const Row& b) {
      return a.e != b.e ? a.e < b.e : a.gpu < b.gpu;  // (epoch, gpu), id order kept within
    });
  }
  int64_t total = 0, nmem = 0;
  for (int r = 0; r < R; ++r) {
    total += (int64_t)rows[r].size();
    for (const Row& w : rows[r]) nmem += w.b->n;
  }
  const int64_t cap = *n_rows;
  *n_rows = total;
  if (total > cap || nmem > members_cap) return ORC_ERANGE;
  int64_t x = 0, m = 0;
  batch_off[0] = 0;
  for (int r = 0; r < R; ++r) {
    size_t k = 0;
    for (int e = 0; e < Ew; ++e) {
      for (int g = 0; g < N; ++g) {
        while (k < rows[r].size() && rows[r][k].e == e && rows[r][k].gpu == g) {
          const Batch& b = *rows[r][k].b;
          b_ready[x] = (uint32_t)b.ready;
          b_req_off[x] = (uint32_t)m;
          b_n[x] = b.n;
          b_model[x] = b.model;
          b_strict[x] = b.strict ? 1 : 0;
          b_gpu[x] = g;
          for (uint32_t a : b.arr) members[m++] = a;
          ++x;
          ++k;
        }
        batch_off[((int64_t)r * Ew + e) * N + g + 1] = (int32_t)x;
      }
    }
  }
  return ORC_OK;
}

}  // extern "C"
