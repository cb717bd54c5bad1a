// oracle/epoch.cpp — TEST INFRASTRUCTURE ONLY (see pem.hpp).
// O4/O5: one replica's epoch-by-epoch replay.  Per epoch of length W (Alg 2's Monitor_Interval,
// P:L291, reading Q1): VM events (O11) -> installs -> round-robin dispatch (Q18) -> actual Alg 1
// placement + request accounting (O6, O7) -> scoring of every candidate geometry for every
// decidable GPU, from idle, on that GPU's epoch batches (O8, readings Q19-Q21, the paper's
// "Oracle" scheme P:L485) -> Alg 2 hysteresis + ~30% cap (O9, O10).
// policy 2 (N1) replaces the scoring by Alg 2's own heuristic (lines 1-23, readings
// R10-R17 of DESIGN.md): EWMA of the observed BE load -> small-slice set -> thresholds -> geometry.
// N3 (cold_us > 0): the Autoscaler's container pools (readings R22-R27): one container
// per batch, reactive scale-up with a cold start t_cold, delayed termination of surplus containers.
#include "pem.hpp"
#include <algorithm>
#include <climits>

namespace pem {

int64_t num_epochs(const Tables& tb, int64_t trace_len, int64_t W) {
  int64_t maxT = 0;
  for (int m = 0; m < tb.M; ++m) maxT = std::max<int64_t>(maxT, tb.tmo[m]);
  return (trace_len + W - 1) / W + (maxT + W - 1) / W;
}

namespace {
enum { VM_NONE = 0, VM_OD = 1, VM_SPOT = 2 };
constexpr int64_t kForever = LLONG_MAX;

struct Node {
  int vm = VM_OD;
  int bill = VM_OD;
  int64_t bill_since = 0;
  int64_t avail_from = 0, avail_until = kForever;
};

struct Gpu {
  GpuState S;
  int target = -1;          // pending reconfiguration target
  int ctr = 0;              // Alg 2 wait_ctr
  int64_t rs = 0, re = 0;   // reconfiguration window [rs, re)
  Node node;
  int64_t pred_num = 0;     // Alg 2 history_info (N1): EWMA of BE batches, milli-batches
  int64_t pred_mem = 0;     //   and of their total footprint, milli-MiB (R11)
  std::vector<std::vector<int64_t>> pool;  // N3: per model, busy-until of every container (R22)
  std::vector<int> surplus_ctr;            // N3: consecutive epochs with surplus containers (R26)
};

struct Replay {
  const Tables& tb;
  const ReplayCfg& cfg;
  uint64_t replica;
  int64_t H;
  ReplayOut* out;
  std::vector<Gpu> gpu;

  Replay(const Tables& t, const ReplayCfg& c, uint64_t r, int64_t h, ReplayOut* o)
      : tb(t), cfg(c), replica(r), H(h), out(o), gpu(c.N) {}

  int64_t clipH(int64_t x) const { return std::min(x, H); }

  void bill_switch(Node& nd, int type, int64_t at) {
    if (nd.bill == VM_OD) out->accum[2] += clipH(at) - clipH(nd.bill_since);
    if (nd.bill == VM_SPOT) out->accum[3] += clipH(at) - clipH(nd.bill_since);
    nd.bill = type;
    nd.bill_since = at;
  }

  bool has_vm(const Gpu& g, int64_t t) const { return g.node.avail_from <= t && t < g.node.avail_until; }
  bool available(const Gpu& g, int64_t t) const { return has_vm(g, t) && !(g.rs <= t && t < g.re); }

  void install(Gpu& g) {  // at recfg_end: new geometry, idle, wait_ctr reset (reading Q24)
    GpuState fresh;
    fresh.geom = g.target;
    g.S = fresh;
    g.target = -1;
    g.ctr = 0;
  }

  // O11 — one revocation boundary tau = k * T_rev for node n.
  void vm_event(int n, int64_t k, int64_t tau) {
    Gpu& g = gpu[n];
    Node& nd = g.node;
    const uint64_t thr = (uint64_t)(cfg.p_rev * 9007199254740992.0);  // p_rev * 2^53
    const bool revoked = vm_draw(cfg.seed, replica, n, k, 0) < thr;
    const bool spot_ok = vm_draw(cfg.seed, replica, n, k, 1) >= thr;
    if (cfg.vm_policy == 1) {  // PROTEAN: retry spot, else on-demand; seamless redirect
      if (nd.vm == VM_SPOT) {
        if (revoked && !spot_ok) {
          nd.vm = VM_OD;
          bill_switch(nd, VM_OD, tau + cfg.notice);
        }
      } else if (nd.vm == VM_OD) {
        if (spot_ok) {  // spot whenever possible
          nd.vm = VM_SPOT;
          bill_switch(nd, VM_SPOT, tau);
        }
      }
    } else if (cfg.vm_policy == 2) {  // Spot Only
      if (nd.vm == VM_SPOT) {
        if (revoked && !spot_ok) {  // node lost: no dispatch from tau, billed through the notice
          nd.vm = VM_NONE;
          nd.avail_until = tau;
          bill_switch(nd, VM_NONE, tau + cfg.notice);
          g.target = -1;
          g.rs = g.re = 0;
          reset_pool(g);  // the node's containers go with it (R27)
        }
      } else if (nd.vm == VM_NONE) {
        if (spot_ok) {  // a new spot VM: initial geometry, idle, wait_ctr 0
          nd.vm = VM_SPOT;
          nd.avail_from = tau;
          nd.avail_until = kForever;
          bill_switch(nd, VM_SPOT, tau);
          GpuState fresh;
          fresh.geom = cfg.init_geom;
          g.S = fresh;
          g.target = -1;
          g.ctr = 0;
          g.rs = g.re = 0;
          reset_pool(g);  // a new VM starts with the prewarmed pool only (R27)
        }
      }
    }
  }

  void reset_pool(Gpu& g) {  // R22: prewarm idle containers per model (busy-until 0)
    g.pool.assign(tb.M, std::vector<int64_t>(cfg.prewarm, 0));
    g.surplus_ctr.assign(tb.M, 0);
  }

  // R23: the container a batch of model m dispatched at t runs in: the first idle one (busy-until
  // <= t), else a new one after a cold start.  Returns its index; *t_eff = t (+ cold_us if spawned).
  size_t acquire(Gpu& g, int m, int64_t t, int64_t* t_eff) {
    std::vector<int64_t>& P = g.pool[m];
    for (size_t i = 0; i < P.size(); ++i)
      if (P[i] <= t) {
        *t_eff = t;
        return i;
      }
    if ((int)P.size() >= kPoolCap) out->pool_overflow = true;  // R22 capacity (ERANGE)
    P.push_back(t);  // reactive scale-up: one container per batch
    out->cold_starts += 1;
    *t_eff = t + cfg.cold_us;  // t = t_cold + t_queue + t_exec
    return P.size() - 1;
  }

  void account(const Batch& b, const PlaceOut* po, int drop_kind) {
    int64_t* c = out->counters;
    if (b.strict) c[0] += b.n; else c[4] += b.n;
    if (drop_kind != 0) {
      if (b.strict) c[3] += b.n; else c[6] += b.n;
      return;
    }
    for (uint32_t a : b.arr) {
      int64_t lat = po->end - (int64_t)a;  // t_queue + t_exec, t_cold = 0 (reading Q15)
      if (b.strict) {
        if (lat <= tb.slo[b.model]) c[1]++; else c[2]++;   // SLO compliance
        out->hist[bucket_of((uint64_t)lat)]++;
      } else {
        c[5]++;
        out->hist[kBuckets + bucket_of((uint64_t)lat)]++;
      }
    }
  }

  void run(const std::vector<Batch>& batches, int64_t E, bool want_keys, bool want_log) {
    const int N = cfg.N;
    const int G = (int)tb.geoms.size();
    for (int n = 0; n < N; ++n) {
      gpu[n].S.geom = cfg.init_geom;  // (4g,2g,1g) by default
      Node& nd = gpu[n].node;
      nd.vm = nd.bill = (cfg.vm_policy == 0) ? VM_OD : VM_SPOT;
      reset_pool(gpu[n]);
    }
    out->hist.assign(2 * kBuckets, 0);
    out->decisions.assign((size_t)E * N, 0xFF);
    if (want_keys) out->cand_keys.assign((size_t)E * N * G, -1);
    Accum acc;
    int cursor = 0;
    size_t bi = 0;

    for (int64_t e = 0; e < E; ++e) {
      const int64_t eW = e * cfg.W, T = eW + cfg.W;

      // 1. VM events at revocation boundaries inside this epoch (installs due earlier first)
      if (cfg.vm_policy != 0) {
        for (int64_t k = (eW + cfg.rev_interval - 1) / cfg.rev_interval; k * cfg.rev_interval < T; ++k) {
          const int64_t tau = k * cfg.rev_interval;
          if (k < 1 || tau >= H) continue;
          for (int n = 0; n < N; ++n) {
            if (gpu[n].target >= 0 && gpu[n].re <= tau) install(gpu[n]);
            vm_event(n, k, tau);
          }
        }
      }
      // pending reconfigurations that complete by the decision time T
      for (int n = 0; n < N; ++n)
        if (gpu[n].target >= 0 && gpu[n].re <= T) install(gpu[n]);

      // 2. dispatch this epoch's batches in id order: round-robin over available GPUs
      std::vector<std::vector<size_t>> list(N);
      const size_t first_bi = bi;
      std::vector<BatchRec> erec;  // this epoch's log rows, in id order
      while (bi < batches.size() && batches[bi].ready < T) {
        const Batch& b = batches[bi];
        int chosen = -1;
        for (int i = 0; i < N; ++i) {
          int n = (cursor + i) % N;
          if (available(gpu[n], b.ready)) { chosen = n; break; }
        }
        erec.push_back({(uint32_t)b.ready, (uint32_t)e, b.n, b.model, b.strict, 0xFF, 0xFF, 1, 0, 0});
        if (chosen < 0) {
          account(b, nullptr, 1);  // dispatch drop (reading Q32)
        } else {
          list[chosen].push_back(bi);
          cursor = (chosen + 1) % N;
        }
        ++bi;
      }

      // 3. actual placement on the current geometry, carried state
      for (int n = 0; n < N; ++n) {
        Gpu& g = gpu[n];
        for (size_t x : list[n]) {
          const Batch& b = batches[x];
          int64_t t_eff = b.ready;
          size_t ci = 0;
          if (cfg.cold_us > 0) ci = acquire(g, b.model, b.ready, &t_eff);  // N3 (R23)
          PlaceOut po = place(tb, tb.geoms[g.S.geom], g.S, t_eff, b.model, b.strict,
                              cfg.max_live, &acc, H);
          if (cfg.cold_us > 0) g.pool[b.model][ci] = po.dropped ? t_eff : po.end;  // R24
          account(b, &po, po.dropped);
          BatchRec& r = erec[x - first_bi];
          r.gpu = n;
          r.dropped = po.dropped;
          if (!po.dropped) {
            r.slice = po.slice;
            r.start = po.start;
            r.end = po.end;
          }
        }
      }
      if (want_log) out->log.insert(out->log.end(), erec.begin(), erec.end());

      // N3 delayed termination (R26): n_c = batches of model m dispatched to the GPU in this
      // epoch; a pool larger than n_c for keepalive_epochs consecutive epochs loses its
      // surplus containers that are idle at T
      if (cfg.cold_us > 0) {
        for (int n = 0; n < N; ++n) {
          Gpu& g = gpu[n];
          std::vector<int64_t> need(tb.M, 0);
          for (size_t x : list[n]) need[batches[x].model] += 1;
          for (int m = 0; m < tb.M; ++m) {
            std::vector<int64_t>& P = g.pool[m];
            const int64_t surplus = (int64_t)P.size() - need[m];
            if (surplus <= 0) {
              g.surplus_ctr[m] = 0;
              continue;
            }
            if (++g.surplus_ctr[m] < cfg.keepalive_epochs) continue;
            int64_t drop = surplus;
            std::vector<int64_t> kept;
            for (int64_t bu : P) {
              if (drop > 0 && bu <= T) { --drop; continue; }  // terminate an idle container
              kept.push_back(bu);
            }
            P = kept;
            g.surplus_ctr[m] = 0;
          }
        }
      }

      // 4. candidate scoring for every decidable GPU (has a VM at T, no open window)
      std::vector<int> wants;
      std::vector<int64_t> key_best(N, -1), key_cur(N, -1);
      std::vector<int> best(N, -1);
      if (cfg.policy == 2) {
        // Alg 2 GPU_Reconfigurator, one decidable GPU at a time
        for (int n = 0; n < N; ++n) {
          Gpu& g = gpu[n];
          if (!(has_vm(g, T) && g.re <= T)) continue;
          const int cur = g.S.geom;
          // line 2: curr_queue_info = the BE batches dispatched to this GPU in the epoch (R10)
          int64_t be_num = 0, be_mem = 0;
          for (size_t x : list[n]) {
            if (batches[x].strict) continue;
            be_num += 1;
            be_mem += tb.mem[batches[x].model];  // footprint per batch (Q36)
          }
          // lines 8-9: pred_BE_num, pred_BE_mem by a light-weight EWMA [95] (R11)
          const int64_t a = cfg.ewma_alpha_pm;
          g.pred_num = (a * 1000 * be_num + (1000 - a) * g.pred_num) / 1000;
          g.pred_mem = (a * 1000 * be_mem + (1000 - a) * g.pred_mem) / 1000;
          // lines 5-7, 10-18: first small-slice set whose summed capacity holds pred_BE_mem (R12)
          const std::vector<std::vector<int>> small_slice_set = {{0, 1}, {2}};  // [[1g,2g],[3g]]
          bool found = false;
          std::vector<int> chosen;
          for (const std::vector<int>& ss : small_slice_set) {
            int64_t sum_max_mem = 0;
            for (int p : ss) sum_max_mem += tb.cap(p);
            if (sum_max_mem * 1000 >= g.pred_mem) {
              chosen = ss;
              found = true;
              break;
            }
          }
          const int64_t pot_occupancy = g.pred_num;  // line 13 (R13)
          const int64_t T_low = cfg.t_low, T_high = cfg.t_high;  // lines 14-15 (R14)
          // lines 19-23 (after the loop, reading Q26)
          std::vector<int> final_geometry;
          if (!found || pot_occupancy < T_low || pot_occupancy > T_high) {
            final_geometry = {2, 3};  // (4g,3g)
          } else {
            final_geometry = chosen;
            final_geometry.push_back(3);  // + 4g
          }
          std::sort(final_geometry.begin(), final_geometry.end());
          int fin = -1;
          for (int j = 0; j < G && fin < 0; ++j)
            if (tb.geoms[j] == final_geometry) fin = j;  // present: checked by the API (R15)
          best[n] = fin;
          out->decisions[(size_t)e * N + n] = (uint8_t)fin;
          // lines 24-30 (reading Q22)
          if (fin != cur) {
            if (g.ctr >= cfg.wait_limit) wants.push_back(n);
            else g.ctr += 1;
          } else {
            g.ctr = 0;
          }
        }
      }
      if (cfg.policy == 0) {
        for (int n = 0; n < N; ++n) {
          Gpu& g = gpu[n];
          if (!(has_vm(g, T) && g.re <= T)) continue;
          const int cur = g.S.geom;
          for (int j = 0; j < G; ++j) {
            GpuState C;  // idle GPU in geometry j (reading Q19)
            C.geom = j;
            int64_t misses = 0, tail = 0;
            for (size_t x : list[n]) {
              const Batch& b = batches[x];
              PlaceOut po = place(tb, tb.geoms[j], C, b.ready, b.model, b.strict, cfg.max_live,
                                  nullptr, H);
              if (po.dropped != 3)  // h5 self-check: co-location pressure on the scored slices
                for (size_t s = 0; s < tb.geoms[j].size(); ++s)
                  if (po.feasible[s]) {
                    out->stats[3] += 1;
                    if (po.s_F[s] > kPpm) out->stats[2] += 1;
                  }
              if (b.strict) {
                if (po.dropped) {
                  misses += b.n;
                } else {
                  int64_t hits = 0;
                  for (uint32_t a : b.arr)
                    if (po.end - (int64_t)a <= tb.slo[b.model]) hits++;
                  misses += b.n - hits;
                }
              } else {
                int64_t t_b = po.dropped ? (int64_t)kSat32 : po.end - (int64_t)b.arr[0];
                tail = std::max(tail, t_b);
              }
            }
            int64_t key = make_key(misses, tail, j == cur ? 0 : j + 1);
            out->counters[8] += (int64_t)list[n].size() * (int64_t)tb.geoms[j].size();
            out->counters[9] += 1;
            if (want_keys) out->cand_keys[((size_t)e * N + n) * G + j] = key;
            if (key_best[n] < 0 || key < key_best[n]) key_best[n] = key;
            if (j == cur) key_cur[n] = key;
          }
          const int tag = (int)(key_best[n] & 255);
          best[n] = tag == 0 ? cur : tag - 1;
          out->stats[0] += 1;
          if (tag != 0) out->stats[1] += 1;
          out->decisions[(size_t)e * N + n] = (uint8_t)best[n];
          // Alg 2 lines 24-30, reading Q22
          if (best[n] != cur) {
            if (g.ctr >= cfg.wait_limit) wants.push_back(n);
            else g.ctr += 1;
          } else {
            g.ctr = 0;
          }
        }
      }
      if (cfg.policy != 1) {
        // ~30% of GPUs may reconfigure simultaneously, reading Q23; under policy 2 there
        // is no miss estimate, so the order is by GPU only (R16)
        int alive = 0, open = 0;
        for (int n = 0; n < N; ++n) {
          if (has_vm(gpu[n], T)) alive++;
          if (gpu[n].re > T) open++;
        }
        int cap = std::max(1, cfg.cap_pct * alive / 100);
        int free_slots = std::max(0, cap - open);
        std::stable_sort(wants.begin(), wants.end(), [&](int a, int b) {
          int64_t da = cfg.policy == 0 ? (key_cur[a] >> 40) - (key_best[a] >> 40) : 0;
          int64_t db = cfg.policy == 0 ? (key_cur[b] >> 40) - (key_best[b] >> 40) : 0;
          if (da != db) return da > db;
          return a < b;
        });
        for (int i = 0; i < (int)wants.size() && i < free_slots; ++i) {
          Gpu& g = gpu[wants[i]];
          int64_t drain_end = T;  // the GPU must be idle to reconfigure
          for (const Resident& r : g.S.res) drain_end = std::max(drain_end, r.end);
          g.rs = T;
          g.re = drain_end + cfg.reconfig_us;  // ~2 s downtime
          g.target = best[wants[i]];
          out->counters[7] += 1;
        }
      }
    }

    // (delayed termination runs inside the epoch loop, see terminate_surplus)
    // close billing at H and finalize (O12)
    for (int n = 0; n < N; ++n) bill_switch(gpu[n].node, VM_NONE, H);
    out->accum[0] = acc.busy_w;
    out->accum[1] = acc.mem_num;
    for (int c = 0; c < 2; ++c) {
      out->p[c][0] = (int64_t)percentile(&out->hist[c * kBuckets], 50);
      out->p[c][1] = (int64_t)percentile(&out->hist[c * kBuckets], 99);
    }
    out->cost = ((double)out->accum[2] * cfg.price_od + (double)out->accum[3] * cfg.price_spot) / 3.6e9;
    out->util[0] = (double)out->accum[0] / (7.0 * (double)N * (double)H);
    out->util[1] = (double)out->accum[1] / ((double)tb.gpu_mem * (double)N * (double)H);
  }
};
}  // namespace

void replay_replica(const Tables& tb, const ReplayCfg& cfg, uint64_t replica_id,
                    const uint32_t* arrival, const uint8_t* meta, int64_t n, bool want_keys,
                    bool want_log, ReplayOut* out) {
  const int64_t E = num_epochs(tb, cfg.trace_len, cfg.W);
  std::vector<Batch> batches = form_batches(tb, arrival, meta, n);
  Replay rp(tb, cfg, replica_id, E * cfg.W, out);
  rp.run(batches, E, want_keys, want_log);
  out->n_batches = (int64_t)batches.size();
}

}  // namespace pem
