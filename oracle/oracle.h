/* oracle/oracle.h — TEST INFRASTRUCTURE ONLY.
 *
 * C interface of the CPU oracle (plain C++17 reading of the PROTEAN epoch model, see pem.hpp and
 * DESIGN.md).  Loaded by tests/ (via oracle/oracle.py), __graft_entry__.smoke() and bench.py's
 * cpu_baseline / --impl reference legs only.  Independent of include/protean.h: its own structs,
 * its own validation (same numeric error codes, defined here separately).  Host pointers only.
 */
#ifndef PEM_ORACLE_H_
#define PEM_ORACLE_H_
#include <stdint.h>
#ifdef __cplusplus
extern "C" {
#endif

enum { ORC_OK = 0, ORC_EINVAL = -1, ORC_ERANGE = -2, ORC_ENOMEM = -3, ORC_EUNSUP = -7 };

typedef struct {
  int32_t M;
  const int32_t *solo, *fbr;      /* [M][5] */
  const int32_t *mem, *bsz, *slo, *tmo;  /* [M] */
  int32_t geometry_set;           /* 0: 12 multiset-maximal, 1: all 37, 2: explicit */
  int32_t n_geoms;
  const uint8_t *geoms;           /* explicit: [G][8] */
  int32_t gpu_mem_mib;            /* N4c: GPU memory (0 = A100-40GB 40960); profile p holds
                                     gpu_mem * {1,2,4,4,8}[p] / 8; multiple of 8, <= 2^24 */
} orc_tables;

typedef struct { int64_t start, end; int32_t mem, slice, model, strict; } orc_res;  /* 32 B */

typedef struct {
  int32_t geom, target, wait_ctr, has_vm;
  int64_t recfg_start, recfg_end;
  int64_t last_start[7], busy_until[7], busy_us[7];
  int32_t vm_type;                /* 0 none, 1 on-demand, 2 spot (billing type this epoch) */
  int32_t n_res;
  orc_res res[64];
} orc_state;

/* O2.  stats = {feasible, maximal placements, placement-maximal multisets, multiset-maximal}. */
int orc_enumerate(int32_t set, int32_t *n, uint8_t *out, int32_t *stats);
/* geometry table a tables struct resolves to (after validation) */
int orc_table_geometries(const orc_tables *t, int32_t *n, uint8_t *out);

int64_t orc_exec_us(int64_t solo, int64_t F_ppm);

/* O6 on an explicit state; diagnostics per slice position.  accum[2] += busy_w, mem_num. */
int orc_place(const orc_tables *t, orc_state *S, int64_t t_ready, int32_t model, int32_t strict,
              int32_t max_live, int64_t H, int32_t *slice, int64_t *start, int64_t *end,
              int32_t *dropped, int64_t *s_start, int64_t *s_end, int32_t *feasible,
              int32_t *eligible, int64_t *accum);

/* O3; returns the number of batches (id order), writes at most cap rows; < 0 on error. */
int64_t orc_form_batches(const orc_tables *t, const uint32_t *arrival, const uint8_t *meta,
                         int64_t n, uint32_t *ready, int32_t *nreq, int32_t *model,
                         int32_t *strict, int64_t *first_raw, int64_t cap);

/* Second formulation of O6a/b: 1-us time-stepped FIFO simulator with fixed slice choices. */
int orc_tick_simulate(const orc_tables *t, int32_t geom, int32_t nb, const int64_t *t_ready,
                      const int32_t *model, const int32_t *slice, int64_t *start, int64_t *end);

int32_t orc_bucket(uint64_t x);
uint64_t orc_bucket_lower(int32_t b);
uint64_t orc_percentile(const uint32_t *hist, int32_t q_percent);
uint64_t orc_vm_draw(uint64_t seed, uint64_t replica, uint64_t node, uint64_t k, uint64_t d);
int64_t orc_key(int64_t misses, int64_t tail, int32_t tag);
int64_t orc_num_epochs(const orc_tables *t, int64_t trace_len, int64_t W);

typedef struct {
  int32_t R, N;
  int64_t replica_base, trace_len, W;
  const uint32_t *arrival; const uint8_t *meta; const int64_t *replica_off;
  int32_t policy, wait_limit, cap_pct, init_geom, max_live, vm_policy;
  int64_t reconfig_us;
  double p_rev, price_od, price_spot;
  int64_t rev_interval, notice;
  uint64_t seed;
  int32_t shard_mode, nthreads;
  int32_t ewma_alpha_pm, pad;   /* policy 2 (N1): EWMA weight per mille, 1..1000 */
  int64_t t_low, t_high;        /* policy 2: T_low <= T_high, milli-BE-batches per epoch */
  int64_t cold_us;              /* N3: container cold start (0 = warm containers, Q15) */
  int32_t keepalive_epochs;     /* N3: delayed termination after this many surplus epochs, >= 1 */
  int32_t prewarm;              /* N3: idle containers per (sim-GPU, model) at t = 0, 0..128 */
} orc_replay_in;

typedef struct {
  uint32_t ready, epoch; int32_t n, model, strict, gpu, slice, dropped; int64_t start, end;
} orc_batch_rec;  /* 48 B */

typedef struct {
  int64_t *counters;   /* [R][10] */
  int64_t *accum;      /* [R][4] */
  uint32_t *hist;      /* [R][2][3328] */
  int64_t *p50_p99;    /* [R][2][2] */
  double *cost;        /* [R] */
  double *util;        /* [R][2] */
  uint8_t *decisions;  /* [R][E][N] or NULL */
  int64_t *cand_keys;  /* [R][E][N][G] or NULL */
  orc_batch_rec *log;  /* [R][log_cap] or NULL */
  int64_t log_cap;
  int64_t *n_batches;  /* [R] or NULL */
  int64_t *cold_starts; /* [R] or NULL (N3) */
  int64_t *stats;       /* [R][4] or NULL: workload self-checks, not a method output:
                           0 decidable GPU-epochs scored, 1 of them with best != current geometry,
                           2 candidate (batch, feasible slice) evaluations with Eq 1's F > 10^6,
                           3 candidate (batch, feasible slice) evaluations */
} orc_replay_out;

int orc_replay(const orc_tables *t, const orc_replay_in *in, orc_replay_out *out);

/* One epoch (O5 steps 3-4) on given batches.  Batches are SoA, ordered by (replica, gpu, id). */
int orc_score_epoch(const orc_tables *t, int32_t R, int32_t N, int32_t epoch, int32_t max_live,
                    int64_t W, int64_t H, const uint32_t *b_ready, const uint32_t *b_req_off,
                    const int32_t *b_n, const int32_t *b_model, const int32_t *b_strict,
                    const int32_t *batch_off, const uint32_t *arrival, orc_state *state,
                    int32_t geom_lo, int32_t geom_hi, int64_t *best_key, int64_t *cand_key,
                    int64_t *p_start, int64_t *p_end, int32_t *p_slice, int32_t *p_dropped,
                    int64_t *counters, int64_t *accum, double price_od, double price_spot,
                    double *cost);

/* O3 batch formation + O5.2 round-robin dispatch for epochs [e_lo, e_hi) (the form_batches
 * helper of SURVEY §8(b)): rows ordered by (replica, epoch, gpu, batch id), batch_off CSR over
 * (replica, epoch - e_lo, gpu); avail [R][N][2] {from, until} or NULL (always available); dispatch
 * drops are not emitted.  members: every row's member arrivals, contiguous and ascending, at
 * req_off.  *n_rows: capacity in, rows out (ERANGE if too small, *n_rows = rows needed). */
int orc_form_dispatch(const orc_tables *t, int32_t R, int32_t N, int64_t W, int64_t trace_len,
                     const uint32_t *arrival, const uint8_t *meta, const int64_t *replica_off,
                     int32_t e_lo, int32_t e_hi, const int64_t *avail, uint32_t *b_ready,
                     uint32_t *b_req_off, int32_t *b_n, int32_t *b_model, int32_t *b_strict,
                     int32_t *b_gpu, int32_t *batch_off, int64_t *n_rows, uint32_t *members,
                     int64_t members_cap);

/* N4a exhaustive assignment sweep (readings R18-R21): per (replica, gpu) and geometry j in
 * [geom_lo, geom_hi) the min key over every assignment of the GPU's batches (<= max_batches <= 8)
 * to j's slices, scheduled from idle with the slice forced; assign = slice of batch x in bits
 * 3x..3x+2 of the lowest-index minimiser; best_key = min over the range, tag 0 when j == cur_geom. */
/* N4b: BE-reserve depths (reading R28): per (replica, gpu, geometry j in range) the keys of Alg 1
 * replays from idle with strict eligibility "position >= d" for d = 0..S_j-1, plus the tag walk
 * (code 0); depth_key [R*N*nc][8] (code 0 = auto, 1 + d; -1 beyond S_j), depth_code = argmin code
 * (ties -> lowest code), best_key = min over the range; n_eval += replays. */
int orc_sweep_depths(const orc_tables *t, int32_t R, int32_t N, int32_t max_live,
                     const uint32_t *b_ready, const uint32_t *b_req_off, const int32_t *b_n,
                     const int32_t *b_model, const int32_t *b_strict, const int32_t *batch_off,
                     const uint32_t *arrival, const uint8_t *cur_geom, int32_t geom_lo, int32_t geom_hi,
                     int64_t *depth_key, uint8_t *depth_code, int64_t *best_key, int64_t *n_eval);
int orc_sweep(const orc_tables *t, int32_t R, int32_t N, int32_t max_live, int32_t max_batches,
              const uint32_t *b_ready, const uint32_t *b_req_off, const int32_t *b_n,
              const int32_t *b_model, const int32_t *b_strict, const int32_t *batch_off,
              const uint32_t *arrival, const uint8_t *cur_geom, int32_t geom_lo, int32_t geom_hi,
              int64_t *sweep_key, uint32_t *assign, int64_t *best_key, int64_t *n_assign);

#ifdef __cplusplus
}
#endif
#endif
