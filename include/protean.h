/*
 * protean.h — C ABI of the B200-native PROTEAN placement scorer and trace replayer.
 *
 * What this library computes is the "PROTEAN epoch model" (PEM): the paper's slowdown model
 * (Eq 1 / Eq 2), Job Distribution (Alg 1), the GPU Reconfigurator's decision step (Alg 2,
 * hysteresis + ~30% cap) and cost-aware procurement, driven by an exhaustive per-epoch search
 * over MIG geometries (the paper's "Oracle" scheme run online) or by Alg 2's own heuristic
 * (policy 2), optionally with the Autoscaler's container pools and cold starts; plus the
 * exhaustive assignment sweep (section 3b) and a batch formation / dispatch helper (3a).
 * Entry points: protean_load_profiles, protean_score_epoch, protean_replay_traces,
 * protean_form_batches, protean_sweep_assignments, the mode-G exchange set-up (section 4) and
 * small helpers (errors, geometries, epochs, timings, defaults).  Paper citations are
 * "P:L<n>" = line n of PAPER.md (Bhasi et al., "Towards SLO-Compliant and Cost-Effective
 * Serverless Computing on Emerging GPU Architectures", MIDDLEWARE '24).  Every reading of a
 * silent / ambiguous passage is listed in DESIGN.md §3 (Q1..Q39 follow SURVEY.md §8(c)).
 *
 * Units everywhere: time in integer microseconds (int64 inside, uint32 for stored arrivals and
 * batch ready times), memory in MiB, fractional bandwidth (FBR) in ppm (10^6 == 1.0), prices
 * in USD per node-hour.  No floating point enters any decision; cost and utilisation are
 * converted to double once, from integer accumulators.
 *
 * Ownership: the caller owns every input and output buffer.  The library owns only the handle,
 * its device copy of the tables, its scratch memory and (mode G / virtual ranks) its exchange
 * buffers; all are released by protean_free().  The library never frees or reallocates caller memory.
 *
 * Pointers: every pointer inside protean_epoch_in / protean_epoch_out / protean_replay_cfg /
 * protean_replay_out is a DEVICE pointer (cudaMalloc'd or torch CUDA tensor data) on the
 * handle's device, unless the field comment says "host".  protean_profiles holds host pointers.
 *
 * Errors: every call returns an int code (PROTEAN_OK == 0 or a negative PROTEAN_E*).  There are
 * no exceptions or aborts across the ABI.  On a non-OK return the outputs are undefined.
 * PROTEAN_ECUDA / PROTEAN_ENCCL poison the handle: every later call returns PROTEAN_ESTATE until
 * protean_free().  protean_last_error() gives a human-readable detail of the last failure.
 *
 * Threading: a handle is not thread-safe; distinct handles are independent.
 */
#ifndef PROTEAN_H_
#define PROTEAN_H_

#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

#define PROTEAN_ABI_VERSION 1

enum {
  PROTEAN_OK = 0,
  PROTEAN_EINVAL = -1,  /* bad pointer / size / ordering / value (e.g. unsorted arrivals,
                           model id >= n_models, fbr > 10^6, solo <= 0, geometry violating T2) */
  PROTEAN_ERANGE = -2,  /* a value does not fit its field: time >= 2^32 us in a uint32 field,
                           n_gpus > 255, G > 254, live residents > max_live in a given state */
  PROTEAN_ENOMEM = -3,  /* device / host allocation failed */
  PROTEAN_ECUDA = -4,   /* a CUDA runtime call failed (handle poisoned) */
  PROTEAN_ENCCL = -5,   /* a cross-rank exchange failed or timed out (handle poisoned) */
  PROTEAN_ESTATE = -6,  /* handle poisoned, or bad call order */
  PROTEAN_EUNSUP = -7   /* valid request this build does not implement (reserved) */
};

/* MIG slice profiles of the A100-40GB, T2, in ascending-resource order (the order
 * Alg 1 walks; 3g < 4g by compute since both hold 20 GB, reading Q3).
 *   compute (sevenths) 1,2,3,4,7;  memory MiB 5120,10240,20480,20480,40960;  max count 7,3,2,1,1 */
enum { PROTEAN_P_1G = 0, PROTEAN_P_2G, PROTEAN_P_3G, PROTEAN_P_4G, PROTEAN_P_7G, PROTEAN_NPROF };

#define PROTEAN_MAX_MODELS 64
#define PROTEAN_MAX_SLICES 7      /* a geometry has at most 7 slices (T2: "maximum of 7") */
#define PROTEAN_MAX_LIVE 64       /* max live batches per simulated GPU (reading Q39) */
#define PROTEAN_NBUCKETS 3328     /* log-linear latency histogram buckets (O7, reading Q30) */
#define PROTEAN_NCOUNTERS 10
#define PROTEAN_NACCUM 4

typedef struct protean_handle protean_handle;

/* ---------------------------------------------------------------------------------------------
 * 1. Profiles: per model x per slice profile tables + the candidate geometry set.
 *    Solo/FBR per slice are the "prerequisites ... estimated through profiling";
 *    FBR = bw*sm of Eq 1; RDF = solo[p]/solo[7g].
 *    All pointers are HOST pointers; the library copies them.                                  */
typedef struct {
  int32_t abi_version;             /* must be PROTEAN_ABI_VERSION */
  int32_t n_models;                /* M, 1..64 */
  const int32_t *solo_us;          /* [M][5] solo (isolated) batch exec time per profile, > 0 */
  const int32_t *fbr_ppm;          /* [M][5] fractional bandwidth requirement per profile, 0..10^6 */
  const int32_t *mem_mib;          /* [M] memory footprint of one batch, 1..gpu_mem_mib (40960) */
  const int32_t *batch_size;       /* [M] B_m, 1..65535 (128 vision, 4 language) */
  const int32_t *slo_us;           /* [M] strict SLO, > 0 (paper: 3 x solo on 7g) */
  const int32_t *batch_timeout_us; /* [M] T_m >= 0: a batch closes at B_m requests or first+T_m (Q14) */
  int32_t geometry_set;            /* 0: the 12 multiset-maximal geometries (default)
                                      1: all 37 feasible geometries
                                      2: explicit list (geoms) */
  int32_t n_geoms;                 /* explicit only: G, 1..254 */
  const uint8_t *geoms;            /* explicit only: [G][8] profile ids ascending, 0xFF padded;
                                      each validated against T2 (counts, compute <= 7/7, mem <= 40 GB) */
  int32_t device;                  /* CUDA device ordinal */
  int32_t gpu_mem_mib;             /* N4c, MIG profile table of the simulated GPU (P:L495
                                      "Generalizability"; NVIDIA's MIG tables, not in the paper):
                                      its memory in MiB, a multiple of 8, <= 2^24.  Profile p holds
                                      gpu_mem * {1,2,4,4,8}[p] / 8 MiB; compute sevenths, max counts
                                      and hence the geometry sets are T2's.  0 = A100-40GB (40960);
                                      81920 = A100-80GB / H100-80GB, 144384 = H200-141GB,
                                      184320 = B200-180GB (nominal GiB x 1024).  The double-memory
                                      1g profiles (1g.20gb, 1g.45gb) are not modelled.  Footprints
                                      (mem_mib) must be <= gpu_mem_mib; mem utilisation divides by it. */
} protean_profiles;

/* Validates the tables, enumerates the geometry set (canonical order: count vectors
 * (c7g,c4g,c3g,c2g,c1g) descending lexicographically; index 0 = (7g), 1 = (4g,3g),
 * 2 = (4g,2g,1g) in both built-in sets), uploads everything to the device and returns a handle.
 * Synchronous.  Errors: EINVAL (bad table value / pointer / geometry), ERANGE (G > 254),
 * ENOMEM, ECUDA. */
int protean_load_profiles(const protean_profiles *p, protean_handle **out);
void protean_free(protean_handle *h);
const char *protean_strerror(int code);
const char *protean_last_error(const protean_handle *h);

/* Geometry table of the handle: *n_geoms = G; if geoms != NULL it receives [G][8] host bytes
 * (profile ids ascending, 0xFF padded).  Host pointers. */
int protean_get_geometries(const protean_handle *h, int32_t *n_geoms, uint8_t *geoms);

/* Number of epochs of a replay: E = ceil(trace_len/W) + ceil(max_m T_m / W) (O4).  Host. */
int protean_num_epochs(const protean_handle *h, int64_t trace_len_us, int64_t epoch_len_us,
                       int64_t *n_epochs);

/* ---------------------------------------------------------------------------------------------
 * 2. One epoch of the search for R replicas x N simulated GPUs (§8(a) S4, S6, S7, S8).
 *    For every GPU: the pending reconfiguration is installed if recfg_end <= T = (epoch+1)W;
 *    its batches are placed on its CURRENT geometry with Alg 1 on the carried state (the actual
 *    placement, which advances `state`); and if the GPU is decidable at T (has_vm and
 *    recfg_end <= T) every candidate geometry j in [geom_lo, geom_hi) replays the same batch list
 *    from an idle GPU and is scored by key = misses<<40 | BE_tail<<8 | tag, tag 0 = current
 *    geometry, else j+1 (O8); each node-epoch's VM cost price(vm_type) x W is reported (T3,
 *    P:L173-179; cost projection P:L333; reading Q35: reported, not keyed).
 *    Enqueue-only: validation runs in the kernel and the call returns once the work is enqueued on
 *    `stream` (cudaStream_t; NULL = legacy default); outputs (and `state`) are valid after a sync of
 *    that stream.  The kernel's validation verdict (EINVAL: bad state / batch / offsets; ERANGE:
 *    n_live > max_live) is latched in a device word of the handle: protean_score_epoch_status()
 *    reads it after the caller's sync.  An invalid CTA (replica) writes none of its outputs and
 *    leaves its states untouched.  Host-detectable argument errors are still returned directly. */
typedef struct {           /* 16 B */
  uint32_t ready_us;       /* batch ready time (O3): last member's arrival if full, else first + T_m */
  uint32_t req_off;        /* index of the batch's first member in arrival_us */
  uint16_t n_req;          /* members; they are arrival_us[req_off .. req_off + n_req), sorted */
  uint8_t model;           /* model id < M */
  uint8_t strict;          /* 1 = strict (SLO), 0 = best effort (BE) */
  uint32_t gpu;            /* informational: the GPU it was dispatched to */
} protean_batch;

typedef struct {           /* 24 B: one batch resident on a simulated GPU */
  int64_t start_us, end_us;/* [start, end) on its slice; end = start + exec (Eq 1, frozen at start) */
  int32_t mem_mib;
  uint8_t slice;           /* slice position within the geometry (ascending profile order) */
  uint8_t model, strict, pad;
} protean_resident;

typedef struct {           /* one simulated GPU's carried state; caller-allocated */
  uint8_t geom;            /* current geometry index */
  uint8_t target;          /* pending reconfiguration target, 0xFF = none */
  uint8_t wait_ctr;        /* Alg 2 wait_ctr — not modified by score_epoch */
  uint8_t n_live;          /* residents in live[] (<= max_live) */
  uint8_t has_vm;          /* 1 = the node holds a VM at the decision time */
  uint8_t vm_type;         /* billing type of the node's VM this epoch: 0 none, 1 on-demand, 2 spot */
  uint8_t pad[2];
  int64_t recfg_start_us, recfg_end_us;  /* reconfiguration window [start, end), 0/0 = none */
  int64_t last_start_us[PROTEAN_MAX_SLICES];   /* FIFO: latest start on each slice */
  int64_t busy_until_us[PROTEAN_MAX_SLICES];   /* busy-time union bookkeeping (O6e) */
  int64_t busy_us[PROTEAN_MAX_SLICES];         /* ACCUMULATED busy us of each slice instance: the
                                                  union of its batches' [start, end) clipped to
                                                  [0, H) (O6e, "percentage non-idle time");
                                                  cleared with the state on a reconfiguration install */
  protean_resident live[PROTEAN_MAX_LIVE];  /* the live residents as a set: order unspecified
                                               (score_epoch writes them back grouped by slice) */
} protean_gpu_state;

typedef struct {           /* 24 B */
  int64_t start_us, end_us;
  uint8_t slice;           /* chosen slice position (valid when dropped == 0) */
  uint8_t dropped;         /* 0 placed, 2 placement drop (no slice fits), 3 overflow (max_live) */
  uint8_t pad[6];
} protean_placement;

typedef struct {
  int32_t n_replicas, n_gpus, epoch;   /* R >= 1, 1 <= N <= 255, epoch >= 0 */
  int32_t max_live;                    /* 1..64 (default 64) */
  int64_t epoch_len_us;                /* W > 0 */
  int64_t horizon_us;                  /* H: busy/memory accounting is clipped to [0, H) */
  const protean_batch *batches;        /* ordered by (replica, gpu, batch id) */
  const int32_t *batch_off;            /* [R*N+1] CSR offsets into batches */
  const uint32_t *arrival_us;          /* member arrivals referenced by req_off */
  protean_gpu_state *state;            /* [R*N] in/out */
  int32_t geom_lo, geom_hi;            /* candidate range; [0, G) = all */
  double price_od_node_hr;             /* USD per node-hour of an on-demand VM (T3 / 8, Q27), >= 0 */
  double price_spot_node_hr;           /* USD per node-hour of a spot VM, >= 0 */
} protean_epoch_in;

typedef struct {
  int64_t *best_key;          /* [R*N] min key over the range; -1 if the GPU is not decidable */
  int64_t *cand_key;          /* [R*N*(hi-lo)] every candidate key (-1 if not decidable), or NULL */
  protean_placement *placement; /* [n_batches] actual placement, same order as batches */
  int64_t *counters;          /* [R][10] ACCUMULATED (+=): see protean_replay_out.counters */
  int64_t *accum;             /* [R][4] ACCUMULATED, or NULL: busy_w, mem_num (see replay) */
  double *cost_usd;           /* [R*N] node-epoch VM cost, or NULL: has_vm ? price(vm_type) * W /
                                 3.6e9 : 0, evaluated as (price * (double)W) / 3.6e9 */
} protean_epoch_out;

int protean_score_epoch(protean_handle *h, const protean_epoch_in *in, protean_epoch_out *out,
                        void *stream);

/* Verdict of the score_epoch calls enqueued since the last status call (host; synchronises the
 * handle's device): PROTEAN_OK, or EINVAL / ERANGE if any enqueued kernel rejected its input (the
 * detail goes to protean_last_error).  Clears the latched word. */
int protean_score_epoch_status(protean_handle *h);

/* ---------------------------------------------------------------------------------------------
 * 3. Trace replay, epoch by epoch, of many independent replicas (the north-star path, §8(a)
 *    S2..S11 fused).  Per replica, for e = 0..E-1 (O5): VM events -> batch formation (O3) ->
 *    round-robin dispatch (Q18) -> actual Alg-1 placement + per-request accounting (O6, O7) ->
 *    candidate scoring of every geometry for every decidable GPU (O8) -> hysteresis + 30% cap +
 *    reconfiguration windows (O9, O10).  Then percentiles, cost and utilisation (O12).
 *    Synchronous (returns after the outputs are written).                                      */
typedef struct {
  int32_t n_replicas;          /* replicas in THIS call */
  int32_t n_gpus;              /* N simulated GPUs per replica, 1..255 */
  int64_t replica_base;        /* global id of the first replica (RNG stream of O11); mode R
                                  sharding passes each rank its own slice of replicas */
  int64_t trace_len_us;        /* arrivals lie in [0, trace_len) */
  int64_t epoch_len_us;        /* W, Monitor_Interval of Alg 2; default 1'000'000 (Q1) */
  const uint32_t *arrival_us;  /* device: per replica, sorted non-decreasing */
  const uint8_t *meta;         /* device: bits 0..5 model id, bit 7 strict (user-annotated) */
  const int64_t *replica_off;  /* device: [R+1] offsets into arrival_us / meta */
  int32_t policy;              /* 0 = geometry search (default); 1 = fixed geometry (no search);
                                  2 = Alg 2 heuristic (N1, R10-R17): EWMA of
                                  the observed BE load -> small-slice set -> T_low/T_high ->
                                  (4g,2g,1g) or (4g,3g); EINVAL if the geometry set lacks either */
  int32_t wait_limit;          /* Alg 2 wait_limit, default 3 (reading Q22) */
  int32_t reconfig_cap_pct;    /* default 30 (reading Q23) */
  int32_t init_geom;           /* default 2 = (4g,2g,1g) (reading Q25) */
  int32_t max_live;            /* 1..64, default 64 */
  int32_t vm_policy;           /* 0 on-demand only; 1 PROTEAN spot + on-demand fallback;
                                  2 spot only */
  int64_t reconfig_us;         /* MIG reconfiguration downtime, default 2'000'000 */
  double p_rev;                /* revocation probability per interval, 0..1 */
  double price_od_node_hr, price_spot_node_hr; /* default AWS T3 / 8: 4.096575, 1.228975 (Q27) */
  int64_t rev_interval_us;     /* revocation interval T_rev (default 300 s, Q28); must be >= W */
  int64_t notice_us;           /* eviction notice (default 30 s); must be < T_rev */
  uint64_t seed;               /* VM RNG seed (O11) */
  int32_t shard_mode;          /* 0 = replicas (mode R); 1 = geometry ranges (mode G, section 4) */
  int32_t rank, nranks;        /* mode G only: must match the handle's exchange set-up */
  int32_t max_ctas;            /* 0 = the resident capacity of the device; else caps the replay
                                  grid (lets several mode-G ranks share one GPU) */
  int32_t ewma_alpha_pm;       /* policy 2: EWMA weight of the newest epoch, per mille, 1..1000
                                  (default 500; R11) */
  int64_t t_low_milli;         /* policy 2: T_low, thousandths of a BE batch per epoch (default 500) */
  int64_t t_high_milli;        /* policy 2: T_high >= T_low (default 4000; R14) */
  int64_t cold_start_us;       /* N3 Autoscaler (R22-R27): container
                                  cold start; 0 (default) = warm containers (reading Q15), no pools.
                                  > 0: per (sim-GPU, model) pools of <= 128 containers, one per
                                  batch; a batch finding none idle waits cold_start_us (PROTEAN_ERANGE
                                  if a pool would exceed 128) */
  int32_t keepalive_epochs;    /* N3: surplus containers terminated after this many consecutive
                                  surplus epochs, >= 1 (default 600 = ~10 min at W = 1 s) */
  int32_t prewarm;             /* N3: idle containers per (sim-GPU, model) at t = 0, 0..128 */
  int32_t ctas_per_replica;    /* search policy, shard_mode 0: CTAs sharing one replica, each scoring
                                  a slot-balanced geometry range and exchanging min-loc keys per
                                  epoch in device memory (mode G inside one launch).  0 = auto
                                  (min(16, G, SMs / replicas) when replicas < SMs, else 1); 1 = off;
                                  k = min(k, 16, G).  Outputs are identical for every setting.  The
                                  CTAs of a replica must run concurrently: a device shared with other
                                  work can delay them past the exchange timeout (PROTEAN_ENCCL). */
  int32_t reserved2;           /* must be 0 */
} protean_replay_cfg;

/* counters[10] per replica (O7/O8/O10):
 *   0 strict_arr  1 strict_met  2 strict_missed  3 strict_drop
 *   4 be_arr      5 be_served   6 be_drop        7 reconfigs
 *   8 slot_evals (sum over candidate x batch of the geometry's slice count)
 *   9 geom_candidates (replica x epoch x decidable GPU x geometry schedules)
 * accum[4] per replica: 0 busy_w  = sum over slices of compute7 x busy us (clipped to [0,H))
 *                       1 mem_num = sum over batches of mem_mib x |[start,end) ∩ [0,H)|
 *                       2 vm_od_us, 3 vm_spot_us (billed node-us over [0,H))              */
typedef struct {
  uint32_t ready_us;
  uint32_t epoch;
  uint16_t n_req; uint8_t model, strict;
  uint8_t gpu, slice, dropped, pad;  /* dropped: 0 placed, 1 dispatch, 2 placement, 3 overflow */
  int64_t start_us, end_us;
} protean_batch_rec;         /* 32 B, debug log of every batch in id order */

typedef struct {             /* caller-allocated, one row per replica of this call */
  int64_t *counters;         /* [R][10] */
  int64_t *accum;            /* [R][4] */
  uint32_t *hist;            /* [R][2][3328] latency histograms (0 strict, 1 BE) */
  int64_t *p50_p99_us;       /* [R][2][2] nearest-rank P50/P99 (bucket lower edges, O12) */
  double *cost_usd;          /* [R] */
  double *util;              /* [R][2]: compute-weighted busy, memory-time */
  uint8_t *decisions;        /* [R][E][N] best geometry per decidable GPU-epoch, 0xFF otherwise;
                                or NULL */
  int64_t *cand_keys;        /* [R][E][N][G] every candidate key (-1 when not scored), or NULL */
  protean_batch_rec *batch_log; /* [R][batch_log_cap] or NULL */
  int64_t batch_log_cap;
  int64_t *n_batches;        /* [R] batches formed (also when batch_log is NULL), or NULL */
  int64_t *cold_starts;      /* [R] N3 cold starts (containers spawned), or NULL */
} protean_replay_out;

int protean_replay_traces(protean_handle *h, const protean_replay_cfg *cfg,
                          protean_replay_out *out, void *stream);

/* Device time (CUDA events on the launching stream) of the last protean_replay_traces call:
 * prepass_ms = the prepass (epoch offsets) + the trace-level stream partition (per-(replica, epoch,
 * stream) counts, run indices, stable scatter into a stream-sorted copy of the arrivals, request
 * validation); replay_ms = the fused replay kernel; launch = {grid, block, dynamic smem bytes,
 * resident CTAs per SM} of the replay kernel (any pointer may be NULL).  Host.
 * Device memory: besides its scratch, a call holds a stream-sorted copy of the arrivals
 * (4 B/request) and two [R][E(+1)][2M] uint32 index tables, grown with the stream-ordered allocator
 * and kept by the handle for the next call. */
int protean_last_timings(const protean_handle *h, float *prepass_ms, float *replay_ms,
                         int32_t *launch);

/* Device time (ms, CUDA events on the call's stream) of the candidate search the last
 * protean_replay_traces ran ahead of its epoch chain: batch-aligned stream cursors (O3)
 * and the O8 keys of every (replica, epoch, residue class, geometry) replayed from idle (Alg 1,
 * P:L251-277; the "Oracle" scheme), used for the epochs whose dispatch is the closed form
 * of Q18 (every sim-GPU available all epoch).  0 when the call scored every epoch inside
 * the chain (mode G, virtual ranks, policy != 0, n_gpus > 32, or PROTEAN_PRECAND=0).  The search
 * holds R*(E+1)*2M uint32 cursors and R*E*N*G int64 keys in handle scratch.  *walk_ms (may be
 * NULL) = the cursor pass alone.  When the call ran the lean chain (a warp per replica on the
 * search's id-ordered batch rows; many-replica mode R, policy 0, no container pools, N*G even, no
 * epoch above 96 batches), protean_last_timings' replay_ms is the chain and *acct_ms (may be NULL)
 * the per-request accounting pass after it (O7: histograms, SLO hits, P50/P99); else 0.
 * EINVAL for a NULL handle or search_ms. */
int protean_last_search_ms(const protean_handle *h, float *search_ms, float *walk_ms,
                           float *acct_ms);

/* ---------------------------------------------------------------------------------------------
 * 3c. End-to-end replay from HOST buffers: the computation of protean_replay_traces (mode R), with
 *     cfg->arrival_us, cfg->meta, cfg->replica_off and every output pointer of `out` being HOST
 *     pointers (cand_keys and batch_log must be NULL).  The replicas are cut into `chunks`
 *     contiguous ranges (1..R); chunk k+1's trace is copied host -> device on an internal copy
 *     stream while chunk k replays on `stream`, and chunk k's outputs are copied back on an
 *     internal return stream while chunk k+1 replays (two device staging slots owned by the
 *     handle, grown on demand).  Replicas keep their global ids (replica_base + r), so the outputs
 *     equal one device call over all replicas.  Host trace and output buffers should be
 *     page-locked (cudaHostAlloc / cudaHostRegister) for the copies to overlap; pageable memory is
 *     correct but serialises.  protean_last_timings then reports the device time summed over the
 *     chunks.  Synchronous.  Errors as protean_replay_traces; EINVAL for shard_mode != 0.       */
int protean_replay_traces_host(protean_handle *h, const protean_replay_cfg *cfg,
                               protean_replay_out *out, int32_t chunks, void *stream);

/* Fill a replay config with the defaults listed above (host). */
void protean_replay_cfg_defaults(protean_replay_cfg *cfg);

/* ---------------------------------------------------------------------------------------------
 * 3a. Batch formation + dispatch helper (SURVEY §8(b) protean_form_batches) for callers of
 *     protean_score_epoch: O3 batch formation (a batch of model m closes at B_m requests or at its
 *     first arrival + T_m, reading Q14) and O5.2 batch-level round-robin dispatch over the
 *     sim-GPUs available at the batch's ready time (reading Q18; cursor from epoch 0) for
 *     epochs [e_lo, e_hi) (a batch belongs to epoch ready / W, Q31).  Uses n_replicas, n_gpus,
 *     trace_len_us, epoch_len_us, arrival_us, meta, replica_off of cfg (device); the trace is
 *     validated as by protean_replay_traces.
 *       avail_windows  device int64 [R][N][2] {from, until}: GPU n is available at t iff
 *                      from <= t < until; NULL = always available.  Dispatch drops are not emitted.
 *       batches        device, *n_batches rows of capacity; rows ordered by (replica, epoch, gpu,
 *                      batch id); gpu = the sim-GPU; req_off indexes `members`
 *       batch_off      device int32 [R * (e_hi - e_lo) * N + 1] CSR over (replica, epoch - e_lo, gpu)
 *       n_batches      host: capacity in, rows out (PROTEAN_ERANGE if too small; *n_batches then
 *                      holds the rows needed)
 *       members        device uint32, members_cap >= requests + 4 per replica: the member arrivals
 *                      of every batch, contiguous and ascending (a stream-sorted copy of the
 *                      trace; its layout is otherwise unspecified)
 *     Synchronous.  Host-side scan between the count and write passes; not a bench path.        */
int protean_form_batches(protean_handle *h, const protean_replay_cfg *cfg, int32_t e_lo, int32_t e_hi,
                         const int64_t *avail_windows, protean_batch *batches, int32_t *batch_off,
                         int64_t *n_batches, uint32_t *members, int64_t members_cap, void *stream);

/* ---------------------------------------------------------------------------------------------
 * 3b. Exhaustive assignment sweep (N4a): the paper's "Oracle" scheme, "ideal GPU configurations
 *     ... obtained through multiple offline ... scheduling sweeps".  For every
 *     (replica, sim-GPU) with b <= max_batches dispatched batches of one epoch and every geometry j
 *     in [geom_lo, geom_hi), all S_j^b assignments of the batches to j's slices are scheduled from
 *     idle with the slice forced (Place O6 restricted to that slice: live bound, footprint, FIFO +
 *     memory wait, Eq 1 at the start instant over the slice's co-runners; R18-R21) and
 *     scored with the O8 key; the minimum is kept.  Alg 1's greedy choice is one of the
 *     assignments, so sweep_key[j] never exceeds protean_score_epoch's cand_key[j].
 *     Synchronous (returns after the outputs are written).  Device pointers.                     */
typedef struct {
  int32_t n_replicas, n_gpus;      /* R >= 1, 1 <= N <= 255 */
  int32_t max_live;                /* 1..64 (reading Q39) */
  int32_t max_batches;             /* 1..8: a GPU with more batches -> PROTEAN_ERANGE */
  const protean_batch *batches;    /* ordered by (replica, gpu, batch id); ready non-decreasing per GPU */
  const int32_t *batch_off;        /* [R*N+1] CSR offsets into batches */
  const uint32_t *arrival_us;      /* members referenced by req_off: sorted, each <= the batch's ready */
  const uint8_t *cur_geom;         /* [R*N] current geometry (its key carries tag 0), 0xFF = none */
  int32_t geom_lo, geom_hi;        /* geometry range; [0, G) = all */
} protean_sweep_in;

typedef struct {
  int64_t *sweep_key;   /* [R*N*(hi-lo)] min key over the assignments (tag 0 if j == cur, else j+1), or NULL */
  uint32_t *assign;     /* [R*N*(hi-lo)] the lowest-index minimiser: slice of batch x in bits 3x..3x+2, or NULL */
  int64_t *best_key;    /* [R*N] min over the range */
  int64_t *n_assign;    /* [1] ACCUMULATED (+=): assignments scored, sum over (GPU, j) of S_j^b */
} protean_sweep_out;

/* Errors: EINVAL (sizes, range, null pointers, batch_off[0] != 0 or decreasing, model id >= M,
 * n_req < 1, ready not sorted per GPU, members unsorted or after ready, cur_geom >= G),
 * ERANGE (a GPU with more than max_batches batches).  With several faults, the code of one. */
int protean_sweep_assignments(protean_handle *h, const protean_sweep_in *in, protean_sweep_out *out,
                              void *stream);

/* ---------------------------------------------------------------------------------------------
 * 3c'. BE-reserve depth sweep (N4b; SURVEY §8(f) N4 "BE-reserve depth as an enumerated dimension";
 *     reading R28 of DESIGN.md).  Alg 1 lines 1-8 tag slices from the BE memory in
 *     ascending order and choose_strict_slice avoids the BE-full ones.  Here the reserve is
 *     an enumerated parameter instead: for every (replica, sim-GPU) and every geometry j in
 *     [geom_lo, geom_hi), the GPU-epoch's batches are replayed from idle with Alg 1's greedy Place
 *     (O6) under depth code c: c = 0 keeps the tag walk, c = 1 + d reserves the d smallest slices for
 *     BE (strict eligible on positions >= d; with none eligible, every fitting slice, as Q6), for
 *     d = 0 .. S_j - 1; each replay is scored with the O8 key (tag 0 = current geometry).  Code 0 is
 *     exactly protean_score_epoch's candidate key.  Same input as the assignment sweep (3b);
 *     max_batches is ignored (no batch-count limit).  Synchronous.  Device pointers.
 *     Errors: EINVAL (sizes, range, null pointers, batch_off, model id, n_req, unsorted ready or
 *     members, cur_geom >= G).                                                                  */
typedef struct {
  int64_t *depth_key;   /* [R*N*(hi-lo)][8] key per depth code (-1 for codes beyond S_j), or NULL */
  uint8_t *depth_code;  /* [R*N*(hi-lo)] the minimising code (lowest among equal keys), or NULL */
  int64_t *best_key;    /* [R*N] min over the range and every code */
  int64_t *n_eval;      /* [1] ACCUMULATED (+=): replays scored, sum over (GPU, j) of S_j + 1 */
} protean_depth_out;

int protean_sweep_depths(protean_handle *h, const protean_sweep_in *in, protean_depth_out *out,
                         void *stream);

/* ---------------------------------------------------------------------------------------------
 * 4. Mode G: geometry-range sharding with one min-loc exchange per replica-epoch (SURVEY §8(e),
 *    S8 "argmin over geometries + cross-rank min-loc"; the search is the Oracle's sweep).
 *
 * Rank k of n scores only geometries [bounds[k], bounds[k+1]) of protean_geometry_split and
 * redundantly runs everything else (dispatch, actual placement, accounting, decisions), so no
 * state is exchanged: per (replica, epoch, sim-GPU) each rank contributes its best key and the
 * current geometry's key (INT64_MAX when not in its range), and every rank takes the min of each.
 * The packed key (O8) makes min-loc a plain min, so every rank reaches the decision a 1-rank run
 * reaches: decisions, histograms, counters 0..7 and accumulators are identical to mode R / one
 * rank; counters 8 and 9 count the rank's own candidates (their sum over ranks is the 1-rank
 * value) and cand_keys is written for the rank's range only.
 *
 * The exchange is fused into the replay kernel (no host round trip, no NCCL launch per epoch):
 * every CTA stores its 16-byte (best, current) pairs straight into every rank's exchange buffer
 * (peer stores over NVLink through CUDA IPC mappings), publishes a per-(source rank, replica)
 * sequence number with release semantics at system scope, and reduces after acquiring every
 * source's flag.  Keys are double-buffered by sequence parity; sequence numbers continue across
 * calls, so all ranks must issue the same sequence of mode-G replay calls (same R, N and E), and
 * the kernels of one call must run concurrently (one GPU per rank, or grids that fit together on
 * one GPU: cfg.max_ctas; ranks sharing a process must use non-default streams, since the legacy
 * default stream serialises; the library grows its scratch with the stream-ordered allocator and
 * sets kernel attributes once, so it adds no implicit device-wide synchronisation itself).  A source whose flag does not arrive within 30 s makes the call return
 * PROTEAN_ENCCL (the handle is poisoned).                                                        */

/* Balanced geometry ranges: bounds[0] = 0, bounds[nranks] = G, every range non-empty, cut where
 * the running slice count first reaches k/nranks of the total (slot-balanced; host only, no
 * device needed).  EINVAL for nranks < 1 or nranks > G; geometry set as protean_load_profiles. */
int protean_geometry_split(const protean_profiles *p, int32_t nranks, int32_t *bounds);

/* Allocate (zeroed) this rank's exchange buffer for up to max_replicas replicas per call and
 * max_gpus sim-GPUs, and write its 64-byte cudaIpcMemHandle_t to ipc_handle (host). */
int protean_xchg_export(protean_handle *h, int32_t nranks, int32_t rank, int32_t max_replicas,
                        int32_t max_gpus, void *ipc_handle);

/* Map every rank's buffer: ipc_handles = [nranks][64] bytes gathered from every rank's
 * protean_xchg_export (this rank's own entry is not opened).  Host; synchronous. */
int protean_xchg_import(protean_handle *h, const void *ipc_handles);

/* Single-process set-up: handles[k] is rank k (one handle per rank, any devices that can access
 * each other's memory); allocates and cross-wires all buffers.  Host; synchronous. */
int protean_xchg_attach(protean_handle *const *handles, int32_t nranks, int32_t max_replicas,
                        int32_t max_gpus);

#ifdef __cplusplus
}
#endif
#endif /* PROTEAN_H_ */
