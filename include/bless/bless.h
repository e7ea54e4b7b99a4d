/*
 * bless.h -- C ABI of the B200-native BLESS hot path.
 *
 * BLESS = "Improving GPU Sharing Performance through Adaptive Bubbleless
 * Spatial-Temporal Sharing" (Zhang et al., EuroSys '25).  Citations "L<n>" are
 * lines of that paper's text; "R<n>" are the readings of the paper
 * recorded in DESIGN.md §3.
 *
 * The calls follow the paper's problem statement (L143, L145, L157, L259,
 * L276): an application registers with a GPU quota, its kernels are profiled
 * offline at every SM count, requests are submitted into per-application FIFO
 * queues, a scheduler groups kernels of concurrent requests into kernel squads,
 * picks an execution configuration (no restriction, or a spatial SM split) from
 * the profile, launches the kernels confined to their SM ranges, and the
 * caller polls for completion.
 *
 * Conventions
 *  - One bl_ctx per GPU ("replicating its runtime components for each active
 *    GPU", L171).  device = BL_DEVICE_NONE builds a CUDA-free context that runs
 *    the same C++ scheduler on a virtual clock (CPU parity tests).
 *  - Every call returns bl_status; on failure bl_last_error() returns a
 *    thread-local message.  No C++ exception crosses this boundary.
 *  - All times are int64 nanoseconds.  Host times use bl_now_ns()
 *    (CLOCK_MONOTONIC).  Quotas are converted once to integer parts-per-million;
 *    no floating point enters a scheduling decision.
 *  - Pointers inside bl_op are DEVICE pointers, allocated by the caller
 *    (PyTorch) and BORROWED: they must stay valid until bl_destroy.  All other
 *    pointer arguments are host pointers owned by the caller and only read or
 *    written during the call.
 *  - Thread safety: bl_submit / bl_poll / bl_now_ns may be called from any
 *    thread after bl_start (bl_submit: at most one producer per tenant).
 *    Everything else is single-threaded setup/teardown.
 */
#ifndef BLESS_BLESS_H
#define BLESS_BLESS_H

#include <stddef.h>
#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

#define BL_MAX_TENANTS 16   /* per GPU */
#define BL_MAX_SQUAD 128    /* squad_max upper bound */
#define BL_DEVICE_NONE (-1)

typedef struct bl_ctx bl_ctx;

typedef enum {
  BL_OK = 0,
  BL_PENDING = 1,       /* bl_poll: request not finished yet */
  BL_E_INVALID = -1,    /* bad argument (null pointer, out-of-range index, bad op) */
  BL_E_QUOTA = -2,      /* quota <= 0, > 1, sum > 1 + 1e-9, or < 1 SM after apportionment */
  BL_E_STATE = -3,      /* call not allowed in the current state (see each call) */
  BL_E_CUDA = -4,       /* a CUDA call failed; the ctx is unusable afterwards */
  BL_E_OOM = -5,        /* host/device allocation failed or workspace too small */
  BL_E_FULL = -6,       /* request table / ring full */
  BL_E_NOTFOUND = -7,   /* unknown request id / file */
  BL_E_TIMEOUT = -8     /* bl_drain timed out */
} bl_status;

/* Scheduling policies.  BLESS is the paper's method (§4.3-§4.5).  The others
 * are the in-run baselines of §6.1 (L300-L304) on the same executor/kernels:
 *  ISO/STATIC - each tenant confined to its quota SM range, whole request
 *               launched at arrival (ISO = run with one tenant's sub-trace);
 *  TEMPORAL   - time slices of quota*period on the full GPU (L41, R22);
 *  UNBOUND    - every request launched at arrival on [0,S) (native CUDA
 *               stream concurrency, L103). */
typedef enum {
  BL_POLICY_BLESS = 0,
  BL_POLICY_ISO = 1,
  BL_POLICY_STATIC = 2,
  BL_POLICY_TEMPORAL = 3,
  BL_POLICY_UNBOUND = 4
} bl_policy;

/* R17.  VIRTUAL: 'now' of each decision is the predicted-time chain (exactly
 * the oracle DES); all requests must be submitted before bl_start; on a GPU a
 * squad is never launched before the wall time of its newest arrival.
 * WALL: 'now' = max(host time, predicted end of the in-flight squad); every
 * decision's inputs are logged so the oracle can replay it. */
typedef enum { BL_CLOCK_WALL = 0, BL_CLOCK_VIRTUAL = 1 } bl_clock;

typedef struct {
  int32_t sm_unit;            /* g: SMs per partition (R8; default 4 -> N = 37 on B200) */
  int32_t squad_max;          /* max kernels per squad (L181, L408; R5; default 50) */
  int32_t split_pct;          /* Semi-SP ratio c% (L255; R16; default 50) */
  int32_t seed_all;           /* R6: seed every active request first (default 1) */
  int32_t policy;             /* bl_policy */
  int32_t clock;              /* bl_clock */
  int64_t squad_overhead_ns;  /* VIRTUAL clock: added to 'now' after each squad (L432) */
  int64_t temporal_period_ns; /* TEMPORAL period P (R22; default 2 ms) */
  int32_t temporal_work_conserving; /* 0 = T-cap, 1 = T-wc (R22) */
  int32_t max_inflight_squads;      /* WALL: squads queued on the GPU ahead (default 2) */
  int64_t lookahead_ns;       /* WALL: decide the next squad this long before the
                                 predicted end of the in-flight one (default 20 us) */
  int64_t max_requests;       /* request-table capacity (default 1<<20) */
  int32_t ablate;             /* §6.8 ablation study (L424-L426, reading R32; default 0):
                                 bit 0 = no multi-task scheduler (picks round-robin over
                                 the active requests, one kernel each per round, no
                                 progress order); bit 1 = no execution configuration
                                 determiner (every squad NSP on [0,S)).  BL_E_INVALID
                                 outside 0..3 at bl_create. */
  int32_t sm_limit;           /* f4 SM-count sweep (L420): 0 = all S SMs; else the whole
                                 system (every policy, the profile columns, quota
                                 apportionment, N = sm_limit / g) is restricted to logical
                                 SMs [0, sm_limit) for the run, the way the paper restricts
                                 the GPU with MIG.  BL_E_INVALID at bl_start unless
                                 g <= sm_limit <= S. */
  int32_t squad_max_solo;     /* reading R36 (L57/L121: a request arriving while another
                                 runs alone should get its SMs "instantly"): a squad with a
                                 single active request closes after min(squad_max,
                                 squad_max_solo) kernels, bounding how long an arrival
                                 waits for the next decision; 0 = squad_max (default). */
  int32_t barrier;            /* squad barrier (BLESS policy), bit flags.  0 (default):
                                 every participant of squad s+1 waits for every other
                                 participant of squad s.  Bit 0 (reading R37):
                                 a participant's chain waits for the latest in-flight chain
                                 of every other tenant whose kernels ran on logical SMs its
                                 own kernels will use, so on every SM the squads still run
                                 one after the other.  Bit 1 (reading R38, L57): a request
                                 that arrives while the GPU runs only another tenant's solo
                                 NSP squads is decided at once and its squad does not wait
                                 for them (the solo kernels keep running and share the SMs).
                                 BL_E_INVALID outside 0..3 at bl_create / bl_reset. */
} bl_params;

/* Fill *p with the defaults listed above. */
void bl_params_default(bl_params* p);

/* ---- tenant layers (the applications' kernels, L143 "invoke GPU functions at
 * the granularity of GPU kernels") ------------------------------------------ */
typedef enum {
  BL_OP_GEMM = 0,    /* Y[M,N] = act((X[M,K] W[N,K]^T) * scale + shift + R)          */
  BL_OP_CONV = 1,    /* NHWC conv, KRSC weights, same epilogue                        */
  BL_OP_POOL = 2,    /* max / avg / global-avg pooling, NHWC                          */
  BL_OP_ELTWISE = 3, /* Y = act(X * scale + shift (+ R)), per-channel, any layout      */
  BL_OP_IM2COL = 4,  /* Y[m, k] = im2col of an NHWC input, zero-padded to Kpad columns */
  BL_OP_LAYERNORM = 5, /* Y = LN(X (+ R)) * gamma + beta over the last dim (eps = fparam[0]) */
  BL_OP_ATTENTION = 6, /* per head: O = softmax(Q K^T * scale) V (all-ones mask)          */
  BL_OP_EMBED = 7,     /* Y = LN(word[ids] + pos[0:L] + type[0]) * gamma + beta            */
  BL_OP_DWCONV = 8,    /* depthwise NHWC conv (groups = C), weights [C, R, S, 1] + epilogue */
  BL_OP_VIRTUAL = 15 /* no device work (BL_DEVICE_NONE contexts / profile-only)       */
} bl_op_kind;

typedef enum { BL_F32 = 0, BL_BF16 = 1 } bl_dtype;
typedef enum { BL_ACT_NONE = 0, BL_ACT_RELU = 1, BL_ACT_RELU6 = 2, BL_ACT_GELU = 3 } bl_act;
typedef enum { BL_POOL_MAX = 0, BL_POOL_AVG = 1, BL_POOL_GLOBAL_AVG = 2 } bl_pool_mode;

/* Operation descriptor.  Layouts are row-major, contiguous unless an ld* is
 * given.  Element types: X/W/R/Y in 'dtype'; scale/shift are always fp32
 * per-output-channel vectors (nullable: scale = 1, shift = 0).
 *
 *  GEMM  dims = {M, N, K, ldx(0=K), ldy(0=N), ldr(0=N), split_k(0=auto)}
 *        ptr  = {X, W, scale, shift, R, Y}
 *  CONV  dims = {Nb, H, W, C, K, R, S, stride, pad, groups, ldx(0=C), ldy(0=K)}
 *        ptr  = {X, W(KRSC), scale, shift, R(ld = ldy), Y}
 *        (channel slices: offset the pointers, give ld*)
 *  POOL  dims = {Nb, H, W, C, k, stride, pad, mode(bl_pool_mode), ldy(0=C)}
 *        ptr  = {X, Y}   (ldy: output channel stride of window pools)
 *  ELTWISE dims = {rows, C, ldx(0=C), ldy(0=C)}  ptr = {X, scale, shift, R(ld = ldy), Y}
 *  LAYERNORM dims = {rows, C, ldx(0=C), ldy(0=C)}  ptr = {X, gamma, beta, R(ld = ldx), Y}
 *        fparam[0] = eps (0 -> 1e-12)
 *  ATTENTION dims = {L, heads, dh, ld_qkv, ld_o}  ptr = {QKV, O}
 *        QKV row t = [Q (heads*dh) | K (heads*dh) | V (heads*dh)], head h at
 *        column h*dh of each block; O[t, h*dh + i]; fparam[0] = scale
 *        (0 -> 1/sqrt(dh)); L <= 512, dh = 64
 *  EMBED dims = {L, C, vocab}  ptr = {ids (int32), word [vocab, C], pos [>=L, C],
 *        type [>=1, C], gamma, beta, Y}  fparam[0] = eps (0 -> 1e-12)
 *  DWCONV dims = {Nb, H, W, C, R, S, stride, pad}  ptr = {X, W [C,R,S,1], scale,
 *        shift, R, Y}  (epilogue as CONV)
 *  IM2COL dims = {Nb, H, W, C, R, S, stride, pad, Kpad}  ptr = {X, Y}
 *        Y[(n*OH + oh)*OW + ow, (r*S + s)*C + c] = X[n, oh*stride - pad + r,
 *        ow*stride - pad + s, c] (0 outside the image and for k >= R*S*C);
 *        used for first layers with C < 16 so the conv runs as a tensor-core GEMM
 */
typedef struct {
  int32_t kind;     /* bl_op_kind */
  int32_t dtype;    /* bl_dtype */
  int32_t act;      /* bl_act */
  int32_t flags;    /* reserved, 0 */
  int64_t dims[12];
  void* ptr[8];
  float fparam[4];
} bl_op;

typedef struct {
  uint64_t req;
  int32_t tenant;
  int32_t status;     /* BL_OK or BL_PENDING */
  int64_t arrival_ns; /* as submitted (host clock, or trace time in VIRTUAL) */
  int64_t start_ns;   /* first kernel's first CTA (host clock), or model time */
  int64_t finish_ns;  /* last kernel's last CTA (host clock), or model time */
} bl_req_info;

/* One scheduling decision (BLESS policy), for bit-exact replay by the oracle.
 * config_sp = 0 -> NSP (no spatial restriction), 1 -> SP split p[0..K-1]
 * (partitions of g SMs per participant, participants in tenant-id order). */
typedef struct {
  int64_t now;
  int64_t t_hat;   /* chosen predicted squad duration */
  int64_t t_nsp;   /* Eq. 2 prediction (NSP) */
  int32_t n_active;
  int32_t n_part;
  int32_t config_sp;
  int32_t n_picks;
  int32_t act_tenant[BL_MAX_TENANTS];
  int32_t act_next[BL_MAX_TENANTS];
  int64_t act_arrival[BL_MAX_TENANTS];
  int32_t part_tenant[BL_MAX_TENANTS];
  int32_t part_p[BL_MAX_TENANTS];
  int32_t pick_tenant[BL_MAX_SQUAD];
  int32_t pick_kernel[BL_MAX_SQUAD];
  int16_t pick_lo[BL_MAX_SQUAD];
  int16_t pick_hi[BL_MAX_SQUAD];
} bl_decision;

/* One executed kernel launch (device timestamps converted to host clock). */
typedef struct {
  uint64_t seq;
  int32_t tenant;
  int32_t kernel;
  int16_t lo, hi;     /* logical SM range */
  int32_t nsm;        /* distinct SMs that processed >= 1 tile; -1 = unknown (a light-exit
                         launch older than the last 2^18 of the run: its stats record was
                         reused, so no times or mask are reported) */
  int32_t fallback;   /* bit 0: no in-range CTA ran and the last CTA did the work; bit 1:
                         lingering out-of-range CTAs helped (linger timeout); bit 2: a
                         software-dependency wait timed out and fell back to
                         griddepcontrol.wait (never expected; 0 = clean launch) */
  int64_t start_ns;   /* first tile claimed */
  int64_t end_ns;     /* last CTA exit */
  uint64_t req;
  uint32_t sm_mask[8]; /* logical SMs that processed >= 1 tile (bit i = SM i) */
} bl_launch_rec;

/* One TEMPORAL-policy launch decision (reading R22), for
 * replay by the oracle's slice rule.  Times are ns relative to the loop's
 * start (host clock).  A record is written for every kernel the loop launches. */
typedef struct {
  int64_t t;           /* host time of the decision */
  int64_t gpu_free;    /* predicted time the GPU becomes free before this launch */
  int64_t slice_end;   /* end of the slice the launch is charged to */
  int64_t dur;         /* predicted kernel duration t[j][k][S] */
  int64_t sid;         /* slice id (T-cap: cycle * n_tenants + j; T-wc: turn counter) */
  int64_t last_sid;    /* slice id of the previous launch (-1 before the first) */
  int64_t turn_end;    /* T-wc: end of the running turn before this decision (0 if none) */
  int32_t turn;        /* T-wc: tenant of the running turn before this decision (-1 if none) */
  int32_t work_mask;   /* bit j: tenant j had an active or arrived request at t */
  int32_t tenant, kernel;
  int32_t work_conserving;
  int32_t reserved;
} bl_temporal_rec;

/* Launch descriptor summary of one appended kernel (roofline accounting). */
typedef struct {
  char family[32];     /* e.g. "tc_conv_bf16", "gemv_bf16", "simt_mm_f32" */
  int32_t tiles;       /* work tiles per launch (tile queue length) */
  int32_t grid, block, smem;
  double flops;        /* algorithmic FLOPs per launch */
  double bytes;        /* algorithmic HBM bytes per launch (inputs + weights + outputs once) */
} bl_kernel_info;

/* Device facts from the probe kernel (A1). */
typedef struct {
  int32_t device;
  int32_t sm_count;        /* S */
  int32_t max_smid;        /* %nsmid - 1 */
  int32_t cc_major, cc_minor;
  int32_t tpc_pairs_found; /* cluster-2 probe: pairs whose smids differ by 1 */
  int64_t globaltimer_res_ns; /* smallest observed globaltimer step */
  int64_t clock_offset_ns;    /* globaltimer - host clock */
  int64_t l2_bytes;
  int64_t smem_per_block_optin;
  uint8_t smid_to_lid[256];   /* 255 = not a usable SM */
} bl_device_info;

/* ---- lifecycle ---------------------------------------------------------------
 * bl_create: device >= 0 selects a CUDA device and runs the SM probe (A1);
 * BL_DEVICE_NONE makes a CUDA-free ctx (S, g come from bl_load_profile).
 * workspace/ws_bytes: optional caller-owned device buffer for the launch-slot
 * ring (>= 8 MiB: 2^19 slots x 16 B; more with BLESS_STATS_RING_LOG2); NULL
 * lets the library cudaMalloc it.  Errors: BL_E_INVALID,
 * BL_E_CUDA, BL_E_OOM. */
bl_status bl_create(int device, const bl_params* params, void* workspace, size_t ws_bytes, bl_ctx** out);
bl_status bl_destroy(bl_ctx* ctx);               /* stops threads, frees library memory */
bl_status bl_device_info_get(bl_ctx* ctx, bl_device_info* out);

/* Register an application with a GPU quota in (0, 1] (L143, L157).  Before
 * bl_start only.  Sum of quotas must be <= 1 + 1e-9 (BL_E_QUOTA). */
bl_status bl_register_tenant(bl_ctx* ctx, double quota, const char* name, int* tenant_out);
/* SLO mode (§6.5: "replacing the isolated latency T[n%] in §4.3.1 with
 * the required QoS target").  slo_ns > 0 is the tenant's latency target: the
 * progress order then paces the tenant against tau_prog[k] =
 * floor(tau[k] * slo_ns / T) instead of tau[k] (reading R30), so a tenant
 * with a tight target is scheduled as if it were further behind.  slo_ns = 0
 * restores the default (pace = isolated latency T).  Nothing else changes
 * (quota SMs, predictors, ranges).  Before bl_start; BL_E_INVALID for a bad
 * tenant or slo_ns < 0, BL_E_STATE after bl_start.  A profile file may also
 * carry it ("slo <ns>" after the tenant line; bl_load_profile adopts it). */
bl_status bl_set_tenant_slo(bl_ctx* ctx, int tenant, int64_t slo_ns);
/* Optional: run tenant's kernels on a caller-owned cudaStream_t (torch stream). */
bl_status bl_set_stream(bl_ctx* ctx, int tenant, void* cuda_stream);
/* Append one kernel to the tenant's per-request kernel sequence.  Validates
 * the op and builds its launch descriptor (tiles, grid, TMA maps).  Before
 * bl_start; BL_E_INVALID on a malformed op. */
bl_status bl_append_kernel(bl_ctx* ctx, int tenant, const bl_op* op, int* kernel_idx_out);
/* Run one kernel (not a request) once, unrestricted, on the tenant's stream and
 * wait: parity tests use it to compare a single layer with the oracle. */
bl_status bl_run_kernel(bl_ctx* ctx, int tenant, int kernel_idx, int lo, int hi);
/* Per-request host I/O (the paper's memory-management kernels, L87, L229):
 * when set, every request of the tenant copies in_bytes from host_in to
 * dev_in on the tenant's stream right before its first kernel, and out_bytes
 * from dev_out to host_out right after its last kernel; the request finishes
 * when that copy has landed.  host_in/host_out should be pinned
 * (cudaHostAlloc / torch pin_memory) and stay valid until bl_destroy.
 * Pass in_bytes = out_bytes = 0 to disable.  Before bl_start. */
bl_status bl_set_tenant_io(bl_ctx* ctx, int tenant, const void* host_in, void* dev_in, size_t in_bytes,
                           const void* dev_out, void* host_out, size_t out_bytes);
/* Summary of kernel kernel_idx's launch descriptor.  BL_E_STATE without a device. */
bl_status bl_kernel_info_get(bl_ctx* ctx, int tenant, int kernel_idx, bl_kernel_info* out);

/* ---- offline profiler (L155-L161 §4.2.1; A2) ------------------------------------
 * bl_profile_kernel: time kernel on logical SMs [0, sm_count) with CUDA events:
 * median over 3 batches of the mean of 'reps' back-to-back launches; *d_out =
 * distinct SMs used in an unrestricted run (R19).  bl_profile_tenant fills
 * t[k][s] for every kernel and every s = 1..S.  Before bl_start. */
bl_status bl_profile_kernel(bl_ctx* ctx, int tenant, int kernel_idx, int sm_count, int reps,
                            int64_t* ns_out, int* d_out);
bl_status bl_profile_tenant(bl_ctx* ctx, int tenant, int reps);
/* Direct access to the table: t_ns has S entries (s = 1..S). */
bl_status bl_set_profile_row(bl_ctx* ctx, int tenant, int kernel_idx, const int64_t* t_ns, int d);
bl_status bl_get_profile_row(bl_ctx* ctx, int tenant, int kernel_idx, int64_t* t_ns, int* d);
/* Text format documented in synth/profile.py.  bl_load_profile on a
 * BL_DEVICE_NONE ctx with no tenants also registers the tenants and virtual
 * kernels it describes. */
bl_status bl_save_profile(bl_ctx* ctx, const char* path);
bl_status bl_load_profile(bl_ctx* ctx, const char* path);
/* Derived quantities (R18): SMs per tenant and tau/T (tau[k] at quota SMs). */
bl_status bl_tenant_info(bl_ctx* ctx, int tenant, int* quota_sms, int* n_kernels, int64_t* T_iso_ns);

/* ---- runtime ----------------------------------------------------------------------- */
bl_status bl_start(bl_ctx* ctx);   /* spawns the scheduler/launch thread; requires a full profile */
/* Submit one request (one pass over the tenant's kernel sequence).  WALL: any
 * time after bl_start, arrival_ns = host clock of the arrival.  VIRTUAL: before
 * bl_start, arrival_ns = trace time (non-decreasing per tenant). */
bl_status bl_submit(bl_ctx* ctx, int tenant, int64_t arrival_ns, uint64_t* req_out);
bl_status bl_poll(bl_ctx* ctx, uint64_t req, bl_req_info* out);    /* BL_OK / BL_PENDING */
bl_status bl_drain(bl_ctx* ctx, int64_t timeout_ns);               /* all submitted finished */
bl_status bl_stop(bl_ctx* ctx);
/* Copy out decision records / launch records (from index 'first'). */
bl_status bl_decisions(bl_ctx* ctx, size_t first, bl_decision* buf, size_t cap, size_t* n_out);
bl_status bl_launches(bl_ctx* ctx, size_t first, bl_launch_rec* buf, size_t cap, size_t* n_out);
/* TEMPORAL launch decisions of the last run (policy BL_POLICY_TEMPORAL). */
bl_status bl_temporal_log(bl_ctx* ctx, size_t first, bl_temporal_rec* buf, size_t cap, size_t* n_out);
/* Reset request table, logs and queues (between runs with the same tenants). */
bl_status bl_reset(bl_ctx* ctx, const bl_params* params);

/* ---- pure scheduler entry point (no ctx state; CPU parity) --------------------------
 * decide() of the C++ scheduler on a loaded profile: active arrays of length
 * n_active (tenant ids, arrivals, next kernel indices). */
bl_status bl_decide(bl_ctx* ctx, int64_t now, int n_active, const int32_t* tenants,
                    const int64_t* arrivals, const int32_t* next_kernel, bl_decision* out);

/* Host cost of the C++ scheduler (3.7 + 2 + 1 us per kernel on
 * the paper's host): re-runs decide() 'reps' times on the inputs (now, active
 * set) of each of the n logged records on the calling thread and returns the
 * total wall time and the total number of kernels those decisions picked
 * (so ns/decision = total_ns / (n * reps), ns/kernel = total_ns / total_picks).
 * BL_E_INVALID on a record whose active set does not fit the ctx. */
bl_status bl_time_decide(bl_ctx* ctx, const bl_decision* recs, size_t n, int reps, int64_t* total_ns,
                         int64_t* total_picks);

/* ---- predictor study -------------
 * bl_predict: predicted duration of one squad given as n picks (tenant,
 * kernel) in pick order: p == NULL -> Eq. 2 (NSP, L224, reading R12); else
 * Eq. 1 (L211) for the spatial split p[0..K-1] over the K participants in
 * tenant-id order (partitions of g SMs, each >= 1, summing to N; the last
 * participant gets the remaining S - g*(N - p_last) SMs).  Needs a complete
 * profile; BL_E_INVALID on a bad pick or split.
 * bl_run_squad: executes one squad as given on the device (ctx not started):
 * each participant's picks in pick order on its stream, SM range [lo[i],
 * hi[i]) per pick, all chains released together by one event, every launch
 * stamped; repeated reps times.  makespan_ns = median over reps of (last end
 * - first start); kernel_ns[i] (may be NULL) = median duration of pick i.
 * This is how the study measures NSP, SP, Semi-SP and SEQ squads (L197-L203,
 * L382) against the predictions. */
bl_status bl_predict(bl_ctx* ctx, int n_picks, const int32_t* tenants, const int32_t* kernels, const int32_t* p,
                     int64_t* ns_out);
bl_status bl_run_squad(bl_ctx* ctx, int n_picks, const int32_t* tenants, const int32_t* kernels, const int16_t* lo,
                       const int16_t* hi, int reps, int64_t* makespan_ns, int64_t* kernel_ns);

/* ---- deployment (§4.2.2) --------------------
 * Reading R33.  A tenant's average kernel duration is T_j / m_j (isolated
 * latency at its quota over its kernel count, from the profile).  A set of
 * tenants may share one GPU iff (a) the largest average kernel duration is at
 * most span_x times the smallest (L163: co-locating short-kernel with
 * extremely long-kernel applications starves the former in every squad; the
 * paper's working range is 10 us to 300 us, i.e. span_x = 30), and (b) their
 * memory fits the device's free memory (L169).
 * bl_deployment_check: the ctx's registered, profiled tenants; mem_bytes[j]
 * per tenant; free_bytes <= 0 queries the device (cudaMemGetInfo; BL_E_STATE
 * on a device-less ctx).  *ok_out = 1 admissible, 0 not; *reason_out (may be
 * NULL) = 0 ok, 1 kernel-duration span, 2 memory.
 * bl_place (L171, "a central controller can leverage the memory requirement
 * and profiled kernel information to decide which specific GPU to place
 * applications"): apps in order of decreasing memory (ties: smaller index),
 * each to the GPU with the most remaining free memory among those where it
 * fits and keeps rule (a) (ties: smaller GPU index); gpu_out[i] = -1 if none.
 * Pure host function (no ctx). */
bl_status bl_deployment_check(bl_ctx* ctx, const int64_t* mem_bytes, int64_t free_bytes, int32_t span_x,
                              int32_t* ok_out, int32_t* reason_out);
bl_status bl_place(int n_apps, const int64_t* mem_bytes, const int64_t* avg_kernel_ns, int n_gpus,
                   const int64_t* gpu_free_bytes, int32_t span_x, int32_t* gpu_out);

/* ---- box-wide trace dispatcher ("replicating
 * its runtime components for each active GPU") -----------------------------------
 * One host thread routes a merged trace of several GPUs' tenants: entry i goes
 * to ctxs[entries[i].ctx] as a request of entries[i].tenant.  Entries must be
 * sorted by arrival_ns (trace time).  WALL-clock ctxs: the call busy-waits on
 * the host clock until base_ns + arrival_ns, then submits with that arrival
 * (the ctxs must be started); VIRTUAL ctxs: submits at once with arrival_ns
 * (before bl_start).  req_out[i] receives the request id (may be NULL).
 * Returns when every entry is submitted; errors stop at the failing entry. */
typedef struct {
  int32_t ctx;
  int32_t tenant;
  int64_t arrival_ns;
} bl_dispatch_entry;
bl_status bl_dispatch(bl_ctx* const* ctxs, int n_ctx, const bl_dispatch_entry* entries, size_t n, int64_t base_ns,
                      uint64_t* req_out);

/* Diagnostics: mean per-launch device time of 'reps' back-to-back S-CTA
 * launches of an executor skeleton (variant 0: empty kernel, 1: SM gate + tile
 * queue + exit protocol, 2: 1 + device completion stamps, 3: 2 with
 * programmatic dependent launch).  variant | 4 (4..7) returns instead the
 * mean HOST time per launch call of the same loop (enqueue cost, ns).
 * variant | 8 captures the reps launches into one CUDA graph and launches
 * that instead (capture untimed).
 * BL_E_INVALID for variant outside 0..15 or reps < 1. */
bl_status bl_debug_overhead(bl_ctx* ctx, int variant, int reps, int64_t* ns_out);

/* Diagnostics: one whole request of 'tenant' (every kernel, in order, on
 * logical SMs [lo, hi), light exits for the middle kernels, programmatic
 * dependent launch) launched on the tenant's stream (graph = 0) or captured
 * into a CUDA graph and launched as one graph (graph = 1; capture and
 * instantiation untimed).  Medians over reps: device_ns = CUDA-event time of
 * the chain, host_ns = host time spent enqueueing it.  BL_E_STATE while
 * running; BL_E_INVALID for a bad tenant/range or reps < 1. */
bl_status bl_debug_chain(bl_ctx* ctx, int tenant, int lo, int hi, int graph, int reps, int64_t* device_ns,
                         int64_t* host_ns);

int64_t bl_now_ns(void);
const char* bl_last_error(void);
const char* bl_version(void);

#ifdef __cplusplus
}
#endif
#endif /* BLESS_BLESS_H */
