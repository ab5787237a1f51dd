/*
 * stencil.h -- C ABI of the B200-native in-plane stencil library
 * (libstencil.so, built from paper_conf_ipps_tangtkwkgtw13_b200/csrc/).
 *
 * The operation (PAPER.md = Tang et al., IPDPS 2013; "P:L<n>" = line n):
 *   Eq. (1), P:L59-64 (Sec. III-A): for every interior point
 *     out[i,j,k] = c0*in[i,j,k] + sum_{m=1..r} c_m*(in[i+-m,j,k] + in[i,j+-m,k] + in[i,j,k+-m])
 *   iterated Jacobi-style with two grids and a swap (Fig. 1).
 *   The in-plane method (Sec. III-C, Eqs. 3-5) computes exactly
 *   this (up to rounding order); the forward-plane kernel is the SDK FDTD3d
 *   shape the paper compares against.
 *
 * Domain (reading R1): nx, ny, nz are the INTERIOR (updated)
 * extents; every buffer holds the OUTER grid (n + 2r per axis) whose r-wide
 * shell is a frozen Dirichlet boundary -- it is copied, never computed.
 *
 * Memory layout of every device buffer (query with stencil_plan_layout):
 *   element size s = 4 (STENCIL_F32) or 8 (STENCIL_F64); A = 128 / s;
 *   pitch_x  = round_up(A + nx + r, A)  elements per row (a multiple of 128 B);
 *   rows_y   = ny + 2r rows per plane;  planes_z = nz + 2r planes;
 *   outer point (x, y, z), each in [-r, n + r), lives at element
 *       ((z + r) * rows_y + (y + r)) * pitch_x + A + x
 *   so interior x = 0 starts every row on a 128-byte boundary.  Elements of a
 *   row outside [A - r, A + nx + r) are padding: never read for results, never
 *   written.  bytes = planes_z * rows_y * pitch_x * s.
 *
 * Conventions for every call:
 *   - Return a stencil_status_t; on failure nothing observable is modified and
 *     stencil_last_error_detail() (thread-local) says why.
 *   - Device pointers are caller-owned, on the plan's device, 128-byte aligned
 *     (else STENCIL_ERROR_MISALIGNED), at least layout.bytes long, and must
 *     not overlap each other.
 *   - Calls taking a stream are asynchronous and stream-ordered (no host sync)
 *     unless documented as synchronous.  Kernel faults surface on the stream
 *     (CUDA convention).
 *   - A plan is used by one host thread at a time; distinct plans are
 *     independent.
 */
#ifndef STENCIL_H_
#define STENCIL_H_

#include <stddef.h>
#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

#define STENCIL_ABI_VERSION 7
#define STENCIL_MAX_RADIUS 6 /* orders 2..12: Table I / Table IV */

typedef struct stencil_plan_s *stencil_plan_t;
typedef void *stencil_stream_t; /* a cudaStream_t (NULL = legacy default stream) */

typedef enum { STENCIL_F32 = 0, STENCIL_F64 = 1 } stencil_dtype_t;

typedef enum {
    STENCIL_SUCCESS = 0,
    STENCIL_ERROR_INVALID_VALUE = 1,
    STENCIL_ERROR_NOT_SUPPORTED = 2,
    STENCIL_ERROR_MISALIGNED = 3,
    STENCIL_ERROR_OUT_OF_MEMORY = 4,
    STENCIL_ERROR_CUDA = 5,
    STENCIL_ERROR_NCCL = 6
} stencil_status_t;

/* Which sweep kernel a plan launches. */
typedef enum {
    STENCIL_KERNEL_INPLANE = 0,    /* in-plane full-slice + register tiling (Sec. III-C, Fig. 6d);
                                      one elected compute thread issues the TMA loads, predicated
                                      128-bit global stores */
    STENCIL_KERNEL_FORWARD = 1,    /* forward-plane, SDK FDTD3d shape */
    STENCIL_KERNEL_INPLANE_WS = 2, /* the same in-plane method, warp-specialized for B200: a producer
                                      warpgroup issues the full-slice TMA loads and hands its registers
                                      to the compute warps (setmaxnreg); planes per TMA box compiled in;
                                      branch-free step body; bit-identical to INPLANE.  tx*ty (a
                                      multiple of 32) compute threads */
    /* The paper's in-plane loading variants with per-thread global loads (Fig. 6), one
     * point per thread in x, ry rows per thread (register blocking), double-buffered plane tile; the
     * ablation of Fig. 7 / Fig. 10 (NEXT-2).  rx = zbox = stages = 1.  Bit-identical to INPLANE. */
    STENCIL_KERNEL_IP_CLASSIC = 3,    /* interior + four separately loaded halos (Fig. 6a) */
    STENCIL_KERNEL_IP_VERTICAL = 4,   /* columns with their top/bottom halos (Fig. 6b) */
    STENCIL_KERNEL_IP_HORIZONTAL = 5, /* rows with their left/right halos (Fig. 6c) */
    STENCIL_KERNEL_IP_FULLSLICE = 6,  /* the whole slice incl. corners, flat warp-aligned (Fig. 6d) */
    STENCIL_KERNEL_IP_FULLSLICE_V = 7, /* the full slice in 16-byte vector loads */
    /* The forward-plane method (Eq. 2) with INPLANE's loads: full-slice TMA boxes into the same
     * mbarrier ring, rx = one 16-byte vector, ry rows per thread, FP32x2 arithmetic; the (2r+1)-deep
     * input queue in registers.  The ring holds planes z..z+r, so stages >= ceil(r/zbox) + 2.
     * Ablation only (NEXT-2: "forward plane + the same loads"); bit-identical to INPLANE. */
    STENCIL_KERNEL_FP_TMA = 8
} stencil_kernel_t;

typedef struct {
    int64_t nx, ny, nz;  /* interior extents (nz = LOCAL slab extent for distributed plans) */
    int32_t radius;      /* r */
    int32_t dtype;       /* stencil_dtype_t */
    int64_t elem_size;   /* s */
    int64_t pitch_x;     /* elements per row */
    int64_t rows_y;      /* ny + 2r */
    int64_t planes_z;    /* nz + 2r */
    int64_t interior_x0; /* A: element offset of interior x = 0 within a row */
    int64_t x_origin;    /* A - r: element offset of outer x = -r within a row */
    int64_t bytes;       /* planes_z * rows_y * pitch_x * s */
} stencil_layout_t;

/*
 * Tuning tuple of a sweep kernel: the paper's (TX, TY, RX, RY) (P:L193,
 * P:L256, Table IV) plus the B200 extras.  Thread block = tx * ty threads;
 * each thread computes rx (x, contiguous) * ry (y, contiguous) points per
 * plane; tile = (tx*rx) x (ty*ry).  stages = depth of the shared-memory
 * ring fed by TMA (in-plane only); zbox = planes brought by one TMA load (the
 * box depth; in-plane only); zsegs = number of z segments the sweep is split
 * into so that tiles x zsegs thread blocks fill the 148 SMs (each segment
 * re-reads r planes on each side); ytiles = number of tiles along y (0 =
 * ceil(ny / (ty*ry))); with ytiles set, tile t owns the interior rows
 * [t*ny/ytiles, (t+1)*ny/ytiles) -- a balanced partition that lets the tile
 * count match the 148 SMs.  Forward-plane kernels use rx = 1, stages =
 * zbox = 1, ytiles = 0, ry in {1, 2, 4} (rows per thread, register blocking of
 * Fig. 10 case (i)); the loading-variant kernels (STENCIL_KERNEL_IP_*) the same
 * with zsegs free.
 */
typedef struct {
    int32_t kernel; /* stencil_kernel_t */
    int32_t tx, ty;
    int32_t rx, ry;
    int32_t stages;
    int32_t zsegs;
    int32_t zbox;
    int32_t ytiles;
} stencil_config_t;

typedef struct {
    int64_t launches;          /* sweep-kernel launches issued by this plan so far */
    int64_t aux_launches;      /* shell-copy / halo / copy kernels issued so far */
    int32_t timing_enabled;    /* timing mode (stencil_plan_set_timing) */
    int32_t last_run_sweeps;   /* sweep launches in the last stencil_run */
    double last_run_sweep_ms;  /* CUDA-event time from the start of the first to the end of the
                                  last sweep launch of the last timed stencil_run (-1 if none) */
    int64_t timed_sweeps;      /* sweeps of all timed runs since stencil_plan_set_timing */
    double timed_sweep_ms;     /* their summed CUDA-event time (ms; -1 if none): the average
                                  sweep-launch duration is timed_sweep_ms / timed_sweeps */
    double sweep_ms_min;       /* mode 2 only: shortest / longest single sweep (-1 otherwise) */
    double sweep_ms_max;
} stencil_stats_t;

/* ----------------------------------------------------------------------- */
/* Status strings                                                           */
/* ----------------------------------------------------------------------- */

const char *stencil_status_string(stencil_status_t status);
/* Thread-local detail of the last failure on this thread ("" if none). */
const char *stencil_last_error_detail(void);
int stencil_abi_version(void);

/* ----------------------------------------------------------------------- */
/* Host-only helpers (no GPU required)                                      */
/* ----------------------------------------------------------------------- */

/* The pitched layout described above for the given problem.  INVALID_VALUE
 * if n < 1, r not in [1, STENCIL_MAX_RADIUS], or dtype unknown. */
stencil_status_t stencil_layout_compute(int64_t nx, int64_t ny, int64_t nz, int radius,
                                        stencil_dtype_t dtype, stencil_layout_t *out);

/* ----------------------------------------------------------------------- */
/* Plans                                                                    */
/* ----------------------------------------------------------------------- */

/*
 * Create a single-GPU plan bound to the CURRENT CUDA device.
 *   coeffs: host array of radius+1 values c0..cr of Eq. (1) (isotropic),
 *           copied and rounded to dtype.
 * Errors: NULL plan/coeffs, bad sizes or radius outside [1, 6] -> INVALID_VALUE;
 * a device that is not sm_100 -> NOT_SUPPORTED; CUDA failures -> CUDA.
 * The plan starts with a default configuration chosen by the B200 model
 * (no timing); stencil_tune replaces it with a measured one.
 */
stencil_status_t stencil_plan_create(stencil_plan_t *plan, int64_t nx, int64_t ny, int64_t nz,
                                     int radius, const double *coeffs, stencil_dtype_t dtype);

/*
 * Create a single-GPU plan for the PER-AXIS symmetric stencil (BASELINE north
 * star "symmetric per-axis coefficients"; reading R3b):
 *   out = c0*x + sum_{m=1..r} [ cx_m (x[i-m]+x[i+m]) + cy_m (y[j-m]+y[j+m])
 *                               + cz_m (z[k-m]+z[k+m]) ]
 * which is Eq. (1) when cx = cy = cz.
 *   coeffs: host array of 1 + 3*radius values c0, cx_1..cx_r, cy_1..cy_r,
 *           cz_1..cz_r, copied and rounded to dtype.
 * Run with stencil_run / stencil_tune like any Jacobi plan; the kernels are
 * the per-axis instantiations (same 6r+1 FP instructions per point; the
 * in-plane terms are fma(cx_m, x-pair) then fma(cy_m, y-pair)).  Single-GPU
 * only in this version.  Errors: as stencil_plan_create; a non-finite
 * coefficient -> INVALID_VALUE.
 */
stencil_status_t stencil_plan_create_axes(stencil_plan_t *plan, int64_t nx, int64_t ny, int64_t nz,
                                          int radius, const double *coeffs, stencil_dtype_t dtype);

/* Free every plan-owned object (coefficients, tensor maps, scratch grid,
 * events, NCCL communicator).  NULL-safe.  Synchronises the plan's device. */
void stencil_destroy(stencil_plan_t plan);

stencil_status_t stencil_plan_layout(stencil_plan_t plan, stencil_layout_t *out);

/* Select the sweep kernel and its tuning tuple.  The tuple is validated
 * (thread limits, shared memory, TMA box limits <= 256 per dimension,
 * available template instantiations); INVALID_VALUE / NOT_SUPPORTED if not
 * launchable. */
stencil_status_t stencil_plan_set_config(stencil_plan_t plan, const stencil_config_t *cfg);
stencil_status_t stencil_plan_get_config(stencil_plan_t plan, stencil_config_t *cfg);

/*
 * Run `iters` Jacobi sweeps (Fig. 1) of Eq. (1):  out <- S^iters(in).
 *   in : device buffer with the initial outer grid (shell included); NOT
 *        modified.
 *   out: device buffer receiving the result; its shell equals in's shell.
 * iters == 0 copies in to out.  For iters >= 2 the plan ping-pongs between
 * out and a plan-owned scratch grid (allocated on first need, layout.bytes;
 * see stencil_plan_reserve) so that the last sweep lands in out.
 * Asynchronous on `stream`.  Errors: NULL/misaligned/overlapping buffers,
 * iters < 0 -> INVALID_VALUE / MISALIGNED; launch failures -> CUDA.
 */
stencil_status_t stencil_run(stencil_plan_t plan, const void *in, void *out, int iters,
                             stencil_stream_t stream);

/*
 * Host-to-host run: host_out <- S^iters(host_in), both HOST buffers of
 * layout.bytes (pinned -- cudaMallocHost / cudaHostRegister -- for the copies
 * to be asynchronous).  Pipelined across calls: the plan keeps two device
 * slots (4 grids, allocated on first use) and three internal streams, so the
 * upload of call n+1, the sweeps of call n and the download of call n-1
 * overlap.  Ordering: the upload starts after the caller's prior work on
 * `stream`; the call returns at once and does NOT make `stream` wait -- call
 * stencil_run_host_wait(plan, stream) to make `stream` wait for every
 * download issued so far (then host_out of every call is complete and its
 * host_in reusable once `stream` reaches that point).  Single-GPU Jacobi
 * plans; errors as stencil_run.
 */
stencil_status_t stencil_run_host(stencil_plan_t plan, const void *host_in, void *host_out, int iters,
                                  stencil_stream_t stream);
stencil_status_t stencil_run_host_wait(stencil_plan_t plan, stencil_stream_t stream);

/* max over interior points |a - b| of two grids of the plan's layout, in the
 * plan's dtype (the stop-criterion residual of stencil_run_until, for callers
 * that drive their own loop, e.g. distributed plans: all-reduce the per-rank
 * values with MAX).  HOST-SYNCHRONOUS on `stream`.  Errors: NULL / misaligned
 * buffers -> INVALID_VALUE / MISALIGNED. */
stencil_status_t stencil_residual(stencil_plan_t plan, const void *a, const void *b,
                                  stencil_stream_t stream, double *residual);

/*
 * Fig. 1 with its stop criterion ("until stop criteria"; the
 * paper does not define it -- DESIGN.md reading R5b): Jacobi sweeps of the
 * plan's stencil until the update residual
 *     rho_t = max over interior points |u_t - u_{t-1}|   (computed in the plan's dtype)
 * evaluated after every check_every-th sweep (and after sweep max_iters)
 * satisfies rho_t <= tol, or max_iters sweeps have run.
 *   in, out     : as stencil_run (in is not modified; out receives u_T)
 *   max_iters   : >= 1;  check_every: >= 1;  tol: >= 0
 *   iters_done  : T, the number of sweeps run
 *   residual    : rho at the last check (rho_T)
 * HOST-SYNCHRONOUS: blocks at every check (8-byte read back).  Jacobi plans
 * (isotropic or per-axis), single GPU or distributed (stencil_plan_create_dist):
 * a distributed plan reduces rho over the ranks with one NCCL all-reduce (max)
 * per check, so every rank returns the same T and rho -- collective, every
 * rank calls it with the same arguments.  Errors: as stencil_run; bad counts or
 * tol -> INVALID_VALUE; application plans -> INVALID_VALUE; in-process rank
 * groups -> NOT_SUPPORTED.  A NaN residual never satisfies tol.
 */
stencil_status_t stencil_run_until(stencil_plan_t plan, const void *in, void *out, int max_iters,
                                   double tol, int check_every, stencil_stream_t stream,
                                   int *iters_done, double *residual);

/* ----------------------------------------------------------------------- */
/* Application stencils with a second input grid (Sec. V, Table V,          */
/* P:L284-321; BASELINE config 3 "3D wave")                                 */
/* ----------------------------------------------------------------------- */

typedef enum {
    STENCIL_APP_JACOBI = 0, /* Fig. 1 sweeps of Eq. (1): stencil_run */
    STENCIL_APP_SOURCE = 1, /* Table V "Poisson" (2 in -> 1 out): the Jacobi
                               iteration u <- S(u) + d f with a fixed source grid f */
    STENCIL_APP_WAVE = 2,   /* leapfrog wave step u_{n+1} = S(u_n) + d u_{n-1} (d = -1 for
                               u_tt = c^2 Lap u with c0 = 2 + k*3a_0, c_m = k*a_m) */
    STENCIL_APP_DIV = 3,    /* Table V "Div" (3 in -> 1 out): stencil_plan_create_divgrad / stencil_run_div */
    STENCIL_APP_GRAD = 4    /* Table V "Grad" (1 in -> 3 out): stencil_plan_create_divgrad / stencil_run_grad */
} stencil_app_t;

/*
 * Create a plan for an application stencil: like stencil_plan_create, plus
 *   app: the application kind (JACOBI gives exactly stencil_plan_create);
 *   d  : coefficient of the second grid (f for SOURCE, u_{n-1} for WAVE),
 *        rounded to dtype; ignored for JACOBI.
 * Per point the output is Eq. (1) on the first grid followed by + d * g at the
 * same point (the fixed order of DESIGN.md R7 with this term last).  The
 * second grid uses the plan's layout; its shell is never read.  The kernels
 * are the same in-plane / forward-plane sweeps with the second grid streamed
 * centre-only beside the in-plane tile (configurations are validated and
 * tuned for that variant).  Errors: as stencil_plan_create; unknown app or a
 * non-finite d -> INVALID_VALUE.
 */
stencil_status_t stencil_plan_create_app(stencil_plan_t *plan, int64_t nx, int64_t ny, int64_t nz,
                                         int radius, const double *coeffs, stencil_dtype_t dtype,
                                         stencil_app_t app, double d);

/*
 * SOURCE plans: `iters` Jacobi sweeps u <- S(u) + d f starting from `in`;
 * the result lands in `out` (shell = in's shell); `in` and `f` are not
 * modified (f may alias in).  Same buffer rules, scratch use and errors as
 * stencil_run; a plan of another kind -> INVALID_VALUE.
 */
stencil_status_t stencil_run_source(stencil_plan_t plan, const void *in, const void *f, void *out,
                                    int iters, stencil_stream_t stream);

/*
 * WAVE plans: `iters` leapfrog steps in place.  On entry u_prev, u hold the
 * states n-1 and n (outer grids); on completion they hold the states
 * n+iters-1 and n+iters.  Both buffers (and every intermediate state) carry
 * u's shell (frozen Dirichlet boundary): u_prev's shell is overwritten with
 * u's.  The states rotate through u_prev, u and the plan scratch grid; if
 * iters is not a multiple of 3 the last two states are copied into place at
 * the end (two grid copies).  Errors: NULL / misaligned / overlapping
 * buffers, iters < 0, or a plan of another kind -> INVALID_VALUE /
 * MISALIGNED; launch failures -> CUDA.
 */
stencil_status_t stencil_run_wave(stencil_plan_t plan, void *u_prev, void *u, int iters,
                                  stencil_stream_t stream);

/* Allocate the scratch grid now (synchronous), e.g. before CUDA-graph capture. */
stencil_status_t stencil_plan_reserve(stencil_plan_t plan);

/* Timing of the sweep launches with CUDA events on the run stream (off by
 * default).  mode 0: off; 1: one event before the first and one after the
 * last sweep of every stencil_run; 2: also an event after every sweep (gives
 * the per-sweep min/max).  Setting a mode resets the totals of
 * stencil_stats_t.  Errors: mode outside 0..2 -> INVALID_VALUE. */
stencil_status_t stencil_plan_set_timing(stencil_plan_t plan, int mode);
/* Statistics; when timing is on, synchronises on the end event of the last
 * timed run and folds every run recorded since the previous call into the
 * totals (timed_sweeps, timed_sweep_ms). */
stencil_status_t stencil_plan_stats(stencil_plan_t plan, stencil_stats_t *out);

/* ----------------------------------------------------------------------- */
/* Auto-tuning (Sec. IV-C exhaustive search, Sec. VI model-based pruning)   */
/* ----------------------------------------------------------------------- */

typedef enum {
    STENCIL_MODEL_PAPER = 0, /* Eqs. (6)-(14) with the DESIGN.md readings R12-R15 */
    STENCIL_MODEL_B200 = 1   /* the re-derived B200 model */
} stencil_model_t;

typedef struct {
    int32_t model;           /* stencil_model_t used for ranking */
    double beta_percent;     /* beta of P:L372; 0 or >= 100 -> exhaustive */
    int32_t space_size;      /* M: valid configurations of the searched kernel */
    int32_t timed;           /* N: configurations timed */
    stencil_config_t best;   /* winner (stored in the plan) */
    double best_ms_per_iter; /* measured */
    double best_predicted_gpts; /* model prediction of the winner (Gpts/s) */
    double best_measured_gpts;  /* the winner at the sustained clock (the refinement runs) */
    int32_t best_rank_by_model; /* 0-based rank of the winner in the model ordering */
    double best_burst_gpts;     /* the winner's short-run (boost clock) rate */
} stencil_tune_report_t;

/* One candidate of the search space with its model predictions and (if timed)
 * its measurement; see stencil_tune_results. */
typedef struct {
    stencil_config_t cfg;
    double pred_paper_gpts;  /* model-P prediction, Gpts/s */
    double pred_b200_gpts;   /* model-B prediction, Gpts/s */
    double measured_gpts;    /* < 0 if not timed */
    int32_t regs_per_thread; /* from cudaFuncGetAttributes */
    int32_t smem_bytes;      /* dynamic shared memory per block */
    int32_t active_blocks;   /* cudaOccupancyMaxActiveBlocksPerMultiprocessor */
} stencil_tune_entry_t;

/*
 * Tune the plan's sweep kernel (SYNCHRONOUS).  Enumerates the tuning space of
 * `kernel` (constraints (i)-(iv) of P:L256 in their B200 form), ranks it by
 * `model`, times the top N = max(1, ceil(beta*M/100)) with CUDA
 * events (median of `reps` runs of `iters_per_rep` sweeps each, after one
 * warm-up), then re-times the twelve fastest, plus the four fastest of the
 * largest register tiles (RX*RY) not among them, at the sustained clock: after
 * ~0.5 s of sweeps, two interleaved rounds of ~300 ms runs each
 * (STENCIL_TUNE_SUSTAIN_MS; 0 disables), whose mean decides.  The winner is
 * stored in the plan; best_ms_per_iter / best_measured_gpts are its sustained
 * timing, best_burst_gpts its short-run rate.  If the environment variable
 * STENCIL_TUNE_CACHE names a file, the winner is appended to it and plans
 * created later with the same (dtype, radius, extents, plan kind, SM count)
 * start from the best cached configuration (tuning results persisted, reading
 * of the optional cache of SURVEY.md section 8(b)).
 * scratch_in / scratch_out: two device grids of layout.bytes (clobbered).
 * report may be NULL.
 */
stencil_status_t stencil_tune(stencil_plan_t plan, stencil_kernel_t kernel, stencil_model_t model,
                              double beta_percent, int iters_per_rep, int reps, void *scratch_in,
                              void *scratch_out, stencil_stream_t stream,
                              stencil_tune_report_t *report);

/* Copy up to `cap` entries of the last stencil_tune's candidate list, in model
 * order, into `out`; *count receives the number available. */
stencil_status_t stencil_tune_results(stencil_plan_t plan, stencil_tune_entry_t *out, int cap,
                                      int *count);

/* ----------------------------------------------------------------------- */
/* Performance models, host-only                               */
/* ----------------------------------------------------------------------- */

/* GPU parameter set of P:L331-333 (D6). */
typedef struct {
    int32_t sm;          /* SM */
    double bw;           /* BW, bytes/s */
    int32_t smem;        /* Smem per SM, bytes */
    int32_t reg;         /* Reg per SM */
    int32_t blk_sm;      /* Blk_SM */
    int32_t warp_sm;     /* Warp_SM */
    double lat_cycles;   /* Lat */
    double clock_hz;     /* Clock */
} stencil_gpu_params_t;

/* Kernel description for the model (one candidate). */
typedef struct {
    int64_t lx, ly, lz;  /* interior extents (LZ used by the B200 model only) */
    int32_t tx, ty, rx, ry;
    int32_t radius;
    int32_t elem_size;
    int32_t regs_per_thread;   /* K_R = regs_per_thread * tx * ty (reading R12) */
    int32_t smem_per_block;    /* K_S (reading R12) */
    int32_t ops_per_point;     /* Ops: 8r+1 for in-plane (Table II) */
    int32_t stages;            /* B200 model: TMA ring depth (0 = forward-plane kernel) */
    int32_t zbox;              /* B200 model: planes per TMA load */
    int32_t zsegs;             /* B200 model: z segments */
    int32_t ytiles;            /* B200 model: tiles along y (0 = ceil(ly / (ty*ry))) */
    int32_t active_blocks;     /* B200 model: occupancy from the CUDA runtime; <= 0 -> Eq. (7) */
    int32_t inputs;            /* B200 model: input grids (1; 2 for application plans) */
} stencil_model_kernel_t;

/* Eqs. (6)-(14): predicted points/s.  literal_tc != 0 keeps ActBlks in
 * Eq. (11) (reading R13).  Also returns the intermediate Eqs. (6)-(9) if the
 * pointers are non-NULL. */
double stencil_model_paper(const stencil_gpu_params_t *g, const stencil_model_kernel_t *k,
                           int literal_tc, double *blks, int *act_blks, int *stages,
                           int *rem_blks);
/* The B200 model: predicted points/s. */
double stencil_model_b200(const stencil_gpu_params_t *g, const stencil_model_kernel_t *k);

/* ----------------------------------------------------------------------- */
/* z-slab decomposition over GPUs (north star (3); not in the paper)         */
/* ----------------------------------------------------------------------- */

/* Rank `rank` of `nranks` owns interior planes [*z0, *z0 + *nz_local) of
 * nz_global: the first nz_global % nranks ranks get one extra plane.
 * INVALID_VALUE if nz_local would be < radius (the exchange needs r planes). */
stencil_status_t stencil_slab_partition(int64_t nz_global, int nranks, int rank, int radius,
                                        int64_t *z0, int64_t *nz_local);

/*
 * Halo-exchange plan of one rank for the local layout (host-only).  After each
 * sweep, rank p sends its first r owned planes to p-1 and its last r owned
 * planes to p+1, and receives the neighbours' planes into its r-plane halos.
 * Each message is one contiguous span of r*rows_y*pitch_x elements.  Byte
 * offsets are relative to the buffer start; a neighbour that does not exist
 * has peer = -1 (its halo is the global Dirichlet shell and stays frozen).
 */
typedef struct {
    int32_t peer_lo, peer_hi;      /* ranks p-1, p+1 or -1 */
    int64_t send_lo_off, recv_lo_off;
    int64_t send_hi_off, recv_hi_off;
    int64_t msg_bytes;
} stencil_exchange_plan_t;

stencil_status_t stencil_exchange_plan(const stencil_layout_t *local_layout, int nranks, int rank,
                                       stencil_exchange_plan_t *out);

/*
 * In-process rank group (test mode of the distributed plan, SURVEY.md section 4
 * T5): create the `nranks` slab plans of stencil_plan_create_dist on the
 * current device in one process, plans[k] = rank k, with the same partition,
 * local layouts, exchange plan and boundary/interior split; the transport is
 * cudaMemcpyAsync into the neighbour's buffer instead of NCCL.  Destroy each
 * plan with stencil_destroy.  Run them only through stencil_run_dist_local
 * (stencil_run on a member -> NOT_SUPPORTED).
 */
stencil_status_t stencil_plan_create_dist_local(stencil_plan_t *plans, int64_t nx, int64_t ny,
                                                int64_t nz_global, int radius, const double *coeffs,
                                                stencil_dtype_t dtype, int nranks);

/*
 * stencil_run of every rank of an in-process group, issued sweep by sweep in
 * lock step: per sweep each rank launches its boundary z segments, records an
 * event, copies its first / last r owned planes into the neighbours' halo
 * planes of the same sweep's output on its comm stream (after its own and the
 * target rank's boundary events), launches its interior segments, and its
 * next sweep waits for its own and both neighbours' exchange events.
 *   in[k], out[k] : rank k's buffers (local layout; in holds the global field's
 *                   slab [z0, z0+nz_local+2r) including inner halo planes)
 *   streams[k]    : rank k's run stream.  Asynchronous.
 */
stencil_status_t stencil_run_dist_local(stencil_plan_t *plans, int nranks, const void *const *in,
                                        void *const *out, int iters, const stencil_stream_t *streams);

/* NCCL unique id (128 bytes) for stencil_plan_create_dist; call on rank 0 and
 * broadcast the bytes (e.g. over a torch.distributed process group).  Loads
 * libnccl.so.2 at run time; NCCL if unavailable. */
stencil_status_t stencil_nccl_unique_id(void *uid128);

/*
 * Distributed plan: rank `rank` of `nranks` (one process per GPU, current
 * device) owns a z-slab of the nx*ny*nz_global interior.  The local buffers
 * use stencil_layout_compute(nx, ny, nz_local, r, dtype): local plane z
 * corresponds to global plane z0 + z.  stencil_run keeps its contract per
 * rank; inner halo planes are refreshed by NCCL send/recv after every sweep
 * (the boundary segments are swept first and their exchange overlaps the
 * interior sweep).  Collective: every rank must call stencil_run with the same
 * iters.  NCCL errors -> STENCIL_ERROR_NCCL.
 */
stencil_status_t stencil_plan_create_dist(stencil_plan_t *plan, int64_t nx, int64_t ny,
                                          int64_t nz_global, int radius, const double *coeffs,
                                          stencil_dtype_t dtype, const void *nccl_uid128,
                                          int rank, int nranks);

/* ----------------------------------------------------------------------- */
/* Fused peer-store slab plans: the halo exchange rides on  */
/* the sweep kernel's own stores into the neighbours' grids                 */
/* ----------------------------------------------------------------------- */

/* Host-only: where a slab's fused peer stores land (no GPU needed; the p2p
 * plan uses exactly these numbers).  For the local layout `local` of rank
 * `rank`: the output planes z in [0, planes) are also stored at element
 * index (our element index + lo_delta) of rank lo_rank's grid, the planes z in
 * [nz_local - planes, nz_local) at (our element index + hi_delta) of rank
 * hi_rank's grid (both layouts share pitch and rows); a missing neighbour is
 * -1 with delta 0. */
typedef struct {
    int32_t lo_rank, hi_rank;
    int32_t planes;        /* r */
    int64_t lo_delta;      /* + nz_{rank-1} * rows_y * pitch_x elements */
    int64_t hi_delta;      /* - nz_local * rows_y * pitch_x elements */
} stencil_p2p_targets_t;

stencil_status_t stencil_p2p_targets(const stencil_layout_t *local, int64_t nz_global, int nranks,
                                     int rank, stencil_p2p_targets_t *out);

/* What a slab plan shares with its neighbours: its two ping-pong grids (local
 * layout of stencil_layout_compute(nx, ny, nz_local, r, dtype)) and its two
 * incoming flag words (word 0 written by rank-1, word 1 by rank+1), all
 * device pointers valid in the process that holds them. */
typedef struct {
    void *grid[2];
    void *flags;
    int32_t rank;
    int64_t nz_local;
} stencil_p2p_endpoint_t;

/*
 * Create the slab plan of rank `rank` of `nranks` (same partition as
 * stencil_slab_partition) on the current device.  The plan allocates both of
 * its grids (zeroed) and its flags.  No NCCL: the exchange is fused into the
 * in-plane sweep (PS kernels) -- a completed output plane z < r is also
 * stored into rank-1's grid at its plane nz_lo + z, a plane z >= nz_local - r
 * into rank+1's grid at its plane z - nz_local, over NVLink peer memory.
 * Errors: as stencil_plan_create_dist (minus NCCL); NOT_SUPPORTED if the
 * driver lacks stream memory operations.
 */
stencil_status_t stencil_plan_create_p2p(stencil_plan_t *plan, int64_t nx, int64_t ny,
                                         int64_t nz_global, int radius, const double *coeffs,
                                         stencil_dtype_t dtype, int rank, int nranks);
stencil_status_t stencil_p2p_endpoint(stencil_plan_t plan, stencil_p2p_endpoint_t *out);
/* Wire the neighbours (pointers valid in THIS process; lo iff rank > 0, hi iff
 * rank < nranks-1; rank and nz_local are checked against the partition).  For
 * plans in one process (e.g. several slabs on one GPU) pass the other plans'
 * endpoints; across processes use stencil_p2p_export / stencil_p2p_import. */
stencil_status_t stencil_p2p_connect(stencil_plan_t plan, const stencil_p2p_endpoint_t *lo,
                                     const stencil_p2p_endpoint_t *hi);
/* 3 x 64 bytes of CUDA IPC handles (grid 0, grid 1, flags) to send to the neighbours. */
stencil_status_t stencil_p2p_export(stencil_plan_t plan, void *handles192);
/* Open the neighbours' exported handles (NULL where no neighbour) and connect. */
stencil_status_t stencil_p2p_import(stencil_plan_t plan, const void *lo_handles192,
                                    const void *hi_handles192);
/*
 * Run `iters` sweeps on the plan's grids, continuing from the grid that holds
 * the latest state (grid 0 before the first run): sweep e reads grid[(e-1)%2]
 * and writes grid[e%2]; *current = index of the grid holding the result.
 * Before the first run the caller fills the local outer field (shell and halo
 * planes included) into BOTH grids on every rank and makes every rank's fill
 * complete before any rank's first run (e.g. device sync + process barrier).
 * Asynchronous: sweep e >= 2 waits on the stream (cuStreamWaitValue32) until
 * both neighbours have finished sweep e-1; after sweep e the plan writes e
 * into the neighbours' flag words (cuStreamWriteValue32).  The waits carry
 * CU_STREAM_WAIT_VALUE_FLUSH where the device reports
 * cudaDevAttrCanFlushRemoteWrites (the halo planes and the flag both arrive
 * as remote writes, which a device may reorder).  Collective: every rank runs
 * the same sweep counts.
 */
stencil_status_t stencil_p2p_run(stencil_plan_t plan, int iters, stencil_stream_t stream,
                                 int *current);
/* Make `stream` wait (stream-side, no host block) until both neighbours have
 * finished every sweep this plan has issued, i.e. no peer store into this
 * plan's grids is still in flight -- call before overwriting or reading a
 * whole grid (including its halo planes) between runs. */
stencil_status_t stencil_p2p_quiesce(stencil_plan_t plan, stencil_stream_t stream);
/* Local part of the Fig. 1 stop criterion (reading R5b) for a slab: max over
 * this rank's interior of |u_e - u_{e-1}| after its latest sweep e, in the
 * plan's dtype.  HOST-SYNCHRONOUS on `stream`.  INVALID_VALUE before the
 * first sweep. */
stencil_status_t stencil_p2p_residual(stencil_plan_t plan, stencil_stream_t stream, double *residual);

/* Fig. 1 with its stop criterion (reading R5b) across the slabs:
 * sweep (stencil_p2p_run) in blocks of check_every (the last block shorter so
 * that exactly max_iters can run); after each block the GLOBAL residual =
 * max over ranks of the slab residuals, reduced on the devices without any
 * host collective: nranks-1 rounds in which every slab sends its running max
 * into both neighbours' mapped flag buffers and merges theirs (stream-ordered
 * flag words, as the sweeps).  Stops when it is <= tol.  Collective: every
 * rank calls it with the same arguments.  HOST-SYNCHRONOUS at every check.
 *   iters_done : sweeps run;  residual : the global residual at the last check. */
stencil_status_t stencil_p2p_run_until(stencil_plan_t plan, int max_iters, double tol, int check_every,
                                       stencil_stream_t stream, int *iters_done, double *residual);

/* ----------------------------------------------------------------------- */
/* Div / Grad: application stencils with 3 inputs / 3 outputs (Table V,     */
/* P:L284-289, speedup vs number of grids P:L321; reading R19)    */
/* ----------------------------------------------------------------------- */

/*
 * Plan of a Div (app = STENCIL_APP_DIV) or Grad (STENCIL_APP_GRAD) stencil of
 * radius r on an nx*ny*nz interior (same pitched layout as stencil_plan_create;
 * r in [1, 4]).  a = host array of the r weights a_1..a_r of the central first
 * derivative (a_m multiplies f[+m] - f[-m]; the order-2r FD weights for h = 1
 * are (-1)^(m+1) (r!)^2 / (m (r-m)! (r+m)!)), copied and rounded to dtype.
 * The kernels are the in-plane method with one producer warpgroup (divgrad.cuh);
 * configurations use kernel STENCIL_KERNEL_INPLANE_WS with rx = one 16-byte
 * vector, tx in {16, 32}, ry in {2, 4}, zbox = 2.  Errors: as
 * stencil_plan_create; an unknown app -> INVALID_VALUE; r > 4 -> NOT_SUPPORTED.
 */
stencil_status_t stencil_plan_create_divgrad(stencil_plan_t *plan, int64_t nx, int64_t ny, int64_t nz,
                                             int radius, const double *a, stencil_dtype_t dtype,
                                             stencil_app_t app);

/* out <- Div(u, v, w) at every interior point:
 *   out = sum_m a_m ((u[i+m]-u[i-m]) + (v[j+m]-v[j-m]) + (w[k+m]-w[k-m]))
 * One sweep, asynchronous on `stream`.  u, v, w, out: device grids of the plan
 * layout (bytes), 128-byte aligned, out distinct from the inputs; u, v, w are
 * read on their x / y / z axis only (their shells supply the boundary
 * neighbours); out's shell is not written.  Per-point order: the z terms of
 * the planes behind (m = r..1), the x then y differences (m = 1..r), the z
 * terms of the planes ahead (m = 1..r). */
stencil_status_t stencil_run_div(stencil_plan_t plan, const void *u, const void *v, const void *w, void *out,
                                 stencil_stream_t stream);

/* (gx, gy, gz) <- Grad(f): gx = sum_m a_m (f[i+m]-f[i-m]) (m = 1..r), gy, gz likewise
 * (gz: behind terms m = r..1, then ahead terms m = 1..r).  One sweep, asynchronous;
 * buffers as stencil_run_div, the three outputs distinct from f and each other;
 * output shells not written. */
stencil_status_t stencil_run_grad(stencil_plan_t plan, const void *f, void *gx, void *gy, void *gz,
                                  stencil_stream_t stream);

/* ----------------------------------------------------------------------- */
/* Synthetic inputs on the device                                           */
/* ----------------------------------------------------------------------- */

/* Fill the outer grid of `buf` (plan layout) with the counter-based field of
 * stencil_inputs.counter: value(i, j, kg) = top bits of
 * splitmix64(seed * 2^40 + (kg*(ny+2r) + j)*(nx+2r) + i), kg = outer plane
 * index in the GLOBAL grid (local plane + z0 for distributed plans).  Padding
 * elements are set to 0.  Asynchronous. */
stencil_status_t stencil_fill_counter(stencil_plan_t plan, void *buf, uint64_t seed,
                                      stencil_stream_t stream);

#ifdef __cplusplus
}
#endif

#endif /* STENCIL_H_ */
