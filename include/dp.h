/*
 * dp.h — C ABI of the B200-native DREAMPlace objective/gradient evaluation library (libdp).
 *
 * One call evaluates the global-placement objective of eq (2)
 *     obj = sum_e w_e WA_e(x, y)  +  lambda * D(x, y)
 * and its gradient with respect to every cell's lower-left corner, where
 *   - WA_e is the weighted-average wirelength of eq (3) with the overflow-safe shift
 *     of P:159 and the gradient of eq (6), evaluated net-parallel, x and y fused;
 *   - D is the electrostatic density energy of the ePlace model: the four steps of
 *     density map, DCT spectrum a_uv (eqs 5a/9a), potential and field
 *     (eqs 5b-d / 9b-d via eqs 7-8), force gather.
 * Readings of passages the paper leaves silent or garbled are listed in DESIGN.md §3 and are
 * cited below as A1..A26.
 *
 * Conventions
 *   - All functions return dp_status; nothing throws across the ABI.  On failure
 *     dp_last_error() returns a thread-local, NUL-terminated message (valid until the next
 *     call on the same thread).
 *   - "device" pointers are CUDA device (or managed) pointers on the context's device;
 *     "host" pointers are ordinary host memory (pinned memory is faster for dp_eval_host).
 *   - dp_stream_t is a cudaStream_t passed as void* (NULL = the legacy default stream).
 *     Evaluation calls only enqueue work on that stream and never synchronise the host
 *     (except dp_eval_host), so they may be captured into CUDA graphs by the caller.
 *   - Scalar outputs (double*) are DEVICE pointers written on-stream; NULL skips the output.
 *   - Coordinates: x[c], y[c] are the lower-left corner of cell c in the grid's length
 *     units; pin location = (x[c] + pin_dx[p], y[c] + pin_dy[p])  (reading A1).
 *   - Gradients gx, gy are OVERWRITTEN (not accumulated).
 *   - One context may be used by one stream at a time (it owns scratch buffers).
 *     Different contexts are independent.
 *   - The library runs only on sm_100a (B200).  There is no CPU fallback: without a usable
 *     device every call that needs one returns DP_ERR_CUDA.
 */
#ifndef DP_H_
#define DP_H_

#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

typedef enum dp_status {
    DP_OK = 0,
    DP_ERR_INVALID_ARG = 1,   /* null pointer, bad CSR, gamma <= 0, lambda < 0, ...         */
    DP_ERR_UNSUPPORTED = 2,   /* valid input outside what this build implements (bin counts) */
    DP_ERR_OUT_OF_MEMORY = 3, /* device or host allocation failed                             */
    DP_ERR_CUDA = 4,          /* a CUDA runtime error (no device, launch failure, ...)         */
    DP_ERR_NCCL = 5           /* NCCL missing or a collective failed (distributed contexts)    */
} dp_status;

typedef void *dp_stream_t;     /* cudaStream_t */
typedef struct dp_ctx dp_ctx;  /* opaque */

/* The hypergraph H = (V, E) of P:27 in CSR form, plus per-pin offsets and cell sizes.
 * All arrays are HOST arrays; dp_create deep-copies them (the caller may free them after
 * dp_create returns).                                                                    */
typedef struct dp_netlist {
    int32_t num_cells;         /* |V| >= 1                                                 */
    int32_t num_nets;          /* |E| >= 0                                                 */
    int32_t num_pins;          /* |P| >= 0, < 2^31                                         */
    const int32_t *net_start;  /* [num_nets+1]; net_start[0] = 0, nondecreasing,
                                  net_start[num_nets] = num_pins.  Net e owns pin slots
                                  net_start[e] .. net_start[e+1]-1                          */
    const int32_t *net2pin;    /* [num_pins] permutation mapping slot -> pin id, or NULL
                                  (identity: pins already stored in net order)              */
    const int32_t *pin2cell;   /* [num_pins] indexed by pin id; values in [0, num_cells)    */
    const float *pin_dx;       /* [num_pins] pin offset from the cell's lower-left corner   */
    const float *pin_dy;       /* [num_pins]                                               */
    const float *cell_w;       /* [num_cells] finite, >= 0                                 */
    const float *cell_h;       /* [num_cells] finite, >= 0                                 */
    const float *net_weight;   /* [num_nets] finite, >= 0, or NULL (all 1).  Scales WL_e
                                  and its gradient (reading A4); HPWL is unweighted         */
} dp_netlist;

/* The placement region [xl, xh] x [yl, yh] split into bins_x x bins_y bins.
 * Maps are stored [bins_x][bins_y], y contiguous (reading A20).
 * This build supports bins_x, bins_y powers of two in [16, 4096] (even lengths are what
 * Alg 3 requires; reading A23); anything else -> DP_ERR_UNSUPPORTED.
 * stretch = 1: cells smaller than sqrt(2) bins are stretched to sqrt(2) bins with their
 * charge scaled to keep the area (reading A10); stretch = 0: literal overlap.       */
typedef struct dp_grid {
    double xl, yl, xh, yh;     /* xh > xl, yh > yl, finite                                 */
    int32_t bins_x, bins_y;
    int32_t stretch;           /* 0 or 1                                                   */
} dp_grid;

/* Thread-local message describing the last failure on this thread ("" if none). */
const char *dp_last_error(void);

/* Library version (major*10000 + minor*100 + patch). */
int32_t dp_version(void);

/* Validate the netlist and grid, copy them to `device`, reorder pins into the kernels'
 * layout (degree-binned, locality-sorted nets), precompute the per-cell stretched footprint
 * sizes and transform twiddles, allocate scratch.  One-time host-side cost.
 * Side effect: raises the device's persisting-L2 limit (cudaLimitPersistingL2CacheSize) to
 * cover the context's gradient / force arena (~35 MB at bigblue4), which the evaluation's
 * streams mark persisting; the limit is never lowered (DP_L2_PERSIST=0 skips both).
 * Errors: DP_ERR_INVALID_ARG (null, CSR not monotone / out of range, sizes negative or
 * non-finite, degenerate region, stretch not 0/1), DP_ERR_UNSUPPORTED (bin counts),
 * DP_ERR_OUT_OF_MEMORY, DP_ERR_CUDA.  *out is set only on success.                       */
dp_status dp_create(const dp_netlist *nl, const dp_grid *grid, int device, dp_ctx **out);

/* Distributed context for rank `rank` of `world` (one process per GPU; BASELINE north_star:
 * "nets are partitioned for WA, with the cell-gradient vector reduced; cells are partitioned for
 * the density scatter, with the bin map all-reduced").  Every rank passes the full netlist.
 * WA: the WA work units (nets of degree > 1024 one each, blocks of 8 nets of degree 129..1024,
 * chunks of <= 4096 pins of the smaller nets in locality order; a pure function of the
 * netlist) are split into contiguous pin-balanced ranges, one per rank; each rank evaluates
 * its units' nets (each net on exactly one rank) into a gradient over all cells, summed into
 * per-rank cell blocks by one ncclReduceScatter.  Cells: rank r owns the block
 * [r B, min((r+1) B, num_cells)), B = ceil(num_cells / world), for the density scatter, the
 * force gather and the output.  The int64 bin map is summed with one ncclAllReduce (exact);
 * the Poisson solve is replicated (maps up to 1024^2) or row-sharded (larger maps).  The WA
 * partials (one slot per unit, written by one rank) and the HPWL limbs are all-reduced exactly,
 * so WA, D and HPWL are bit-identical for every world size, and in deterministic mode
 * (dp_set_deterministic) so is the gradient.
 * nccl_unique_id: 128-byte ncclUniqueId from dp_nccl_unique_id() on rank 0, broadcast by the
 * caller (e.g. torch.distributed); NULL builds a "virtual shard" whose collectives are skipped
 * (tests on one GPU): its gx, gy then hold the shard's partial WA gradient on every cell plus
 * lambda times the force on its own cells (the sum over shards is the full gradient).  world
 * = 1 with a real id gives a one-rank communicator: the whole distributed path (direct
 * launches, every collective) on one GPU.
 * In a distributed context gx, gy are written only on [cell_begin, cell_end) and the scalar
 * outputs are global.                                                                       */
dp_status dp_create_dist(const dp_netlist *nl, const dp_grid *grid, int device, int rank,
                         int world, const void *nccl_unique_id, dp_ctx **out);

/* Fill out128 (128 bytes, host) with a fresh ncclUniqueId (NCCL loaded at run time). */
dp_status dp_nccl_unique_id(void *out128);

/* Host-only partition plan used by dp_create_dist (no GPU needed; exposed for tests).
 * cell block of `rank` -> *cell_begin, *cell_end.  net_mask (host, [num_nets], nullable)
 * receives per net: 3 = evaluated and counted (WA, HPWL, gradient) on this rank, 0 = not
 * (every net of degree >= 2 has 3 on exactly one rank).                                      */
dp_status dp_partition_plan(const dp_netlist *nl, int rank, int world, int32_t *cell_begin,
                            int32_t *cell_end, uint8_t *net_mask);

/* Free everything the context owns.  NULL is accepted. */
dp_status dp_destroy(dp_ctx *ctx);

/* Full evaluation (eq 2):
 *   gx, gy   (device, [num_cells]) <- dWA/dx + lambda dD/dx,  dWA/dy + lambda dD/dy
 *   d_obj    (device double, nullable) <- WA + lambda D
 *   d_wl     (device double, nullable) <- WA = sum_e w_e (WL_e^x + WL_e^y)
 *   d_energy (device double, nullable) <- D = 1/2 b_x b_y sum_b rho_b psi_b   (reading A8)
 *   d_hpwl   (device double, nullable) <- HPWL, correctly rounded fp64 (reading A7); NULL
 *            skips it (the fused HPWL costs one extra int64 limb reduction)
 * gamma > 0 (length units, reading A5), lambda >= 0, finite.  x, y, gx, gy must not alias.
 * Errors: DP_ERR_INVALID_ARG, DP_ERR_CUDA, DP_ERR_NCCL.                                  */
dp_status dp_eval(dp_ctx *ctx, const float *x, const float *y, float gamma, float lambda,
                  float *gx, float *gy, double *d_obj, double *d_wl, double *d_energy,
                  double *d_hpwl, dp_stream_t stream);

/* WA wirelength only (eqs 3, 6): gx, gy <- dWA/dx, dWA/dy; d_wl <- WA.                    */
dp_status dp_wl_grad(dp_ctx *ctx, const float *x, const float *y, float gamma, float *gx,
                     float *gy, double *d_wl, dp_stream_t stream);

/* Wirelength model used by dp_eval / dp_wl_grad from the next call on (default DP_WL_WA).
 *   DP_WL_WA   weighted-average wirelength, eqs 3 and 6
 *   DP_WL_LSE  log-sum-exp wirelength ("also implemented"; reading A27: the
 *              definition of [29], LSE_e = gamma ln sum e^{x/gamma} + gamma ln sum e^{-x/gamma},
 *              with the P:159 shift), gradient a_i^+/b^+ - a_i^-/b^-
 * With DP_WL_LSE the d_wl output is the LSE total; a fused HPWL (d_hpwl != NULL) runs as a
 * separate HPWL-only pass of the same kernel.  Errors: DP_ERR_INVALID_ARG (unknown model). */
enum { DP_WL_WA = 0, DP_WL_LSE = 1 };
dp_status dp_set_wl_model(dp_ctx *ctx, int32_t model);

/* Deterministic mode (the paper's future work P:706): on != 0 makes the
 * WA gradient an exact integer sum (each pin's fp32 contribution, or each chunk's exact
 * int32 slot sum, converted to int64 in units of 2^-F, F <= 30, and added with integer
 * atomics), so gx, gy are bit-identical from run to run and independent of stream timing.
 * The density map is always exact (int64, 2^-29) and the force gather writes each cell once.
 * Costs one extra 8-byte-per-coordinate accumulator pass (measured in bench.py).
 * Errors: DP_ERR_INVALID_ARG, DP_ERR_OUT_OF_MEMORY.                                         */
dp_status dp_set_deterministic(dp_ctx *ctx, int32_t on);

/* Fixed cells (fixed macros; reading A34).  h_fixed (host, [num_cells],
 * nonzero = fixed; NULL clears) marks cells that are charges of the density constraint (eq
 * 1b) but not variables of (1a).  Their charge at the positions x, y given here
 * (device, [num_cells]; only the fixed cells' entries are read) is scattered once into a
 * precomputed fixed-charge map (exact int64, like every map); later evaluations start their
 * map from it and sort / scatter / gather only the movable cells, so the fixed cells'
 * positions passed to later calls are used for wirelength only.  gx, gy are 0 for fixed
 * cells.  Single-GPU contexts only (DP_ERR_UNSUPPORTED for dp_create_dist contexts).
 * Synchronises `stream`.  Errors: DP_ERR_INVALID_ARG, DP_ERR_OUT_OF_MEMORY, DP_ERR_CUDA.      */
dp_status dp_set_fixed(dp_ctx *ctx, const uint8_t *h_fixed, const float *x, const float *y,
                       dp_stream_t stream);

/* Density only: gx, gy <- dD/dx, dD/dy; d_energy <- D.                        */
dp_status dp_density_grad(dp_ctx *ctx, const float *x, const float *y, float *gx, float *gy,
                          double *d_energy, dp_stream_t stream);

/* Standalone HPWL (reading A6/A7), correctly rounded fp64.                                */
dp_status dp_hpwl(dp_ctx *ctx, const float *x, const float *y, double *d_hpwl,
                  dp_stream_t stream);

/* End-to-end variant of dp_eval on HOST buffers: copies x, y host->device, evaluates,
 * copies gx, gy and the four scalars device->host, and synchronises `stream` before
 * returning.  h_scalars (host, [4], nullable) <- {obj, wl, energy, hpwl}; with_hpwl = 0
 * skips HPWL (h_scalars[3] = NaN).                                                        */
dp_status dp_eval_host(dp_ctx *ctx, const float *hx, const float *hy, float gamma,
                       float lambda, float *hgx, float *hgy, double *h_scalars,
                       int with_hpwl, dp_stream_t stream);

/* Pipelined variant of dp_eval_host (the e2e path): enqueues the H2D copy of hx, hy (host,
 * [num_cells], PINNED: the copies are asynchronous), the evaluation on `stream`, and the D2H copy
 * of gx, gy (own cells) and of {obj, wl, energy, hpwl} into h_scalars (host PINNED double[4],
 * nullable; hpwl is written only with with_hpwl) and returns without waiting.  Inputs and
 * results pass through two device staging slots and two internal copy streams, so the H2D of
 * call k + 1, the evaluation of call k and the D2H of call k - 1 overlap (PCIe is full duplex).
 * The host buffers of a call must stay untouched until dp_eval_host_wait returns; calls on one
 * context must come from one thread.  Errors as dp_eval_host (argument errors before anything is
 * enqueued).                                                                                  */
dp_status dp_eval_host_async(dp_ctx *ctx, const float *hx, const float *hy, float gamma,
                             float lambda, float *hgx, float *hgy, double *h_scalars,
                             int with_hpwl, dp_stream_t stream);
/* Waits until every dp_eval_host_async call on ctx has delivered its results to the host.  */
dp_status dp_eval_host_wait(dp_ctx *ctx);

/* ---- GP loop --------------------------------------------------------
 * The global-placement iterations around the evaluation, entirely on the device: "the loop
 * that involves the computation of wirelength and density gradient, optimization engines,
 * and cell location updating", with ePlace's Nesterov method and Lipschitz step
 * prediction and the eq (18) density-weight update with DREAMPlace's change for
 * p < 0.  Readings A28-A33 fix what the paper leaves to ePlace /
 * RePlAce: step A28, preconditioner A29, overflow A30, gamma schedule A31, lambda_0 A32,
 * clamp / first step A33.  One iteration is captured once into a CUDA graph and replayed
 * (no host synchronisation per iteration).  Single-GPU contexts only (DP_ERR_UNSUPPORTED for
 * dp_create_dist contexts).  The context's wirelength model (dp_set_wl_model) applies.      */
typedef struct dp_gp_params {
    float target_density;    /* t of the overflow (A30); default 1.0                         */
    float gamma_base_scale;  /* gamma_base = scale (b_x + b_y) (A31); default 4.0            */
    float lambda_scale;      /* lambda_0 = scale |grad WL|_1 / |grad D|_1 (A32); default 8e-5 */
    float mu_min, mu_max;    /* eq (18a); defaults 0.95, 1.05                        */
    float dhpwl_ref;         /* p = dHPWL / dhpwl_ref; default 3.5e5                 */
    float init_rms_bins;     /* rms displacement of v_{-1}, in bins (A33); default 0.01     */
    int32_t max_history;     /* iterations kept in the device history ring; default 4096    */
    float stop_overflow;     /* converged below this overflow: the state then stays (A36);
                                default 0.07 (DREAMPlace's stop criterion); 0 = never       */
} dp_gp_params;
typedef struct dp_gp dp_gp;  /* opaque; owns ~12 float vectors of num_cells + scalars       */

/* Fill *p with the defaults above. */
void dp_gp_default_params(dp_gp_params *p);

/* Create a GP loop on ctx (params NULL = defaults).  The loop borrows ctx: destroy it first.
 * Errors: DP_ERR_INVALID_ARG (null, out-of-range params), DP_ERR_UNSUPPORTED (distributed
 * context), DP_ERR_OUT_OF_MEMORY / DP_ERR_CUDA.                                            */
dp_status dp_gp_create(dp_ctx *ctx, const dp_gp_params *params, dp_gp **out);

/* Start from x0, y0 (device, [num_cells], lower-left corners; clamped into the region):
 * tau_0 and gamma_0 from the density map, lambda_0 (A32), g_0, HPWL_0, and the first
 * Lipschitz reference point v_{-1} (A33).  Asynchronous on `stream`.                        */
dp_status dp_gp_init(dp_gp *gp, const float *x0, const float *y0, dp_stream_t stream);

/* Run `iterations` GP iterations (A28: step, Nesterov update, evaluation at v_{k+1},
 * preconditioner, overflow, lambda and gamma updates).  Asynchronous on `stream`.            */
dp_status dp_gp_run(dp_gp *gp, int32_t iterations, dp_stream_t stream);

/* Copy the major solution u (device) into x, y (device, [num_cells]).  Asynchronous.        */
dp_status dp_gp_positions(dp_gp *gp, float *x, float *y, dp_stream_t stream);

/* Synchronise the device and copy the history of the last min(max_rows, iterations,
 * max_history) iterations, oldest first, into h_rows (host, [max_rows][8]):
 *   {k, HPWL(v_{k+1}), overflow(v_{k+1}), lambda_{k+1}, gamma_{k+1}, obj, alpha_k, WL}.
 * *rows <- rows written.                                                                    */
dp_status dp_gp_history(dp_gp *gp, double *h_rows, int32_t max_rows, int32_t *rows);

/* Fence regions ("multiple electric fields, e.g., one for each region",
 * P:549; reading A38).  h_boxes (host, [n_regions][4] = xl, yl, xh, yh, disjoint rectangles);
 * h_cell_region (host, [num_cells]) in [0, n_regions]: 0 = the default region (the layout
 * minus the fences), r >= 1 = fence r.  Every region has its own density map, Poisson solve
 * and field: rho_r = a blockage of density 1 on the part of each bin outside region r (exact
 * int64, like every map) + the charge of region r's cells; D = sum_r D_r; a cell's density
 * gradient is the force gather in its own region's field.  Wirelength is unchanged.
 * n_regions = 0 clears.  Single-GPU contexts only; not combined with dp_set_fixed.
 * Errors: DP_ERR_INVALID_ARG (null, degenerate boxes, region ids out of range),
 * DP_ERR_UNSUPPORTED, DP_ERR_OUT_OF_MEMORY / DP_ERR_CUDA.                                    */
dp_status dp_set_regions(dp_ctx *ctx, int32_t n_regions, const double *h_boxes, const int32_t *h_cell_region);

/* Test-only hook (no part of the metric): synchronise and copy the loop state at the start of
 * the next iteration.  u, v, vp (= v_{k-1}), g (preconditioned gradient at v), gp_prev (at vp):
 * device, [2 num_cells] (x entries, then y), each may be NULL.  h_scalars (host, [9]):
 * {a_{k+1}, lambda, gamma, HPWL(v), overflow(v), alpha_k (the next step's), k, converged flag,
 * Nesterov coefficient (a_k - 1) / a_{k+1}}.                                                 */
dp_status dp_gp_debug_state(dp_gp *gp, float *u, float *v, float *vp, float *g, float *gp_prev,
                            double *h_scalars);

/* Free the loop's buffers (synchronises the device).  NULL is accepted. */
dp_status dp_gp_destroy(dp_gp *gp);

/* ---- introspection -------------------------------------------------------------------- */
typedef struct dp_info {
    int32_t num_cells, num_nets, num_pins;       /* as stored on this rank                 */
    int32_t cell_begin, cell_end;                /* owned cells ([0, num_cells) if 1 rank) */
    int32_t bins_x, bins_y;
    int32_t rank, world;
    int32_t launches_eval;       /* kernels launched by one dp_eval (d_hpwl = NULL)        */
    int32_t launches_eval_hpwl;  /* ... with d_hpwl != NULL                                */
    int64_t device_bytes;        /* device memory owned by the context                     */
    int32_t num_sms;
    int32_t l2_bytes;
} dp_info;

dp_status dp_get_info(const dp_ctx *ctx, dp_info *info);

/* ---- stage timing (CUDA events on the streams each stage runs on) ----------------------
 * While enabled, every evaluation records a start/stop event pair per stage on the stream
 * the stage is launched on:
 *   DP_STAGE_WA       WA + gradient (+ HPWL) kernels               (WA stream)
 *   DP_STAGE_MAP      density map: count, scan, place, scatter     (density stream)
 *   DP_STAGE_FIELDS   DCT / scaling / IDCT-IDXST transforms        (density stream)
 *   DP_STAGE_GATHER   force gather                                 (density stream)
 *   DP_STAGE_COMBINE  gradient combine + scalar finalize           (caller stream)
 *   DP_STAGE_EVAL     the whole call, fork to join                  (caller stream)
 * dp_profile_read synchronises the recorded events, writes the summed milliseconds per
 * stage to ms[DP_NSTAGES] (host) and the number of evaluations to *count, and resets.  */
enum { DP_STAGE_WA = 0, DP_STAGE_MAP = 1, DP_STAGE_FIELDS = 2, DP_STAGE_GATHER = 3,
       DP_STAGE_COMBINE = 4, DP_STAGE_EVAL = 5, DP_NSTAGES = 6 };
dp_status dp_profile_enable(dp_ctx *ctx, int on);
dp_status dp_profile_read(dp_ctx *ctx, double *ms, int64_t *count);

/* ---- test-only hooks (not part of the metric) ------------------------------------------
 * Expose single stages so parity tests can localise a failure.  All pointers device.     */

/* rho (device, [bins_x*bins_y]) <- the density map of step 1.                     */
dp_status dp_debug_density_map(dp_ctx *ctx, const float *x, const float *y, float *rho,
                               dp_stream_t stream);

/* From a given map rho: psi, xi_x, xi_y (device, [bins_x*bins_y], each nullable)
 * <- eqs 9b-9d;  d_energy (device double, nullable) <- 1/2 b_x b_y sum rho psi
 * (computed spectrally by Parseval, the way dp_eval does).                                */
dp_status dp_debug_fields(dp_ctx *ctx, const float *rho, float *psi, float *xi_x, float *xi_y,
                          double *d_energy, dp_stream_t stream);

/* Single 2-D transform of a bins_x x bins_y map (device in/out, may not alias):
 *   DP_T_DCT2       a = DCT_x DCT_y (in)         (eq 9a, 2/N per axis, reading A13)
 *   DP_T_IDCT2      IDCT_x IDCT_y (in)           (eq 9b without the scaling)
 *   DP_T_IDXST_IDCT IDXST_x IDCT_y (in)          (eq 9c without the scaling)
 *   DP_T_IDCT_IDXST IDCT_x IDXST_y (in)          (eq 9d without the scaling)          */
enum { DP_T_DCT2 = 0, DP_T_IDCT2 = 1, DP_T_IDXST_IDCT = 2, DP_T_IDCT_IDXST = 3 };
dp_status dp_debug_transform(dp_ctx *ctx, int kind, const float *in, float *out,
                             dp_stream_t stream);

/* The row-sharded Poisson solve of `world` ranks emulated on one GPU (test hook):
 * the same kernels with the per-rank layouts, the reduce-scatter / all-to-all / all-gather
 * replaced by device copies.  rho (device, [bins_x*bins_y] float); xi_x, xi_y (device,
 * nullable) and d_energy (device double, nullable) as dp_debug_fields.  Errors:
 * DP_ERR_UNSUPPORTED when the map is not shardable (maps of the warp-FFT path, bins not
 * divisible by world into whole CTA blocks).                                                 */
dp_status dp_debug_sharded_fields(dp_ctx *ctx, int32_t world, const float *rho, float *xi_x, float *xi_y,
                                  double *d_energy, dp_stream_t stream);

/* The WA gradient accumulator of the last evaluation (test hook): out (device)
 * <- in deterministic mode the int64 sums in units 2^-30 ([2 n] long long: x, y per cell),
 * otherwise the fp32 sums ([2 n] float); n = num_cells, or world * ceil(num_cells / world)
 * for a distributed context (a virtual shard's partial sums before the skipped
 * reduce-scatter).  *n_out <- n.  Synchronises the stream.                                  */
dp_status dp_debug_wa_accumulator(dp_ctx *ctx, void *out, int64_t *n_out, dp_stream_t stream);

/* Sort-reuse counters (test / bench hook).  The density scatter keeps the
 * tile-ordered list of small cells between evaluations and rebuilds it (the count / scan /
 * place sort) only when a configuration change requests it or when more than DP_RESORT_PCT
 * percent (environment, read at dp_create; default 5) of the small cells were outside the tile
 * they are listed in during the previous evaluation; such "strays" are scattered and gathered
 * through the global map / field with the same arithmetic, so results do not depend on the list
 * (DP_REUSE_SORT=0: sort on every evaluation).  out (host, int32[4]) <- {sort requested, strays
 * of the last completed evaluation, strays accumulated by a scatter not yet gathered, sorts
 * performed since dp_create}.  Synchronises the context's work.                              */
dp_status dp_debug_sort_stats(dp_ctx *ctx, int32_t *out);

#ifdef __cplusplus
}
#endif
#endif /* DP_H_ */
