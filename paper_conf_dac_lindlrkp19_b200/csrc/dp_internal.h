// dp_internal.h — private definitions of libdp (context layout, kernel entry points).
// Not part of the ABI; see include/dp.h for the public contract and DESIGN.md for the design.
#pragma once

#include <cuda_runtime.h>
#include <stdint.h>

#include <string>
#include <utility>
#include <vector>

#include "../../include/dp.h"

namespace dp {

// ---- programmatic dependent launch (PDL) on the density chain ------------------------------
// A chain kernel launched with launch_chain() may be scheduled while its stream predecessor is
// still finishing (its CTAs are placed once every predecessor CTA has started); griddep_wait()
// at the top of the kernel then blocks until the predecessor has completed and its writes are
// visible, so the semantics are those of plain stream order.  Without the launch attribute
// (DP_PDL=0) both instructions are no-ops.
__device__ __forceinline__ void griddep_wait() { asm volatile("griddepcontrol.wait;" ::: "memory"); }
__device__ __forceinline__ void griddep_launch_dependents() {
  asm volatile("griddepcontrol.launch_dependents;" ::: "memory");
}

template <typename... KArgs, typename... Args>
inline void launch_chain(bool pdl, void (*kernel)(KArgs...), dim3 grid, dim3 block, size_t smem, cudaStream_t s,
                         Args &&...args) {
  cudaLaunchConfig_t cfg = {};
  cfg.gridDim = grid;
  cfg.blockDim = block;
  cfg.dynamicSmemBytes = smem;
  cfg.stream = s;
  cudaLaunchAttribute at[1];
  at[0].id = cudaLaunchAttributeProgrammaticStreamSerialization;
  at[0].val.programmaticStreamSerializationAllowed = 1;
  cfg.attrs = at;
  cfg.numAttrs = pdl ? 1 : 0;
  cudaLaunchKernelEx(&cfg, kernel, std::forward<Args>(args)...);
}

// ---------------------------------------------------------------------------------------
// Compile-time layout parameters.
// ---------------------------------------------------------------------------------------
constexpr int kWaThreads = 256;       // threads per WA chunk CTA (8 warps)
constexpr int kWaPpl = 4;             // pin slots per lane (registers)
constexpr int kWaMaxDeg = 128;        // nets up to this degree go through the chunk kernel (G <= 32)
constexpr int kWaChunkPins = 4096;    // max pins per chunk (staged in shared memory)
constexpr int kWaWindow = 1024;       // consecutive cells per chunk window held in shared memory
constexpr int kBigThreads = 256;      // CTA-per-net kernel for nets > kWaMaxDeg
constexpr int kBigStage = 4096;       // big-net pins whose exact positions stay in shared memory
constexpr int kWarpNetMax = 1024;     // nets of degree (kWaMaxDeg, kWarpNetMax] take a warp each; larger a CTA
constexpr int kWarpNetThreads = 256;  // warp-per-net kernel CTA size
constexpr int kHpwlLimbs = 9;         // limbs 0..kHpwlLimbs (10) of 32-bit digits, LSB 2^-149 (reading A7)

constexpr int kTile = 64;             // density tile = kTile x kTile bins (smaller maps: the map)
constexpr int kHalo = 2;              // small-cell footprints extend <= 2 bins past their first bin
// the walkers' shared tiles extend kMargin bins past the tile on every side: a listed cell whose
// first bin has drifted up to kMargin bins out of its tile since the sort still accumulates in
// shared memory (even, so that the field tile's rows stay 16-byte aligned)
#ifndef DP_MARGIN
#define DP_MARGIN 2   // -DDP_MARGIN=m: A/B builds (0 / 2 / 4 measured)
#endif
constexpr int kMargin = DP_MARGIN;
#ifndef DP_WALK_THREADS
#define DP_WALK_THREADS 512   // -DDP_WALK_THREADS=256: A/B builds
#endif
constexpr int kStageRecs = DP_WALK_THREADS;   // records per staging buffer of the scatter/gather walkers (one per thread)
// Tile bins accumulate each contribution v in (0, 1] as u = floor(v 2^29) in one native 32-bit
// shared atomic (modulo 2^32; the thread whose add wraps carries 2^32 units to the int64 map).
constexpr int kRhoScaleLog2 = 29;   // global bin map: int64 units of 2^-29
// per-tile counters / cursors one 128-byte line apart: every CTA of count / place adds to every
// tile's counter, and counters sharing a line serialise in one L2 slice
constexpr int kCntStride = 32;
constexpr int kCountThreads = 256;
constexpr int kCountCells = 2048;     // cells per count/place CTA (staged in shared memory)

// Per warp-group metadata of the WA chunk layout (16 bytes, bulk-copied per chunk).
struct WarpGroup {
  int32_t pin_base;   // first pin entry of the group, relative to its chunk's pin_begin
  int32_t net_base;   // first net, relative to its chunk's net_begin
  int32_t nnets;      // nets in the group (<= 32 / g)
  int32_t g_log2 : 8; // log2 of lanes per net
  int32_t slots : 8;  // pin slots per lane (<= kWaPpl)
  int32_t flags : 16; // bit 0: all nets of the group have degree 2 (closed-form path)
};

// One CTA's work in the WA kernel (48 bytes).  Pin records hold a chunk-local position slot:
// [0, kWaWindow) = window cell win_lo + i, kWaWindow + f = far cell far_cells[far_begin + f];
// bit 31 marks a foreign pin (distributed: no gradient for that cell on this rank).
struct Chunk {
  int32_t wg_begin, wg_n;     // warp groups (16-byte records)
  int32_t pin_begin, pin_n;   // pin records (16-byte aligned, padded to 4)
  int32_t net_begin, net_n;   // net degrees / weights (16-byte aligned, padded to 4)
  int32_t far_begin, far_n;   // deduplicated cells outside the window
  int32_t far_pad;            // far_n padded to 4 (bulk copy size)
  int32_t win_lo, win_n;      // window [win_lo, win_lo + win_n), win_lo a multiple of 4
  int32_t scale_log2;         // window / far gradients accumulate int32 units of 2^-scale_log2
};

// Shared-memory capacities of the WA chunk kernel (maxima over chunks, multiples of 4).
struct WaCaps {
  int pins, nets, groups, far;
};

// Arguments a captured evaluation graph was built for (kernel parameters are baked in).
struct GraphKey {
  const void *x = nullptr, *y = nullptr, *gx = nullptr, *gy = nullptr;
  const void *obj = nullptr, *wl = nullptr, *en = nullptr, *hpwl = nullptr;
  float gamma = 0.f, lambda = 0.f;
  bool wa = false, den = false;
  int wl_model = 0;
  bool det = false;
  bool sort = true;   // the sort kernels are in the graph
  bool operator==(const GraphKey &o) const {
    return x == o.x && y == o.y && gx == o.gx && gy == o.gy && obj == o.obj && wl == o.wl && en == o.en &&
           hpwl == o.hpwl && gamma == o.gamma && lambda == o.lambda && wa == o.wa && den == o.den &&
           wl_model == o.wl_model && det == o.det && sort == o.sort;
  }
};

struct Ctx {
  // ---- identity ----
  int device = 0;
  int rank = 0, world = 1;
  int num_sms = 0, l2_bytes = 0;
  int32_t num_cells = 0, num_nets_in = 0, num_pins_in = 0;
  int32_t cell_begin = 0, cell_end = 0;
  bool has_weights = false;
  bool dist = false;

  // ---- grid ----
  double xl = 0, yl = 0, xh = 0, yh = 0, bx = 0, by = 0;
  int mx = 0, my = 0, log2mx = 0, log2my = 0, stretch = 1;
  int tiles_x = 0, tiles_y = 0, tile = kTile;

  // ---- WA layout (device) ----
  int32_t n_chunks = 0, n_wgroups = 0, n_wa_nets = 0, n_wa_pins = 0;
  WaCaps wa_caps{4, 4, 4, 4};          // per-chunk staging capacities
  int32_t *d_far_cells = nullptr;      // far-cell lists of all chunks
  Chunk *d_chunks = nullptr;
  WarpGroup *d_wgroups = nullptr;
  int32_t *d_net_deg = nullptr;     // degree | counted<<31 per reordered net
  float *d_net_w = nullptr;         // weights per reordered net (if has_weights)
  int32_t *d_pin_cell = nullptr;    // chunk-local position slot | foreign<<31 per pin entry
  float *d_pin_dx = nullptr, *d_pin_dy = nullptr;
  // big nets (degree > kWaMaxDeg): plain CSR, one CTA per net
  int32_t n_big = 0;
  int32_t n_huge = 0;               // big nets [0, n_huge) (degree > kWarpNetMax) take a CTA each
  int32_t big_stage = 0;            // staged pins per big-net CTA (min(max degree, kBigStage))
  int32_t *d_big_start = nullptr;   // [n_big + 1]
  int32_t *d_big_flags = nullptr;   // counted flag per big net
  float *d_big_w = nullptr;
  int32_t *d_big_cell = nullptr;
  float *d_big_dx = nullptr, *d_big_dy = nullptr;

  // ---- density layout (device) ----
  float *d_cell_w = nullptr, *d_cell_h = nullptr;   // own cells (index from cell_begin)
  float *d_cell_pins = nullptr;
  // fixed cells (NEXT-4, dp_set_fixed): mask per own cell, precomputed fixed-charge map, and
  // the large-cell lists split by mobility
  bool has_fixed = false;
  bool fixed_small = false;     // some fixed cell is a small cell (the count / place kernels need the mask)
  uint8_t *d_fixed = nullptr;
  unsigned long long *d_rho_fixed = nullptr;
  int32_t *d_large_mov = nullptr, *d_large_fix = nullptr;
  // fence regions (NEXT-4, dp_set_regions; reading A38): one density map / Poisson solve / field
  // per region r in [0, n_regions]; cells carry their region, region r's map starts from its
  // blockage map (density 1 outside the region, exact int64)
  int32_t n_regions = 0;                       // fences; 0 = none
  uint8_t *d_region = nullptr;                 // [n_own] region of each own cell
  unsigned long long *d_rho_block = nullptr;   // [n_regions + 1][mx my]
  int32_t *d_large_reg = nullptr;              // large cells grouped by region
  std::vector<int32_t> large_reg_off;          // [n_regions + 2]
  mutable int cur_region = -1;                 // region of the density pass being enqueued
  // GP loop over fence regions: each region pass adds its A30 overflow partials here
  // ([n_regions + 1][ovf_blocks][2], null = not requested), with the target density ovf_target
  double *ovf_part = nullptr;
  int ovf_blocks = 0;
  double ovf_target = 1.0;
  bool walk_sync = false;                      // DP_WALK_SYNC=1: block barrier per walker ring refill
  int n_en_slots() const { return n_en_part * (n_regions + 1); }
  int32_t n_large_mov = 0, n_large_fix = 0;                     // [num_cells] net-weighted pin count (GP preconditioner)
  int32_t n_own = 0;                // cells owned by this rank
  int32_t n_large = 0;              // large cells (footprint > 3 bins on an axis)
  int32_t *d_large = nullptr;       // ids of large own cells
  uint8_t *d_is_large = nullptr;    // per own cell
  int32_t *d_tile_cnt = nullptr;      // [tiles * kCntStride] small-cell counts (reset by the scan)
  int32_t *d_tile_cursor = nullptr;   // [tiles * kCntStride] placement cursors
  int32_t *d_tile_off = nullptr;      // [tiles + 1]
  float4 *d_rec = nullptr;            // per slot: footprint box in tile-local bin units
  int2 *d_rec_rc = nullptr;           // per slot: (charge ratio r as float bits, i0 | j0 << 16)
  int32_t *d_rec_cell = nullptr;      // per slot: own cell index (tile-ordered list, kept between sorts)
  float2 *d_rec_wh = nullptr;         // per slot: (w, h) of the listed cell
  // sort reuse: {re-sort requested, strays of the last evaluation, strays of this
  // one, sorts performed}; the sort kernels run when a sort is requested or the last evaluation's
  // strays (cells outside the tile they were listed in) exceed resort_thr
  int32_t *d_sortctl = nullptr;
  int32_t resort_thr = 0;
  bool reuse_sort = true;             // DP_REUSE_SORT=0: sort on every evaluation (default: keep the list between sorts)
  bool gather_rc = false;             // DP_GATHER_RC=1: the gather recomputes footprints (no records)
  bool sort_cond = false;
  int scatter_merge = 1;              // DP_SCATTER_MERGE=2: the scatter runs one CTA per two walker slices (A/B)
  bool rec_hint = false;              // DP_REC_HINT=1: L2 evict-last records (scatter) / evict-first reads (gather)
  bool early_gather = true;           // DP_EARLY_GATHER=0: the gather waits for its predecessor at the top
  bool early_scatter = true;          // DP_EARLY=0: the no-sort variant keeps the memset and a plain dependency
  bool sort_host = true;              // DP_SORT_HOST=0: every captured evaluation carries the sort kernels
  bool sorted_once = false;           // a graph with the sort kernels has run since the last sort request
  int32_t *h_ctl = nullptr;           // mapped pinned host word: strays of the last evaluation (the gather writes it)
  int32_t *h_ctl_dev = nullptr;       // its device address
  int32_t sort_every = 8;             // DP_SORT_EVERY: every k-th captured evaluation carries the sort kernels anyway
  int64_t sort_tick = 0;
  // the graph variant of the next captured evaluation (or GP iteration): 1 = with the sort kernels
  int sort_variant() {
    const bool kept = sort_host && sorted_once && reuse_sort && n_regions == 0 && h_ctl &&
                      *reinterpret_cast<volatile int32_t *>(h_ctl) <= resort_thr;
    return (!kept || ++sort_tick % sort_every == 0) ? 1 : 0;
  }
  mutable bool omit_sort = false;     // set while capturing a graph without the sort kernels             // DP_SORT_COND=1: the sort in an IF node of captured evaluations (A/B)
  cudaStream_t s_body = nullptr;      // captures the body of the sort's IF node
  bool serial = false;
  bool use_graph = true;   // DP_GRAPH=0 disables the captured-graph evaluation path
  cudaStream_t s_cap = nullptr;
  // captured evaluations: [1] with the sort kernels (they return at once unless a sort is due),
  // [0] without them (the host saw few strays in the last evaluations)
  cudaGraphExec_t gexec_v[2] = {nullptr, nullptr};
  GraphKey gkey_v[2];
  int wl_model = 0;        // DP_WL_WA / DP_WL_LSE (dp_set_wl_model)
  bool deterministic = false;     // dp_set_deterministic (NEXT-2): WA gradient as exact int64 sums
  bool hpwl_fast = false;         // GP loop: HPWL from fp32 pin positions fused into the fast WA path (A37)
  bool pdl = true;                // programmatic dependent launch along the density chain (DP_PDL=0: off)
  bool direct = false;            // DP_DIRECT=1: WA and gather add into the caller's gx, gy (no combine pass)
  float *direct_gx = nullptr, *direct_gy = nullptr;   // set for the duration of one eval_body
  bool fuse_combine = false;      // DP_FUSE_COMBINE=1: the gather waits for WA and writes gx, gy (no combine pass)
  float *fused_gx = nullptr, *fused_gy = nullptr;     // set for the duration of one eval_body
  float direct_lambda = 0.f;
  int det_frac = 30;              // its units 2^-det_frac (>= every chunk's slot scale in practice: exact shifts)
  long long *d_g2i = nullptr;     // [2 num_cells] int64 WA gradient (allocated on first enable)
  // GP loop (gp.cu): while non-null, the evaluation kernels read gamma / lambda from these
  // device scalars instead of their by-value arguments (one captured graph per GP iteration)
  const float *gamma_dev = nullptr, *lambda_dev = nullptr;
  int sched = 0;           // DP_SCHED: 0 = WA from the fork, 1 = WA after the density map (overlaps the transforms)     // DP_SERIAL=1: density chain after WA (no stream overlap; measurement)
  int32_t walk_grid = 0;
  int32_t count_grid = 0;           // resident CTAs of the persistent count kernel
  int32_t *d_walk_tile = nullptr;   // [walk_grid]   // CTAs of the persistent scatter / gather walkers (SMs x resident)
  unsigned long long *d_rho = nullptr;  // bin map, int64 fixed point in units of 2^-kRhoScaleLog2 (exact, deterministic)
  float *d_t = nullptr, *d_sx = nullptr, *d_sy = nullptr;
  float2 *d_xi = nullptr;
  float2 *d_force = nullptr;          // per own cell: -(sum ov xi)
  float2 *d_tw_x = nullptr, *d_tw_y = nullptr;     // FFT twiddles W_N^k, k < N/2
  float2 *d_ph_x = nullptr, *d_ph_y = nullptr;     // e^{-i pi k / 2N}, k < N
  float2 *d_spec = nullptr;                         // T2a -> T2b (A_X, A_Y) transposed [y][x]
  int wa_ctas_per_sm = 0;                           // DP_WA_CTAS_PER_SM: residency cap of the WA kernel (0 = none)
  bool l2_hint = true;                              // DP_L2_HINT=0: no evict-first policy on the WA pin stream (A/B)
  bool row_tma = true;                              // DP_ROW_TMA=0: per-lane loads in the row-inverse passes (A/B)
  bool t1_tma = false;                              // DP_T1_TMA=1: bulk-copied rows in the forward row pass (A/B; not faster inside the overlapped step)
  bool fused_t2 = false;
  int t2b_warps = 4;
  // split WA launch (DP_WA_SPLIT = percent of the chunk units in the first part): the first part
  // (big units + that share of the chunks) runs beside the density map, the rest after the field
  // transforms (beside the gather), so the latency-bound transforms run without WA CTAs
  int wa_split_chunks = 0;
  bool wa_split = false;
  cudaEvent_t ev_fields = nullptr;                                // DP_T2B_WARPS=2: 2-warp T2b CTAs (fit beside two WA CTAs; A/B)                            // DP_FUSED_T2=1: one column kernel (T2) instead of T2a + T2b (A/B)
  float2 *d_sxy = nullptr;                          // T2 -> T3 interleaved (sX, sY) [x][y] (warp-FFT path)
  float2 *d_twf_x = nullptr, *d_twf_y = nullptr;   // CTA FFT: W_N^k, k < N
  bool fft_cta = true;                              // fields by the CTA-FFT passes P1 P2 P3 (fields.cu)
  bool fft_hybrid = false;                          // warp-FFT T1 and T3 around the CTA-FFT column pass P2
  float2 *d_tw2_x = nullptr, *d_tw2_y = nullptr;   // warp FFT: W_N^{n1 k2} at [k2 * 32 + n1] (N <= 1024)
  float *d_kx = nullptr, *d_ky = nullptr;          // wavenumbers (reading A12)

  // ---- shared scratch ----
  float2 *d_g2 = nullptr;             // WA gradient accumulator, interleaved, cleared per call (hot arena head)
  size_t hot_bytes = 0;               // g2 + force arena (L2 persisting window)
  bool l2_persist = true;             // DP_L2_PERSIST=0: no persisting window (A/B)
  bool l2_persist_maps = false;       // DP_L2_PERSIST=2: the density stream's window covers the maps
  void *d_maps = nullptr;             // arena: rho, spec, sxy, xi, t
  size_t maps_bytes = 0;
  double *d_part = nullptr;           // partial sums: [0, n_wa_part) WA, then energy
  int32_t n_wa_part = 0, n_en_part = 0;   // WA partials: one slot per global WA unit (all ranks)
  int32_t part_base = 0;                   // this rank's first WA unit
  int32_t cell_blk = 0;                    // cells per rank block of the gradient reduce-scatter
  int64_t config_gen = 0;                  // bumped by every dp_set_*: graphs captured earlier are stale
  bool shard_poisson = false;              // row-sharded Poisson solve (dist, maps > 1024)
  int64_t g2_cells = 0;                    // WA accumulator length (dist: world blocks; else num_cells)
  unsigned long long *d_limbs = nullptr;  // HPWL fixed-point limbs
  double *d_scal = nullptr;           // {wl, energy, hpwl, obj} staging
  float *d_hx = nullptr, *d_hy = nullptr, *d_hgx = nullptr, *d_hgy = nullptr;  // e2e buffers
  // dp_eval_host_async: two staging slots per direction (inputs x|y, outputs gx|gy + 4 scalars),
  // a copy stream each way; allocated on first use
  float *d_in2[2] = {nullptr, nullptr}, *d_out2[2] = {nullptr, nullptr};
  double *d_osc2[2] = {nullptr, nullptr};
  cudaStream_t s_h2d = nullptr, s_d2h = nullptr;
  cudaEvent_t ev_in_ready[2] = {}, ev_in_free[2] = {}, ev_out_ready[2] = {}, ev_out_free[2] = {};
  int64_t async_k = 0;

  // ---- streams / events ----
  cudaStream_t s_wa = nullptr, s_den = nullptr;
  cudaEvent_t ev_fork = nullptr, ev_wa = nullptr, ev_den = nullptr;
  cudaEvent_t ev_map = nullptr;
  cudaEvent_t ev_sched = nullptr;   // DP_SCHED=2/3: WA start after the placement / the count (A/B)
  cudaStream_t s_aux = nullptr;    // large cells and the finalize, beside the main chains
  cudaEvent_t ev_aux_a = nullptr, ev_aux_b = nullptr, ev_join = nullptr, ev_fin = nullptr;    // density map complete (DP_SCHED=1 start of WA)
  cudaEvent_t ev_done = nullptr;   // end of the last call: serialises use from several streams

  // ---- NCCL (distributed) ----
  void *nccl_comm = nullptr;

  // ---- stage profiling (dp_profile_enable) ----
  bool profiling = false;
  std::vector<cudaEvent_t> prof_pool;          // free events
  std::vector<std::pair<cudaEvent_t, cudaEvent_t>> prof_pairs[DP_NSTAGES];
  int64_t prof_evals = 0;

  int64_t device_bytes = 0;
  int launches_eval = 0, launches_eval_hpwl = 0;
  std::vector<void *> allocations;
};

// error handling ---------------------------------------------------------------------------
void set_error(const std::string &msg);
dp_status fail(dp_status st, const std::string &msg);
dp_status cuda_fail(cudaError_t e, const char *what);

#define DP_CUDA(call)                                               \
  do {                                                              \
    cudaError_t _e = (call);                                        \
    if (_e != cudaSuccess) return ::dp::cuda_fail(_e, #call);        \
  } while (0)

// kernel launchers (defined in the .cu files) ---------------------------------------------
// WA (wa.cu)
// part 0: all WA units; 1 / 2: the two halves of a split launch (Ctx::wa_split_chunks)
void launch_wa(const Ctx &c, const float *x, const float *y, float gamma, bool hpwl_only,
               bool with_hpwl, cudaStream_t s, int part = 0);
// density (density.cu)
void launch_density_map(const Ctx &c, const float *x, const float *y, cudaStream_t s, cudaStream_t aux = nullptr,
                        int build_fixed = 0);
void launch_density_gather(const Ctx &c, const float *x, const float *y, cudaStream_t s, cudaStream_t aux = nullptr);
// transforms (dct.cu)
void launch_fields(const Ctx &c, const float *rho, cudaStream_t s);            // rho as float (debug hook)
void launch_fields_fixed(const Ctx &c, cudaStream_t s);                          // rho = c.d_rho (hot path)
void launch_rho_to_float(const Ctx &c, float *out, cudaStream_t s);
void launch_transform(const Ctx &c, int kind, const float *in, float *out, cudaStream_t s);
void launch_split_fields(const Ctx &c, float *xi_x, float *xi_y, cudaStream_t s);
void launch_psi(const Ctx &c, const float *rho, float *psi, cudaStream_t s);
// CTA-FFT field passes (fields.cu): P1 rows, P2 columns (+ energy), P3 rows
cudaError_t fields_configure();
bool fields_cta_ok(int log2mx, int log2my);
int p2_ctas(int mx, int my, bool hybrid = false);
void launch_fields_cta(const Ctx &c, const void *rho, bool int_map, cudaStream_t s);
void launch_p2_rowmajor(const Ctx &c, cudaStream_t s);
bool fields_shardable(const Ctx &c, int G);
void launch_fields_shard(const Ctx &c, int pass, const void *rho, bool int_map, int r, int G, float *s1,
                         const float *r1, float2 *s2, const float2 *r2, cudaStream_t s);
// combine / finalize (finalize.cu)
dp_status eval_body_ext(Ctx &c, const float *x, const float *y, float gamma, float lambda, float *gx, float *gy,
                        double *d_obj, double *d_wl, double *d_energy, double *d_hpwl, cudaStream_t s, bool do_wa,
                        bool do_den);
dp_status ctx_call_begin(Ctx &c, cudaStream_t s);
dp_status ctx_call_end(Ctx &c, cudaStream_t s);
void launch_combine(const Ctx &c, float lambda, float *gx, float *gy, bool use_wa,
                    bool use_density, cudaStream_t s);
void launch_finalize(const Ctx &c, float lambda, bool with_wl, bool with_energy,
                     bool with_hpwl, double *d_obj, double *d_wl, double *d_energy,
                     double *d_hpwl, cudaStream_t s);
void launch_finalize_phase(const Ctx &c, int phase, float lambda, bool with_wl, bool with_energy,
                           bool with_hpwl, double *d_obj, double *d_wl, double *d_energy,
                           double *d_hpwl, cudaStream_t s);
// configuration (shared-memory opt-in), called from dp_create
cudaError_t dct_configure(int mx, int my);
cudaError_t wa_configure(const WaCaps &caps);
int wa_smem_bytes(const WaCaps &caps);
cudaError_t density_configure(int ntiles, int tile);
int density_walk_grid(int tile);
int density_count_grid(int ntiles);
int density_launches(const Ctx &c);
void launch_region_overflow(const Ctx &c, cudaStream_t s);
dp_status request_sort(Ctx &c, cudaStream_t s);   // the next evaluation rebuilds the tile-ordered list
// NCCL (nccl_dyn.cpp)
dp_status nccl_get_unique_id(void *out128);
dp_status nccl_init(Ctx &c, const void *id);
dp_status nccl_allreduce_f32(Ctx &c, float *buf, size_t n, cudaStream_t s);
dp_status nccl_allreduce_f64(Ctx &c, double *buf, size_t n, cudaStream_t s);
dp_status nccl_allreduce_u64(Ctx &c, unsigned long long *buf, size_t n, cudaStream_t s);
dp_status nccl_reduce_scatter_f32(Ctx &c, float *buf, size_t n, cudaStream_t s);
dp_status nccl_reduce_scatter_i64(Ctx &c, long long *buf, size_t n, cudaStream_t s);
dp_status nccl_reduce_scatter_u64(Ctx &c, unsigned long long *buf, size_t n, cudaStream_t s);
dp_status nccl_all_gather_bytes(Ctx &c, void *buf, size_t n, cudaStream_t s);
dp_status nccl_all_to_all_bytes(Ctx &c, const void *send, void *recv, size_t n, cudaStream_t s);
void nccl_destroy(Ctx &c);

}  // namespace dp
