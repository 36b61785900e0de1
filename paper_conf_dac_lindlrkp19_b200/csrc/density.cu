// density.cu — density map scatter (step 1 of P:253) and electric-force gather (step 4,
// P:256) on sm_100a.
//
// Method: the density map is a 2-D histogram / "dynamic bipartite graph forward"
// where each cell adds its overlap area to the bins it covers; the force on a cell
// is the overlap-weighted sum of the bin field.  The paper sorts cells by area and
// uses 2x2 threads per cell with global atomics.  Readings: A9 (rho in units of
// bin area), A10 (stretch to sqrt2 bins), A11 (clip to region), A21 (gradient sign).
//
// B200 design: random global red.add runs at ~0.18 Gop/ms on B200
// (tools/microbench), which would cost ~70 us for the ~13M bin updates of bigblue4.  So every
// evaluation sorts the small cells by spatial tile (kTile x kTile bins):
//   D1 count   per-CTA shared histogram of tile ids -> global tile counts
//   D2 scan    one CTA: tile offsets and per-tile cursors
//   D3 place   recompute tile ids, reserve ranges per CTA, write tile-local footprint
//              records in tile order
//   D4 scatter persistent walkers (SMs x resident CTAs) each take an equal slice of the
//              tile-ordered records, stream it through double-buffered bulk copies and
//              accumulate into a (tile+2)^2 shared tile, flushed with coalesced red.add into
//              rho only where the slice leaves a tile
//   D5 gather  same walkers; the (tile+2)^2 float2 field tile is reloaded only where the slice
//              enters a new tile; each cell's force is written once
// Large cells (footprint wider than 3 bins) take a CTA-per-cell path with global reds.
// The tile accumulators (one 32-bit word per bin, 2^-29 units modulo 2^32, wraps carried to the
// map by the wrapping thread) flush into an int64 global map (2^-29 units) with red.global.add.u64: the density map is exact up to one rounding
// per contribution and independent of execution order (deterministic; bit-identical after an
// int64 all-reduce).
// Footprint geometry is computed in fp64 (B200 runs FP64 at half rate); records hold the
// footprint in fractions of the cell's first bin (|v| < 3) plus that bin's tile-local index.
#include <algorithm>
#include <cmath>

#include <cstdlib>

#include "async_copy.cuh"
#include "dp_internal.h"

namespace dp {

namespace {

constexpr int kTileThreads = DP_WALK_THREADS;   // scatter / gather CTA size (smem-bound at 2 CTAs per SM)

struct DenArgs {
  const float *x, *y;   // global cell arrays
  const float *w, *h;   // own cells
  int cell_begin, n_own;
  double xl, yl, xh, yh, bx, by, sx, sy, ibx, iby;   // ibx = 1 / bx (no fp64 divisions on the hot path)
  double cx0, cy0;     // -xl / bx, -yl / by: bin coordinate of x is x * ibx + cx0
  float sxf, syf;      // stretched minimum sizes sqrt2 b (fp32)
  float w_large, h_large;   // largest floats <= 2 b_x, 2 b_y: w > w_large <=> (double)w > 2 b_x (dp_create's test)
  int mx, my, tile, tile_log2, tiles_y, ntiles, stretch;
  int *tile_cnt, *tile_cursor, *tile_off;
  int *walk_tile;   // [walk_grid] first tile of each walker's slice (D2)
  int walk_grid;
  float4 *rec;
  int2 *rec_rc;   // (r as float bits, tile-local first bin i0 | j0 << 16; stray: absolute i0 | j0 << 16 | 1 << 31)
  int *rec_cell;  // own cell index (the tile-ordered list, kept between sorts)
  float2 *rec_wh; // (w, h) of the listed cell
  // sort reuse: [0] re-sort requested, [1] strays of the last evaluation, [2]
  // strays of this one (scatter), [3] sorts performed.  The sort kernels run when force_sort,
  // [0] or [1] > resort_thr, and return at once otherwise
  int *sortctl;
  int *host_ctl;   // mapped pinned host word: the gather publishes the last evaluation's strays to the host
  int force_sort, resort_thr;
  int early_gather;   // (gather) the ring starts before griddepcontrol.wait (DP_EARLY_GATHER=0: at the top)
  int early;       // (scatter) the predecessor writes only the map: ring start, list copies and the first
                   // position loads run before griddepcontrol.wait
  int merge;       // walker slices per CTA (the scatter with DP_SCATTER_MERGE = 2: one CTA per SM)
  int rec_hint;    // DP_REC_HINT=1: records stored evict-last by the scatter, read evict-first by the gather
  int write_rec;   // the scatter writes footprint records (the gather reads them; 0: it recomputes)
  unsigned long long *rho;   // int64 fixed point, 2^-kRhoScaleLog2 units
  const float2 *xi;
  float2 *force;
  const int *large;
  // direct output (DP_DIRECT): the gather adds lambda * dD/dx straight into the caller's gx, gy
  // (zeroed at the head of the call, the WA kernel adds into them too) instead of storing force
  float *gxo, *gyo;
  // fused combine (DP_FUSE_COMBINE): the gather writes gx = g2.x + lambda force.x (the WA
  // accumulator is complete: the gather waits for the WA stream) and no force / combine pass
  float *gxf, *gyf;
  const float2 *g2f;
  float lambda;
  const float *lambda_dev;
  // fixed cells (NEXT-4, dp_set_fixed): with a mask, only cells whose flag equals sel are
  // sorted and scattered (sel = 0: the movable cells of an evaluation, whose map starts from
  // the precomputed fixed-charge map; sel = 1: building that map)
  const uint8_t *fixed;
  int sel;
  int keep;   // fence regions: cells of other regions are skipped without writing their force
  int sync_ring;   // DP_WALK_SYNC=1: a block barrier before each ring refill (racecheck diagnostics)
  int n_large;
};

__device__ __forceinline__ bool selected(const DenArgs &a, int i) { return !a.fixed || a.fixed[i] == a.sel; }

__device__ __forceinline__ void red_f32(float *p, float v) {
  asm volatile("red.global.add.f32 [%0], %1;" ::"l"(p), "f"(v) : "memory");
}

// Stretched, clipped footprint of a cell in BIN units (readings A10, A11):
//   lo = (x - xl)/b_x + (w - w')/2 / b_x, hi = lo + w'/b_x, clipped to [0, M].
// Formulated as a few fp64 FMAs from the fp32 inputs; count and place evaluate it identically,
// so their tile choices agree.  The charge ratio r = w h / (w' h') is fp32 (stored as fp32).
struct Foot {
  double lo_x, hi_x, lo_y, hi_y;
  float r;
  bool large, empty;
};

__device__ __forceinline__ Foot footprint_v(const DenArgs &a, float x, float y, float w, float h) {
  Foot f;
  const float ws = a.stretch ? fmaxf(w, a.sxf) : w;
  const float hs = a.stretch ? fmaxf(h, a.syf) : h;
  f.large = ((double)w > 2.0 * a.bx) || ((double)h > 2.0 * a.by);   // same test as dp_create's list
  f.r = (ws * hs > 0.f) ? __fdividef(w * h, ws * hs) : 0.f;
  const double lx = fma((double)(0.5f * (w - ws)), a.ibx, fma((double)x, a.ibx, a.cx0));
  const double ly = fma((double)(0.5f * (h - hs)), a.iby, fma((double)y, a.iby, a.cy0));
  f.hi_x = fmin(fma((double)ws, a.ibx, lx), (double)a.mx);
  f.hi_y = fmin(fma((double)hs, a.iby, ly), (double)a.my);
  f.lo_x = fmax(lx, 0.0);
  f.lo_y = fmax(ly, 0.0);
  f.empty = !(f.hi_x > f.lo_x && f.hi_y > f.lo_y && f.r > 0.f);
  return f;
}

__device__ __forceinline__ Foot footprint(const DenArgs &a, int i) {
  return footprint_v(a, __ldg(a.x + a.cell_begin + i), __ldg(a.y + a.cell_begin + i), __ldg(a.w + i), __ldg(a.h + i));
}

// Small-cell classification shared by count (D1), place (D3) and the scatter walker (D4), which
// must agree exactly: returns -2 for a large cell (CTA-per-cell path), else the tile of the
// footprint's first bin clamped to the map; f.ok is false for an empty footprint (outside the
// region or zero area: the cell stays listed, in the clamped tile, so that it is found again when
// it moves back, and the gather writes its zero force).  Only the lower corner (lx, ly) and the upper
// corner (hx, hy) are formed in fp64 (unclipped); ok equals footprint_v's "not empty" (hi > lo
// after clipping to [0, M]) without fp64 min/max.
struct SmallFoot {
  double lx, ly, hx, hy;
  float ws, hs;
  int bi, bj;
  bool ok;
};

__device__ __forceinline__ int classify_small(const DenArgs &a, float x, float y, float w, float h, SmallFoot &f) {
  if (w > a.w_large || h > a.h_large) return -2;
  f.ws = a.stretch ? fmaxf(w, a.sxf) : w;
  f.hs = a.stretch ? fmaxf(h, a.syf) : h;
  f.lx = fma((double)(0.5f * (w - f.ws)), a.ibx, fma((double)x, a.ibx, a.cx0));
  f.ly = fma((double)(0.5f * (h - f.hs)), a.iby, fma((double)y, a.iby, a.cy0));
  f.hx = fma((double)f.ws, a.ibx, f.lx);
  f.hy = fma((double)f.hs, a.iby, f.ly);
  f.ok = f.hx > f.lx && f.hx > 0.0 && f.lx < (double)a.mx && f.hy > f.ly && f.hy > 0.0 && f.ly < (double)a.my &&
         w * h > 0.f;
  f.bi = max(0, min(__double2int_rz(f.lx), a.mx - 1));
  f.bj = max(0, min(__double2int_rz(f.ly), a.my - 1));
  return (f.bi >> a.tile_log2) * a.tiles_y + (f.bj >> a.tile_log2);
}

// D1-D3 run only when the tile-ordered list must be rebuilt (every CTA reads the same words: they
// change only in the scatter and the gather, after the sort)
__device__ __forceinline__ bool sort_needed(const DenArgs &a) {
  return a.force_sort || *(volatile int *)a.sortctl != 0 || *(volatile int *)(a.sortctl + 1) > a.resort_thr;
}

// first bin of a (non-empty) footprint and its tile
__device__ __forceinline__ int small_tile(const DenArgs &a, const Foot &f, int &bx0, int &by0) {
  bx0 = min((int)f.lo_x, a.mx - 1);
  by0 = min((int)f.lo_y, a.my - 1);
  return (bx0 >> a.tile_log2) * a.tiles_y + (by0 >> a.tile_log2);
}

// Each thread of a count / place CTA holds kCellsPerThread cells (cell i0 + k * blockDim + tid,
// coalesced loads, all issued before the first use); out-of-range cells are empty.
constexpr int kCellsPerThread = kCountCells / kCountThreads;

__device__ __forceinline__ void load_cells(const DenArgs &a, int i0, float (&x)[kCellsPerThread],
                                           float (&y)[kCellsPerThread], float (&w)[kCellsPerThread],
                                           float (&h)[kCellsPerThread]) {
#pragma unroll
  for (int k = 0; k < kCellsPerThread; k++) {
    const int i = i0 + k * kCountThreads + threadIdx.x;
    const bool ok = i < a.n_own;
    x[k] = ok ? __ldg(a.x + a.cell_begin + i) : 0.f;
    y[k] = ok ? __ldg(a.y + a.cell_begin + i) : 0.f;
    w[k] = ok ? __ldg(a.w + i) : 0.f;
    h[k] = ok ? __ldg(a.h + i) : 0.f;
  }
}

// D1: per-CTA shared histogram of tile ids
// MASK: a fixed-cell mask is in effect (dp_set_fixed with fixed small cells); a separate
// instantiation keeps the default path's register budget (and occupancy) unchanged
template <bool MASK>
__global__ void __launch_bounds__(kCountThreads) k_count(DenArgs a) {
  griddep_wait();
  if (!sort_needed(a)) return;
  extern __shared__ int s_hist[];
  for (int t = threadIdx.x; t < a.ntiles; t += kCountThreads) s_hist[t] = 0;
  __syncthreads();
  // persistent: one CTA per resident slot walks cell blocks blockIdx.x, + gridDim.x, ... (no
  // partial last wave) and flushes its histogram once
  const int nblk = (a.n_own + kCountCells - 1) / kCountCells;
  for (int blk = blockIdx.x; blk < nblk; blk += gridDim.x) {
    const int i0 = blk * kCountCells;
    float x[kCellsPerThread], y[kCellsPerThread], w[kCellsPerThread], h[kCellsPerThread];
    load_cells(a, i0, x, y, w, h);
#pragma unroll
    for (int k = 0; k < kCellsPerThread; k++) {
      SmallFoot f;
      const int i = i0 + k * kCountThreads + threadIdx.x;
      const int t = classify_small(a, x[k], y[k], w[k], h[k], f);
      // (lanes past n_own load w = h = 0 and classify like a zero-area cell: not counted)
      if (t >= 0 && i < a.n_own && (!MASK || selected(a, i))) atomicAdd(&s_hist[t], 1);
    }
  }
  __syncthreads();
  for (int t = threadIdx.x; t < a.ntiles; t += kCountThreads)
    if (s_hist[t]) atomicAdd(a.tile_cnt + t * kCntStride, s_hist[t]);
}

// D2 (single CTA of 1024 threads): exclusive scan of the tile counts with warp shuffles (two
// barriers) -> tile offsets and cursors; resets the counts for the next call.
__device__ __forceinline__ int warp_incl_scan(int v, int lane) {
#pragma unroll
  for (int o = 1; o < 32; o <<= 1) {
    const int t = __shfl_up_sync(0xffffffffu, v, o);
    if (lane >= o) v += t;
  }
  return v;
}

__global__ void __launch_bounds__(1024) k_scan(DenArgs a) {
  griddep_wait();
  if (!sort_needed(a)) return;
  if (threadIdx.x == 0) a.sortctl[3]++;
  __shared__ int s_wa[32];
  constexpr int T = 1024;
  const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
  const int per = (a.ntiles + T - 1) / T;
  const int t0 = threadIdx.x * per;
  int cnt_sum = 0;
  for (int k = 0; k < per; k++)
    if (t0 + k < a.ntiles) cnt_sum += a.tile_cnt[(t0 + k) * kCntStride];
  const int ia = warp_incl_scan(cnt_sum, lane);
  if (lane == 31) s_wa[warp] = ia;
  __syncthreads();
  if (warp == 0) s_wa[lane] = warp_incl_scan(s_wa[lane], lane);
  __syncthreads();
  const long long N = s_wa[31], G = a.walk_grid;
  int off_c = (warp ? s_wa[warp - 1] : 0) + ia - cnt_sum;
  for (int k = 0; k < per; k++) {
    const int t = t0 + k;
    if (t < a.ntiles) {
      const int c = a.tile_cnt[t * kCntStride];
      a.tile_off[t] = off_c;
      a.tile_cursor[t * kCntStride] = off_c;
      // walkers whose slice [N g / G, N (g + 1) / G) starts in this tile:
      // off <= floor(N g / G) < off + c  <=>  ceil(off G / N) <= g < ceil((off + c) G / N)
      if (c > 0) {
        const long long g0 = ((long long)off_c * G + N - 1) / N, g1 = ((long long)(off_c + c) * G + N - 1) / N;
        for (long long g = g0; g < g1; g++) a.walk_tile[g] = t;
      }
      off_c += c;
      a.tile_cnt[t * kCntStride] = 0;  // ready for the next evaluation
    }
  }
  if (threadIdx.x == T - 1) a.tile_off[a.ntiles] = off_c;
}

// D3: the same cells as D1.  The shared histogram's atomicAdd returns each cell's rank inside
// its tile; a block scan of the histogram (with one global reservation per non-empty tile) gives
// the local tile-ordered slots; the list entries (cell, w, h) are assembled in shared memory and
// written out in contiguous per-tile runs (random per-record stores were measured 3x slower).
// The footprints themselves are formed by the scatter walker on every evaluation (the list is
// kept while the cells stay in their tiles).
struct PlaceOut {
  float2 wh[kCountCells];
  int cell[kCountCells];
  int tile[kCountCells];
};

int place_smem_bytes(int ntiles) { return (int)sizeof(PlaceOut) + 8 * ntiles; }

template <bool MASK>
__global__ void __launch_bounds__(kCountThreads) k_place(DenArgs a) {
  griddep_wait();
  if (!sort_needed(a)) return;
  extern __shared__ __align__(16) unsigned char psm[];
  PlaceOut &po = *reinterpret_cast<PlaceOut *>(psm);
  int *s_hist = reinterpret_cast<int *>(psm + sizeof(PlaceOut));   // [ntiles] counts -> local offsets
  int *s_base = s_hist + a.ntiles;                                  // [ntiles] global bases
  __shared__ int s_warp[kCountThreads / 32];
  const int i0 = blockIdx.x * kCountCells;
  for (int t = threadIdx.x; t < a.ntiles; t += kCountThreads) s_hist[t] = 0;
  float x[kCellsPerThread], y[kCellsPerThread], w[kCellsPerThread], h[kCellsPerThread];
  load_cells(a, i0, x, y, w, h);
  __syncthreads();
  int tl[kCellsPerThread], rank[kCellsPerThread];
#pragma unroll
  for (int k = 0; k < kCellsPerThread; k++) {
    const int i = i0 + k * kCountThreads + threadIdx.x;
    SmallFoot f;
    int t = classify_small(a, x[k], y[k], w[k], h[k], f);
    tl[k] = -1;
    if (i >= a.n_own || t == -2) continue;
    if (MASK && !selected(a, i)) {   // fixed cell of an evaluation: not listed, force 0;
      if (a.keep) continue;          // another region's cell: its own pass writes its force
      t = -3;
    }
    if (t == -3) {   // a fixed cell of an evaluation (never in the map): force 0, kept until the next sort
      a.force[i] = make_float2(0.f, 0.f);
      continue;
    }
    tl[k] = t;
    rank[k] = atomicAdd(&s_hist[t], 1);
  }
  __syncthreads();
  // reservation + block exclusive scan of the histogram (tiles split evenly over the threads)
  const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
  const int per = (a.ntiles + kCountThreads - 1) / kCountThreads, t0 = threadIdx.x * per;
  int sum = 0;
  for (int q = 0; q < per; q++) {
    const int t = t0 + q;
    if (t < a.ntiles) {
      const int cnt = s_hist[t];
      if (cnt) s_base[t] = atomicAdd(a.tile_cursor + t * kCntStride, cnt);
      sum += cnt;
    }
  }
  const int incl = warp_incl_scan(sum, lane);
  if (lane == 31) s_warp[warp] = incl;
  __syncthreads();
  if (warp == 0) {
    const int v = lane < kCountThreads / 32 ? s_warp[lane] : 0;
    const int ws = warp_incl_scan(v, lane);
    if (lane < kCountThreads / 32) s_warp[lane] = ws;
  }
  __syncthreads();
  int run = (warp ? s_warp[warp - 1] : 0) + incl - sum;
  for (int q = 0; q < per; q++) {
    const int t = t0 + q;
    if (t < a.ntiles) {
      const int cnt = s_hist[t];
      s_hist[t] = run;
      run += cnt;
    }
  }
  __syncthreads();
#pragma unroll
  for (int k = 0; k < kCellsPerThread; k++) {
    if (tl[k] < 0) continue;
    const int slot = s_hist[tl[k]] + rank[k];
    po.wh[slot] = make_float2(w[k], h[k]);
    po.cell[slot] = i0 + k * kCountThreads + threadIdx.x;
    po.tile[slot] = tl[k];
  }
  __syncthreads();
  const int total = s_warp[kCountThreads / 32 - 1];
  for (int j = threadIdx.x; j < total; j += kCountThreads) {
    const int t = po.tile[j];
    const int pos = s_base[t] + (j - s_hist[t]);
    a.rec_wh[pos] = po.wh[j];
    a.rec_cell[pos] = po.cell[j];
  }
}

// Record staging ring: kStages buffers of up to kStageRecs records, each completing on its own
// mbarrier: the scatter stages the list (rec_cell 4 B, rec_wh 8 B in the rc slot), the gather the
// footprint records the scatter wrote (rec 16 B, rec_rc 8 B, rec_cell 4 B).  Thread 0 owns the walker and keeps
// kStages - 1 chunks in flight; the chunk descriptors live in shared memory next to the data.
// The copied range is rounded out to 4-record multiples (the record arrays are padded by 8).
constexpr int kStages = 4;
struct RecBufG {   // gather: footprint records
  float4 rec[kStageRecs + 8];
  int2 rc[kStageRecs + 8];
  int cell[kStageRecs + 8];
};
struct RecBufS {   // scatter: list entries
  float2 wh[kStageRecs + 8];
  int cell[kStageRecs + 8];
};
struct WalkChunk {
  int begin, end, tile, off;
};
template <class Buf>
struct RecStage {
  Buf buf[kStages];
  WalkChunk ch[kStages];
  uint64_t bar[kStages];     // full: descriptor + records landed (one arrival by the producer + tx bytes)
  uint64_t empty[kStages];   // released: every warp has consumed the buffer (one arrival per warp)
  uint64_t bar_xi;
};
using StageG = RecStage<RecBufG>;
using StageS = RecStage<RecBufS>;

template <class St>
__host__ __device__ constexpr int stage_bytes() { return (int)((sizeof(St) + 15) & ~(size_t)15); }
__host__ __device__ constexpr int walk_span(int tile) { return tile + kHalo + 2 * kMargin; }   // shared tile side
// the scatter's CTA is the smaller (12-byte list entries, a 32-bit word per bin), so WA CTAs fit
// beside it; both walkers run the same grid (the gather's occupancy)
int scatter_smem_bytes(int tile) { return stage_bytes<StageS>() + walk_span(tile) * walk_span(tile) * 4; }
int walk_smem_bytes(int tile) { return stage_bytes<StageG>() + walk_span(tile) * walk_span(tile) * 8; }

__device__ __forceinline__ unsigned issue_copies(const DenArgs &a, RecBufG &B, int b0, int n, uint64_t *bar) {
  if (n > 0) {
    if (a.rec_hint) {   // the records' last use: evict-first
      const uint64_t pol = l2_evict_first_policy();
      bulk_g2s_hint(B.rec, a.rec + b0, 16u * n, bar, pol);
      bulk_g2s_hint(B.rc, a.rec_rc + b0, 8u * n, bar, pol);
    } else {
      bulk_g2s(B.rec, a.rec + b0, 16u * n, bar);
      bulk_g2s(B.rc, a.rec_rc + b0, 8u * n, bar);
    }
    bulk_g2s(B.cell, a.rec_cell + b0, 4u * n, bar);
  }
  return 28u;
}
__device__ __forceinline__ unsigned issue_copies(const DenArgs &a, RecBufS &B, int b0, int n, uint64_t *bar) {
  if (n > 0) {
    bulk_g2s(B.wh, a.rec_wh + b0, 8u * n, bar);
    bulk_g2s(B.cell, a.rec_cell + b0, 4u * n, bar);
  }
  return 12u;
}

// A walker's slice [rb, re) of the tile-ordered small-cell records, cut into chunks of at most
// kStageRecs records that never straddle a tile.
struct Walker {
  int cur, re, t, tend;
};

__device__ __forceinline__ void walk_init(const DenArgs &a, Walker &w) {
  // a CTA covers a.merge consecutive walker slices (the scatter with DP_SCATTER_MERGE; else 1)
  const int N = a.tile_off[a.ntiles];
  const int m = a.merge, G = gridDim.x * m, g0 = blockIdx.x * m;
  w.cur = (int)(((long long)N * g0) / G);
  w.re = (int)(((long long)N * (g0 + m)) / G);
  w.t = 0;
  w.tend = 0;
  if (w.cur >= w.re) return;
  w.t = a.walk_tile[g0];   // from D2: tile_off[t] <= cur < tile_off[t + 1]
  w.tend = a.tile_off[w.t + 1];
}

// (thread 0) next chunk of the slice -> descriptor slot b, copies issued on bar[b].  The
// descriptor is written before the arrival, so a consumer that sees the phase complete sees it;
// an empty chunk (end of the slice) completes its phase with no bytes.
template <class St>
__device__ __forceinline__ void walk_issue(const DenArgs &a, Walker &w, St &st, int b) {
  WalkChunk c;
  c.begin = c.end = w.cur;
  c.tile = w.t;
  c.off = 0;
  int b0 = 0, n = 0;
  if (w.cur < w.re) {
    while (w.tend <= w.cur) w.tend = a.tile_off[++w.t + 1];   // skip finished / empty tiles
    c.tile = w.t;
    c.end = min(min(w.cur + kStageRecs, w.tend), w.re);
    w.cur = c.end;
    b0 = c.begin & ~3;
    n = ((c.end + 3) & ~3) - b0;
    c.off = c.begin - b0;
  }
  st.ch[b] = c;
  // the arrival (with the byte count) precedes the copies; an empty chunk completes with no bytes
  constexpr unsigned per = sizeof(st.buf[0]) == sizeof(RecBufG) ? 28u : 12u;
  mbar_expect_tx(&st.bar[b], (unsigned)n * per);
  issue_copies(a, st.buf[b], b0, n, &st.bar[b]);
}

// (thread 0) barriers + the first kStages - 1 chunks; the caller synchronises
template <class St>
__device__ __forceinline__ void walk_start(const DenArgs &a, Walker &w, St &st) {
  walk_init(a, w);
  for (int b = 0; b < kStages; b++) {
    mbar_init(&st.bar[b]);
    mbar_init_count(&st.empty[b], blockDim.x >> 5);
  }
  mbar_init(&st.bar_xi);
  for (int b = 0; b < kStages - 1; b++) walk_issue(a, w, st, b);
}

// Ring step of chunk c (every thread): wait until chunk c has landed; thread 0 then refills the
// buffer of chunk c - 1 with chunk c + kStages - 1 once every warp has released chunk c - 1.
// Warps move through the ring independently: there is no block barrier per chunk.  The ordering
// of a warp's reads of buffer b2 (and of its descriptor st.ch[b2]) before thread 0 refills it is
// the empty[b2] mbarrier: each warp's mbarrier.arrive (release, CTA scope) after its last read,
// thread 0's try_wait (acquire) before the refill.  compute-sanitizer racecheck does not model
// mbarrier ordering and reports the descriptor refill as a WAR hazard; a.sync_ring
// (DP_WALK_SYNC=1, diagnostics only) adds a block barrier before each refill, under which
// racecheck reports none (profiles/r02_sanitizer_racecheck*.log).
template <class St>
__device__ __forceinline__ WalkChunk walk_next(const DenArgs &a, Walker &w, St &st, int c) {
  const int b = c % kStages;
  mbar_wait(&st.bar[b], (c / kStages) & 1);
  const WalkChunk cc = st.ch[b];
  if (a.sync_ring) __syncthreads();   // uniform: every thread reaches it
  if (threadIdx.x == 0 && cc.begin < cc.end) {
    const int b2 = (c + kStages - 1) % kStages;
    if (c >= 1) mbar_wait(&st.empty[b2], ((c - 1) / kStages) & 1);
    walk_issue(a, w, st, b2);
  }
  return cc;
}

// this warp is done with chunk c's buffer
template <class St>
__device__ __forceinline__ void walk_release(St &st, int c) {
  __syncwarp();
  if ((threadIdx.x & 31) == 0) mbar_arrive(&st.empty[c % kStages]);
}

// overlaps (bin units) of a record's footprint with the 3 bins from its first bin, per axis;
// clipping makes out-of-map / non-covered overlaps 0
__device__ __forceinline__ void rec_overlaps(const float4 q, float ox3[3], float oy3[3]) {
#pragma unroll
  for (int d = 0; d < 3; d++) {
    ox3[d] = fmaxf(fminf(q.z, (float)(d + 1)) - fmaxf(q.x, (float)d), 0.f);
    oy3[d] = fmaxf(fminf(q.w, (float)(d + 1)) - fmaxf(q.y, (float)d), 0.f);
  }
}

// flush the shared tile accumulators into rho and clear them (caller synchronises before and
// after).  Each word holds its bin's sum modulo 2^32 (units 2^-29); the wraps were already added
// to rho by the threads whose atomic crossed 2^32, so rho + word is the exact int64 sum.
__device__ __forceinline__ void flush_tile(const DenArgs &a, unsigned *s_acc, int tile) {
  const int P = walk_span(a.tile);   // even: word pairs (8-byte shared loads / stores)
  const int ox = (tile / a.tiles_y) * a.tile - kMargin, oy = (tile % a.tiles_y) * a.tile - kMargin;
  const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5, nw = blockDim.x >> 5;
  uint2 *s2 = reinterpret_cast<uint2 *>(s_acc);
  for (int i = warp; i < P; i += nw) {
    const int gi = ox + i;
    const bool row_in = (unsigned)gi < (unsigned)a.mx;
    for (int j2 = lane; j2 < P / 2; j2 += 32) {
      const int k2 = i * (P / 2) + j2;
      const uint2 v = s2[k2];
      s2[k2] = make_uint2(0u, 0u);
      const int gj = oy + 2 * j2;
      if (row_in && (v.x | v.y)) {
        unsigned long long *dst = a.rho + (size_t)gi * a.my + gj;
        if (v.x && (unsigned)gj < (unsigned)a.my)
          asm volatile("red.global.add.u64 [%0], %1;" ::"l"(dst), "l"((unsigned long long)v.x) : "memory");
        if (v.y && (unsigned)(gj + 1) < (unsigned)a.my)
          asm volatile("red.global.add.u64 [%0], %1;" ::"l"(dst + 1), "l"((unsigned long long)v.y) : "memory");
      }
    }
  }
}

// shared-memory add returning the old word (native 32-bit ATOMS.ADD on sm_100a)
__device__ __forceinline__ unsigned atom_shared_add(unsigned *p, unsigned v) {
  unsigned old;
  asm volatile("atom.shared.add.u32 %0, [%1], %2;" : "=r"(old) : "r"(smem_u32(p)), "r"(v) : "memory");
  return old;
}

// m <- 2 m + carry(old + u): the wrap mask of a record's nine adds in two instructions per add
// (the carry out of the 32-bit sum, shifted in; the first add ends up in bit 8)
__device__ __forceinline__ unsigned carry_in(unsigned m, unsigned old, unsigned u) {
  unsigned t, r;
  asm("{\n\tadd.cc.u32 %0, %2, %3;\n\taddc.u32 %1, %4, %4;\n\t}" : "=r"(t), "=r"(r) : "r"(old), "r"(u), "r"(m));
  return r;
}

// D4: persistent scatter walker.  Each listed cell's footprint is formed here from its current
// position (the classifier of D1-D3, fp64 corners): the record (fractions of the first bin, r,
// first bin) is written to the cell's slot for the gather.  A cell whose first bin is still in
// the walker's tile adds into the (tile+2)^2 shared tile: one 32-bit word per bin accumulating
// u = floor(v 2^29) (v <= 1, so u <= 2^29) with a native shared atomic add that returns the old
// word; the (rare) thread whose add wraps past 2^32 adds 2^32 units to the int64 map itself.  A
// cell that has left its tile since the last sort (a stray) adds the same u straight to the int64
// map.  The word is flushed when the slice leaves the tile.  The map is the exact sum of the
// per-contribution roundings whatever the order or path (bit-identical to a fresh sort).
static_assert(kStageRecs == kTileThreads, "the scatter walker holds one record per thread and chunk");

// (scatter) this thread's list entry of a landed chunk and the cell's current position: the
// position loads are random L2 reads, issued one chunk ahead of their use
struct ScatterIn {
  int cell;
  float2 wh;
  float x, y;
};

__device__ __forceinline__ void scatter_fetch(const DenArgs &a, const StageS &st, int b, const WalkChunk &cc,
                                              ScatterIn &in) {
  if ((int)threadIdx.x < cc.end - cc.begin) {
    in.cell = st.buf[b].cell[cc.off + threadIdx.x];
    in.wh = st.buf[b].wh[cc.off + threadIdx.x];
    in.x = __ldg(a.x + a.cell_begin + in.cell);
    in.y = __ldg(a.y + a.cell_begin + in.cell);
  }
}

// The record of a listed cell at its current position, relative to a shared tile whose origin is
// (tox, toy) and which takes first bins [0, span) per axis: fractions of the first bin q, charge
// ratio rr, the first bin (tile-local, or absolute for a stray).  The scatter and the recomputing
// gather form it with this one function, so both see the same footprint bit for bit.
struct FootRec {
  float4 q;
  float rr;
  int i0, j0;
  bool ok, stray;
};

__device__ __forceinline__ FootRec make_rec(const DenArgs &a, const ScatterIn &in, int tox, int toy, int span) {
  FootRec fr;
  SmallFoot f;
  classify_small(a, in.x, in.y, in.wh.x, in.wh.y, f);   // listed cells are small
  fr.q = make_float4(0.f, 0.f, 0.f, 0.f);
  fr.rr = 0.f;
  fr.i0 = fr.j0 = 0;
  fr.ok = f.ok;
  fr.stray = false;
  if (f.ok) {
    const int bi = f.bi, bj = f.bj;
    // bin-local fractions (|v| < 3) of the clipped footprint [max(l, 0), min(h, M)]: fp32 keeps
    // ~2e-7 bin absolute precision, which the force gather needs where large opposite bin
    // fields cancel (the 'initial' placement).  fl(max(l, 0) - b) = max(fl(l - b), -b)
    fr.q = make_float4(fmaxf((float)(f.lx - bi), (float)-bi), fmaxf((float)(f.ly - bj), (float)-bj),
                       fminf((float)(f.hx - bi), (float)(a.mx - bi)), fminf((float)(f.hy - bj), (float)(a.my - bj)));
    fr.rr = __fdividef(in.wh.x * in.wh.y, f.ws * f.hs);
    fr.i0 = bi - tox;
    fr.j0 = bj - toy;
    fr.stray = (unsigned)fr.i0 >= (unsigned)span || (unsigned)fr.j0 >= (unsigned)span;
    if (fr.stray) {
      fr.i0 = bi;
      fr.j0 = bj;
    }
  }
  return fr;
}

__global__ void __launch_bounds__(kTileThreads) k_scatter_walk(DenArgs a) {
  if (!a.early) griddep_wait();
  extern __shared__ __align__(16) unsigned char dsm[];
  StageS &st = *reinterpret_cast<StageS *>(dsm);
  unsigned *s_acc = reinterpret_cast<unsigned *>(dsm + stage_bytes<StageS>());   // 2^-29 units, mod 2^32
  const int P = walk_span(a.tile);
  const int span = a.tile + 2 * kMargin;   // first bins the shared tile takes
  Walker w;
  if (threadIdx.x == 0) {
    if (blockIdx.x == 0) a.sortctl[0] = 0;   // a requested sort has run (D1-D3 precede this kernel)
    walk_start(a, w, st);
  }
  for (int k = threadIdx.x; k < P * P; k += blockDim.x) s_acc[k] = 0u;
  __syncthreads();
  const float scale_fx = (float)(1u << kRhoScaleLog2);
  uint64_t pol_last = 0;
  if (a.rec_hint) asm volatile("createpolicy.fractional.L2::evict_last.b64 %0, 1.0;" : "=l"(pol_last));
  int cur_tile = -1;
  int tox = 0, toy = 0;   // origin of the shared tile (first bin of the tile - kMargin)
  unsigned strays = 0;
  WalkChunk cc = walk_next(a, w, st, 0);
  ScatterIn in = {0, make_float2(0.f, 0.f), 0.f, 0.f};
  scatter_fetch(a, st, 0, cc, in);
  if (a.early) griddep_wait();   // the map is zeroed: from here on it is written
  for (int c = 0; cc.begin < cc.end; c++) {
    const int n = cc.end - cc.begin;
    if (cc.tile != cur_tile) {   // uniform: every warp sees the same chunks
      if (cur_tile >= 0) {
        __syncthreads();   // the tile is complete
        flush_tile(a, s_acc, cur_tile);
        __syncthreads();   // flushed and cleared
      }
      cur_tile = cc.tile;
      tox = (cur_tile / a.tiles_y) * a.tile - kMargin;
      toy = (cur_tile % a.tiles_y) * a.tile - kMargin;
    }
    // chunk c + 1 was issued (non-empty chunks c, c - 1, c - 2 refilled the ring): its entries and
    // positions are fetched now and arrive while this chunk is processed
    const int b1 = (c + 1) % kStages;
    mbar_wait(&st.bar[b1], ((c + 1) / kStages) & 1);
    const WalkChunk cn = st.ch[b1];
    ScatterIn nx = in;
    scatter_fetch(a, st, b1, cn, nx);
    if ((int)threadIdx.x < n) {
      const FootRec fr = make_rec(a, in, tox, toy, span);
      const float4 q = fr.q;
      const int2 rc = make_int2(__float_as_int(fr.rr), fr.stray ? (int)(fr.i0 | (fr.j0 << 16) | 0x80000000u)
                                                                : (fr.i0 | (fr.j0 << 16)));
      if (fr.ok) {
        const bool stray = fr.stray;
        const int i0 = fr.i0, j0 = fr.j0, bi = fr.i0 + (stray ? 0 : tox), bj = fr.j0 + (stray ? 0 : toy);
        const float rr = fr.rr;
        const float r = rr * scale_fx;   // r 2^29
        float ox3[3], oy3[3];
        rec_overlaps(q, ox3, oy3);
        if (!stray) {
          const int base = i0 * P + j0;
          unsigned wrapped = 0u;   // bit 8 - (3 di + dj): that word's add wrapped past 2^32
#pragma unroll
          for (int di = 0; di < 3; di++) {
            const float rx = r * ox3[di];
#pragma unroll
            for (int dj = 0; dj < 3; dj++) {
              const unsigned u = (unsigned)(rx * oy3[dj]);   // floor(v 2^29) <= 2^29 (power-of-two scaling is exact)
              const unsigned old = atom_shared_add(s_acc + base + di * P + dj, u);
              wrapped = carry_in(wrapped, old, u);
            }
          }
          // wrapped words (rare): 2^32 units (8 bin areas) each go straight to the map.  Collected
          // as a mask so that the map addresses are formed only here (as predicated reductions
          // inside the loop, they were computed for all nine bins of every record)
          if (wrapped) {
            while (wrapped) {
              const int bit = 8 - (__ffs(wrapped) - 1);   // add index 3 di + dj
              wrapped &= wrapped - 1;
              asm volatile("red.global.add.u64 [%0], %1;" ::"l"(a.rho + (size_t)(bi + bit / 3) * a.my + bj + bit % 3),
                           "l"(1ull << 32)
                           : "memory");
            }
          }
        } else {   // stray: the same units straight into the map (bins past the map have zero overlap)
          strays++;
#pragma unroll
          for (int di = 0; di < 3; di++) {
            const float rx = r * ox3[di];
#pragma unroll
            for (int dj = 0; dj < 3; dj++) {
              const unsigned u = (unsigned)(rx * oy3[dj]);
              if (u)
                asm volatile("red.global.add.u64 [%0], %1;" ::"l"(a.rho + (size_t)(bi + di) * a.my + bj + dj),
                             "l"((unsigned long long)u)
                             : "memory");
            }
          }
        }
      }
      if (a.write_rec) {   // the records of the record-reading gather
        if (a.rec_hint) {   // kept in L2 for the gather (evict-last)
          asm volatile("st.global.L2::cache_hint.v4.f32 [%0], {%1, %2, %3, %4}, %5;" ::"l"(a.rec + cc.begin + threadIdx.x),
                       "f"(q.x), "f"(q.y), "f"(q.z), "f"(q.w), "l"(pol_last)
                       : "memory");
          asm volatile("st.global.L2::cache_hint.v2.s32 [%0], {%1, %2}, %3;" ::"l"(a.rec_rc + cc.begin + threadIdx.x),
                       "r"(rc.x), "r"(rc.y), "l"(pol_last)
                       : "memory");
        } else {
          a.rec[cc.begin + threadIdx.x] = q;
          a.rec_rc[cc.begin + threadIdx.x] = rc;
        }
      }
    }
    walk_release(st, c);
    cc = walk_next(a, w, st, c + 1);   // landed already; thread 0 refills the ring
    in = nx;
  }
  __syncthreads();
  if (cur_tile >= 0) flush_tile(a, s_acc, cur_tile);
  strays = __reduce_add_sync(0xffffffffu, strays);
  if ((threadIdx.x & 31) == 0 && strays) atomicAdd(a.sortctl + 2, (int)strays);
}

// sum over the record's 3x3 bins of ov(bin) xi(bin), from the shared field tile (first bin
// (i0, j0) tile-local) or, for a stray, the global field (absolute first bin); bins without
// overlap are not read (those past the map have none)
__device__ __forceinline__ float2 field_sum(const DenArgs &a, const float2 *s_xi, int P, float4 q, bool stray, int i0,
                                            int j0) {
  float ox3[3], oy3[3];
  rec_overlaps(q, ox3, oy3);
  float fx = 0.f, fy = 0.f;
  if (!stray) {
    const float2 *row = s_xi + i0 * P + j0;   // in bounds: i0, j0 < tile + 2 kMargin, P = that + 2
#pragma unroll
    for (int di = 0; di < 3; di++) {
      float sx = 0.f, sy = 0.f;
#pragma unroll
      for (int dj = 0; dj < 3; dj++) {
        const float2 e2 = (ox3[di] > 0.f && oy3[dj] > 0.f) ? row[di * P + dj] : make_float2(0.f, 0.f);
        sx = fmaf(oy3[dj], e2.x, sx);
        sy = fmaf(oy3[dj], e2.y, sy);
      }
      fx = fmaf(ox3[di], sx, fx);
      fy = fmaf(ox3[di], sy, fy);
    }
  } else {
    const float2 *row = a.xi + (size_t)i0 * a.my + j0;
#pragma unroll
    for (int di = 0; di < 3; di++) {
      float sx = 0.f, sy = 0.f;
#pragma unroll
      for (int dj = 0; dj < 3; dj++) {
        const float2 e2 = (ox3[di] > 0.f && oy3[dj] > 0.f) ? row[(size_t)di * a.my + dj] : make_float2(0.f, 0.f);
        sx = fmaf(oy3[dj], e2.x, sx);
        sy = fmaf(oy3[dj], e2.y, sy);
      }
      fx = fmaf(ox3[di], sx, fx);
      fy = fmaf(ox3[di], sy, fy);
    }
  }
  return make_float2(fx, fy);
}

// (gather) the force of one cell: fused combine, direct output or the force vector
__device__ __forceinline__ void gather_out(const DenArgs &a, int cell, float lam, float area, float r, float fx,
                                           float fy) {
  // dD/dx = - r sum_b ov(i,b) xi^X_b  (reading A21), ov in length^2
  if (a.gxf) {   // fused combine: exactly k_combine's fmaf(lambda, force, g2)
    const int gc = a.cell_begin + cell;
    const float2 g = a.g2f[gc];
    a.gxf[gc] = fmaf(lam, -area * r * fx, g.x);
    a.gyf[gc] = fmaf(lam, -area * r * fy, g.y);
  } else if (a.gxo) {
    const int gc = a.cell_begin + cell;
    red_f32(a.gxo + gc, lam * (-area * r * fx));
    red_f32(a.gyo + gc, lam * (-area * r * fy));
  } else {
    a.force[cell] = make_float2(-area * r * fx, -area * r * fy);
  }
}

// D5: persistent gather walker; the (tile+2)^2 float2 field tile is (re)loaded with one bulk copy
// per tile row whenever the slice enters a tile; bins outside the map read as zero.
template <class St>
__device__ __forceinline__ void load_xi_tile(const DenArgs &a, St &st, float2 *s_xi, int tile,
                                             unsigned phase) {
  const int P = walk_span(a.tile);
  const int ox = (tile / a.tiles_y) * a.tile - kMargin, oy = (tile % a.tiles_y) * a.tile - kMargin;
  // rows [r0, r1) and columns [c0, c1) of the shared tile lie in the map (c0, c1 even: 16-byte rows)
  const int r0 = max(0, -ox), r1 = min(P, a.mx - ox), c0 = max(0, -oy), c1 = min(P, a.my - oy);
  if (threadIdx.x == 0) mbar_expect_tx(&st.bar_xi, (unsigned)((r1 - r0) * (c1 - c0) * 8));
  __syncthreads();   // armed before any copy can complete
  const int row = r0 + (int)threadIdx.x;
  if (row < r1)
    bulk_g2s(s_xi + row * P + c0, a.xi + (size_t)(ox + row) * a.my + (oy + c0), 8u * (c1 - c0), &st.bar_xi);
  if (r0 > 0 || r1 < P || c0 > 0 || c1 < P) {
    const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5, nw = blockDim.x >> 5;
    for (int i = warp; i < P; i += nw)
      for (int j = lane; j < P; j += 32)
        if (i < r0 || i >= r1 || j < c0 || j >= c1) s_xi[i * P + j] = make_float2(0.f, 0.f);
    __syncthreads();
  }
  mbar_wait(&st.bar_xi, phase);
}

__global__ void __launch_bounds__(kTileThreads) k_gather_walk(DenArgs a) {
  if (!a.early_gather) griddep_wait();
  // the records were written by the scatter, which completed before the transforms began: the ring
  // starts before griddepcontrol.wait, which only the field (the predecessor's output) needs
  extern __shared__ __align__(16) unsigned char dsm[];
  StageG &st = *reinterpret_cast<StageG *>(dsm);
  float2 *s_xi = reinterpret_cast<float2 *>(dsm + stage_bytes<StageG>());
  const int P = walk_span(a.tile);
  Walker w;
  if (threadIdx.x == 0) {
    if (blockIdx.x == 0) {   // the scatter has completed: its stray count decides the next sort
      const int strays = a.sortctl[2];
      a.sortctl[1] = strays;
      a.sortctl[2] = 0;
      if (a.host_ctl) *(volatile int *)a.host_ctl = strays;   // the host's view (graph choice, §5.5)
    }
    walk_start(a, w, st);
  }
  __syncthreads();   // barriers initialised, first descriptors visible
  if (a.early_gather) griddep_wait();   // the field of the transform pass before this kernel
  int cur_tile = -1;
  unsigned xi_phase = 0;
  const float area = (float)(a.bx * a.by);
  const float lam = a.lambda_dev ? __ldg(a.lambda_dev) : a.lambda;
  for (int c = 0;; c++) {
    const int b = c % kStages;
    const WalkChunk cc = walk_next(a, w, st, c);
    if (cc.begin >= cc.end) break;
    if (cc.tile != cur_tile) {   // uniform; load_xi_tile's barrier waits until every warp left the old tile
      load_xi_tile(a, st, s_xi, cc.tile, xi_phase);
      xi_phase ^= 1u;
      cur_tile = cc.tile;
    }
    const RecBufG &B = st.buf[b];
    const int n = cc.end - cc.begin;
    for (int k = threadIdx.x; k < n; k += blockDim.x) {
      const float4 q = B.rec[cc.off + k];
      const int2 rc = B.rc[cc.off + k];
      const float r = __int_as_float(rc.x);
      const bool stray = rc.y < 0;
      const float2 fs = field_sum(a, s_xi, P, q, stray, rc.y & 0xffff, (rc.y >> 16) & 0x7fff);
      const float fx = fs.x, fy = fs.y;
      gather_out(a, B.cell[cc.off + k], lam, area, r, fx, fy);
    }
    walk_release(st, c);
  }
}

// D5' (DP_GATHER_RC): the gather walker recomputes each listed cell's footprint from its position
// (make_rec, as the scatter did) instead of reading the scatter's records: it stages the 12-byte
// list entries and prefetches the positions one chunk ahead like the scatter; no record traffic.
int gather_rc_smem_bytes(int tile) { return stage_bytes<StageS>() + walk_span(tile) * walk_span(tile) * 8; }

__global__ void __launch_bounds__(kTileThreads) k_gather_walk_rc(DenArgs a) {
  if (!a.early_gather) griddep_wait();
  extern __shared__ __align__(16) unsigned char dsm[];
  StageS &st = *reinterpret_cast<StageS *>(dsm);
  float2 *s_xi = reinterpret_cast<float2 *>(dsm + stage_bytes<StageS>());
  const int P = walk_span(a.tile);
  const int span = a.tile + 2 * kMargin;
  Walker w;
  if (threadIdx.x == 0) {
    if (blockIdx.x == 0) {   // the scatter has completed: its stray count decides the next sort
      const int strays = a.sortctl[2];
      a.sortctl[1] = strays;
      a.sortctl[2] = 0;
      if (a.host_ctl) *(volatile int *)a.host_ctl = strays;   // the host's view (graph choice, §5.5)
    }
    walk_start(a, w, st);
  }
  __syncthreads();   // barriers initialised, first descriptors visible
  if (a.early_gather) griddep_wait();   // the field of the transform pass before this kernel
  int cur_tile = -1, tox = 0, toy = 0;
  unsigned xi_phase = 0;
  const float area = (float)(a.bx * a.by);
  const float lam = a.lambda_dev ? __ldg(a.lambda_dev) : a.lambda;
  WalkChunk cc = walk_next(a, w, st, 0);
  ScatterIn in = {0, make_float2(0.f, 0.f), 0.f, 0.f};
  scatter_fetch(a, st, 0, cc, in);
  for (int c = 0; cc.begin < cc.end; c++) {
    const int n = cc.end - cc.begin;
    if (cc.tile != cur_tile) {   // uniform; load_xi_tile's barrier waits until every warp left the old tile
      load_xi_tile(a, st, s_xi, cc.tile, xi_phase);
      xi_phase ^= 1u;
      cur_tile = cc.tile;
      tox = (cur_tile / a.tiles_y) * a.tile - kMargin;
      toy = (cur_tile % a.tiles_y) * a.tile - kMargin;
    }
    const int b1 = (c + 1) % kStages;   // chunk c + 1: entries and positions fetched ahead
    mbar_wait(&st.bar[b1], ((c + 1) / kStages) & 1);
    const WalkChunk cn = st.ch[b1];
    ScatterIn nx = in;
    scatter_fetch(a, st, b1, cn, nx);
    if ((int)threadIdx.x < n) {
      const FootRec fr = make_rec(a, in, tox, toy, span);
      const float2 fs = fr.ok ? field_sum(a, s_xi, P, fr.q, fr.stray, fr.i0, fr.j0) : make_float2(0.f, 0.f);
      gather_out(a, in.cell, lam, area, fr.rr, fs.x, fs.y);
    }
    walk_release(st, c);
    cc = walk_next(a, w, st, c + 1);
    in = nx;
  }
}

// Large cells: one CTA per cell, fp64 overlaps, global reductions.
__global__ void __launch_bounds__(256) k_scatter_large(DenArgs a) {
  const int i = a.large[blockIdx.x];
  const Foot f = footprint(a, i);
  if (f.empty) return;
  const int i0 = (int)f.lo_x, i1 = min((int)ceil(f.hi_x), a.mx) - 1;
  const int j0 = (int)f.lo_y, j1 = min((int)ceil(f.hi_y), a.my) - 1;
  const int nj = j1 - j0 + 1, n = (i1 - i0 + 1) * nj;
  for (int k = threadIdx.x; k < n; k += blockDim.x) {
    const int bi = i0 + k / nj, bj = j0 + k % nj;
    const double ox = fmin(f.hi_x, (double)(bi + 1)) - fmax(f.lo_x, (double)bi);
    const double oy = fmin(f.hi_y, (double)(bj + 1)) - fmax(f.lo_y, (double)bj);
    if (ox <= 0.0 || oy <= 0.0) continue;
    const unsigned long long v =
        (unsigned long long)__double2ll_rn((double)f.r * ox * oy * (double)(1ll << kRhoScaleLog2));
    asm volatile("red.global.add.u64 [%0], %1;" ::"l"(a.rho + (size_t)bi * a.my + bj), "l"(v) : "memory");
  }
}

__global__ void __launch_bounds__(256) k_gather_large(DenArgs a) {
  const int i = a.large[blockIdx.x];
  const Foot f = footprint(a, i);
  __shared__ double s_x[8], s_y[8];
  double fx = 0.0, fy = 0.0;
  if (!f.empty) {
    const int i0 = (int)f.lo_x, i1 = min((int)ceil(f.hi_x), a.mx) - 1;
    const int j0 = (int)f.lo_y, j1 = min((int)ceil(f.hi_y), a.my) - 1;
    const int nj = j1 - j0 + 1, n = (i1 - i0 + 1) * nj;
    for (int k = threadIdx.x; k < n; k += blockDim.x) {
      const int bi = i0 + k / nj, bj = j0 + k % nj;
      const double ox = fmin(f.hi_x, (double)(bi + 1)) - fmax(f.lo_x, (double)bi);
      const double oy = fmin(f.hi_y, (double)(bj + 1)) - fmax(f.lo_y, (double)bj);
      if (ox <= 0.0 || oy <= 0.0) continue;
      const float2 e = a.xi[(size_t)bi * a.my + bj];
      fx += ox * oy * e.x;
      fy += ox * oy * e.y;
    }
  }
#pragma unroll
  for (int o = 16; o > 0; o >>= 1) {
    fx += __shfl_xor_sync(0xffffffffu, fx, o);
    fy += __shfl_xor_sync(0xffffffffu, fy, o);
  }
  if ((threadIdx.x & 31) == 0) {
    s_x[threadIdx.x >> 5] = fx;
    s_y[threadIdx.x >> 5] = fy;
  }
  __syncthreads();
  if (threadIdx.x == 0) {
    double tx = 0.0, ty = 0.0;
    for (int w = 0; w < (int)(blockDim.x >> 5); w++) {
      tx += s_x[w];
      ty += s_y[w];
    }
    const double area = a.bx * a.by;   // overlaps above are in bin units
    const float2 v = make_float2((float)(-(double)f.r * area * tx), (float)(-(double)f.r * area * ty));
    if (a.gxf) {
      const float lam = a.lambda_dev ? __ldg(a.lambda_dev) : a.lambda;
      const int gc = a.cell_begin + i;
      const float2 g = a.g2f[gc];
      a.gxf[gc] = fmaf(lam, v.x, g.x);
      a.gyf[gc] = fmaf(lam, v.y, g.y);
    } else if (a.gxo) {
      const float lam = a.lambda_dev ? __ldg(a.lambda_dev) : a.lambda;
      red_f32(a.gxo + a.cell_begin + i, lam * v.x);
      red_f32(a.gyo + a.cell_begin + i, lam * v.y);
    } else {
      a.force[i] = v;
    }
  }
}

// A30 of a fence region's map (the GP loop with dp_set_regions): the blockage counts at the
// target density like a fixed macro (A30'), rho_eff = rho - (1 - t) blockage, so only cells
// overflow; per-block partials [region][block][2] summed in a fixed order by the GP.
__global__ void __launch_bounds__(256) k_region_overflow(const unsigned long long *rho, const unsigned long long *blk,
                                                         long long nbins, double t, double *part) {
  const double unit = 1.0 / (double)(1ll << kRhoScaleLog2);
  double s = 0.0;
  for (long long b = blockIdx.x * 256ll + threadIdx.x; b < nbins; b += (long long)gridDim.x * 256)
    s += fmax(((double)rho[b] - (1.0 - t) * (double)blk[b]) * unit - t, 0.0);
  __shared__ double r0[8];
#pragma unroll
  for (int o = 16; o > 0; o >>= 1) s += __shfl_xor_sync(0xffffffffu, s, o);
  if ((threadIdx.x & 31) == 0) r0[threadIdx.x >> 5] = s;
  __syncthreads();
  if (threadIdx.x == 0) {
    double tot = 0.0;
    for (int w = 0; w < 8; w++) tot += r0[w];
    part[2 * blockIdx.x] = tot;
    part[2 * blockIdx.x + 1] = 0.0;
  }
}

// rho <- 0 as a kernel (not a memset node), so that the scatter walker can follow it with a
// programmatic dependency and run its prologue while the map is cleared
__global__ void __launch_bounds__(256) k_zero_map(unsigned long long *rho, long long nbins) {
  ulonglong2 *d = reinterpret_cast<ulonglong2 *>(rho);
  const long long n2 = nbins >> 1;   // maps are even-sized
  for (long long i = blockIdx.x * 256ll + threadIdx.x; i < n2; i += (long long)gridDim.x * 256)
    d[i] = make_ulonglong2(0ull, 0ull);
}

// Start of the map in a captured evaluation: rho <- src (the fixed-charge map) or 0, and the
// graph's IF node around D1-D3 is set to "sort needed" (sort reuse: the count, scan and place
// launches are skipped altogether when the list is kept).
__global__ void __launch_bounds__(256) k_map_init(DenArgs a, const unsigned long long *src, long long nbins,
                                                  cudaGraphConditionalHandle sort_if) {
  if (blockIdx.x == 0 && threadIdx.x == 0) cudaGraphSetConditional(sort_if, sort_needed(a) ? 1u : 0u);
  ulonglong2 *d = reinterpret_cast<ulonglong2 *>(a.rho);
  const ulonglong2 *s2 = reinterpret_cast<const ulonglong2 *>(src);
  const long long n2 = nbins >> 1;   // maps are even-sized
  for (long long i = blockIdx.x * 256ll + threadIdx.x; i < n2; i += (long long)gridDim.x * 256)
    d[i] = src ? s2[i] : make_ulonglong2(0ull, 0ull);
}

// largest float f with (double)f <= v, so that for any float w: w > f <=> (double)w > v
float float_at_most(double v) {
  float f = (float)v;
  if ((double)f > v) f = std::nextafter(f, -INFINITY);
  return f;
}

DenArgs make_args(const Ctx &c, const float *x, const float *y) {
  DenArgs a;
  a.x = x;
  a.y = y;
  a.w = c.d_cell_w;
  a.h = c.d_cell_h;
  a.cell_begin = c.cell_begin;
  a.n_own = c.n_own;
  a.xl = c.xl; a.yl = c.yl; a.xh = c.xh; a.yh = c.yh; a.bx = c.bx; a.by = c.by;
  a.sx = 1.4142135623730951 * c.bx;
  a.sy = 1.4142135623730951 * c.by;
  a.ibx = 1.0 / c.bx;
  a.iby = 1.0 / c.by;
  a.cx0 = -c.xl * a.ibx;
  a.cy0 = -c.yl * a.iby;
  a.sxf = (float)a.sx;
  a.syf = (float)a.sy;
  a.w_large = float_at_most(2.0 * c.bx);
  a.h_large = float_at_most(2.0 * c.by);
  a.mx = c.mx; a.my = c.my; a.tile = c.tile; a.tiles_y = c.tiles_y;
  a.tile_log2 = 0;
  while ((1 << a.tile_log2) < c.tile) a.tile_log2++;
  a.ntiles = c.tiles_x * c.tiles_y;
  a.stretch = c.stretch;
  a.tile_cnt = c.d_tile_cnt;
  a.tile_cursor = c.d_tile_cursor;
  a.tile_off = c.d_tile_off;
  a.walk_tile = c.d_walk_tile;
  a.walk_grid = c.walk_grid;
  a.rec = c.d_rec;
  a.rec_rc = c.d_rec_rc;
  a.rec_cell = c.d_rec_cell;
  a.rec_wh = c.d_rec_wh;
  a.sortctl = c.d_sortctl;
  a.host_ctl = c.h_ctl_dev;
  a.force_sort = c.reuse_sort ? 0 : 1;
  a.write_rec = c.gather_rc ? 0 : 1;
  a.rec_hint = c.rec_hint ? 1 : 0;
  a.merge = 1;
  a.early = 0;
  a.early_gather = c.early_gather ? 1 : 0;
  a.resort_thr = c.resort_thr;
  a.rho = c.d_rho;
  a.xi = c.d_xi;
  a.force = c.d_force;
  a.gxo = c.direct_gx;
  a.gyo = c.direct_gy;
  a.gxf = c.fused_gx;
  a.gyf = c.fused_gy;
  a.g2f = c.d_g2;
  a.lambda = c.direct_lambda;
  a.lambda_dev = c.lambda_dev;
  a.large = c.d_large;
  a.n_large = c.n_large;
  a.fixed = c.has_fixed && c.fixed_small ? c.d_fixed : nullptr;
  a.sel = 0;
  a.keep = 0;
  a.sync_ring = c.walk_sync ? 1 : 0;
  if (c.has_fixed) {
    a.large = c.d_large_mov;
    a.n_large = c.n_large_mov;
  }
  if (c.n_regions > 0 && c.cur_region >= 0) {   // fence regions: this pass's cells only
    a.fixed = c.d_region;
    a.sel = c.cur_region;
    a.keep = 1;
    a.force_sort = 1;   // one list per region pass: sorted every time
    a.large = c.d_large_reg + c.large_reg_off[c.cur_region];
    a.n_large = c.large_reg_off[c.cur_region + 1] - c.large_reg_off[c.cur_region];
  }
  return a;
}

}  // namespace

cudaError_t density_configure(int ntiles, int tile) {
  cudaError_t e = cudaFuncSetAttribute(k_count<false>, cudaFuncAttributeMaxDynamicSharedMemorySize, ntiles * 4);
  if (e != cudaSuccess) return e;
  e = cudaFuncSetAttribute(k_count<true>, cudaFuncAttributeMaxDynamicSharedMemorySize, ntiles * 4);
  if (e != cudaSuccess) return e;
  e = cudaFuncSetAttribute(k_place<false>, cudaFuncAttributeMaxDynamicSharedMemorySize, place_smem_bytes(ntiles));
  if (e != cudaSuccess) return e;
  e = cudaFuncSetAttribute(k_place<true>, cudaFuncAttributeMaxDynamicSharedMemorySize, place_smem_bytes(ntiles));
  if (e != cudaSuccess) return e;
  e = cudaFuncSetAttribute(k_scatter_walk, cudaFuncAttributeMaxDynamicSharedMemorySize, scatter_smem_bytes(tile));
  if (e != cudaSuccess) return e;
  e = cudaFuncSetAttribute(k_gather_walk_rc, cudaFuncAttributeMaxDynamicSharedMemorySize, gather_rc_smem_bytes(tile));
  if (e != cudaSuccess) return e;
  return cudaFuncSetAttribute(k_gather_walk, cudaFuncAttributeMaxDynamicSharedMemorySize, walk_smem_bytes(tile));
}

// grid of the walkers: every SM filled with as many CTAs as fit (the smaller of the two kernels'
// occupancies, so both see the same slices)
// resident CTAs of the persistent count kernel
int density_count_grid(int ntiles) {
  int dev = 0, sms = 0, o = 0;
  if (cudaGetDevice(&dev) != cudaSuccess) return 0;
  if (cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev) != cudaSuccess) return 0;
  if (cudaOccupancyMaxActiveBlocksPerMultiprocessor(&o, k_count<false>, kCountThreads, ntiles * 4) != cudaSuccess)
    return 0;
  return sms * std::max(1, o);
}

int density_walk_grid(int tile) {
  int dev = 0, sms = 0, o1 = 0, o2 = 0;
  if (cudaGetDevice(&dev) != cudaSuccess) return 0;
  if (cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev) != cudaSuccess) return 0;
  if (cudaOccupancyMaxActiveBlocksPerMultiprocessor(&o1, k_scatter_walk, kTileThreads, scatter_smem_bytes(tile)) != cudaSuccess)
    return 0;
  if (cudaOccupancyMaxActiveBlocksPerMultiprocessor(&o2, k_gather_walk, kTileThreads, walk_smem_bytes(tile)) != cudaSuccess)
    return 0;
  int per_sm = std::max(1, std::min(o1, o2));
  // DP_WALK_CTAS = k (measurement knob): at most k walker CTAs per SM, leaving shared memory for
  // the WA kernel that runs beside the scatter and the gather
  if (const char *e = std::getenv("DP_WALK_CTAS")) per_sm = std::max(1, std::min(per_sm, std::atoi(e)));
  return sms * per_sm;
}

void launch_region_overflow(const Ctx &c, cudaStream_t s) {
  if (!c.ovf_part || c.n_regions == 0 || c.cur_region < 0) return;
  const size_t nb = (size_t)c.mx * c.my;
  k_region_overflow<<<c.ovf_blocks, 256, 0, s>>>(c.d_rho, c.d_rho_block + (size_t)c.cur_region * nb, (long long)nb,
                                                 c.ovf_target, c.ovf_part + 2 * (size_t)c.cur_region * c.ovf_blocks);
}

// kernels of one evaluation's density map + gather: count, scan, place, scatter, gather, and the
// large-cell scatter / gather when there are large cells
int density_launches(const Ctx &c) { return 5 + (c.n_large > 0 ? 2 : 0); }

// aux (optional): a second stream for the large-cell CTAs, which then overlap the sort and the
// tile walkers (joined back into s before return)
void launch_density_map(const Ctx &c, const float *x, const float *y, cudaStream_t s, cudaStream_t aux,
                        int build_fixed) {
  DenArgs a = make_args(c, x, y);
  if (build_fixed) {   // dp_set_fixed: the map of the fixed cells alone (its own list: the caller
    a.fixed = c.d_fixed;   // requests a sort for the next evaluation)
    a.sel = 1;
    a.force_sort = 1;
    a.large = c.d_large_fix;
    a.n_large = c.n_large_fix;
  }
  const int ntiles = a.ntiles;
  const int nblk = (c.n_own + kCountCells - 1) / kCountCells;
  const size_t nb = (size_t)c.mx * c.my;
  const unsigned long long *src = nullptr;   // the map starts from this (or 0)
  if (c.n_regions > 0 && c.cur_region >= 0)   // the region's blockage map (exact int64)
    src = c.d_rho_block + (size_t)c.cur_region * nb;
  else if (c.has_fixed && !build_fixed)       // the precomputed fixed-charge map (exact int64)
    src = c.d_rho_fixed;
  // in a captured evaluation whose list may be kept, D1-D3 sit in a conditional (IF) node set by
  // k_map_init: no launches at all when the list is kept (DP_SORT_COND=0: the kernels return early)
  cudaStreamCaptureStatus cs = cudaStreamCaptureStatusNone;
  cudaStreamIsCapturing(s, &cs);
  const bool cond = nblk > 0 && !a.force_sort && !c.omit_sort && c.sort_cond && c.s_body &&
                    cs == cudaStreamCaptureStatusActive;
  cudaStream_t ss = s;   // stream of D1-D3
  // the graph variant without the sort kernels: the scatter follows a zeroing kernel
  // programmatically and starts its prologue early (DP_EARLY=0: memset and a plain dependency)
  const bool early = nblk > 0 && c.omit_sort && !a.force_sort && !cond && c.pdl && c.early_scatter;
  if (cond) {
    cudaGraph_t g = nullptr;
    const cudaGraphNode_t *deps = nullptr;
    size_t nd = 0;
    cudaGraphConditionalHandle h = 0;
    cudaGraphConditionalHandleCreate(&h, (cudaStreamGetCaptureInfo(s, &cs, nullptr, &g), g), 0, 0);
    k_map_init<<<2 * c.num_sms, 256, 0, s>>>(a, src, (long long)nb, h);
    cudaStreamGetCaptureInfo(s, &cs, nullptr, &g, &deps, &nd);
    cudaGraphNodeParams p = {};
    p.type = cudaGraphNodeTypeConditional;
    p.conditional.handle = h;
    p.conditional.type = cudaGraphCondTypeIf;
    p.conditional.size = 1;
    cudaGraphNode_t node = nullptr;
    cudaGraphAddNode(&node, g, deps, nd, &p);
    cudaStreamUpdateCaptureDependencies(s, &node, 1, cudaStreamSetCaptureDependencies);
    cudaStreamBeginCaptureToGraph(c.s_body, p.conditional.phGraph_out[0], nullptr, nullptr, 0,
                                  cudaStreamCaptureModeRelaxed);
    ss = c.s_body;
  } else if (src) {
    cudaMemcpyAsync(c.d_rho, src, sizeof(unsigned long long) * nb, cudaMemcpyDeviceToDevice, s);
  } else if (early) {
    k_zero_map<<<2 * c.num_sms, 256, 0, s>>>(c.d_rho, (long long)nb);
  } else {
    cudaMemsetAsync(c.d_rho, 0, sizeof(unsigned long long) * nb, s);
  }
  const bool side = aux && a.n_large > 0;
  if (side && !cond) {
    cudaEventRecord(c.ev_aux_a, s);
    cudaStreamWaitEvent(aux, c.ev_aux_a, 0);
    k_scatter_large<<<a.n_large, 256, 0, aux>>>(a);
    cudaEventRecord(c.ev_aux_b, aux);
  }
  if (nblk > 0 && c.omit_sort && !a.force_sort) {   // captured while the list is kept: no sort kernels (§5.5)
    if (c.sched == 2 || c.sched == 3) cudaEventRecord(c.ev_sched, s);
    a.early = early && !src ? 1 : 0;
    a.merge = c.scatter_merge;
    launch_chain(c.pdl, k_scatter_walk, c.walk_grid / c.scatter_merge, kTileThreads, scatter_smem_bytes(c.tile), s, a);
  } else if (nblk > 0) {
    const int cgrid = std::min(nblk, c.count_grid > 0 ? c.count_grid : nblk);
    if (a.fixed)
      launch_chain(c.pdl, k_count<true>, cgrid, kCountThreads, ntiles * 4, ss, a);
    // (k_count<true> counts only selected cells; k_place<true> records only selected cells)
    else
      launch_chain(c.pdl, k_count<false>, cgrid, kCountThreads, ntiles * 4, ss, a);
    if (c.sched == 3 && !cond) cudaEventRecord(c.ev_sched, ss);   // DP_SCHED=3: WA starts after the count
    launch_chain(c.pdl, k_scan, 1, 1024, 0, ss, a);
    if (a.fixed)
      launch_chain(c.pdl, k_place<true>, nblk, kCountThreads, place_smem_bytes(ntiles), ss, a);
    else
      launch_chain(c.pdl, k_place<false>, nblk, kCountThreads, place_smem_bytes(ntiles), ss, a);
    if (cond) {
      cudaGraph_t body = nullptr;
      cudaStreamEndCapture(c.s_body, &body);
      if (side) {   // the large cells beside the conditional sort and the walkers
        cudaEventRecord(c.ev_aux_a, s);
        cudaStreamWaitEvent(aux, c.ev_aux_a, 0);
        k_scatter_large<<<a.n_large, 256, 0, aux>>>(a);
        cudaEventRecord(c.ev_aux_b, aux);
      }
    }
    if (c.sched == 2 || (c.sched == 3 && cond)) cudaEventRecord(c.ev_sched, s);   // DP_SCHED=2: WA starts after the placement
    // after the IF node the walker is an ordinary dependent (programmatic edges join kernel nodes)
    a.merge = c.scatter_merge;
    launch_chain(c.pdl && !cond, k_scatter_walk, c.walk_grid / c.scatter_merge, kTileThreads, scatter_smem_bytes(c.tile), s, a);
  }
  if (side)
    cudaStreamWaitEvent(s, c.ev_aux_b, 0);
  else if (a.n_large > 0)
    k_scatter_large<<<a.n_large, 256, 0, s>>>(a);
}

void launch_density_gather(const Ctx &c, const float *x, const float *y, cudaStream_t s, cudaStream_t aux) {
  const DenArgs a = make_args(c, x, y);
  const bool side = aux && a.n_large > 0;
  if (side) {
    cudaEventRecord(c.ev_aux_a, s);
    cudaStreamWaitEvent(aux, c.ev_aux_a, 0);
    k_gather_large<<<a.n_large, 256, 0, aux>>>(a);
    cudaEventRecord(c.ev_aux_b, aux);
  }
  if (c.n_own > 0 && c.gather_rc)
    launch_chain(c.pdl, k_gather_walk_rc, c.walk_grid, kTileThreads, gather_rc_smem_bytes(c.tile), s, a);
  else if (c.n_own > 0)
    launch_chain(c.pdl, k_gather_walk, c.walk_grid, kTileThreads, walk_smem_bytes(c.tile), s, a);
  if (side)
    cudaStreamWaitEvent(s, c.ev_aux_b, 0);
  else if (a.n_large > 0)
    k_gather_large<<<a.n_large, 256, 0, s>>>(a);
}

}  // namespace dp
