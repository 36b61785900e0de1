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
//   D2 scan    one CTA: tile offsets, per-tile cursors, work segments (<= kSegCells cells)
//   D3 place   recompute tile ids, reserve ranges per CTA, write tile-local footprint
//              records in tile order
//   D4 scatter one CTA per segment accumulates its records into a (tile+2)^2 shared tile,
//              flushed with coalesced red.add into rho
//   D5 gather  one CTA per segment stages the (tile+2)^2 float2 field tile in shared memory
//              and writes each cell's force
// Large cells (footprint wider than 3 bins) take a CTA-per-cell path with global reds.
// The tile accumulators (int32, 2^-19) flush into an int64 global map (2^-24) with native
// red.global.add.u64: the density map is exact up to one rounding per contribution and
// independent of execution order (deterministic; bit-identical after an int64 all-reduce).
// Footprint geometry is computed in fp64 (B200 runs FP64 at half rate); records hold the
// footprint in fractions of the cell's first bin (|v| < 3) plus that bin's tile-local index.
#include "dp_internal.h"

namespace dp {

namespace {

struct DenArgs {
  const float *x, *y;   // global cell arrays
  const float *w, *h;   // own cells
  int cell_begin, n_own;
  double xl, yl, xh, yh, bx, by, sx, sy, ibx, iby;   // ibx = 1 / bx (no fp64 divisions on the hot path)
  int mx, my, tile, tile_log2, tiles_y, ntiles, stretch;
  int *tile_cnt, *tile_cursor, *tile_off;
  Segment *segs;
  int *nsegs;
  float4 *rec;
  int2 *rec_rc;   // (r as float bits, tile-local first bin i0 | j0 << 16)
  int *rec_cell;  // own cell index
  unsigned long long *rho;   // int64 fixed point, 2^-kRhoScaleLog2 units
  const float2 *xi;
  float2 *force;
  const int *large;
};

struct Foot {
  double lx, hx, ly, hy;
  float r;
  bool large, empty;
};

// Stretched, clipped footprint of a cell (readings A10, A11) from its loaded values.
__device__ __forceinline__ Foot footprint_v(const DenArgs &a, float xf, float yf, float wf, float hf) {
  Foot f;
  const double x = xf, y = yf, w = wf, h = hf;
  double ws = w, hs = h;
  float wsf = wf, hsf = hf;
  if (a.stretch) {
    ws = fmax(w, a.sx);
    hs = fmax(h, a.sy);
    wsf = fmaxf(wf, (float)a.sx);
    hsf = fmaxf(hf, (float)a.sy);
  }
  f.large = (w > 2.0 * a.bx) || (h > 2.0 * a.by);
  // charge ratio r = w h / (w' h') in fp32 (only its fp32 rounding is stored)
  f.r = (wsf * hsf > 0.f) ? __fdividef(wf * hf, wsf * hsf) : 0.f;
  const double cx = x + 0.5 * w, cy = y + 0.5 * h;
  f.lx = fmax(cx - 0.5 * ws, a.xl);
  f.hx = fmin(cx + 0.5 * ws, a.xh);
  f.ly = fmax(cy - 0.5 * hs, a.yl);
  f.hy = fmin(cy + 0.5 * hs, a.yh);
  f.empty = !(f.hx > f.lx && f.hy > f.ly && f.r > 0.f);
  return f;
}

__device__ __forceinline__ Foot footprint(const DenArgs &a, int i) {
  return footprint_v(a, __ldg(a.x + a.cell_begin + i), __ldg(a.y + a.cell_begin + i), __ldg(a.w + i), __ldg(a.h + i));
}

// Loads x, y, w, h of own cells [i0, i0 + 8) (i0 a multiple of 8) with 16-byte vector loads
// when the global index is aligned; out-of-range cells get w = h = 0 (empty).
struct Cells8 { float x[8], y[8], w[8], h[8]; };

__device__ __forceinline__ void load_cells8(const DenArgs &a, int i0, Cells8 &c) {
  const int g0 = a.cell_begin + i0;
  if (i0 + 8 <= a.n_own && (g0 & 3) == 0) {
#pragma unroll
    for (int v = 0; v < 2; v++) {
      const float4 X = __ldg(reinterpret_cast<const float4 *>(a.x + g0) + v);
      const float4 Y = __ldg(reinterpret_cast<const float4 *>(a.y + g0) + v);
      const float4 W = __ldg(reinterpret_cast<const float4 *>(a.w + i0) + v);
      const float4 H = __ldg(reinterpret_cast<const float4 *>(a.h + i0) + v);
      c.x[4 * v] = X.x; c.x[4 * v + 1] = X.y; c.x[4 * v + 2] = X.z; c.x[4 * v + 3] = X.w;
      c.y[4 * v] = Y.x; c.y[4 * v + 1] = Y.y; c.y[4 * v + 2] = Y.z; c.y[4 * v + 3] = Y.w;
      c.w[4 * v] = W.x; c.w[4 * v + 1] = W.y; c.w[4 * v + 2] = W.z; c.w[4 * v + 3] = W.w;
      c.h[4 * v] = H.x; c.h[4 * v + 1] = H.y; c.h[4 * v + 2] = H.z; c.h[4 * v + 3] = H.w;
    }
  } else {
#pragma unroll
    for (int k = 0; k < 8; k++) {
      const int i = i0 + k;
      const bool ok = i < a.n_own;
      c.x[k] = ok ? __ldg(a.x + a.cell_begin + i) : 0.f;
      c.y[k] = ok ? __ldg(a.y + a.cell_begin + i) : 0.f;
      c.w[k] = ok ? __ldg(a.w + i) : 0.f;
      c.h[k] = ok ? __ldg(a.h + i) : 0.f;
    }
  }
}

__device__ __forceinline__ int small_tile(const DenArgs &a, const Foot &f, int &ox, int &oy) {
  int bx0 = (int)floor((f.lx - a.xl) * a.ibx), by0 = (int)floor((f.ly - a.yl) * a.iby);
  bx0 = min(max(bx0, 0), a.mx - 1);
  by0 = min(max(by0, 0), a.my - 1);
  const int tx = bx0 >> a.tile_log2, ty = by0 >> a.tile_log2;
  ox = tx << a.tile_log2;
  oy = ty << a.tile_log2;
  return tx * a.tiles_y + ty;
}

// D1: 8 cells per thread, all loads issued up front
__global__ void __launch_bounds__(kCountThreads) k_count(DenArgs a) {
  extern __shared__ int s_hist[];
  for (int t = threadIdx.x; t < a.ntiles; t += kCountThreads) s_hist[t] = 0;
  __syncthreads();
  const int i0 = (blockIdx.x * kCountThreads + threadIdx.x) * 8;
  if (i0 < a.n_own) {
    Cells8 c;
    load_cells8(a, i0, c);
#pragma unroll
    for (int k = 0; k < 8; k++) {
      if (i0 + k >= a.n_own) break;
      const Foot f = footprint_v(a, c.x[k], c.y[k], c.w[k], c.h[k]);
      if (f.empty || f.large) continue;
      int ox, oy;
      atomicAdd(&s_hist[small_tile(a, f, ox, oy)], 1);
    }
  }
  __syncthreads();
  for (int t = threadIdx.x; t < a.ntiles; t += kCountThreads)
    if (s_hist[t]) atomicAdd(a.tile_cnt + t, s_hist[t]);
}

// D2 (single CTA of 1024 threads)
__global__ void __launch_bounds__(1024) k_scan(DenArgs a) {
  __shared__ int s_a[1024], s_b[1024];
  constexpr int T = 1024;
  const int per = (a.ntiles + T - 1) / T;
  const int t0 = threadIdx.x * per;
  int cnt_sum = 0, seg_sum = 0;
  for (int k = 0; k < per; k++) {
    const int t = t0 + k;
    if (t < a.ntiles) {
      const int c = a.tile_cnt[t];
      cnt_sum += c;
      seg_sum += (c + kSegCells - 1) / kSegCells;
    }
  }
  s_a[threadIdx.x] = cnt_sum;
  s_b[threadIdx.x] = seg_sum;
  __syncthreads();
  for (int off = 1; off < T; off <<= 1) {  // inclusive Hillis-Steele scan
    int va = 0, vb = 0;
    if ((int)threadIdx.x >= off) {
      va = s_a[threadIdx.x - off];
      vb = s_b[threadIdx.x - off];
    }
    __syncthreads();
    s_a[threadIdx.x] += va;
    s_b[threadIdx.x] += vb;
    __syncthreads();
  }
  int off_c = s_a[threadIdx.x] - cnt_sum, off_s = s_b[threadIdx.x] - seg_sum;
  for (int k = 0; k < per; k++) {
    const int t = t0 + k;
    if (t < a.ntiles) {
      const int c = a.tile_cnt[t];
      a.tile_off[t] = off_c;
      a.tile_cursor[t] = off_c;
      const int ns = (c + kSegCells - 1) / kSegCells;
      for (int q = 0; q < ns; q++) {
        Segment sg;
        sg.tile = t;
        sg.begin = off_c + q * kSegCells;
        sg.end = min(off_c + c, sg.begin + kSegCells);
        sg.pad = 0;
        a.segs[off_s + q] = sg;
      }
      off_c += c;
      off_s += ns;
      a.tile_cnt[t] = 0;  // ready for the next evaluation
    }
  }
  if (threadIdx.x == T - 1) {
    a.tile_off[a.ntiles] = s_a[T - 1];
    *a.nsegs = s_b[T - 1];
  }
}

// D3: same 8-cells-per-thread traversal as D1; records stay in registers while the CTA
// reserves its ranges in the tile cursors.
__global__ void __launch_bounds__(kCountThreads) k_place(DenArgs a) {
  extern __shared__ int s_hist[];
  for (int t = threadIdx.x; t < a.ntiles; t += kCountThreads) s_hist[t] = 0;
  __syncthreads();
  const int i0 = (blockIdx.x * kCountThreads + threadIdx.x) * 8;
  int tl[8], rk[8], ij[8];
  float4 rec[8];
  float rr[8];
#pragma unroll
  for (int k = 0; k < 8; k++) tl[k] = -1;
  if (i0 < a.n_own) {
    Cells8 c;
    load_cells8(a, i0, c);
#pragma unroll
    for (int k = 0; k < 8; k++) {
      const int i = i0 + k;
      if (i >= a.n_own) break;
      const Foot f = footprint_v(a, c.x[k], c.y[k], c.w[k], c.h[k]);
      if (f.large) continue;
      if (f.empty) {
        a.force[i] = make_float2(0.f, 0.f);
        continue;
      }
      int ox, oy;
      tl[k] = small_tile(a, f, ox, oy);
      rk[k] = atomicAdd(&s_hist[tl[k]], 1);
      // bin-local fractions (|v| < 3): fp32 keeps ~2e-7 bin absolute precision, which the force
      // gather needs where large opposite bin fields cancel (the 'initial' placement)
      const double ux0 = (f.lx - a.xl) * a.ibx, uy0 = (f.ly - a.yl) * a.iby;
      const int bi = min(max((int)floor(ux0), 0), a.mx - 1);
      const int bj = min(max((int)floor(uy0), 0), a.my - 1);
      rec[k] = make_float4((float)(ux0 - bi), (float)(uy0 - bj), (float)((f.hx - a.xl) * a.ibx - bi),
                           (float)((f.hy - a.yl) * a.iby - bj));
      rr[k] = f.r;
      ij[k] = (bi - ox) | ((bj - oy) << 16);
    }
  }
  __syncthreads();
  for (int t = threadIdx.x; t < a.ntiles; t += kCountThreads) {
    const int c = s_hist[t];
    if (c) s_hist[t] = atomicAdd(a.tile_cursor + t, c);
  }
  __syncthreads();
#pragma unroll
  for (int k = 0; k < 8; k++) {
    if (tl[k] < 0) continue;
    const int pos = s_hist[tl[k]] + rk[k];
    a.rec[pos] = rec[k];
    a.rec_rc[pos] = make_int2(__float_as_int(rr[k]), ij[k]);
    a.rec_cell[pos] = i0 + k;
  }
}

// D4
__global__ void __launch_bounds__(256) k_scatter_tiles(DenArgs a) {
  extern __shared__ int s_t[];   // int32 fixed point, 2^-kTileScaleLog2 units (native ATOMS.ADD)
  const int sg = blockIdx.x;
  if (sg >= *a.nsegs) return;
  const Segment seg = a.segs[sg];
  const int P = a.tile + kHalo;
  const int tx = seg.tile / a.tiles_y, ty = seg.tile % a.tiles_y;
  const int ox = tx * a.tile, oy = ty * a.tile;
  for (int k = threadIdx.x; k < P * P; k += blockDim.x) s_t[k] = 0;
  __syncthreads();
  const float scale = (float)(1 << kTileScaleLog2);
  for (int p = seg.begin + threadIdx.x; p < seg.end; p += blockDim.x) {
    const float4 q = a.rec[p];
    const int2 rc = a.rec_rc[p];
    const float r = __int_as_float(rc.x);
    const int i0 = rc.y & 0xffff, j0 = rc.y >> 16;
#pragma unroll
    for (int di = 0; di < 3; di++) {
      const int i = i0 + di;
      const float ovx = fminf(q.z, (float)(di + 1)) - fmaxf(q.x, (float)di);
      if (ovx <= 0.f || i >= P || ox + i >= a.mx) break;
#pragma unroll
      for (int dj = 0; dj < 3; dj++) {
        const int j = j0 + dj;
        const float ovy = fminf(q.w, (float)(dj + 1)) - fmaxf(q.y, (float)dj);
        if (ovy <= 0.f || j >= P || oy + j >= a.my) break;
        atomicAdd(&s_t[i * P + j], __float2int_rn(r * ovx * ovy * scale));
      }
    }
  }
  __syncthreads();
  for (int k = threadIdx.x; k < P * P; k += blockDim.x) {
    const int iv = s_t[k];
    const int gi = ox + k / P, gj = oy + k % P;
    if (iv != 0 && gi < a.mx && gj < a.my)
      asm volatile("red.global.add.u64 [%0], %1;" ::"l"(a.rho + (size_t)gi * a.my + gj),
                   "l"((unsigned long long)iv << (kRhoScaleLog2 - kTileScaleLog2))
                   : "memory");
  }
}

// D5
__global__ void __launch_bounds__(256) k_gather_tiles(DenArgs a) {
  extern __shared__ float2 s_xi[];
  const int sg = blockIdx.x;
  if (sg >= *a.nsegs) return;
  const Segment seg = a.segs[sg];
  const int P = a.tile + kHalo;
  const int tx = seg.tile / a.tiles_y, ty = seg.tile % a.tiles_y;
  const int ox = tx * a.tile, oy = ty * a.tile;
  for (int k = threadIdx.x; k < P * P; k += blockDim.x) {
    const int gi = ox + k / P, gj = oy + k % P;
    s_xi[k] = (gi < a.mx && gj < a.my) ? a.xi[(size_t)gi * a.my + gj] : make_float2(0.f, 0.f);
  }
  __syncthreads();
  const float area = (float)(a.bx * a.by);
  for (int p = seg.begin + threadIdx.x; p < seg.end; p += blockDim.x) {
    const float4 q = a.rec[p];
    const int2 rc = a.rec_rc[p];
    const float r = __int_as_float(rc.x);
    const int i0 = rc.y & 0xffff, j0 = rc.y >> 16;
    float fx = 0.f, fy = 0.f;
#pragma unroll
    for (int di = 0; di < 3; di++) {
      const int i = i0 + di;
      const float ovx = fminf(q.z, (float)(di + 1)) - fmaxf(q.x, (float)di);
      if (ovx <= 0.f || i >= P) break;
#pragma unroll
      for (int dj = 0; dj < 3; dj++) {
        const int j = j0 + dj;
        const float ovy = fminf(q.w, (float)(dj + 1)) - fmaxf(q.y, (float)dj);
        if (ovy <= 0.f || j >= P) break;
        const float2 e = s_xi[i * P + j];
        const float ov = ovx * ovy;
        fx += ov * e.x;
        fy += ov * e.y;
      }
    }
    // dD/dx = - r sum_b ov(i,b) xi^X_b  (reading A21), ov in length^2
    a.force[a.rec_cell[p]] = make_float2(-area * r * fx, -area * r * fy);
  }
}

// Large cells: one CTA per cell, fp64 overlaps, global reductions.
__global__ void __launch_bounds__(256) k_scatter_large(DenArgs a) {
  const int i = a.large[blockIdx.x];
  const Foot f = footprint(a, i);
  if (f.empty) return;
  const int i0 = max((int)floor((f.lx - a.xl) * a.ibx), 0), i1 = min((int)floor((f.hx - a.xl) * a.ibx), a.mx - 1);
  const int j0 = max((int)floor((f.ly - a.yl) * a.iby), 0), j1 = min((int)floor((f.hy - a.yl) * a.iby), a.my - 1);
  const int nj = j1 - j0 + 1, n = (i1 - i0 + 1) * nj;
  for (int k = threadIdx.x; k < n; k += blockDim.x) {
    const int bi = i0 + k / nj, bj = j0 + k % nj;
    const double ox = fmin(f.hx, a.xl + (bi + 1) * a.bx) - fmax(f.lx, a.xl + bi * a.bx);
    const double oy = fmin(f.hy, a.yl + (bj + 1) * a.by) - fmax(f.ly, a.yl + bj * a.by);
    if (ox <= 0.0 || oy <= 0.0) continue;
    const unsigned long long v =
        (unsigned long long)__double2ll_rn((double)f.r * ox * oy * a.ibx * a.iby * (double)(1ll << kRhoScaleLog2));
    asm volatile("red.global.add.u64 [%0], %1;" ::"l"(a.rho + (size_t)bi * a.my + bj), "l"(v) : "memory");
  }
}

__global__ void __launch_bounds__(256) k_gather_large(DenArgs a) {
  const int i = a.large[blockIdx.x];
  const Foot f = footprint(a, i);
  __shared__ double s_x[8], s_y[8];
  double fx = 0.0, fy = 0.0;
  if (!f.empty) {
    const int i0 = max((int)floor((f.lx - a.xl) * a.ibx), 0), i1 = min((int)floor((f.hx - a.xl) * a.ibx), a.mx - 1);
    const int j0 = max((int)floor((f.ly - a.yl) * a.iby), 0), j1 = min((int)floor((f.hy - a.yl) * a.iby), a.my - 1);
    const int nj = j1 - j0 + 1, n = (i1 - i0 + 1) * nj;
    for (int k = threadIdx.x; k < n; k += blockDim.x) {
      const int bi = i0 + k / nj, bj = j0 + k % nj;
      const double ox = fmin(f.hx, a.xl + (bi + 1) * a.bx) - fmax(f.lx, a.xl + bi * a.bx);
      const double oy = fmin(f.hy, a.yl + (bj + 1) * a.by) - fmax(f.ly, a.yl + bj * a.by);
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
    a.force[i] = make_float2((float)(-(double)f.r * tx), (float)(-(double)f.r * ty));
  }
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
  a.mx = c.mx; a.my = c.my; a.tile = c.tile; a.tiles_y = c.tiles_y;
  a.tile_log2 = 0;
  while ((1 << a.tile_log2) < c.tile) a.tile_log2++;
  a.ntiles = c.tiles_x * c.tiles_y;
  a.stretch = c.stretch;
  a.tile_cnt = c.d_tile_cnt;
  a.tile_cursor = c.d_tile_cursor;
  a.tile_off = c.d_tile_off;
  a.segs = c.d_segs;
  a.nsegs = c.d_nsegs;
  a.rec = c.d_rec;
  a.rec_rc = c.d_rec_rc;
  a.rec_cell = c.d_rec_cell;
  a.rho = c.d_rho;
  a.xi = c.d_xi;
  a.force = c.d_force;
  a.large = c.d_large;
  return a;
}

}  // namespace

cudaError_t density_configure(int ntiles, int tile) {
  const int P = tile + kHalo;
  cudaError_t e = cudaFuncSetAttribute(k_count, cudaFuncAttributeMaxDynamicSharedMemorySize, ntiles * 4);
  if (e != cudaSuccess) return e;
  e = cudaFuncSetAttribute(k_place, cudaFuncAttributeMaxDynamicSharedMemorySize, ntiles * 4);
  if (e != cudaSuccess) return e;
  e = cudaFuncSetAttribute(k_scatter_tiles, cudaFuncAttributeMaxDynamicSharedMemorySize, P * P * 4);
  if (e != cudaSuccess) return e;
  return cudaFuncSetAttribute(k_gather_tiles, cudaFuncAttributeMaxDynamicSharedMemorySize, P * P * 8);
}

int density_launches(const Ctx &c) { return 6 + (c.n_large > 0 ? 1 : 0); }

void launch_density_map(const Ctx &c, const float *x, const float *y, cudaStream_t s) {
  const DenArgs a = make_args(c, x, y);
  const int P = c.tile + kHalo;
  const int ntiles = a.ntiles;
  const int nblk = (c.n_own + kCountThreads * 8 - 1) / (kCountThreads * 8);
  cudaMemsetAsync(c.d_rho, 0, sizeof(unsigned long long) * (size_t)c.mx * c.my, s);
  if (nblk > 0) {
    k_count<<<nblk, kCountThreads, ntiles * 4, s>>>(a);
    k_scan<<<1, 1024, 0, s>>>(a);
    k_place<<<nblk, kCountThreads, ntiles * 4, s>>>(a);
    k_scatter_tiles<<<c.max_segs, 256, P * P * 4, s>>>(a);
  }
  if (c.n_large > 0) k_scatter_large<<<c.n_large, 256, 0, s>>>(a);
}

void launch_density_gather(const Ctx &c, const float *x, const float *y, cudaStream_t s) {
  const DenArgs a = make_args(c, x, y);
  const int P = c.tile + kHalo;
  if (c.n_own > 0) k_gather_tiles<<<c.max_segs, 256, P * P * 8, s>>>(a);
  if (c.n_large > 0) k_gather_large<<<c.n_large, 256, 0, s>>>(a);
}

}  // namespace dp
