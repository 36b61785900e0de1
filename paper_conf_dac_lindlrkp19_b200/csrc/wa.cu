// wa.cu — weighted-average wirelength, its gradient and HPWL on sm_100a.
//
// Method: WA of eq (3) with the overflow-safe shift of P:159 and Table I
// notation; gradient of eq (6); merged forward+backward per net as in
// Alg 2 so no per-net intermediate touches global memory; HPWL.
//
// B200 design, differences from the paper's Alg 2:
//  * nets are locality-sorted into chunks at dp_create; a CTA owns one chunk and keeps the
//    positions and gradients of the chunk's cell window in shared memory, so the pin->cell
//    gradient reduction is a shared-memory atomic instead of a global one (random L2 reds
//    run at ~0.2 Gop/ms on B200 — tools/microbench), flushed once with coalesced red.v4;
//  * nets are processed by groups of G = 1..32 lanes (by degree), each lane holding up to 8
//    pins in registers: a^+- are computed once and kept (Alg 2 recomputes them);
//  * x and y are fused in one pass (the paper uses two streams);
//  * the shift is done in net-local coordinates with an exact TwoSum of (x_cell + dx), so
//    fp32 keeps full relative precision even at |x| ~ 1e6 (reading A2);
//  * HPWL uses the exact per-net extremes and a 2^-149 fixed-point int64 limb sum, which
//    makes the total correctly rounded and order independent (reading A7).
#include "dp_internal.h"

namespace dp {

namespace {

constexpr float kLog2e = 1.4426950408889634f;

struct WaArgs {
  const Chunk *chunks;
  const WarpGroup *wgs;
  const int32_t *net_deg;
  const float *net_w;
  const int32_t *pin_cell;
  const float *pin_dx, *pin_dy;
  const float *x, *y;
  float2 *g2;
  float gamma, inv_gamma, k2;   // k2 = log2(e) / gamma
  double *part;                 // WA partial per CTA
  unsigned long long *limbs;    // HPWL limbs
  int has_w;
  // big nets
  const int32_t *big_start, *big_flags, *big_cell;
  const float *big_w, *big_dx, *big_dy;
  int part_offset;
};

// Exact sum s + e = a + b (Knuth TwoSum, fp32, no contraction).
__device__ __forceinline__ void two_sum(float a, float b, float &s, float &e) {
  s = __fadd_rn(a, b);
  float bb = __fsub_rn(s, a);
  e = __fadd_rn(__fsub_rn(a, __fsub_rn(s, bb)), __fsub_rn(b, bb));
}

// (h1,l1) > (h2,l2) for TwoSum-normalised pairs: the fp32 rounding of the value is
// monotone, so comparing hi then lo compares the exact values.
__device__ __forceinline__ bool pair_gt(float h1, float l1, float h2, float l2) {
  return h1 > h2 || (h1 == h2 && l1 > l2);
}

__device__ __forceinline__ float ex2(float v) {
  float r;
  asm("ex2.approx.ftz.f32 %0, %1;" : "=f"(r) : "f"(v));
  return r;
}

__device__ __forceinline__ void red_v2(float2 *p, float a, float b) {
  asm volatile("red.global.add.v2.f32 [%0], {%1, %2};" ::"l"(p), "f"(a), "f"(b) : "memory");
}

__device__ __forceinline__ void red_v4(float4 *p, float a, float b, float c, float d) {
  asm volatile("red.global.add.v4.f32 [%0], {%1, %2, %3, %4};" ::"l"(p), "f"(a), "f"(b), "f"(c),
               "f"(d)
               : "memory");
}

// Add h (>= 0, a multiple of 2^-149 below 2^131) to 10 int64 limbs of 32-bit digits with
// weight 2^(32 j - 149) (reading A7).
__device__ __forceinline__ void limbs_add(unsigned long long (&L)[kHpwlLimbs + 1], double h) {
  if (!(h > 0.0)) return;
  unsigned long long bits = (unsigned long long)__double_as_longlong(h);
  int ex = (int)((bits >> 52) & 0x7ff);
  unsigned long long m = bits & ((1ull << 52) - 1);
  int e;
  if (ex == 0) {
    e = -1074;
  } else {
    m |= 1ull << 52;
    e = ex - 1075;
  }
  int s = e + 149;
  if (s < 0) {
    m >>= -s;
    s = 0;
  }
  int q = s >> 5, r = s & 31;
  unsigned __int128 v = (unsigned __int128)m << r;
  unsigned long long d0 = (unsigned long long)(v & 0xffffffffu);
  unsigned long long d1 = (unsigned long long)((v >> 32) & 0xffffffffu);
  unsigned long long d2 = (unsigned long long)(v >> 64);
#pragma unroll
  for (int k = 0; k <= kHpwlLimbs; k++) {
    unsigned long long add = (k == q ? d0 : 0ull) + (k == q + 1 ? d1 : 0ull) + (k == q + 2 ? d2 : 0ull);
    L[k] += add;
  }
}

template <int THREADS>
__device__ void block_flush_scalars(double wl, unsigned long long (&L)[kHpwlLimbs + 1],
                                    bool hpwl, double *part_slot, unsigned long long *limbs) {
  __shared__ double s_wl[THREADS / 32];
  __shared__ unsigned long long s_l[THREADS / 32][kHpwlLimbs + 1];
  const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
#pragma unroll
  for (int o = 16; o > 0; o >>= 1) wl += __shfl_xor_sync(0xffffffffu, wl, o);
  if (hpwl) {
#pragma unroll
    for (int k = 0; k <= kHpwlLimbs; k++) {
#pragma unroll
      for (int o = 16; o > 0; o >>= 1) L[k] += __shfl_xor_sync(0xffffffffu, L[k], o);
    }
  }
  if (lane == 0) {
    s_wl[warp] = wl;
    if (hpwl)
#pragma unroll
      for (int k = 0; k <= kHpwlLimbs; k++) s_l[warp][k] = L[k];
  }
  __syncthreads();
  if (threadIdx.x == 0) {
    double t = 0.0;
    for (int w = 0; w < THREADS / 32; w++) t += s_wl[w];
    if (part_slot) *part_slot = t;
  }
  if (hpwl && threadIdx.x <= kHpwlLimbs) {
    unsigned long long t = 0;
    for (int w = 0; w < THREADS / 32; w++) t += s_l[w][threadIdx.x];
    if (t) atomicAdd(limbs + threadIdx.x, t);
  }
}

// Fast2Sum (3 flops): exact when |a| >= |b| (cell coordinate vs pin offset, the usual case);
// otherwise still accurate to ~ulp of the sum, which is all the WA value/gradient needs.
__device__ __forceinline__ void fast_sum(float a, float b, float &s, float &e) {
  s = __fadd_rn(a, b);
  e = __fadd_rn(__fsub_rn(a, s), b);
}

// Per-lane running extremes of one axis as (hi, lo) pairs.
struct Axis { float Ph, Pl, Mh, Ml; };

template <bool EXACT>
__device__ __forceinline__ void ext_update(Axis &A, float h, float l) {
  if (EXACT) {
    if (pair_gt(h, l, A.Ph, A.Pl)) { A.Ph = h; A.Pl = l; }
    if (pair_gt(A.Mh, A.Ml, h, l)) { A.Mh = h; A.Ml = l; }
  } else {  // the shift only needs a pin at (or within an ulp of) the extreme
    if (h > A.Ph) { A.Ph = h; A.Pl = l; }
    if (h < A.Mh) { A.Mh = h; A.Ml = l; }
  }
}

template <bool EXACT>
__device__ __forceinline__ void ext_shfl(Axis &A, int o) {
  const float ph = __shfl_xor_sync(0xffffffffu, A.Ph, o), pl = __shfl_xor_sync(0xffffffffu, A.Pl, o);
  const float mh = __shfl_xor_sync(0xffffffffu, A.Mh, o), ml = __shfl_xor_sync(0xffffffffu, A.Ml, o);
  if (EXACT) {
    if (pair_gt(ph, pl, A.Ph, A.Pl)) { A.Ph = ph; A.Pl = pl; }
    if (pair_gt(A.Mh, A.Ml, mh, ml)) { A.Mh = mh; A.Ml = ml; }
  } else {
    if (ph > A.Ph || (ph == A.Ph && pl > A.Pl)) { A.Ph = ph; A.Pl = pl; }
    if (mh < A.Mh || (mh == A.Mh && ml < A.Ml)) { A.Mh = mh; A.Ml = ml; }
  }
}

struct GroupCtx {
  const Chunk &ch;
  const float2 *s_pos;
  float *s_g;
  int lane;
  unsigned lt_mask;
};

// One warp group: 32/G nets, G lanes per net, S pin slots per lane.
template <int MODE, int S>
__device__ __forceinline__ void wa_group(const WaArgs &a, const WarpGroup &wg, const GroupCtx &gc, double &wl_acc,
                                         unsigned long long (&L)[kHpwlLimbs + 1]) {
  constexpr bool kGrad = MODE != 2;
  constexpr bool kHpwl = MODE != 0;
  const int glog = wg.g_log2, G = 1 << glog;
  const int gi = gc.lane >> glog, j = gc.lane & (G - 1);
  int d = 0, counted = 0;
  float we = 1.f;
  if (gi < wg.nnets) {
    const int raw = __ldg(a.net_deg + wg.net_base + gi);
    d = raw & 0x7fffffff;
    counted = (raw >> 31) & 1;
    if (a.has_w) we = __ldg(a.net_w + wg.net_base + gi);
  }
  // ---- phase A: pin records of all slots (slot-major compressed layout, coalesced) ----
  int cell[S];
  float dxs[S], dys[S];
  unsigned vm = 0;
  int base = wg.pin_base;
#pragma unroll
  for (int s = 0; s < S; s++) {
    const bool valid = s * G + j < d;
    const unsigned m = __ballot_sync(0xffffffffu, valid);
    cell[s] = 0;
    dxs[s] = dys[s] = 0.f;
    if (valid) {
      const int p = base + __popc(m & gc.lt_mask);
      cell[s] = __ldg(a.pin_cell + p);
      dxs[s] = __ldg(a.pin_dx + p);
      dys[s] = __ldg(a.pin_dy + p);
      vm |= 1u << s;
    }
    base += __popc(m);
  }
  // ---- phase B: pin positions px = x_cell + dx as (hi, lo) pairs ----
  float hx[S], lx[S], hy[S], ly[S];
  Axis X{-INFINITY, 0.f, INFINITY, 0.f}, Y{-INFINITY, 0.f, INFINITY, 0.f};
#pragma unroll
  for (int s = 0; s < S; s++) {
    hx[s] = lx[s] = hy[s] = ly[s] = 0.f;
    if (vm & (1u << s)) {
      const int c = cell[s] & 0x7fffffff;
      const int wi = c - gc.ch.win_lo;
      float xc, yc;
      if ((unsigned)wi < (unsigned)gc.ch.win_n) {
        const float2 q = gc.s_pos[wi];
        xc = q.x;
        yc = q.y;
      } else {
        xc = __ldg(a.x + c);
        yc = __ldg(a.y + c);
      }
      if (kHpwl) {
        two_sum(xc, dxs[s], hx[s], lx[s]);
        two_sum(yc, dys[s], hy[s], ly[s]);
      } else {
        fast_sum(xc, dxs[s], hx[s], lx[s]);
        fast_sum(yc, dys[s], hy[s], ly[s]);
      }
      ext_update<kHpwl>(X, hx[s], lx[s]);
      ext_update<kHpwl>(Y, hy[s], ly[s]);
    }
  }
  for (int o = 1; o < G; o <<= 1) {
    ext_shfl<kHpwl>(X, o);
    ext_shfl<kHpwl>(Y, o);
  }
  const bool leader = (j == 0) && d >= 2;
  if (kHpwl && leader && counted) {
    // px = fl64(x + dx) as the oracle forms it: (double)hi + (double)lo rounds the exact
    // real x + dx once (reading A7)
    const double xp = __dadd_rn((double)X.Ph, (double)X.Pl), xm = __dadd_rn((double)X.Mh, (double)X.Ml);
    const double yp = __dadd_rn((double)Y.Ph, (double)Y.Pl), ym = __dadd_rn((double)Y.Mh, (double)Y.Ml);
    limbs_add(L, __dadd_rn(__dsub_rn(xp, xm), __dsub_rn(yp, ym)));
  }
  if (!kGrad) return;
  // ---- shifted exponentials a^+- and sums b^+-, c~^+- (Table I) ----
  float lxp[S], lxm[S], lyp[S], lym[S], axp[S], axm[S], ayp[S], aym[S];
  float bxp = 0.f, bxm = 0.f, cxp = 0.f, cxm = 0.f, byp = 0.f, bym = 0.f, cyp = 0.f, cym = 0.f;
#pragma unroll
  for (int s = 0; s < S; s++) {
    lxp[s] = lxm[s] = lyp[s] = lym[s] = 0.f;
    axp[s] = axm[s] = ayp[s] = aym[s] = 0.f;
    if (vm & (1u << s)) {
      lxp[s] = __fadd_rn(__fsub_rn(hx[s], X.Ph), __fsub_rn(lx[s], X.Pl));   // <= 0 (net-local)
      lxm[s] = __fadd_rn(__fsub_rn(hx[s], X.Mh), __fsub_rn(lx[s], X.Ml));   // >= 0
      lyp[s] = __fadd_rn(__fsub_rn(hy[s], Y.Ph), __fsub_rn(ly[s], Y.Pl));
      lym[s] = __fadd_rn(__fsub_rn(hy[s], Y.Mh), __fsub_rn(ly[s], Y.Ml));
      axp[s] = ex2(lxp[s] * a.k2);
      axm[s] = ex2(-lxm[s] * a.k2);
      ayp[s] = ex2(lyp[s] * a.k2);
      aym[s] = ex2(-lym[s] * a.k2);
      bxp += axp[s]; cxp = fmaf(lxp[s], axp[s], cxp);
      bxm += axm[s]; cxm = fmaf(lxm[s], axm[s], cxm);
      byp += ayp[s]; cyp = fmaf(lyp[s], ayp[s], cyp);
      bym += aym[s]; cym = fmaf(lym[s], aym[s], cym);
    }
  }
  for (int o = 1; o < G; o <<= 1) {
    bxp += __shfl_xor_sync(0xffffffffu, bxp, o);
    cxp += __shfl_xor_sync(0xffffffffu, cxp, o);
    bxm += __shfl_xor_sync(0xffffffffu, bxm, o);
    cxm += __shfl_xor_sync(0xffffffffu, cxm, o);
    byp += __shfl_xor_sync(0xffffffffu, byp, o);
    cyp += __shfl_xor_sync(0xffffffffu, cyp, o);
    bym += __shfl_xor_sync(0xffffffffu, bym, o);
    cym += __shfl_xor_sync(0xffffffffu, cym, o);
  }
  if (d < 2) return;  // lanes without a net; degree-1 nets are dropped at create
  const float ibxp = __frcp_rn(bxp), ibxm = __frcp_rn(bxm), ibyp = __frcp_rn(byp), ibym = __frcp_rn(bym);
  const float mxp = cxp * ibxp, mxm = cxm * ibxm, myp = cyp * ibyp, mym = cym * ibym;
  if (leader && counted) {
    // WL_e = c+/b+ - c-/b- = (x+ - x-) + c~+/b+ - c~-/b-   (eq 3 in net-local coordinates)
    const float spanx = __fadd_rn(__fsub_rn(X.Ph, X.Mh), __fsub_rn(X.Pl, X.Ml));
    const float spany = __fadd_rn(__fsub_rn(Y.Ph, Y.Mh), __fsub_rn(Y.Pl, Y.Ml));
    wl_acc += (double)(we * ((spanx + mxp - mxm) + (spany + myp - mym)));
  }
  // eq (6): dWL/dx_i = a+_i/b+ (1 + (l+_i - m+)/g) - a-_i/b- (1 - (l-_i - m-)/g)
  //                  = a+_i (P+ + l+_i Q+) - a-_i (P- - l-_i Q-)
  const float ig = a.inv_gamma;
  const float qxp = we * ibxp * ig, pxp = we * ibxp * (1.f - mxp * ig);
  const float qxm = we * ibxm * ig, pxm = we * ibxm * (1.f + mxm * ig);
  const float qyp = we * ibyp * ig, pyp = we * ibyp * (1.f - myp * ig);
  const float qym = we * ibym * ig, pym = we * ibym * (1.f + mym * ig);
#pragma unroll
  for (int s = 0; s < S; s++) {
    if ((vm & (1u << s)) && cell[s] >= 0) {  // cell < 0: foreign pin (another rank owns it)
      const float gx = axp[s] * fmaf(lxp[s], qxp, pxp) - axm[s] * fmaf(-lxm[s], qxm, pxm);
      const float gy = ayp[s] * fmaf(lyp[s], qyp, pyp) - aym[s] * fmaf(-lym[s], qym, pym);
      const int wi = cell[s] - gc.ch.win_lo;
      if ((unsigned)wi < (unsigned)gc.ch.win_n) {
        atomicAdd(gc.s_g + 2 * wi, gx);
        atomicAdd(gc.s_g + 2 * wi + 1, gy);
      } else {
        red_v2(a.g2 + cell[s], gx, gy);
      }
    }
  }
}

// MODE 0: WA + gradient; 1: WA + gradient + HPWL; 2: HPWL only.
template <int MODE>
__global__ void __launch_bounds__(kWaThreads, 3) k_wa_chunks(WaArgs a) {
  constexpr bool kGrad = MODE != 2;
  constexpr bool kHpwl = MODE != 0;
  __shared__ float2 s_pos[kWaWindow];
  __shared__ float s_g[kGrad ? 2 * kWaWindow : 1];
  __shared__ int s_next;

  const Chunk ch = a.chunks[blockIdx.x];
  const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
  for (int i = tid; i < ch.win_n; i += kWaThreads) {
    s_pos[i] = make_float2(__ldg(a.x + ch.win_lo + i), __ldg(a.y + ch.win_lo + i));
    if (kGrad) {
      s_g[2 * i] = 0.f;
      s_g[2 * i + 1] = 0.f;
    }
  }
  if (tid == 0) s_next = ch.wg_begin + kWaThreads / 32;
  __syncthreads();

  double wl_acc = 0.0;
  unsigned long long L[kHpwlLimbs + 1];
#pragma unroll
  for (int k = 0; k <= kHpwlLimbs; k++) L[k] = 0ull;
  const GroupCtx gc{ch, s_pos, s_g, lane, (1u << lane) - 1u};

  // warp groups are handed out dynamically inside the CTA (self-balancing)
  int wgi = ch.wg_begin + warp;
  while (wgi < ch.wg_end) {
    const WarpGroup wg = a.wgs[wgi];
    switch (wg.slots) {
      case 1: wa_group<MODE, 1>(a, wg, gc, wl_acc, L); break;
      case 2: wa_group<MODE, 2>(a, wg, gc, wl_acc, L); break;
      case 3: wa_group<MODE, 3>(a, wg, gc, wl_acc, L); break;
      default: wa_group<MODE, 4>(a, wg, gc, wl_acc, L); break;
    }
    int nx = 0;
    if (lane == 0) nx = atomicAdd(&s_next, 1);
    wgi = __shfl_sync(0xffffffffu, nx, 0);
  }
  __syncthreads();
  if (kGrad) {
    // flush the window: cells [win_lo, win_lo + win_n) as 16-byte vector reductions
    float4 *g4 = reinterpret_cast<float4 *>(a.g2);
    const int lo = ch.win_lo, n = ch.win_n;
    const int head = lo & 1;  // an odd first cell is flushed alone
    if (head && tid == 0 && n > 0) {
      const float gx = s_g[0], gy = s_g[1];
      if (gx != 0.f || gy != 0.f) red_v2(a.g2 + lo, gx, gy);
    }
    const int npair = (n - head) >> 1;
    for (int i = tid; i < npair; i += kWaThreads) {
      const int w = head + 2 * i;
      const float v0 = s_g[2 * w], v1 = s_g[2 * w + 1], v2 = s_g[2 * w + 2], v3 = s_g[2 * w + 3];
      if (v0 != 0.f || v1 != 0.f || v2 != 0.f || v3 != 0.f) red_v4(g4 + ((lo + w) >> 1), v0, v1, v2, v3);
    }
    if (((n - head) & 1) && tid == 0) {
      const int w = n - 1;
      const float gx = s_g[2 * w], gy = s_g[2 * w + 1];
      if (gx != 0.f || gy != 0.f) red_v2(a.g2 + lo + w, gx, gy);
    }
  }
  block_flush_scalars<kWaThreads>(wl_acc, L, kHpwl, kGrad ? a.part + blockIdx.x : nullptr, a.limbs);
}

// ---------------------------------------------------------------------------------------
// Nets with degree > kWaMaxDeg: one CTA per net, three passes over the pins (Alg 2's
// structure, a^+- recomputed in the gradient pass because they do not fit in registers).
// ---------------------------------------------------------------------------------------
struct Ext { float Xh, Xl, xh, xl, Yh, Yl, yh, yl; };

__device__ __forceinline__ void ext_merge(Ext &e, const Ext &o) {
  if (pair_gt(o.Xh, o.Xl, e.Xh, e.Xl)) { e.Xh = o.Xh; e.Xl = o.Xl; }
  if (pair_gt(e.xh, e.xl, o.xh, o.xl)) { e.xh = o.xh; e.xl = o.xl; }
  if (pair_gt(o.Yh, o.Yl, e.Yh, e.Yl)) { e.Yh = o.Yh; e.Yl = o.Yl; }
  if (pair_gt(e.yh, e.yl, o.yh, o.yl)) { e.yh = o.yh; e.yl = o.yl; }
}

template <int MODE>
__global__ void __launch_bounds__(kBigThreads) k_wa_big(WaArgs a) {
  constexpr bool kGrad = MODE != 2;
  constexpr bool kHpwl = MODE != 0;
  const int net = blockIdx.x, tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
  constexpr int NW = kBigThreads / 32;
  const int s0 = a.big_start[net], d = a.big_start[net + 1] - s0;
  const int counted = a.big_flags[net];
  const float we = a.has_w ? a.big_w[net] : 1.f;
  __shared__ Ext s_ext[NW];
  __shared__ float s_sum[NW][8];

  Ext e{-INFINITY, 0.f, INFINITY, 0.f, -INFINITY, 0.f, INFINITY, 0.f};
  for (int p = tid; p < d; p += kBigThreads) {
    const int c = a.big_cell[s0 + p] & 0x7fffffff;
    float h, l, H, Lo;
    two_sum(__ldg(a.x + c), a.big_dx[s0 + p], h, l);
    two_sum(__ldg(a.y + c), a.big_dy[s0 + p], H, Lo);
    Ext o{h, l, h, l, H, Lo, H, Lo};
    ext_merge(e, o);
  }
#pragma unroll
  for (int o = 16; o > 0; o >>= 1) {
    Ext t;
    t.Xh = __shfl_xor_sync(0xffffffffu, e.Xh, o); t.Xl = __shfl_xor_sync(0xffffffffu, e.Xl, o);
    t.xh = __shfl_xor_sync(0xffffffffu, e.xh, o); t.xl = __shfl_xor_sync(0xffffffffu, e.xl, o);
    t.Yh = __shfl_xor_sync(0xffffffffu, e.Yh, o); t.Yl = __shfl_xor_sync(0xffffffffu, e.Yl, o);
    t.yh = __shfl_xor_sync(0xffffffffu, e.yh, o); t.yl = __shfl_xor_sync(0xffffffffu, e.yl, o);
    ext_merge(e, t);
  }
  if (lane == 0) s_ext[warp] = e;
  __syncthreads();
  e = s_ext[0];
  for (int w = 1; w < NW; w++) ext_merge(e, s_ext[w]);

  unsigned long long L[kHpwlLimbs + 1];
#pragma unroll
  for (int k = 0; k <= kHpwlLimbs; k++) L[k] = 0ull;
  if (kHpwl && tid == 0 && counted) {
    const double xp = __dadd_rn((double)e.Xh, (double)e.Xl), xm = __dadd_rn((double)e.xh, (double)e.xl);
    const double yp = __dadd_rn((double)e.Yh, (double)e.Yl), ym = __dadd_rn((double)e.yh, (double)e.yl);
    limbs_add(L, __dadd_rn(__dsub_rn(xp, xm), __dsub_rn(yp, ym)));
  }
  double wl_acc = 0.0;
  if (kGrad) {
    float sm[8] = {0, 0, 0, 0, 0, 0, 0, 0};  // bxp cxp bxm cxm byp cyp bym cym
    for (int p = tid; p < d; p += kBigThreads) {
      const int c = a.big_cell[s0 + p] & 0x7fffffff;
      float hx, lx, hy, ly;
      two_sum(__ldg(a.x + c), a.big_dx[s0 + p], hx, lx);
      two_sum(__ldg(a.y + c), a.big_dy[s0 + p], hy, ly);
      const float lxp = __fadd_rn(__fsub_rn(hx, e.Xh), __fsub_rn(lx, e.Xl));
      const float lxm = __fadd_rn(__fsub_rn(hx, e.xh), __fsub_rn(lx, e.xl));
      const float lyp = __fadd_rn(__fsub_rn(hy, e.Yh), __fsub_rn(ly, e.Yl));
      const float lym = __fadd_rn(__fsub_rn(hy, e.yh), __fsub_rn(ly, e.yl));
      const float axp = ex2(lxp * a.k2), axm = ex2(-lxm * a.k2);
      const float ayp = ex2(lyp * a.k2), aym = ex2(-lym * a.k2);
      sm[0] += axp; sm[1] += lxp * axp; sm[2] += axm; sm[3] += lxm * axm;
      sm[4] += ayp; sm[5] += lyp * ayp; sm[6] += aym; sm[7] += lym * aym;
    }
#pragma unroll
    for (int k = 0; k < 8; k++) {
#pragma unroll
      for (int o = 16; o > 0; o >>= 1) sm[k] += __shfl_xor_sync(0xffffffffu, sm[k], o);
    }
    __syncthreads();
    if (lane == 0)
#pragma unroll
      for (int k = 0; k < 8; k++) s_sum[warp][k] = sm[k];
    __syncthreads();
#pragma unroll
    for (int k = 0; k < 8; k++) {
      float t = 0.f;
      for (int w = 0; w < NW; w++) t += s_sum[w][k];
      sm[k] = t;
    }
    const float ibxp = 1.f / sm[0], ibxm = 1.f / sm[2], ibyp = 1.f / sm[4], ibym = 1.f / sm[6];
    const float mxp = sm[1] * ibxp, mxm = sm[3] * ibxm, myp = sm[5] * ibyp, mym = sm[7] * ibym;
    if (tid == 0 && counted) {
      const float spanx = __fadd_rn(__fsub_rn(e.Xh, e.xh), __fsub_rn(e.Xl, e.xl));
      const float spany = __fadd_rn(__fsub_rn(e.Yh, e.yh), __fsub_rn(e.Yl, e.yl));
      wl_acc = (double)(we * ((spanx + mxp - mxm) + (spany + myp - mym)));
    }
    for (int p = tid; p < d; p += kBigThreads) {
      const int raw = a.big_cell[s0 + p];
      if (raw < 0) continue;
      float hx, lx, hy, ly;
      two_sum(__ldg(a.x + raw), a.big_dx[s0 + p], hx, lx);
      two_sum(__ldg(a.y + raw), a.big_dy[s0 + p], hy, ly);
      const float lxp = __fadd_rn(__fsub_rn(hx, e.Xh), __fsub_rn(lx, e.Xl));
      const float lxm = __fadd_rn(__fsub_rn(hx, e.xh), __fsub_rn(lx, e.xl));
      const float lyp = __fadd_rn(__fsub_rn(hy, e.Yh), __fsub_rn(ly, e.Yl));
      const float lym = __fadd_rn(__fsub_rn(hy, e.yh), __fsub_rn(ly, e.yl));
      const float axp = ex2(lxp * a.k2), axm = ex2(-lxm * a.k2);
      const float ayp = ex2(lyp * a.k2), aym = ex2(-lym * a.k2);
      const float gx = we * (axp * ibxp * (1.f + (lxp - mxp) * a.inv_gamma) -
                             axm * ibxm * (1.f - (lxm - mxm) * a.inv_gamma));
      const float gy = we * (ayp * ibyp * (1.f + (lyp - myp) * a.inv_gamma) -
                             aym * ibym * (1.f - (lym - mym) * a.inv_gamma));
      red_v2(a.g2 + raw, gx, gy);
    }
  }
  __syncthreads();
  block_flush_scalars<kBigThreads>(wl_acc, L, kHpwl, kGrad ? a.part + a.part_offset + net : nullptr,
                                   a.limbs);
}

template <int MODE>
void launch_mode(const Ctx &c, const WaArgs &a, cudaStream_t s) {
  if (c.n_chunks > 0) k_wa_chunks<MODE><<<c.n_chunks, kWaThreads, 0, s>>>(a);
  if (c.n_big > 0) k_wa_big<MODE><<<c.n_big, kBigThreads, 0, s>>>(a);
}

}  // namespace

void launch_wa(const Ctx &c, const float *x, const float *y, float gamma, bool hpwl_only,
               bool with_hpwl, cudaStream_t s) {
  WaArgs a;
  a.chunks = c.d_chunks;
  a.wgs = c.d_wgroups;
  a.net_deg = c.d_net_deg;
  a.net_w = c.d_net_w;
  a.pin_cell = c.d_pin_cell;
  a.pin_dx = c.d_pin_dx;
  a.pin_dy = c.d_pin_dy;
  a.x = x;
  a.y = y;
  a.g2 = c.d_g2;
  a.gamma = gamma;
  a.inv_gamma = 1.f / gamma;
  a.k2 = kLog2e / gamma;
  a.part = c.d_part;
  a.limbs = c.d_limbs;
  a.has_w = c.has_weights ? 1 : 0;
  a.big_start = c.d_big_start;
  a.big_flags = c.d_big_flags;
  a.big_cell = c.d_big_cell;
  a.big_w = c.d_big_w;
  a.big_dx = c.d_big_dx;
  a.big_dy = c.d_big_dy;
  a.part_offset = c.n_chunks;
  if (hpwl_only)
    launch_mode<2>(c, a, s);
  else if (with_hpwl)
    launch_mode<1>(c, a, s);
  else
    launch_mode<0>(c, a, s);
}

}  // namespace dp
