// wa.cu — weighted-average wirelength, its gradient and HPWL on sm_100a.
//
// Method: WA of eq (3) with the overflow-safe shift of P:159 and Table I
// notation; gradient of eq (6); merged forward+backward per net as in
// Alg 2 so no per-net intermediate touches global memory; HPWL.
//
// B200 design, differences from the paper's Alg 2:
//  * nets are locality-sorted into chunks at dp_create (~2048 pins).  A CTA owns one chunk and
//    stages it in shared memory with bulk async copies (cp.async.bulk + mbarrier): pin records,
//    net degrees, warp-group metadata, the chunk's window of 1024 consecutive cells and a
//    deduplicated list of its "far" cells.  Every pin refers to a chunk-local position slot
//    [window | far | trash], so the inner loop touches shared memory only and has no
//    data-dependent branches;
//  * pin -> cell gradients accumulate in shared memory as int32 fixed point (sm_100a has a
//    native 32-bit integer ATOMS.ADD; shared float atomics are CAS loops), with a per-chunk
//    scale chosen at create from a bound on the cell sums, then flush once per cell with
//    coalesced red.global.add.v4.f32 (window) / v2 (far cells);
//  * nets are processed by groups of G = 1..32 lanes (by degree), each lane holding up to 4
//    pins in registers (slot count templated): a^+- are computed once and kept (Alg 2
//    recomputes them); x and y fused (the paper uses two streams);
//  * 2-pin nets (55% of nets) use the closed form of eqs (3)/(6) for two pins;
//  * numerics: the shift reference is the rounded extreme P = max fl(x + dx); for every pin
//    whose exponential matters, x_cell - P is exact (Sterbenz) and the rounding of P is a
//    common shift that cancels exactly (reading A2).  Values are carried in log2 units;
//  * HPWL mode uses exact (TwoSum) pin positions and extremes and a 2^-149 fixed-point int64
//    limb sum: correctly rounded and order independent (reading A7).
#include <algorithm>

#include "async_copy.cuh"
#include "dp_internal.h"

namespace dp {

namespace {

constexpr float kLog2e = 1.4426950408889634f;
constexpr float kLn2 = 0.6931471805599453f;

constexpr int kWaSmemOptIn = 227 * 1024 - 8192;   // dynamic opt-in, leaving room for the static shared arrays

struct WaArgs {
  const Chunk *chunks;
  const WarpGroup *wgs;
  const int32_t *net_deg;
  const float *net_w;
  const int32_t *pin_slot;
  const float *pin_dx, *pin_dy;
  const int32_t *far_cells;
  const float *x, *y;
  float2 *g2;
  long long *g2i;               // deterministic mode (NEXT-2): int64 gradient in units 2^-det_frac, else null
  float *gxo, *gyo;             // direct output (DP_DIRECT): add into the caller's gx, gy (16-byte aligned)
  int det_frac;
  float gamma, inv_gamma, k2;   // k2 = log2(e) / gamma
  const float *gamma_dev;       // non-null: gamma read from device memory (GP loop, graph-replayed)
  double *part;                 // WA partial per CTA
  unsigned long long *limbs;    // HPWL limbs
  int has_w;
  int stream_hint;              // evict-first L2 policy on the staged netlist data (DP_L2_HINT=0: off)
  // big nets
  const int32_t *big_start, *big_flags, *big_cell;
  const float *big_w, *big_dx, *big_dy;
  int part_base;                // global WA unit of this context's unit 0: unit u writes part[part_base + u]
  int unit0;                    // unit of this launch's CTA 0 (a split WA launch: CTA b runs unit unit0 + b)
  int hp_offset;                // MODE 4: fast-HPWL partials at part[hp_offset + the WA partial's index]
  int big_stage;   // pins staged in shared memory per big-net CTA
  int n_huge, n_big, n_warp_blocks;
  WaCaps caps;
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

__device__ __forceinline__ float lg2(float v) {
  float r;
  asm("lg2.approx.ftz.f32 %0, %1;" : "=f"(r) : "f"(v));
  return r;
}

__device__ __forceinline__ float rcp(float v) {
  float r;
  asm("rcp.approx.ftz.f32 %0, %1;" : "=f"(r) : "f"(v));
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

__device__ __forceinline__ void red_f1(float *p, float v) {
  asm volatile("red.global.add.f32 [%0], %1;" ::"l"(p), "f"(v) : "memory");
}

__device__ __forceinline__ void red_s64(long long *p, long long v) {
  asm volatile("red.global.add.u64 [%0], %1;" ::"l"(p), "l"(v) : "memory");
}

// Deterministic mode (NEXT-2): a per-pin contribution becomes an int64 in units 2^-F (one
// rounding of the fp32 value, independent of order), summed with integer atomics: the cell
// gradient is then bit-identical from run to run whatever the atomic order.
template <class A>
__device__ __forceinline__ void grad_out(const A &a, int cell, float gx, float gy) {
  if (a.g2i) {
    red_s64(a.g2i + 2 * cell, __double2ll_rn(ldexp((double)gx, a.det_frac)));
    red_s64(a.g2i + 2 * cell + 1, __double2ll_rn(ldexp((double)gy, a.det_frac)));
  } else if (a.gxo) {
    red_f1(a.gxo + cell, gx);
    red_f1(a.gyo + cell, gy);
  } else {
    red_v2(a.g2 + cell, gx, gy);
  }
}

// int32 slot sum in units 2^-scale -> int64 in units 2^-F (exact when F >= scale)
__device__ __forceinline__ long long to_det(int v, int shift) {
  return shift >= 0 ? ((long long)v << shift) : ((long long)v >> -shift);
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
                                    bool hpwl, double *part_slot, unsigned long long *limbs,
                                    double hp = 0.0, double *hp_slot = nullptr) {
  __shared__ double s_wl[THREADS / 32];
  __shared__ double s_hp[THREADS / 32];
  __shared__ unsigned long long s_l[THREADS / 32][kHpwlLimbs + 1];
  const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
#pragma unroll
  for (int o = 16; o > 0; o >>= 1) wl += __shfl_xor_sync(0xffffffffu, wl, o);
  if (hp_slot) {
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) hp += __shfl_xor_sync(0xffffffffu, hp, o);
  }
  if (hpwl) {
#pragma unroll
    for (int k = 0; k <= kHpwlLimbs; k++) {
#pragma unroll
      for (int o = 16; o > 0; o >>= 1) L[k] += __shfl_xor_sync(0xffffffffu, L[k], o);
    }
  }
  if (lane == 0) {
    s_wl[warp] = wl;
    s_hp[warp] = hp;
    if (hpwl)
#pragma unroll
      for (int k = 0; k <= kHpwlLimbs; k++) s_l[warp][k] = L[k];
  }
  __syncthreads();
  if (threadIdx.x == 0) {
    double t = 0.0;
    for (int w = 0; w < THREADS / 32; w++) t += s_wl[w];
    if (part_slot) *part_slot = t;
    if (hp_slot) {
      double h = 0.0;
      for (int w = 0; w < THREADS / 32; w++) h += s_hp[w];
      *hp_slot = h;
    }
  }
  if (hpwl && threadIdx.x <= kHpwlLimbs) {
    unsigned long long t = 0;
    for (int w = 0; w < THREADS / 32; w++) t += s_l[w][threadIdx.x];
    if (t) atomicAdd(limbs + threadIdx.x, t);
  }
}

// Per-lane running extremes of one axis as exact (hi, lo) pairs (HPWL mode).
struct Axis { float Ph, Pl, Mh, Ml; };

__device__ __forceinline__ void ext_update(Axis &A, float h, float l) {
  if (pair_gt(h, l, A.Ph, A.Pl)) { A.Ph = h; A.Pl = l; }
  if (pair_gt(A.Mh, A.Ml, h, l)) { A.Mh = h; A.Ml = l; }
}

__device__ __forceinline__ void ext_shfl(Axis &A, int o) {
  const float ph = __shfl_xor_sync(0xffffffffu, A.Ph, o), pl = __shfl_xor_sync(0xffffffffu, A.Pl, o);
  const float mh = __shfl_xor_sync(0xffffffffu, A.Mh, o), ml = __shfl_xor_sync(0xffffffffu, A.Ml, o);
  if (pair_gt(ph, pl, A.Ph, A.Pl)) { A.Ph = ph; A.Pl = pl; }
  if (pair_gt(A.Mh, A.Ml, mh, ml)) { A.Mh = mh; A.Ml = ml; }
}

// Shared-memory view of one staged chunk.
struct GroupCtx {
  const int *slot;       // [pins] position slot
  const float *dx, *dy;  // [pins]
  const int *deg;        // [nets] degree | counted << 31
  const float *w;        // [nets]
  const float *px, *py;  // [slots] cell positions: window cells, then far cells
  int *g;                // [2 * slots] int32 fixed-point gradient (x, y interleaved)
  int trash;             // gradient slot of foreign pins (never flushed)
  float scale;           // 2^scale_log2
  int lane;
  unsigned lt_mask;
};

__device__ __forceinline__ void grad_add(const GroupCtx &gc, int raw, float gx, float gy) {
  atomicAdd(gc.g + 2 * raw, __float2int_rn(gx * gc.scale));
  atomicAdd(gc.g + 2 * raw + 1, __float2int_rn(gy * gc.scale));
}

// the same with gx, gy already in the chunk's fixed-point units (the scale folded into the
// per-net coefficients)
__device__ __forceinline__ void grad_add_scaled(const GroupCtx &gc, int raw, float gx, float gy) {
  atomicAdd(gc.g + 2 * raw, __float2int_rn(gx));
  atomicAdd(gc.g + 2 * raw + 1, __float2int_rn(gy));
}

// Pin records of one warp group, slot-major compressed layout (32/G nets, G lanes per net):
// slot s holds, in lane order, the pins s G + j < d of every net.  (A ballot-free variant for
// groups of one degree measured no faster: the arithmetic replacing the ballot costs as much.)
template <int S>
__device__ __forceinline__ unsigned load_pins(const WarpGroup &wg, const GroupCtx &gc, int G, int j, int d,
                                              int (&raw)[S], float (&xc)[S], float (&yc)[S], float (&dxs)[S],
                                              float (&dys)[S]) {
  unsigned vm = 0;
  int base = wg.pin_base;
#pragma unroll
  for (int s = 0; s < S; s++) {
    const bool valid = s * G + j < d;
    const unsigned m = __ballot_sync(0xffffffffu, valid);
    const int p = valid ? base + __popc(m & gc.lt_mask) : wg.pin_base;
    raw[s] = gc.slot[p];
    dxs[s] = gc.dx[p];
    dys[s] = gc.dy[p];
    xc[s] = gc.px[raw[s]];
    yc[s] = gc.py[raw[s]];
    vm |= (valid ? 1u : 0u) << s;
    base += __popc(m);
  }
  return vm;
}

// HPWL modes (MODE 1: WA + gradient + HPWL, MODE 2: HPWL only): exact TwoSum positions.
template <int MODE, int S>
__device__ __forceinline__ void wa_group_exact(const WaArgs &a, const WarpGroup &wg, const GroupCtx &gc, float &wl_acc,
                                               unsigned long long (&L)[kHpwlLimbs + 1]) {
  constexpr bool kGrad = MODE != 2;
  const int glog = wg.g_log2, G = 1 << glog;
  const int gi = gc.lane >> glog, j = gc.lane & (G - 1);
  int d = 0, counted = 0;
  float we = 1.f;
  if (gi < wg.nnets) {
    const int r = gc.deg[wg.net_base + gi];
    d = r & 0x7fffffff;
    counted = (r >> 31) & 1;
    if (a.has_w) we = gc.w[wg.net_base + gi];
  }
  int raw[S];
  float xc[S], yc[S], dxs[S], dys[S];
  const unsigned vm = load_pins<S>(wg, gc, G, j, d, raw, xc, yc, dxs, dys);
  float hx[S], lx[S], hy[S], ly[S];
  Axis X{-INFINITY, 0.f, INFINITY, 0.f}, Y{-INFINITY, 0.f, INFINITY, 0.f};
#pragma unroll
  for (int s = 0; s < S; s++) {
    two_sum(xc[s], dxs[s], hx[s], lx[s]);
    two_sum(yc[s], dys[s], hy[s], ly[s]);
    if (vm & (1u << s)) {
      ext_update(X, hx[s], lx[s]);
      ext_update(Y, hy[s], ly[s]);
    }
  }
  for (int o = 1; o < G; o <<= 1) {
    ext_shfl(X, o);
    ext_shfl(Y, o);
  }
  if (j == 0 && d >= 2 && counted) {
    // px = fl64(x + dx) as the oracle forms it: (double)hi + (double)lo rounds the exact real
    // x + dx once (reading A7)
    const double xp = __dadd_rn((double)X.Ph, (double)X.Pl), xm = __dadd_rn((double)X.Mh, (double)X.Ml);
    const double yp = __dadd_rn((double)Y.Ph, (double)Y.Pl), ym = __dadd_rn((double)Y.Mh, (double)Y.Ml);
    limbs_add(L, __dadd_rn(__dsub_rn(xp, xm), __dsub_rn(yp, ym)));
  }
  if (!kGrad) return;
  float lxp[S], lxm[S], lyp[S], lym[S], axp[S], axm[S], ayp[S], aym[S];
  float bxp = 0.f, bxm = 0.f, cxp = 0.f, cxm = 0.f, byp = 0.f, bym = 0.f, cyp = 0.f, cym = 0.f;
#pragma unroll
  for (int s = 0; s < S; s++) {
    const bool v = vm & (1u << s);
    lxp[s] = v ? __fadd_rn(__fsub_rn(hx[s], X.Ph), __fsub_rn(lx[s], X.Pl)) * a.k2 : -1e30f;
    lxm[s] = v ? __fadd_rn(__fsub_rn(hx[s], X.Mh), __fsub_rn(lx[s], X.Ml)) * a.k2 : 1e30f;
    lyp[s] = v ? __fadd_rn(__fsub_rn(hy[s], Y.Ph), __fsub_rn(ly[s], Y.Pl)) * a.k2 : -1e30f;
    lym[s] = v ? __fadd_rn(__fsub_rn(hy[s], Y.Mh), __fsub_rn(ly[s], Y.Ml)) * a.k2 : 1e30f;
    axp[s] = ex2(lxp[s]);
    axm[s] = ex2(-lxm[s]);
    ayp[s] = ex2(lyp[s]);
    aym[s] = ex2(-lym[s]);
    bxp += axp[s]; cxp = fmaf(lxp[s], axp[s], cxp);
    bxm += axm[s]; cxm = fmaf(lxm[s], axm[s], cxm);
    byp += ayp[s]; cyp = fmaf(lyp[s], ayp[s], cyp);
    bym += aym[s]; cym = fmaf(lym[s], aym[s], cym);
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
  if (d < 2) return;
  const float ibxp = rcp(bxp), ibxm = rcp(bxm), ibyp = rcp(byp), ibym = rcp(bym);
  const float mxp = cxp * ibxp, mxm = cxm * ibxm, myp = cyp * ibyp, mym = cym * ibym;
  if (j == 0 && counted) {
    const float ig2 = a.gamma * kLn2;
    const float spanx = __fadd_rn(__fsub_rn(X.Ph, X.Mh), __fsub_rn(X.Pl, X.Ml));
    const float spany = __fadd_rn(__fsub_rn(Y.Ph, Y.Mh), __fsub_rn(Y.Pl, Y.Ml));
    wl_acc += we * ((spanx + (mxp - mxm) * ig2) + (spany + (myp - mym) * ig2));
  }
  const float wl2 = we * kLn2;
  const float qxp = ibxp * wl2, pxp = we * ibxp - mxp * qxp;
  const float qxm = ibxm * wl2, pxm = we * ibxm + mxm * qxm;
  const float qyp = ibyp * wl2, pyp = we * ibyp - myp * qyp;
  const float qym = ibym * wl2, pym = we * ibym + mym * qym;
#pragma unroll
  for (int s = 0; s < S; s++) {
    if (vm & (1u << s)) {
      const float gx = axp[s] * fmaf(lxp[s], qxp, pxp) - axm[s] * fmaf(-lxm[s], qxm, pxm);
      const float gy = ayp[s] * fmaf(lyp[s], qyp, pyp) - aym[s] * fmaf(-lym[s], qym, pym);
      grad_add(gc, raw[s], gx, gy);
    }
  }
}

// Headline path (no HPWL).  Shift reference = the rounded extreme P = max fl(x_c + dx): for
// every pin whose exponential matters, (x_c - P) is exact (Sterbenz) and the one rounding of
// P is a common shift that cancels in eq (3)/(6).  Everything is carried in log2 units
// lambda = (x - P) log2(e)/gamma, so a = 2^lambda and (x - m)/gamma = (lambda - mu) ln 2.
// Invalid slots get lambda = -+1e30 (a = 0, lambda a = 0): no per-slot branches.
//
// LSE (NEXT-3, reading A27): the same b^+- sums; LSE_e = (x+ - x-) + gamma ln 2 (log2 b+ + log2 b-)
// and dLSE/dx_i = a_i^+/b^+ - a_i^-/b^-; the c sums are not formed.
template <int S, bool LSE, bool HP>
__device__ __forceinline__ void wa_group_fast(const WaArgs &a, const WarpGroup &wg, const GroupCtx &gc,
                                              float &wl_acc, float &hp_acc) {
  const int glog = wg.g_log2, G = 1 << glog;
  const int gi = gc.lane >> glog, j = gc.lane & (G - 1);
  int d = 0, counted = 0;
  float we = 1.f;
  if (gi < wg.nnets) {
    const int r = gc.deg[wg.net_base + gi];
    d = r & 0x7fffffff;
    counted = (r >> 31) & 1;
    if (a.has_w) we = gc.w[wg.net_base + gi];
  }
  int raw[S];
  float xc[S], yc[S], dxs[S], dys[S];
  const unsigned vm = load_pins<S>(wg, gc, G, j, d, raw, xc, yc, dxs, dys);
  float Px = -INFINITY, Mx = INFINITY, Py = -INFINITY, My = INFINITY;
#pragma unroll
  for (int s = 0; s < S; s++) {
    const bool v = vm & (1u << s);
    const float px = xc[s] + dxs[s], py = yc[s] + dys[s];
    Px = fmaxf(Px, v ? px : -INFINITY);
    Mx = fminf(Mx, v ? px : INFINITY);
    Py = fmaxf(Py, v ? py : -INFINITY);
    My = fminf(My, v ? py : INFINITY);
  }
  for (int o = 1; o < G; o <<= 1) {
    Px = fmaxf(Px, __shfl_xor_sync(0xffffffffu, Px, o));
    Mx = fminf(Mx, __shfl_xor_sync(0xffffffffu, Mx, o));
    Py = fmaxf(Py, __shfl_xor_sync(0xffffffffu, Py, o));
    My = fminf(My, __shfl_xor_sync(0xffffffffu, My, o));
  }
  const float k2 = a.k2;
  float lxp[S], lxm[S], lyp[S], lym[S], axp[S], axm[S], ayp[S], aym[S];
  float bxp = 0.f, bxm = 0.f, cxp = 0.f, cxm = 0.f, byp = 0.f, bym = 0.f, cyp = 0.f, cym = 0.f;
#pragma unroll
  for (int s = 0; s < S; s++) {
    const bool v = vm & (1u << s);
    const float dkx = dxs[s] * k2, dky = dys[s] * k2;
    lxp[s] = v ? fmaf(xc[s] - Px, k2, dkx) : -1e30f;   // <= 0 (to an ulp of P)
    lxm[s] = v ? fmaf(xc[s] - Mx, k2, dkx) : 1e30f;    // >= 0
    lyp[s] = v ? fmaf(yc[s] - Py, k2, dky) : -1e30f;
    lym[s] = v ? fmaf(yc[s] - My, k2, dky) : 1e30f;
    axp[s] = ex2(lxp[s]);
    axm[s] = ex2(-lxm[s]);
    ayp[s] = ex2(lyp[s]);
    aym[s] = ex2(-lym[s]);
    bxp += axp[s];
    bxm += axm[s];
    byp += ayp[s];
    bym += aym[s];
    if (!LSE) {
      cxp = fmaf(lxp[s], axp[s], cxp);
      cxm = fmaf(lxm[s], axm[s], cxm);
      cyp = fmaf(lyp[s], ayp[s], cyp);
      cym = fmaf(lym[s], aym[s], cym);
    }
  }
  for (int o = 1; o < G; o <<= 1) {
    bxp += __shfl_xor_sync(0xffffffffu, bxp, o);
    bxm += __shfl_xor_sync(0xffffffffu, bxm, o);
    byp += __shfl_xor_sync(0xffffffffu, byp, o);
    bym += __shfl_xor_sync(0xffffffffu, bym, o);
    if (!LSE) {
      cxp += __shfl_xor_sync(0xffffffffu, cxp, o);
      cxm += __shfl_xor_sync(0xffffffffu, cxm, o);
      cyp += __shfl_xor_sync(0xffffffffu, cyp, o);
      cym += __shfl_xor_sync(0xffffffffu, cym, o);
    }
  }
  if (d < 2) return;
  const float ibxp = rcp(bxp), ibxm = rcp(bxm), ibyp = rcp(byp), ibym = rcp(bym);
  if (LSE) {
    if (j == 0 && counted) {
      const float ig2 = a.gamma * kLn2;
      wl_acc += we * ((Px - Mx) + (Py - My) + (lg2(bxp) + lg2(bxm) + lg2(byp) + lg2(bym)) * ig2);
    }
    const float wxp = we * ibxp, wxm = we * ibxm, wyp = we * ibyp, wym = we * ibym;
#pragma unroll
    for (int s = 0; s < S; s++) {
      if (vm & (1u << s)) grad_add(gc, raw[s], axp[s] * wxp - axm[s] * wxm, ayp[s] * wyp - aym[s] * wym);
    }
    return;
  }
  const float mxp = cxp * ibxp, mxm = cxm * ibxm, myp = cyp * ibyp, mym = cym * ibym;  // log2 units
  if (j == 0 && counted) {
    // WL_e = (x+ - x-) + (mu+ - mu-) gamma ln 2   (eq 3 in shifted coordinates)
    if (HP) hp_acc += (Px - Mx) + (Py - My);   // fast HPWL (GP schedule; reading A37)
    const float ig2 = a.gamma * kLn2;
    wl_acc += we * ((Px - Mx) + (mxp - mxm) * ig2 + (Py - My) + (myp - mym) * ig2);
  }
  // eq (6) in log2 units: a+ (P+ + lambda+ Q+) - a- (P- - lambda- Q-), in the chunk's
  // fixed-point units (w_e times the slot scale 2^k: exact power-of-two scaling)
  const float ws = we * gc.scale, wl2 = ws * kLn2;
  const float qxp = ibxp * wl2, pxp = ws * ibxp - mxp * qxp;
  const float qxm = ibxm * wl2, pxm = ws * ibxm + mxm * qxm;
  const float qyp = ibyp * wl2, pyp = ws * ibyp - myp * qyp;
  const float qym = ibym * wl2, pym = ws * ibym + mym * qym;
#pragma unroll
  for (int s = 0; s < S; s++) {
    if (vm & (1u << s)) {
      const float gx = axp[s] * fmaf(lxp[s], qxp, pxp) - axm[s] * fmaf(-lxm[s], qxm, pxm);
      const float gy = ayp[s] * fmaf(lyp[s], qyp, pyp) - aym[s] * fmaf(-lym[s], qym, pym);
      grad_add_scaled(gc, raw[s], gx, gy);
    }
  }
}

// tanh(u/2) for u = t ln2 >= 0 given e = 2^-t: series for small u (1 - e loses digits),
// (1 - e)/(1 + e) otherwise.
__device__ __forceinline__ float tanh_half(float t, float e) {
  const float h = 0.5f * kLn2 * t;
  if (h < 0.0625f) {
    const float h2 = h * h;
    return h * fmaf(h2, fmaf(h2, 2.f / 15.f, -1.f / 3.f), 1.f);
  }
  return (1.f - e) * rcp(1.f + e);
}

// Warp groups of 2-pin nets (G = 1): the closed form of eqs (3)/(6) for two pins at
// separation delta, WA = |delta| tanh(|delta| / 2 gamma) and dWA/dx_2 = -dWA/dx_1 =
// sign(delta) [tanh(u/2) + (u/2) sech^2(u/2)], u = |delta| / gamma (pinned against the oracle
// in tests/test_oracle_wa.py::test_two_pin_closed_form).
//
// LSE (reading A27): LSE = |delta| + 2 gamma ln(1 + e^-u) per axis and dLSE/dx_2 = sign(delta) tanh(u/2).
//
// EX (MODE 1): the exact HPWL of the pair as the exact-HPWL groups form it (TwoSum positions,
// exact extremes, fp64 span, int64 limbs; reading A7) beside the fp32 closed form for WA.
template <bool LSE, bool HP, bool EX>
__device__ __forceinline__ void wa_group_pairs(const WaArgs &a, const WarpGroup &wg, const GroupCtx &gc,
                                               float &wl_acc, float &hp_acc,
                                               unsigned long long (&L)[kHpwlLimbs + 1]) {
  const int lane = gc.lane;
  if (lane >= wg.nnets) return;
  const int r = gc.deg[wg.net_base + lane];
  const int counted = (r >> 31) & 1;
  const float we = a.has_w ? gc.w[wg.net_base + lane] : 1.f;
  // slot-major: pin 0 of net L at pin_base + L, pin 1 at pin_base + nnets + L
  const int p0 = wg.pin_base + lane, p1 = p0 + wg.nnets;
  const int r0 = gc.slot[p0], r1 = gc.slot[p1];
  const int s0 = r0, s1 = r1;
  const float ddx = (gc.px[s1] - gc.px[s0]) + (gc.dx[p1] - gc.dx[p0]);
  const float ddy = (gc.py[s1] - gc.py[s0]) + (gc.dy[p1] - gc.dy[p0]);
  const float tx = fabsf(ddx) * a.k2, ty = fabsf(ddy) * a.k2;   // u log2(e)
  const float ex = ex2(-tx), ey = ex2(-ty);
  const float thx = tanh_half(tx, ex), thy = tanh_half(ty, ey);
  if (LSE) {
    if (counted)
      wl_acc += we * (fabsf(ddx) + fabsf(ddy) + (2.f * kLn2) * a.gamma * (lg2(1.f + ex) + lg2(1.f + ey)));
    const float gx = copysignf(we * thx, ddx), gy = copysignf(we * thy, ddy);
    grad_add(gc, r1, gx, gy);
    grad_add(gc, r0, -gx, -gy);
    return;
  }
  if (counted) wl_acc += we * (fabsf(ddx) * thx + fabsf(ddy) * thy);
  if (HP && counted) hp_acc += fabsf(ddx) + fabsf(ddy);
  if (EX && counted) {
    float h0x, l0x, h1x, l1x, h0y, l0y, h1y, l1y;
    two_sum(gc.px[s0], gc.dx[p0], h0x, l0x);
    two_sum(gc.px[s1], gc.dx[p1], h1x, l1x);
    two_sum(gc.py[s0], gc.dy[p0], h0y, l0y);
    two_sum(gc.py[s1], gc.dy[p1], h1y, l1y);
    const bool ox = pair_gt(h1x, l1x, h0x, l0x), oy = pair_gt(h1y, l1y, h0y, l0y);
    const double xp = __dadd_rn((double)(ox ? h1x : h0x), (double)(ox ? l1x : l0x));
    const double xm = __dadd_rn((double)(ox ? h0x : h1x), (double)(ox ? l0x : l1x));
    const double yp = __dadd_rn((double)(oy ? h1y : h0y), (double)(oy ? l1y : l0y));
    const double ym = __dadd_rn((double)(oy ? h0y : h1y), (double)(oy ? l0y : l1y));
    limbs_add(L, __dadd_rn(__dsub_rn(xp, xm), __dsub_rn(yp, ym)));
  }
  const float hx = 0.5f * kLn2 * tx, hy = 0.5f * kLn2 * ty;
  const float gx = copysignf(we * fmaf(hx, fmaf(-thx, thx, 1.f), thx), ddx);   // d/dx of pin 1
  const float gy = copysignf(we * fmaf(hy, fmaf(-thy, thy, 1.f), thy), ddy);
  grad_add(gc, r1, gx, gy);
  grad_add(gc, r0, -gx, -gy);
}

// (A compile-time lanes-per-net variant of wa_group_fast, 24 instantiations, measured 85 -> 107
// us: the kernel's code outgrows the instruction caches.)
template <bool LSE, bool HP>
__device__ __forceinline__ void wa_group_fast_dispatch(const WaArgs &a, const WarpGroup &wg, const GroupCtx &gc,
                                                       float &wl_acc, float &hp_acc) {
  switch (wg.slots) {
    case 1: wa_group_fast<1, LSE, HP>(a, wg, gc, wl_acc, hp_acc); break;
    case 2: wa_group_fast<2, LSE, HP>(a, wg, gc, wl_acc, hp_acc); break;
    case 3: wa_group_fast<3, LSE, HP>(a, wg, gc, wl_acc, hp_acc); break;
    default: wa_group_fast<4, LSE, HP>(a, wg, gc, wl_acc, hp_acc); break;
  }
}

// Dynamic shared-memory layout of the chunk kernel (capacities fixed at create).
struct WaSmem {
  WaCaps c;
  __host__ __device__ int slots() const { return kWaWindow + c.far + 4; }   // + trash, padded
  __host__ __device__ int off_slot() const { return 0; }
  __host__ __device__ int off_dx() const { return 4 * c.pins; }
  __host__ __device__ int off_dy() const { return 8 * c.pins; }
  __host__ __device__ int off_deg() const { return 12 * c.pins; }
  __host__ __device__ int off_w() const { return off_deg() + 4 * c.nets; }
  __host__ __device__ int off_wg() const { return off_w() + 4 * c.nets; }
  __host__ __device__ int off_far() const { return off_wg() + 16 * c.groups; }
  __host__ __device__ int off_px() const { return off_far() + 4 * c.far; }
  __host__ __device__ int off_py() const { return off_px() + 4 * slots(); }
  __host__ __device__ int off_g() const { return off_py() + 4 * slots(); }
  __host__ __device__ int off_bar() const { return off_g() + 8 * slots(); }
  __host__ __device__ int bytes() const { return off_bar() + 16; }   // two mbarriers
};

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

// Exact shifted coordinates of big-net pin p: (hx, lx) = TwoSum(x_c, dx), (hy, ly) likewise.
__device__ __forceinline__ float4 big_pin(const WaArgs &a, int c, int s) {
  float4 v;
  two_sum(__ldg(a.x + c), __ldg(a.big_dx + s), v.x, v.y);
  two_sum(__ldg(a.y + c), __ldg(a.big_dy + s), v.z, v.w);
  return v;
}

// CTA per net of degree > kWaMaxDeg (largest first).  Pass 1 loads every pin once (4 loads in
// flight per thread) and keeps the exact coordinates in shared memory (nets up to kBigStage
// pins; larger nets reload), pass 2 forms the eq-6 sums, pass 3 the gradient.
static_assert(kBigThreads == kWaThreads && kWarpNetThreads == kWaThreads, "big / warp nets run in chunk-kernel CTAs");

template <int MODE>
__device__ __forceinline__ void wa_big_net(const WaArgs &a, int net, float4 *s_pin) {
  constexpr bool kGrad = MODE != 2;
  constexpr bool kHpwl = MODE == 1 || MODE == 2;
  constexpr bool kLse = MODE == 3;
  double hp_b = 0.0;
  const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
  constexpr int NW = kBigThreads / 32;
  const int s0 = a.big_start[net], d = a.big_start[net + 1] - s0;
  const bool staged = d <= a.big_stage;
  const int counted = a.big_flags[net];
  const float we = a.has_w ? a.big_w[net] : 1.f;
  __shared__ Ext s_ext[NW];
  __shared__ float s_sum[NW][8];

  Ext e{-INFINITY, 0.f, INFINITY, 0.f, -INFINITY, 0.f, INFINITY, 0.f};
  for (int p0 = tid; p0 < d; p0 += 4 * kBigThreads) {
    int c[4];
#pragma unroll
    for (int k = 0; k < 4; k++) {
      const int p = p0 + k * kBigThreads;
      c[k] = p < d ? (__ldg(a.big_cell + s0 + p) & 0x7fffffff) : -1;
    }
    float4 v[4];
#pragma unroll
    for (int k = 0; k < 4; k++)
      if (c[k] >= 0) v[k] = big_pin(a, c[k], s0 + p0 + k * kBigThreads);
#pragma unroll
    for (int k = 0; k < 4; k++) {
      if (c[k] < 0) continue;
      if (staged) s_pin[p0 + k * kBigThreads] = v[k];
      const Ext o{v[k].x, v[k].y, v[k].x, v[k].y, v[k].z, v[k].w, v[k].z, v[k].w};
      ext_merge(e, o);
    }
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
  __syncthreads();   // also publishes s_pin
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
      const float4 v = staged ? s_pin[p] : big_pin(a, __ldg(a.big_cell + s0 + p) & 0x7fffffff, s0 + p);
      const float lxp = __fadd_rn(__fsub_rn(v.x, e.Xh), __fsub_rn(v.y, e.Xl));
      const float lxm = __fadd_rn(__fsub_rn(v.x, e.xh), __fsub_rn(v.y, e.xl));
      const float lyp = __fadd_rn(__fsub_rn(v.z, e.Yh), __fsub_rn(v.w, e.Yl));
      const float lym = __fadd_rn(__fsub_rn(v.z, e.yh), __fsub_rn(v.w, e.yl));
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
      if (MODE == 4) hp_b = (double)(spanx + spany);
      if (kLse)   // reading A27: (x+ + gamma ln b+) - (x- - gamma ln b-)
        wl_acc = (double)(we * ((spanx + spany) + a.gamma * (logf(sm[0]) + logf(sm[2]) + logf(sm[4]) + logf(sm[6]))));
      else
        wl_acc = (double)(we * ((spanx + mxp - mxm) + (spany + myp - mym)));
    }
    for (int p = tid; p < d; p += kBigThreads) {
      const int raw = __ldg(a.big_cell + s0 + p);
      if (raw < 0) continue;
      const float4 v = staged ? s_pin[p] : big_pin(a, raw, s0 + p);
      const float lxp = __fadd_rn(__fsub_rn(v.x, e.Xh), __fsub_rn(v.y, e.Xl));
      const float lxm = __fadd_rn(__fsub_rn(v.x, e.xh), __fsub_rn(v.y, e.xl));
      const float lyp = __fadd_rn(__fsub_rn(v.z, e.Yh), __fsub_rn(v.w, e.Yl));
      const float lym = __fadd_rn(__fsub_rn(v.z, e.yh), __fsub_rn(v.w, e.yl));
      const float axp = ex2(lxp * a.k2), axm = ex2(-lxm * a.k2);
      const float ayp = ex2(lyp * a.k2), aym = ex2(-lym * a.k2);
      const float gx = kLse ? we * (axp * ibxp - axm * ibxm)
                            : we * (axp * ibxp * (1.f + (lxp - mxp) * a.inv_gamma) -
                                    axm * ibxm * (1.f - (lxm - mxm) * a.inv_gamma));
      const float gy = kLse ? we * (ayp * ibyp - aym * ibym)
                            : we * (ayp * ibyp * (1.f + (lyp - myp) * a.inv_gamma) -
                                    aym * ibym * (1.f - (lym - mym) * a.inv_gamma));
      grad_out(a, raw, gx, gy);
    }
  }
  __syncthreads();
  const int slot = a.part_base + a.unit0 + blockIdx.x;
  block_flush_scalars<kBigThreads>(wl_acc, L, kHpwl, kGrad ? a.part + slot : nullptr, a.limbs, hp_b,
                                   MODE == 4 ? a.part + a.hp_offset + slot : nullptr);
}

// Warp per net for degrees (kWaMaxDeg, kWarpNetMax]: three passes over the pins with warp
// shuffles only (no block barriers); passes 2 and 3 reload the pin data (L1 / L2 resident).
// MODE 0 uses the log2-unit fast path of the chunk kernel (shift reference P = max fl(x + dx));
// the HPWL modes form exact TwoSum coordinates as k_wa_big does.
__device__ __forceinline__ float warp_max(float v) {
#pragma unroll
  for (int o = 16; o > 0; o >>= 1) v = fmaxf(v, __shfl_xor_sync(0xffffffffu, v, o));
  return v;
}
__device__ __forceinline__ float warp_min(float v) {
#pragma unroll
  for (int o = 16; o > 0; o >>= 1) v = fminf(v, __shfl_xor_sync(0xffffffffu, v, o));
  return v;
}
__device__ __forceinline__ float warp_sum(float v) {
#pragma unroll
  for (int o = 16; o > 0; o >>= 1) v += __shfl_xor_sync(0xffffffffu, v, o);
  return v;
}

template <int MODE>
__device__ __forceinline__ void wa_warp_nets(const WaArgs &a, int wb) {
  constexpr bool kGrad = MODE != 2;
  constexpr bool kHpwl = MODE == 1 || MODE == 2;
  constexpr bool kLse = MODE == 3;
  double hp_w = 0.0;
  const int lane = threadIdx.x & 31;
  const int net = a.n_huge + wb * (kWarpNetThreads / 32) + (threadIdx.x >> 5);
  double wl_acc = 0.0;
  unsigned long long L[kHpwlLimbs + 1];
#pragma unroll
  for (int k = 0; k <= kHpwlLimbs; k++) L[k] = 0ull;
  if (net < a.n_big) {
    const int s0 = a.big_start[net], d = a.big_start[net + 1] - s0;
    const int counted = a.big_flags[net];
    const float we = a.has_w ? a.big_w[net] : 1.f;
    const int *cell = a.big_cell + s0;
    const float *pdx = a.big_dx + s0, *pdy = a.big_dy + s0;
    if (MODE == 0 || MODE == 3 || MODE == 4) {
      float Px = -INFINITY, Mx = INFINITY, Py = -INFINITY, My = INFINITY;
#pragma unroll 4
      for (int p = lane; p < d; p += 32) {
        const int c = __ldg(cell + p) & 0x7fffffff;
        const float px = __ldg(a.x + c) + __ldg(pdx + p), py = __ldg(a.y + c) + __ldg(pdy + p);
        Px = fmaxf(Px, px); Mx = fminf(Mx, px);
        Py = fmaxf(Py, py); My = fminf(My, py);
      }
      Px = warp_max(Px); Mx = warp_min(Mx); Py = warp_max(Py); My = warp_min(My);
      const float k2 = a.k2;
      float bxp = 0.f, bxm = 0.f, cxp = 0.f, cxm = 0.f, byp = 0.f, bym = 0.f, cyp = 0.f, cym = 0.f;
#pragma unroll 4
      for (int p = lane; p < d; p += 32) {
        const int c = __ldg(cell + p) & 0x7fffffff;
        const float xc = __ldg(a.x + c), yc = __ldg(a.y + c);
        const float dkx = __ldg(pdx + p) * k2, dky = __ldg(pdy + p) * k2;
        const float lxp = fmaf(xc - Px, k2, dkx), lxm = fmaf(xc - Mx, k2, dkx);
        const float lyp = fmaf(yc - Py, k2, dky), lym = fmaf(yc - My, k2, dky);
        const float axp = ex2(lxp), axm = ex2(-lxm), ayp = ex2(lyp), aym = ex2(-lym);
        bxp += axp; cxp = fmaf(lxp, axp, cxp);
        bxm += axm; cxm = fmaf(lxm, axm, cxm);
        byp += ayp; cyp = fmaf(lyp, ayp, cyp);
        bym += aym; cym = fmaf(lym, aym, cym);
      }
      bxp = warp_sum(bxp); cxp = warp_sum(cxp); bxm = warp_sum(bxm); cxm = warp_sum(cxm);
      byp = warp_sum(byp); cyp = warp_sum(cyp); bym = warp_sum(bym); cym = warp_sum(cym);
      const float ibxp = rcp(bxp), ibxm = rcp(bxm), ibyp = rcp(byp), ibym = rcp(bym);
      const float mxp = cxp * ibxp, mxm = cxm * ibxm, myp = cyp * ibyp, mym = cym * ibym;   // log2 units
      if (lane == 0 && counted) {
        const float ig2 = a.gamma * kLn2;
        if (MODE == 4) hp_w = (double)((Px - Mx) + (Py - My));
        if (kLse)
          wl_acc = (double)(we * ((Px - Mx) + (Py - My) + (lg2(bxp) + lg2(bxm) + lg2(byp) + lg2(bym)) * ig2));
        else
          wl_acc = (double)(we * ((Px - Mx) + (mxp - mxm) * ig2 + (Py - My) + (myp - mym) * ig2));
      }
      const float wl2 = we * kLn2;
      const float qxp = ibxp * wl2, pxp = we * ibxp - mxp * qxp;
      const float qxm = ibxm * wl2, pxm = we * ibxm + mxm * qxm;
      const float qyp = ibyp * wl2, pyp = we * ibyp - myp * qyp;
      const float qym = ibym * wl2, pym = we * ibym + mym * qym;
#pragma unroll 4
      for (int p = lane; p < d; p += 32) {
        const int raw = __ldg(cell + p);
        if (raw < 0) continue;
        const float xc = __ldg(a.x + raw), yc = __ldg(a.y + raw);
        const float dkx = __ldg(pdx + p) * k2, dky = __ldg(pdy + p) * k2;
        const float lxp = fmaf(xc - Px, k2, dkx), lxm = fmaf(xc - Mx, k2, dkx);
        const float lyp = fmaf(yc - Py, k2, dky), lym = fmaf(yc - My, k2, dky);
        const float axp = ex2(lxp), axm = ex2(-lxm), ayp = ex2(lyp), aym = ex2(-lym);
        const float gx = kLse ? we * (axp * ibxp - axm * ibxm) : axp * fmaf(lxp, qxp, pxp) - axm * fmaf(-lxm, qxm, pxm);
        const float gy = kLse ? we * (ayp * ibyp - aym * ibym) : ayp * fmaf(lyp, qyp, pyp) - aym * fmaf(-lym, qym, pym);
        grad_out(a, raw, gx, gy);
      }
    } else {
      Ext e{-INFINITY, 0.f, INFINITY, 0.f, -INFINITY, 0.f, INFINITY, 0.f};
      for (int p = lane; p < d; p += 32) {
        const float4 v = big_pin(a, __ldg(cell + p) & 0x7fffffff, s0 + p);
        const Ext o{v.x, v.y, v.x, v.y, v.z, v.w, v.z, v.w};
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
      if (lane == 0 && counted) {
        const double xp = __dadd_rn((double)e.Xh, (double)e.Xl), xm = __dadd_rn((double)e.xh, (double)e.xl);
        const double yp = __dadd_rn((double)e.Yh, (double)e.Yl), ym = __dadd_rn((double)e.yh, (double)e.yl);
        limbs_add(L, __dadd_rn(__dsub_rn(xp, xm), __dsub_rn(yp, ym)));
      }
      if (kGrad) {
        float sm[8] = {0, 0, 0, 0, 0, 0, 0, 0};  // bxp cxp bxm cxm byp cyp bym cym
        for (int p = lane; p < d; p += 32) {
          const float4 v = big_pin(a, __ldg(cell + p) & 0x7fffffff, s0 + p);
          const float lxp = __fadd_rn(__fsub_rn(v.x, e.Xh), __fsub_rn(v.y, e.Xl));
          const float lxm = __fadd_rn(__fsub_rn(v.x, e.xh), __fsub_rn(v.y, e.xl));
          const float lyp = __fadd_rn(__fsub_rn(v.z, e.Yh), __fsub_rn(v.w, e.Yl));
          const float lym = __fadd_rn(__fsub_rn(v.z, e.yh), __fsub_rn(v.w, e.yl));
          const float axp = ex2(lxp * a.k2), axm = ex2(-lxm * a.k2);
          const float ayp = ex2(lyp * a.k2), aym = ex2(-lym * a.k2);
          sm[0] += axp; sm[1] += lxp * axp; sm[2] += axm; sm[3] += lxm * axm;
          sm[4] += ayp; sm[5] += lyp * ayp; sm[6] += aym; sm[7] += lym * aym;
        }
#pragma unroll
        for (int k = 0; k < 8; k++) sm[k] = warp_sum(sm[k]);
        const float ibxp = 1.f / sm[0], ibxm = 1.f / sm[2], ibyp = 1.f / sm[4], ibym = 1.f / sm[6];
        const float mxp = sm[1] * ibxp, mxm = sm[3] * ibxm, myp = sm[5] * ibyp, mym = sm[7] * ibym;
        if (lane == 0 && counted) {
          const float spanx = __fadd_rn(__fsub_rn(e.Xh, e.xh), __fsub_rn(e.Xl, e.xl));
          const float spany = __fadd_rn(__fsub_rn(e.Yh, e.yh), __fsub_rn(e.Yl, e.yl));
          wl_acc = (double)(we * ((spanx + mxp - mxm) + (spany + myp - mym)));
        }
        for (int p = lane; p < d; p += 32) {
          const int raw = __ldg(cell + p);
          if (raw < 0) continue;
          const float4 v = big_pin(a, raw, s0 + p);
          const float lxp = __fadd_rn(__fsub_rn(v.x, e.Xh), __fsub_rn(v.y, e.Xl));
          const float lxm = __fadd_rn(__fsub_rn(v.x, e.xh), __fsub_rn(v.y, e.xl));
          const float lyp = __fadd_rn(__fsub_rn(v.z, e.Yh), __fsub_rn(v.w, e.Yl));
          const float lym = __fadd_rn(__fsub_rn(v.z, e.yh), __fsub_rn(v.w, e.yl));
          const float axp = ex2(lxp * a.k2), axm = ex2(-lxm * a.k2);
          const float ayp = ex2(lyp * a.k2), aym = ex2(-lym * a.k2);
          const float gx = we * (axp * ibxp * (1.f + (lxp - mxp) * a.inv_gamma) -
                                 axm * ibxm * (1.f - (lxm - mxm) * a.inv_gamma));
          const float gy = we * (ayp * ibyp * (1.f + (lyp - myp) * a.inv_gamma) -
                                 aym * ibym * (1.f - (lym - mym) * a.inv_gamma));
          grad_out(a, raw, gx, gy);
        }
      }
    }
  }
  const int slot = a.part_base + a.unit0 + blockIdx.x;
  block_flush_scalars<kWarpNetThreads>(wl_acc, L, kHpwl, kGrad ? a.part + slot : nullptr, a.limbs, hp_w,
                                       MODE == 4 ? a.part + a.hp_offset + slot : nullptr);
}

// MODE 0: WA + gradient; 1: WA + gradient + HPWL; 2: HPWL only; 3: LSE + gradient (NEXT-3);
// 4: WA + gradient + fast HPWL (fp32 pin positions, per-CTA partials; the GP loop, reading A37).
template <int MODE>
// at least 2 CTAs per SM (4096-pin chunks: shared memory allows 2; the register cap of 3 per SM
// measured 0.5 % slower, 4 per SM at 64 registers slower still)
__global__ void __launch_bounds__(kWaThreads, 2) k_wa_chunks(const WaArgs a0) {
  WaArgs a = a0;
  if (a.gamma_dev) {   // uniform branch: the GP loop's gamma lives on the device
    const float g = __ldg(a.gamma_dev);
    a.gamma = g;
    a.inv_gamma = 1.f / g;
    a.k2 = kLog2e / g;
  }
  constexpr bool kGrad = MODE != 2;
  constexpr bool kHpwl = MODE == 1 || MODE == 2;
  extern __shared__ __align__(16) unsigned char smem[];
  const WaSmem L_{a.caps};
  int *s_slot = reinterpret_cast<int *>(smem + L_.off_slot());
  float *s_dx = reinterpret_cast<float *>(smem + L_.off_dx());
  float *s_dy = reinterpret_cast<float *>(smem + L_.off_dy());
  int *s_deg = reinterpret_cast<int *>(smem + L_.off_deg());
  float *s_w = reinterpret_cast<float *>(smem + L_.off_w());
  WarpGroup *s_wg = reinterpret_cast<WarpGroup *>(smem + L_.off_wg());
  int *s_far = reinterpret_cast<int *>(smem + L_.off_far());
  float *s_px = reinterpret_cast<float *>(smem + L_.off_px());
  float *s_py = reinterpret_cast<float *>(smem + L_.off_py());
  int *s_g = reinterpret_cast<int *>(smem + L_.off_g());
  uint64_t *bar = reinterpret_cast<uint64_t *>(smem + L_.off_bar());

  // one launch for all nets: CTAs [0, n_huge) take a net of degree > kWarpNetMax each, the next
  // n_warp_blocks CTAs 8 nets of degree (kWaMaxDeg, kWarpNetMax] each (a warp per net), the rest
  // the staged chunks; the long big-net CTAs are dispatched first and overlap the chunks.
  const int unit = a.unit0 + blockIdx.x;
  if (unit < a.n_huge) {
    wa_big_net<MODE>(a, unit, reinterpret_cast<float4 *>(smem));
    return;
  }
  if (unit < a.n_huge + a.n_warp_blocks) {
    wa_warp_nets<MODE>(a, unit - a.n_huge);
    return;
  }
  const int chunk = unit - a.n_huge - a.n_warp_blocks;
  const Chunk ch = a.chunks[chunk];
  const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
  // window positions by bulk copy when 16-byte aligned (the caller's x / y), else by threads
  const int wbulk = ch.win_n & ~3;
  const bool win_bulk = ((((uintptr_t)(a.x + ch.win_lo)) | ((uintptr_t)(a.y + ch.win_lo))) & 15) == 0 && wbulk > 0;
  // two barriers: bar[0] = the far-cell list (small, issued first: the far-position gather
  // starts while the pin records are still in flight), bar[1] = everything else
  if (tid == 0) {
    mbar_init(bar);
    mbar_init(bar + 1);
    mbar_expect_tx(bar, 4u * ch.far_pad);
    if (ch.far_pad) bulk_g2s(s_far, a.far_cells + ch.far_begin, 4u * ch.far_pad, bar);
    const unsigned tx = 12u * ch.pin_n + (a.has_w ? 8u : 4u) * ch.net_n + 16u * ch.wg_n + (win_bulk ? 8u * wbulk : 0u);
    mbar_expect_tx(bar + 1, tx);
    // the chunk's netlist data is read once per evaluation: streamed with an evict-first L2 policy
    const uint64_t pol = a.stream_hint ? l2_evict_first_policy() : 0;
    auto copy = [&](void *dst, const void *src, unsigned bytes) {
      if (a.stream_hint)
        bulk_g2s_hint(dst, src, bytes, bar + 1, pol);
      else
        bulk_g2s(dst, src, bytes, bar + 1);
    };
    if (ch.pin_n) {
      copy(s_slot, a.pin_slot + ch.pin_begin, 4u * ch.pin_n);
      copy(s_dx, a.pin_dx + ch.pin_begin, 4u * ch.pin_n);
      copy(s_dy, a.pin_dy + ch.pin_begin, 4u * ch.pin_n);
    }
    if (ch.net_n) {
      copy(s_deg, a.net_deg + ch.net_begin, 4u * ch.net_n);
      if (a.has_w) copy(s_w, a.net_w + ch.net_begin, 4u * ch.net_n);
    }
    if (ch.wg_n) copy(s_wg, a.wgs + ch.wg_begin, 16u * ch.wg_n);
    if (win_bulk) {
      bulk_g2s(s_px, a.x + ch.win_lo, 4u * wbulk, bar + 1);
      bulk_g2s(s_py, a.y + ch.win_lo, 4u * wbulk, bar + 1);
    }
  }
  const int nslots = L_.slots();
  if (kGrad)   // 2 * nslots is a multiple of 8, s_g 16-byte aligned
    for (int i = tid; i < nslots / 2; i += kWaThreads) reinterpret_cast<int4 *>(s_g)[i] = make_int4(0, 0, 0, 0);
  for (int i = (win_bulk ? wbulk : 0) + tid; i < ch.win_n; i += kWaThreads) {
    s_px[i] = __ldg(a.x + ch.win_lo + i);
    s_py[i] = __ldg(a.y + ch.win_lo + i);
  }
  __syncthreads();   // barrier initialised before anyone waits on it
  mbar_wait(bar, 0);
  // far cells: positions gathered once per chunk
#ifndef DP_WA_FAR_LDG
  // 4-byte cp.async global -> shared (no register round trip), completed before the barrier
  // (the register path below, -DDP_WA_FAR_LDG: 5047-5055 vs 5064-5065 evals/s)
  for (int f = tid; f < ch.far_n; f += kWaThreads) {
    const int c = s_far[f];
    asm volatile("cp.async.ca.shared.global [%0], [%1], 4;" ::"r"(smem_u32(s_px + kWaWindow + f)), "l"(a.x + c) : "memory");
    asm volatile("cp.async.ca.shared.global [%0], [%1], 4;" ::"r"(smem_u32(s_py + kWaWindow + f)), "l"(a.y + c) : "memory");
  }
  asm volatile("cp.async.wait_all;" ::: "memory");
#else
  for (int f0 = tid; f0 < ch.far_n; f0 += 4 * kWaThreads) {   // 8 loads in flight per thread
    float fx[4], fy[4];
#pragma unroll
    for (int k = 0; k < 4; k++) {
      const int f = f0 + k * kWaThreads;
      const int c = f < ch.far_n ? s_far[f] : 0;
      fx[k] = __ldg(a.x + c);
      fy[k] = __ldg(a.y + c);
    }
#pragma unroll
    for (int k = 0; k < 4; k++) {
      const int f = f0 + k * kWaThreads;
      if (f < ch.far_n) {
        s_px[kWaWindow + f] = fx[k];
        s_py[kWaWindow + f] = fy[k];
      }
    }
  }
#endif
  mbar_wait(bar + 1, 0);
  __syncthreads();

  float wl_acc = 0.f, hp_acc = 0.f;
  unsigned long long L[kHpwlLimbs + 1];
#pragma unroll
  for (int k = 0; k <= kHpwlLimbs; k++) L[k] = 0ull;
  const GroupCtx gc{s_slot, s_dx, s_dy, s_deg, s_w, s_px, s_py, s_g, nslots - 1, exp2f((float)ch.scale_log2),
                    lane, (1u << lane) - 1u};

  // warp groups are dealt round-robin (the host orders them by decreasing cost)
  for (int gi = warp; gi < ch.wg_n; gi += kWaThreads / 32) {
    const WarpGroup wg = s_wg[gi];
    if (MODE == 0 || MODE == 3 || MODE == 4) {
      constexpr bool kL = MODE == 3, kH = MODE == 4;
      if (wg.flags & 1) {
        wa_group_pairs<kL, kH, false>(a, wg, gc, wl_acc, hp_acc, L);
      } else {
        wa_group_fast_dispatch<kL, kH>(a, wg, gc, wl_acc, hp_acc);
      }
    } else {
      if (MODE == 1 && (wg.flags & 1)) {   // 2-pin nets: closed-form WA + exact HPWL
        wa_group_pairs<false, false, true>(a, wg, gc, wl_acc, hp_acc, L);
        continue;
      }
      switch (wg.slots) {
        case 1: wa_group_exact<MODE, 1>(a, wg, gc, wl_acc, L); break;
        case 2: wa_group_exact<MODE, 2>(a, wg, gc, wl_acc, L); break;
        case 3: wa_group_exact<MODE, 3>(a, wg, gc, wl_acc, L); break;
        default: wa_group_exact<MODE, 4>(a, wg, gc, wl_acc, L); break;
      }
    }
  }
  __syncthreads();
  if (kGrad && a.g2i) {   // deterministic flush: exact int32 -> int64 conversion, integer reds
    const int sh = a.det_frac - ch.scale_log2;
    for (int w = tid; w < ch.win_n; w += kWaThreads) {
      const int gx = s_g[2 * w], gy = s_g[2 * w + 1];
      if (gx) red_s64(a.g2i + 2 * (ch.win_lo + w), to_det(gx, sh));
      if (gy) red_s64(a.g2i + 2 * (ch.win_lo + w) + 1, to_det(gy, sh));
    }
    for (int f = tid; f < ch.far_n; f += kWaThreads) {
      const int gx = s_g[2 * (kWaWindow + f)], gy = s_g[2 * (kWaWindow + f) + 1];
      if (gx) red_s64(a.g2i + 2 * s_far[f], to_det(gx, sh));
      if (gy) red_s64(a.g2i + 2 * s_far[f] + 1, to_det(gy, sh));
    }
  } else if (kGrad && a.gxo) {   // direct output: 4-cell vector reds into gx and gy (win_lo % 4 == 0)
    const float inv = exp2f(-(float)ch.scale_log2);
    const int nq = ch.win_n >> 2;
    const int4 *s4 = reinterpret_cast<const int4 *>(s_g);
    for (int q = tid; q < nq; q += kWaThreads) {
      const int4 v0 = s4[2 * q], v1 = s4[2 * q + 1];   // x0 y0 x1 y1 | x2 y2 x3 y3
      const int c0 = ch.win_lo + 4 * q;
      if (v0.x | v0.z | v1.x | v1.z)
        red_v4(reinterpret_cast<float4 *>(a.gxo + c0), v0.x * inv, v0.z * inv, v1.x * inv, v1.z * inv);
      if (v0.y | v0.w | v1.y | v1.w)
        red_v4(reinterpret_cast<float4 *>(a.gyo + c0), v0.y * inv, v0.w * inv, v1.y * inv, v1.w * inv);
    }
    for (int w = 4 * nq + tid; w < ch.win_n; w += kWaThreads) {
      if (s_g[2 * w]) red_f1(a.gxo + ch.win_lo + w, s_g[2 * w] * inv);
      if (s_g[2 * w + 1]) red_f1(a.gyo + ch.win_lo + w, s_g[2 * w + 1] * inv);
    }
    for (int f = tid; f < ch.far_n; f += kWaThreads) {
      const int gx = s_g[2 * (kWaWindow + f)], gy = s_g[2 * (kWaWindow + f) + 1];
      if (gx) red_f1(a.gxo + s_far[f], gx * inv);
      if (gy) red_f1(a.gyo + s_far[f], gy * inv);
    }
  } else if (kGrad) {
    const float inv = exp2f(-(float)ch.scale_log2);
    // window: cells [win_lo, win_lo + win_n), win_lo a multiple of 4 -> 16-byte vector reductions
    float4 *g4 = reinterpret_cast<float4 *>(a.g2 + ch.win_lo);
    const int npair = ch.win_n >> 1;
    for (int i = tid; i < npair; i += kWaThreads) {
      const int4 v = *reinterpret_cast<const int4 *>(s_g + 4 * i);
      if (v.x | v.y | v.z | v.w) red_v4(g4 + i, v.x * inv, v.y * inv, v.z * inv, v.w * inv);
    }
    if ((ch.win_n & 1) && tid == 0) {
      const int w = ch.win_n - 1;
      if (s_g[2 * w] | s_g[2 * w + 1]) red_v2(a.g2 + ch.win_lo + w, s_g[2 * w] * inv, s_g[2 * w + 1] * inv);
    }
    for (int f = tid; f < ch.far_n; f += kWaThreads) {
      const int gx = s_g[2 * (kWaWindow + f)], gy = s_g[2 * (kWaWindow + f) + 1];
      if (gx | gy) red_v2(a.g2 + s_far[f], gx * inv, gy * inv);
    }
  }
  block_flush_scalars<kWaThreads>((double)wl_acc, L, kHpwl, kGrad ? a.part + a.part_base + unit : nullptr,
                                  a.limbs, (double)hp_acc,
                                  MODE == 4 ? a.part + a.hp_offset + a.part_base + unit : nullptr);
}

template <int MODE>
void launch_mode(const Ctx &c, const WaArgs &a0, cudaStream_t s, int part) {
  const WaSmem L{a0.caps};
  const int units = c.n_chunks + a0.n_huge + a0.n_warp_blocks;
  // part 0: every unit; part 1 / 2: units [0, U_A) / [U_A, units) of a split launch (the big
  // units, then the first chunks, in part 1)
  const int ua = std::min(units, a0.n_huge + a0.n_warp_blocks + c.wa_split_chunks);
  WaArgs a = a0;
  a.unit0 = part == 2 ? ua : 0;
  const int grid = part == 0 ? units : part == 1 ? ua : units - ua;
  int bytes = L.bytes();
  // DP_WA_CTAS_PER_SM = k (measurement knob): pad the dynamic shared memory so that at most k
  // WA CTAs are resident per SM, leaving room for the concurrently running density kernels
  if (c.wa_ctas_per_sm > 0)
    bytes = std::max(bytes, std::min(kWaSmemOptIn, ((228 * 1024) / c.wa_ctas_per_sm - 4096) & ~127));
  if (grid > 0) k_wa_chunks<MODE><<<grid, kWaThreads, bytes, s>>>(a);
}

}  // namespace

int wa_smem_bytes(const WaCaps &caps) { return WaSmem{caps}.bytes(); }

cudaError_t wa_configure(const WaCaps &caps) {
  const int b = std::max(WaSmem{caps}.bytes(), kWaSmemOptIn);   // launches may pad (DP_WA_CTAS_PER_SM)
  cudaError_t e = cudaFuncSetAttribute(k_wa_chunks<0>, cudaFuncAttributeMaxDynamicSharedMemorySize, b);
  if (e != cudaSuccess) return e;
  e = cudaFuncSetAttribute(k_wa_chunks<1>, cudaFuncAttributeMaxDynamicSharedMemorySize, b);
  if (e != cudaSuccess) return e;
  e = cudaFuncSetAttribute(k_wa_chunks<3>, cudaFuncAttributeMaxDynamicSharedMemorySize, b);
  if (e != cudaSuccess) return e;
  e = cudaFuncSetAttribute(k_wa_chunks<4>, cudaFuncAttributeMaxDynamicSharedMemorySize, b);
  if (e != cudaSuccess) return e;
  return cudaFuncSetAttribute(k_wa_chunks<2>, cudaFuncAttributeMaxDynamicSharedMemorySize, b);
}

void launch_wa(const Ctx &c, const float *x, const float *y, float gamma, bool hpwl_only, bool with_hpwl,
               cudaStream_t s, int part) {
  WaArgs a;
  a.unit0 = 0;
  a.chunks = c.d_chunks;
  a.wgs = c.d_wgroups;
  a.net_deg = c.d_net_deg;
  a.net_w = c.d_net_w;
  a.pin_slot = c.d_pin_cell;
  a.pin_dx = c.d_pin_dx;
  a.pin_dy = c.d_pin_dy;
  a.far_cells = c.d_far_cells;
  a.x = x;
  a.y = y;
  a.g2 = c.d_g2;
  a.g2i = c.deterministic ? c.d_g2i : nullptr;
  a.gxo = c.direct_gx;
  a.gyo = c.direct_gy;
  a.det_frac = c.det_frac;
  a.gamma = gamma;
  a.gamma_dev = c.gamma_dev;
  a.inv_gamma = 1.f / gamma;
  a.k2 = kLog2e / gamma;
  a.part = c.d_part;
  a.limbs = c.d_limbs;
  a.has_w = c.has_weights ? 1 : 0;
  a.stream_hint = c.l2_hint ? 1 : 0;
  a.big_start = c.d_big_start;
  a.big_flags = c.d_big_flags;
  a.big_cell = c.d_big_cell;
  a.big_w = c.d_big_w;
  a.big_dx = c.d_big_dx;
  a.big_dy = c.d_big_dy;
  a.part_base = c.part_base;
  a.hp_offset = c.n_wa_part + c.n_en_slots() + 1;
  a.n_huge = c.n_huge;
  a.n_big = c.n_big;
  a.n_warp_blocks = (c.n_big - c.n_huge + kWarpNetThreads / 32 - 1) / (kWarpNetThreads / 32);
  // big-net pins staged in the chunk kernel's dynamic shared memory (larger nets reload)
  a.big_stage = std::min(c.big_stage, wa_smem_bytes(c.wa_caps) / 16);
  a.caps = c.wa_caps;
  if (hpwl_only) {
    launch_mode<2>(c, a, s, part);
  } else if (c.wl_model == DP_WL_LSE) {   // LSE: fast path; a fused HPWL is a second, HPWL-only pass
    launch_mode<3>(c, a, s, part);
    if (with_hpwl) launch_mode<2>(c, a, s, part);
  } else if (with_hpwl && c.hpwl_fast && c.wl_model == DP_WL_WA) {   // GP loop: fast HPWL in the fast path
    launch_mode<4>(c, a, s, part);
  } else if (with_hpwl) {
    launch_mode<1>(c, a, s, part);
  } else {
    launch_mode<0>(c, a, s, part);
  }
}

}  // namespace dp
