// dct.cu — DCT / IDCT / IDXST transforms and the spectral Poisson solve on sm_100a.
//
// Method: potential and field by eqs (5a)-(5d) computed as the
// separable transforms of eqs (9a)-(9d) built from the 1-D DCT of eq (7a),
// IDCT of eq (7b) and IDXST of eq (8a)/(8e); N-point FFT evaluation in the
// spirit of Alg 3 (Makhoul [32]).  Readings: A12 (wavenumbers k = pi u / W),
// A13 (2/N per axis), A14 (half weight of the u = 0 term), A15 (DC term dropped),
// A16/A17 (the garbled eqs 11/12 are not used: every transform here is checked against the
// naive eq 7/8 definitions), A20 (1-D ops along y = the contiguous axis first).
//
// B200 design: the three transforms of a density evaluation are three
// kernels over maps that stay L2-resident:
//   T1  rows:     DCT over y of rho                                   -> t
//   T2  columns:  DCT over x of t, spectral scaling, Parseval energy, and BOTH inverse
//                 column transforms (IDXST_x of a k_u/k^2, IDCT_x of a k_v/k^2)  -> sX, sY
//   T3  rows:     IDCT_y of sX and IDXST_y of sY, written interleaved (xi_X, xi_Y)
// Two real sequences always share one complex FFT (z = p + i q).  The FFT is a shared-memory
// radix-2 DIT with bit-reversed loads and fp32 twiddles computed in fp64 at create.
// The energy D = 1/2 b_x b_y sum rho psi is taken in the spectral domain (Parseval), so psi
// is never materialised on the hot path (reading A8).
#include <type_traits>

#include "async_copy.cuh"
#include "dp_internal.h"
#include "fft_warp.cuh"

namespace dp {

namespace {

constexpr int kRowThreads = 256;
constexpr int kColThreads = 256;
// columns per CTA in the column kernels (even: pairs share a complex FFT); sized so the
// shared-memory slab fits and the grid has >= 256 CTAs at 1024 columns
__host__ __device__ inline int col_slab(int mx) { (void)mx; return 2; }

__device__ __forceinline__ float2 cmul(float2 a, float2 b) {
  return make_float2(a.x * b.x - a.y * b.y, a.x * b.y + a.y * b.x);
}
__device__ __forceinline__ int brev(int n, int log2n) { return (int)(__brev((unsigned)n) >> (32 - log2n)); }
// Makhoul reordering (Alg 3 lines 3-8): v[n] = x[2n], v[N-1-n] = x[2n+1]; position of x[t] in v
__device__ __forceinline__ int mk_pos(int t, int n) { return (t & 1) ? n - ((t + 1) >> 1) : (t >> 1); }

// In-place DIT FFT of nseq sequences of length n = 2^log2n stored back to back in buf, input
// already in bit-reversed order.  tw[k] = exp(-2 pi i k / n), k < n/2.  inverse = true uses
// conjugate twiddles (unnormalised inverse DFT).  Two radix-2 levels are fused per shared-
// memory round trip (a radix-4 step on {i, i+h, i+2h, i+3h}), so a 1024-point transform takes
// 5 barriers instead of 10.
__device__ void fft_block(float2 *buf, int n, int log2n, int nseq, const float2 *__restrict__ tw,
                          bool inverse) {
  const int quarter_n = n >> 2, lq = log2n - 2;
  const int total4 = nseq * quarter_n;
  int s = 1;
  for (; s + 1 <= log2n; s += 2) {
    const int h = 1 << (s - 1), lh = s - 1;
    const int st1 = n >> s, st2 = n >> (s + 1);   // twiddle strides of W_{2h} and W_{4h}
    for (int q = threadIdx.x; q < total4; q += blockDim.x) {
      const int seq = q >> lq, r = q & (quarter_n - 1);
      const int blk = r >> lh, k = r & (h - 1);
      const int base = seq * n + (blk << (lh + 2)) + k;
      float2 w1 = __ldg(tw + k * st1), w2 = __ldg(tw + k * st2);
      if (inverse) {
        w1.y = -w1.y;
        w2.y = -w2.y;
      }
      // W_{4h}^{k+h} = W_{4h}^k * (-i) forward, (+i) inverse
      const float2 w3 = inverse ? make_float2(-w2.y, w2.x) : make_float2(w2.y, -w2.x);
      const float2 a0 = buf[base], a1 = buf[base + h], a2 = buf[base + 2 * h], a3 = buf[base + 3 * h];
      const float2 t1 = cmul(w1, a1), t3 = cmul(w1, a3);
      const float2 b0 = make_float2(a0.x + t1.x, a0.y + t1.y), b1 = make_float2(a0.x - t1.x, a0.y - t1.y);
      const float2 b2 = make_float2(a2.x + t3.x, a2.y + t3.y), b3 = make_float2(a2.x - t3.x, a2.y - t3.y);
      const float2 u2 = cmul(w2, b2), u3 = cmul(w3, b3);
      buf[base] = make_float2(b0.x + u2.x, b0.y + u2.y);
      buf[base + 2 * h] = make_float2(b0.x - u2.x, b0.y - u2.y);
      buf[base + h] = make_float2(b1.x + u3.x, b1.y + u3.y);
      buf[base + 3 * h] = make_float2(b1.x - u3.x, b1.y - u3.y);
    }
    __syncthreads();
  }
  if (s == log2n) {  // odd log2n: one last radix-2 level
    const int half = 1 << (s - 1), half_n = n >> 1, total = nseq * half_n;
    for (int b = threadIdx.x; b < total; b += blockDim.x) {
      const int seq = b >> (log2n - 1), r = b & (half_n - 1);
      const int k = r;  // one group: grp = 0, len = n
      const int i = seq * n + k, jx = i + half;
      float2 w = __ldg(tw + k);
      if (inverse) w.y = -w.y;
      const float2 u = buf[i], v = cmul(w, buf[jx]);
      buf[i] = make_float2(u.x + v.x, u.y + v.y);
      buf[jx] = make_float2(u.x - v.x, u.y - v.y);
    }
    __syncthreads();
  }
}

// Forward DCT post-processing for a pair packed as z = p + i q (Alg 3 lines 10-16, split
// of the two real spectra): returns (DCT(p)_k, DCT(q)_k) with the 2/N factor (reading A13).
__device__ __forceinline__ float2 dct_post(const float2 *Z, int k, int n, float2 ph, float scale) {
  const float2 z = Z[k], zc = Z[(n - k) & (n - 1)];
  // V0 = (z + conj zc)/2, V1 = (z - conj zc) * (-i/2)
  const float v0x = 0.5f * (z.x + zc.x), v0y = 0.5f * (z.y - zc.y);
  const float dx = z.x - zc.x, dy = z.y + zc.y;
  const float v1x = 0.5f * dy, v1y = -0.5f * dx;
  // Re(V e^{-i pi k / 2N}), ph = (cos, -sin)
  return make_float2(scale * (v0x * ph.x - v0y * ph.y), scale * (v1x * ph.x - v1y * ph.y));
}

// Inverse pre-processing for two IDCT-type sequences p (real part) and q (imag part), both
// already reversed if they are IDXST inputs (eq 8e):  Z_k = e^{+i pi k/2N} [(p_k + q_{N-k})
// + i (q_k - p_{N-k})] with p_N = q_N = 0.  ph = e^{-i pi k/2N} (conjugated here).
__device__ __forceinline__ float2 inv_pre(float pk, float qk, float pnk, float qnk, float2 ph) {
  const float re = pk + qnk, im = qk - pnk;
  return make_float2(re * ph.x + im * ph.y, im * ph.x - re * ph.y);
}

// ---------------------------------------------------------------------------------------
// T1 / debug: forward DCT over rows, rows (2r, 2r+1) share one complex FFT.
// ---------------------------------------------------------------------------------------
// IN = float, or unsigned long long = int64 fixed point in 2^-kRhoScaleLog2 units (the bin map)
__device__ __forceinline__ float load_map(const float *p) { return __ldg(p); }
__device__ __forceinline__ float load_map(const unsigned long long *p) {
  return (float)((double)(long long)__ldg(p) * (1.0 / (double)(1ll << kRhoScaleLog2)));
}

__device__ __forceinline__ float smem_map(const float *p) { return *p; }
__device__ __forceinline__ float smem_map(const unsigned long long *p) {
  return (float)((double)(long long)*p * (1.0 / (double)(1ll << kRhoScaleLog2)));
}

template <class IN>
__global__ void __launch_bounds__(kRowThreads) k_row_dct(const IN *__restrict__ in, float *__restrict__ out,
                                                         int n, int log2n, const float2 *__restrict__ tw,
                                                         const float2 *__restrict__ ph) {
  extern __shared__ float2 zbuf[];
  const IN *r0 = in + (size_t)(2 * blockIdx.x) * n, *r1 = r0 + n;
  for (int t = threadIdx.x; t < n; t += kRowThreads)
    zbuf[brev(mk_pos(t, n), log2n)] = make_float2(load_map(r0 + t), load_map(r1 + t));
  __syncthreads();
  fft_block(zbuf, n, log2n, 1, tw, false);
  float *o0 = out + (size_t)(2 * blockIdx.x) * n, *o1 = o0 + n;
  const float scale = 2.f / n;
  for (int k = threadIdx.x; k < n; k += kRowThreads) {
    const float2 v = dct_post(zbuf, k, n, __ldg(ph + k), scale);
    o0[k] = v.x;
    o1[k] = v.y;
  }
}

// ---------------------------------------------------------------------------------------
// T3 / debug: inverse over rows.  Row r of A (op opA) and row r of B (op opB) share one
// complex IFFT.  op: 1 = IDCT (eq 7b), 2 = IDXST (eq 8a via 8e).  Output either two planes
// or one interleaved float2 plane (xi_X, xi_Y).
// ---------------------------------------------------------------------------------------
struct RowInvArgs {
  const float *inA, *inB;
  long long stepA, stepB;   // row r of A at inA + r * stepA
  int opA, opB;
  float *outA, *outB;       // planes (row step n), used if outI == nullptr
  long long ostepA, ostepB;
  float2 *outI;             // interleaved output (row step n)
  const float2 *inI;        // if set: interleaved input (A, B) with row step n (warp kernel only)
  long long ostepT;         // if > 0 (warp kernel): outI[t * ostepT + r] (transposed store)
  int tma;                  // interleaved input by bulk copy (DP_ROW_TMA=0: per-lane loads, A/B)
  int n, log2n;
  const float2 *tw, *ph;
};

__global__ void __launch_bounds__(kRowThreads) k_row_inv(RowInvArgs a) {
  extern __shared__ float2 zbuf[];
  const int n = a.n;
  float *p = reinterpret_cast<float *>(zbuf + n);
  float *q = p + n;
  const float *ra = a.inA + (long long)blockIdx.x * a.stepA;
  const float *rb = a.inB + (long long)blockIdx.x * a.stepB;
  for (int t = threadIdx.x; t < n; t += kRowThreads) {
    // IDXST input reversal (eq 8e): x'_t = x_{N-t}, x'_0 = 0
    p[t] = (a.opA == 2) ? (t ? __ldg(ra + n - t) : 0.f) : __ldg(ra + t);
    q[t] = (a.opB == 2) ? (t ? __ldg(rb + n - t) : 0.f) : __ldg(rb + t);
  }
  __syncthreads();
  for (int k = threadIdx.x; k < n; k += kRowThreads) {
    const float pnk = k ? p[n - k] : 0.f, qnk = k ? q[n - k] : 0.f;
    zbuf[brev(k, a.log2n)] = inv_pre(p[k], q[k], pnk, qnk, __ldg(a.ph + k));
  }
  __syncthreads();
  fft_block(zbuf, n, a.log2n, 1, a.tw, true);
  for (int t = threadIdx.x; t < n; t += kRowThreads) {
    const float2 v = zbuf[mk_pos(t, n)];
    float va = 0.5f * v.x, vb = 0.5f * v.y;
    if (t & 1) {
      if (a.opA == 2) va = -va;
      if (a.opB == 2) vb = -vb;
    }
    if (a.outI) {
      a.outI[(size_t)blockIdx.x * n + t] = make_float2(va, vb);
    } else {
      a.outA[(long long)blockIdx.x * a.ostepA + t] = va;
      a.outB[(long long)blockIdx.x * a.ostepB + t] = vb;
    }
  }
}

// ---------------------------------------------------------------------------------------
// Warp-FFT row kernels (N = 2^LOGN in [32, 1024]); every warp owns B = 1024 / N row pairs (T1)
// or rows (T3) and never waits on a block barrier.
// ---------------------------------------------------------------------------------------
constexpr int kWRowWarps = 2;   // warps per CTA: a 1024-row map gives 256-512 CTAs
constexpr int kTStoreWarps = 4; // T2b (transposed output): 4 adjacent columns -> 32-byte row segments

// 1/x to ~1 ulp on the MUFU (the IEEE __frcp_rn slow path stalled the column pass)
__device__ __forceinline__ float fast_rcp(float x) {
  float r;
  asm("rcp.approx.f32 %0, %1;" : "=f"(r) : "f"(x));
  return r;
}

// dct_post on values already loaded: z = Z[k], zc = Z[N - k]
__device__ __forceinline__ float2 dct_post_v(float2 z, float2 zc, float2 ph, float scale) {
  const float v0x = 0.5f * (z.x + zc.x), v0y = 0.5f * (z.y - zc.y);
  const float dx = z.x - zc.x, dy = z.y + zc.y;
  const float v1x = 0.5f * dy, v1y = -0.5f * dx;
  return make_float2(scale * (v0x * ph.x - v0y * ph.y), scale * (v1x * ph.x - v1y * ph.y));
}

// T1: rows (2p, 2p+1) packed as one complex sequence (Makhoul order), DCT over y
template <class IN, int LOGN>
__global__ void __launch_bounds__(32 * kWRowWarps) k_row_dct_w(const IN *__restrict__ in, float *__restrict__ out,
                                                             const float2 *__restrict__ tw2,
                                                             const float2 *__restrict__ ph, int npairs, int tma) {
  griddep_wait();
  constexpr int N = 1 << LOGN, K = N / 32, B = wfft::kPts / N;
  extern __shared__ float2 wsm[];
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  float2 *buf = wsm + warp * wfft::kBufPad;
  const int p0 = (blockIdx.x * kWRowWarps + warp) * B;
  if (p0 >= npairs) return;
  // the warp's B row pairs (contiguous: rows 2 p0 .. 2 (p0 + B) - 1) land in its staging area by
  // one bulk copy (the TMA queue keeps the whole transfer in flight; per-lane loads were
  // limited by outstanding misses per SM)
  IN *stage = reinterpret_cast<IN *>(wsm + kWRowWarps * wfft::kBufPad) + (size_t)warp * 2 * wfft::kPts;
  __shared__ uint64_t s_bar[kWRowWarps];
  const int nvalid = min(B, npairs - p0);
  if (tma && lane == 0) {
    mbar_init(&s_bar[warp]);
    const unsigned bytes = (unsigned)(2 * N * nvalid * sizeof(IN));
    mbar_expect_tx(&s_bar[warp], bytes);
    bulk_g2s(stage, in + (size_t)(2 * p0) * N, bytes, &s_bar[warp]);
  }
  // twiddle / phase tables are read right before use (L1-resident; registers kept low)
  float2 a[32];
  if (tma) {
    __syncwarp();
    mbar_wait(&s_bar[warp], 0);
#pragma unroll
    for (int s = 0; s < B; s++) {
      const bool ok = s < nvalid;
      const IN *r0 = stage + (size_t)(2 * s) * N, *r1 = r0 + N;
#pragma unroll
      for (int j = 0; j < K; j++) {
        const int n = lane + 32 * j;
        const int src = n < N / 2 ? 2 * n : 2 * (N - 1 - n) + 1;   // v[n] = x[2n], v[N-1-n] = x[2n+1]
        a[s * K + j] = ok ? make_float2(smem_map(r0 + src), smem_map(r1 + src)) : make_float2(0.f, 0.f);
      }
    }
  } else {
#pragma unroll
    for (int s = 0; s < B; s++) {
      const bool ok = s < nvalid;
      const IN *r0 = in + (size_t)(2 * (p0 + s)) * N, *r1 = r0 + N;
#pragma unroll
      for (int j = 0; j < K; j++) {
        const int n = lane + 32 * j;
        const int src = n < N / 2 ? 2 * n : 2 * (N - 1 - n) + 1;
        a[s * K + j] = ok ? make_float2(load_map(r0 + src), load_map(r1 + src)) : make_float2(0.f, 0.f);
      }
    }
  }
  wfft::warp_fft<LOGN, false>(a, buf, tw2);
  const float scale = 2.f / N;
#pragma unroll
  for (int s = 0; s < B; s++) {
    if (p0 + s >= npairs) break;
    float *o0 = out + (size_t)(2 * (p0 + s)) * N, *o1 = o0 + N;
#pragma unroll
    for (int j = 0; j < K; j++) {
      const int k = lane + 32 * j;
      const float2 v = dct_post_v(buf[wfft::pad(s * N + k)], buf[wfft::pad(s * N + ((N - k) & (N - 1)))],
                                  __ldg(ph + k), scale);
      o0[k] = v.x;
      o1[k] = v.y;
    }
  }
}

// T3 / debug: row r of A (op opA) and row r of B (op opB) as one complex inverse sequence
// TSTORE (T2b, transposed output outI[t * ostepT + r]): the CTA's WARPS * B consecutive rows r
// are written together after a block barrier, WARPS * B adjacent float2 per output row (full
// 32-byte sectors at WARPS = 4), instead of one 8-byte store per lane and row.
template <int LOGN, int WARPS = kWRowWarps, bool TSTORE = false>
__global__ void __launch_bounds__(32 * WARPS) k_row_inv_w(RowInvArgs a, const float2 *__restrict__ tw2, int rows) {
  griddep_wait();
  constexpr int N = 1 << LOGN, K = N / 32, B = wfft::kPts / N;
  extern __shared__ float2 wsm[];
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  float2 *buf = wsm + warp * wfft::kBufPad;
  const int r0 = (blockIdx.x * WARPS + warp) * B;
  if (!TSTORE && r0 >= rows) return;   // TSTORE: idle warps still reach the block barrier
  // interleaved input: the warp's B rows (contiguous) land in its buffer by one bulk copy;
  // planar input (debug transforms): per-lane loads, staged through the buffer.  Either way each
  // row is read once and the mirrored element N - k comes from the buffer.
  __shared__ uint64_t s_bar[WARPS];
  const int nvalid = max(0, min(B, rows - r0));
  if (a.inI && a.tma && lane == 0 && nvalid > 0) {
    mbar_init(&s_bar[warp]);
    const unsigned bytes = (unsigned)(N * nvalid * sizeof(float2));
    mbar_expect_tx(&s_bar[warp], bytes);
    bulk_g2s(buf, a.inI + (size_t)r0 * N, bytes, &s_bar[warp]);
  }
  // twiddle / phase tables are read right before use (L1-resident; registers kept low)
  float2 v[32];
  if (a.inI && a.tma) {
    __syncwarp();
    if (nvalid > 0) mbar_wait(&s_bar[warp], 0);
#pragma unroll
    for (int s = 0; s < B; s++)
#pragma unroll
      for (int j = 0; j < K; j++) v[s * K + j] = s < nvalid ? buf[s * N + lane + 32 * j] : make_float2(0.f, 0.f);
  } else {
#pragma unroll
    for (int s = 0; s < B; s++) {
      const bool ok = s < nvalid;
      const float *ra = a.inA + (long long)(r0 + s) * a.stepA, *rb = a.inB + (long long)(r0 + s) * a.stepB;
      const float2 *ri = a.inI ? a.inI + (size_t)(r0 + s) * N : nullptr;
#pragma unroll
      for (int j = 0; j < K; j++) {
        const int k = lane + 32 * j;
        v[s * K + j] = !ok ? make_float2(0.f, 0.f) : ri ? __ldg(ri + k) : make_float2(__ldg(ra + k), __ldg(rb + k));
      }
    }
#pragma unroll
    for (int q = 0; q < B * K; q++) buf[q * 32 + lane] = v[q];
    __syncwarp();
  }
#pragma unroll
  for (int s = 0; s < B; s++) {
#pragma unroll
    for (int j = 0; j < K; j++) {
      const int k = lane + 32 * j;
      const float2 vk = v[s * K + j];
      const float2 vn = k ? buf[s * N + N - k] : make_float2(0.f, 0.f);
      // IDXST input reversal (eq 8e): x'_t = x_{N-t}, x'_0 = 0
      const float pk = (a.opA == 2) ? vn.x : vk.x;
      const float pnk = k ? ((a.opA == 2) ? vk.x : vn.x) : 0.f;
      const float qk = (a.opB == 2) ? vn.y : vk.y;
      const float qnk = k ? ((a.opB == 2) ? vk.y : vn.y) : 0.f;
      v[s * K + j] = inv_pre(pk, qk, pnk, qnk, __ldg(a.ph + lane + 32 * j));
    }
  }
  __syncwarp();
  wfft::warp_fft<LOGN, true>(v, buf, tw2);
  if constexpr (TSTORE) {
    constexpr int C = WARPS * B;   // consecutive output columns of this CTA
    const int rc0 = blockIdx.x * C;
    __syncthreads();
    for (int idx = threadIdx.x; idx < N * C; idx += 32 * WARPS) {
      const int c = idx % C, t = idx / C, r = rc0 + c;
      if (r >= rows) continue;
      const float2 z = wsm[(c / B) * wfft::kBufPad + wfft::pad((c % B) * N + mk_pos(t, N))];
      float va = 0.5f * z.x, vb = 0.5f * z.y;
      if (t & 1) {
        if (a.opA == 2) va = -va;
        if (a.opB == 2) vb = -vb;
      }
      a.outI[(size_t)t * a.ostepT + r] = make_float2(va, vb);
    }
    return;
  }
#pragma unroll
  for (int s = 0; s < B; s++) {
    const int r = r0 + s;
    if (r >= rows) break;
#pragma unroll
    for (int j = 0; j < K; j++) {
      const int t = lane + 32 * j;
      const float2 z = buf[wfft::pad(s * N + mk_pos(t, N))];
      float va = 0.5f * z.x, vb = 0.5f * z.y;
      if (t & 1) {
        if (a.opA == 2) va = -va;
        if (a.opB == 2) vb = -vb;
      }
      if (a.outI) {
        if (a.ostepT > 0)
          a.outI[(size_t)t * a.ostepT + r] = make_float2(va, vb);
        else
          a.outI[(size_t)r * N + t] = make_float2(va, vb);
      } else {
        a.outA[(long long)r * a.ostepA + t] = va;
        a.outB[(long long)r * a.ostepB + t] = vb;
      }
    }
  }
}

// ---------------------------------------------------------------------------------------
// Column kernels: a CTA owns kColSlab adjacent columns (pairs share a complex FFT).
// ---------------------------------------------------------------------------------------
// Generic column transform (debug transforms): op 0 = DCT, 1 = IDCT, 2 = IDXST.
__global__ void __launch_bounds__(kColThreads) k_col_generic(const float *__restrict__ in, float *__restrict__ out,
                                                             int op, int mx, int log2mx, int my,
                                                             const float2 *__restrict__ tw,
                                                             const float2 *__restrict__ ph) {
  extern __shared__ float2 zbuf[];  // [sc/2][mx] complex + [sc][mx] real
  const int kColSlab = col_slab(mx);
  float *rbuf = reinterpret_cast<float *>(zbuf + (kColSlab / 2) * mx);
  const int c0 = blockIdx.x * kColSlab;
  for (int idx = threadIdx.x; idx < mx * kColSlab; idx += kColThreads) {
    const int row = idx / kColSlab, col = idx % kColSlab;
    rbuf[col * mx + row] = __ldg(in + (size_t)row * my + c0 + col);
  }
  __syncthreads();
  if (op == 0) {
    for (int idx = threadIdx.x; idx < mx * (kColSlab / 2); idx += kColThreads) {
      const int pr = idx >> log2mx, t = idx & (mx - 1);
      zbuf[pr * mx + brev(mk_pos(t, mx), log2mx)] = make_float2(rbuf[(2 * pr) * mx + t], rbuf[(2 * pr + 1) * mx + t]);
    }
  } else {
    for (int idx = threadIdx.x; idx < mx * (kColSlab / 2); idx += kColThreads) {
      const int pr = idx >> log2mx, k = idx & (mx - 1);
      const float *pp = rbuf + (2 * pr) * mx, *qq = rbuf + (2 * pr + 1) * mx;
      float pk, qk, pnk, qnk;
      if (op == 2) {  // reversed inputs x'_t = x_{N-t}
        pk = k ? pp[mx - k] : 0.f;
        qk = k ? qq[mx - k] : 0.f;
        pnk = k ? pp[k] : 0.f;
        qnk = k ? qq[k] : 0.f;
      } else {
        pk = pp[k];
        qk = qq[k];
        pnk = k ? pp[mx - k] : 0.f;
        qnk = k ? qq[mx - k] : 0.f;
      }
      zbuf[pr * mx + brev(k, log2mx)] = inv_pre(pk, qk, pnk, qnk, __ldg(ph + k));
    }
  }
  __syncthreads();
  fft_block(zbuf, mx, log2mx, kColSlab / 2, tw, op != 0);
  for (int idx = threadIdx.x; idx < mx * kColSlab; idx += kColThreads) {
    const int row = idx / kColSlab, col = idx % kColSlab, pr = col >> 1;
    float v;
    if (op == 0) {
      const float2 d = dct_post(zbuf + pr * mx, row, mx, __ldg(ph + row), 2.f / mx);
      v = (col & 1) ? d.y : d.x;
    } else {
      const float2 z = zbuf[pr * mx + mk_pos(row, mx)];
      v = 0.5f * ((col & 1) ? z.y : z.x);
      if (op == 2 && (row & 1)) v = -v;
    }
    out[(size_t)row * my + c0 + col] = v;
  }
}

// T2: fused column pass.  For each column v of t = DCT_y(rho):
//   a[u][v]   = DCT_x(t[.][v])                                  (eq 9a)
//   energy   += omega_u omega_v a^2 / (k_u^2 + k_v^2)           (Parseval form of D, A8)
//   sX[.][v]  = IDXST_x( a k_u / k^2 )                          (eq 9c, x part)
//   sY[.][v]  = IDCT_x ( a k_v / k^2 )                          (eq 9d, x part)
// with a_00 / k^2 := 0 (eq 4c, A15).  The IDXST of column v and the IDCT of column v share
// one complex IFFT.
struct ColFieldArgs {
  const float *t;
  float *sx, *sy;
  int mx, log2mx, my;
  const float2 *tw_x, *ph_x;
  const float *kx, *ky;
  double *energy_part;   // one slot per CTA
  double energy_scale;   // 1/2 b_x b_y
};

__global__ void __launch_bounds__(kColThreads) k_col_fields(ColFieldArgs a) {
  extern __shared__ float2 zbuf[];  // [sc][mx] complex; the first half doubles as the forward buffer
  const int mx = a.mx, log2mx = a.log2mx, my = a.my;
  const int kColSlab = col_slab(mx);
  float *abuf = reinterpret_cast<float *>(zbuf + kColSlab * mx);  // [kColSlab][mx] real spectrum
  __shared__ double s_red[kColThreads / 32];
  const int c0 = blockIdx.x * kColSlab;
  // load + Makhoul reorder along x, pairs of columns -> complex
  for (int idx = threadIdx.x; idx < mx * kColSlab; idx += kColThreads) {
    const int row = idx / kColSlab, col = idx % kColSlab, pr = col >> 1;
    const float v = __ldg(a.t + (size_t)row * my + c0 + col);
    float2 *slot = &zbuf[pr * mx + brev(mk_pos(row, mx), log2mx)];
    if (col & 1) slot->y = v; else slot->x = v;
  }
  __syncthreads();
  fft_block(zbuf, mx, log2mx, kColSlab / 2, a.tw_x, false);
  const float scale = 2.f / mx;
  double e = 0.0;
  // DCT_x spectrum, Parseval energy term and the spectral scaling of eqs (9c)/(9d) in one pass:
  // A_X = a k_u / k^2 -> abuf, A_Y = a k_v / k^2 -> ybuf; a_00 / k^2 := 0 (A15)
  float *ybuf = abuf + kColSlab * mx;
  for (int idx = threadIdx.x; idx < mx * (kColSlab / 2); idx += kColThreads) {
    const int pr = idx >> log2mx, u = idx & (mx - 1);
    const float2 d = dct_post(zbuf + pr * mx, u, mx, __ldg(a.ph_x + u), scale);
    const float kx = __ldg(a.kx + u);
    const double wu = (u == 0) ? 0.25 * mx : 0.5 * mx;
#pragma unroll
    for (int h = 0; h < 2; h++) {
      const int col = 2 * pr + h, v = c0 + col;
      const float ky = __ldg(a.ky + v);
      const float ik2 = (u == 0 && v == 0) ? 0.f : fast_rcp(kx * kx + ky * ky);
      const float av = h ? d.y : d.x;
      const double wv = (v == 0) ? 0.25 * my : 0.5 * my;
      e += wu * wv * (double)(av * av * ik2);
      abuf[col * mx + u] = av * kx * ik2;
      ybuf[col * mx + u] = av * ky * ik2;
    }
  }
  __syncthreads();
  // inverse pre-processing: per column, p = reversed A_X (IDXST via eq 8e), q = A_Y (IDCT)
  for (int idx = threadIdx.x; idx < mx * kColSlab; idx += kColThreads) {
    const int col = idx >> log2mx, k = idx & (mx - 1);
    const float *ax = abuf + col * mx, *ay = ybuf + col * mx;
    const float pk = k ? ax[mx - k] : 0.f;
    const float pnk = k ? ax[k] : 0.f;
    const float qk = ay[k];
    const float qnk = k ? ay[mx - k] : 0.f;
    zbuf[col * mx + brev(k, log2mx)] = inv_pre(pk, qk, pnk, qnk, __ldg(a.ph_x + k));
  }
  __syncthreads();
  fft_block(zbuf, mx, log2mx, kColSlab, a.tw_x, true);
  for (int idx = threadIdx.x; idx < mx * kColSlab; idx += kColThreads) {
    const int row = idx / kColSlab, col = idx % kColSlab;
    const float2 z = zbuf[col * mx + mk_pos(row, mx)];
    const float vx = (row & 1) ? -0.5f * z.x : 0.5f * z.x;  // IDXST sign (-1)^x
    a.sx[(size_t)row * my + c0 + col] = vx;
    a.sy[(size_t)row * my + c0 + col] = 0.5f * z.y;
  }
  // energy partial
#pragma unroll
  for (int o = 16; o > 0; o >>= 1) e += __shfl_xor_sync(0xffffffffu, e, o);
  if ((threadIdx.x & 31) == 0) s_red[threadIdx.x >> 5] = e;
  __syncthreads();
  if (threadIdx.x == 0) {
    double t = 0.0;
    for (int w = 0; w < kColThreads / 32; w++) t += s_red[w];
    a.energy_part[blockIdx.x] = t * a.energy_scale;
  }
}

// T2a (warp FFT, M = mx = 2^LOGM in [32, 1024]): every warp owns B = 1024 / M column pairs of
// t.  DCT_x of the pair as one complex sequence, the Parseval energy term and the spectral
// scaling of eqs (9c)/(9d); writes (A_X, A_Y) transposed, specT[v][u] (row v contiguous), for
// the inverse x pass (T2b = the row-inverse kernel on specT: IDXST_x of A_X + i IDCT_x of A_Y,
// stored transposed into (sX, sY)[x][y]).  Splitting the column work in two keeps one FFT per
// warp per kernel: these transforms are latency-bound at 512-1024 warps per map.
constexpr int kWColWarps = 2;

template <int LOGM>
__global__ void __launch_bounds__(32 * kWColWarps) k_col_fwd_w(ColFieldArgs a, float2 *__restrict__ specT,
                                                             const float2 *__restrict__ tw2) {
  griddep_wait();
  constexpr int M = 1 << LOGM, K = M / 32, B = wfft::kPts / M;
  extern __shared__ float2 wsm[];
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  float2 *buf = wsm + warp * wfft::kBufPad;
  const int gw = blockIdx.x * kWColWarps + warp;   // global warp: energy slot
  const int p0 = gw * B;                           // first column pair
  const int my = a.my, npairs = my / 2;
  if (p0 >= npairs) return;
  float kxr[K];   // twiddle / phase tables are read right before use (L1-resident)
#pragma unroll
  for (int j = 0; j < K; j++) kxr[j] = __ldg(a.kx + lane + 32 * j);
  float2 z[32];
#pragma unroll
  for (int s = 0; s < B; s++) {
    const bool ok = p0 + s < npairs;
#pragma unroll
    for (int j = 0; j < K; j++) {
      const int n = lane + 32 * j;
      const int src = n < M / 2 ? 2 * n : 2 * (M - 1 - n) + 1;   // Makhoul order along x
      z[s * K + j] = ok ? __ldg(reinterpret_cast<const float2 *>(a.t + (size_t)src * my) + (p0 + s)) : make_float2(0.f, 0.f);
    }
  }
  wfft::warp_fft<LOGM, false>(z, buf, tw2);
  const float scale = 2.f / M;
  double e = 0.0;
#pragma unroll
  for (int s = 0; s < B; s++) {
    const int p = p0 + s;
    if (p >= npairs) break;
    const float ky0 = __ldg(a.ky + 2 * p), ky1 = __ldg(a.ky + 2 * p + 1);
    const double wv0 = (p == 0) ? 0.25 * my : 0.5 * my, wv1 = 0.5 * my;
#pragma unroll
    for (int j = 0; j < K; j++) {
      const int u = lane + 32 * j;
      const float2 d = dct_post_v(buf[wfft::pad(s * M + u)], buf[wfft::pad(s * M + ((M - u) & (M - 1)))],
                                  __ldg(a.ph_x + lane + 32 * j), scale);   // (a_2p[u], a_2p+1[u])
      const float kx = kxr[j];
      const double wu = (u == 0) ? 0.25 * M : 0.5 * M;
      const float ik0 = (u == 0 && p == 0) ? 0.f : fast_rcp(kx * kx + ky0 * ky0);   // a_00 / k^2 := 0
      const float ik1 = fast_rcp(kx * kx + ky1 * ky1);
      e += wu * (wv0 * (double)(d.x * d.x * ik0) + wv1 * (double)(d.y * d.y * ik1));
      specT[(size_t)(2 * p) * M + u] = make_float2(d.x * kx * ik0, d.x * ky0 * ik0);
      specT[(size_t)(2 * p + 1) * M + u] = make_float2(d.y * kx * ik1, d.y * ky1 * ik1);
    }
  }
#pragma unroll
  for (int o = 16; o > 0; o >>= 1) e += __shfl_xor_sync(0xffffffffu, e, o);
  if (lane == 0) a.energy_part[gw] = e * a.energy_scale;
}

// T2 fused (warp FFT, M = mx = 2^LOGM in [32, 1024]): every warp owns B = 1024 / M column pairs
// of t and runs, per pair, the forward DCT_x of both columns as one complex FFT, the Parseval
// energy term and the spectral scaling of eqs (9c)/(9d) (a_00 / k^2 := 0), then per column the
// inverse x pass IDXST_x(A_X) + i IDCT_x(A_Y) as one complex IFFT (eq 8e reversal), and writes
// (sX, sY) of both columns as one 16-byte store per row: sxy[x][2p], sxy[x][2p+1].  One kernel
// instead of T2a + T2b: the spectrum never leaves shared memory.
template <int LOGM>
__global__ void __launch_bounds__(32 * kWColWarps) k_col_fields_w(ColFieldArgs a, float2 *__restrict__ sxy,
                                                                const float2 *__restrict__ tw2) {
  griddep_wait();
  constexpr int M = 1 << LOGM, K = M / 32, B = wfft::kPts / M;
  extern __shared__ float2 wsm[];
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  float2 *buf = wsm + warp * (wfft::kBufPad + 2 * wfft::kPts);
  float2 *spec = buf + wfft::kBufPad;   // [2][kPts]: (A_X, A_Y) of column 2p (h = 0) / 2p + 1 (h = 1)
  const int gw = blockIdx.x * kWColWarps + warp;   // global warp: energy slot
  const int p0 = gw * B;                           // first column pair
  const int my = a.my, npairs = my / 2;
  if (p0 >= npairs) return;
  float kxr[K];   // twiddle / phase tables are read right before use (L1-resident)
#pragma unroll
  for (int j = 0; j < K; j++) kxr[j] = __ldg(a.kx + lane + 32 * j);
  float2 z[32];
#pragma unroll
  for (int s = 0; s < B; s++) {
    const bool ok = p0 + s < npairs;
#pragma unroll
    for (int j = 0; j < K; j++) {
      const int n = lane + 32 * j;
      const int src = n < M / 2 ? 2 * n : 2 * (M - 1 - n) + 1;   // Makhoul order along x
      z[s * K + j] = ok ? __ldg(reinterpret_cast<const float2 *>(a.t + (size_t)src * my) + (p0 + s)) : make_float2(0.f, 0.f);
    }
  }
  wfft::warp_fft<LOGM, false>(z, buf, tw2);
  const float scale = 2.f / M;
  double e = 0.0;
#pragma unroll
  for (int s = 0; s < B; s++) {
    const int p = p0 + s;
    const bool ok = p < npairs;
    const float ky0 = ok ? __ldg(a.ky + 2 * p) : 0.f, ky1 = ok ? __ldg(a.ky + 2 * p + 1) : 0.f;
    const double wv0 = (p == 0) ? 0.25 * my : 0.5 * my, wv1 = 0.5 * my;
#pragma unroll
    for (int j = 0; j < K; j++) {
      const int u = lane + 32 * j;
      const float2 d = dct_post_v(buf[wfft::pad(s * M + u)], buf[wfft::pad(s * M + ((M - u) & (M - 1)))],
                                  __ldg(a.ph_x + lane + 32 * j), scale);   // (a_2p[u], a_2p+1[u])
      const float kx = kxr[j];
      const double wu = (u == 0) ? 0.25 * M : 0.5 * M;
      const float ik0 = (!ok || (u == 0 && p == 0)) ? 0.f : fast_rcp(kx * kx + ky0 * ky0);   // a_00 / k^2 := 0
      const float ik1 = ok ? fast_rcp(kx * kx + ky1 * ky1) : 0.f;
      e += wu * (wv0 * (double)(d.x * d.x * ik0) + wv1 * (double)(d.y * d.y * ik1));
      spec[s * M + u] = make_float2(d.x * kx * ik0, d.x * ky0 * ik0);
      spec[wfft::kPts + s * M + u] = make_float2(d.y * kx * ik1, d.y * ky1 * ik1);
    }
  }
#pragma unroll
  for (int o = 16; o > 0; o >>= 1) e += __shfl_xor_sync(0xffffffffu, e, o);
  if (lane == 0) a.energy_part[gw] = e * a.energy_scale;
  __syncwarp();
  float2 r0[32];
#pragma unroll
  for (int h = 0; h < 2; h++) {
    const float2 *A = spec + h * wfft::kPts;
    float2 v[32];
#pragma unroll
    for (int s = 0; s < B; s++) {
#pragma unroll
      for (int j = 0; j < K; j++) {
        const int k = lane + 32 * j;
        const float2 ak = A[s * M + k], ank = k ? A[s * M + M - k] : make_float2(0.f, 0.f);
        // p = A_X reversed (IDXST via eq 8e: x'_t = x_{N-t}, x'_0 = 0), q = A_Y (IDCT)
        v[s * K + j] = inv_pre(ank.x, ak.y, k ? ak.x : 0.f, ank.y, __ldg(a.ph_x + lane + 32 * j));
      }
    }
    wfft::warp_fft<LOGM, true>(v, buf, tw2);
#pragma unroll
    for (int s = 0; s < B; s++) {
#pragma unroll
      for (int j = 0; j < K; j++) {
        const int t = lane + 32 * j;
        const float2 zz = buf[wfft::pad(s * M + mk_pos(t, M))];
        const float2 o = make_float2((t & 1) ? -0.5f * zz.x : 0.5f * zz.x, 0.5f * zz.y);   // IDXST sign (-1)^x
        if (h == 0) {
          r0[s * K + j] = o;
        } else if (p0 + s < npairs) {
          const float2 q = r0[s * K + j];
          *reinterpret_cast<float4 *>(sxy + (size_t)t * my + 2 * (p0 + s)) = make_float4(q.x, q.y, o.x, o.y);
        }
      }
    }
    __syncwarp();   // buf is reused by the next inverse
  }
}

size_t col_fields_w_smem() { return (size_t)kWColWarps * (wfft::kBufPad + 2 * wfft::kPts) * sizeof(float2); }

// psi spectrum scaling for the debug hook: out = a / k^2 (0 at the DC term)
__global__ void k_scale_psi(const float *a, float *out, const float *kx, const float *ky, int mx, int my) {
  const size_t n = (size_t)mx * my;
  for (size_t i = blockIdx.x * (size_t)blockDim.x + threadIdx.x; i < n; i += (size_t)gridDim.x * blockDim.x) {
    const int u = (int)(i / my), v = (int)(i % my);
    const float k2 = kx[u] * kx[u] + ky[v] * ky[v];
    out[i] = (u == 0 && v == 0) ? 0.f : a[i] / k2;
  }
}

__global__ void k_split_xi(const float2 *xi, float *xx, float *xy, size_t n) {
  for (size_t i = blockIdx.x * (size_t)blockDim.x + threadIdx.x; i < n; i += (size_t)gridDim.x * blockDim.x) {
    const float2 v = xi[i];
    if (xx) xx[i] = v.x;
    if (xy) xy[i] = v.y;
  }
}

size_t row_smem(int n) { return (size_t)n * sizeof(float2) + 2 * (size_t)n * sizeof(float); }
size_t col_generic_smem(int mx) { return (size_t)(col_slab(mx) / 2) * mx * sizeof(float2) + (size_t)col_slab(mx) * mx * sizeof(float); }
size_t col_fields_smem(int mx) { return (size_t)col_slab(mx) * mx * sizeof(float2) + 2 * (size_t)col_slab(mx) * mx * sizeof(float); }

bool warp_fft_ok(int log2n) { return log2n >= 5 && log2n <= 10; }
size_t wrow_smem() { return (size_t)kWRowWarps * wfft::kBufPad * sizeof(float2); }
// T1: FFT buffers + per-warp staging of 2 * 1024 input values (8 bytes each at most)
size_t wrow_dct_smem() { return wrow_smem() + (size_t)kWRowWarps * 2 * wfft::kPts * sizeof(unsigned long long); }
int wrow_ctas(int units, int log2n) {   // units = row pairs (T1) or rows (T3)
  const int per_warp = wfft::kPts >> log2n, per_cta = per_warp * kWRowWarps;
  return (units + per_cta - 1) / per_cta;
}

void row_inv(const Ctx &c, const float *inA, long long stepA, int opA, const float *inB, long long stepB,
             int opB, float *outA, long long ostepA, float *outB, long long ostepB, float2 *outI,
             int rows, cudaStream_t s, const float2 *inI = nullptr, bool x_axis = false, long long ostepT = 0) {
  RowInvArgs a;
  a.inA = inA; a.inB = inB; a.stepA = stepA; a.stepB = stepB; a.opA = opA; a.opB = opB;
  a.outA = outA; a.outB = outB; a.ostepA = ostepA; a.ostepB = ostepB; a.outI = outI;
  a.inI = inI;
  a.ostepT = ostepT;
  a.tma = c.row_tma ? 1 : 0;
  const int log2n = x_axis ? c.log2mx : c.log2my;
  const float2 *tw2 = x_axis ? c.d_tw2_x : c.d_tw2_y;
  a.n = 1 << log2n; a.log2n = log2n;
  a.tw = x_axis ? c.d_tw_x : c.d_tw_y;
  a.ph = x_axis ? c.d_ph_x : c.d_ph_y;
  if (!warp_fft_ok(log2n)) {
    k_row_inv<<<rows, kRowThreads, row_smem(a.n), s>>>(a);
    return;
  }
  if (ostepT > 0 && inI) {   // T2b: 4-warp CTAs, coalesced transposed stores (DP_T2B_WARPS=2: 2-warp, A/B)
    auto go = [&](auto wtag) {
      constexpr int W = decltype(wtag)::value;
      const int per_cta = (wfft::kPts >> log2n) * W;
      const int g = (rows + per_cta - 1) / per_cta;
      const size_t sm = (size_t)W * wfft::kBufPad * sizeof(float2);
      switch (log2n) {
        case 5: launch_chain(c.pdl, k_row_inv_w<5, W, true>, g, 32 * W, sm, s, a, tw2, rows); break;
        case 6: launch_chain(c.pdl, k_row_inv_w<6, W, true>, g, 32 * W, sm, s, a, tw2, rows); break;
        case 7: launch_chain(c.pdl, k_row_inv_w<7, W, true>, g, 32 * W, sm, s, a, tw2, rows); break;
        case 8: launch_chain(c.pdl, k_row_inv_w<8, W, true>, g, 32 * W, sm, s, a, tw2, rows); break;
        case 9: launch_chain(c.pdl, k_row_inv_w<9, W, true>, g, 32 * W, sm, s, a, tw2, rows); break;
        default: launch_chain(c.pdl, k_row_inv_w<10, W, true>, g, 32 * W, sm, s, a, tw2, rows); break;
      }
    };
    if (c.t2b_warps == 2)
      go(std::integral_constant<int, 2>{});
    else
      go(std::integral_constant<int, kTStoreWarps>{});
    return;
  }
  const int g = wrow_ctas(rows, log2n);
  const size_t sm = wrow_smem();
  switch (log2n) {
    case 5: launch_chain(c.pdl, k_row_inv_w<5>, g, 32 * kWRowWarps, sm, s, a, tw2, rows); break;
    case 6: launch_chain(c.pdl, k_row_inv_w<6>, g, 32 * kWRowWarps, sm, s, a, tw2, rows); break;
    case 7: launch_chain(c.pdl, k_row_inv_w<7>, g, 32 * kWRowWarps, sm, s, a, tw2, rows); break;
    case 8: launch_chain(c.pdl, k_row_inv_w<8>, g, 32 * kWRowWarps, sm, s, a, tw2, rows); break;
    case 9: launch_chain(c.pdl, k_row_inv_w<9>, g, 32 * kWRowWarps, sm, s, a, tw2, rows); break;
    default: launch_chain(c.pdl, k_row_inv_w<10>, g, 32 * kWRowWarps, sm, s, a, tw2, rows); break;
  }
}

// T1 dispatcher: DCT over y of every row of `in` (IN = float or the int64 map)
template <class IN>
void row_dct(const Ctx &c, const IN *in, float *out, cudaStream_t s) {
  if (!warp_fft_ok(c.log2my)) {
    k_row_dct<IN><<<c.mx / 2, kRowThreads, row_smem(c.my), s>>>(in, out, c.my, c.log2my, c.d_tw_y, c.d_ph_y);
    return;
  }
  const int np = c.mx / 2, g = wrow_ctas(np, c.log2my);
  const size_t sm = c.t1_tma ? wrow_dct_smem() : wrow_smem();
  switch (c.log2my) {
    case 5: launch_chain(c.pdl, k_row_dct_w<IN, 5>, g, 32 * kWRowWarps, sm, s, in, out, c.d_tw2_y, c.d_ph_y, np, c.t1_tma ? 1 : 0); break;
    case 6: launch_chain(c.pdl, k_row_dct_w<IN, 6>, g, 32 * kWRowWarps, sm, s, in, out, c.d_tw2_y, c.d_ph_y, np, c.t1_tma ? 1 : 0); break;
    case 7: launch_chain(c.pdl, k_row_dct_w<IN, 7>, g, 32 * kWRowWarps, sm, s, in, out, c.d_tw2_y, c.d_ph_y, np, c.t1_tma ? 1 : 0); break;
    case 8: launch_chain(c.pdl, k_row_dct_w<IN, 8>, g, 32 * kWRowWarps, sm, s, in, out, c.d_tw2_y, c.d_ph_y, np, c.t1_tma ? 1 : 0); break;
    case 9: launch_chain(c.pdl, k_row_dct_w<IN, 9>, g, 32 * kWRowWarps, sm, s, in, out, c.d_tw2_y, c.d_ph_y, np, c.t1_tma ? 1 : 0); break;
    default: launch_chain(c.pdl, k_row_dct_w<IN, 10>, g, 32 * kWRowWarps, sm, s, in, out, c.d_tw2_y, c.d_ph_y, np, c.t1_tma ? 1 : 0); break;
  }
}

}  // namespace

// smem opt-in (called once from dp_create)
cudaError_t dct_configure(int mx, int my) {
  cudaError_t e;
  e = cudaFuncSetAttribute(k_row_dct<float>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)row_smem(my));
  if (e != cudaSuccess) return e;
  e = cudaFuncSetAttribute(k_row_dct<unsigned long long>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)row_smem(my));
  if (e != cudaSuccess) return e;
  e = cudaFuncSetAttribute(k_row_inv, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)row_smem(my));
  if (e != cudaSuccess) return e;
  e = cudaFuncSetAttribute(k_col_generic, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)col_generic_smem(mx));
  if (e != cudaSuccess) return e;
  e = cudaFuncSetAttribute(k_col_fields, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)col_fields_smem(mx));
  if (e != cudaSuccess) return e;
  const int dsm = (int)wrow_dct_smem();
  for (auto f : {k_row_dct_w<float, 5>, k_row_dct_w<float, 6>, k_row_dct_w<float, 7>, k_row_dct_w<float, 8>,
                 k_row_dct_w<float, 9>, k_row_dct_w<float, 10>}) {
    e = cudaFuncSetAttribute(f, cudaFuncAttributeMaxDynamicSharedMemorySize, dsm);
    if (e != cudaSuccess) return e;
  }
  for (auto f : {k_row_dct_w<unsigned long long, 5>, k_row_dct_w<unsigned long long, 6>,
                 k_row_dct_w<unsigned long long, 7>, k_row_dct_w<unsigned long long, 8>,
                 k_row_dct_w<unsigned long long, 9>, k_row_dct_w<unsigned long long, 10>}) {
    e = cudaFuncSetAttribute(f, cudaFuncAttributeMaxDynamicSharedMemorySize, dsm);
    if (e != cudaSuccess) return e;
  }
  const int wsm = (int)col_fields_w_smem();
  for (auto f : {k_col_fields_w<5>, k_col_fields_w<6>, k_col_fields_w<7>, k_col_fields_w<8>, k_col_fields_w<9>,
                 k_col_fields_w<10>}) {
    e = cudaFuncSetAttribute(f, cudaFuncAttributeMaxDynamicSharedMemorySize, wsm);
    if (e != cudaSuccess) return e;
  }
  return cudaSuccess;
}

int col_fields_ctas(int mx, int my) { return my / col_slab(mx); }

namespace {
void fields_after_t1(const Ctx &c, cudaStream_t s);
}

void launch_fields(const Ctx &c, const float *rho, cudaStream_t s) {
  if (c.fft_cta) {
    launch_fields_cta(c, rho, false, s);
    return;
  }
  // T1: t = DCT_y(rho)
  row_dct<float>(c, rho, c.d_t, s);
  fields_after_t1(c, s);
}

void launch_fields_fixed(const Ctx &c, cudaStream_t s) {
  if (c.fft_cta) {
    launch_fields_cta(c, c.d_rho, true, s);
    return;
  }
  row_dct<unsigned long long>(c, c.d_rho, c.d_t, s);
  fields_after_t1(c, s);
}

__global__ void k_rho_to_float(const unsigned long long *in, float *out, size_t n) {
  for (size_t i = blockIdx.x * (size_t)blockDim.x + threadIdx.x; i < n; i += (size_t)gridDim.x * blockDim.x)
    out[i] = load_map(in + i);
}

void launch_rho_to_float(const Ctx &c, float *out, cudaStream_t s) {
  k_rho_to_float<<<c.num_sms * 4, 256, 0, s>>>(c.d_rho, out, (size_t)c.mx * c.my);
}

namespace {
void fields_after_t1(const Ctx &c, cudaStream_t s) {
  // T2: columns (DCT_x, scaling, energy, inverse x)
  ColFieldArgs a;
  a.t = c.d_t; a.sx = c.d_sx; a.sy = c.d_sy;
  a.mx = c.mx; a.log2mx = c.log2mx; a.my = c.my;
  a.tw_x = c.d_tw_x; a.ph_x = c.d_ph_x; a.kx = c.d_kx; a.ky = c.d_ky;
  a.energy_part = c.d_part + c.n_wa_part + (c.n_regions > 0 && c.cur_region > 0 ? c.cur_region * c.n_en_part : 0);
  a.energy_scale = 0.5 * c.bx * c.by;
  if (c.fft_hybrid) {   // the CTA-FFT column pass on t[x][y], then T3
    launch_p2_rowmajor(c, s);
    row_inv(c, nullptr, 0, 1, nullptr, 0, 2, nullptr, 0, nullptr, 0, c.d_xi, c.mx, s, c.d_sxy);
    return;
  }
  if (warp_fft_ok(c.log2mx) && warp_fft_ok(c.log2my)) {
    const int warps = ((c.my / 2) + (wfft::kPts >> c.log2mx) - 1) / (wfft::kPts >> c.log2mx);
    const int g = (warps + kWColWarps - 1) / kWColWarps;
    float2 *sxy = c.d_sxy;
    if (c.fused_t2) {   // measured slower at 1024^2 (longer per-warp latency chain); kept for A/B
      const size_t sm = col_fields_w_smem();
      switch (c.log2mx) {   // T2: DCT_x, scaling, energy, IDXST_x / IDCT_x in one pass
        case 5: launch_chain(c.pdl, k_col_fields_w<5>, g, 32 * kWColWarps, sm, s, a, sxy, c.d_tw2_x); break;
        case 6: launch_chain(c.pdl, k_col_fields_w<6>, g, 32 * kWColWarps, sm, s, a, sxy, c.d_tw2_x); break;
        case 7: launch_chain(c.pdl, k_col_fields_w<7>, g, 32 * kWColWarps, sm, s, a, sxy, c.d_tw2_x); break;
        case 8: launch_chain(c.pdl, k_col_fields_w<8>, g, 32 * kWColWarps, sm, s, a, sxy, c.d_tw2_x); break;
        case 9: launch_chain(c.pdl, k_col_fields_w<9>, g, 32 * kWColWarps, sm, s, a, sxy, c.d_tw2_x); break;
        default: launch_chain(c.pdl, k_col_fields_w<10>, g, 32 * kWColWarps, sm, s, a, sxy, c.d_tw2_x); break;
      }
    } else {
      const size_t sm = (size_t)kWColWarps * wfft::kBufPad * sizeof(float2);
      float2 *spec = c.d_spec;
      switch (c.log2mx) {   // T2a
        case 5: launch_chain(c.pdl, k_col_fwd_w<5>, g, 32 * kWColWarps, sm, s, a, spec, c.d_tw2_x); break;
        case 6: launch_chain(c.pdl, k_col_fwd_w<6>, g, 32 * kWColWarps, sm, s, a, spec, c.d_tw2_x); break;
        case 7: launch_chain(c.pdl, k_col_fwd_w<7>, g, 32 * kWColWarps, sm, s, a, spec, c.d_tw2_x); break;
        case 8: launch_chain(c.pdl, k_col_fwd_w<8>, g, 32 * kWColWarps, sm, s, a, spec, c.d_tw2_x); break;
        case 9: launch_chain(c.pdl, k_col_fwd_w<9>, g, 32 * kWColWarps, sm, s, a, spec, c.d_tw2_x); break;
        default: launch_chain(c.pdl, k_col_fwd_w<10>, g, 32 * kWColWarps, sm, s, a, spec, c.d_tw2_x); break;
      }
      // T2b: per column v (row v of specT): sX = IDXST_x(A_X), sY = IDCT_x(A_Y), stored [x][y]
      row_inv(c, nullptr, 0, 2, nullptr, 0, 1, nullptr, 0, nullptr, 0, sxy, c.my, s, spec, true, c.my);
    }
    // T3: rows: xi_X = IDCT_y(sX), xi_Y = IDXST_y(sY), interleaved in and out
    row_inv(c, nullptr, 0, 1, nullptr, 0, 2, nullptr, 0, nullptr, 0, c.d_xi, c.mx, s, sxy);
    return;
  }
  k_col_fields<<<c.my / col_slab(c.mx), kColThreads, col_fields_smem(c.mx), s>>>(a);
  // T3: rows: xi_X = IDCT_y(sX), xi_Y = IDXST_y(sY), interleaved
  row_inv(c, c.d_sx, c.my, 1, c.d_sy, c.my, 2, nullptr, 0, nullptr, 0, c.d_xi, c.mx, s);
}
}  // namespace

void launch_split_fields(const Ctx &c, float *xi_x, float *xi_y, cudaStream_t s) {
  k_split_xi<<<c.num_sms * 4, 256, 0, s>>>(c.d_xi, xi_x, xi_y, (size_t)c.mx * c.my);
}

void launch_transform(const Ctx &c, int kind, const float *in, float *out, cudaStream_t s) {
  const int mx = c.mx, my = c.my;
  float *tmp = c.d_t;  // scratch (debug path only)
  switch (kind) {
    case DP_T_DCT2:
      row_dct<float>(c, in, tmp, s);
      k_col_generic<<<my / col_slab(mx), kColThreads, col_generic_smem(mx), s>>>(tmp, out, 0, mx, c.log2mx, my, c.d_tw_x, c.d_ph_x);
      break;
    case DP_T_IDCT2:
    case DP_T_IDXST_IDCT:
    case DP_T_IDCT_IDXST: {
      const int op_y = (kind == DP_T_IDCT_IDXST) ? 2 : 1;
      const int op_x = (kind == DP_T_IDXST_IDCT) ? 2 : 1;
      // rows (2r, 2r+1) share a complex IFFT
      row_inv(c, in, 2LL * my, op_y, in + my, 2LL * my, op_y, tmp, 2LL * my, tmp + my, 2LL * my, nullptr, mx / 2, s);
      k_col_generic<<<my / col_slab(mx), kColThreads, col_generic_smem(mx), s>>>(tmp, out, op_x, mx, c.log2mx, my, c.d_tw_x, c.d_ph_x);
      break;
    }
    default:
      break;
  }
}

void launch_psi(const Ctx &c, const float *rho, float *psi, cudaStream_t s) {
  // debug only: a = DCT2(rho) -> psi = IDCT2(a / k^2).  Uses sx / sy as scratch.
  launch_transform(c, DP_T_DCT2, rho, c.d_sx, s);
  k_scale_psi<<<c.num_sms * 4, 256, 0, s>>>(c.d_sx, c.d_sy, c.d_kx, c.d_ky, c.mx, c.my);
  launch_transform(c, DP_T_IDCT2, c.d_sy, psi, s);
}

}  // namespace dp
