// fields.cu — the spectral Poisson solve of one evaluation (steps 2-3 of P:253-256) in three
// passes over the bin map, each a CTA-level FFT (fft_cta.cuh: radix 16, 16 points per thread,
// in place).
//
// Method: a = DCT2(rho) (eq 9a; DCT of eq 7a with 2/N per axis, readings
// A13/A20), A_X = a k_u / k^2 and A_Y = a k_v / k^2 with a_00 / k^2 := 0 (eqs 9c/9d, A12, A15),
// xi_X = IDXST_x IDCT_y (A_X), xi_Y = IDCT_x IDXST_y (A_Y) (eqs 9c/9d with eqs 7b/8a/8e), and
// the energy D = 1/2 b_x b_y sum rho psi taken in the spectral domain by Parseval (A8), so psi
// is never formed.  Each 1-D transform is an N-point complex FFT in Makhoul's order (Alg 3,
// P:367-437, without the garbled eqs 11/12, readings A16-A18): two real sequences share one
// complex FFT (z = p + i q).
//
//   P1  rows x:     t = DCT_y(rho) of rows (2p, 2p+1)           -> tT[y][x]   (transposed store)
//   P2  columns y:  a = DCT_x(t) of columns (2p, 2p+1); energy; A_X, A_Y; per column
//                   IDXST_x(A_X) + i IDCT_x(A_Y)                  -> sxy[x][y]  (transposed store)
//   P3  rows x:     IDCT_y(sX) + i IDXST_y(sY)                      -> xi[x][y] = (xi_X, xi_Y)
//
// Every pass reads whole rows (contiguous) and the two transposed stores write 2 SEQ adjacent
// values per output row (16-32 bytes): no strided column reads.  P2 takes the forward
// post-processing, the scaling and the inverse pre-processing of both columns per spectral pair
// (u, M - u) in one thread, in place: the spectrum is never stored.  The per-element phase,
// twiddle and wavenumber loads are issued together (unrolled loops, twiddles ahead of each
// stage's barrier): one table latency per stage instead of one per element.
#include "dp_internal.h"
#include "fft_cta.cuh"

namespace dp {

namespace {

int ilog2_int(int v) {
  int l = 0;
  while ((1 << l) < v) l++;
  return l;
}

using cfft::buf_len;
using cfft::pad;

// Makhoul reordering (Alg 3 lines 3-8): v[n] = x[2n], v[N-1-n] = x[2n+1]; position of x[t] in v
__device__ __forceinline__ int mk_pos(int t, int n) { return (t & 1) ? n - ((t + 1) >> 1) : (t >> 1); }

__device__ __forceinline__ float map_value(float v) { return v; }
// one rounding of the integer, then an exact power-of-two scale: the same value as the fp64
// route (exact below 2^53) without the fp64 conversions
__device__ __forceinline__ float map_value(unsigned long long v) {
  return __ll2float_rn((long long)v) * (1.0f / (float)(1ll << kRhoScaleLog2));
}

// forward DCT post-processing of a pair packed as z = p + i q (Alg 3 lines 10-16): returns
// (DCT(p)_k, DCT(q)_k) with the 2/N factor (A13); z = Z[k], zc = Z[N - k], ph = e^{-i pi k / 2N}
__device__ __forceinline__ float2 dct_post(float2 z, float2 zc, float2 ph, float scale) {
  const float v0x = 0.5f * (z.x + zc.x), v0y = 0.5f * (z.y - zc.y);
  const float dx = z.x - zc.x, dy = z.y + zc.y;
  const float v1x = 0.5f * dy, v1y = -0.5f * dx;
  return make_float2(scale * (v0x * ph.x - v0y * ph.y), scale * (v1x * ph.x - v1y * ph.y));
}

// inverse pre-processing of two IDCT-type sequences p (real) and q (imag), IDXST inputs already
// reversed (eq 8e): Z_k = e^{+i pi k / 2N} [(p_k + q_{N-k}) + i (q_k - p_{N-k})]
__device__ __forceinline__ float2 inv_pre(float pk, float qk, float pnk, float qnk, float2 ph) {
  const float re = pk + qnk, im = qk - pnk;
  return make_float2(re * ph.x + im * ph.y, im * ph.x - re * ph.y);
}

__device__ __forceinline__ float fast_rcp(float x) {
  float r;
  asm("rcp.approx.f32 %0, %1;" : "=f"(r) : "f"(x));
  return r;
}

// Layouts.  Unsharded: tT[y][x] (P1 -> P2), sxy[x][y] (P2 -> P3).  Row-sharded over G ranks
// (R = mx / G rows and C = my / G columns per rank, rank offsets x_base, y_base):
// P1 writes its rows' t as the all-to-all send blocks S1[q][y - qC][x - x_base], P2 reads the
// received blocks R1[p][y - y_base][x - pR] and writes S2[q][x - qR][y - y_base], P3 reads
// R2[p][x - x_base][y - pC].  With G = 1 (R = mx, C = my) these are exactly the unsharded
// layouts, so one indexing serves both.
struct FieldArgs {
  const void *rho;        // [mx][my], IN = float or int64 (2^-29 units); rows [x_base, x_base + nrows) used
  float *t_out;           // P1 output (tT / S1)
  const float *t_in;      // P2 input (tT / R1)
  float2 *s_out;          // P2 output (sxy / S2)
  const float2 *s_in;     // P3 input (sxy / R2)
  float2 *xi;             // [mx][my] (xi_X, xi_Y); P3 writes rows [x_base, x_base + nrows)
  int mx, my;
  int R, C;               // rows / columns per rank block (powers of two)
  int lR, lC;             // log2 R, log2 C
  int x_base, y_base;     // this rank's first row / column
  int nrows, ncols;       // rows of P1 / P3, columns of P2
  const float2 *twf_x, *twf_y;   // exp(-2 pi i k / N), k < N
  const float2 *ph_x, *ph_y;     // exp(-i pi k / 2N), k < N
  const float *kx, *ky;          // wavenumbers (A12)
  double *energy_part;           // one slot per P2 CTA
  double energy_scale;           // 1/2 b_x b_y
};

// Layout helpers (one code path for the unsharded and the row-sharded block layouts, so both
// run the same instructions: shifts, R and C are powers of two)
__device__ __forceinline__ size_t t_index(const FieldArgs &a, int y, int xl) {   // tT / S1 / R1, xl = x - x_base
  return ((size_t)(y >> a.lC) << (a.lC + a.lR)) + ((size_t)(y & (a.C - 1)) << a.lR) + xl;
}
__device__ __forceinline__ size_t s_index(const FieldArgs &a, int x, int yl) {   // sxy / S2 / R2, yl = y - y_base
  return ((size_t)(x >> a.lR) << (a.lC + a.lR)) + ((size_t)(x & (a.R - 1)) << a.lC) + yl;
}

// ---- P1: rows (2p, 2p+1) of rho -> DCT over y -> tT[y][x] ----------------------------------
template <class IN, int LOGN>
__global__ void __launch_bounds__(cfft::seq_per_cta(LOGN) * cfft::threads_per_seq(LOGN))
    k_p1(FieldArgs a) {
  griddep_wait();
  constexpr int N = 1 << LOGN, T = cfft::threads_per_seq(LOGN), SEQ = cfft::seq_per_cta(LOGN);
  constexpr int NT = SEQ * T, ROWS = 2 * SEQ, L = buf_len(N);
  extern __shared__ __align__(16) float2 sm1[];
  float *out = reinterpret_cast<float *>(sm1 + SEQ * L);   // [N][ROWS]
  const IN *rho = reinterpret_cast<const IN *>(a.rho);
  const int tid = threadIdx.x, s = tid / T, t = tid % T;
  const int x0 = a.x_base + blockIdx.x * ROWS, xend = a.x_base + a.nrows;
  // load: row x0 + rr (coalesced) -> real (rr even) / imaginary (rr odd) part of sequence rr/2,
  // at its Makhoul position; every load is issued before the first use
  constexpr int PER = ROWS * N / NT;
  IN v[PER];
#pragma unroll
  for (int q = 0; q < PER; q++) {
    const int idx = tid + q * NT, x = x0 + (idx >> LOGN);
    v[q] = x < xend ? rho[(size_t)x * N + (idx & (N - 1))] : (IN)0;
  }
#pragma unroll
  for (int q = 0; q < PER; q++) {
    const int idx = tid + q * NT, rr = idx >> LOGN, col = idx & (N - 1);
    float *slot = reinterpret_cast<float *>(sm1 + (rr >> 1) * L + pad(mk_pos(col, N)));
    slot[rr & 1] = map_value(v[q]);
  }
  __syncthreads();
  float2 *const A[1] = {sm1 + s * L};
  cfft::fft<LOGN, false>(A, t, a.twf_y);
  const float scale = 2.f / N;
#pragma unroll
  for (int m = 0; m < 16; m++) {   // unrolled: the 16 phase loads are issued together
    const int k = t + m * T;
    const float2 d = dct_post(A[0][pad(k)], A[0][pad((N - k) & (N - 1))], __ldg(a.ph_y + k), scale);
    *reinterpret_cast<float2 *>(out + k * ROWS + 2 * s) = d;
  }
  __syncthreads();
  // transposed store: tT[k][x0 .. x0 + ROWS) (unsharded) / S1[k / C][k % C][x0 - x_base ..]
  if (ROWS % 4 == 0 && x0 + ROWS <= xend) {
    for (int idx = tid; idx < N * (ROWS / 4); idx += NT) {
      const int k = idx / (ROWS / 4), q = idx % (ROWS / 4);
      *reinterpret_cast<float4 *>(a.t_out + t_index(a, k, x0 - a.x_base) + 4 * q) =
          *reinterpret_cast<const float4 *>(out + k * ROWS + 4 * q);
    }
  } else {
    for (int idx = tid; idx < N * ROWS; idx += NT) {
      const int k = idx / ROWS, c = idx % ROWS;
      if (x0 + c < xend) a.t_out[t_index(a, k, x0 - a.x_base) + c] = out[idx];
    }
  }
}

// ---- P2: columns (2p, 2p+1) (rows of tT) -> DCT over x, energy, scaling, inverse over x ----
// TIN: t stored transposed, tT[y][x] (after P1); otherwise t[x][y] (after the warp-FFT T1):
// the CTA then reads its COLS adjacent columns as 4 COLS-byte row segments.
// P2 of the hybrid path runs one column pair per CTA (SEQ = 1).
// Per column pair: one forward FFT (the two columns packed as z = p + i q), then, per spectral
// pair (u, M - u) held by one thread, the DCT post-processing, the energy terms, the scaling
// (9c/9d) and the inverse pre-processing of BOTH columns written in place (even column) and
// into the second buffer (odd column): the spectrum never needs its own storage.  The two
// inverse FFTs then run in lockstep.
template <int LOGM, bool TIN>
constexpr int p2_seq() { return TIN ? cfft::seq_per_cta(LOGM) : 1; }

// at most 128 registers for a 128-thread CTA (min 4 CTAs / SM by registers): the column pass
// then fits beside two WA CTAs in the overlapped evaluation (their 2 x 256 x 92 registers)
template <int LOGM, bool TIN>
__global__ void __launch_bounds__(p2_seq<LOGM, TIN>() * cfft::threads_per_seq(LOGM),
                                  p2_seq<LOGM, TIN>() * cfft::threads_per_seq(LOGM) <= 128 ? 4 : 1)
    k_p2(FieldArgs a) {
  griddep_wait();
  constexpr int M = 1 << LOGM, T = cfft::threads_per_seq(LOGM), SEQ = p2_seq<LOGM, TIN>();
  constexpr int NT = SEQ * T, COLS = 2 * SEQ, L = buf_len(M);
  extern __shared__ __align__(16) float2 sm2[];   // per group: buffers (even, odd column)
  __shared__ double s_red[NT / 32 > 0 ? NT / 32 : 1];
  const int tid = threadIdx.x, s = tid / T, t = tid % T;
  const int y0 = a.y_base + blockIdx.x * COLS, my = a.my, yend = a.y_base + a.ncols;
  float2 *const A0 = sm2 + (2 * s) * L, *const A1 = A0 + L;
  constexpr int PER = COLS * M / NT;
  float v[PER];
#pragma unroll
  for (int q = 0; q < PER; q++) {
    const int idx = tid + q * NT;
    const int c = TIN ? idx >> LOGM : idx % COLS, x = TIN ? idx & (M - 1) : idx / COLS;
    // received blocks R1[x / R][y - y_base][x % R] (unsharded: tT[y][x])
    v[q] = (y0 + c < yend) ? (TIN ? a.t_in[((size_t)(x >> a.lR) << (a.lC + a.lR)) +
                                           ((size_t)(y0 + c - a.y_base) << a.lR) + (x & (a.R - 1))]
                                  : a.t_in[(size_t)x * my + y0 + c])
                           : 0.f;
  }
#pragma unroll
  for (int q = 0; q < PER; q++) {
    const int idx = tid + q * NT;
    const int c = TIN ? idx >> LOGM : idx % COLS, x = TIN ? idx & (M - 1) : idx / COLS;
    float *slot = reinterpret_cast<float *>(sm2 + (c & ~1) * L + pad(mk_pos(x, M)));
    slot[c & 1] = v[q];
  }
  __syncthreads();
  {
    float2 *const F[1] = {A0};
    cfft::fft<LOGM, false>(F, t, a.twf_x);
  }
  // spectrum of columns v0 = y0 + 2s, v1 = v0 + 1: energy (Parseval, A8) and scaling (9c/9d)
  const float scale = 2.f / M;
  const int v0 = y0 + 2 * s, v1 = v0 + 1;
  const bool ok = v1 < yend;
  const float ky0 = ok ? __ldg(a.ky + v0) : 0.f, ky1 = ok ? __ldg(a.ky + v1) : 0.f;
  const double wv0 = (v0 == 0) ? 0.25 * my : 0.5 * my, wv1 = 0.5 * my;
  double e = 0.0;
  // pairs (u, M - u), u = t + m T < M / 2 (unrolled: the phase / wavenumber loads issue
  // together); u = M / 2 (its own partner) by thread 0 of the group
#pragma unroll
  for (int m = 0; m <= 8; m++) {
    if (m == 8 && t != 0) break;
    const int u = m < 8 ? t + m * T : M / 2;
    const int n = (M - u) & (M - 1);   // partner M - u (u = 0, M / 2: itself)
    const float2 zu = A0[pad(u)], zn = A0[pad(n)];
    // (a_{u,v0}, a_{u,v1}) and the scaled spectra of frequency u
    float2 AXu, AYu, AXn, AYn;   // .x: column v0, .y: column v1
    {
      const float2 d = dct_post(zu, zn, __ldg(a.ph_x + u), scale);
      const float kx = __ldg(a.kx + u);
      const double wu = (u == 0) ? 0.25 * M : 0.5 * M;
      const float ik0 = (!ok || (u == 0 && v0 == 0)) ? 0.f : fast_rcp(kx * kx + ky0 * ky0);   // a_00 / k^2 := 0
      const float ik1 = ok ? fast_rcp(kx * kx + ky1 * ky1) : 0.f;
      e += wu * (wv0 * (double)(d.x * d.x * ik0) + wv1 * (double)(d.y * d.y * ik1));
      AXu = make_float2(d.x * kx * ik0, d.y * kx * ik1);
      AYu = make_float2(d.x * ky0 * ik0, d.y * ky1 * ik1);
    }
    if (n != u) {
      const float2 d = dct_post(zn, zu, __ldg(a.ph_x + n), scale);
      const float kx = __ldg(a.kx + n);
      const double wu = 0.5 * M;
      const float ik0 = ok ? fast_rcp(kx * kx + ky0 * ky0) : 0.f;
      const float ik1 = ok ? fast_rcp(kx * kx + ky1 * ky1) : 0.f;
      e += wu * (wv0 * (double)(d.x * d.x * ik0) + wv1 * (double)(d.y * d.y * ik1));
      AXn = make_float2(d.x * kx * ik0, d.y * kx * ik1);
      AYn = make_float2(d.x * ky0 * ik0, d.y * ky1 * ik1);
    } else {
      AXn = AXu;
      AYn = AYu;
    }
    // inverse pre-processing, p = A_X reversed (IDXST via eq 8e: p_k = A_X[M - k], p_0 = 0),
    // q = A_Y (IDCT): Z_k = inv_pre(p_k, q_k, p_{M-k}, q_{M-k})
    if (u == 0) {
      A0[pad(0)] = inv_pre(0.f, AYu.x, 0.f, 0.f, __ldg(a.ph_x));
      A1[pad(0)] = inv_pre(0.f, AYu.y, 0.f, 0.f, __ldg(a.ph_x));
    } else {
      const float2 phu = __ldg(a.ph_x + u);
      A0[pad(u)] = inv_pre(AXn.x, AYu.x, AXu.x, AYn.x, phu);
      A1[pad(u)] = inv_pre(AXn.y, AYu.y, AXu.y, AYn.y, phu);
      if (n != u) {
        const float2 phn = __ldg(a.ph_x + n);
        A0[pad(n)] = inv_pre(AXu.x, AYn.x, AXn.x, AYu.x, phn);
        A1[pad(n)] = inv_pre(AXu.y, AYn.y, AXn.y, AYu.y, phn);
      }
    }
  }
  __syncthreads();
  {
    float2 *const I[2] = {A0, A1};
    cfft::fft<LOGM, true, 2>(I, t, a.twf_x);
  }
  // transposed store: sxy[x][y0 .. y0 + COLS) (unsharded) / S2[x / R][x % R][y0 - y_base ..];
  // column c = 2 g + h lives in buffer h of group g, at the Makhoul position of x
  if (y0 + COLS <= yend) {
    for (int idx = tid; idx < M * SEQ; idx += NT) {
      const int x = idx / SEQ, g = idx % SEQ;
      const float2 *G = sm2 + (2 * g) * L;
      const int px = pad(mk_pos(x, M));
      const float2 z0 = G[px], z1 = G[L + px];
      const float sg = (x & 1) ? -0.5f : 0.5f;   // IDXST sign (-1)^x
      *reinterpret_cast<float4 *>(a.s_out + s_index(a, x, y0 - a.y_base) + 2 * g) =
          make_float4(sg * z0.x, 0.5f * z0.y, sg * z1.x, 0.5f * z1.y);
    }
  } else {
    for (int idx = tid; idx < M * COLS; idx += NT) {
      const int x = idx / COLS, c = idx % COLS;
      if (y0 + c < yend) {
        const float2 z = sm2[c * L + pad(mk_pos(x, M))];
        a.s_out[s_index(a, x, y0 - a.y_base) + c] = make_float2((x & 1) ? -0.5f * z.x : 0.5f * z.x, 0.5f * z.y);
      }
    }
  }
  // energy partial of this CTA (fixed order: deterministic)
#pragma unroll
  for (int o = 16; o > 0; o >>= 1) e += __shfl_xor_sync(0xffffffffu, e, o);
  if ((tid & 31) == 0) s_red[tid >> 5] = e;
  __syncthreads();
  if (tid == 0) {
    double tot = 0.0;
    for (int w = 0; w < (NT + 31) / 32; w++) tot += s_red[w];
    a.energy_part[y0 / COLS] = tot * a.energy_scale;   // global column-slab slot: the same for any sharding
  }
}

// ---- P3: rows x of sxy -> IDCT_y(sX) + i IDXST_y(sY) -> xi[x][y] ---------------------------
template <int LOGN>
__global__ void __launch_bounds__(cfft::seq_per_cta(LOGN) * cfft::threads_per_seq(LOGN))
    k_p3(FieldArgs a) {
  griddep_wait();
  constexpr int N = 1 << LOGN, T = cfft::threads_per_seq(LOGN), SEQ = cfft::seq_per_cta(LOGN);
  constexpr int NT = SEQ * T, L = buf_len(N);
  extern __shared__ __align__(16) float2 sm3[];
  const int tid = threadIdx.x, s = tid / T, t = tid % T;
  const int x0 = a.x_base + blockIdx.x * SEQ, xend = a.x_base + a.nrows;
  constexpr int PER = SEQ * N / NT;
  float2 v[PER];
#pragma unroll
  for (int q = 0; q < PER; q++) {
    const int idx = tid + q * NT, x = x0 + (idx >> LOGN), k = idx & (N - 1);
    v[q] = x < xend ? a.s_in[((size_t)(k >> a.lC) << (a.lC + a.lR)) + ((size_t)(x - a.x_base) << a.lC) + (k & (a.C - 1))]
                    : make_float2(0.f, 0.f);
  }
#pragma unroll
  for (int q = 0; q < PER; q++) {
    const int idx = tid + q * NT;
    sm3[(idx >> LOGN) * L + pad(idx & (N - 1))] = v[q];
  }
  __syncthreads();
  float2 *const A[1] = {sm3 + s * L};
  // in place, pairs (k, N - k) per thread: p = sX (IDCT), q = sY reversed (IDXST, eq 8e)
#pragma unroll
  for (int m = 0; m <= 8; m++) {   // k = t + m T < N / 2 (unrolled), k = N / 2 by thread 0
    if (m == 8 && t != 0) break;
    const int k = m < 8 ? t + m * T : N / 2;
    const float2 vk = A[0][pad(k)], vn = k ? A[0][pad(N - k)] : make_float2(0.f, 0.f);
    const float2 zk = inv_pre(vk.x, vn.y, vn.x, k ? vk.y : 0.f, __ldg(a.ph_y + k));
    if (k && k < N / 2) A[0][pad(N - k)] = inv_pre(vn.x, vk.y, vk.x, vn.y, __ldg(a.ph_y + N - k));
    A[0][pad(k)] = zk;
  }
  __syncthreads();
  cfft::fft<LOGN, true>(A, t, a.twf_y);
  const int x = x0 + s;
  if (x < xend)
#pragma unroll
    for (int m = 0; m < 16; m++) {
      const int y = t + m * T;
      const float2 z = A[0][pad(mk_pos(y, N))];
      a.xi[(size_t)x * N + y] = make_float2(0.5f * z.x, (y & 1) ? -0.5f * z.y : 0.5f * z.y);   // IDXST sign on xi_Y
    }
}

template <int LOGN>
constexpr size_t p1_smem() {
  return sizeof(float2) * cfft::seq_per_cta(LOGN) * buf_len(1 << LOGN) +
         sizeof(float) * (size_t)(1 << LOGN) * 2 * cfft::seq_per_cta(LOGN);
}
template <int LOGN, bool TIN = true>
constexpr size_t p2_smem() {
  return sizeof(float2) * 2 * p2_seq<LOGN, TIN>() * buf_len(1 << LOGN);
}
template <int LOGN>
constexpr size_t p3_smem() {
  return sizeof(float2) * cfft::seq_per_cta(LOGN) * buf_len(1 << LOGN);
}

template <class K>
cudaError_t set_smem(K kernel, size_t bytes) {
  return cudaFuncSetAttribute(kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)bytes);
}

template <int LOGN>
cudaError_t configure_one() {
  cudaError_t e;
  if ((e = set_smem(k_p1<unsigned long long, LOGN>, p1_smem<LOGN>())) != cudaSuccess) return e;
  if ((e = set_smem(k_p1<float, LOGN>, p1_smem<LOGN>())) != cudaSuccess) return e;
  if ((e = set_smem(k_p2<LOGN, true>, p2_smem<LOGN>())) != cudaSuccess) return e;
  if ((e = set_smem(k_p2<LOGN, false>, p2_smem<LOGN, false>())) != cudaSuccess) return e;
  return set_smem(k_p3<LOGN>, p3_smem<LOGN>());
}

template <int LOGN>
void launch_p1(const Ctx &c, const FieldArgs &a, bool int_map, cudaStream_t s) {
  constexpr int NT = cfft::seq_per_cta(LOGN) * cfft::threads_per_seq(LOGN);
  const int g = (a.nrows + 2 * cfft::seq_per_cta(LOGN) - 1) / (2 * cfft::seq_per_cta(LOGN));
  if (int_map)
    launch_chain(c.pdl, k_p1<unsigned long long, LOGN>, g, NT, p1_smem<LOGN>(), s, a);
  else
    launch_chain(c.pdl, k_p1<float, LOGN>, g, NT, p1_smem<LOGN>(), s, a);
}
template <int LOGN>
void launch_p2(const Ctx &c, const FieldArgs &a, bool tin, cudaStream_t s) {
  if (tin) {
    constexpr int SEQ = p2_seq<LOGN, true>(), NT = SEQ * cfft::threads_per_seq(LOGN);
    launch_chain(c.pdl, k_p2<LOGN, true>, (a.ncols + 2 * SEQ - 1) / (2 * SEQ), NT, p2_smem<LOGN, true>(), s, a);
  } else {
    constexpr int SEQ = p2_seq<LOGN, false>(), NT = SEQ * cfft::threads_per_seq(LOGN);
    launch_chain(c.pdl, k_p2<LOGN, false>, (a.ncols + 2 * SEQ - 1) / (2 * SEQ), NT, p2_smem<LOGN, false>(), s, a);
  }
}
template <int LOGN>
void launch_p3(const Ctx &c, const FieldArgs &a, cudaStream_t s) {
  constexpr int NT = cfft::seq_per_cta(LOGN) * cfft::threads_per_seq(LOGN);
  const int g = (a.nrows + cfft::seq_per_cta(LOGN) - 1) / cfft::seq_per_cta(LOGN);
  launch_chain(c.pdl, k_p3<LOGN>, g, NT, p3_smem<LOGN>(), s, a);
}

#define DP_FIELDS_DISPATCH(logn, call) \
  switch (logn) {                      \
    case 4: call(4); break;            \
    case 5: call(5); break;            \
    case 6: call(6); break;            \
    case 7: call(7); break;            \
    case 8: call(8); break;            \
    case 9: call(9); break;            \
    case 10: call(10); break;          \
    case 11: call(11); break;          \
    default: call(12); break;          \
  }

}  // namespace

// energy partials of P2: one per CTA
int p2_ctas(int mx, int my, bool hybrid) {
  const int logm = ilog2_int(mx);
  const int cols = 2 * (hybrid ? 1 : cfft::seq_per_cta(logm));
  return (my + cols - 1) / cols;
}

cudaError_t fields_configure() {
  cudaError_t e;
#define DP_CFG(L) \
  if ((e = configure_one<L>()) != cudaSuccess) return e;
  DP_CFG(4) DP_CFG(5) DP_CFG(6) DP_CFG(7) DP_CFG(8) DP_CFG(9) DP_CFG(10) DP_CFG(11) DP_CFG(12)
#undef DP_CFG
  return cudaSuccess;
}

bool fields_cta_ok(int log2mx, int log2my) { return log2mx >= 4 && log2mx <= 12 && log2my >= 4 && log2my <= 12; }

namespace {
FieldArgs field_args(const Ctx &c, const void *rho) {
  FieldArgs a;
  a.rho = rho;
  a.t_out = c.d_t;
  a.t_in = c.d_t;
  a.s_out = c.d_sxy;
  a.s_in = c.d_sxy;
  a.xi = c.d_xi;
  a.mx = c.mx;
  a.my = c.my;
  a.R = c.mx;
  a.C = c.my;
  a.lR = c.log2mx;
  a.lC = c.log2my;
  a.x_base = a.y_base = 0;
  a.nrows = c.mx;
  a.ncols = c.my;
  a.twf_x = c.d_twf_x;
  a.twf_y = c.d_twf_y;
  a.ph_x = c.d_ph_x;
  a.ph_y = c.d_ph_y;
  a.kx = c.d_kx;
  a.ky = c.d_ky;
  a.energy_part = c.d_part + c.n_wa_part + (c.n_regions > 0 && c.cur_region > 0 ? c.cur_region * c.n_en_part : 0);
  a.energy_scale = 0.5 * c.bx * c.by;
  return a;
}

// rank r of G: rows [r R, (r+1) R), columns [r C, (r+1) C); buffers as in the layout comment
FieldArgs shard_args(const Ctx &c, const void *rho, int r, int G, float *s1, const float *r1, float2 *s2,
                     const float2 *r2) {
  FieldArgs a = field_args(c, rho);
  a.R = c.mx / G;
  a.C = c.my / G;
  a.lR = ilog2_int(a.R);
  a.lC = ilog2_int(a.C);
  a.x_base = r * a.R;
  a.y_base = r * a.C;
  a.nrows = a.R;
  a.ncols = a.C;
  a.t_out = s1;
  a.t_in = r1;
  a.s_out = s2;
  a.s_in = r2;
  return a;
}
}  // namespace

// P1 -> P2 -> P3 on stream s; rho is the int64 map (c.d_rho) or a float map (debug hook)
void launch_fields_cta(const Ctx &c, const void *rho, bool int_map, cudaStream_t s) {
  const FieldArgs a = field_args(c, rho);
#define DP_P1(L) launch_p1<L>(c, a, int_map, s)
#define DP_P2(L) launch_p2<L>(c, a, true, s)
#define DP_P3(L) launch_p3<L>(c, a, s)
  DP_FIELDS_DISPATCH(c.log2my, DP_P1)
  DP_FIELDS_DISPATCH(c.log2mx, DP_P2)
  DP_FIELDS_DISPATCH(c.log2my, DP_P3)
#undef DP_P1
#undef DP_P2
#undef DP_P3
}

// P2 alone on t[x][y] as the warp-FFT row pass T1 writes it (the hybrid field path)
void launch_p2_rowmajor(const Ctx &c, cudaStream_t s) {
  const FieldArgs a = field_args(c, nullptr);
#define DP_P2(L) launch_p2<L>(c, a, false, s)
  DP_FIELDS_DISPATCH(c.log2mx, DP_P2)
#undef DP_P2
}

bool fields_shardable(const Ctx &c, int G) {
  if (!c.fft_cta || G < 1 || (G & (G - 1)) || c.mx % G || c.my % G) return false;   // R, C powers of two
  const int R = c.mx / G, C = c.my / G;
  // every P1 / P2 CTA lies inside one rank block: rows by 2 SEQ_y, columns by 2 SEQ_x
  return R % (2 * cfft::seq_per_cta(c.log2my)) == 0 && C % (2 * cfft::seq_per_cta(c.log2mx)) == 0;
}

// One rank's passes of the row-sharded solve (the caller moves the blocks between them):
// pass 1 = P1 on the rank's rows -> s1; pass 2 = P2 on its columns from r1 -> s2 (+ its energy
// slots); pass 3 = P3 on its rows from r2 -> its rows of xi.
void launch_fields_shard(const Ctx &c, int pass, const void *rho, bool int_map, int r, int G, float *s1,
                         const float *r1, float2 *s2, const float2 *r2, cudaStream_t s) {
  const FieldArgs a = shard_args(c, rho, r, G, s1, r1, s2, r2);
#define DP_P1(L) launch_p1<L>(c, a, int_map, s)
#define DP_P2(L) launch_p2<L>(c, a, true, s)
#define DP_P3(L) launch_p3<L>(c, a, s)
  if (pass == 1) DP_FIELDS_DISPATCH(c.log2my, DP_P1)
  if (pass == 2) DP_FIELDS_DISPATCH(c.log2mx, DP_P2)
  if (pass == 3) DP_FIELDS_DISPATCH(c.log2my, DP_P3)
#undef DP_P1
#undef DP_P2
#undef DP_P3
}

}  // namespace dp
