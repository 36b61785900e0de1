// fields.cu — the spectral Poisson solve of one evaluation (steps 2-3 of P:253-256) in three
// passes over the bin map, each a CTA-level FFT (fft_cta.cuh) with 8 points per thread.
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
// values per output row (16-32 bytes): no strided column reads.  The spectrum of P2 stays in
// shared memory between the forward and the inverse x transforms.
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
__device__ __forceinline__ float map_value(unsigned long long v) {
  return (float)((double)(long long)v * (1.0 / (double)(1ll << kRhoScaleLog2)));
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
  int R, C;               // rows / columns per rank block
  int x_base, y_base;     // this rank's first row / column
  int nrows, ncols;       // rows of P1 / P3, columns of P2
  const float2 *twf_x, *twf_y;   // exp(-2 pi i k / N), k < N
  const float2 *ph_x, *ph_y;     // exp(-i pi k / 2N), k < N
  const float *kx, *ky;          // wavenumbers (A12)
  double *energy_part;           // one slot per P2 CTA
  double energy_scale;           // 1/2 b_x b_y
};

// ---- P1: rows (2p, 2p+1) of rho -> DCT over y -> tT[y][x] ----------------------------------
template <class IN, int LOGN>
__global__ void __launch_bounds__(cfft::seq_per_cta(LOGN) * cfft::threads_per_seq(LOGN))
    k_p1(FieldArgs a) {
  griddep_wait();
  constexpr int N = 1 << LOGN, T = cfft::threads_per_seq(LOGN), SEQ = cfft::seq_per_cta(LOGN);
  constexpr int NT = SEQ * T, ROWS = 2 * SEQ, L = buf_len(N);
  extern __shared__ __align__(16) float2 sm1[];
  float *out = reinterpret_cast<float *>(sm1 + 2 * SEQ * L);   // [N][ROWS]
  const IN *rho = reinterpret_cast<const IN *>(a.rho);
  const int tid = threadIdx.x, s = tid / T, t = tid % T;
  const int x0 = a.x_base + blockIdx.x * ROWS, xend = a.x_base + a.nrows;
  float2 *A = sm1 + (2 * s) * L, *B = A + L;
  // load: row x0 + rr (coalesced) -> real (rr even) / imaginary (rr odd) part of sequence rr/2,
  // at its Makhoul position.  Every load is issued before the first use (unrolled: a loop
  // that waits on each load serialises the global latency)
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
    float *slot = reinterpret_cast<float *>(sm1 + (rr & ~1) * L + pad(mk_pos(col, N)));
    slot[rr & 1] = map_value(v[q]);
  }
  __syncthreads();
  const float2 *Z = cfft::fft<LOGN, false>(A, B, t, a.twf_y);
  const float scale = 2.f / N;
  for (int k = t; k < N; k += T) {
    const float2 d = dct_post(Z[pad(k)], Z[pad((N - k) & (N - 1))], __ldg(a.ph_y + k), scale);
    out[k * ROWS + 2 * s] = d.x;
    out[k * ROWS + 2 * s + 1] = d.y;
  }
  __syncthreads();
  // transposed store: tT[k][x0 .. x0 + ROWS) (unsharded) / S1[k / C][k % C][x0 - x_base ..]
  const size_t CR = (size_t)a.C * a.R;
  if (ROWS % 4 == 0 && x0 + ROWS <= xend) {
    for (int idx = tid; idx < N * (ROWS / 4); idx += NT) {
      const int k = idx / (ROWS / 4), q = idx % (ROWS / 4);
      *reinterpret_cast<float4 *>(a.t_out + (size_t)(k / a.C) * CR + (size_t)(k % a.C) * a.R + (x0 - a.x_base) + 4 * q) =
          *reinterpret_cast<const float4 *>(out + k * ROWS + 4 * q);
    }
  } else {
    for (int idx = tid; idx < N * ROWS; idx += NT) {
      const int k = idx / ROWS, c = idx % ROWS;
      if (x0 + c < xend)
        a.t_out[(size_t)(k / a.C) * CR + (size_t)(k % a.C) * a.R + (x0 - a.x_base) + c] = out[idx];
    }
  }
}

// ---- P2: columns (2p, 2p+1) (rows of tT) -> DCT over x, energy, scaling, inverse over x ----
// TIN: t stored transposed, tT[y][x] (after P1); otherwise t[x][y] (after the warp-FFT T1):
// the CTA then reads its COLS adjacent columns as 4 COLS-byte row segments.
// P2 of the hybrid path runs one column pair per CTA (SEQ = 1): half the shared memory and
// threads of a CTA, so its CTAs fit beside the WA kernel's (the unsharded / sharded CTA-FFT
// path keeps seq_per_cta)
template <int LOGM, bool TIN>
constexpr int p2_seq() { return TIN ? cfft::seq_per_cta(LOGM) : 1; }

template <int LOGM, bool TIN = true>
__global__ void __launch_bounds__(p2_seq<LOGM, TIN>() * cfft::threads_per_seq(LOGM))
    k_p2(FieldArgs a) {
  griddep_wait();
  constexpr int M = 1 << LOGM, T = cfft::threads_per_seq(LOGM), SEQ = p2_seq<LOGM, TIN>();
  constexpr int NT = SEQ * T, COLS = 2 * SEQ, L = buf_len(M);
  extern __shared__ __align__(16) float2 sm2[];
  float2 *spec = sm2 + 2 * SEQ * L;    // [COLS][M] (A_X, A_Y)
  float2 *out = spec + COLS * M;       // [M][COLS] (sX, sY)
  __shared__ double s_red[NT / 32 > 0 ? NT / 32 : 1];
  const int tid = threadIdx.x, s = tid / T, t = tid % T;
  const int y0 = a.y_base + blockIdx.x * COLS, my = a.my, yend = a.y_base + a.ncols;
  const size_t CR = (size_t)a.C * a.R;
  float2 *A = sm2 + (2 * s) * L, *B = A + L;
  constexpr int PER = COLS * M / NT;
  float v[PER];
#pragma unroll
  for (int q = 0; q < PER; q++) {
    const int idx = tid + q * NT;
    const int c = TIN ? idx >> LOGM : idx % COLS, x = TIN ? idx & (M - 1) : idx / COLS;
    v[q] = (y0 + c < yend) ? (TIN ? a.t_in[(size_t)(x / a.R) * CR + (size_t)(y0 + c - a.y_base) * a.R + (x % a.R)]
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
  const float2 *Z = cfft::fft<LOGM, false>(A, B, t, a.twf_x);
  // spectrum of columns v0 = y0 + 2s, v1 = v0 + 1: energy (Parseval, A8) and scaling (9c/9d)
  const float scale = 2.f / M;
  const int v0 = y0 + 2 * s, v1 = v0 + 1;
  const bool ok = v1 < yend;
  const float ky0 = ok ? __ldg(a.ky + v0) : 0.f, ky1 = ok ? __ldg(a.ky + v1) : 0.f;
  const double wv0 = (v0 == 0) ? 0.25 * my : 0.5 * my, wv1 = 0.5 * my;
  double e = 0.0;
  for (int u = t; u < M; u += T) {
    const float2 d = dct_post(Z[pad(u)], Z[pad((M - u) & (M - 1))], __ldg(a.ph_x + u), scale);
    const float kx = __ldg(a.kx + u);
    const double wu = (u == 0) ? 0.25 * M : 0.5 * M;
    const float ik0 = (!ok || (u == 0 && v0 == 0)) ? 0.f : fast_rcp(kx * kx + ky0 * ky0);   // a_00 / k^2 := 0
    const float ik1 = ok ? fast_rcp(kx * kx + ky1 * ky1) : 0.f;
    e += wu * (wv0 * (double)(d.x * d.x * ik0) + wv1 * (double)(d.y * d.y * ik1));
    spec[(2 * s) * M + u] = make_float2(d.x * kx * ik0, d.x * ky0 * ik0);
    spec[(2 * s + 1) * M + u] = make_float2(d.y * kx * ik1, d.y * ky1 * ik1);
  }
  __syncthreads();
  // inverse over x, two rounds (even, then odd columns): IDXST_x(A_X) + i IDCT_x(A_Y)
#pragma unroll 1
  for (int h = 0; h < 2; h++) {
    const int c = 2 * s + h;
    const float2 *S = spec + c * M;
    for (int k = t; k < M; k += T) {
      const float2 ak = S[k], ank = k ? S[M - k] : make_float2(0.f, 0.f);
      // p = A_X reversed (IDXST via eq 8e: x'_t = x_{N-t}, x'_0 = 0), q = A_Y (IDCT)
      A[pad(k)] = inv_pre(ank.x, ak.y, k ? ak.x : 0.f, ank.y, __ldg(a.ph_x + k));
    }
    __syncthreads();
    const float2 *W = cfft::fft<LOGM, true>(A, B, t, a.twf_x);
    for (int x = t; x < M; x += T) {
      const float2 z = W[pad(mk_pos(x, M))];
      out[x * COLS + c] = make_float2((x & 1) ? -0.5f * z.x : 0.5f * z.x, 0.5f * z.y);   // IDXST sign (-1)^x
    }
    __syncthreads();
  }
  // transposed store: sxy[x][y0 .. y0 + COLS) (unsharded) / S2[x / R][x % R][y0 - y_base ..]
  if (COLS % 2 == 0 && y0 + COLS <= yend) {
    for (int idx = tid; idx < M * (COLS / 2); idx += NT) {
      const int x = idx / (COLS / 2), q = idx % (COLS / 2);
      *reinterpret_cast<float4 *>(a.s_out + (size_t)(x / a.R) * CR + (size_t)(x % a.R) * a.C + (y0 - a.y_base) + 2 * q) =
          *reinterpret_cast<const float4 *>(out + x * COLS + 2 * q);
    }
  } else {
    for (int idx = tid; idx < M * COLS; idx += NT) {
      const int x = idx / COLS, c = idx % COLS;
      if (y0 + c < yend) a.s_out[(size_t)(x / a.R) * CR + (size_t)(x % a.R) * a.C + (y0 - a.y_base) + c] = out[idx];
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
  const size_t CR = (size_t)a.C * a.R;
  float2 *A = sm3 + (2 * s) * L, *B = A + L;
  constexpr int PER = SEQ * N / NT;
  float2 v[PER];
#pragma unroll
  for (int q = 0; q < PER; q++) {
    const int idx = tid + q * NT, x = x0 + (idx >> LOGN), k = idx & (N - 1);
    v[q] = x < xend ? a.s_in[(size_t)(k / a.C) * CR + (size_t)(x - a.x_base) * a.C + (k % a.C)] : make_float2(0.f, 0.f);
  }
#pragma unroll
  for (int q = 0; q < PER; q++) {
    const int idx = tid + q * NT;
    sm3[(2 * (idx >> LOGN)) * L + pad(idx & (N - 1))] = v[q];
  }
  __syncthreads();
  // in place, pairs (k, N - k) per thread: p = sX (IDCT), q = sY reversed (IDXST, eq 8e)
  for (int k = t; k <= N / 2; k += T) {
    const float2 vk = A[pad(k)], vn = k ? A[pad(N - k)] : make_float2(0.f, 0.f);
    const float2 zk = inv_pre(vk.x, vn.y, vn.x, k ? vk.y : 0.f, __ldg(a.ph_y + k));
    if (k && k < N / 2) A[pad(N - k)] = inv_pre(vn.x, vk.y, vk.x, vn.y, __ldg(a.ph_y + N - k));
    A[pad(k)] = zk;
  }
  __syncthreads();
  const float2 *W = cfft::fft<LOGN, true>(A, B, t, a.twf_y);
  const int x = x0 + s;
  if (x < xend)
    for (int y = t; y < N; y += T) {
      const float2 z = W[pad(mk_pos(y, N))];
      a.xi[(size_t)x * N + y] = make_float2(0.5f * z.x, (y & 1) ? -0.5f * z.y : 0.5f * z.y);   // IDXST sign on xi_Y
    }
}

template <int LOGN>
constexpr size_t p1_smem() {
  return sizeof(float2) * 2 * cfft::seq_per_cta(LOGN) * buf_len(1 << LOGN) +
         sizeof(float) * (size_t)(1 << LOGN) * 2 * cfft::seq_per_cta(LOGN);
}
template <int LOGN, bool TIN = true>
constexpr size_t p2_smem() {
  return sizeof(float2) * (2 * p2_seq<LOGN, TIN>() * buf_len(1 << LOGN) +
                           2 * (size_t)(2 * p2_seq<LOGN, TIN>()) * (1 << LOGN));
}
template <int LOGN>
constexpr size_t p3_smem() {
  return sizeof(float2) * 2 * cfft::seq_per_cta(LOGN) * buf_len(1 << LOGN);
}

template <int LOGN>
cudaError_t configure_one() {
  cudaError_t e;
  if ((e = cudaFuncSetAttribute(k_p1<unsigned long long, LOGN>, cudaFuncAttributeMaxDynamicSharedMemorySize,
                                (int)p1_smem<LOGN>())) != cudaSuccess)
    return e;
  if ((e = cudaFuncSetAttribute(k_p1<float, LOGN>, cudaFuncAttributeMaxDynamicSharedMemorySize,
                                (int)p1_smem<LOGN>())) != cudaSuccess)
    return e;
  if ((e = cudaFuncSetAttribute(k_p2<LOGN, true>, cudaFuncAttributeMaxDynamicSharedMemorySize,
                                (int)p2_smem<LOGN>())) != cudaSuccess)
    return e;
  if ((e = cudaFuncSetAttribute(k_p2<LOGN, false>, cudaFuncAttributeMaxDynamicSharedMemorySize,
                                (int)p2_smem<LOGN, false>())) != cudaSuccess)
    return e;
  return cudaFuncSetAttribute(k_p3<LOGN>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)p3_smem<LOGN>());
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
  if (!c.fft_cta || G < 1 || c.mx % G || c.my % G) return false;
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
