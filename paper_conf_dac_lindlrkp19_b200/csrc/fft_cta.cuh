// fft_cta.cuh — CTA-level complex FFT (Stockham autosort, radix 8) for the field transforms.
//
// One sequence of N = 2^LOGN points is transformed by T = N/8 threads (8 points per thread)
// through shared memory: an optional first stage of radix 2^(LOGN mod 3), then radix-8 stages
// (Stockham DIT: stage with sub-length Ns reads src[j + r N/R], twiddles W_{Ns R}^{r (j mod Ns)},
// a radix-R DFT in registers, writes dst[(j - j mod Ns) R + j mod Ns + r Ns]; output in
// natural order, no bit reversal).  A CTA runs SEQ sequences side by side (SEQ T threads) and
// every stage ends in one block barrier.  Buffers are padded by one float2 per 8 entries, which
// makes the strided stage writes bank-conflict free.
//
// Why not the warp FFT (fft_warp.cuh): a warp holding 1024 points leaves a 1024^2 map with 512
// to 1024 warps per pass (<= 7 per SM), and the transforms were latency bound at 10-16 us per
// pass; at 8 points per thread the same pass has 4x the warps in flight.
#pragma once

#include "fft_warp.cuh"

namespace dp {
namespace cfft {

__host__ __device__ constexpr int pad(int e) { return e + (e >> 3); }
__host__ __device__ constexpr int buf_len(int n) { return n + (n >> 3); }   // float2 per padded buffer
__host__ __device__ constexpr int threads_per_seq(int logn) { return logn >= 3 ? (1 << logn) / 8 : 1; }
// sequences per CTA: about 256 threads, at most 16 sequences
__host__ __device__ constexpr int seq_per_cta(int logn) {
  return threads_per_seq(logn) >= 256 ? 1 : (256 / threads_per_seq(logn) > 16 ? 16 : 256 / threads_per_seq(logn));
}

__device__ __forceinline__ float2 cmul(float2 a, float2 b) {
  return make_float2(a.x * b.x - a.y * b.y, a.x * b.y + a.y * b.x);
}

// One Stockham DIT stage of radix R for group j (j < N / R).  twf[k] = exp(-2 pi i k / N), k < N
// (fp64-rounded table); INV uses the conjugate (unnormalised inverse DFT).
template <int N, int R, bool INV>
__device__ __forceinline__ void stage(const float2 *src, float2 *dst, int Ns, int j, const float2 *__restrict__ twf) {
  constexpr int LR = wfft::log2_c(R);
  float2 v[R];
  const int jm = j & (Ns - 1);
#pragma unroll
  for (int r = 0; r < R; r++) v[r] = src[pad(j + r * (N / R))];
  if (Ns > 1) {
    const int k0 = jm * (N / (Ns * R));   // W_{Ns R}^{r jm} = W_N^{r k0}, r k0 < N
#pragma unroll
    for (int r = 1; r < R; r++) {
      float2 w = __ldg(twf + r * k0);
      if (INV) w.y = -w.y;
      v[r] = cmul(v[r], w);
    }
  }
  wfft::reg_dft<R, INV>(v);   // v[m] = X[brev(m)]
  const int base = (j - jm) * R + jm;
#pragma unroll
  for (int r = 0; r < R; r++) dst[pad(base + r * Ns)] = v[wfft::brev_c(r, LR)];
}

// FFT of the sequence in A (natural order, padded) by thread t in [0, T) of its group; B is the
// second buffer.  Every thread of the CTA must call it (block barriers); returns the buffer
// holding the result (natural order).  The caller synchronises before (input written).
template <int LOGN, bool INV>
__device__ __forceinline__ float2 *fft(float2 *A, float2 *B, int t, const float2 *__restrict__ twf) {
  constexpr int N = 1 << LOGN, T = threads_per_seq(LOGN), REM = LOGN % 3;
  float2 *src = A, *dst = B;
  int Ns = 1;
  if (REM) {
    constexpr int R = 1 << REM;
#pragma unroll
    for (int g = 0; g < (N / R) / T; g++) stage<N, R, INV>(src, dst, 1, t + g * T, twf);
    __syncthreads();
    float2 *tmp = src; src = dst; dst = tmp;
    Ns = R;
  }
#pragma unroll
  for (int s = 0; s < (LOGN - REM) / 3; s++) {
    stage<N, 8, INV>(src, dst, Ns, t, twf);
    __syncthreads();
    float2 *tmp = src; src = dst; dst = tmp;
    Ns *= 8;
  }
  return src;
}

}  // namespace cfft
}  // namespace dp
