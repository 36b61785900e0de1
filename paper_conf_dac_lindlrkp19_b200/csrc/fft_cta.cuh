// fft_cta.cuh — CTA-level complex FFT (Stockham autosort, radix 16, in place) for the field
// transforms.
//
// One sequence of N = 2^LOGN points is transformed by T = N/16 threads (16 points per thread)
// through one padded shared buffer: radix-16 stages, then one stage of radix 2^(LOGN mod 4)
// (each thread then runs 16/R butterflies).  Stockham DIT: the stage with sub-length Ns reads
// src[j + r N/R], multiplies by W_{Ns R}^{r (j mod Ns)}, runs a radix-R DFT in registers and
// writes dst[(j - j mod Ns) R + j mod Ns + r Ns]; output in natural order, no bit reversal.
// Every stage reads the 16 points t + m T (m < 16) of its thread whatever R is, so a stage is
// read all -> barrier -> compute -> write all -> barrier on ONE buffer (in place).  NB buffers
// can be transformed in lockstep (two independent sequences per thread: the column pass's pair
// of inverse transforms), which doubles the work between two barriers.  A CTA runs SEQ
// sequences side by side (SEQ T threads, about 128).  Buffers are padded by one float2 per 16
// entries: the radix-16 stride-16 writes of the first stage then fall on distinct bank pairs.
//
// Round 2 replaced the radix-8 / 8-points-per-thread / ping-pong version (4 stages, 2 buffers,
// 256-thread CTAs): at 1024 points it ran one CTA of 256 threads per two sequences and measured
// 13-26 us per pass alone.
#pragma once

#include "fft_warp.cuh"

namespace dp {
namespace cfft {

__host__ __device__ constexpr int pad(int e) { return e + (e >> 4); }
__host__ __device__ constexpr int buf_len(int n) { return n + (n >> 4) + 1; }   // float2 per padded buffer
__host__ __device__ constexpr int threads_per_seq(int logn) { return logn >= 4 ? (1 << logn) / 16 : 1; }
// sequences per CTA: about 128 threads, at most 16 sequences
__host__ __device__ constexpr int seq_per_cta(int logn) {
  return threads_per_seq(logn) >= 128 ? 1 : (128 / threads_per_seq(logn) > 16 ? 16 : 128 / threads_per_seq(logn));
}

__device__ __forceinline__ float2 cmul(float2 a, float2 b) {
  return make_float2(a.x * b.x - a.y * b.y, a.x * b.y + a.y * b.x);
}

// One in-place Stockham DIT stage of radix R on NB buffers (thread t of T = N/16).
// twf[k] = exp(-2 pi i k / N), k < N (fp64-rounded table); INV uses the conjugate
// (unnormalised inverse DFT).  Ends with a block barrier (the output is visible).
template <int N, int R, bool INV, int NB>
__device__ __forceinline__ void stage(float2 *const (&A)[NB], int Ns, int t, const float2 *__restrict__ twf) {
  constexpr int T = N / 16, B = 16 / R, LR = wfft::log2_c(R);
  // twiddles first: they depend on t only, so their (L1 / L2) latency overlaps the shared reads
  // and the barrier instead of following them
  float2 w[B][R];
  if (Ns > 1) {
#pragma unroll
    for (int q = 0; q < B; q++) {
      const int k0 = ((t + q * T) & (Ns - 1)) * (N / (Ns * R));   // W_{Ns R}^{r jm} = W_N^{r k0}, r k0 < N
#pragma unroll
      for (int r = 1; r < R; r++) w[q][r] = __ldg(twf + r * k0);
    }
  }
  float2 v[NB][16];
#pragma unroll
  for (int b = 0; b < NB; b++)
#pragma unroll
    for (int m = 0; m < 16; m++) v[b][m] = A[b][pad(t + m * T)];   // m = q + B r: j_q + r N / R
  __syncthreads();
#pragma unroll
  for (int q = 0; q < B; q++) {
    const int j = t + q * T, jm = j & (Ns - 1);
    float2 u[NB][R];
#pragma unroll
    for (int b = 0; b < NB; b++)
#pragma unroll
      for (int r = 0; r < R; r++) u[b][r] = v[b][q + B * r];
    if (Ns > 1) {
#pragma unroll
      for (int r = 1; r < R; r++) {
        float2 wr = w[q][r];
        if (INV) wr.y = -wr.y;
#pragma unroll
        for (int b = 0; b < NB; b++) u[b][r] = cmul(u[b][r], wr);
      }
    }
    const int base = (j - jm) * R + jm;
#pragma unroll
    for (int b = 0; b < NB; b++) {
      wfft::reg_dft<R, INV>(u[b]);   // u[m] = X[brev(m)]
#pragma unroll
      for (int r = 0; r < R; r++) A[b][pad(base + r * Ns)] = u[b][wfft::brev_c(r, LR)];
    }
  }
  __syncthreads();
}

// In-place FFT of the NB sequences in A (natural order, padded) by thread t in [0, T) of its
// group.  Every thread of the CTA must call it (block barriers); the caller synchronises before
// (input written); the output is in natural order and visible to the whole CTA on return.
template <int LOGN, bool INV, int NB = 1>
__device__ __forceinline__ void fft(float2 *const (&A)[NB], int t, const float2 *__restrict__ twf) {
  constexpr int N = 1 << LOGN, S16 = LOGN / 4, REM = LOGN % 4;
#pragma unroll
  for (int s = 0; s < S16; s++) stage<N, 16, INV, NB>(A, 1 << (4 * s), t, twf);
  if constexpr (REM != 0) stage<N, (1 << REM), INV, NB>(A, 1 << (4 * S16), t, twf);
}

}  // namespace cfft
}  // namespace dp
