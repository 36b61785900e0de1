// fft_warp.cuh — warp-level complex FFT for the DCT/IDCT/IDXST transforms (sm_100a).
//
// One warp transforms 1024 complex points at a time: B = 1024 / N independent sequences of
// length N = 32 K (K = 1 .. 32).  Four-step decomposition n = n1 + 32 n2, k = K k1 + k2:
//   pass 1  every lane (n1) runs a K-point DFT over its K registers (n2)         [registers]
//   twiddle multiply by W_N^{n1 k2} (table [k2][n1], coalesced)
//   transpose through the warp's padded shared buffer (conflict-free both ways)
//   pass 2  every lane (one (sequence, k2) pair) runs a 32-point DFT over n1     [registers]
//   output  X[K k1 + k2] written to the shared buffer in natural order.
// No block barriers: only __syncwarp.  Both passes are radix-2 DIF with compile-time twiddles
// (W_32^t constants).  Replaces the shared-memory radix-4 FFT whose 5 block barriers per
// transform and index arithmetic made the transforms latency-bound.
#pragma once

namespace dp {
namespace wfft {

constexpr int kPts = 1024;                       // complex points per warp call
constexpr int kBufPad = kPts + kPts / 32;        // padded buffer length (float2)

// padded position of logical index q (one float2 of padding per 32)
__device__ __forceinline__ int pad(int q) { return q + (q >> 5); }

// W_32^t = exp(-2 pi i t / 32) for t in [0, 16)
__host__ __device__ constexpr float cos32(int t) {
  return t == 0 ? 1.000000000e+00f : t == 1 ? 9.807852804e-01f : t == 2 ? 9.238795325e-01f
       : t == 3 ? 8.314696123e-01f : t == 4 ? 7.071067812e-01f : t == 5 ? 5.555702330e-01f
       : t == 6 ? 3.826834324e-01f : t == 7 ? 1.950903220e-01f : t == 8 ? 0.0f
       : t == 9 ? -1.950903220e-01f : t == 10 ? -3.826834324e-01f : t == 11 ? -5.555702330e-01f
       : t == 12 ? -7.071067812e-01f : t == 13 ? -8.314696123e-01f : t == 14 ? -9.238795325e-01f
       : -9.807852804e-01f;
}
__host__ __device__ constexpr float sin32(int t) { return t <= 8 ? cos32(8 - t) : cos32(t - 8); }

__host__ __device__ constexpr int brev_c(int v, int bits) {
  int r = 0;
  for (int b = 0; b < bits; b++) r |= ((v >> b) & 1) << (bits - 1 - b);
  return r;
}
__host__ __device__ constexpr int log2_c(int v) { return v <= 1 ? 0 : 1 + log2_c(v >> 1); }

// a *= W_32^t (forward) or conj (inverse); t compile-time after unrolling
template <bool INV>
__device__ __forceinline__ float2 tw32(float2 a, int t) {
  if (t == 0) return a;
  if (t == 8) return INV ? make_float2(-a.y, a.x) : make_float2(a.y, -a.x);   // * (+-i)
  const float c = cos32(t), s = INV ? sin32(t) : -sin32(t);                    // w = c + i s
  return make_float2(a.x * c - a.y * s, a.x * s + a.y * c);
}

// In-register radix-2 DIF DFT of a[base .. base + S): afterwards a[base + m] = X[brev(m)].
template <int S, bool INV>
__device__ __forceinline__ void reg_dft(float2 *a) {
#pragma unroll
  for (int len = S; len >= 2; len >>= 1) {
#pragma unroll
    for (int st = 0; st < S; st += len) {
#pragma unroll
      for (int i = 0; i < len / 2; i++) {
        const float2 u = a[st + i], v = a[st + i + len / 2];
        a[st + i] = make_float2(u.x + v.x, u.y + v.y);
        a[st + i + len / 2] = tw32<INV>(make_float2(u.x - v.x, u.y - v.y), i * (32 / len));
      }
    }
  }
}

// Per-lane twiddles of pass 1, loaded up front so their latency overlaps the data loads:
// tw[k2] = W_N^{lane k2} for k2 in [1, K) (tw[0] unused).
template <int LOGN>
__device__ __forceinline__ void load_twiddles(float2 (&tw)[32], const float2 *__restrict__ tw2) {
  constexpr int K = (1 << LOGN) / 32;
  const int lane = threadIdx.x & 31;
#pragma unroll
  for (int k2 = 1; k2 < K; k2++) tw[k2] = __ldg(tw2 + k2 * 32 + lane);
}

// Warp FFT of B = 1024 / N sequences.  In: a[s K + j] = x_s[lane + 32 j].  tw = this lane's
// twiddles from load_twiddles (tw2[k2 * 32 + n1] = W_N^{n1 k2}, an fp64-rounded table).  Out: buf[pad(s N + k)] = X_s[k] (unnormalised; INV uses
// conjugate twiddles).  buf is this warp's kBufPad-entry shared buffer; a[] is clobbered.
// Twiddles are read from the (L1-resident) table right before use: holding all 31 of them in
// registers for the whole transform cost ~60 registers per thread, which kept the WA kernel's
// CTAs off the SMs that run a transform.
template <int LOGN, bool INV>
__device__ __forceinline__ void warp_fft(float2 (&a)[32], float2 *buf, const float2 *__restrict__ tw2) {
  constexpr int N = 1 << LOGN, K = N / 32, B = kPts / N, LK = LOGN - 5;
  static_assert(K >= 1 && K <= 32, "warp_fft: N in [32, 1024]");
  const int lane = threadIdx.x & 31;
  // pass 1: K-point DFTs per lane; twiddle; scatter to the transpose rows
#pragma unroll
  for (int s = 0; s < B; s++) {
    reg_dft<K, INV>(a + s * K);
#pragma unroll
    for (int m = 0; m < K; m++) {
      const int k2 = brev_c(m, LK);
      float2 v = a[s * K + m];
      if (k2 != 0) {
        float2 w = __ldg(tw2 + k2 * 32 + lane);
        if (INV) w.y = -w.y;
        v = make_float2(v.x * w.x - v.y * w.y, v.x * w.y + v.y * w.x);
      }
      buf[(s * K + k2) * 33 + lane] = v;
    }
  }
  __syncwarp();
  // pass 2: lane L = s K + k2 takes the 32 values over n1
  float2 z[32];
#pragma unroll
  for (int n1 = 0; n1 < 32; n1++) z[n1] = buf[lane * 33 + n1];
  __syncwarp();
  reg_dft<32, INV>(z);
  const int s = lane >> LK, k2 = lane & (K - 1);
#pragma unroll
  for (int m = 0; m < 32; m++) buf[pad(s * N + K * brev_c(m, 5) + k2)] = z[m];
  __syncwarp();
}

}  // namespace wfft
}  // namespace dp
