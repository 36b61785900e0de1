// Design-probe microbenchmark (not product code): on-chip op rates on B200 that decide the
// WA / scatter kernel structure — shared-memory float atomics, shuffles, MUFU ex2, FP64,
// and coalesced vector red.global.add (the privatised-tile flush).
#include <cstdio>
#include <cstdlib>
#include <cuda_runtime.h>
#define CK(x) do { cudaError_t e = (x); if (e != cudaSuccess) { printf("CUDA %s at %d\n", cudaGetErrorString(e), __LINE__); exit(1);} } while (0)

__global__ void k_smem_atomic(float* out, int iters, int mask, int stride) {
  __shared__ float s[8192];
  for (int i = threadIdx.x; i < 8192; i += blockDim.x) s[i] = 0.f;
  __syncthreads();
  unsigned h = threadIdx.x * 2654435761u + blockIdx.x;
  for (int i = 0; i < iters; i++) {
    h = h * 1664525u + 1013904223u;
    int a = stride ? ((threadIdx.x * stride + i) & mask) : ((h >> 8) & mask);
    atomicAdd(&s[a], 1.0f);
  }
  __syncthreads();
  if (threadIdx.x == 0) out[blockIdx.x] = s[5];
}
__global__ void k_shfl(float* out, int iters) {
  float v = threadIdx.x;
  for (int i = 0; i < iters; i++) {
    v += __shfl_xor_sync(0xffffffff, v, 1);
    v += __shfl_xor_sync(0xffffffff, v, 2);
    v += __shfl_xor_sync(0xffffffff, v, 4);
    v += __shfl_xor_sync(0xffffffff, v, 8);
  }
  if (v == 1.2345f) out[0] = v;
}
__global__ void k_ex2(float* out, int iters) {
  float a = threadIdx.x * 1e-3f, b = a + 0.1f, c = a + 0.2f, d = a + 0.3f;
  for (int i = 0; i < iters; i++) {
    asm volatile("ex2.approx.ftz.f32 %0, %0;" : "+f"(a)); asm volatile("ex2.approx.ftz.f32 %0, %0;" : "+f"(b));
    asm volatile("ex2.approx.ftz.f32 %0, %0;" : "+f"(c)); asm volatile("ex2.approx.ftz.f32 %0, %0;" : "+f"(d));
    a *= -0.5f; b *= -0.5f; c *= -0.5f; d *= -0.5f;
  }
  if (a + b + c + d == 1.2345f) out[0] = a;
}
__global__ void k_dfma(double* out, int iters) {
  double a = threadIdx.x, b = a + 1, c = a + 2, d = a + 3;
  for (int i = 0; i < iters; i++) { a = fma(a, 0.999, 1e-3); b = fma(b, 0.999, 1e-3); c = fma(c, 0.999, 1e-3); d = fma(d, 0.999, 1e-3); }
  if (a + b + c + d == 1.2345) out[0] = a;
}
__global__ void k_red_coalesced_v4(float4* dst, int n4, int reps) {
  for (int r = 0; r < reps; r++)
    for (int i = blockIdx.x * blockDim.x + threadIdx.x; i < n4; i += gridDim.x * blockDim.x)
      asm volatile("red.global.add.v4.f32 [%0], {%1, %2, %3, %4};" :: "l"(dst + i), "f"(1.0f), "f"(2.0f), "f"(1.0f), "f"(2.0f) : "memory");
}
__global__ void k_red_coalesced_f1(float* dst, int n, int reps) {
  for (int r = 0; r < reps; r++)
    for (int i = blockIdx.x * blockDim.x + threadIdx.x; i < n; i += gridDim.x * blockDim.x)
      asm volatile("red.global.add.f32 [%0], %1;" :: "l"(dst + i), "f"(1.0f) : "memory");
}
__global__ void k_store_coalesced_v4(float4* dst, int n4, int reps) {
  for (int r = 0; r < reps; r++)
    for (int i = blockIdx.x * blockDim.x + threadIdx.x; i < n4; i += gridDim.x * blockDim.x)
      dst[i] = make_float4(1.f, 2.f, 1.f, (float)r);
}

template <class F> float timeit(F f, int reps = 10) {
  cudaEvent_t a, b; CK(cudaEventCreate(&a)); CK(cudaEventCreate(&b));
  f(); CK(cudaDeviceSynchronize());
  CK(cudaEventRecord(a)); for (int i = 0; i < reps; i++) f(); CK(cudaEventRecord(b)); CK(cudaEventSynchronize(b));
  float ms; CK(cudaEventElapsedTime(&ms, a, b)); return ms * 1000.f / reps;
}

int main() {
  int sms; CK(cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0));
  float* out; CK(cudaMalloc(&out, 1 << 24));
  double* dout; CK(cudaMalloc(&dout, 1 << 20));
  const int blocks = sms * 4, threads = 256, iters = 4096;
  double lanes = (double)blocks * threads * iters;
  float t;
  t = timeit([&] { k_smem_atomic<<<blocks, threads>>>(out, iters, 8191, 0); });
  printf("smem atomicAdd f32 random/8K: %.1f us  -> %.2f lane-ops/clk/SM @1.965GHz (%.1f G lane-op/s)\n", t, lanes / (t * 1e-6) / sms / 1.965e9, lanes / t / 1e3);
  t = timeit([&] { k_smem_atomic<<<blocks, threads>>>(out, iters, 8191, 1); });
  printf("smem atomicAdd f32 lane-distinct: %.1f us -> %.2f lane-ops/clk/SM (%.1f G/s)\n", t, lanes / (t * 1e-6) / sms / 1.965e9, lanes / t / 1e3);
  t = timeit([&] { k_smem_atomic<<<blocks, threads>>>(out, iters, 63, 0); });
  printf("smem atomicAdd f32 random/64 (contended): %.1f us -> %.2f lane-ops/clk/SM\n", t, lanes / (t * 1e-6) / sms / 1.965e9);
  t = timeit([&] { k_shfl<<<blocks, threads>>>(out, iters); });
  printf("shfl: %.1f us -> %.2f warp-shfl/clk/SM\n", t, lanes * 4 / 32 / (t * 1e-6) / sms / 1.965e9);
  t = timeit([&] { k_ex2<<<blocks, threads>>>(out, iters); });
  printf("ex2: %.1f us -> %.1f lane-ex2/clk/SM (%.0f G/s)\n", t, lanes * 4 / (t * 1e-6) / sms / 1.965e9, lanes * 4 / t / 1e3);
  t = timeit([&] { k_dfma<<<blocks, threads>>>(dout, iters); });
  printf("dfma: %.1f us -> %.1f lane-dfma/clk/SM (%.1f TFLOP/s)\n", t, lanes * 4 / (t * 1e-6) / sms / 1.965e9, lanes * 8 / t / 1e6);
  int n4 = (8 << 20) / 16;  // 8 MB window, L2 resident
  float4* dst; CK(cudaMalloc(&dst, 64 << 20)); CK(cudaMemset(dst, 0, 64 << 20));
  t = timeit([&] { k_red_coalesced_v4<<<sms * 8, 256>>>(dst, n4, 8); });
  printf("coalesced red.v4 8MB x8: %.1f us -> %.0f G ops/s, %.0f GB/s\n", t, n4 * 8.0 / t / 1e3, n4 * 8.0 * 16 / t / 1e3);
  t = timeit([&] { k_red_coalesced_f1<<<sms * 8, 256>>>((float*)dst, n4 * 4, 8); });
  printf("coalesced red.f32 8MB x8: %.1f us -> %.0f G ops/s, %.0f GB/s\n", t, n4 * 32.0 / t / 1e3, n4 * 32.0 * 4 / t / 1e3);
  t = timeit([&] { k_store_coalesced_v4<<<sms * 8, 256>>>(dst, n4, 8); });
  printf("coalesced st.v4 8MB x8: %.1f us -> %.0f GB/s\n", t, n4 * 8.0 * 16 / t / 1e3);
  return 0;
}
