// Design probe (not product code): which part of the gradient-combine pass is slow?
// g2 (float2, read + zeroed), force (float2, read), gx / gy (float, written), 2.18M cells.
#include <cstdio>
#include <cstdlib>
#include <cuda_runtime.h>
#define CK(x) do { cudaError_t e = (x); if (e != cudaSuccess) { printf("CUDA %s at %d\n", cudaGetErrorString(e), __LINE__); exit(1);} } while (0)

template <int MODE>
__global__ void k_comb(float2 *g2, const float2 *force, float *gx, float *gy, float4 *gxy, int n) {
  const int c0 = 2 * (blockIdx.x * blockDim.x + threadIdx.x);
  if (c0 + 1 >= n) return;
  float4 g = *reinterpret_cast<const float4 *>(g2 + c0);
  float4 f = MODE == 3 ? make_float4(0, 0, 0, 0) : *reinterpret_cast<const float4 *>(force + c0);
  if (MODE != 1) *reinterpret_cast<float4 *>(g2 + c0) = make_float4(0.f, 0.f, 0.f, 0.f);
  if (MODE == 2) {
    gxy[c0 >> 1] = make_float4(g.x + f.x, g.y + f.y, g.z + f.z, g.w + f.w);
  } else {
    *reinterpret_cast<float2 *>(gx + c0) = make_float2(g.x + f.x, g.z + f.z);
    *reinterpret_cast<float2 *>(gy + c0) = make_float2(g.y + f.y, g.w + f.w);
  }
}
// 4 cells per thread, loads first
__global__ void k_comb4(float2 *g2, const float2 *force, float *gx, float *gy, int n) {
  const int c0 = 4 * (blockIdx.x * blockDim.x + threadIdx.x);
  if (c0 + 3 >= n) return;
  float4 g0 = *reinterpret_cast<const float4 *>(g2 + c0), g1 = *reinterpret_cast<const float4 *>(g2 + c0 + 2);
  float4 f0 = *reinterpret_cast<const float4 *>(force + c0), f1 = *reinterpret_cast<const float4 *>(force + c0 + 2);
  *reinterpret_cast<float4 *>(g2 + c0) = make_float4(0, 0, 0, 0);
  *reinterpret_cast<float4 *>(g2 + c0 + 2) = make_float4(0, 0, 0, 0);
  *reinterpret_cast<float4 *>(gx + c0) = make_float4(g0.x + f0.x, g0.z + f0.z, g1.x + f1.x, g1.z + f1.z);
  *reinterpret_cast<float4 *>(gy + c0) = make_float4(g0.y + f0.y, g0.w + f0.w, g1.y + f1.y, g1.w + f1.w);
}
__global__ void k_flush_w(float4 *p, size_t n) {
  for (size_t i = blockIdx.x * (size_t)blockDim.x + threadIdx.x; i < n; i += (size_t)gridDim.x * blockDim.x) p[i] = make_float4(0, 0, 0, 0);
}
__global__ void k_touch(float2 *g2, const float2 *force, int n) {  // leave g2 / force in L2 like the real pipeline
  for (int i = blockIdx.x * blockDim.x + threadIdx.x; i < n; i += gridDim.x * blockDim.x) { g2[i].x += force[i].y; }
}

int main() {
  const int n = 2180000;
  float2 *g2, *force; float *gx, *gy; float4 *gxy, *fl;
  CK(cudaMalloc(&g2, n * 8)); CK(cudaMalloc(&force, n * 8)); CK(cudaMalloc(&gx, n * 4)); CK(cudaMalloc(&gy, n * 4));
  CK(cudaMalloc(&gxy, n * 8)); size_t fb = 512ull << 20; CK(cudaMalloc(&fl, fb));
  CK(cudaMemset(g2, 0, n * 8)); CK(cudaMemset(force, 0, n * 8)); CK(cudaMemset(gx, 0, n * 4)); CK(cudaMemset(gy, 0, n * 4));
  cudaEvent_t a, b; CK(cudaEventCreate(&a)); CK(cudaEventCreate(&b));
  auto run = [&](const char *name, int pre, auto kern) {
    float tot = 0; const int reps = 20;
    for (int r = 0; r < reps; r++) {
      if (pre == 1) k_flush_w<<<1184, 512>>>(fl, fb / 16);
      if (pre == 2) k_touch<<<1184, 256>>>(g2, force, n);
      CK(cudaEventRecord(a)); kern(); CK(cudaEventRecord(b)); CK(cudaEventSynchronize(b));
      float ms; CK(cudaEventElapsedTime(&ms, a, b)); tot += ms;
    }
    printf("%-44s pre=%d  %7.2f us\n", name, pre, tot * 1000 / reps);
  };
  const int g2b = (n / 2 + 255) / 256, g4b = (n / 4 + 255) / 256;
  for (int pre = 0; pre < 3; pre++) {
    run("combine full (2 rd, 3 wr)", pre, [&] { k_comb<0><<<g2b, 256>>>(g2, force, gx, gy, gxy, n); });
    run("no g2 zeroing", pre, [&] { k_comb<1><<<g2b, 256>>>(g2, force, gx, gy, gxy, n); });
    run("interleaved output gxy", pre, [&] { k_comb<2><<<g2b, 256>>>(g2, force, gx, gy, gxy, n); });
    run("no force read", pre, [&] { k_comb<3><<<g2b, 256>>>(g2, force, gx, gy, gxy, n); });
    run("4 cells / thread", pre, [&] { k_comb4<<<g4b, 256>>>(g2, force, gx, gy, n); });
    run("memset g2 only", pre, [&] { cudaMemsetAsync(g2, 0, n * 8); });
  }
  return 0;
}
