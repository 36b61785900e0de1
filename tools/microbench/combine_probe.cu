// Design probe (not product code): is a streaming read of an array slow right after that
// array received random red.global.add / scattered 8-byte stores?
#include <cstdio>
#include <cstdlib>
#include <cuda_runtime.h>
#define CK(x) do { cudaError_t e = (x); if (e != cudaSuccess) { printf("CUDA %s at %d\n", cudaGetErrorString(e), __LINE__); exit(1);} } while (0)

__global__ void k_combine(float2 *g2, const float2 *force, float *gx, float *gy, int n, float lam) {
  const int c0 = 2 * (blockIdx.x * blockDim.x + threadIdx.x);
  if (c0 + 1 >= n) return;
  float4 g = *reinterpret_cast<const float4 *>(g2 + c0);
  *reinterpret_cast<float4 *>(g2 + c0) = make_float4(0.f, 0.f, 0.f, 0.f);
  float4 f = *reinterpret_cast<const float4 *>(force + c0);
  *reinterpret_cast<float2 *>(gx + c0) = make_float2(g.x + lam * f.x, g.z + lam * f.z);
  *reinterpret_cast<float2 *>(gy + c0) = make_float2(g.y + lam * f.y, g.w + lam * f.w);
}
__global__ void k_read_only(const float4 *a, const float4 *b, float *out, int n4) {
  const int i = blockIdx.x * blockDim.x + threadIdx.x;
  if (i >= n4) return;
  float4 x = a[i], y = b[i];
  if (x.x + y.y == 1234.5f) out[0] = x.z;
}
__global__ void k_rand_red(float2 *g2, int n, int ops) {
  for (int i = blockIdx.x * blockDim.x + threadIdx.x; i < ops; i += gridDim.x * blockDim.x) {
    unsigned h = (unsigned)i * 2654435761u;
    int c = (int)(h % (unsigned)n);
    asm volatile("red.global.add.v2.f32 [%0], {%1, %2};" ::"l"(g2 + c), "f"(1.f), "f"(2.f) : "memory");
  }
}
__global__ void k_rand_store(float2 *f, int n) {
  for (int i = blockIdx.x * blockDim.x + threadIdx.x; i < n; i += gridDim.x * blockDim.x) {
    unsigned h = (unsigned)i * 2654435761u;
    int c = (int)(h % (unsigned)n);
    f[c] = make_float2(1.f, 2.f);
  }
}
__global__ void k_seq_store(float2 *f, int n) {
  for (int i = blockIdx.x * blockDim.x + threadIdx.x; i < n; i += gridDim.x * blockDim.x) f[i] = make_float2(1.f, 2.f);
}
__global__ void k_flush(float4 *p, size_t n) {
  for (size_t i = blockIdx.x * (size_t)blockDim.x + threadIdx.x; i < n; i += (size_t)gridDim.x * blockDim.x) p[i] = make_float4(0, 0, 0, 0);
}

int main() {
  const int n = 2180000;
  float2 *g2, *force; float *gx, *gy, *out; float4 *fl;
  CK(cudaMalloc(&g2, n * 8)); CK(cudaMalloc(&force, n * 8)); CK(cudaMalloc(&gx, n * 4)); CK(cudaMalloc(&gy, n * 4));
  CK(cudaMalloc(&out, 64)); size_t fb = 512ull << 20; CK(cudaMalloc(&fl, fb));
  CK(cudaMemset(g2, 0, n * 8)); CK(cudaMemset(force, 0, n * 8));
  cudaEvent_t a, b; CK(cudaEventCreate(&a)); CK(cudaEventCreate(&b));
  auto flush = [&] { k_flush<<<1184, 512>>>(fl, fb / 16); };
  auto time_combine = [&](const char *label, auto pre) {
    float tot = 0; int reps = 20;
    for (int r = 0; r < reps; r++) {
      pre(); flush();
      CK(cudaEventRecord(a)); k_combine<<<(n / 2 + 255) / 256, 256>>>(g2, force, gx, gy, n, 1.f); CK(cudaEventRecord(b));
      CK(cudaEventSynchronize(b)); float ms; CK(cudaEventElapsedTime(&ms, a, b)); tot += ms;
    }
    printf("%-40s combine %.2f us\n", label, tot * 1000 / reps);
  };
  time_combine("fresh", [] {});
  time_combine("after seq store force", [&] { k_seq_store<<<1184, 256>>>(force, n); });
  time_combine("after random 8B stores force", [&] { k_rand_store<<<1184, 256>>>(force, n); });
  time_combine("after random red.v2 g2 (8.9M)", [&] { k_rand_red<<<1184, 256>>>(g2, n, 8900000); });
  time_combine("after both", [&] { k_rand_store<<<1184, 256>>>(force, n); k_rand_red<<<1184, 256>>>(g2, n, 8900000); });
  // no flush, right after
  {
    float tot = 0; int reps = 20;
    for (int r = 0; r < reps; r++) {
      flush(); k_rand_store<<<1184, 256>>>(force, n); k_rand_red<<<1184, 256>>>(g2, n, 8900000);
      CK(cudaEventRecord(a)); k_combine<<<(n / 2 + 255) / 256, 256>>>(g2, force, gx, gy, n, 1.f); CK(cudaEventRecord(b));
      CK(cudaEventSynchronize(b)); float ms; CK(cudaEventElapsedTime(&ms, a, b)); tot += ms;
    }
    printf("%-40s combine %.2f us\n", "both, no flush in between", tot * 1000 / reps);
  }
  {
    float tot = 0;
    for (int r = 0; r < 20; r++) {
      flush(); CK(cudaEventRecord(a)); k_read_only<<<(n / 2 + 255) / 256, 256>>>((float4 *)g2, (float4 *)force, out, n / 2); CK(cudaEventRecord(b));
      CK(cudaEventSynchronize(b)); float ms; CK(cudaEventElapsedTime(&ms, a, b)); tot += ms;
    }
    printf("%-40s %.2f us\n", "read-only 2 arrays", tot * 1000 / 20);
  }
  return 0;
}
