// Design probe (not product code): achievable bandwidth for ~35 MB read + ~35 MB write
// streaming kernels on B200 as a function of work per thread and store flavour.
#include <cstdio>
#include <cstdlib>
#include <cuda_runtime.h>
#define CK(x) do { cudaError_t e = (x); if (e != cudaSuccess) { printf("CUDA %s at %d\n", cudaGetErrorString(e), __LINE__); exit(1);} } while (0)

template <int U>
__global__ void k_copy(const float4 *__restrict__ a, float4 *__restrict__ b, int n4) {
  const int base = (blockIdx.x * blockDim.x) * U + threadIdx.x;
  float4 v[U];
#pragma unroll
  for (int u = 0; u < U; u++) { int i = base + u * blockDim.x; if (i < n4) v[u] = a[i]; }
#pragma unroll
  for (int u = 0; u < U; u++) { int i = base + u * blockDim.x; if (i < n4) b[i] = v[u]; }
}
template <int U>
__global__ void k_read(const float4 *__restrict__ a, float *out, int n4) {
  const int base = (blockIdx.x * blockDim.x) * U + threadIdx.x;
  float s = 0;
#pragma unroll
  for (int u = 0; u < U; u++) { int i = base + u * blockDim.x; if (i < n4) { float4 v = a[i]; s += v.x + v.y + v.z + v.w; } }
  if (s == 1234.5f) out[0] = s;
}
template <int U>
__global__ void k_write(float4 *__restrict__ b, int n4) {
  const int base = (blockIdx.x * blockDim.x) * U + threadIdx.x;
#pragma unroll
  for (int u = 0; u < U; u++) { int i = base + u * blockDim.x; if (i < n4) b[i] = make_float4(1, 2, 3, 4); }
}
__global__ void k_flush_w(float4 *p, size_t n) {
  for (size_t i = blockIdx.x * (size_t)blockDim.x + threadIdx.x; i < n; i += (size_t)gridDim.x * blockDim.x) p[i] = make_float4(0, 0, 0, 0);
}
__global__ void k_flush_r(const float4 *p, size_t n, float *out) {
  float s = 0;
  for (size_t i = blockIdx.x * (size_t)blockDim.x + threadIdx.x; i < n; i += (size_t)gridDim.x * blockDim.x) s += p[i].x;
  if (s == 1234.5f) out[0] = s;
}

int main() {
  const size_t bytes = 35ull << 20;
  const int n4 = (int)(bytes / 16);
  float4 *a, *b, *fl; float *out;
  CK(cudaMalloc(&a, bytes)); CK(cudaMalloc(&b, bytes)); CK(cudaMalloc(&out, 64));
  size_t fb = 512ull << 20; CK(cudaMalloc(&fl, fb)); CK(cudaMemset(a, 0, bytes)); CK(cudaMemset(b, 0, bytes)); CK(cudaMemset(fl, 0, fb));
  cudaEvent_t e0, e1; CK(cudaEventCreate(&e0)); CK(cudaEventCreate(&e1));
  auto run = [&](const char *name, int flush, auto kern) {
    float tot = 0; const int reps = 20;
    for (int r = 0; r < reps; r++) {
      if (flush == 1) k_flush_w<<<1184, 512>>>(fl, fb / 16);
      if (flush == 2) k_flush_r<<<1184, 512>>>(fl, fb / 16, out);
      CK(cudaEventRecord(e0)); kern(); CK(cudaEventRecord(e1)); CK(cudaEventSynchronize(e1));
      float ms; CK(cudaEventElapsedTime(&ms, e0, e1)); tot += ms;
    }
    printf("%-34s flush=%s  %7.2f us\n", name, flush == 0 ? "none " : (flush == 1 ? "write" : "read "), tot * 1000 / reps);
  };
  for (int f = 0; f < 3; f++) {
    run("read 35MB U=1", f, [&] { k_read<1><<<(n4 + 255) / 256, 256>>>(a, out, n4); });
    run("read 35MB U=4", f, [&] { k_read<4><<<(n4 + 1023) / 1024, 256>>>(a, out, n4); });
    run("write 35MB U=1", f, [&] { k_write<1><<<(n4 + 255) / 256, 256>>>(b, n4); });
    run("write 35MB U=4", f, [&] { k_write<4><<<(n4 + 1023) / 1024, 256>>>(b, n4); });
    run("copy 35MB U=1", f, [&] { k_copy<1><<<(n4 + 255) / 256, 256>>>(a, b, n4); });
    run("copy 35MB U=4", f, [&] { k_copy<4><<<(n4 + 1023) / 1024, 256>>>(a, b, n4); });
    run("copy 35MB U=8", f, [&] { k_copy<8><<<(n4 + 2047) / 2048, 256>>>(a, b, n4); });
  }
  return 0;
}
