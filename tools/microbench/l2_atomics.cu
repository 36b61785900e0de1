// Design-probe microbenchmark (not product code): L2 gather / red.add throughput on B200.
// Answers: how many random 4B/8B gathers and red.global.add ops per second does the chip
// sustain when the target array is L2-resident (8.7-17.4 MB) — the WA pin->cell gradient
// and the density scatter/gather are bounded by exactly this.
#include <cstdio>
#include <cstdlib>
#include <cstdint>
#include <vector>
#include <random>
#include <algorithm>
#include <cuda_runtime.h>

#define CK(x) do { cudaError_t e = (x); if (e != cudaSuccess) { printf("CUDA %s at %d\n", cudaGetErrorString(e), __LINE__); exit(1);} } while (0)

__global__ void k_gather_f1(const int* __restrict__ idx, const float* __restrict__ src, float* __restrict__ out, int n) {
  float acc = 0.f;
  for (int i = blockIdx.x * blockDim.x + threadIdx.x; i < n; i += gridDim.x * blockDim.x) acc += src[idx[i]];
  if (acc == 1234.5f) out[0] = acc;
}
__global__ void k_gather_f2(const int* __restrict__ idx, const float2* __restrict__ src, float* __restrict__ out, int n) {
  float acc = 0.f;
  for (int i = blockIdx.x * blockDim.x + threadIdx.x; i < n; i += gridDim.x * blockDim.x) { float2 v = src[idx[i]]; acc += v.x + v.y; }
  if (acc == 1234.5f) out[0] = acc;
}
__global__ void k_red_f1(const int* __restrict__ idx, float* dst, int n) {
  for (int i = blockIdx.x * blockDim.x + threadIdx.x; i < n; i += gridDim.x * blockDim.x)
    asm volatile("red.global.add.f32 [%0], %1;" :: "l"(dst + idx[i]), "f"(1.0f) : "memory");
}
__global__ void k_red_f2(const int* __restrict__ idx, float2* dst, int n) {
  for (int i = blockIdx.x * blockDim.x + threadIdx.x; i < n; i += gridDim.x * blockDim.x)
    asm volatile("red.global.add.v2.f32 [%0], {%1, %2};" :: "l"(dst + idx[i]), "f"(1.0f), "f"(2.0f) : "memory");
}
__global__ void k_red_f4(const int* __restrict__ idx, float4* dst, int n) {
  for (int i = blockIdx.x * blockDim.x + threadIdx.x; i < n; i += gridDim.x * blockDim.x)
    asm volatile("red.global.add.v4.f32 [%0], {%1, %2, %3, %4};" :: "l"(dst + (idx[i] >> 1)), "f"(1.0f), "f"(2.0f), "f"(1.0f), "f"(2.0f) : "memory");
}
__global__ void k_copy(const float4* __restrict__ a, float4* __restrict__ b, size_t n) {
  for (size_t i = blockIdx.x * (size_t)blockDim.x + threadIdx.x; i < n; i += (size_t)gridDim.x * blockDim.x) b[i] = a[i];
}

template <class F> float timeit(F f, int reps = 20) {
  cudaEvent_t a, b; CK(cudaEventCreate(&a)); CK(cudaEventCreate(&b));
  for (int i = 0; i < 3; i++) f();
  CK(cudaEventRecord(a));
  for (int i = 0; i < reps; i++) f();
  CK(cudaEventRecord(b)); CK(cudaEventSynchronize(b));
  float ms; CK(cudaEventElapsedTime(&ms, a, b));
  return ms * 1000.f / reps;  // us
}

int main() {
  const int NC = 2180000, NP = 8900000, M = 1024;
  std::mt19937_64 rng(1);
  std::vector<int> rnd(NP), loc(NP), sorted_loc(NP), bins(13000000);
  std::uniform_int_distribution<int> U(0, NC - 1);
  std::normal_distribution<double> G(0, 64);
  // locality pattern like the generator: per net centre c0, 90% near, 10% uniform; nets of 4 pins
  for (int i = 0; i < NP; i += 4) {
    int c0 = U(rng);
    for (int j = 0; j < 4 && i + j < NP; j++) {
      int c = (rng() % 10 == 0) ? U(rng) : (int)((c0 + (long)llround(G(rng)) + NC) % NC);
      loc[i + j] = c;
    }
  }
  for (int i = 0; i < NP; i++) rnd[i] = U(rng);
  // nets sorted by centre: emulate by sorting groups by first cell
  {
    std::vector<std::pair<int,int>> key(NP / 4);
    for (int g = 0; g < NP / 4; g++) key[g] = {loc[g * 4], g};
    std::sort(key.begin(), key.end());
    int o = 0;
    for (auto& kv : key) for (int j = 0; j < 4; j++) sorted_loc[o++] = loc[kv.second * 4 + j];
    for (; o < NP; o++) sorted_loc[o] = loc[o];
  }
  std::uniform_int_distribution<int> UB(0, M * M - 1);
  for (auto& b : bins) b = UB(rng);

  int *d_rnd, *d_loc, *d_sloc, *d_bins; float *d_src, *d_out; float2* d_src2;
  CK(cudaMalloc(&d_rnd, NP * 4)); CK(cudaMalloc(&d_loc, NP * 4)); CK(cudaMalloc(&d_sloc, NP * 4));
  CK(cudaMalloc(&d_bins, bins.size() * 4));
  CK(cudaMalloc(&d_src, NC * 4 * 2)); CK(cudaMalloc(&d_src2, NC * 8)); CK(cudaMalloc(&d_out, 4 * M * M));
  CK(cudaMemcpy(d_rnd, rnd.data(), NP * 4, cudaMemcpyHostToDevice));
  CK(cudaMemcpy(d_loc, loc.data(), NP * 4, cudaMemcpyHostToDevice));
  CK(cudaMemcpy(d_sloc, sorted_loc.data(), NP * 4, cudaMemcpyHostToDevice));
  CK(cudaMemcpy(d_bins, bins.data(), bins.size() * 4, cudaMemcpyHostToDevice));
  CK(cudaMemset(d_src, 0, NC * 8)); CK(cudaMemset(d_src2, 0, NC * 8)); CK(cudaMemset(d_out, 0, 4 * M * M));
  int sms; CK(cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0));
  int l2; CK(cudaDeviceGetAttribute(&l2, cudaDevAttrL2CacheSize, 0));
  printf("SMs %d L2 %d bytes\n", sms, l2);
  dim3 g(sms * 8), b(256);
  const char* names[3] = {"uniform", "locality", "locality+sorted"};
  int* idxs[3] = {d_rnd, d_loc, d_sloc};
  for (int v = 0; v < 3; v++) {
    int* id = idxs[v];
    float t1 = timeit([&] { k_gather_f1<<<g, b>>>(id, d_src, d_out, NP); });
    float t2 = timeit([&] { k_gather_f2<<<g, b>>>(id, d_src2, d_out, NP); });
    float t3 = timeit([&] { k_red_f1<<<g, b>>>(id, d_src, NP); });
    float t4 = timeit([&] { k_red_f2<<<g, b>>>(id, d_src2, NP); });
    float t5 = timeit([&] { k_red_f4<<<g, b>>>(id, (float4*)d_src2, NP); });
    printf("[%s] NP=%d  gather f32 %.1f us (%.0f G/s) | gather f2 %.1f us (%.0f G/s) | red f32 %.1f us (%.0f G/s) | red v2 %.1f us (%.0f G/s) | red v4 %.1f us (%.0f G/s)\n",
           names[v], NP, t1, NP / t1 / 1e3, t2, NP / t2 / 1e3, t3, NP / t3 / 1e3, t4, NP / t4 / 1e3, t5, NP / t5 / 1e3);
  }
  int nb = (int)bins.size();
  float tb = timeit([&] { k_red_f1<<<g, b>>>(d_bins, d_out, nb); });
  printf("density-like red f32 into 4MB map: %d ops %.1f us (%.0f G/s)\n", nb, tb, nb / tb / 1e3);
  size_t nbytes = 512ull << 20; float4 *ca, *cb; CK(cudaMalloc(&ca, nbytes)); CK(cudaMalloc(&cb, nbytes));
  float tc = timeit([&] { k_copy<<<sms * 4, 512>>>(ca, cb, nbytes / 16); }, 10);
  printf("copy 512MB: %.1f us  %.0f GB/s\n", tc, 2.0 * nbytes / tc / 1e3);
  return 0;
}
