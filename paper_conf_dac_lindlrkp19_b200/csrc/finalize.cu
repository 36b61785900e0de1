// finalize.cu — gradient combine (eq 2: grad WA + lambda grad D) and the scalar
// outputs (WA, D, obj, HPWL) on sm_100a.
//
// The WA kernels accumulate into the interleaved scratch g2 (cleared at the head of the WA
// stream), which this pass reads and splits into the caller's gx / gy.  Scalars are reduced from per-CTA partials in a fixed order, so
// WA and D are run-to-run deterministic given the partials; HPWL is converted from the
// exact int64 limb sum with one correctly rounded step (reading A7).
#include "dp_internal.h"

namespace dp {

namespace {

// Four cells per thread: 16-byte loads of g2 / force issued together, 16-byte stores of gx / gy,
// no grid-stride loop.  g2 is only read here (zeroing it in the same pass, a store to the
// lines just loaded, measured 2.5x slower on B200); the WA stream clears it before the next
// accumulation.  force[i] is stored with the parity offset of cell_begin (dp_create), so even
// global cells are 16-byte aligned in both arrays.
// Deterministic mode (NEXT-2): the WA gradient arrives as int64 in units 2^-F (exact sums).
__global__ void __launch_bounds__(256) k_combine_det(const long long *__restrict__ g2i, int frac,
                                                     const float2 *__restrict__ force, float *__restrict__ gx,
                                                     float *__restrict__ gy, int cell_begin, int n_own, float lambda,
                                                     const float *__restrict__ lambda_dev, int use_wa, int use_den,
                                                     const uint8_t *__restrict__ fixed) {
  if (lambda_dev) lambda = __ldg(lambda_dev);
  const int i = blockIdx.x * blockDim.x + threadIdx.x;
  if (i >= n_own) return;
  const int c = cell_begin + i;
  float vx = 0.f, vy = 0.f;
  if (use_wa) {
    const longlong2 q = reinterpret_cast<const longlong2 *>(g2i)[c];
    vx = (float)ldexp((double)q.x, -frac);
    vy = (float)ldexp((double)q.y, -frac);
  }
  if (use_den) {
    const float2 f = force[i];
    vx = fmaf(lambda, f.x, vx);
    vy = fmaf(lambda, f.y, vy);
  }
  if (fixed && fixed[i]) vx = vy = 0.f;
  gx[c] = vx;
  gy[c] = vy;
}

// Virtual shard (dp_create_dist without NCCL, tests): the gradient reduce-scatter is skipped, so
// the shard's partial WA gradient is written for every cell (the sum over shards is the full
// gradient) and lambda times the force for its own cells.
__global__ void __launch_bounds__(256) k_combine_virtual(const float2 *__restrict__ g2, const long long *__restrict__ g2i,
                                                         int frac, const float2 *__restrict__ force,
                                                         float *__restrict__ gx, float *__restrict__ gy, int n,
                                                         int cell_begin, int n_own, float lambda, int use_wa,
                                                         int use_den) {
  const int c = blockIdx.x * blockDim.x + threadIdx.x;
  if (c >= n) return;
  float vx = 0.f, vy = 0.f;
  if (use_wa) {
    if (g2i) {
      const longlong2 q = reinterpret_cast<const longlong2 *>(g2i)[c];
      vx = (float)ldexp((double)q.x, -frac);
      vy = (float)ldexp((double)q.y, -frac);
    } else {
      const float2 q = g2[c];
      vx = q.x;
      vy = q.y;
    }
  }
  if (use_den && c >= cell_begin && c < cell_begin + n_own) {
    const float2 f = force[c - cell_begin];
    vx = fmaf(lambda, f.x, vx);
    vy = fmaf(lambda, f.y, vy);
  }
  gx[c] = vx;
  gy[c] = vy;
}

__global__ void __launch_bounds__(256) k_combine(const float2 *__restrict__ g2, const float2 *__restrict__ force,
                                                 float *__restrict__ gx, float *__restrict__ gy, int cell_begin,
                                                 int n_own, float lambda, const float *__restrict__ lambda_dev,
                                                 int use_wa, int use_den, const uint8_t *__restrict__ fixed) {
  if (lambda_dev) lambda = __ldg(lambda_dev);   // GP loop: lambda on the device
  const int c0 = (cell_begin & ~3) + 4 * (blockIdx.x * blockDim.x + threadIdx.x);
  const int cend = cell_begin + n_own;
  if (c0 >= cend) return;
  const float2 *fb = force - cell_begin;   // fb[c] = force of global cell c
  const bool aligned4 = (((uintptr_t)(fb + c0)) & 15) == 0 && (((uintptr_t)(gx + c0)) & 15) == 0 &&
                        (((uintptr_t)(gy + c0)) & 15) == 0;
  if (c0 >= cell_begin && c0 + 3 < cend && aligned4) {
    float4 g0 = make_float4(0.f, 0.f, 0.f, 0.f), g1 = g0, f0 = g0, f1 = g0;
    if (use_wa) {
      g0 = __ldcs(reinterpret_cast<const float4 *>(g2 + c0));
      g1 = __ldcs(reinterpret_cast<const float4 *>(g2 + c0 + 2));
    }
    if (use_den) {
      f0 = __ldcs(reinterpret_cast<const float4 *>(fb + c0));
      f1 = __ldcs(reinterpret_cast<const float4 *>(fb + c0 + 2));
    }
    float4 ox = make_float4(fmaf(lambda, f0.x, g0.x), fmaf(lambda, f0.z, g0.z), fmaf(lambda, f1.x, g1.x),
                            fmaf(lambda, f1.z, g1.z));
    float4 oy = make_float4(fmaf(lambda, f0.y, g0.y), fmaf(lambda, f0.w, g0.w), fmaf(lambda, f1.y, g1.y),
                            fmaf(lambda, f1.w, g1.w));
    if (fixed) {   // NEXT-4: fixed cells are not variables -> gradient 0 (single-context: own = global)
      const uchar4 m = *reinterpret_cast<const uchar4 *>(fixed + c0);
      if (m.x) ox.x = oy.x = 0.f;
      if (m.y) ox.y = oy.y = 0.f;
      if (m.z) ox.z = oy.z = 0.f;
      if (m.w) ox.w = oy.w = 0.f;
    }
    __stcs(reinterpret_cast<float4 *>(gx + c0), ox);
    __stcs(reinterpret_cast<float4 *>(gy + c0), oy);
    return;
  }
  for (int c = c0; c < c0 + 4; c++) {  // ragged ends of the own range / unaligned caller buffers
    if (c < cell_begin || c >= cend) continue;
    float vx = 0.f, vy = 0.f;
    if (use_wa) {
      const float2 q = g2[c];
      vx = q.x;
      vy = q.y;
    }
    if (use_den) {
      const float2 q = fb[c];
      vx = fmaf(lambda, q.x, vx);
      vy = fmaf(lambda, q.y, vy);
    }
    if (fixed && fixed[c - cell_begin]) vx = vy = 0.f;
    gx[c] = vx;
    gy[c] = vy;
  }
}

// Correctly rounded double of sum_j L[j] 2^(32 j - 149), L[j] < 2^63 (reading A7).
__device__ double limbs_to_double(const unsigned long long *L) {
  unsigned int D[kHpwlLimbs + 3];
  unsigned long long carry = 0;
  for (int j = 0; j <= kHpwlLimbs; j++) {
    const unsigned __int128 v = (unsigned __int128)L[j] + carry;
    D[j] = (unsigned int)(v & 0xffffffffu);
    carry = (unsigned long long)(v >> 32);
  }
  D[kHpwlLimbs + 1] = (unsigned int)(carry & 0xffffffffu);
  D[kHpwlLimbs + 2] = (unsigned int)(carry >> 32);
  int top = -1;
  for (int j = kHpwlLimbs + 2; j >= 0; j--)
    if (D[j]) {
      top = j;
      break;
    }
  if (top < 0) return 0.0;
  auto dig = [&](int j) -> unsigned __int128 { return (j >= 0) ? (unsigned __int128)D[j] : (unsigned __int128)0; };
  unsigned __int128 W = (dig(top) << 96) | (dig(top - 1) << 64) | (dig(top - 2) << 32) | dig(top - 3);
  bool sticky = false;
  for (int j = 0; j < top - 3; j++) sticky |= (D[j] != 0);
  const int lz = __clz(D[top]);  // leading zeros of the top digit
  W <<= lz;
  int pos = 32 * (top - 3) + 127 - lz;  // bit index of the MSB in the 2^-149 scaled integer
  unsigned long long mant = (unsigned long long)(W >> 75);
  const unsigned __int128 rem = W & (((unsigned __int128)1 << 75) - 1);
  const unsigned __int128 half = (unsigned __int128)1 << 74;
  if (rem > half || (rem == half && (sticky || (mant & 1ull)))) mant++;
  if (mant == (1ull << 53)) {
    mant >>= 1;
    pos++;
  }
  return ldexp((double)mant, pos - 52 - 149);
}

struct FinArgs {
  const double *part;
  int n_wa, n_en;
  const double *hp_part;   // fast-HPWL partials (GP loop, reading A37) or null: exact limbs
  unsigned long long *limbs;
  double *scal;   // staging {wl, energy, hpwl, obj}
  double *d_obj, *d_wl, *d_energy, *d_hpwl;
  float lambda;
  const float *lambda_dev;
  int with_wl, with_energy, with_hpwl, phase;  // phase 0: local sums -> scal (dist), 1: outputs, 2: both
};

__global__ void __launch_bounds__(256) k_finalize(FinArgs a) {
  __shared__ double s_a[256], s_b[256], s_c[256];
  if (a.phase != 1) {
    double wl = 0.0, en = 0.0, hp = 0.0;
    // fixed assignment of partials to threads and a fixed tree -> deterministic
    if (a.with_wl)
      for (int i = threadIdx.x; i < a.n_wa; i += 256) wl += a.part[i];
    if (a.with_energy)
      for (int i = threadIdx.x; i < a.n_en; i += 256) en += a.part[a.n_wa + i];
    if (a.hp_part)
      for (int i = threadIdx.x; i < a.n_wa; i += 256) hp += a.hp_part[i];
    s_a[threadIdx.x] = wl;
    s_b[threadIdx.x] = en;
    s_c[threadIdx.x] = hp;
    __syncthreads();
    for (int o = 128; o > 0; o >>= 1) {
      if ((int)threadIdx.x < o) {
        s_a[threadIdx.x] += s_a[threadIdx.x + o];
        s_b[threadIdx.x] += s_b[threadIdx.x + o];
        s_c[threadIdx.x] += s_c[threadIdx.x + o];
      }
      __syncthreads();
    }
    if (threadIdx.x == 0) {
      a.scal[0] = s_a[0];
      a.scal[1] = s_b[0];
      a.scal[4] = s_c[0];
    }
  }
  if (a.phase == 0) return;
  __syncthreads();
  if (a.lambda_dev) a.lambda = *a.lambda_dev;
  if (threadIdx.x == 0) {
    const double wl = a.scal[0], en = a.scal[1];
    double hp = __longlong_as_double(0x7ff8000000000000ll);
    if (a.with_hpwl && a.hp_part) {
      hp = a.scal[4];
    } else if (a.with_hpwl) {
      hp = limbs_to_double(a.limbs);
      for (int k = 0; k <= kHpwlLimbs; k++) a.limbs[k] = 0ull;
    }
    if (a.d_wl) *a.d_wl = wl;
    if (a.d_energy) *a.d_energy = en;
    if (a.d_hpwl) *a.d_hpwl = hp;
    if (a.d_obj) *a.d_obj = (a.with_wl ? wl : 0.0) + (a.with_energy ? (double)a.lambda * en : 0.0);
    a.scal[2] = hp;
    a.scal[3] = (a.with_wl ? wl : 0.0) + (a.with_energy ? (double)a.lambda * en : 0.0);
  }
}

}  // namespace

void launch_combine(const Ctx &c, float lambda, float *gx, float *gy, bool use_wa, bool use_density,
                    cudaStream_t s) {
  if (c.dist && !c.nccl_comm) {
    k_combine_virtual<<<(c.num_cells + 255) / 256, 256, 0, s>>>(c.d_g2, c.deterministic ? c.d_g2i : nullptr,
                                                                c.det_frac, c.d_force, gx, gy, c.num_cells,
                                                                c.cell_begin, c.n_own, lambda, use_wa ? 1 : 0,
                                                                use_density ? 1 : 0);
    return;
  }
  if (c.n_own <= 0) return;
  if (c.deterministic) {
    k_combine_det<<<(c.n_own + 255) / 256, 256, 0, s>>>(c.d_g2i, c.det_frac, c.d_force, gx, gy, c.cell_begin, c.n_own,
                                                        lambda, use_density ? c.lambda_dev : nullptr, use_wa ? 1 : 0,
                                                        use_density ? 1 : 0, c.has_fixed ? c.d_fixed : nullptr);
    return;
  }
  const int quads = (c.n_own + 6) / 4 + 1;
  const int blocks = (quads + 255) / 256;
  k_combine<<<blocks, 256, 0, s>>>(c.d_g2, c.d_force, gx, gy, c.cell_begin, c.n_own, lambda,
                                   use_density ? c.lambda_dev : nullptr, use_wa ? 1 : 0, use_density ? 1 : 0,
                                   c.has_fixed ? c.d_fixed : nullptr);
}

void launch_finalize_phase(const Ctx &c, int phase, float lambda, bool with_wl, bool with_energy, bool with_hpwl,
                           double *d_obj, double *d_wl, double *d_energy, double *d_hpwl, cudaStream_t s) {
  FinArgs a;
  a.part = c.d_part;
  a.n_wa = c.n_wa_part;
  a.n_en = c.n_en_slots();
  a.hp_part = (with_hpwl && c.hpwl_fast && c.wl_model == DP_WL_WA) ? c.d_part + c.n_wa_part + c.n_en_slots() + 1 : nullptr;
  a.limbs = c.d_limbs;
  a.scal = c.d_scal;
  a.d_obj = d_obj;
  a.d_wl = d_wl;
  a.d_energy = d_energy;
  a.d_hpwl = d_hpwl;
  a.lambda = lambda;
  a.lambda_dev = with_energy ? c.lambda_dev : nullptr;
  a.with_wl = with_wl;
  a.with_energy = with_energy;
  a.with_hpwl = with_hpwl;
  a.phase = phase;
  k_finalize<<<1, 256, 0, s>>>(a);
}

void launch_finalize(const Ctx &c, float lambda, bool with_wl, bool with_energy, bool with_hpwl, double *d_obj,
                     double *d_wl, double *d_energy, double *d_hpwl, cudaStream_t s) {
  launch_finalize_phase(c, 2, lambda, with_wl, with_energy, with_hpwl, d_obj, d_wl, d_energy, d_hpwl, s);
}

}  // namespace dp
