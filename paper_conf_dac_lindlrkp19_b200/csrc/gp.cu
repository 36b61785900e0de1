// gp.cu — the global-placement loop around the evaluation on sm_100a.
//
// PAPER.md: the kernel GP iterations "involve the computation of wirelength and density
// gradient, optimization engines, and cell location updating"; the optimizer is
// ePlace's Nesterov method with a Lipschitz-constant step prediction; the
// density weight follows eq (18) with DREAMPlace's change for p < 0.  What the
// paper leaves to ePlace/RePlAce is taken as readings A28-A33 (oracle/gp.py):
//   A28 alpha_k = |v_k - v_{k-1}| / |g_k - g_{k-1}|, u_{k+1} = clamp(v_k - alpha_k g_k),
//       a_{k+1} = (1 + sqrt(4 a_k^2 + 1))/2, v_{k+1} = clamp(u_{k+1} + (a_k - 1)/a_{k+1} (u_{k+1} - u_k))
//   A29 g_i = grad_i / max(1, P_i + lambda w_i h_i)
//   A30 overflow = sum_b max(rho_b - t, 0) b_x b_y / sum_i w_i h_i (the evaluation's own map)
//   A31 gamma = 4 (b_x + b_y) 10^((tau - 0.1) 20/9 - 1)
//   A32 lambda_0 = 8e-5 |grad WL|_1 / |grad D|_1, then eq (18) with p = dHPWL / 3.5e5
//   A33 HPWL / overflow at v; clamp to [xl, xh - w]; v_{-1} = v_0 - eta g_0 (rms 0.01 b_x)
//   A36 converged once overflow < stop_overflow: later iterations leave the state unchanged;
//       lambda capped at 1e30
//   A37 the HPWL the schedule uses (eq 18's p) and the history reports is the "fast HPWL": the
//       same per-net spans from the fp32 pin positions of the WA pass, summed in fp64 per CTA
//       (the exact, correctly rounded HPWL stays dp_eval's d_hpwl; they differ by ~1e-7 rel.)
//
// B200 design: every step runs on the device.  gamma and lambda live in device memory and
// the evaluation kernels read them there (Ctx::gamma_dev / lambda_dev), so one iteration —
// Lipschitz norms, step, Nesterov update, the full evaluation (both streams), the
// preconditioner, the overflow reduction and the scalar schedule — is captured ONCE into a
// CUDA graph and replayed per iteration with no host synchronisation.  Reductions are
// per-block fp64 partials combined in a fixed order (run-to-run deterministic).
#include <cmath>
#include <cstdlib>

#include "dp_internal.h"

namespace dp {
namespace {

constexpr int kGpThreads = 256;
constexpr int kHistCols = 8;   // k, hpwl, overflow, lambda, gamma, obj, alpha, wl

struct GpDev {      // device-resident loop state (scalars)
  double a, lam, gamma, hpwl, tau, alpha, coef, eta;
  double l1_wl, l1_d, area_total, gamma_base;
  long long k;
  float f_gamma, f_lambda, f_alpha, f_coef, f_eta;
  int frozen;                       // A36: converged (the step kernel and the schedule stop)
  float pad_[2];
};

struct GpArgs {
  int n;
  const uint8_t *fixed;    // NEXT-4 (reading A34): fixed cells are not variables (null: none)
  float *ux, *uy, *vx, *vy, *vpx, *vpy, *gx, *gy, *gpx, *gpy, *rgx, *rgy;
  const float *w, *h, *pins;
  float xl, yl, xh, yh;
  const unsigned long long *rho;
  const unsigned long long *rho_fixed;   // fixed-charge map (dp_set_fixed), null if none
  long long nbins;
  double rho_unit;         // 2^-kRhoScaleLog2
  double target;
  double *part;            // [nblk][2]
  int nblk;
  double *part_ovf;        // [oblk][2] overflow partials of k_gp_post
  int oblk;
  const double *region_ovf;   // fence regions: the density passes' overflow partials ([region_blk][2])
  int region_blk;
  GpDev *dev;
  const double *out;       // eval outputs {obj, wl, energy, hpwl}
  double *hist;
  int hist_cap;
  double bxby;
  double mu_min, mu_max, dhpwl_ref, lambda_scale, init_rms_bins, bx, stop_overflow;
};

// fixed-order block reduction of two fp64 values into part[2 * blockIdx.x + {0,1}]
__device__ __forceinline__ void block_pair(double s0, double s1, double *part) {
  __shared__ double r0[kGpThreads / 32], r1[kGpThreads / 32];
#pragma unroll
  for (int o = 16; o > 0; o >>= 1) {
    s0 += __shfl_xor_sync(0xffffffffu, s0, o);
    s1 += __shfl_xor_sync(0xffffffffu, s1, o);
  }
  const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
  if (lane == 0) {
    r0[warp] = s0;
    r1[warp] = s1;
  }
  __syncthreads();
  if (threadIdx.x == 0) {
    double t0 = 0.0, t1 = 0.0;
    for (int w = 0; w < kGpThreads / 32; w++) {
      t0 += r0[w];
      t1 += r1[w];
    }
    part[2 * blockIdx.x] = t0;
    part[2 * blockIdx.x + 1] = t1;
  }
}

enum { R_NORMS = 0, R_L1 = 1, R_SQ = 2, R_OVF = 3 };

// A30 with fixed macros (the DREAMPlace convention): the fixed charge counts at the
// target density, rho_eff = rho_movable + t rho_fixed = rho - (1 - t) rho_fixed, so a bin that a
// macro covers overflows only by its movable charge; the sum is divided by the movable area
__device__ __forceinline__ double ovf_term(const GpArgs &a, long long b) {
  double r = (double)a.rho[b] * a.rho_unit;
  if (a.rho_fixed) r -= (1.0 - a.target) * ((double)a.rho_fixed[b] * a.rho_unit);
  return fmax(r - a.target, 0.0);
}

// Per-block partial sums.  R_NORMS: (|v - vp|^2, |g - gp|^2); R_L1: (|rg|_1, 0);
// R_SQ: (|g|^2, 0); R_OVF: (sum_b max(rho_b - t, 0), 0).
__global__ void __launch_bounds__(kGpThreads) k_gp_partials(GpArgs a, int mode) {
  double s0 = 0.0, s1 = 0.0;
  const int stride = gridDim.x * kGpThreads;
  if (mode == R_OVF) {
    for (long long b = blockIdx.x * kGpThreads + threadIdx.x; b < a.nbins; b += stride) s0 += ovf_term(a, b);
  } else {
    for (int i = blockIdx.x * kGpThreads + threadIdx.x; i < a.n; i += stride) {
      if (mode == R_NORMS) {
        const double dx = (double)a.vx[i] - a.vpx[i], dy = (double)a.vy[i] - a.vpy[i];
        const double ex = (double)a.gx[i] - a.gpx[i], ey = (double)a.gy[i] - a.gpy[i];
        s0 += dx * dx + dy * dy;
        s1 += ex * ex + ey * ey;
      } else if (mode == R_L1) {
        s0 += fabs((double)a.rgx[i]) + fabs((double)a.rgy[i]);
      } else {
        s0 += (double)a.gx[i] * a.gx[i] + (double)a.gy[i] * a.gy[i];
      }
    }
  }
  block_pair(s0, s1, a.part);
}

// Fixed-order block reduction of n (x, y) partial pairs (every thread of the block calls it;
// the result is valid in all threads).  Thread t sums pairs t, t + T, ... in order, then a
// fixed shared-memory tree: deterministic, and far shorter than one thread walking the list.
__device__ __forceinline__ void sum_parts(const double *part, int n, double &t0, double &t1) {
  __shared__ double s0[kGpThreads], s1[kGpThreads];
  double a0 = 0.0, a1 = 0.0;
  for (int b = threadIdx.x; b < n; b += kGpThreads) {
    a0 += part[2 * b];
    a1 += part[2 * b + 1];
  }
  s0[threadIdx.x] = a0;
  s1[threadIdx.x] = a1;
  __syncthreads();
  for (int o = kGpThreads / 2; o > 0; o >>= 1) {
    if ((int)threadIdx.x < o) {
      s0[threadIdx.x] += s0[threadIdx.x + o];
      s1[threadIdx.x] += s1[threadIdx.x + o];
    }
    __syncthreads();
  }
  t0 = s0[0];
  t1 = s1[0];
  __syncthreads();
}

__device__ __forceinline__ double gamma_of(const GpArgs &a, double tau) {   // A31
  return a.dev->gamma_base * pow(10.0, (tau - 0.1) * 20.0 / 9.0 - 1.0);
}

enum { S_ALPHA = 0, S_ITER_END = 1, S_INIT_TAU = 2, S_INIT_L1D = 3, S_INIT_LAMBDA = 4, S_INIT_ETA = 5,
       S_INIT_DONE = 6 };

// A28: Lipschitz step prediction from the norms (t0 = |v - vp|^2, t1 = |g - gp|^2) and the
// Nesterov coefficient for the next update
__device__ __forceinline__ void step_scalars(GpDev &d, double t0, double t1) {
  const double num = sqrt(t0), den = sqrt(t1);
  if (den > 0.0) d.alpha = num / den;
  const double an = (1.0 + sqrt(4.0 * d.a * d.a + 1.0)) / 2.0;
  d.coef = (d.a - 1.0) / an;
  d.a = an;
  d.f_alpha = (float)d.alpha;
  d.f_coef = (float)d.coef;
}

// Scalar steps of the schedule (one block; partials summed in a fixed order, thread 0 writes).
__global__ void __launch_bounds__(kGpThreads) k_gp_scalar(GpArgs a, int op) {
  GpDev &d = *a.dev;
  double t0, t1, o0 = 0.0, o1 = 0.0;
  sum_parts(a.part, a.nblk, t0, t1);
  if (op == S_ITER_END) {
    if (a.region_ovf)
      sum_parts(a.region_ovf, a.region_blk, o0, o1);
    else
      sum_parts(a.part_ovf, a.oblk, o0, o1);
  }
  if (op == S_INIT_TAU && a.region_ovf) sum_parts(a.region_ovf, a.region_blk, t0, t1);
  if (threadIdx.x != 0) return;
  switch (op) {
    case S_ALPHA:
      step_scalars(d, t0, t1);
      break;
    case S_ITER_END: {   // A30 overflow, eq (18) lambda, A31 gamma, history row; then A28 for the next step
      const double tau = o0 * a.bxby / d.area_total;
      const double hp = a.out[3];
      if (d.frozen) {   // A36: converged, the state stays; the row repeats it
        if (a.hist_cap > 0) {
          double *r = a.hist + (size_t)(d.k % a.hist_cap) * kHistCols;
          r[0] = (double)d.k; r[1] = hp; r[2] = d.tau; r[3] = d.lam;
          r[4] = d.gamma; r[5] = a.out[0]; r[6] = d.alpha; r[7] = a.out[1];
        }
        d.k += 1;
        break;
      }
      const double p = (hp - d.hpwl) / a.dhpwl_ref;
      const double mu = p < 0.0 ? a.mu_max * fmax(pow(0.9999, (double)d.k), 0.98)
                                : fmax(a.mu_min, pow(a.mu_max, 1.0 - p));            // eq (18a)
      d.lam = fmin(d.lam * mu, 1e30);
      d.tau = tau;
      d.gamma = gamma_of(a, tau);
      if (a.hist_cap > 0) {
        double *r = a.hist + (size_t)(d.k % a.hist_cap) * kHistCols;
        r[0] = (double)d.k; r[1] = hp; r[2] = tau; r[3] = d.lam;
        r[4] = d.gamma; r[5] = a.out[0]; r[6] = d.alpha; r[7] = a.out[1];
      }
      d.hpwl = hp;
      d.k += 1;
      d.f_gamma = (float)d.gamma;
      d.f_lambda = (float)d.lam;
      step_scalars(d, t0, t1);
      if (tau < a.stop_overflow) d.frozen = 1;
      break;
    }
    case S_INIT_TAU:
      d.tau = t0 * a.bxby / d.area_total;
      d.gamma = gamma_of(a, d.tau);
      d.f_gamma = (float)d.gamma;
      break;
    case S_INIT_L1D:
      d.l1_d = t0;
      break;
    case S_INIT_LAMBDA:   // A32
      d.l1_wl = t0;
      d.lam = d.l1_d > 0.0 ? a.lambda_scale * d.l1_wl / d.l1_d : 0.0;
      d.f_lambda = (float)d.lam;
      break;
    case S_INIT_ETA: {    // A33: v_{-1} = v_0 - eta g_0 with rms displacement init_rms_bins b_x
      const double rms = sqrt(t0 / (2.0 * a.n));
      d.eta = rms > 0.0 ? a.init_rms_bins * a.bx / rms : 0.0;
      d.f_eta = (float)d.eta;
      d.hpwl = a.out[3];
      break;
    }
    case S_INIT_DONE:
      d.a = 1.0;
      d.alpha = 0.0;
      d.k = 0;
      d.frozen = 0;
      break;
  }
}

__device__ __forceinline__ float clampf(float v, float lo, float hi) { return fminf(fmaxf(v, lo), hi); }

// A28 per cell: u' = clamp(v - alpha g); v' = clamp(u' + coef (u' - u)); vp = v; gp = g.
__global__ void __launch_bounds__(kGpThreads) k_gp_update(GpArgs a) {
  const int i = blockIdx.x * kGpThreads + threadIdx.x;
  if (i >= a.n || a.dev->frozen) return;
  if (a.fixed && a.fixed[i]) {   // not a variable: u, v stay (its gradient is 0 as well)
    a.vpx[i] = a.vx[i]; a.vpy[i] = a.vy[i];
    a.gpx[i] = a.gx[i]; a.gpy[i] = a.gy[i];
    return;
  }
  const float alpha = a.dev->f_alpha, coef = a.dev->f_coef;
  const float hx = a.xh - a.w[i], hy = a.yh - a.h[i];
  const float vx = a.vx[i], vy = a.vy[i], gx = a.gx[i], gy = a.gy[i];
  const float ux = clampf(fmaf(-alpha, gx, vx), a.xl, hx), uy = clampf(fmaf(-alpha, gy, vy), a.yl, hy);
  const float nx = clampf(fmaf(coef, ux - a.ux[i], ux), a.xl, hx), ny = clampf(fmaf(coef, uy - a.uy[i], uy), a.yl, hy);
  a.vpx[i] = vx; a.vpy[i] = vy;
  a.gpx[i] = gx; a.gpy[i] = gy;
  a.ux[i] = ux; a.uy[i] = uy;
  a.vx[i] = nx; a.vy[i] = ny;
}

// A29: g = raw / max(1, P_i + lambda w h)
__global__ void __launch_bounds__(kGpThreads) k_gp_precond(GpArgs a) {
  const int i = blockIdx.x * kGpThreads + threadIdx.x;
  if (i >= a.n) return;
  const float lam = a.dev->f_lambda;
  const float inv = 1.f / fmaxf(1.f, fmaf(lam, a.w[i] * a.h[i], a.pins[i]));
  a.gx[i] = a.rgx[i] * inv;
  a.gy[i] = a.rgy[i] * inv;
}

// After the evaluation at v: blocks [0, nblk) precondition (A29) and form the Lipschitz norms
// |v - vp|^2, |g - gp|^2 of the next step (grid-stride, fixed order); blocks [nblk, nblk + oblk)
// form the overflow partials (A30) from the evaluation's bin map.
__global__ void __launch_bounds__(kGpThreads) k_gp_post(GpArgs a) {
  double s0 = 0.0, s1 = 0.0;
  if ((int)blockIdx.x < a.nblk) {
    const float lam = a.dev->f_lambda;
    for (int i = blockIdx.x * kGpThreads + threadIdx.x; i < a.n; i += a.nblk * kGpThreads) {
      const float inv = 1.f / fmaxf(1.f, fmaf(lam, a.w[i] * a.h[i], a.pins[i]));
      const float gx = a.rgx[i] * inv, gy = a.rgy[i] * inv;
      a.gx[i] = gx;
      a.gy[i] = gy;
      const double dx = (double)a.vx[i] - a.vpx[i], dy = (double)a.vy[i] - a.vpy[i];
      const double ex = (double)gx - a.gpx[i], ey = (double)gy - a.gpy[i];
      s0 += dx * dx + dy * dy;
      s1 += ex * ex + ey * ey;
    }
    block_pair(s0, s1, a.part);
  } else {
    if (a.region_ovf) return;   // fence regions: the density passes wrote the overflow partials
    const int b0 = blockIdx.x - a.nblk;
    for (long long b = (long long)b0 * kGpThreads + threadIdx.x; b < a.nbins; b += (long long)a.oblk * kGpThreads)
      s0 += ovf_term(a, b);
    __shared__ double r0[kGpThreads / 32];
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) s0 += __shfl_xor_sync(0xffffffffu, s0, o);
    if ((threadIdx.x & 31) == 0) r0[threadIdx.x >> 5] = s0;
    __syncthreads();
    if (threadIdx.x == 0) {
      double t = 0.0;
      for (int w = 0; w < kGpThreads / 32; w++) t += r0[w];
      a.part_ovf[2 * b0] = t;
      a.part_ovf[2 * b0 + 1] = 0.0;
    }
  }
}

// init helpers: u = v = clamp(x0); vp = v - eta g
__global__ void __launch_bounds__(kGpThreads) k_gp_start(GpArgs a, const float *x0, const float *y0) {
  const int i = blockIdx.x * kGpThreads + threadIdx.x;
  if (i >= a.n) return;
  const float x = clampf(x0[i], a.xl, a.xh - a.w[i]), y = clampf(y0[i], a.yl, a.yh - a.h[i]);
  a.ux[i] = x; a.uy[i] = y; a.vx[i] = x; a.vy[i] = y;
}
__global__ void __launch_bounds__(kGpThreads) k_gp_back(GpArgs a) {
  const int i = blockIdx.x * kGpThreads + threadIdx.x;
  if (i >= a.n) return;
  const float eta = a.dev->f_eta;
  a.vpx[i] = fmaf(-eta, a.gx[i], a.vx[i]);
  a.vpy[i] = fmaf(-eta, a.gy[i], a.vy[i]);
}
__global__ void __launch_bounds__(kGpThreads) k_gp_copy(float *dx, float *dy, const float *sx, const float *sy, int n) {
  const int i = blockIdx.x * kGpThreads + threadIdx.x;
  if (i < n) {
    dx[i] = sx[i];
    dy[i] = sy[i];
  }
}

}  // namespace

struct Gp {
  Ctx *c = nullptr;
  dp_gp_params p{};
  GpArgs a{};
  GpDev *dev = nullptr;
  double *out = nullptr;     // {obj, wl, energy, hpwl}
  cudaStream_t s_cap = nullptr;
  cudaGraphExec_t gexec_v[2] = {nullptr, nullptr};   // captured iterations without / with the sort kernels
  int64_t gexec_gen_v[2] = {-1, -1};   // Ctx::config_gen the iteration graphs were captured with
  int64_t gen = -1;          // Ctx::config_gen of the last gp_refresh
  double *region_ovf_buf = nullptr;   // fence regions: overflow partials of the density passes
  size_t region_ovf_cap = 0;
  bool initialised = false;
  std::vector<void *> allocs;
  int cell_blocks = 0;
};

namespace {

template <class T>
dp_status gp_alloc(Gp &g, T **p, size_t n) {
  void *q = nullptr;
  const cudaError_t e = cudaMalloc(&q, (n ? n : 1) * sizeof(T));
  if (e != cudaSuccess) return cuda_fail(e, "cudaMalloc (gp)");
  g.allocs.push_back(q);
  *p = static_cast<T *>(q);
  return DP_OK;
}

void gp_free(Gp *g) {
  if (!g) return;
  for (int v = 0; v < 2; v++)
    if (g->gexec_v[v]) cudaGraphExecDestroy(g->gexec_v[v]);
  if (g->s_cap) cudaStreamDestroy(g->s_cap);
  for (void *q : g->allocs) cudaFree(q);
  delete g;
}

struct GpDeviceGuard {
  int prev = -1;
  explicit GpDeviceGuard(int dev) {
    if (cudaGetDevice(&prev) != cudaSuccess) prev = -1;
    cudaSetDevice(dev);
  }
  ~GpDeviceGuard() {
    if (prev >= 0) cudaSetDevice(prev);
  }
};

void partials(Gp &g, int mode, cudaStream_t s) { k_gp_partials<<<g.a.nblk, kGpThreads, 0, s>>>(g.a, mode); }
void scalar(Gp &g, int op, cudaStream_t s) { k_gp_scalar<<<1, kGpThreads, 0, s>>>(g.a, op); }

// evaluation at (x, y) -> raw gradient rg; gamma / lambda from the device unless given
dp_status gp_eval(Gp &g, const float *x, const float *y, bool wa, bool den, bool dev_scalars, cudaStream_t s) {
  Ctx &c = *g.c;
  c.gamma_dev = dev_scalars || (wa && !den) ? &g.dev->f_gamma : nullptr;
  c.lambda_dev = dev_scalars ? &g.dev->f_lambda : nullptr;
  c.hpwl_fast = true;   // A37: the schedule's HPWL from fp32 pin positions, fused into the WA pass
  const dp_status st = eval_body_ext(c, x, y, 1.f, 1.f, g.a.rgx, g.a.rgy, g.out, g.out + 1, g.out + 2,
                                     wa ? g.out + 3 : nullptr, s, wa, den);
  c.gamma_dev = nullptr;
  c.lambda_dev = nullptr;
  c.hpwl_fast = false;
  return st;
}

// Constants that depend on the context's configuration (refreshed at init and whenever a
// dp_set_* changed it): the fixed cells (A34) and the movable area of A30's normalisation.
dp_status gp_refresh(Gp &g) {
  Ctx &c = *g.c;
  const int n = g.a.n;
  g.a.fixed = c.has_fixed ? c.d_fixed : nullptr;
  g.a.rho_fixed = c.has_fixed ? c.d_rho_fixed : nullptr;
  if (c.n_regions > 0) {   // A30 per region pass (density.cu k_region_overflow), summed by the schedule
    const size_t nreg = (size_t)(c.n_regions + 1) * g.a.oblk;
    if (!g.region_ovf_buf || g.region_ovf_cap < nreg) {
      double *p = nullptr;
      dp_status st = gp_alloc(g, &p, 2 * nreg);
      if (st != DP_OK) return st;
      DP_CUDA(cudaMemset(p, 0, sizeof(double) * 2 * nreg));
      g.region_ovf_buf = p;
      g.region_ovf_cap = nreg;
    }
    c.ovf_part = g.region_ovf_buf;
    c.ovf_blocks = g.a.oblk;
    c.ovf_target = g.a.target;
    g.a.region_ovf = g.region_ovf_buf;
    g.a.region_blk = (int)nreg;
  } else {
    c.ovf_part = nullptr;
    g.a.region_ovf = nullptr;
    g.a.region_blk = 0;
  }
  std::vector<float> w(n), h(n);
  std::vector<uint8_t> m(n, 0);
  DP_CUDA(cudaMemcpy(w.data(), c.d_cell_w, sizeof(float) * n, cudaMemcpyDeviceToHost));
  DP_CUDA(cudaMemcpy(h.data(), c.d_cell_h, sizeof(float) * n, cudaMemcpyDeviceToHost));
  if (c.has_fixed) DP_CUDA(cudaMemcpy(m.data(), c.d_fixed, n, cudaMemcpyDeviceToHost));
  double area = 0.0;
  for (int i = 0; i < n; i++)
    if (!m[i]) area += (double)w[i] * (double)h[i];
  DP_CUDA(cudaMemcpy(&g.dev->area_total, &area, sizeof(double), cudaMemcpyHostToDevice));
  g.gen = c.config_gen;
  return DP_OK;
}

// one GP iteration (the captured body): the step with alpha_k / coef from the previous scalar
// pass, the evaluation at v_{k+1}, one fused pass (preconditioner, next step's norms, overflow
// partials), one scalar pass (eq 18, gamma, history, alpha_{k+1}, a_{k+2})
dp_status gp_iteration(Gp &g, cudaStream_t s) {
  const int cb = g.cell_blocks;
  k_gp_update<<<cb, kGpThreads, 0, s>>>(g.a);
  dp_status st = gp_eval(g, g.a.vx, g.a.vy, true, true, true, s);
  if (st != DP_OK) return st;
  k_gp_post<<<g.a.nblk + g.a.oblk, kGpThreads, 0, s>>>(g.a);
  scalar(g, S_ITER_END, s);
  DP_CUDA(cudaGetLastError());
  return DP_OK;
}

}  // namespace
}  // namespace dp

using dp::Ctx;
using dp::Gp;

extern "C" {

void dp_gp_default_params(dp_gp_params *p) {
  if (!p) return;
  p->target_density = 1.0f;
  p->gamma_base_scale = 4.0f;
  p->lambda_scale = 8e-5f;
  p->mu_min = 0.95f;
  p->mu_max = 1.05f;
  p->dhpwl_ref = 3.5e5f;
  p->init_rms_bins = 0.01f;
  p->max_history = 4096;
  p->stop_overflow = 0.07f;
}

dp_status dp_gp_create(dp_ctx *ctx, const dp_gp_params *params, dp_gp **out) {
  if (!ctx || !out) return dp::fail(DP_ERR_INVALID_ARG, "ctx / out is NULL");
  *out = nullptr;
  Ctx *c = reinterpret_cast<Ctx *>(ctx);
  if (c->dist) return dp::fail(DP_ERR_UNSUPPORTED, "the GP loop runs on single-GPU contexts");
  dp_gp_params p;
  dp_gp_default_params(&p);
  if (params) p = *params;
  if (!(p.target_density > 0.f) || !(p.gamma_base_scale > 0.f) || !(p.lambda_scale >= 0.f) ||
      !(p.mu_min > 0.f) || !(p.mu_max >= p.mu_min) || !(p.dhpwl_ref > 0.f) || !(p.init_rms_bins > 0.f) ||
      p.max_history < 0 || !(p.stop_overflow >= 0.f))
    return dp::fail(DP_ERR_INVALID_ARG, "invalid dp_gp_params");
  dp::GpDeviceGuard guard(c->device);
  Gp *g = new Gp();
  g->c = c;
  g->p = p;
  const int n = c->num_cells;
  auto bail = [&](dp_status st) {
    dp::gp_free(g);
    return st;
  };
  dp::GpArgs &a = g->a;
  a.n = n;
  float **bufs[] = {&a.ux, &a.uy, &a.vx, &a.vy, &a.vpx, &a.vpy, &a.gx, &a.gy, &a.gpx, &a.gpy, &a.rgx, &a.rgy};
  for (float **b : bufs) {
    dp_status st = dp::gp_alloc(*g, b, (size_t)n);
    if (st != DP_OK) return bail(st);
  }
  a.w = c->d_cell_w;
  a.h = c->d_cell_h;
  a.pins = c->d_cell_pins;
  a.xl = (float)c->xl; a.yl = (float)c->yl; a.xh = (float)c->xh; a.yh = (float)c->yh;
  a.rho = c->d_rho;
  a.nbins = (long long)c->mx * c->my;
  a.rho_unit = std::ldexp(1.0, -dp::kRhoScaleLog2);
  a.target = p.target_density;
  // post-pass grid: 8 CTAs per SM for the cells (each thread a few cells, 11 loads each in flight;
  // 2 per SM left it latency-bound at 58 us for bigblue4), 4 per SM for the bins
  a.nblk = std::max(1, std::min(c->num_sms * 8, (n + dp::kGpThreads - 1) / dp::kGpThreads));
  a.bxby = c->bx * c->by;
  a.mu_min = p.mu_min; a.mu_max = p.mu_max; a.dhpwl_ref = p.dhpwl_ref;
  a.lambda_scale = p.lambda_scale; a.init_rms_bins = p.init_rms_bins; a.bx = c->bx;
  a.hist_cap = p.max_history;
  a.stop_overflow = p.stop_overflow;
  dp_status st;
  if ((st = dp::gp_alloc(*g, &a.part, 2 * (size_t)a.nblk)) != DP_OK) return bail(st);
  a.oblk = (int)std::max<long long>(1, std::min<long long>(c->num_sms * 4, (a.nbins + dp::kGpThreads - 1) / dp::kGpThreads));
  if ((st = dp::gp_alloc(*g, &a.part_ovf, 2 * (size_t)a.oblk)) != DP_OK) return bail(st);
  if ((st = dp::gp_alloc(*g, &g->dev, 1)) != DP_OK) return bail(st);
  if ((st = dp::gp_alloc(*g, &g->out, 4)) != DP_OK) return bail(st);
  if ((st = dp::gp_alloc(*g, &a.hist, (size_t)std::max(1, p.max_history) * dp::kHistCols)) != DP_OK) return bail(st);
  // zeroed: dp_gp_history copies the whole ring (compute-sanitizer initcheck)
  if (cudaMemset(a.hist, 0, sizeof(double) * (size_t)std::max(1, p.max_history) * dp::kHistCols) != cudaSuccess)
    return bail(dp::fail(DP_ERR_CUDA, "history memset"));
  a.dev = g->dev;
  a.out = g->out;
  g->cell_blocks = (n + dp::kGpThreads - 1) / dp::kGpThreads;
  // constants of the schedule: total cell area (A30) and gamma_base (A31), computed on the host
  {
    std::vector<float> w(n), h(n);
    if (cudaMemcpy(w.data(), c->d_cell_w, sizeof(float) * n, cudaMemcpyDeviceToHost) != cudaSuccess ||
        cudaMemcpy(h.data(), c->d_cell_h, sizeof(float) * n, cudaMemcpyDeviceToHost) != cudaSuccess)
      return bail(dp::fail(DP_ERR_CUDA, "cell sizes"));
    dp::GpDev d{};
    for (int i = 0; i < n; i++) d.area_total += (double)w[i] * (double)h[i];
    d.gamma_base = (double)p.gamma_base_scale * (c->bx + c->by);
    d.a = 1.0;
    if (cudaMemcpy(g->dev, &d, sizeof(d), cudaMemcpyHostToDevice) != cudaSuccess)
      return bail(dp::fail(DP_ERR_CUDA, "gp state upload"));
  }
  if (cudaStreamCreateWithFlags(&g->s_cap, cudaStreamNonBlocking) != cudaSuccess)
    return bail(dp::fail(DP_ERR_CUDA, "stream creation"));
  *out = reinterpret_cast<dp_gp *>(g);
  return DP_OK;
}

dp_status dp_gp_destroy(dp_gp *gp) {
  Gp *g = reinterpret_cast<Gp *>(gp);
  if (g) {
    dp::GpDeviceGuard guard(g->c->device);
    cudaDeviceSynchronize();
    dp::gp_free(g);
  }
  return DP_OK;
}

dp_status dp_gp_init(dp_gp *gp, const float *x0, const float *y0, dp_stream_t stream) {
  Gp *g = reinterpret_cast<Gp *>(gp);
  if (!g || !x0 || !y0) return dp::fail(DP_ERR_INVALID_ARG, "gp / x0 / y0 is NULL");
  Ctx &c = *g->c;
  dp::GpDeviceGuard guard(c.device);
  cudaStream_t s = (cudaStream_t)stream;
  DP_CUDA(cudaStreamSynchronize(s));
  dp_status st = dp::gp_refresh(*g);
  if (st != DP_OK) return st;
  st = dp::ctx_call_begin(c, s);
  if (st != DP_OK) return st;
  const int cb = g->cell_blocks;
  auto &a = g->a;
  DP_CUDA(cudaMemsetAsync(g->out, 0, 4 * sizeof(double), s));
  dp::k_gp_start<<<cb, dp::kGpThreads, 0, s>>>(a, x0, y0);
  // density alone at v: grad D, the map -> tau_0 -> gamma_0 (A31)
  if ((st = dp::gp_eval(*g, a.vx, a.vy, false, true, false, s)) != DP_OK) return st;
  if (!a.region_ovf) dp::partials(*g, dp::R_OVF, s);
  dp::scalar(*g, dp::S_INIT_TAU, s);
  dp::partials(*g, dp::R_L1, s);
  dp::scalar(*g, dp::S_INIT_L1D, s);
  // wirelength alone at v with gamma_0 -> lambda_0 (A32)
  if ((st = dp::gp_eval(*g, a.vx, a.vy, true, false, false, s)) != DP_OK) return st;
  dp::partials(*g, dp::R_L1, s);
  dp::scalar(*g, dp::S_INIT_LAMBDA, s);
  // full evaluation at v -> g_0, HPWL_0; v_{-1} and g_{-1} (A33)
  if ((st = dp::gp_eval(*g, a.vx, a.vy, true, true, true, s)) != DP_OK) return st;
  dp::k_gp_precond<<<cb, dp::kGpThreads, 0, s>>>(a);
  dp::partials(*g, dp::R_SQ, s);
  dp::scalar(*g, dp::S_INIT_ETA, s);
  dp::k_gp_back<<<cb, dp::kGpThreads, 0, s>>>(a);
  // evaluate at v_{-1}: swap the roles of (v, g) and (vp, gp) for one evaluation + precondition
  std::swap(a.vx, a.vpx); std::swap(a.vy, a.vpy); std::swap(a.gx, a.gpx); std::swap(a.gy, a.gpy);
  st = dp::gp_eval(*g, a.vx, a.vy, true, true, true, s);
  if (st == DP_OK) dp::k_gp_precond<<<cb, dp::kGpThreads, 0, s>>>(a);
  std::swap(a.vx, a.vpx); std::swap(a.vy, a.vpy); std::swap(a.gx, a.gpx); std::swap(a.gy, a.gpy);
  if (st != DP_OK) return st;
  dp::scalar(*g, dp::S_INIT_DONE, s);
  dp::partials(*g, dp::R_NORMS, s);   // alpha_0, a_1 and the first Nesterov coefficient (A28)
  dp::scalar(*g, dp::S_ALPHA, s);
  DP_CUDA(cudaGetLastError());
  g->initialised = true;
  return dp::ctx_call_end(c, s);
}

dp_status dp_gp_run(dp_gp *gp, int32_t iterations, dp_stream_t stream) {
  Gp *g = reinterpret_cast<Gp *>(gp);
  if (!g) return dp::fail(DP_ERR_INVALID_ARG, "gp is NULL");
  if (!g->initialised) return dp::fail(DP_ERR_INVALID_ARG, "dp_gp_init has not been called");
  if (iterations < 0) return dp::fail(DP_ERR_INVALID_ARG, "iterations < 0");
  Ctx &c = *g->c;
  dp::GpDeviceGuard guard(c.device);
  cudaStream_t s = (cudaStream_t)stream;
  if (g->gen != c.config_gen) {
    DP_CUDA(cudaStreamSynchronize(s));
    dp_status st = dp::gp_refresh(*g);
    if (st != DP_OK) return st;
  }
  if (c.profiling) {   // per-stage events: direct launches
    dp_status st = dp::ctx_call_begin(c, s);
    if (st != DP_OK) return st;
    for (int it = 0; it < iterations; it++)
      if ((st = dp::gp_iteration(*g, s)) != DP_OK) return st;
    return dp::ctx_call_end(c, s);
  }
  for (int v = 0; v < 2; v++)
    if (g->gexec_v[v] && g->gexec_gen_v[v] != c.config_gen) {   // dp_set_* since the capture: the body changed
      cudaGraphExecDestroy(g->gexec_v[v]);
      g->gexec_v[v] = nullptr;
    }
  // two captured iterations: [1] with the density sort kernels, [0] without (the list is kept;
  // chosen per iteration like the evaluation graphs)
  auto capture = [&](int v) -> dp_status {
    cudaGraph_t graph = nullptr;
    DP_CUDA(cudaStreamBeginCapture(g->s_cap, cudaStreamCaptureModeThreadLocal));
    c.omit_sort = v == 0;
    dp_status st = dp::gp_iteration(*g, g->s_cap);
    c.omit_sort = false;
    const cudaError_t ce = cudaStreamEndCapture(g->s_cap, &graph);
    if (st != DP_OK) {
      if (graph) cudaGraphDestroy(graph);
      return st;
    }
    if (ce != cudaSuccess) return dp::cuda_fail(ce, "cudaStreamEndCapture (gp)");
    const cudaError_t ie = cudaGraphInstantiateWithFlags(&g->gexec_v[v], graph, cudaGraphInstantiateFlagUseNodePriority);
    cudaGraphDestroy(graph);
    if (ie != cudaSuccess) {
      g->gexec_v[v] = nullptr;
      return dp::cuda_fail(ie, "cudaGraphInstantiate (gp)");
    }
    g->gexec_gen_v[v] = c.config_gen;
    return DP_OK;
  };
  dp_status st = dp::ctx_call_begin(c, s);
  if (st != DP_OK) return st;
  for (int it = 0; it < iterations; it++) {
    const int v = c.sort_variant();
    if (!g->gexec_v[v] && (st = capture(v)) != DP_OK) return st;
    DP_CUDA(cudaGraphLaunch(g->gexec_v[v], s));
    if (v == 1) c.sorted_once = true;
  }
  return dp::ctx_call_end(c, s);
}

dp_status dp_gp_positions(dp_gp *gp, float *x, float *y, dp_stream_t stream) {
  Gp *g = reinterpret_cast<Gp *>(gp);
  if (!g || !x || !y) return dp::fail(DP_ERR_INVALID_ARG, "gp / x / y is NULL");
  dp::GpDeviceGuard guard(g->c->device);
  cudaStream_t s = (cudaStream_t)stream;
  dp_status st = dp::ctx_call_begin(*g->c, s);
  if (st != DP_OK) return st;
  dp::k_gp_copy<<<g->cell_blocks, dp::kGpThreads, 0, s>>>(x, y, g->a.ux, g->a.uy, g->a.n);
  DP_CUDA(cudaGetLastError());
  return dp::ctx_call_end(*g->c, s);
}

dp_status dp_gp_debug_state(dp_gp *gp, float *u, float *v, float *vp, float *g, float *gp_prev, double *h_scalars) {
  Gp *G = reinterpret_cast<Gp *>(gp);
  if (!G || !h_scalars) return dp::fail(DP_ERR_INVALID_ARG, "gp / h_scalars is NULL");
  dp::GpDeviceGuard guard(G->c->device);
  DP_CUDA(cudaDeviceSynchronize());
  const size_t n = (size_t)G->a.n, b = n * sizeof(float);
  auto pair = [&](float *dst, const float *sx, const float *sy) -> cudaError_t {
    if (!dst) return cudaSuccess;
    cudaError_t e = cudaMemcpy(dst, sx, b, cudaMemcpyDeviceToDevice);
    return e != cudaSuccess ? e : cudaMemcpy(dst + n, sy, b, cudaMemcpyDeviceToDevice);
  };
  DP_CUDA(pair(u, G->a.ux, G->a.uy));
  DP_CUDA(pair(v, G->a.vx, G->a.vy));
  DP_CUDA(pair(vp, G->a.vpx, G->a.vpy));
  DP_CUDA(pair(g, G->a.gx, G->a.gy));
  DP_CUDA(pair(gp_prev, G->a.gpx, G->a.gpy));
  dp::GpDev d{};
  DP_CUDA(cudaMemcpy(&d, G->dev, sizeof(d), cudaMemcpyDeviceToHost));
  const double sc[9] = {d.a, d.lam, d.gamma, d.hpwl, d.tau, d.alpha, (double)d.k, (double)d.frozen, d.coef};
  for (int i = 0; i < 9; i++) h_scalars[i] = sc[i];
  return DP_OK;
}

dp_status dp_gp_history(dp_gp *gp, double *h_rows, int32_t max_rows, int32_t *rows) {
  Gp *g = reinterpret_cast<Gp *>(gp);
  if (!g || !rows || (max_rows > 0 && !h_rows)) return dp::fail(DP_ERR_INVALID_ARG, "gp / rows / h_rows is NULL");
  dp::GpDeviceGuard guard(g->c->device);
  DP_CUDA(cudaDeviceSynchronize());
  dp::GpDev d{};
  DP_CUDA(cudaMemcpy(&d, g->dev, sizeof(d), cudaMemcpyDeviceToHost));
  const int cap = g->a.hist_cap;
  const long long total = d.k;
  const long long avail = std::min<long long>(total, cap);
  const long long first = total - avail;
  const int n = (int)std::min<long long>(avail, max_rows);
  std::vector<double> all((size_t)std::max(cap, 1) * dp::kHistCols);
  if (n > 0) DP_CUDA(cudaMemcpy(all.data(), g->a.hist, all.size() * sizeof(double), cudaMemcpyDeviceToHost));
  for (int r = 0; r < n; r++) {   // oldest first
    const long long k = first + r;
    const double *src = all.data() + (size_t)(k % cap) * dp::kHistCols;
    for (int j = 0; j < dp::kHistCols; j++) h_rows[(size_t)r * dp::kHistCols + j] = src[j];
  }
  *rows = n;
  return DP_OK;
}

}  // extern "C"
