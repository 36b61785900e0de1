// dp_api.cu — the C ABI of libdp (include/dp.h): validation, dp_create (host-side layout
// building), evaluation orchestration over two streams, and the test hooks.
//
// dp_create does all data-dependent preparation once:
//   * pins are put in net order (net2pin applied), degree 0/1 nets are dropped (reading A3);
//   * nets of degree <= kWaMaxDeg are sorted by the median cell index of their pins and cut
//     into chunks of ~kWaChunkPins pins; each chunk gets the densest window of kWaWindow
//     consecutive cells (its positions and gradients live in shared memory);
//   * inside a chunk nets are grouped by lanes-per-net G (degree <= 8 G) and sorted by degree,
//     32/G nets form a warp group whose pins are stored slot-major so every load coalesces;
//   * nets of larger degree keep a CSR list for the CTA-per-net kernel;
//   * the own-cell range, large-cell list, tile grid, FFT twiddles and wavenumbers.
// dp_eval forks the caller stream into a WA stream and a density stream, joins, combines.
#include <dlfcn.h>

#include <algorithm>
#include <cmath>
#include <cstdlib>
#include <cstring>
#include <numeric>
#include <string>
#include <vector>
#include <map>
#include <mutex>
#include <cstring>

#include "dp_internal.h"

namespace dp {

static thread_local std::string g_err;

void set_error(const std::string &msg) { g_err = msg; }
dp_status fail(dp_status st, const std::string &msg) {
  g_err = msg;
  return st;
}
dp_status cuda_fail(cudaError_t e, const char *what) {
  g_err = std::string("CUDA error ") + cudaGetErrorName(e) + " (" + cudaGetErrorString(e) + ") in " + what;
  return e == cudaErrorMemoryAllocation ? DP_ERR_OUT_OF_MEMORY : DP_ERR_CUDA;
}

namespace {

struct DeviceGuard {
  int prev = -1;
  explicit DeviceGuard(int dev) {
    if (cudaGetDevice(&prev) != cudaSuccess) prev = -1;
    if (prev != dev) cudaSetDevice(dev);
  }
  ~DeviceGuard() {
    int cur = -1;
    if (prev >= 0 && cudaGetDevice(&cur) == cudaSuccess && cur != prev) cudaSetDevice(prev);
  }
};

template <class T>
dp_status dev_alloc(Ctx &c, T **p, size_t n) {
  *p = nullptr;
  if (n == 0) n = 1;
  void *q = nullptr;
  cudaError_t e = cudaMalloc(&q, n * sizeof(T));
  if (e != cudaSuccess) return cuda_fail(e, "cudaMalloc");
  c.allocations.push_back(q);
  c.device_bytes += (int64_t)(n * sizeof(T));
  *p = static_cast<T *>(q);
  return DP_OK;
}

template <class T>
dp_status dev_upload(Ctx &c, T **p, const std::vector<T> &v) {
  dp_status st = dev_alloc(c, p, v.size());
  if (st != DP_OK) return st;
  if (!v.empty()) DP_CUDA(cudaMemcpy(*p, v.data(), v.size() * sizeof(T), cudaMemcpyHostToDevice));
  return DP_OK;
}

bool is_pow2(int v) { return v > 0 && (v & (v - 1)) == 0; }
int ilog2(int v) {
  int r = 0;
  while ((1 << r) < v) r++;
  return r;
}

dp_status validate(const dp_netlist *nl, const dp_grid *g) {
  if (!nl || !g) return fail(DP_ERR_INVALID_ARG, "netlist or grid is NULL");
  if (nl->num_cells < 1) return fail(DP_ERR_INVALID_ARG, "num_cells must be >= 1");
  if (nl->num_nets < 0 || nl->num_pins < 0) return fail(DP_ERR_INVALID_ARG, "negative net or pin count");
  if (!nl->net_start || !nl->cell_w || !nl->cell_h) return fail(DP_ERR_INVALID_ARG, "net_start, cell_w and cell_h are required");
  if (nl->num_pins > 0 && (!nl->pin2cell || !nl->pin_dx || !nl->pin_dy))
    return fail(DP_ERR_INVALID_ARG, "pin2cell, pin_dx, pin_dy are required when num_pins > 0");
  if (nl->net_start[0] != 0) return fail(DP_ERR_INVALID_ARG, "net_start[0] must be 0");
  for (int32_t e = 0; e < nl->num_nets; e++)
    if (nl->net_start[e + 1] < nl->net_start[e]) return fail(DP_ERR_INVALID_ARG, "net_start must be nondecreasing (net " + std::to_string(e) + ")");
  if (nl->net_start[nl->num_nets] != nl->num_pins) return fail(DP_ERR_INVALID_ARG, "net_start[num_nets] must equal num_pins");
  for (int32_t p = 0; p < nl->num_pins; p++) {
    const int32_t c = nl->pin2cell[p];
    if (c < 0 || c >= nl->num_cells) return fail(DP_ERR_INVALID_ARG, "pin2cell out of range at pin " + std::to_string(p));
    if (!std::isfinite(nl->pin_dx[p]) || !std::isfinite(nl->pin_dy[p])) return fail(DP_ERR_INVALID_ARG, "non-finite pin offset at pin " + std::to_string(p));
  }
  if (nl->net2pin) {
    std::vector<uint8_t> seen(nl->num_pins, 0);
    for (int32_t s = 0; s < nl->num_pins; s++) {
      const int32_t p = nl->net2pin[s];
      if (p < 0 || p >= nl->num_pins || seen[p]) return fail(DP_ERR_INVALID_ARG, "net2pin is not a permutation");
      seen[p] = 1;
    }
  }
  for (int32_t c = 0; c < nl->num_cells; c++) {
    const float w = nl->cell_w[c], h = nl->cell_h[c];
    if (!std::isfinite(w) || !std::isfinite(h) || w < 0.f || h < 0.f) return fail(DP_ERR_INVALID_ARG, "cell sizes must be finite and >= 0 (cell " + std::to_string(c) + ")");
  }
  if (nl->net_weight)
    for (int32_t e = 0; e < nl->num_nets; e++)
      if (!std::isfinite(nl->net_weight[e]) || nl->net_weight[e] < 0.f) return fail(DP_ERR_INVALID_ARG, "net weights must be finite and >= 0");
  if (!(std::isfinite(g->xl) && std::isfinite(g->xh) && std::isfinite(g->yl) && std::isfinite(g->yh)) || !(g->xh > g->xl) || !(g->yh > g->yl))
    return fail(DP_ERR_INVALID_ARG, "degenerate or non-finite placement region");
  if (g->stretch != 0 && g->stretch != 1) return fail(DP_ERR_INVALID_ARG, "stretch must be 0 or 1");
  if (!is_pow2(g->bins_x) || !is_pow2(g->bins_y) || g->bins_x < 16 || g->bins_y < 16 || g->bins_x > 4096 || g->bins_y > 4096)
    return fail(DP_ERR_UNSUPPORTED, "bins_x and bins_y must be powers of two in [16, 4096]");
  return DP_OK;
}

// Dynamic shared-memory opt-ins are per device: the maxima configured so far on each device
// (several contexts, possibly on several GPUs, in one process).
struct DeviceConfig {
  WaCaps wa{4, 4, 4, 4};
  bool wa_set = false;
  int max_m = 0, max_tiles = 0, max_tile = 0;
};
std::mutex g_cfg_mutex;
std::map<int, DeviceConfig> g_cfg;

int g_class(int d) {  // log2 of lanes per net
  int g = 0;
  while ((kWaPpl << g) < d) g++;
  return g;
}

// The global WA work plan, a pure function of the netlist — identical on every
// rank and for every number of ranks.  Units, in CTA order of the WA kernel:
//   [nets of degree > kWarpNetMax, one CTA each | blocks of 8 nets of degree (kWaMaxDeg,
//    kWarpNetMax], a warp each | chunks of <= kWaChunkPins pins of the small nets in locality
//    order (median cell index)]
// Ranks take contiguous unit ranges balanced by pin count ("nets are partitioned for WA",
// BASELINE north_star); a unit's WA partial has one global slot, so partial sums, chunk fixed-
// point scales and hence the deterministic-mode gradient are the same for any world size.
struct WaPlan {
  std::vector<int32_t> small;                         // locality order
  std::vector<std::pair<size_t, size_t>> chunk_rng;   // [i, j) into small
  std::vector<int32_t> big;                           // degree-descending
  int32_t n_huge = 0, n_wblk = 0;
  std::vector<int64_t> unit_pins;
  std::vector<int32_t> unit_lo;                       // [world + 1]
  int32_t units() const { return n_huge + n_wblk + (int32_t)chunk_rng.size(); }
};

WaPlan wa_plan(const dp_netlist *nl, int world) {
  WaPlan P;
  // DP_WA_CHUNK = pins per chunk (A/B; smaller chunks stage less shared memory per CTA)
  const char *ce = std::getenv("DP_WA_CHUNK");
  const int chunk_pins = ce ? std::max(256, std::min(kWaChunkPins, std::atoi(ce))) : kWaChunkPins;
  auto pin_of = [&](int32_t slot) { return nl->net2pin ? nl->net2pin[slot] : slot; };
  auto deg = [&](int32_t e) { return nl->net_start[e + 1] - nl->net_start[e]; };
  for (int32_t e = 0; e < nl->num_nets; e++) {
    const int d = deg(e);
    if (d < 2) continue;  // reading A3: degree 0/1 contribute nothing
    (d > kWaMaxDeg ? P.big : P.small).push_back(e);
  }
  std::vector<int32_t> key(nl->num_nets, 0), tmp;
  for (int32_t e : P.small) {
    tmp.clear();
    for (int32_t k = nl->net_start[e]; k < nl->net_start[e + 1]; k++) tmp.push_back(nl->pin2cell[pin_of(k)]);
    std::nth_element(tmp.begin(), tmp.begin() + tmp.size() / 2, tmp.end());
    key[e] = tmp[tmp.size() / 2];
  }
  std::stable_sort(P.small.begin(), P.small.end(), [&](int32_t a, int32_t b) { return key[a] < key[b]; });
  std::stable_sort(P.big.begin(), P.big.end(), [&](int32_t a, int32_t b) { return deg(a) > deg(b); });
  while (P.n_huge < (int32_t)P.big.size() && deg(P.big[P.n_huge]) > kWarpNetMax) P.n_huge++;
  constexpr int kWarpNets = kWarpNetThreads / 32;
  P.n_wblk = ((int32_t)P.big.size() - P.n_huge + kWarpNets - 1) / kWarpNets;
  for (size_t i = 0; i < P.small.size();) {   // nets until the pin budget is reached (at least one)
    size_t j = i;
    int pins = 0;
    while (j < P.small.size()) {
      const int d = deg(P.small[j]);
      if (j > i && pins + d > chunk_pins) break;
      pins += d;
      j++;
    }
    P.chunk_rng.push_back({i, j});
    i = j;
  }
  for (int32_t u = 0; u < P.n_huge; u++) P.unit_pins.push_back(deg(P.big[u]));
  for (int32_t b = 0; b < P.n_wblk; b++) {
    int64_t n = 0;
    for (int32_t q = P.n_huge + b * kWarpNets; q < std::min<int32_t>((int32_t)P.big.size(), P.n_huge + (b + 1) * kWarpNets); q++)
      n += deg(P.big[q]);
    P.unit_pins.push_back(n);
  }
  for (const auto &r : P.chunk_rng) {
    int64_t n = 0;
    for (size_t q = r.first; q < r.second; q++) n += deg(P.small[q]);
    P.unit_pins.push_back(n);
  }
  // rank of a unit: the one whose share of the pin total contains the unit's midpoint
  const int32_t U = P.units();
  int64_t total = 0;
  for (int64_t n : P.unit_pins) total += n;
  P.unit_lo.assign(world + 1, U);
  P.unit_lo[0] = 0;
  int64_t acc = 0;
  int r = 1;
  for (int32_t u = 0; u < U && r < world; u++) {
    const long double mid = (long double)acc + 0.5L * (long double)P.unit_pins[u];
    while (r < world && mid * world >= (long double)total * r) P.unit_lo[r++] = u;
    acc += P.unit_pins[u];
  }
  while (r < world) P.unit_lo[r++] = U;
  return P;
}

// Cells: world equal blocks of ceil(num_cells / world) (the gradient reduce-scatter's blocks);
// rank r owns [r B, min((r+1) B, num_cells)) for the density scatter and gather.  Nets: the nets
// of the rank's WA units (mask 3 = evaluated and counted; every net of degree >= 2 on exactly
// one rank).
int32_t cell_block(int32_t n, int world) { return (int32_t)(((int64_t)n + world - 1) / world); }

void plan(const dp_netlist *nl, int rank, int world, int32_t &cb, int32_t &ce, std::vector<uint8_t> *mask,
          const WaPlan *wp = nullptr) {
  const int32_t B = cell_block(nl->num_cells, world);
  cb = (int32_t)std::min<int64_t>(nl->num_cells, (int64_t)B * rank);
  ce = (int32_t)std::min<int64_t>(nl->num_cells, (int64_t)B * (rank + 1));
  if (!mask) return;
  WaPlan local;
  if (!wp) {
    local = wa_plan(nl, world);
    wp = &local;
  }
  mask->assign(nl->num_nets, 0);
  constexpr int kWarpNets = kWarpNetThreads / 32;
  for (int32_t u = wp->unit_lo[rank]; u < wp->unit_lo[rank + 1]; u++) {
    if (u < wp->n_huge) {
      (*mask)[wp->big[u]] = 3;
    } else if (u < wp->n_huge + wp->n_wblk) {
      const int32_t b = u - wp->n_huge;
      for (int32_t q = wp->n_huge + b * kWarpNets; q < std::min<int32_t>((int32_t)wp->big.size(), wp->n_huge + (b + 1) * kWarpNets); q++)
        (*mask)[wp->big[q]] = 3;
    } else {
      const auto &rg = wp->chunk_rng[u - wp->n_huge - wp->n_wblk];
      for (size_t q = rg.first; q < rg.second; q++) (*mask)[wp->small[q]] = 3;
    }
  }
}

dp_status build_wa(Ctx &c, const dp_netlist *nl, const WaPlan &P) {
  const int32_t ncells = nl->num_cells;
  auto pin_of = [&](int32_t slot) { return nl->net2pin ? nl->net2pin[slot] : slot; };
  // this rank's units: huge nets [h0, h1), warp blocks [w0, w1), chunks [k0, k1) (global indices)
  const int32_t u0 = P.unit_lo[c.rank], u1 = P.unit_lo[c.rank + 1];
  auto clip = [&](int32_t lo, int32_t hi, int32_t &a0, int32_t &a1) {
    a0 = std::max(u0, lo) - lo;
    a1 = std::max(a0, std::min(u1, hi) - lo);
  };
  int32_t h0, h1, w0, w1, k0, k1;
  clip(0, P.n_huge, h0, h1);
  clip(P.n_huge, P.n_huge + P.n_wblk, w0, w1);
  clip(P.n_huge + P.n_wblk, P.units(), k0, k1);
  c.part_base = u0;
  c.n_wa_part = P.units();
  const std::vector<int32_t> &small = P.small;
  std::vector<Chunk> chunks;
  std::vector<WarpGroup> wgs;
  std::vector<int32_t> net_deg, pin_cell, far_cells;
  std::vector<float> net_w, pin_dx, pin_dy;
  WaCaps caps{4, 4, 4, 4};
  auto up4 = [](int v) { return (v + 3) & ~3; };
  std::vector<int32_t> cells, far;
  for (int32_t kc = k0; kc < k1; kc++) {
    const size_t i = P.chunk_rng[kc].first, j = P.chunk_rng[kc].second;
    // densest window of kWaWindow consecutive cells, start aligned to 4 cells (16 bytes) so
    // the kernel can stage x / y with bulk async copies
    cells.clear();
    for (size_t q = i; q < j; q++)
      for (int32_t k = nl->net_start[small[q]]; k < nl->net_start[small[q] + 1]; k++) cells.push_back(nl->pin2cell[pin_of(k)]);
    std::sort(cells.begin(), cells.end());
    const int win_n0 = std::min<int32_t>(kWaWindow, ncells);
    int32_t best_lo = cells[0];
    size_t best = 0, lo = 0;
    for (size_t hi = 0; hi < cells.size(); hi++) {
      while (cells[hi] - cells[lo] >= std::max(1, win_n0 - 3)) lo++;
      if (hi - lo + 1 > best) {
        best = hi - lo + 1;
        best_lo = cells[lo];
      }
    }
    best_lo = std::max(0, std::min(best_lo, ncells - win_n0)) & ~3;
    const int win_n = std::min<int32_t>(kWaWindow, ncells - best_lo);
    // far cells: distinct cells of the chunk outside the window
    far.clear();
    for (int32_t cc : cells)
      if (cc < best_lo || cc >= best_lo + win_n) far.push_back(cc);
    far.erase(std::unique(far.begin(), far.end()), far.end());   // cells are sorted
    auto slot_of = [&](int32_t cc) -> int32_t {
      if (cc >= best_lo && cc < best_lo + win_n) return cc - best_lo;
      return kWaWindow + (int32_t)(std::lower_bound(far.begin(), far.end(), cc) - far.begin());
    };
    auto pad4 = [&]() {
      while (pin_cell.size() & 3) {
        pin_cell.push_back(0);
        pin_dx.push_back(0.f);
        pin_dy.push_back(0.f);
      }
      while (net_deg.size() & 3) {
        net_deg.push_back(0);
        net_w.push_back(0.f);
      }
    };
    pad4();
    Chunk ch;
    ch.wg_begin = (int32_t)wgs.size();
    ch.win_lo = best_lo;
    ch.win_n = win_n;
    ch.pin_begin = (int32_t)pin_cell.size();
    ch.net_begin = (int32_t)net_deg.size();
    ch.far_begin = (int32_t)far_cells.size();
    ch.far_n = (int32_t)far.size();
    ch.far_pad = up4(ch.far_n);
    far_cells.insert(far_cells.end(), far.begin(), far.end());
    while ((int32_t)far_cells.size() < ch.far_begin + ch.far_pad) far_cells.push_back(0);
    {
      // int32 fixed-point scale of the gradient slots: |dWL_e/dx_i| <= (2 + d/2) w_e per pin
      // (max pin: 1 + (d-1)/e; others: <= 1 + 1/e, per side), so a slot's sum is bounded by
      // the sum of its pins' bounds; pick 2^k with bound * 2^k < 2^30.
      std::vector<double> bound(kWaWindow + far.size() + 1, 0.0);
      for (size_t q = i; q < j; q++) {
        const int32_t e = small[q];
        const int d = nl->net_start[e + 1] - nl->net_start[e];
        const double we = nl->net_weight ? (double)nl->net_weight[e] : 1.0;
        for (int32_t k = nl->net_start[e]; k < nl->net_start[e + 1]; k++)
          bound[slot_of(nl->pin2cell[pin_of(k)])] += (2.0 + 0.5 * d) * we;
      }
      const double bmax = std::max(1e-30, *std::max_element(bound.begin(), bound.end()));
      int k = (int)std::floor(std::log2(double(1 << 30) / bmax));
      ch.scale_log2 = std::max(-100, std::min(k, 100));
    }
    // group nets by lanes-per-net class, largest class first, degree-descending inside
    std::vector<std::vector<int32_t>> cls(6);
    for (size_t q = i; q < j; q++) {
      const int d = nl->net_start[small[q] + 1] - nl->net_start[small[q]];
      cls[g_class(d)].push_back(small[q]);
    }
    for (int g = 5; g >= 0; g--) {
      auto &v = cls[g];
      std::stable_sort(v.begin(), v.end(), [&](int32_t a, int32_t b) {
        return (nl->net_start[a + 1] - nl->net_start[a]) > (nl->net_start[b + 1] - nl->net_start[b]);
      });
      const int per = 32 >> g, G = 1 << g;
      for (size_t q = 0; q < v.size(); q += per) {
        WarpGroup wg;
        wg.pin_base = (int32_t)pin_cell.size() - ch.pin_begin;
        wg.net_base = (int32_t)net_deg.size() - ch.net_begin;
        wg.nnets = (int32_t)std::min<size_t>(per, v.size() - q);
        wg.g_log2 = g;
        int dmax = 0;
        bool pairs = (g == 0);
        for (int n = 0; n < wg.nnets; n++) {
          const int32_t e = v[q + n];
          const int d = nl->net_start[e + 1] - nl->net_start[e];
          dmax = std::max(dmax, d);
          pairs = pairs && d == 2;
          net_deg.push_back(d | (int32_t)0x80000000u);   // counted: every own net (one rank per net)
          net_w.push_back(nl->net_weight ? nl->net_weight[e] : 1.f);
        }
        wg.slots = (dmax + G - 1) / G;
        wg.flags = pairs ? 1 : 0;
        for (int s = 0; s < wg.slots; s++)
          for (int L = 0; L < 32; L++) {
            const int gi = L >> g, jj = L & (G - 1);
            if (gi >= wg.nnets) continue;
            const int32_t e = v[q + gi];
            const int d = nl->net_start[e + 1] - nl->net_start[e];
            const int k = s * G + jj;
            if (k >= d) continue;
            const int32_t p = pin_of(nl->net_start[e] + k);
            pin_cell.push_back(slot_of(nl->pin2cell[p]));
            pin_dx.push_back(nl->pin_dx[p]);
            pin_dy.push_back(nl->pin_dy[p]);
          }
        wgs.push_back(wg);
      }
    }
    ch.wg_n = (int32_t)wgs.size() - ch.wg_begin;
    pad4();
    ch.pin_n = (int32_t)pin_cell.size() - ch.pin_begin;
    ch.net_n = (int32_t)net_deg.size() - ch.net_begin;
    caps.pins = std::max(caps.pins, ch.pin_n);
    caps.nets = std::max(caps.nets, ch.net_n);
    caps.groups = std::max(caps.groups, up4(ch.wg_n));
    caps.far = std::max(caps.far, ch.far_pad);
    chunks.push_back(ch);
  }
  c.n_chunks = (int32_t)chunks.size();
  c.n_wgroups = (int32_t)wgs.size();
  c.n_wa_nets = (int32_t)net_deg.size();
  c.n_wa_pins = (int32_t)pin_cell.size();
  {   // shared-memory opt-in: per device (cudaFuncSetAttribute is), the maxima over its contexts
    std::lock_guard<std::mutex> lock(g_cfg_mutex);
    DeviceConfig &dc = g_cfg[c.device];
    WaCaps m{std::max(dc.wa.pins, caps.pins), std::max(dc.wa.nets, caps.nets),
             std::max(dc.wa.groups, caps.groups), std::max(dc.wa.far, caps.far)};
    if (wa_smem_bytes(m) > 227 * 1024) return fail(DP_ERR_UNSUPPORTED, "WA chunk staging exceeds shared memory");
    if (!dc.wa_set || m.pins != dc.wa.pins || m.nets != dc.wa.nets || m.groups != dc.wa.groups ||
        m.far != dc.wa.far) {
      DP_CUDA(wa_configure(m));
      dc.wa = m;
      dc.wa_set = true;
    }
    c.wa_caps = caps;
  }
  dp_status st;
  if ((st = dev_upload(c, &c.d_chunks, chunks)) != DP_OK) return st;
  if ((st = dev_upload(c, &c.d_wgroups, wgs)) != DP_OK) return st;
  if ((st = dev_upload(c, &c.d_net_deg, net_deg)) != DP_OK) return st;
  if ((st = dev_upload(c, &c.d_net_w, net_w)) != DP_OK) return st;
  if ((st = dev_upload(c, &c.d_pin_cell, pin_cell)) != DP_OK) return st;
  if ((st = dev_upload(c, &c.d_pin_dx, pin_dx)) != DP_OK) return st;
  if ((st = dev_upload(c, &c.d_pin_dy, pin_dy)) != DP_OK) return st;
  if ((st = dev_upload(c, &c.d_far_cells, far_cells)) != DP_OK) return st;
  // ---- big nets: this rank's huge nets, then its warp-block nets (largest first: the longest
  // CTAs start in the first wave) ----
  constexpr int kWarpNets = kWarpNetThreads / 32;
  std::vector<int32_t> big(P.big.begin() + h0, P.big.begin() + h1);
  for (int32_t q = P.n_huge + w0 * kWarpNets; q < std::min<int32_t>((int32_t)P.big.size(), P.n_huge + w1 * kWarpNets); q++)
    big.push_back(P.big[q]);
  c.big_stage = big.empty() ? 0 : std::min(kBigStage, nl->net_start[big[0] + 1] - nl->net_start[big[0]]);
  std::vector<int32_t> bstart{0}, bflags, bcell;
  std::vector<float> bw, bdx, bdy;
  for (int32_t e : big) {
    for (int32_t k = nl->net_start[e]; k < nl->net_start[e + 1]; k++) {
      const int32_t p = pin_of(k);
      bcell.push_back(nl->pin2cell[p]);
      bdx.push_back(nl->pin_dx[p]);
      bdy.push_back(nl->pin_dy[p]);
    }
    bstart.push_back((int32_t)bcell.size());
    bflags.push_back(1);
    bw.push_back(nl->net_weight ? nl->net_weight[e] : 1.f);
  }
  c.n_big = (int32_t)big.size();
  c.n_huge = h1 - h0;
  if ((st = dev_upload(c, &c.d_big_start, bstart)) != DP_OK) return st;
  if ((st = dev_upload(c, &c.d_big_flags, bflags)) != DP_OK) return st;
  if ((st = dev_upload(c, &c.d_big_w, bw)) != DP_OK) return st;
  if ((st = dev_upload(c, &c.d_big_cell, bcell)) != DP_OK) return st;
  if ((st = dev_upload(c, &c.d_big_dx, bdx)) != DP_OK) return st;
  if ((st = dev_upload(c, &c.d_big_dy, bdy)) != DP_OK) return st;
  return DP_OK;
}

// warp-FFT four-step twiddles W_N^{n1 k2}, n1 < 32, k2 < N / 32, laid out [k2][n1] (fp64-rounded)
std::vector<float2> twiddles2(int n) {
  const int K = std::max(1, n / 32);
  std::vector<float2> t((size_t)K * 32);
  for (int k2 = 0; k2 < K; k2++)
    for (int n1 = 0; n1 < 32; n1++) {
      const double a = -2.0 * M_PI * (double)((n1 * k2) % n) / n;
      t[(size_t)k2 * 32 + n1] = make_float2((float)std::cos(a), (float)std::sin(a));
    }
  return t;
}

std::vector<float2> twiddles(int n) {  // exp(-2 pi i k / n), k < n/2, from fp64
  std::vector<float2> t(n / 2);
  for (int k = 0; k < n / 2; k++) {
    const double a = 2.0 * M_PI * k / n;
    t[k] = make_float2((float)std::cos(a), (float)-std::sin(a));
  }
  return t;
}
std::vector<float2> twiddles_full(int n) {  // exp(-2 pi i k / n), k < n, from fp64 (CTA FFT)
  std::vector<float2> t(n);
  for (int k = 0; k < n; k++) {
    const double a = 2.0 * M_PI * k / n;
    t[k] = make_float2((float)std::cos(a), (float)-std::sin(a));
  }
  return t;
}
std::vector<float2> phases(int n) {  // exp(-i pi k / 2n), k < n
  std::vector<float2> t(n);
  for (int k = 0; k < n; k++) {
    const double a = M_PI * k / (2.0 * n);
    t[k] = make_float2((float)std::cos(a), (float)-std::sin(a));
  }
  return t;
}

dp_status build_density(Ctx &c, const dp_netlist *nl) {
  c.n_own = c.cell_end - c.cell_begin;
  std::vector<float> w(nl->cell_w + c.cell_begin, nl->cell_w + c.cell_end);
  std::vector<float> h(nl->cell_h + c.cell_begin, nl->cell_h + c.cell_end);
  std::vector<int32_t> large;
  for (int32_t i = 0; i < c.n_own; i++)
    if ((double)w[i] > 2.0 * c.bx || (double)h[i] > 2.0 * c.by) large.push_back(i);
  c.n_large = (int32_t)large.size();
  c.tile = std::min(kTile, std::min(c.mx, c.my));
  c.tiles_x = c.mx / c.tile;
  c.tiles_y = c.my / c.tile;
  const int ntiles = c.tiles_x * c.tiles_y;
  const size_t nb = (size_t)c.mx * c.my;
  dp_status st;
  if ((st = dev_upload(c, &c.d_cell_w, w)) != DP_OK) return st;
  if ((st = dev_upload(c, &c.d_cell_h, h)) != DP_OK) return st;
  if ((st = dev_upload(c, &c.d_large, large)) != DP_OK) return st;
  if ((st = dev_alloc(c, &c.d_tile_cnt, (size_t)ntiles * kCntStride)) != DP_OK) return st;
  DP_CUDA(cudaMemset(c.d_tile_cnt, 0, sizeof(int32_t) * ntiles * kCntStride));
  if ((st = dev_alloc(c, &c.d_tile_cursor, (size_t)ntiles * kCntStride)) != DP_OK) return st;
  if ((st = dev_alloc(c, &c.d_tile_off, ntiles + 1)) != DP_OK) return st;
  // sort records; padded by 8 so staged copies may round their range to 4-record multiples
  // (16-byte records with a per-cell-size constant table measured slower inside the step:
  // 4389 vs 4586 evals/s)
  if ((st = dev_alloc(c, &c.d_rec, c.n_own + 8)) != DP_OK) return st;
  if ((st = dev_alloc(c, &c.d_rec_rc, c.n_own + 8)) != DP_OK) return st;
  if ((st = dev_alloc(c, &c.d_rec_cell, c.n_own + 8)) != DP_OK) return st;
  if ((st = dev_alloc(c, &c.d_rec_wh, c.n_own + 8)) != DP_OK) return st;
  if ((st = dev_alloc(c, &c.d_sortctl, 4)) != DP_OK) return st;
  {
    const int32_t ctl[4] = {1, 0, 0, 0};   // the first evaluation sorts
    DP_CUDA(cudaMemcpy(c.d_sortctl, ctl, sizeof(ctl), cudaMemcpyHostToDevice));
    // DP_REUSE_SORT=0: sort on every evaluation.  Reuse is the default at every size since the
    // sort kernels are left out of the captured graph: adaptec1 13210 -> 15350
    // evals/s on the walk, GP 113 -> 112 us per iteration (with the kernels returning early instead,
    // reuse had measured slower there: 114 -> 120 us)
    const char *e = std::getenv("DP_REUSE_SORT");
    c.reuse_sort = e ? std::atoi(e) != 0 : true;
    // DP_SORT_COND=1: the sort kernels inside a graph IF node instead of returning early (measured
    // equal at bigblue4, ~7 us slower per GP iteration at adaptec1)
    const char *he = std::getenv("DP_SORT_HOST");
    c.sort_host = !(he && std::atoi(he) == 0);
    const char *sm = std::getenv("DP_SCATTER_MERGE");
    c.scatter_merge = sm && std::atoi(sm) == 2 ? 2 : 1;
    const char *rh = std::getenv("DP_REC_HINT");
    c.rec_hint = rh && std::atoi(rh) != 0;
    const char *eg = std::getenv("DP_EARLY_GATHER");
    c.early_gather = !(eg && std::atoi(eg) == 0);
    const char *ee = std::getenv("DP_EARLY");
    c.early_scatter = !(ee && std::atoi(ee) == 0);
    const char *se = std::getenv("DP_SORT_EVERY");
    c.sort_every = se ? std::max(1, std::atoi(se)) : 8;
    DP_CUDA(cudaHostAlloc(&c.h_ctl, sizeof(int32_t), cudaHostAllocMapped));
    *c.h_ctl = 0;
    DP_CUDA(cudaHostGetDevicePointer(reinterpret_cast<void **>(&c.h_ctl_dev), c.h_ctl, 0));
    const char *ge = std::getenv("DP_GATHER_RC");
    c.gather_rc = ge && std::atoi(ge) != 0;
    const char *fe = std::getenv("DP_FUSE_COMBINE");
    c.fuse_combine = fe && std::atoi(fe) != 0;
    const char *ce = std::getenv("DP_SORT_COND");
    c.sort_cond = ce && std::atoi(ce) != 0;
    // re-sort once more than this share of the small cells has left its tile (DP_RESORT_PCT,
    // default 5 %: a stray costs its nine map updates as global reductions, a sort ~50 us)
    const char *pe = std::getenv("DP_RESORT_PCT");
    const double pct = pe ? std::atof(pe) : 5.0;
    c.resort_thr = (int32_t)std::min(2.0e9, std::max(0.0, pct * 0.01 * (double)c.n_own));
  }
  // the maps of the hot path in one arena (rho int64, t, spec, sxy, xi): the density
  // stream's L2 persisting window (create)
  {
    unsigned char *arena = nullptr;
    c.maps_bytes = nb * (sizeof(unsigned long long) + sizeof(float) + 3 * sizeof(float2));
    if ((st = dev_alloc(c, &arena, c.maps_bytes)) != DP_OK) return st;
    c.d_maps = arena;
    c.d_rho = reinterpret_cast<unsigned long long *>(arena);
    arena += nb * sizeof(unsigned long long);
    c.d_spec = reinterpret_cast<float2 *>(arena);
    arena += nb * sizeof(float2);
    c.d_sxy = reinterpret_cast<float2 *>(arena);
    arena += nb * sizeof(float2);
    c.d_xi = reinterpret_cast<float2 *>(arena);
    arena += nb * sizeof(float2);
    c.d_t = reinterpret_cast<float *>(arena);
  }
  if ((st = dev_alloc(c, &c.d_sx, nb)) != DP_OK) return st;
  if ((st = dev_alloc(c, &c.d_sy, nb)) != DP_OK) return st;
  if ((st = dev_upload(c, &c.d_tw_x, twiddles(c.mx))) != DP_OK) return st;
  if ((st = dev_upload(c, &c.d_tw_y, twiddles(c.my))) != DP_OK) return st;
  if ((st = dev_upload(c, &c.d_ph_x, phases(c.mx))) != DP_OK) return st;
  if ((st = dev_upload(c, &c.d_ph_y, phases(c.my))) != DP_OK) return st;
  if ((st = dev_upload(c, &c.d_twf_x, twiddles_full(c.mx))) != DP_OK) return st;
  if ((st = dev_upload(c, &c.d_twf_y, twiddles_full(c.my))) != DP_OK) return st;
  if ((st = dev_upload(c, &c.d_tw2_x, twiddles2(c.mx))) != DP_OK) return st;
  if ((st = dev_upload(c, &c.d_tw2_y, twiddles2(c.my))) != DP_OK) return st;
  std::vector<float> kx(c.mx), ky(c.my);
  for (int u = 0; u < c.mx; u++) kx[u] = (float)(M_PI * u / (c.xh - c.xl));   // reading A12
  for (int v = 0; v < c.my; v++) ky[v] = (float)(M_PI * v / (c.yh - c.yl));
  if ((st = dev_upload(c, &c.d_kx, kx)) != DP_OK) return st;
  if ((st = dev_upload(c, &c.d_ky, ky)) != DP_OK) return st;
  {   // shared-memory opt-in: per device, the maxima over its contexts
    std::lock_guard<std::mutex> lock(g_cfg_mutex);
    DeviceConfig &dc = g_cfg[c.device];
    const int m = std::max(c.mx, c.my);
    if (m > dc.max_m || c.mx != c.my) {
      DP_CUDA(dct_configure(std::max(c.mx, dc.max_m), std::max(c.my, dc.max_m)));
      DP_CUDA(fields_configure());
      dc.max_m = std::max(dc.max_m, m);
    }
    if (ntiles > dc.max_tiles || c.tile > dc.max_tile) {
      dc.max_tiles = std::max(dc.max_tiles, ntiles);
      dc.max_tile = std::max(dc.max_tile, c.tile);
      DP_CUDA(density_configure(dc.max_tiles, dc.max_tile));
    }
  }
  c.walk_grid = density_walk_grid(c.tile);
  c.count_grid = density_count_grid(c.tiles_x * c.tiles_y);
  if (c.walk_grid <= 0) return fail(DP_ERR_CUDA, "density walker occupancy query failed");
  {  // DP_WALK_MULT = k: k slices per resident walker slot (finer slices start as SMs free up)
    const char *e = std::getenv("DP_WALK_MULT");
    const int k = e ? std::max(1, std::atoi(e)) : 1;
    c.walk_grid *= k;
  }
  if (c.walk_grid % c.scatter_merge) c.scatter_merge = 1;   // merged scatter slices need an even grid
  if ((st = dev_alloc(c, &c.d_walk_tile, c.walk_grid)) != DP_OK) return st;
  DP_CUDA(cudaMemset(c.d_walk_tile, 0, sizeof(int32_t) * c.walk_grid));
  return DP_OK;
}

void destroy(Ctx *c) {
  if (!c) return;
  DeviceGuard g(c->device);
  if (c->s_wa) cudaStreamSynchronize(c->s_wa);
  if (c->s_den) cudaStreamSynchronize(c->s_den);
  if (c->s_aux) cudaStreamSynchronize(c->s_aux);
  nccl_destroy(*c);
  for (void *p : c->allocations) cudaFree(p);
  if (c->d_hx) cudaFreeHost(c->d_hx);
  if (c->s_h2d) cudaStreamSynchronize(c->s_h2d);
  if (c->s_d2h) cudaStreamSynchronize(c->s_d2h);
  for (int b = 0; b < 2; b++) {
    if (c->ev_in_ready[b]) cudaEventDestroy(c->ev_in_ready[b]);
    if (c->ev_in_free[b]) cudaEventDestroy(c->ev_in_free[b]);
    if (c->ev_out_ready[b]) cudaEventDestroy(c->ev_out_ready[b]);
    if (c->ev_out_free[b]) cudaEventDestroy(c->ev_out_free[b]);
  }
  if (c->s_h2d) cudaStreamDestroy(c->s_h2d);
  if (c->s_d2h) cudaStreamDestroy(c->s_d2h);
  for (int v = 0; v < 2; v++)
    if (c->gexec_v[v]) cudaGraphExecDestroy(c->gexec_v[v]);
  if (c->h_ctl) cudaFreeHost(c->h_ctl);
  if (c->s_cap) cudaStreamDestroy(c->s_cap);
  if (c->s_wa) cudaStreamDestroy(c->s_wa);
  if (c->s_den) cudaStreamDestroy(c->s_den);
  if (c->s_body) cudaStreamDestroy(c->s_body);
  if (c->ev_fork) cudaEventDestroy(c->ev_fork);
  if (c->ev_wa) cudaEventDestroy(c->ev_wa);
  if (c->ev_fields) cudaEventDestroy(c->ev_fields);
  if (c->ev_den) cudaEventDestroy(c->ev_den);
  if (c->ev_done) cudaEventDestroy(c->ev_done);
  if (c->ev_map) cudaEventDestroy(c->ev_map);
  if (c->ev_sched) cudaEventDestroy(c->ev_sched);
  for (cudaEvent_t e : {c->ev_aux_a, c->ev_aux_b, c->ev_join, c->ev_fin})
    if (e) cudaEventDestroy(e);
  if (c->s_aux) cudaStreamDestroy(c->s_aux);
  for (auto &v : c->prof_pairs)
    for (auto &p : v) {
      cudaEventDestroy(p.first);
      cudaEventDestroy(p.second);
    }
  for (cudaEvent_t e : c->prof_pool) cudaEventDestroy(e);
  delete c;
}

dp_status create(const dp_netlist *nl, const dp_grid *grid, int device, int rank, int world, const void *nccl_id,
                 dp_ctx **out) {
  if (!out) return fail(DP_ERR_INVALID_ARG, "out is NULL");
  *out = nullptr;
  dp_status st = validate(nl, grid);
  if (st != DP_OK) return st;
  if (world < 1 || rank < 0 || rank >= world) return fail(DP_ERR_INVALID_ARG, "bad rank / world");
  int ndev = 0;
  cudaError_t e = cudaGetDeviceCount(&ndev);
  if (e != cudaSuccess || ndev == 0) return fail(DP_ERR_CUDA, "no CUDA device available (libdp has no CPU path)");
  if (device < 0 || device >= ndev) return fail(DP_ERR_INVALID_ARG, "device index out of range");
  DeviceGuard guard(device);
  cudaDeviceProp prop;
  DP_CUDA(cudaGetDeviceProperties(&prop, device));
  if (prop.major != 10 || prop.minor != 0)
    return fail(DP_ERR_CUDA, std::string("libdp is built for sm_100a (B200); device is ") + prop.name);
  Ctx *c = new Ctx();
  c->device = device;
  c->rank = rank;
  c->world = world;
  // a distributed context: several ranks, or one rank with a real NCCL communicator (a 1-rank
  // dp_create_dist runs every collective of the distributed path on one GPU)
  c->dist = world > 1 || nccl_id != nullptr;
  c->num_sms = prop.multiProcessorCount;
  c->l2_bytes = prop.l2CacheSize;
  c->num_cells = nl->num_cells;
  c->num_nets_in = nl->num_nets;
  c->num_pins_in = nl->num_pins;
  c->has_weights = nl->net_weight != nullptr;
  c->xl = grid->xl; c->yl = grid->yl; c->xh = grid->xh; c->yh = grid->yh;
  c->mx = grid->bins_x; c->my = grid->bins_y;
  c->log2mx = ilog2(c->mx); c->log2my = ilog2(c->my);
  c->bx = (c->xh - c->xl) / c->mx;
  c->by = (c->yh - c->yl) / c->my;
  c->stretch = grid->stretch;
  const WaPlan wplan = wa_plan(nl, world);
  plan(nl, rank, world, c->cell_begin, c->cell_end, nullptr);
  auto bail = [&](dp_status s) {
    destroy(c);
    return s;
  };
  if ((st = build_wa(*c, nl, wplan)) != DP_OK) return bail(st);
  if ((st = build_density(*c, nl)) != DP_OK) return bail(st);
  {   // net-weighted pin count per cell: the GP preconditioner's P_i (gp.cu, reading A29)
    std::vector<double> acc(nl->num_cells, 0.0);
    for (int32_t e = 0; e < nl->num_nets; e++) {
      const double w = nl->net_weight ? (double)nl->net_weight[e] : 1.0;
      for (int32_t k = nl->net_start[e]; k < nl->net_start[e + 1]; k++)
        acc[nl->pin2cell[nl->net2pin ? nl->net2pin[k] : k]] += w;
    }
    std::vector<float> pins(acc.begin(), acc.end());
    if ((st = dev_upload(*c, &c->d_cell_pins, pins)) != DP_OK) return bail(st);
  }
  {   // field transforms: the warp FFT up to 1024 points (fewer instructions, no block barriers:
      // measured 4599 vs 4041 evals/s at bigblue4 against the CTA FFT), the CTA FFT (fields.cu)
      // beyond, where the warp FFT does not reach; DP_FFT = 0 (warp) / 1 (CTA) / 2 (hybrid: warp
      // rows, CTA column pass) forces one (A/B)
    const char *e = std::getenv("DP_FFT");
    const bool big = std::max(c->mx, c->my) > 1024;
    const int mode = e ? std::atoi(e) : (big ? 1 : 0);
    c->fft_cta = fields_cta_ok(c->log2mx, c->log2my) && (big || mode == 1);
    // the hybrid keeps the warp-FFT T1 / T3: both axes within the warp FFT's 32 .. 1024 points
    c->fft_hybrid = !c->fft_cta && mode == 2 && fields_cta_ok(c->log2mx, c->log2my) && c->log2mx >= 5 &&
                    c->log2my >= 5 && !big;
  }
  // energy partials: one per CTA of the column pass (P2 of the CTA-FFT path; 2-column slabs of
  // the warp-FFT path)
  c->n_en_part = (c->fft_cta || c->fft_hybrid) ? p2_ctas(c->mx, c->my, c->fft_hybrid) : c->my / 2;
  // one "hot" arena for the two per-cell vectors the combine reads: the WA accumulator g2
  // [num_cells] and the force [n_own + 4] (offset by the parity of cell_begin so that even
  // global cells are 16-byte aligned: the combine reads cell pairs as float4).  It is the
  // L2 persisting access-policy window of the evaluation's streams (DP_L2_PERSIST=0: off).
  {
    c->cell_blk = cell_block(c->num_cells, world);
    c->g2_cells = c->dist ? (int64_t)c->cell_blk * world : (int64_t)c->num_cells;
    const size_t g2n = ((size_t)c->g2_cells + 7) & ~(size_t)7;
    const size_t hot_n = g2n + (size_t)c->n_own + 4;
    if ((st = dev_alloc(*c, &c->d_g2, hot_n)) != DP_OK) return bail(st);
    if (cudaMemset(c->d_g2, 0, sizeof(float2) * hot_n) != cudaSuccess) return bail(fail(DP_ERR_CUDA, "memset"));
    c->d_force = c->d_g2 + g2n + (c->cell_begin & 1);
    c->hot_bytes = sizeof(float2) * hot_n;
  }
  // partials: WA [n_wa_part], energy [n_en_part], 1 spare, fast HPWL [n_wa_part] (GP loop)
  if ((st = dev_alloc(*c, &c->d_part, 2 * c->n_wa_part + c->n_en_part + 1)) != DP_OK) return bail(st);
  if (cudaMemset(c->d_part, 0, sizeof(double) * (2 * c->n_wa_part + c->n_en_part + 1)) != cudaSuccess) return bail(fail(DP_ERR_CUDA, "memset"));
  if ((st = dev_alloc(*c, &c->d_limbs, kHpwlLimbs + 1)) != DP_OK) return bail(st);
  if (cudaMemset(c->d_limbs, 0, sizeof(unsigned long long) * (kHpwlLimbs + 1)) != cudaSuccess) return bail(fail(DP_ERR_CUDA, "memset"));
  if ((st = dev_alloc(*c, &c->d_scal, 8)) != DP_OK) return bail(st);
  if ((st = dev_alloc(*c, &c->d_hgx, c->num_cells)) != DP_OK) return bail(st);   // e2e device buffers
  if ((st = dev_alloc(*c, &c->d_hgy, c->num_cells)) != DP_OK) return bail(st);
  if ((st = dev_alloc(*c, &c->d_hy, 2 * (size_t)c->num_cells)) != DP_OK) return bail(st);  // x then y
  c->d_hx = nullptr;
  { const char *e = std::getenv("DP_SERIAL"); c->serial = e && e[0] == '1'; }
  { const char *e = std::getenv("DP_SCHED"); c->sched = e ? std::atoi(e) : 2; }
  int prio_lo = 0, prio_hi = 0;
  cudaDeviceGetStreamPriorityRange(&prio_lo, &prio_hi);
  { const char *e = std::getenv("DP_PRIO"); if (e && e[0] == '0') prio_hi = prio_lo; }   // default: density first
  { const char *e = std::getenv("DP_FUSED_T2"); c->fused_t2 = e && e[0] == '1'; }
  { const char *e = std::getenv("DP_T2B_WARPS"); c->t2b_warps = (e && e[0] == '2') ? 2 : 4; }
  { const char *e = std::getenv("DP_WA_CTAS_PER_SM"); c->wa_ctas_per_sm = e ? std::atoi(e) : 0; }
  { const char *e = std::getenv("DP_L2_HINT"); c->l2_hint = !(e && e[0] == '0'); }
  { const char *e = std::getenv("DP_ROW_TMA"); c->row_tma = !(e && e[0] == '0'); }
  { const char *e = std::getenv("DP_T1_TMA"); c->t1_tma = e && e[0] == '1'; }
  { const char *e = std::getenv("DP_GRAPH"); c->use_graph = !(e && e[0] == '0'); }
  { const char *e = std::getenv("DP_DIRECT"); c->direct = e && e[0] == '1'; }
  { const char *e = std::getenv("DP_PDL"); c->pdl = !(e && e[0] == '0'); }
  { const char *e = std::getenv("DP_WALK_SYNC"); c->walk_sync = e && e[0] == '1'; }
  {
    const char *e = std::getenv("DP_L2_PERSIST");
    c->l2_persist = !(e && e[0] == '0');
    c->l2_persist_maps = e && e[0] == '2';
  }
  if (cudaStreamCreateWithFlags(&c->s_cap, cudaStreamNonBlocking) != cudaSuccess ||
      cudaStreamCreateWithPriority(&c->s_wa, cudaStreamNonBlocking, prio_lo) != cudaSuccess ||
      cudaStreamCreateWithPriority(&c->s_den, cudaStreamNonBlocking, prio_hi) != cudaSuccess ||
      cudaEventCreateWithFlags(&c->ev_map, cudaEventDisableTiming) != cudaSuccess ||
      cudaEventCreateWithFlags(&c->ev_sched, cudaEventDisableTiming) != cudaSuccess ||
      cudaStreamCreateWithPriority(&c->s_aux, cudaStreamNonBlocking, prio_hi) != cudaSuccess ||
      cudaStreamCreateWithPriority(&c->s_body, cudaStreamNonBlocking, prio_hi) != cudaSuccess ||
      cudaEventCreateWithFlags(&c->ev_aux_a, cudaEventDisableTiming) != cudaSuccess ||
      cudaEventCreateWithFlags(&c->ev_aux_b, cudaEventDisableTiming) != cudaSuccess ||
      cudaEventCreateWithFlags(&c->ev_join, cudaEventDisableTiming) != cudaSuccess ||
      cudaEventCreateWithFlags(&c->ev_fin, cudaEventDisableTiming) != cudaSuccess ||
      cudaEventCreateWithFlags(&c->ev_fork, cudaEventDisableTiming) != cudaSuccess ||
      cudaEventCreateWithFlags(&c->ev_wa, cudaEventDisableTiming) != cudaSuccess ||
      cudaEventCreateWithFlags(&c->ev_den, cudaEventDisableTiming) != cudaSuccess ||
      cudaEventCreateWithFlags(&c->ev_done, cudaEventDisableTiming) != cudaSuccess)
    return bail(fail(DP_ERR_CUDA, "stream/event creation failed"));
  // only while the arena is a modest part of L2: at the industrial size (10M cells, a 160 MB
  // arena) a partial window measured 2x slower (365 vs 711 evals/s) than no window
  if (c->l2_persist && (double)c->hot_bytes > 0.4 * (double)c->l2_bytes) c->l2_persist = false;
  if (c->l2_persist && prop.persistingL2CacheMaxSize > 0 && prop.accessPolicyMaxWindowSize > 0) {
    // keep g2 + force (WA reds, gather stores, the combine's reads) and, on the density stream,
    // the transform maps resident in L2 (DP_L2_PERSIST=1: g2 + force only, 2: both)
    const bool maps = c->l2_persist_maps;
    const size_t want = c->hot_bytes + (maps ? c->maps_bytes : 0);
    const size_t setaside = std::min<size_t>((size_t)prop.persistingL2CacheMaxSize, want);
    size_t cur = 0;
    cudaDeviceGetLimit(&cur, cudaLimitPersistingL2CacheSize);
    if (cur < setaside) cudaDeviceSetLimit(cudaLimitPersistingL2CacheSize, setaside);
    const float ratio = (float)std::min(1.0, (double)setaside / (double)want);
    auto window = [&](void *base, size_t bytes) {
      cudaStreamAttrValue v{};
      v.accessPolicyWindow.base_ptr = base;
      v.accessPolicyWindow.num_bytes = std::min<size_t>(bytes, (size_t)prop.accessPolicyMaxWindowSize);
      v.accessPolicyWindow.hitRatio = ratio;
      v.accessPolicyWindow.hitProp = cudaAccessPropertyPersisting;
      v.accessPolicyWindow.missProp = cudaAccessPropertyStreaming;
      return v;
    };
    const cudaStreamAttrValue vh = window(c->d_g2, c->hot_bytes);
    const cudaStreamAttrValue vm = window(c->d_maps, c->maps_bytes);
    for (cudaStream_t s : {c->s_cap, c->s_wa, c->s_aux})
      cudaStreamSetAttribute(s, cudaStreamAttributeAccessPolicyWindow, &vh);
    cudaStreamSetAttribute(c->s_den, cudaStreamAttributeAccessPolicyWindow, maps ? &vm : &vh);
    cudaGetLastError();   // best effort: a refused hint leaves the default policy
  }
  {   // DP_WA_SPLIT = p (0 < p < 100): split WA launch around the field transforms
    const char *e = std::getenv("DP_WA_SPLIT");
    const int p = e ? std::atoi(e) : 0;
    if (p > 0 && p < 100 && !c->dist) {
      if (cudaEventCreateWithFlags(&c->ev_fields, cudaEventDisableTiming) != cudaSuccess)
        return bail(fail(DP_ERR_CUDA, "event creation failed"));
      c->wa_split_chunks = (int)((long long)c->n_chunks * p / 100);
      c->wa_split = true;
    }
  }
  const int wa_k = (c->n_chunks + c->n_big > 0) ? 1 : 0;   // one kernel: big nets, warp nets, chunks
  c->launches_eval = wa_k + density_launches(*c) + ((c->fft_cta || c->fft_hybrid) ? 3 : c->fused_t2 ? 3 : 4) /* P1 P2 P3, T1 P2 T3 or T1 T2a T2b T3 */ + 2 /* combine, finalize */;
  if (c->wa_split && wa_k) c->launches_eval += 1;   // the WA kernel in two launches
  if (c->fuse_combine && !c->dist) c->launches_eval -= 1;   // no combine pass (default configuration)
  c->launches_eval_hpwl = c->launches_eval;
  if (c->dist && nccl_id) {
    if ((st = nccl_init(*c, nccl_id)) != DP_OK) return bail(st);
    // row-sharded Poisson solve for maps above 1024 (replicated below: a redundant <= 4 MB solve
    // is cheaper than its exchanges); DP_SHARD_POISSON = 1 / 0 forces it on / off
    const char *e = std::getenv("DP_SHARD_POISSON");
    const bool want = e ? e[0] == '1' : std::max(c->mx, c->my) > 1024;
    c->shard_poisson = want && fields_shardable(*c, world);
  }
  cudaError_t le = cudaDeviceSynchronize();
  if (le != cudaSuccess) return bail(cuda_fail(le, "dp_create"));
  *out = reinterpret_cast<dp_ctx *>(c);
  return DP_OK;
}

inline Ctx *C(dp_ctx *p) { return reinterpret_cast<Ctx *>(p); }

dp_status check_eval_args(Ctx *c, const void *x, const void *y) {
  if (!c) return fail(DP_ERR_INVALID_ARG, "ctx is NULL");
  if (!x || !y) return fail(DP_ERR_INVALID_ARG, "x / y is NULL");
  return DP_OK;
}

// ---- stage profiling ---------------------------------------------------------------------
cudaEvent_t prof_event(Ctx &c) {
  if (!c.prof_pool.empty()) {
    cudaEvent_t e = c.prof_pool.back();
    c.prof_pool.pop_back();
    return e;
  }
  cudaEvent_t e = nullptr;
  cudaEventCreate(&e);
  return e;
}
struct StageMark {
  Ctx &c;
  int stage;
  cudaStream_t s;
  cudaEvent_t a = nullptr;
  StageMark(Ctx &c_, int st, cudaStream_t s_) : c(c_), stage(st), s(s_) {
    if (c.profiling) {
      a = prof_event(c);
      cudaEventRecord(a, s);
    }
  }
  ~StageMark() {
    if (a) {
      cudaEvent_t b = prof_event(c);
      cudaEventRecord(b, s);
      c.prof_pairs[stage].push_back({a, b});
    }
  }
};

// the density chain on the density stream: map -> (allreduce) -> fields -> gather
// Row-sharded Poisson solve of rank c.rank: the summed map's row block arrives by
// the reduce-scatter; P1 on the rank's rows, all-to-all, P2 on its columns (+ its energy slots),
// all-to-all, P3 on its rows, all-gather of the field rows.
dp_status sharded_fields(Ctx &c, cudaStream_t s) {
  const int G = c.world;
  const size_t nb = (size_t)c.mx * c.my, blk = nb / ((size_t)G * G);   // C R elements per block
  float *s1 = c.d_t, *r1 = c.d_sx;
  float2 *s2 = c.d_sxy, *r2 = c.d_spec;
  DP_CUDA(cudaMemsetAsync(c.d_part + c.n_wa_part, 0, sizeof(double) * c.n_en_part, s));   // other ranks' slots
  launch_fields_shard(c, 1, c.d_rho, true, c.rank, G, s1, r1, s2, r2, s);
  dp_status st = nccl_all_to_all_bytes(c, s1, r1, blk * sizeof(float), s);
  if (st != DP_OK) return st;
  launch_fields_shard(c, 2, c.d_rho, true, c.rank, G, s1, r1, s2, r2, s);
  if ((st = nccl_all_to_all_bytes(c, s2, r2, blk * sizeof(float2), s)) != DP_OK) return st;
  launch_fields_shard(c, 3, c.d_rho, true, c.rank, G, s1, r1, s2, r2, s);
  return nccl_all_gather_bytes(c, c.d_xi, nb / G * sizeof(float2), s);
}

dp_status density_chain_pass(Ctx &c, const float *x, const float *y, bool with_gather = true);

// the density chain; with fence regions (NEXT-4, reading A38) one pass per region, each with its
// own map (from the region's blockage map), Poisson solve (its own energy slots) and gather.
// with_gather = false (fused combine): map and fields only, the caller launches the gather
dp_status density_chain(Ctx &c, const float *x, const float *y, bool with_gather = true) {
  if (c.n_regions == 0) return density_chain_pass(c, x, y, with_gather);
  for (int r = 0; r <= c.n_regions; r++) {
    c.cur_region = r;
    const dp_status st = density_chain_pass(c, x, y);
    c.cur_region = -1;
    if (st != DP_OK) return st;
  }
  return DP_OK;
}

dp_status density_chain_pass(Ctx &c, const float *x, const float *y, bool with_gather) {
  {
    StageMark m(c, DP_STAGE_MAP, c.s_den);
    launch_density_map(c, x, y, c.s_den, c.s_aux);
    if (c.dist && c.nccl_comm) {
      const size_t nb = (size_t)c.mx * c.my;
      dp_status st = c.shard_poisson ? nccl_reduce_scatter_u64(c, c.d_rho, nb / c.world, c.s_den)   // exact
                                     : nccl_allreduce_u64(c, c.d_rho, nb, c.s_den);                 // exact
      if (st != DP_OK) return st;
    }
  }
  DP_CUDA(cudaEventRecord(c.ev_map, c.s_den));
  launch_region_overflow(c, c.s_den);   // GP loop over fence regions: this region's A30 partials
  {
    StageMark m(c, DP_STAGE_FIELDS, c.s_den);
    if (c.shard_poisson) {
      dp_status st = sharded_fields(c, c.s_den);
      if (st != DP_OK) return st;
    } else {
      launch_fields_fixed(c, c.s_den);
    }
  }
  if (c.wa_split) DP_CUDA(cudaEventRecord(c.ev_fields, c.s_den));
  if (!with_gather) return DP_OK;
  StageMark m(c, DP_STAGE_GATHER, c.s_den);
  launch_density_gather(c, x, y, c.s_den, c.s_aux);
  return DP_OK;
}

dp_status finalize(Ctx &c, float lambda, bool with_wl, bool with_energy, bool with_hpwl, double *d_obj, double *d_wl,
                   double *d_energy, double *d_hpwl, cudaStream_t s) {
  if (c.dist && c.nccl_comm) {
    // every WA partial slot is written by exactly one rank (zero elsewhere): the all-reduce is
    // exact and the fixed-order sum below is the same for any number of ranks; the HPWL limbs
    // are integers; the energy is replicated (every rank solves the same Poisson problem)
    dp_status st;
    if (with_wl && (st = nccl_allreduce_f64(c, c.d_part, (size_t)c.n_wa_part, s)) != DP_OK) return st;
    if (with_hpwl && (st = nccl_allreduce_u64(c, c.d_limbs, kHpwlLimbs + 1, s)) != DP_OK) return st;
    // row-sharded solve: each rank holds the energy slots of its column blocks (exact)
    if (with_energy && c.shard_poisson &&
        (st = nccl_allreduce_f64(c, c.d_part + c.n_wa_part, (size_t)c.n_en_part, s)) != DP_OK)
      return st;
  }
  launch_finalize(c, lambda, with_wl, with_energy, with_hpwl, d_obj, d_wl, d_energy, d_hpwl, s);
  return DP_OK;
}

// A context owns scratch (g2, maps, partials): calls issued on different streams are ordered
// by making each call wait for the previous one (skipped while the stream is being captured,
// where the caller's graph already orders the calls).
dp_status call_begin(Ctx &c, cudaStream_t s) {
  cudaStreamCaptureStatus cs = cudaStreamCaptureStatusNone;
  DP_CUDA(cudaStreamIsCapturing(s, &cs));
  if (cs == cudaStreamCaptureStatusNone) DP_CUDA(cudaStreamWaitEvent(s, c.ev_done, 0));
  return DP_OK;
}
dp_status call_end(Ctx &c, cudaStream_t s) {
  cudaStreamCaptureStatus cs = cudaStreamCaptureStatusNone;
  DP_CUDA(cudaStreamIsCapturing(s, &cs));
  if (cs == cudaStreamCaptureStatusNone) DP_CUDA(cudaEventRecord(c.ev_done, s));
  return DP_OK;
}

dp_status eval_body(Ctx &c, const float *x, const float *y, float gamma, float lambda, float *gx, float *gy,
                    double *d_obj, double *d_wl, double *d_energy, double *d_hpwl, cudaStream_t s, bool do_wa,
                    bool do_den);

// Graph path: the whole evaluation (both streams, ~15 launches and their event edges) is
// captured once per argument set into a CUDA graph and replayed with one cudaGraphLaunch;
// a call with different arguments re-captures and updates the executable graph in place
// (cudaGraphExecUpdate).  Skipped while profiling (per-stage events), for distributed
// contexts (collectives) and when the caller is itself capturing.
dp_status eval_graph(Ctx &c, const float *x, const float *y, float gamma, float lambda, float *gx, float *gy,
                     double *d_obj, double *d_wl, double *d_energy, double *d_hpwl, cudaStream_t s, bool do_wa,
                     bool do_den) {
  // the sort kernels are left out of the captured evaluation while the host's (possibly a few
  // evaluations old) view of the stray count is below the re-sort threshold, except on every
  // sort_every-th call (the device decides there); strays are handled exactly either way, so a
  // late view only delays a sort
  const int v = c.sort_variant();
  const bool with_sort = v == 1;
  const GraphKey key{x, y, gx, gy, d_obj, d_wl, d_energy, d_hpwl, gamma, lambda, do_wa, do_den, c.wl_model,
                     c.deterministic, with_sort};
  cudaGraphExec_t &gexec = c.gexec_v[v];
  if (!(gexec && key == c.gkey_v[v])) {
    cudaGraph_t g = nullptr;
    DP_CUDA(cudaStreamBeginCapture(c.s_cap, cudaStreamCaptureModeThreadLocal));
    c.omit_sort = !with_sort;
    dp_status st = eval_body(c, x, y, gamma, lambda, gx, gy, d_obj, d_wl, d_energy, d_hpwl, c.s_cap, do_wa, do_den);
    c.omit_sort = false;
    const cudaError_t ce = cudaStreamEndCapture(c.s_cap, &g);
    if (st != DP_OK) {
      if (g) cudaGraphDestroy(g);
      return st;
    }
    if (ce != cudaSuccess) return cuda_fail(ce, "cudaStreamEndCapture");
    if (gexec) {
      cudaGraphExecUpdateResultInfo info;
      if (cudaGraphExecUpdate(gexec, g, &info) != cudaSuccess) {
        cudaGetLastError();
        cudaGraphExecDestroy(gexec);
        gexec = nullptr;
      }
    }
    if (!gexec) {
      // honour the captured stream priorities (density chain first), as in a stream launch
      const cudaError_t ie = cudaGraphInstantiateWithFlags(&gexec, g, cudaGraphInstantiateFlagUseNodePriority);
      if (ie != cudaSuccess) {
        cudaGraphDestroy(g);
        gexec = nullptr;
        return cuda_fail(ie, "cudaGraphInstantiate");
      }
    }
    cudaGraphDestroy(g);
    c.gkey_v[v] = key;
  }
  dp_status st0 = call_begin(c, s);
  if (st0 != DP_OK) return st0;
  DP_CUDA(cudaGraphLaunch(gexec, s));
  if (with_sort && do_den) c.sorted_once = true;
  return call_end(c, s);
}

dp_status eval_impl(Ctx &c, const float *x, const float *y, float gamma, float lambda, float *gx, float *gy,
                    double *d_obj, double *d_wl, double *d_energy, double *d_hpwl, cudaStream_t s, bool do_wa,
                    bool do_den) {
  cudaStreamCaptureStatus cs = cudaStreamCaptureStatusNone;
  DP_CUDA(cudaStreamIsCapturing(s, &cs));
  if (c.use_graph && !c.profiling && !c.dist && cs == cudaStreamCaptureStatusNone)
    return eval_graph(c, x, y, gamma, lambda, gx, gy, d_obj, d_wl, d_energy, d_hpwl, s, do_wa, do_den);
  dp_status st0 = call_begin(c, s);
  if (st0 != DP_OK) return st0;
  // direct launches (profiling, DP_GRAPH=0, multi-GPU contexts) choose the sort variant per call
  // like the captured graphs (§5.5); a caller's own capture always carries the sort kernels
  const int v = cs == cudaStreamCaptureStatusNone ? c.sort_variant() : 1;
  c.omit_sort = v == 0;
  st0 = eval_body(c, x, y, gamma, lambda, gx, gy, d_obj, d_wl, d_energy, d_hpwl, s, do_wa, do_den);
  c.omit_sort = false;
  if (st0 != DP_OK) return st0;
  if (v == 1 && do_den) c.sorted_once = true;
  return call_end(c, s);
}

dp_status eval_body(Ctx &c, const float *x, const float *y, float gamma, float lambda, float *gx, float *gy,
                    double *d_obj, double *d_wl, double *d_energy, double *d_hpwl, cudaStream_t s, bool do_wa,
                    bool do_den) {
  StageMark whole(c, DP_STAGE_EVAL, s);
  if (c.profiling) c.prof_evals++;
  // direct output (DP_DIRECT=1): both chains add into gx, gy, which are zeroed first; no combine
  const bool direct = c.direct && !c.deterministic && !c.dist && !c.has_fixed &&
                      ((((uintptr_t)gx) | ((uintptr_t)gy)) & 15) == 0;
  struct DirectReset {
    Ctx &c;
    ~DirectReset() { c.direct_gx = c.direct_gy = nullptr; }
  } direct_reset{c};
  c.direct_gx = direct ? gx : nullptr;
  c.direct_gy = direct ? gy : nullptr;
  c.direct_lambda = lambda;
  // fused combine (DP_FUSE_COMBINE=1): the gather waits for the WA stream and writes gx, gy itself
  const bool fused = c.fuse_combine && !direct && do_wa && do_den && !c.deterministic && !c.dist && !c.has_fixed &&
                     c.n_regions == 0 && !c.wa_split;
  struct FusedReset {
    Ctx &c;
    ~FusedReset() { c.fused_gx = c.fused_gy = nullptr; }
  } fused_reset{c};
  const size_t gbytes = sizeof(float) * (size_t)c.num_cells;
  DP_CUDA(cudaEventRecord(c.ev_fork, s));
  if (do_den) {
    DP_CUDA(cudaStreamWaitEvent(c.s_den, c.ev_fork, 0));
    if (direct) {   // before the count: the WA stream starts after the placement (DP_SCHED=2)
      DP_CUDA(cudaMemsetAsync(gx, 0, gbytes, c.s_den));
      DP_CUDA(cudaMemsetAsync(gy, 0, gbytes, c.s_den));
    }
    dp_status st = density_chain(c, x, y, !fused);
    if (st != DP_OK) return st;
    if (!fused) DP_CUDA(cudaEventRecord(c.ev_den, c.s_den));
  }
  if (do_wa) {
    DP_CUDA(cudaStreamWaitEvent(
        c.s_wa,
        !do_den ? c.ev_fork
        : c.serial ? c.ev_den
        : c.sched == 1 ? c.ev_map
        : (c.sched == 2 || c.sched == 3) && c.n_own > 0 ? c.ev_sched
        : c.sched >= 2 ? c.ev_map
                       : c.ev_fork,
        0));
    {
      StageMark m(c, DP_STAGE_WA, c.s_wa);
      // clear the own-cell range of the WA gradient accumulator (read, not reset, by combine)
      if (direct) {
        if (!do_den) {
          DP_CUDA(cudaMemsetAsync(gx, 0, gbytes, c.s_wa));
          DP_CUDA(cudaMemsetAsync(gy, 0, gbytes, c.s_wa));
        } else if (c.sched < 2 || c.serial) {
          return fail(DP_ERR_UNSUPPORTED, "DP_DIRECT needs DP_SCHED >= 2");
        }
      } else if (c.deterministic)
        DP_CUDA(cudaMemsetAsync(c.d_g2i, 0, 2 * sizeof(long long) * (size_t)c.g2_cells, c.s_wa));
      else
        DP_CUDA(cudaMemsetAsync(c.d_g2, 0, sizeof(float2) * (size_t)c.g2_cells, c.s_wa));
      if (c.wa_split && do_den && !c.serial && c.n_regions == 0) {   // around the transforms
        launch_wa(c, x, y, gamma, false, d_hpwl != nullptr, c.s_wa, 1);
        DP_CUDA(cudaStreamWaitEvent(c.s_wa, c.ev_fields, 0));
        launch_wa(c, x, y, gamma, false, d_hpwl != nullptr, c.s_wa, 2);
      } else {
        launch_wa(c, x, y, gamma, false, d_hpwl != nullptr, c.s_wa);
      }
      if (c.dist && c.nccl_comm) {   // nets are partitioned: sum the WA gradient into each cell block
        const size_t n = 2 * (size_t)c.cell_blk;
        dp_status st = c.deterministic ? nccl_reduce_scatter_i64(c, c.d_g2i, n, c.s_wa)
                                       : nccl_reduce_scatter_f32(c, reinterpret_cast<float *>(c.d_g2), n, c.s_wa);
        if (st != DP_OK) return st;
      }
    }
    DP_CUDA(cudaEventRecord(c.ev_wa, c.s_wa));
  }
  if (fused) {   // the gather after the fields and the complete WA accumulator
    DP_CUDA(cudaStreamWaitEvent(c.s_den, c.ev_wa, 0));
    c.fused_gx = gx;
    c.fused_gy = gy;
    {
      StageMark m(c, DP_STAGE_GATHER, c.s_den);
      launch_density_gather(c, x, y, c.s_den, c.s_aux);
    }
    c.fused_gx = c.fused_gy = nullptr;
    DP_CUDA(cudaEventRecord(c.ev_den, c.s_den));
  }
  if (do_wa) DP_CUDA(cudaStreamWaitEvent(s, c.ev_wa, 0));
  if (do_den) DP_CUDA(cudaStreamWaitEvent(s, c.ev_den, 0));
  {
    StageMark m(c, DP_STAGE_COMBINE, s);
    if (c.dist) {   // the finalize carries collectives: keep it on the caller stream
      launch_combine(c, do_den ? lambda : 0.f, gx, gy, do_wa, do_den, s);
      dp_status st = finalize(c, lambda, do_wa, do_den, do_wa && d_hpwl != nullptr, d_obj, d_wl, d_energy, d_hpwl, s);
      if (st != DP_OK) return st;
    } else {        // scalars (aux stream) beside the gradient combine (caller stream)
      DP_CUDA(cudaEventRecord(c.ev_join, s));
      DP_CUDA(cudaStreamWaitEvent(c.s_aux, c.ev_join, 0));
      dp_status st =
          finalize(c, lambda, do_wa, do_den, do_wa && d_hpwl != nullptr, d_obj, d_wl, d_energy, d_hpwl, c.s_aux);
      if (st != DP_OK) return st;
      DP_CUDA(cudaEventRecord(c.ev_fin, c.s_aux));
      if (!direct && !fused) launch_combine(c, do_den ? lambda : 0.f, gx, gy, do_wa, do_den, s);
      DP_CUDA(cudaStreamWaitEvent(s, c.ev_fin, 0));
    }
  }
  DP_CUDA(cudaGetLastError());
  return DP_OK;
}

}  // namespace

// entry points for gp.cu (the GP loop captures one iteration around the evaluation)
dp_status eval_body_ext(Ctx &c, const float *x, const float *y, float gamma, float lambda, float *gx, float *gy,
                        double *d_obj, double *d_wl, double *d_energy, double *d_hpwl, cudaStream_t s, bool do_wa,
                        bool do_den) {
  return eval_body(c, x, y, gamma, lambda, gx, gy, d_obj, d_wl, d_energy, d_hpwl, s, do_wa, do_den);
}
dp_status request_sort(Ctx &c, cudaStream_t s) {
  c.sorted_once = false;   // the next captured evaluation carries the sort kernels
  DP_CUDA(cudaMemsetAsync(c.d_sortctl, 0x01, sizeof(int32_t), s));   // word 0 != 0: sort requested
  return DP_OK;
}

dp_status ctx_call_begin(Ctx &c, cudaStream_t s) { return call_begin(c, s); }
dp_status ctx_call_end(Ctx &c, cudaStream_t s) { return call_end(c, s); }
}  // namespace dp

using dp::C;
using dp::Ctx;
using dp::fail;

extern "C" {

const char *dp_last_error(void) { return dp::g_err.c_str(); }

int32_t dp_version(void) { return 100; }

dp_status dp_create(const dp_netlist *nl, const dp_grid *grid, int device, dp_ctx **out) {
  try {
    return dp::create(nl, grid, device, 0, 1, nullptr, out);
  } catch (const std::bad_alloc &) {
    return fail(DP_ERR_OUT_OF_MEMORY, "host allocation failed in dp_create");
  } catch (...) {
    return fail(DP_ERR_INVALID_ARG, "unexpected exception in dp_create");
  }
}

dp_status dp_create_dist(const dp_netlist *nl, const dp_grid *grid, int device, int rank, int world,
                         const void *nccl_unique_id, dp_ctx **out) {
  try {
    return dp::create(nl, grid, device, rank, world, nccl_unique_id, out);
  } catch (const std::bad_alloc &) {
    return fail(DP_ERR_OUT_OF_MEMORY, "host allocation failed in dp_create_dist");
  } catch (...) {
    return fail(DP_ERR_INVALID_ARG, "unexpected exception in dp_create_dist");
  }
}

dp_status dp_nccl_unique_id(void *out128) {
  if (!out128) return fail(DP_ERR_INVALID_ARG, "out128 is NULL");
  return dp::nccl_get_unique_id(out128);
}

dp_status dp_partition_plan(const dp_netlist *nl, int rank, int world, int32_t *cell_begin, int32_t *cell_end,
                            uint8_t *net_mask) {
  try {
    if (!cell_begin || !cell_end) return fail(DP_ERR_INVALID_ARG, "cell_begin / cell_end NULL");
    if (world < 1 || rank < 0 || rank >= world) return fail(DP_ERR_INVALID_ARG, "bad rank / world");
    if (!nl || !nl->net_start || nl->num_cells < 1 || (nl->num_pins > 0 && !nl->pin2cell))
      return fail(DP_ERR_INVALID_ARG, "netlist incomplete");
    std::vector<uint8_t> mask;
    dp::plan(nl, rank, world, *cell_begin, *cell_end, net_mask ? &mask : nullptr);
    if (net_mask && !mask.empty()) std::memcpy(net_mask, mask.data(), mask.size());
    return DP_OK;
  } catch (...) {
    return fail(DP_ERR_OUT_OF_MEMORY, "exception in dp_partition_plan");
  }
}

dp_status dp_destroy(dp_ctx *ctx) {
  dp::destroy(C(ctx));
  return DP_OK;
}

dp_status dp_eval(dp_ctx *ctx, const float *x, const float *y, float gamma, float lambda, float *gx, float *gy,
                  double *d_obj, double *d_wl, double *d_energy, double *d_hpwl, dp_stream_t stream) {
  Ctx *c = C(ctx);
  dp_status st = dp::check_eval_args(c, x, y);
  if (st != DP_OK) return st;
  if (!gx || !gy) return fail(DP_ERR_INVALID_ARG, "gx / gy is NULL");
  if (!(gamma > 0.f) || !std::isfinite(gamma)) return fail(DP_ERR_INVALID_ARG, "gamma must be finite and > 0");
  if (!(lambda >= 0.f) || !std::isfinite(lambda)) return fail(DP_ERR_INVALID_ARG, "lambda must be finite and >= 0");
  dp::DeviceGuard g(c->device);
  return dp::eval_impl(*c, x, y, gamma, lambda, gx, gy, d_obj, d_wl, d_energy, d_hpwl, (cudaStream_t)stream, true,
                       true);
}

dp_status dp_wl_grad(dp_ctx *ctx, const float *x, const float *y, float gamma, float *gx, float *gy, double *d_wl,
                     dp_stream_t stream) {
  Ctx *c = C(ctx);
  dp_status st = dp::check_eval_args(c, x, y);
  if (st != DP_OK) return st;
  if (!gx || !gy) return fail(DP_ERR_INVALID_ARG, "gx / gy is NULL");
  if (!(gamma > 0.f) || !std::isfinite(gamma)) return fail(DP_ERR_INVALID_ARG, "gamma must be finite and > 0");
  dp::DeviceGuard g(c->device);
  return dp::eval_impl(*c, x, y, gamma, 0.f, gx, gy, nullptr, d_wl, nullptr, nullptr, (cudaStream_t)stream, true,
                       false);
}

dp_status dp_set_wl_model(dp_ctx *ctx, int32_t model) {
  if (ctx) C(ctx)->config_gen++;
  Ctx *c = C(ctx);
  if (!c) return fail(DP_ERR_INVALID_ARG, "ctx is NULL");
  if (model != DP_WL_WA && model != DP_WL_LSE) return fail(DP_ERR_INVALID_ARG, "unknown wirelength model");
  c->wl_model = model;
  return DP_OK;
}

dp_status dp_set_deterministic(dp_ctx *ctx, int32_t on) {
  if (ctx) C(ctx)->config_gen++;
  Ctx *c = C(ctx);
  if (!c) return fail(DP_ERR_INVALID_ARG, "ctx is NULL");
  if (on && !c->d_g2i) {
    dp::DeviceGuard g(c->device);
    dp_status st = dp::dev_alloc(*c, &c->d_g2i, 2 * (size_t)c->g2_cells);
    if (st != DP_OK) return st;
  }
  c->deterministic = on != 0;
  return DP_OK;
}

dp_status dp_set_fixed(dp_ctx *ctx, const uint8_t *h_fixed, const float *x, const float *y, dp_stream_t stream) {
  if (ctx) C(ctx)->config_gen++;
  Ctx *c = C(ctx);
  if (!c) return fail(DP_ERR_INVALID_ARG, "ctx is NULL");
  if (c->dist) return fail(DP_ERR_UNSUPPORTED, "fixed cells are supported on single-GPU contexts");
  if (h_fixed && (!x || !y)) return fail(DP_ERR_INVALID_ARG, "x / y is NULL");
  if (h_fixed && c->n_regions > 0) return fail(DP_ERR_UNSUPPORTED, "fixed cells with fence regions");
  dp::DeviceGuard g(c->device);
  cudaStream_t s = (cudaStream_t)stream;
  dp_status st = dp::call_begin(*c, s);
  if (st != DP_OK) return st;
  DP_CUDA(cudaStreamSynchronize(s));   // the captured evaluation changes (map initialisation, masks): re-capture
  for (int v = 0; v < 2; v++)
    if (c->gexec_v[v]) {
      cudaGraphExecDestroy(c->gexec_v[v]);
      c->gexec_v[v] = nullptr;
      c->gkey_v[v] = dp::GraphKey{};
    }
  if (!h_fixed) {
    c->has_fixed = false;
    if ((st = dp::request_sort(*c, s)) != DP_OK) return st;   // the list lacks the formerly fixed cells
    return dp::call_end(*c, s);
  }
  const int n = c->n_own;
  std::vector<uint8_t> m(((size_t)n + 3) & ~(size_t)3, 0);
  for (int i = 0; i < n; i++) m[i] = h_fixed[c->cell_begin + i] ? 1 : 0;
  std::vector<int32_t> large(c->n_large), mov, fix;
  if (c->n_large)
    DP_CUDA(cudaMemcpy(large.data(), c->d_large, sizeof(int32_t) * c->n_large, cudaMemcpyDeviceToHost));
  for (int32_t i : large) (m[i] ? fix : mov).push_back(i);
  {   // fixed small cells need the mask in the sort; fixed large cells only change the lists
    size_t nfix = 0;
    for (int i = 0; i < n; i++) nfix += m[i];
    c->fixed_small = nfix > fix.size();
  }
  if (!c->d_fixed) {
    if ((st = dp::dev_alloc(*c, &c->d_fixed, m.size())) != DP_OK) return st;
    if ((st = dp::dev_alloc(*c, &c->d_rho_fixed, (size_t)c->mx * c->my)) != DP_OK) return st;
    if ((st = dp::dev_alloc(*c, &c->d_large_mov, (size_t)std::max(1, c->n_large))) != DP_OK) return st;
    if ((st = dp::dev_alloc(*c, &c->d_large_fix, (size_t)std::max(1, c->n_large))) != DP_OK) return st;
  }
  DP_CUDA(cudaStreamSynchronize(s));
  DP_CUDA(cudaMemcpy(c->d_fixed, m.data(), m.size(), cudaMemcpyHostToDevice));
  if (!mov.empty()) DP_CUDA(cudaMemcpy(c->d_large_mov, mov.data(), sizeof(int32_t) * mov.size(), cudaMemcpyHostToDevice));
  if (!fix.empty()) DP_CUDA(cudaMemcpy(c->d_large_fix, fix.data(), sizeof(int32_t) * fix.size(), cudaMemcpyHostToDevice));
  c->n_large_mov = (int32_t)mov.size();
  c->n_large_fix = (int32_t)fix.size();
  c->has_fixed = true;
  // the fixed-charge map: the density map of the fixed cells alone (exact int64), kept
  dp::launch_density_map(*c, x, y, s, nullptr, 1);
  DP_CUDA(cudaMemcpyAsync(c->d_rho_fixed, c->d_rho, sizeof(unsigned long long) * (size_t)c->mx * c->my,
                          cudaMemcpyDeviceToDevice, s));
  if ((st = dp::request_sort(*c, s)) != DP_OK) return st;   // the list now holds the fixed cells
  DP_CUDA(cudaGetLastError());
  return dp::call_end(*c, s);
}

dp_status dp_set_regions(dp_ctx *ctx, int32_t n_regions, const double *h_boxes, const int32_t *h_cell_region) {
  Ctx *c = C(ctx);
  if (!c) return fail(DP_ERR_INVALID_ARG, "ctx is NULL");
  if (c->dist) return fail(DP_ERR_UNSUPPORTED, "fence regions are supported on single-GPU contexts");
  if (n_regions < 0 || n_regions > 254) return fail(DP_ERR_INVALID_ARG, "n_regions must be in [0, 254]");
  if (n_regions > 0 && (!h_boxes || !h_cell_region)) return fail(DP_ERR_INVALID_ARG, "boxes / cell_region is NULL");
  if (n_regions > 0 && c->has_fixed) return fail(DP_ERR_UNSUPPORTED, "fence regions with fixed cells");
  for (int32_t r = 0; r < n_regions; r++) {
    const double *b = h_boxes + 4 * r;
    if (!(std::isfinite(b[0]) && std::isfinite(b[1]) && std::isfinite(b[2]) && std::isfinite(b[3])) ||
        !(b[2] > b[0]) || !(b[3] > b[1]))
      return fail(DP_ERR_INVALID_ARG, "fence box " + std::to_string(r) + " is degenerate or non-finite");
  }
  for (int32_t i = 0; n_regions > 0 && i < c->num_cells; i++)
    if (h_cell_region[i] < 0 || h_cell_region[i] > n_regions)
      return fail(DP_ERR_INVALID_ARG, "cell_region out of [0, n_regions]");
  dp::DeviceGuard g(c->device);
  DP_CUDA(cudaDeviceSynchronize());
  c->config_gen++;
  for (int v = 0; v < 2; v++)   // the captured evaluation changes: re-capture
    if (c->gexec_v[v]) {
      cudaGraphExecDestroy(c->gexec_v[v]);
      c->gexec_v[v] = nullptr;
      c->gkey_v[v] = dp::GraphKey{};
    }
  c->n_regions = 0;
  {   // the list was built for one region pass: the next evaluation sorts
    dp_status rs = dp::request_sort(*c, nullptr);
    if (rs != DP_OK) return rs;
    DP_CUDA(cudaDeviceSynchronize());
  }
  if (n_regions == 0) return DP_OK;
  const int R = n_regions, n = c->n_own;
  const size_t nb = (size_t)c->mx * c->my;
  std::vector<uint8_t> reg(((size_t)n + 3) & ~(size_t)3, 0);
  for (int i = 0; i < n; i++) reg[i] = (uint8_t)h_cell_region[c->cell_begin + i];
  // blockage maps (A38): per bin the fraction outside region r, at density 1, in 2^-29 units
  std::vector<unsigned long long> blk((size_t)(R + 1) * nb, 0ull);
  auto cover = [&](const double *b, int i, int j) {
    const double x0 = c->xl + i * c->bx, y0 = c->yl + j * c->by;
    const double ox = std::max(0.0, std::min(x0 + c->bx, b[2]) - std::max(x0, b[0])) / c->bx;
    const double oy = std::max(0.0, std::min(y0 + c->by, b[3]) - std::max(y0, b[1])) / c->by;
    return ox * oy;
  };
  const double unit = std::ldexp(1.0, dp::kRhoScaleLog2);
  for (int i = 0; i < c->mx; i++)
    for (int j = 0; j < c->my; j++) {
      double in_fences = 0.0;
      for (int r = 1; r <= R; r++) {
        const double f = cover(h_boxes + 4 * (r - 1), i, j);
        in_fences += f;
        blk[(size_t)r * nb + (size_t)i * c->my + j] = (unsigned long long)std::llround((1.0 - f) * unit);
      }
      blk[(size_t)i * c->my + j] = (unsigned long long)std::llround(std::min(1.0, in_fences) * unit);
    }
  std::vector<int32_t> large(c->n_large);
  if (c->n_large) DP_CUDA(cudaMemcpy(large.data(), c->d_large, sizeof(int32_t) * c->n_large, cudaMemcpyDeviceToHost));
  std::vector<int32_t> lreg;
  c->large_reg_off.assign(R + 2, 0);
  for (int r = 0; r <= R; r++) {
    c->large_reg_off[r] = (int32_t)lreg.size();
    for (int32_t i : large)
      if (reg[i] == r) lreg.push_back(i);
  }
  c->large_reg_off[R + 1] = (int32_t)lreg.size();
  if (lreg.empty()) lreg.push_back(0);
  dp_status st;
  if ((st = dp::dev_upload(*c, &c->d_region, reg)) != DP_OK) return st;
  if ((st = dp::dev_upload(*c, &c->d_rho_block, blk)) != DP_OK) return st;
  if ((st = dp::dev_upload(*c, &c->d_large_reg, lreg)) != DP_OK) return st;
  // partial sums with one energy slot range per region
  const size_t np = 2 * (size_t)c->n_wa_part + (size_t)c->n_en_part * (R + 1) + 1;
  double *part = nullptr;
  if ((st = dp::dev_alloc(*c, &part, np)) != DP_OK) return st;
  DP_CUDA(cudaMemset(part, 0, sizeof(double) * np));
  c->d_part = part;
  c->n_regions = R;
  return DP_OK;
}

dp_status dp_density_grad(dp_ctx *ctx, const float *x, const float *y, float *gx, float *gy, double *d_energy,
                          dp_stream_t stream) {
  Ctx *c = C(ctx);
  dp_status st = dp::check_eval_args(c, x, y);
  if (st != DP_OK) return st;
  if (!gx || !gy) return fail(DP_ERR_INVALID_ARG, "gx / gy is NULL");
  dp::DeviceGuard g(c->device);
  return dp::eval_impl(*c, x, y, 1.f, 1.f, gx, gy, nullptr, nullptr, d_energy, nullptr, (cudaStream_t)stream, false,
                       true);
}

dp_status dp_hpwl(dp_ctx *ctx, const float *x, const float *y, double *d_hpwl, dp_stream_t stream) {
  Ctx *c = C(ctx);
  dp_status st = dp::check_eval_args(c, x, y);
  if (st != DP_OK) return st;
  if (!d_hpwl) return fail(DP_ERR_INVALID_ARG, "d_hpwl is NULL");
  dp::DeviceGuard g(c->device);
  cudaStream_t s = (cudaStream_t)stream;
  if ((st = dp::call_begin(*c, s)) != DP_OK) return st;
  dp::launch_wa(*c, x, y, 1.f, true, true, s);
  st = dp::finalize(*c, 0.f, false, false, true, nullptr, nullptr, nullptr, d_hpwl, s);
  if (st != DP_OK) return st;
  DP_CUDA(cudaGetLastError());
  return dp::call_end(*c, s);
}

dp_status dp_eval_host(dp_ctx *ctx, const float *hx, const float *hy, float gamma, float lambda, float *hgx,
                       float *hgy, double *h_scalars, int with_hpwl, dp_stream_t stream) {
  Ctx *c = C(ctx);
  if (!c) return fail(DP_ERR_INVALID_ARG, "ctx is NULL");
  if (!hx || !hy || !hgx || !hgy) return fail(DP_ERR_INVALID_ARG, "host buffer is NULL");
  if (!(gamma > 0.f) || !std::isfinite(gamma)) return fail(DP_ERR_INVALID_ARG, "gamma must be finite and > 0");
  if (!(lambda >= 0.f) || !std::isfinite(lambda)) return fail(DP_ERR_INVALID_ARG, "lambda must be finite and >= 0");
  dp::DeviceGuard g(c->device);
  cudaStream_t s = (cudaStream_t)stream;
  const size_t n = (size_t)c->num_cells;
  float *dx = c->d_hy, *dy = c->d_hy + n;
  DP_CUDA(cudaMemcpyAsync(dx, hx, n * sizeof(float), cudaMemcpyHostToDevice, s));
  DP_CUDA(cudaMemcpyAsync(dy, hy, n * sizeof(float), cudaMemcpyHostToDevice, s));
  double *sc = c->d_scal + 4;
  dp_status st = dp::eval_impl(*c, dx, dy, gamma, lambda, c->d_hgx, c->d_hgy, sc + 0, sc + 1, sc + 2,
                               with_hpwl ? sc + 3 : nullptr, s, true, true);
  if (st != DP_OK) return st;
  const size_t off = (size_t)c->cell_begin, cnt = (size_t)(c->cell_end - c->cell_begin);
  DP_CUDA(cudaMemcpyAsync(hgx + off, c->d_hgx + off, cnt * sizeof(float), cudaMemcpyDeviceToHost, s));
  DP_CUDA(cudaMemcpyAsync(hgy + off, c->d_hgy + off, cnt * sizeof(float), cudaMemcpyDeviceToHost, s));
  double tmp[4];
  DP_CUDA(cudaMemcpyAsync(tmp, sc, 4 * sizeof(double), cudaMemcpyDeviceToHost, s));
  DP_CUDA(cudaStreamSynchronize(s));
  if (h_scalars) {
    h_scalars[0] = tmp[0];
    h_scalars[1] = tmp[1];
    h_scalars[2] = tmp[2];
    h_scalars[3] = with_hpwl ? tmp[3] : std::nan("");
  }
  return DP_OK;
}

dp_status dp_eval_host_async(dp_ctx *ctx, const float *hx, const float *hy, float gamma, float lambda, float *hgx,
                             float *hgy, double *h_scalars, int with_hpwl, dp_stream_t stream) {
  Ctx *c = C(ctx);
  if (!c) return fail(DP_ERR_INVALID_ARG, "ctx is NULL");
  if (!hx || !hy || !hgx || !hgy) return fail(DP_ERR_INVALID_ARG, "host buffer is NULL");
  if (!(gamma > 0.f) || !std::isfinite(gamma)) return fail(DP_ERR_INVALID_ARG, "gamma must be finite and > 0");
  if (!(lambda >= 0.f) || !std::isfinite(lambda)) return fail(DP_ERR_INVALID_ARG, "lambda must be finite and >= 0");
  dp::DeviceGuard g(c->device);
  cudaStream_t s = (cudaStream_t)stream;
  const size_t n = (size_t)c->num_cells;
  if (!c->s_h2d) {   // first use: slots, copy streams, events
    dp_status st;
    for (int b = 0; b < 2; b++) {
      if ((st = dp::dev_alloc(*c, &c->d_in2[b], 2 * n)) != DP_OK) return st;
      if ((st = dp::dev_alloc(*c, &c->d_out2[b], 2 * n)) != DP_OK) return st;
      if ((st = dp::dev_alloc(*c, &c->d_osc2[b], 4)) != DP_OK) return st;
      DP_CUDA(cudaEventCreateWithFlags(&c->ev_in_ready[b], cudaEventDisableTiming));
      DP_CUDA(cudaEventCreateWithFlags(&c->ev_in_free[b], cudaEventDisableTiming));
      DP_CUDA(cudaEventCreateWithFlags(&c->ev_out_ready[b], cudaEventDisableTiming));
      DP_CUDA(cudaEventCreateWithFlags(&c->ev_out_free[b], cudaEventDisableTiming));
      DP_CUDA(cudaEventRecord(c->ev_in_free[b], s));
      DP_CUDA(cudaEventRecord(c->ev_out_free[b], s));
    }
    DP_CUDA(cudaStreamCreateWithFlags(&c->s_h2d, cudaStreamNonBlocking));
    DP_CUDA(cudaStreamCreateWithFlags(&c->s_d2h, cudaStreamNonBlocking));
  }
  const int b = (int)(c->async_k++ & 1);
  // H2D of this call's positions into slot b once the call two back has moved them on
  DP_CUDA(cudaStreamWaitEvent(c->s_h2d, c->ev_in_free[b], 0));
  DP_CUDA(cudaMemcpyAsync(c->d_in2[b], hx, n * sizeof(float), cudaMemcpyHostToDevice, c->s_h2d));
  DP_CUDA(cudaMemcpyAsync(c->d_in2[b] + n, hy, n * sizeof(float), cudaMemcpyHostToDevice, c->s_h2d));
  DP_CUDA(cudaEventRecord(c->ev_in_ready[b], c->s_h2d));
  // the evaluation reads the fixed input buffers (one captured graph for every call)
  DP_CUDA(cudaStreamWaitEvent(s, c->ev_in_ready[b], 0));
  DP_CUDA(cudaMemcpyAsync(c->d_hy, c->d_in2[b], 2 * n * sizeof(float), cudaMemcpyDeviceToDevice, s));
  DP_CUDA(cudaEventRecord(c->ev_in_free[b], s));
  double *sc = c->d_scal + 4;
  dp_status st = dp::eval_impl(*c, c->d_hy, c->d_hy + n, gamma, lambda, c->d_hgx, c->d_hgy, sc + 0, sc + 1, sc + 2,
                               with_hpwl ? sc + 3 : nullptr, s, true, true);
  if (st != DP_OK) return st;
  // results into output slot b once its previous D2H is done, then D2H on the copy stream
  const size_t off = (size_t)c->cell_begin, cnt = (size_t)(c->cell_end - c->cell_begin);
  DP_CUDA(cudaStreamWaitEvent(s, c->ev_out_free[b], 0));
  DP_CUDA(cudaMemcpyAsync(c->d_out2[b] + off, c->d_hgx + off, cnt * sizeof(float), cudaMemcpyDeviceToDevice, s));
  DP_CUDA(cudaMemcpyAsync(c->d_out2[b] + n + off, c->d_hgy + off, cnt * sizeof(float), cudaMemcpyDeviceToDevice, s));
  DP_CUDA(cudaMemcpyAsync(c->d_osc2[b], sc, 4 * sizeof(double), cudaMemcpyDeviceToDevice, s));
  DP_CUDA(cudaEventRecord(c->ev_out_ready[b], s));
  DP_CUDA(cudaStreamWaitEvent(c->s_d2h, c->ev_out_ready[b], 0));
  DP_CUDA(cudaMemcpyAsync(hgx + off, c->d_out2[b] + off, cnt * sizeof(float), cudaMemcpyDeviceToHost, c->s_d2h));
  DP_CUDA(cudaMemcpyAsync(hgy + off, c->d_out2[b] + n + off, cnt * sizeof(float), cudaMemcpyDeviceToHost, c->s_d2h));
  if (h_scalars) DP_CUDA(cudaMemcpyAsync(h_scalars, c->d_osc2[b], 4 * sizeof(double), cudaMemcpyDeviceToHost, c->s_d2h));
  DP_CUDA(cudaEventRecord(c->ev_out_free[b], c->s_d2h));
  return DP_OK;
}

dp_status dp_eval_host_wait(dp_ctx *ctx) {
  Ctx *c = C(ctx);
  if (!c) return fail(DP_ERR_INVALID_ARG, "ctx is NULL");
  dp::DeviceGuard g(c->device);
  if (c->s_h2d) DP_CUDA(cudaStreamSynchronize(c->s_h2d));
  if (c->s_d2h) DP_CUDA(cudaStreamSynchronize(c->s_d2h));
  return DP_OK;
}

dp_status dp_get_info(const dp_ctx *ctx, dp_info *info) {
  const Ctx *c = reinterpret_cast<const Ctx *>(ctx);
  if (!c || !info) return fail(DP_ERR_INVALID_ARG, "NULL argument");
  info->num_cells = c->num_cells;
  info->num_nets = c->n_wa_nets + c->n_big;
  info->num_pins = c->n_wa_pins;
  info->cell_begin = c->cell_begin;
  info->cell_end = c->cell_end;
  info->bins_x = c->mx;
  info->bins_y = c->my;
  info->rank = c->rank;
  info->world = c->world;
  info->launches_eval = c->launches_eval;
  info->launches_eval_hpwl = c->launches_eval_hpwl;
  info->device_bytes = c->device_bytes;
  info->num_sms = c->num_sms;
  info->l2_bytes = c->l2_bytes;
  return DP_OK;
}

dp_status dp_profile_enable(dp_ctx *ctx, int on) {
  Ctx *c = C(ctx);
  if (!c) return fail(DP_ERR_INVALID_ARG, "ctx is NULL");
  c->profiling = on != 0;
  return DP_OK;
}

dp_status dp_profile_read(dp_ctx *ctx, double *ms, int64_t *count) {
  Ctx *c = C(ctx);
  if (!c || !ms) return fail(DP_ERR_INVALID_ARG, "NULL argument");
  dp::DeviceGuard g(c->device);
  for (int st = 0; st < DP_NSTAGES; st++) {
    double tot = 0.0;
    for (auto &p : c->prof_pairs[st]) {
      DP_CUDA(cudaEventSynchronize(p.second));
      float t = 0.f;
      DP_CUDA(cudaEventElapsedTime(&t, p.first, p.second));
      tot += t;
      c->prof_pool.push_back(p.first);
      c->prof_pool.push_back(p.second);
    }
    c->prof_pairs[st].clear();
    ms[st] = tot;
  }
  if (count) *count = c->prof_evals;
  c->prof_evals = 0;
  return DP_OK;
}

dp_status dp_debug_sort_stats(dp_ctx *ctx, int32_t *out) {
  Ctx *c = C(ctx);
  if (!c || !out) return fail(DP_ERR_INVALID_ARG, "NULL argument");
  dp::DeviceGuard g(c->device);
  DP_CUDA(cudaEventSynchronize(c->ev_done));
  DP_CUDA(cudaDeviceSynchronize());
  DP_CUDA(cudaMemcpy(out, c->d_sortctl, 4 * sizeof(int32_t), cudaMemcpyDeviceToHost));
  return DP_OK;
}

dp_status dp_debug_density_map(dp_ctx *ctx, const float *x, const float *y, float *rho, dp_stream_t stream) {
  Ctx *c = C(ctx);
  dp_status st = dp::check_eval_args(c, x, y);
  if (st != DP_OK) return st;
  if (!rho) return fail(DP_ERR_INVALID_ARG, "rho is NULL");
  dp::DeviceGuard g(c->device);
  cudaStream_t s = (cudaStream_t)stream;
  dp::launch_density_map(*c, x, y, s);
  dp::launch_rho_to_float(*c, rho, s);
  DP_CUDA(cudaGetLastError());
  return DP_OK;
}

dp_status dp_debug_fields(dp_ctx *ctx, const float *rho, float *psi, float *xi_x, float *xi_y, double *d_energy,
                          dp_stream_t stream) {
  Ctx *c = C(ctx);
  if (!c || !rho) return fail(DP_ERR_INVALID_ARG, "NULL argument");
  dp::DeviceGuard g(c->device);
  cudaStream_t s = (cudaStream_t)stream;
  dp::launch_fields(*c, rho, s);
  if (xi_x || xi_y) dp::launch_split_fields(*c, xi_x, xi_y, s);
  if (d_energy) dp::launch_finalize(*c, 1.f, false, true, false, nullptr, nullptr, d_energy, nullptr, s);
  if (psi) dp::launch_psi(*c, rho, psi, s);
  DP_CUDA(cudaGetLastError());
  return DP_OK;
}

dp_status dp_debug_sharded_fields(dp_ctx *ctx, int32_t world, const float *rho, float *xi_x, float *xi_y,
                                  double *d_energy, dp_stream_t stream) {
  Ctx *c = C(ctx);
  if (!c || !rho || world < 1) return fail(DP_ERR_INVALID_ARG, "NULL argument or world < 1");
  dp::DeviceGuard g(c->device);
  if (!dp::fields_shardable(*c, world))
    return fail(DP_ERR_UNSUPPORTED, "map not shardable over world ranks (CTA-FFT path, bins divisible by world)");
  cudaStream_t s = (cudaStream_t)stream;
  const int G = world;
  const size_t nb = (size_t)c->mx * c->my, per = nb / G, blk = per / G;
  // every virtual rank's buffers side by side: S1 / R1 in t / sx, S2 / R2 in sxy / spec
  auto S1 = [&](int r) { return c->d_t + r * per; };
  auto R1 = [&](int r) { return c->d_sx + r * per; };
  auto S2 = [&](int r) { return c->d_sxy + r * per; };
  auto R2 = [&](int r) { return c->d_spec + r * per; };
  DP_CUDA(cudaMemsetAsync(c->d_part + c->n_wa_part, 0, sizeof(double) * c->n_en_part, s));
  for (int r = 0; r < G; r++) dp::launch_fields_shard(*c, 1, rho, false, r, G, S1(r), R1(r), S2(r), R2(r), s);
  for (int p = 0; p < G; p++)   // all-to-all: block q of rank p's S1 -> block p of rank q's R1
    for (int q = 0; q < G; q++)
      DP_CUDA(cudaMemcpyAsync(R1(q) + p * blk, S1(p) + q * blk, blk * sizeof(float), cudaMemcpyDeviceToDevice, s));
  for (int r = 0; r < G; r++) dp::launch_fields_shard(*c, 2, rho, false, r, G, S1(r), R1(r), S2(r), R2(r), s);
  for (int p = 0; p < G; p++)
    for (int q = 0; q < G; q++)
      DP_CUDA(cudaMemcpyAsync(R2(q) + p * blk, S2(p) + q * blk, blk * sizeof(float2), cudaMemcpyDeviceToDevice, s));
  for (int r = 0; r < G; r++) dp::launch_fields_shard(*c, 3, rho, false, r, G, S1(r), R1(r), S2(r), R2(r), s);
  if (xi_x || xi_y) dp::launch_split_fields(*c, xi_x, xi_y, s);
  if (d_energy) dp::launch_finalize(*c, 1.f, false, true, false, nullptr, nullptr, d_energy, nullptr, s);
  DP_CUDA(cudaGetLastError());
  return DP_OK;
}

dp_status dp_debug_wa_accumulator(dp_ctx *ctx, void *out, int64_t *n_out, dp_stream_t stream) {
  Ctx *c = C(ctx);
  if (!c || !n_out) return fail(DP_ERR_INVALID_ARG, "NULL argument");
  dp::DeviceGuard g(c->device);
  *n_out = c->g2_cells;
  if (!out) return DP_OK;
  cudaStream_t s = (cudaStream_t)stream;
  if (c->deterministic && c->d_g2i)
    DP_CUDA(cudaMemcpyAsync(out, c->d_g2i, 2 * sizeof(long long) * (size_t)c->g2_cells, cudaMemcpyDeviceToDevice, s));
  else
    DP_CUDA(cudaMemcpyAsync(out, c->d_g2, sizeof(float2) * (size_t)c->g2_cells, cudaMemcpyDeviceToDevice, s));
  DP_CUDA(cudaStreamSynchronize(s));
  return DP_OK;
}

dp_status dp_debug_transform(dp_ctx *ctx, int kind, const float *in, float *out, dp_stream_t stream) {
  Ctx *c = C(ctx);
  if (!c || !in || !out) return fail(DP_ERR_INVALID_ARG, "NULL argument");
  if (kind < DP_T_DCT2 || kind > DP_T_IDCT_IDXST) return fail(DP_ERR_INVALID_ARG, "unknown transform kind");
  if (in == out) return fail(DP_ERR_INVALID_ARG, "in and out must not alias");
  dp::DeviceGuard g(c->device);
  dp::launch_transform(*c, kind, in, out, (cudaStream_t)stream);
  DP_CUDA(cudaGetLastError());
  return DP_OK;
}

}  // extern "C"
