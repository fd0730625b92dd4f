// Window-size solver: the paper's analytic model (§III-D).
//
//   P1 (FP, eq. 1a-1d):  min m  s.t.  (1b) window compute >= fetch of the layer entering it,
//                        (1c) memory <= S_avail (hard), (1d) window compute >= Σc2g + Σg2c (soft)
//   P2 (BP, eq. 2a-2d):  min m  s.t.  (2b) window BP time >= transfers of the layer entering it,
//                        (2c) memory (hard), (2d) soft as (1d)
//   window rule: m meeting P1 and P2 for all layers; otherwise the largest m
//                        the memory permits.
//   eq. 3 / eq. 4 are evaluated and reported, not used to choose m.
//
// Readings (R4-R8): m = w = prefetch distance; the sums of (1b)/(1d) run over the
// w layers before the entering layer j; (2b) uses the decoupled param/grad slot halves of this
// engine, so the entering layer's fetch and the leaving layer's offload proceed in opposite
// link directions and the constraint is max(g2c, c2g) (a GPU-optimised entering layer is
// restaged by K1: t_stage replaces t_c2g); the soft constraints use the paper's half-duplex
// sum unless `duplex` is set (then max); "min m" with soft constraints is lexicographic:
// hard and soft (only for w < L: at w = L nothing moves and every window sum is empty, so the
// soft constraint is vacuous there) -> hard only -> memory maximum.  Optional (cpu_hard, R19):
// the CPU Adam of the host layers must fit in one step's GPU time (the throughput form of eq. 3).  The implementation uses prefix sums; the
// oracle (oracle/autotune_oracle.py) evaluates the same definitions with plain loops.
#include <algorithm>
#include <cmath>
#include <vector>

#include "sh_internal.hpp"

namespace sh {

namespace {
struct Prefix {
  std::vector<double> s;  // s[i] = Σ_{k<i} a[k]
  explicit Prefix(const double* a, int n) : s(n + 1, 0.0) {
    for (int i = 0; i < n; ++i) s[i + 1] = s[i] + (a ? a[i] : 0.0);
  }
  double sum(int b, int e) const {  // Σ_{k=b}^{e-1}
    if (e <= b) return 0.0;
    return s[e] - s[b];
  }
};
inline double at(const double* a, int i) { return a ? a[i] : 0.0; }
}  // namespace

}  // namespace sh

using namespace sh;

extern "C" sh_status sh_solve_window(const sh_profile* P, sh_solve_report* R) {
  clear_error();
  if (!P || !R || P->n_layers < 1) {
    set_error("sh_solve_window: null profile/report or n_layers < 1");
    return SH_ERR_INVALID;
  }
  const int L = P->n_layers;
  const Prefix fp(P->t_fp, L), bp(P->t_bp, L), c2g(P->t_c2g, L), g2c(P->t_g2c, L);
  const Prefix ogpu(P->t_opt_gpu, L);
  int64_t slot = 0;
  for (int i = 0; i < L; ++i) slot = std::max<int64_t>(slot, P->slot_bytes ? P->slot_bytes[i] : 0);

  // d = prefetch distance (ring d+1 slots), g = GPU-optimised layers [0, g).  The paper couples
  // them (d = g = m); `decouple` (R22) lets g exceed d.
  auto mem_ok = [&](int d, int g) {
    int64_t need = P->fixed_bytes + (int64_t)(d + 1) * slot;
    for (int i = 0; i < g; ++i) need += P->gstate_bytes ? P->gstate_bytes[i] : 0;
    return need <= P->s_avail;
  };
  auto fetch = [&](int j, int g) { return j < g ? at(P->t_stage, j) : at(P->t_c2g, j); };
  auto fp_hard = [&](int d, int g) {  // (1b): ∀ j ∈ [d, L): Σ_{i=j-d}^{j-1} t_fp ≥ fetch of j
    for (int j = d; j < L; ++j)
      if (fp.sum(j - d, j) < fetch(j, g)) return false;
    return true;
  };
  auto bp_hard = [&](int d, int g) {  // (2b): ∀ j ∈ [0, L-d-2]: Σ_{i=j+1}^{j+d} t_bp ≥ max(g2c[j+d+1], fetch_j)
    for (int j = 0; j + d + 1 < L; ++j) {
      const double off = j + d + 1 >= g ? at(P->t_g2c, j + d + 1) : 0.0;  // G layers are not offloaded
      if (bp.sum(j + 1, j + d + 1) < std::max(off, fetch(j, g))) return false;
    }
    return true;
  };
  auto soft = [&](int d) {  // (1d) over FP windows, (2d) over BP windows
    for (int j = d; j < L; ++j) {
      const double a = c2g.sum(j - d, j), b = g2c.sum(j - d, j);
      if (fp.sum(j - d, j) < (P->duplex ? std::max(a, b) : a + b)) return false;
    }
    for (int j = 0; j + d + 1 < L; ++j) {
      const double a = c2g.sum(j + 1, j + d + 1), b = g2c.sum(j + 1, j + d + 1);
      if (bp.sum(j + 1, j + d + 1) < (P->duplex ? std::max(a, b) : a + b)) return false;
    }
    return true;
  };
  auto cpu_total = [&](int g) {
    double t = 0;
    for (int k = g; k < L; ++k) t += at(P->t_opt_cpu, k);
    return t;
  };
  auto gpu_step = [&](int g) { return fp.sum(0, L) + bp.sum(0, L) + ogpu.sum(0, g); };
  const double rho = P->cpu_util_max > 0.0 && P->cpu_util_max < 1.0 ? P->cpu_util_max : 1.0;
  auto cpu_ok = [&](int g) { return !P->cpu_hard || cpu_total(g) <= rho * gpu_step(g); };
  // fp_serial (R23): the FP fetches of the host layers share ONE link, so (1b) per layer is
  // not enough when t_c2g > t_fp.  With no stalls position p starts computing at S(p) = Σ_{i<p} t_fp;
  // the fetch of host layer j may start once its slot frees (position j-d-1 done, i.e. S(j-d)) and
  // after the previous fetch: F(j) = max(F(j-1), S(max(0, j-d))) + t_c2g[j], and must land by S(j).
  auto fp_serial_ok = [&](int d, int g) {
    if (!P->fp_serial) return true;
    double F = -INFINITY;
    for (int j = g; j < L; ++j) {
      F = std::max(F, fp.sum(0, std::max(0, j - d))) + at(P->t_c2g, j);
      if (F > fp.sum(0, j)) return false;
    }
    return true;
  };
  auto hard = [&](int d, int g) { return fp_hard(d, g) && bp_hard(d, g) && cpu_ok(g) && fp_serial_ok(d, g); };

  int wmax = -1;
  for (int w = 0; w <= L; ++w)
    if (mem_ok(w, w)) wmax = w;
  if (wmax < 0) {
    set_error("sh_solve_window: even w=0 exceeds S_avail (%lld bytes)", (long long)P->s_avail);
    return SH_ERR_OOM_DEVICE;
  }
  int best_d = -1, best_g = -1, reason = 2;
  if (!P->decouple) {
    for (int w = 0; w < L && best_d < 0; ++w)
      if (mem_ok(w, w) && hard(w, w) && soft(w)) best_d = best_g = w, reason = 0;
    for (int w = 0; w <= L && best_d < 0; ++w)
      if (mem_ok(w, w) && hard(w, w)) best_d = best_g = w, reason = 1;
  } else {
    int gmin = 0;
    while (gmin < L && !cpu_ok(gmin)) ++gmin;
    // g for a ring of d+1: the smallest meeting the CPU constraint (the paper's "min m"), or with
    // fill_gpu the largest the memory leaves (every GPU-optimised layer takes its ~30-40 B/param of
    // CPU-Adam + DMA traffic off the host DRAM); -1 if none fits
    auto g_for = [&](int d) {
      const int lo = std::max(d, gmin);
      if (!P->fill_gpu) return mem_ok(d, lo) ? lo : -1;
      int g = -1;
      for (int x = lo; x <= L; ++x)
        if (mem_ok(d, x)) g = x;
      return g;
    };
    for (int d = 0; d < L && best_d < 0; ++d) {
      const int g = g_for(d);
      if (g >= 0 && hard(d, g) && soft(d)) best_d = d, best_g = g, reason = 0;
    }
    for (int d = 0; d <= L && best_d < 0; ++d) {
      const int g = g_for(d);
      if (g >= 0 && hard(d, g)) best_d = d, best_g = g, reason = 1;
    }
    // R27, link-bound FP (no ring meets the serial form of (1b)): extra slots no longer shorten the FP,
    // they only hold gradients.  The gradient pool (the ring's grad halves) must absorb the backlog of
    // a backward pass that outruns the CPU Adam beyond what the host landing buffers take:
    // B(g) = ceil(Σ_{k>=g} max(0, 1 - t_bp^k / t_opt_cpu^k)) - landing_buffers; every other byte goes to
    // the GPU-optimised set (fill_gpu).  Smallest d with d + 1 >= B(g_for(d)) meeting the per-window
    // (1b) / (2b), g = the largest GPU set the memory leaves next to the ring.
    if (best_d < 0 && P->fill_gpu && P->landing_buffers > 0) {
      auto backlog = [&](int g) {
        double b = 0.0;
        for (int k = g; k < L; ++k) {
          const double tc = at(P->t_opt_cpu, k);
          if (tc > 0.0) b += std::max(0.0, 1.0 - at(P->t_bp, k) / tc);
        }
        return (int)std::ceil(b - 1e-9) - P->landing_buffers;
      };
      // (no CPU constraint here: when no ring meets the hard constraints the CPU Adam is typically the
      // bottleneck too, and then the largest GPU set is what relieves it)
      for (int d = 0; d <= L && best_d < 0; ++d) {
        int g = -1;
        for (int x = d; x <= L; ++x)
          if (mem_ok(d, x)) g = x;
        if (g >= 0 && d + 1 >= backlog(g) && fp_hard(d, g) && bp_hard(d, g)) best_d = d, best_g = g, reason = 3;
      }
    }
  }
  if (best_d < 0) best_d = best_g = wmax, reason = 2;

  R->window = best_g;
  R->ring_slots = best_d + 1;
  R->w_max_memory = wmax;
  R->reason = reason;
  R->fp_hard_ok = fp_hard(best_d, best_g) && fp_serial_ok(best_d, best_g);
  R->bp_hard_ok = bp_hard(best_d, best_g);
  R->soft_ok = soft(best_d);
  // eq. 3: t_opt_cpu^k ≤ Σ_{i=0}^{k}(t_fp^i + t_bp^i) + Σ_{i<g} t_opt_gpu^i,  k ∈ [g, L)
  double slack = INFINITY;
  for (int k = best_g; k < L; ++k) {
    const double rhs = fp.sum(0, k + 1) + bp.sum(0, k + 1) + ogpu.sum(0, best_g);
    slack = std::min(slack, rhs - at(P->t_opt_cpu, k));
  }
  R->eq3_min_slack_ms = std::isinf(slack) ? 0.0 : slack;
  R->eq3_ok = !(slack < 0.0);
  // eq. 4: 5 n t_async ≤ Σ_{i=g}^{n-1} t_opt_gpu
  R->eq4_lhs_ms = 5.0 * L * P->t_async;
  R->eq4_rhs_ms = ogpu.sum(best_g, L);
  R->cpu_total_ms = cpu_total(best_g);
  R->gpu_step_ms = gpu_step(best_g);
  return SH_OK;
}
