// ratel_plan.cpp -- Ratel's traffic-aware activation swapping planner
// (§IV-D), the C ABI of include/ratel_plan.h.
//
// Host-only: the planner runs once per model/batch shape before training (the
// paper drives it with profiled layer sizes and measured bandwidths), so it is
// O(n log n) scalar code.  The layers are sorted once by offloading benefit
// (Eq. 6); prefix sums of A and FLOP in that order give Eq. 7 by one binary
// search and Algorithm 1 by one forward scan that evaluates Eq. 1/4/5 per
// prefix.  Every sum is accumulated in OB order and every formula is
// evaluated in the order the paper writes it, in IEEE double with no FMA
// contraction, so the result is reproducible bit for bit.
#pragma GCC optimize("fp-contract=off")

#include <algorithm>
#include <cmath>
#include <cstdio>
#include <limits>
#include <numeric>
#include <vector>

#include "ratel.h"
#include "ratel_plan.h"
#include "ratel_plan_impl.h"

namespace {

int bad(const char* what) {
  char msg[160];
  std::snprintf(msg, sizeof msg, "ratel swap planner: invalid %s", what);
  return ratel::report_error(RATEL_EINVAL, msg);
}

bool is_fin(double x) { return std::isfinite(x); }

int check_model(const ratel_swap_model* m) {
  if (m == nullptr) return bad("model (NULL)");
  if (!is_fin(m->thp_g) || m->thp_g <= 0) return bad("model.thp_g (THP_G must be finite and > 0)");
  if (!is_fin(m->bw_g) || m->bw_g <= 0) return bad("model.bw_g (BW_G must be finite and > 0)");
  if (!is_fin(m->bw_s2m) || m->bw_s2m <= 0) return bad("model.bw_s2m (BW_S2M must be finite and > 0)");
  if (!is_fin(m->bw_m2s) || m->bw_m2s <= 0) return bad("model.bw_m2s (BW_M2S must be finite and > 0)");
  if (!is_fin(m->mem_m_avail) || m->mem_m_avail < 0) return bad("model.mem_m_avail (must be finite and >= 0)");
  if (!is_fin(m->params) || m->params < 0) return bad("model.params (P must be finite and >= 0)");
  if (!is_fin(m->flop_f) || m->flop_f < 0) return bad("model.flop_f (FLOP_f must be finite and >= 0)");
  return RATEL_OK;
}

int check_layers(const ratel_swap_layer* layers, int n) {
  if (n < 0) return bad("n_layers (< 0)");
  if (n > 0 && layers == nullptr) return bad("layers (NULL)");
  for (int i = 0; i < n; ++i) {
    if (!is_fin(layers[i].act_bytes) || layers[i].act_bytes <= 0) return bad("layer act_bytes (must be finite and > 0)");
    if (!is_fin(layers[i].recompute_flop) || layers[i].recompute_flop < 0)
      return bad("layer recompute_flop (must be finite and >= 0)");
  }
  return RATEL_OK;
}

// Eq. 3 with R18: the activations main memory cannot hold go to the SSDs.
double spilled(const ratel_swap_model& m, double a_g2m) { return std::max(0.0, a_g2m - m.mem_m_avail); }

double max4(double a, double b, double c, double d) { return std::max(std::max(a, b), std::max(c, d)); }

// Eq. 4: GPU compute | GPU->main activations | main->GPU P16 | SSD.
double t_forward(const ratel_swap_model& m, double a_g2m) {
  return max4(m.flop_f / m.thp_g, a_g2m / m.bw_g, 2.0 * m.params / m.bw_g,
              2.0 * m.params / m.bw_s2m + spilled(m, a_g2m) / m.bw_m2s);
}

// Eq. 5: compute incl. recomputation | G16 out | P16 + activations
// in | SSD (14P states + spilled activations read, 14P written; simplex).
double t_backward(const ratel_swap_model& m, double a_g2m, double flop_r) {
  return max4((2.0 * m.flop_f + flop_r) / m.thp_g, 2.0 * m.params / m.bw_g, (2.0 * m.params + a_g2m) / m.bw_g,
              (14.0 * m.params + spilled(m, a_g2m)) / m.bw_s2m + 14.0 * m.params / m.bw_m2s);
}

// Algorithm 1 line 6 (R20): indices by OB = FLOP/A (Eq. 6) descending, stable.
std::vector<int> ob_order(const ratel_swap_layer* layers, int n) {
  std::vector<double> ob(n);
  for (int i = 0; i < n; ++i) ob[i] = layers[i].recompute_flop / layers[i].act_bytes;
  std::vector<int> idx(n);
  std::iota(idx.begin(), idx.end(), 0);
  std::stable_sort(idx.begin(), idx.end(), [&](int a, int b) { return ob[a] > ob[b]; });
  return idx;
}

}  // namespace

extern "C" {

int ratel_swap_iter_time(const ratel_swap_model* model, double a_g2m, double flop_r, double* t_f, double* t_b) {
  if (int rc = check_model(model)) return rc;
  if (!is_fin(a_g2m) || a_g2m < 0) return bad("a_g2m (must be finite and >= 0)");
  if (!is_fin(flop_r)) return bad("flop_r (must be finite)");
  if (t_f) *t_f = t_forward(*model, a_g2m);
  if (t_b) *t_b = t_backward(*model, a_g2m, flop_r);
  return RATEL_OK;
}

int ratel_swap_recompute_flop(const ratel_swap_layer* layers, int n_layers, double flop_f, double a_g2m,
                              double* flop_r) {
  if (int rc = check_layers(layers, n_layers)) return rc;
  if (!is_fin(flop_f) || flop_f < 0) return bad("flop_f (must be finite and >= 0)");
  if (!is_fin(a_g2m) || a_g2m < 0) return bad("a_g2m (must be finite and >= 0)");
  if (flop_r == nullptr) return bad("flop_r (NULL)");
  const std::vector<int> order = ob_order(layers, n_layers);
  // cover[k] = A of the first k layers in OB order, fr[k] = FLOP_f minus their FLOPs
  std::vector<double> cover(n_layers + 1), fr(n_layers + 1);
  cover[0] = 0.0;
  fr[0] = flop_f;
  for (int k = 0; k < n_layers; ++k) {
    cover[k + 1] = cover[k] + layers[order[k]].act_bytes;
    fr[k + 1] = fr[k] - layers[order[k]].recompute_flop;
  }
  // whole layers: the largest k with cover[k] <= a_g2m; then layer k (0-based in
  // OB order) contributes the fraction (a_g2m - cover[k]) / A of its FLOPs (Eq. 7)
  const int k = static_cast<int>(std::upper_bound(cover.begin(), cover.end(), a_g2m) - cover.begin()) - 1;
  if (k >= n_layers) {
    *flop_r = fr[n_layers];  // R19
  } else {
    const ratel_swap_layer& l = layers[order[k]];
    *flop_r = fr[k] - l.recompute_flop * (a_g2m - cover[k]) / l.act_bytes;
  }
  return RATEL_OK;
}

int ratel_plan_activation_swap(const ratel_swap_layer* layers, int n_layers, const ratel_swap_model* model,
                               double a_inter_block, int* order, ratel_swap_plan* plan) {
  if (int rc = check_model(model)) return rc;
  if (int rc = check_layers(layers, n_layers)) return rc;
  if (!is_fin(a_inter_block) || a_inter_block < 0) return bad("a_inter_block (must be finite and >= 0)");
  if (plan == nullptr) return bad("plan (NULL)");
  if (n_layers > 0 && order == nullptr) return bad("order (NULL)");
  const ratel_swap_model& m = *model;
  const std::vector<int> idx = ob_order(layers, n_layers);

  // Algorithm 1: grow the swap list along the OB order while
  // T_iter improves; once the list holds A_interBlock (R21), the first layer
  // that does not lower T_iter ends it -- by convexity no later prefix is better.
  double t_min = std::numeric_limits<double>::infinity();
  double a_g2m = 0.0, flop_r = m.flop_f;  // lines 2-4: nothing swapped = full recomputation
  int n_swap = 0;
  for (; n_swap < n_layers; ++n_swap) {
    const ratel_swap_layer& l = layers[idx[n_swap]];
    const double a_next = a_g2m + l.act_bytes;             // line 8
    const double fr_next = flop_r - l.recompute_flop;      // line 9
    const double t = t_forward(m, a_next) + t_backward(m, a_next, fr_next);  // line 10, Eq. 1
    if (t >= t_min) {
      if (a_g2m >= a_inter_block) break;                   // lines 11-13
    } else {
      t_min = t;                                           // line 16
    }
    a_g2m = a_next;                                        // line 18: swap it
    flop_r = fr_next;
  }
  std::copy(idx.begin(), idx.end(), order);
  plan->n_swap = n_swap;
  plan->a_g2m = a_g2m;
  plan->flop_r = flop_r;
  plan->t_f = t_forward(m, a_g2m);
  plan->t_b = t_backward(m, a_g2m, flop_r);
  plan->t_iter = plan->t_f + plan->t_b;
  plan->t_min = t_min;
  return RATEL_OK;
}

}  // extern "C"
