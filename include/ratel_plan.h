/*
 * ratel_plan.h -- C ABI of Ratel's holistic traffic-aware activation swapping
 * planner (§IV-D "Holistic Traffic-Aware Activation Swapping
 * Management"), exported by libratel.so.
 *
 * Given the model's layers (activation bytes A_i, recompute FLOPs FLOP_i) and
 * the measured machine (Table I), the planner picks the activations
 * to swap GPU -> main memory (the rest are recomputed in backward) so that the
 * iteration time T_iter = T_f + T_b (Eq. 1, 4, 5) is minimal, exploiting that
 * T_iter is convex in the swapped amount A_G2M: Algorithm 1
 * walks the layers by offloading benefit OB = FLOP/A (Eq. 6)
 * and stops at the first layer that no longer lowers T_iter once A_G2M has
 * reached A_interBlock (the minimum safe amount, Case 1).
 *
 * Pure host code: no CUDA, no ratel_init needed, thread-safe (no state), IEEE
 * double arithmetic in the paper's order without FMA contraction.
 *
 * Readings:
 *   R18  alpha*A_G2M = max(0, A_G2M - MEM_M^avail); Eq. 4's MEM_CPU^avail is
 *        Table I's MEM_M^avail.
 *   R19  Eq. 7 clamps at A_G2M >= sum(A): FLOP_r = FLOP_f - sum(FLOP).
 *   R20  layers are sorted by OB descending, stable (equal OB keep input order).
 *   R21  the OOM guard of Algorithm 1 line 12 tests the amount already in the
 *        swap list (before adding the current layer) against A_interBlock.
 *   R22  the plan's A_G2M / FLOP_r / T_iter are the swap list's totals.
 *
 * Errors: RATEL_EINVAL (include/ratel.h) for a NULL pointer, n_layers < 0, a
 * non-finite value, THP_G / BW_* <= 0, MEM_M^avail / P / FLOP_f / FLOP_i < 0,
 * or A_i <= 0 (a layer with no activation has no offloading benefit); nothing
 * is written then and ratel_last_error() says which argument.
 */
#ifndef RATEL_PLAN_H
#define RATEL_PLAN_H

#ifdef __cplusplus
extern "C" {
#endif

/* Table I quantities independent of the swap decision. */
typedef struct {
  double thp_g;        /* THP_G: measured peak GPU throughput, FLOP/s (> 0) */
  double bw_g;         /* BW_G: max unidirectional GPU<->main PCIe bandwidth, B/s (> 0) */
  double bw_s2m;       /* BW_S2M: SSD -> main memory bandwidth, B/s (> 0) */
  double bw_m2s;       /* BW_M2S: main memory -> SSD bandwidth, B/s (> 0) */
  double mem_m_avail;  /* MEM_M^avail: minimum unallocated main memory, bytes (>= 0) */
  double params;       /* P: number of parameters (2P = bytes of a 16-bit copy) (>= 0) */
  double flop_f;       /* FLOP_f: forward FLOPs; backward is 2 FLOP_f (Table I) (>= 0) */
} ratel_swap_model;

typedef struct {
  double act_bytes;       /* A_i: bytes of the layer's activations (> 0) */
  double recompute_flop;  /* FLOP_i: FLOPs to recompute them (>= 0) */
} ratel_swap_layer;

typedef struct {
  int n_swap;          /* swapped layers = order[0 .. n_swap) */
  double a_g2m;        /* A_G2M: their activation bytes (summed in OB order) */
  double flop_r;       /* FLOP_r = FLOP_f - their recompute FLOPs (subtracted in OB order) */
  double t_f, t_b;     /* Eq. 4 and Eq. 5 at (a_g2m, flop_r), seconds */
  double t_iter;       /* Eq. 1: t_f + t_b */
  double t_min;        /* Algorithm 1's Tmin when it stopped (+inf for no layers) */
} ratel_swap_plan;

/* Eq. 1/4/5: T_f and T_b for a given A_G2M (bytes) and FLOP_r.  t_f, t_b:
 * caller-owned outputs (either may be NULL). */
int ratel_swap_iter_time(const ratel_swap_model* model, double a_g2m, double flop_r,
                         double* t_f, double* t_b);

/* Eq. 7: recomputation FLOPs when A_G2M bytes are swapped, the layers taken
 * in OB order and the last one partially (footnote 5's interpolation). */
int ratel_swap_recompute_flop(const ratel_swap_layer* layers, int n_layers, double flop_f,
                              double a_g2m, double* flop_r);

/* Algorithm 1.  layers: n_layers entries (caller-owned, read only).  order:
 * caller-owned array of n_layers ints, receives every layer index in OB
 * order (R20); the swapped layers are its first plan->n_swap entries.
 * a_inter_block: A_interBlock, bytes (>= 0). */
int ratel_plan_activation_swap(const ratel_swap_layer* layers, int n_layers,
                               const ratel_swap_model* model, double a_inter_block,
                               int* order, ratel_swap_plan* plan);

#ifdef __cplusplus
}
#endif

#endif /* RATEL_PLAN_H */
