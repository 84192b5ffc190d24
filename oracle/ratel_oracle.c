/*
 * ratel_oracle.c -- CPU ORACLE for the Ratel active-gradient-offloading step.
 *
 * TEST INFRASTRUCTURE ONLY.  Only tests/, __graft_entry__.smoke() and
 * bench.py's cpu_baseline / --impl reference legs may load this library.
 * It shares no code, header, table or constant with the CUDA library
 * (paper_conf_icde_liaosyxcyww25_b200/csrc) and never includes its headers.
 *
 * What it computes.  PAPER.md never writes the optimizer out: "Adam optimizer
 * [44] is generally adopted ... which introduces auxiliary optimizer states"
 * (§II "LLM Training Stages"); model states are P32 (fp32 master),
 * OS32 (fp32 Adam m and v), G16 (16-bit grads) and P16 (16-bit working copy)
 * (Table II); "the CPU updates the model states of the
 * tensor i and produces a 16-bit parameter copy" (§IV-C).
 * Active gradient offloading only reorders/overlaps that update and "keeps
 * synchronous model updating" (footnote 4 P:L1147-1152), so the
 * oracle is the plain synchronous mixed-precision Adam(W) step, per element,
 * in double, with fp32 storage -- DESIGN.md readings R1-R9:
 *
 *   g  = (double) bf16(G16[i])                      exact widening     (R5)
 *   g *= coef                                       clip, if enabled   (R9)
 *   AdamW + wd: theta = theta * (1 - lr*wd)         decoupled          (R3)
 *   Adam-L2 + wd: g = g + wd*theta                  torch.optim.Adam   (R3)
 *   m = b1*m + (1-b1)*g ;  v = b2*v + (1-b2)*g*g
 *   bc1 = 1 - b1^t ; bc2 = 1 - b2^t                 pow in double      (R6)
 *   delta = lr * (m/bc1) / (sqrt(v/bc2) + eps)       eps outside root   (R2)
 *   theta = theta - delta
 *   P32,M,V = (float) theta,m,v  (round to nearest even)               (R7)
 *   P16 = bf16_rne(P32)          from the STORED fp32 master           (R7)
 *
 * Scales for the condition-aware tolerance (R13): theta_bar and m_bar,
 *   m_bar     = b1*m_bar + (1-b1)*|g|
 *   theta_bar = (1-lr*wd)*theta_bar + |delta|   (AdamW; Adam-L2: + |delta|)
 *
 * Build: gcc -O2 -ffp-contract=off -fopenmp -fPIC -shared (no -ffast-math, no
 * FMA contraction: the double arithmetic is exactly the C expression order).
 * Pinned by tests/test_oracle_pins.py (closed forms, invariants, torch float64
 * AdamW/Adam/clip_grad_norm_, a 50-digit mpmath trace, exhaustive bf16 RNE);
 * the scales by tests/test_oracle_scale_pins.py (step-1 and constant-gradient
 * closed forms, zero-gradient decay, |theta| <= theta_bar and |m| <= m_bar,
 * the Cauchy-Schwarz bound on each step, a 50-digit trace of both scales).
 */
#include <math.h>
#include <stddef.h>
#include <stdint.h>
#include <string.h>

#define ORACLE_ADAMW 0
#define ORACLE_ADAM_L2 1

typedef struct {
  double lr, beta1, beta2, eps, weight_decay;
  int64_t step; /* 1-based t */
  int mode;     /* ORACLE_ADAMW | ORACLE_ADAM_L2 */
} oracle_hparams;

/* bf16 -> double: the bf16 pattern is the top half of an fp32; exact. */
double oracle_bf16_to_double(uint16_t b) {
  uint32_t u = (uint32_t)b << 16;
  float f;
  memcpy(&f, &u, sizeof f);
  return (double)f;
}

/* fp32 -> bf16, round to nearest, ties to even -- the definition written out:
 * the two bf16 neighbours of x are its truncation `lo` and the next pattern
 * up in magnitude `lo+1`; pick the nearer, on a tie the one with an even
 * last bit.  Overflow past the largest finite rounds to Inf like IEEE.
 * NaN -> quiet NaN 0x7FC0 with the sign kept (R7). */
uint16_t oracle_bf16_rne(float x) {
  uint32_t u;
  memcpy(&u, &x, sizeof u);
  if ((u & 0x7F800000u) == 0x7F800000u && (u & 0x007FFFFFu) != 0)
    return (uint16_t)(((u >> 16) & 0x8000u) | 0x7FC0u);
  uint16_t lo = (uint16_t)(u >> 16);   /* truncation toward zero */
  uint32_t rem = u & 0xFFFFu;          /* discarded bits: rem / 2^16 of one bf16 ulp */
  if (rem > 0x8000u) return (uint16_t)(lo + 1);
  if (rem < 0x8000u) return lo;
  return (lo & 1u) ? (uint16_t)(lo + 1) : lo; /* exact tie: to even */
}

void oracle_bf16_rne_array(const float* x, uint16_t* out, size_t n) {
  for (size_t i = 0; i < n; ++i) out[i] = oracle_bf16_rne(x[i]);
}

/* One element of the update in double.  Returns |delta| for the scale. */
static double adam_elem(double g, double* theta, double* m, double* v, int apply_wd,
                        const oracle_hparams* hp, double* g_used) {
  double th = *theta;
  if (apply_wd && hp->weight_decay != 0.0) {
    if (hp->mode == ORACLE_ADAMW)
      th = th * (1.0 - hp->lr * hp->weight_decay);
    else
      g = g + hp->weight_decay * th;
  }
  double mm = hp->beta1 * (*m) + (1.0 - hp->beta1) * g;
  double vv = hp->beta2 * (*v) + (1.0 - hp->beta2) * g * g;
  double t = (double)hp->step;
  double bc1 = 1.0 - pow(hp->beta1, t);
  double bc2 = 1.0 - pow(hp->beta2, t);
  double delta = hp->lr * (mm / bc1) / (sqrt(vv / bc2) + hp->eps);
  th = th - delta;
  *theta = th;
  *m = mm;
  *v = vv;
  *g_used = g;
  return fabs(delta);
}

static void update_scales(size_t i, double g_used, double absdelta, int apply_wd,
                          const oracle_hparams* hp, double* theta_bar, double* m_bar) {
  if (m_bar) m_bar[i] = hp->beta1 * m_bar[i] + (1.0 - hp->beta1) * fabs(g_used);
  if (theta_bar) {
    double d = (apply_wd && hp->mode == ORACLE_ADAMW) ? (1.0 - hp->lr * hp->weight_decay) : 1.0;
    theta_bar[i] = d * theta_bar[i] + absdelta;
  }
}

/* The product semantics: fp32 states, bf16 grads and working copy.
 * g16/p32/m32/v32/p16 are n-element arrays; theta_bar/m_bar may be NULL.
 * threads > 1 parallelises over elements (results are identical: the update
 * is elementwise). */
void oracle_adam_range(size_t n, const uint16_t* g16, double coef, int apply_wd,
                       const oracle_hparams* hp, float* p32, float* m32, float* v32,
                       uint16_t* p16, double* theta_bar, double* m_bar, int threads) {
  (void)threads;
#pragma omp parallel for schedule(static) num_threads(threads > 0 ? threads : 1) if (threads > 1)
  for (size_t i = 0; i < n; ++i) {
    double g = oracle_bf16_to_double(g16[i]) * coef;
    double th = (double)p32[i], m = (double)m32[i], v = (double)v32[i], gu;
    double ad = adam_elem(g, &th, &m, &v, apply_wd, hp, &gu);
    p32[i] = (float)th;
    m32[i] = (float)m;
    v32[i] = (float)v;
    p16[i] = oracle_bf16_rne(p32[i]);
    update_scales(i, gu, ad, apply_wd, hp, theta_bar, m_bar);
  }
}

/* Same update with double states (no fp32 storage) -- used only to pin the
 * arithmetic against a high-precision brute-force trace. */
void oracle_adam_range_f64(size_t n, const double* g, double coef, int apply_wd,
                           const oracle_hparams* hp, double* p, double* m, double* v) {
  for (size_t i = 0; i < n; ++i) {
    double gu;
    adam_elem(g[i] * coef, &p[i], &m[i], &v[i], apply_wd, hp, &gu);
  }
}

/* Sum of squares of the widened bf16 grads, in double, in index order,
 * continuing a running sum s0 (so a sum over several ranges is one
 * index-ordered sum over their concatenation). */
double oracle_grad_sumsq(const uint16_t* g16, size_t n, double s0) {
  double s = s0;
  for (size_t i = 0; i < n; ++i) {
    double g = oracle_bf16_to_double(g16[i]);
    s += g * g;
  }
  return s;
}

/* torch.nn.utils.clip_grad_norm_ semantics (R9): coef = max_norm/(||g||+1e-6),
 * clamped to at most 1. */
double oracle_clip_coef(double sumsq, double max_norm) {
  double c = max_norm / (sqrt(sumsq) + 1e-6);
  return (c < 1.0 || isnan(c)) ? c : 1.0; /* NaN propagates like torch.clamp */
}

/* ---- Data-parallel gradient reduction (R17) ----
 * With the reduce-scatter fused into the update, the gradient of element i is
 * the data-parallel combination of the N ranks' local bf16 gradients,
 *     g[i] = scale * sum_{q=0..nq-1} (double) bf16(G16_q[i]),
 * summed in double in rank order (scale = 1/N gives DDP's mean, 1 the sum).
 * The paper leaves multi-GPU gradient semantics unspecified;
 * this is the plain definition of a sum/mean all-reduce, written out. */
void oracle_reduce_grads(size_t n, const uint16_t* const* g16s, int nq, double scale, double* out) {
  for (size_t i = 0; i < n; ++i) {
    double s = 0.0;
    for (int q = 0; q < nq; ++q) s = s + oracle_bf16_to_double(g16s[q][i]);
    out[i] = scale * s;
  }
}

/* The update of oracle_adam_range from a double gradient (the reduced one):
 * the same per-element steps, g = g[i] * coef instead of the widened bf16. */
void oracle_adam_range_gd(size_t n, const double* gd, double coef, int apply_wd,
                          const oracle_hparams* hp, float* p32, float* m32, float* v32,
                          uint16_t* p16, double* theta_bar, double* m_bar) {
  for (size_t i = 0; i < n; ++i) {
    double g = gd[i] * coef;
    double th = (double)p32[i], m = (double)m32[i], v = (double)v32[i], gu;
    double ad = adam_elem(g, &th, &m, &v, apply_wd, hp, &gu);
    p32[i] = (float)th;
    m32[i] = (float)m;
    v32[i] = (float)v;
    p16[i] = oracle_bf16_rne(p32[i]);
    update_scales(i, gu, ad, apply_wd, hp, theta_bar, m_bar);
  }
}

/* Sum of squares of a double gradient, in index order, continuing s0. */
double oracle_grad_sumsq_d(const double* g, size_t n, double s0) {
  double s = s0;
  for (size_t i = 0; i < n; ++i) s += g[i] * g[i];
  return s;
}
