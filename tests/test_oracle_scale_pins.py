"""Pins for the oracle's tolerance scales theta_bar and m_bar (CPU only).

The scales are the denominators of every parity verdict (R13,
SURVEY §8(c) Z13 / step 10 of the oracle algorithm):

    m_bar_t     = b1 * m_bar_{t-1} + (1 - b1) * |g_t|          (m_bar_0 = 0)
    theta_bar_t = d * theta_bar_{t-1} + |delta_t|               (theta_bar_0 = |theta_0|)

with d = 1 - lr*wd for AdamW (1 for Adam-L2) and, in Adam-L2 mode, g_t the
L2-augmented gradient g + wd*theta.  PAPER.md never writes Adam down (it cites
Adam [44]), so nothing in the paper fixes these numbers; they are
pinned here by what the mathematics fixes independently of the oracle:

  * step-1 closed forms: m_bar_1 = (1-b1)|g|, theta_bar_1 = d|theta_0| +
    lr|g|/(|g|+eps) (m_hat_1 = g, v_hat_1 = g^2), and the Adam-L2 form with
    g' = g + wd*theta_0;
  * constant gradient, wd = 0: m_bar_t = |c|(1 - b1^t) and theta_bar_t =
    |theta_0| + t*lr*|c|/(|c|+eps) (m_hat = c, v_hat = c^2 at every t);
  * zero gradient: m_bar = 0, theta_bar_t = |theta_0|(1-lr*wd)^t;
  * the triangle inequality: |theta_t| <= theta_bar_t and |m_t| <= m_bar_t
    (what makes them scales), and theta_bar grows by at most the bound on
    Adam's step, lr * (1-b1)/sqrt(1-b2) / sqrt(bias terms);
  * a 50-digit mpmath trace of each step from the oracle's stored fp32 state,
    tracking theta_bar and m_bar independently over 10 steps and comparing
    them (not just using them as bounds).
"""
import math

import numpy as np
import pytest

import oracle
import synth

LR, B1, B2, EPS = 1e-3, 0.9, 0.999, 1e-8
REL = 4 * 2.0 ** -52          # a few double roundings


def _g(bits):
    return synth.bf16_bits_to_f32(bits).astype(np.float64)


def g_bits(vals):
    a = np.asarray(vals, np.float32)
    bits = (a.view(np.uint32) >> 16).astype(np.uint16)
    assert np.array_equal(synth.bf16_bits_to_f32(bits), a)
    return bits


def close(got, exp, rel):
    got, exp = np.asarray(got, np.float64), np.asarray(exp, np.float64)
    return np.all(np.abs(got - exp) <= rel * np.abs(exp) + 1e-300)


# ---------------------------------------------------------------- step 1
@pytest.mark.parametrize("wd", [0.0, 1e-2, 0.1])
def test_scales_step1_closed_form_adamw(wd):
    n = 4096
    th0 = synth.theta0(n, block=41)
    g = synth.grad16(n, step=1, block=41)
    r = oracle.Range.fresh(th0)
    assert np.array_equal(r.theta_bar, np.abs(th0.astype(np.float64))) and not r.m_bar.any()
    oracle.adam_range(r, g, oracle.hparams(step=1, lr=LR, eps=EPS, weight_decay=wd))
    gd = _g(g)
    assert close(r.m_bar, (1 - B1) * np.abs(gd), REL)
    exp = (1 - LR * wd) * np.abs(th0.astype(np.float64)) + LR * np.abs(gd) / (np.abs(gd) + EPS)
    # |delta_1| comes from m1, v1 rounded to fp32 storage: relative 2^-24 each
    assert close(r.theta_bar, exp, 2.0 ** -21)
    # |delta_1| -> lr as eps -> 0 (SURVEY §8(c) pins): theta_bar_1 - d|theta_0| <= lr
    assert np.all(r.theta_bar - (1 - LR * wd) * np.abs(th0.astype(np.float64)) <= LR * (1 + 2.0 ** -20))


def test_scales_step1_closed_form_adam_l2():
    n, wd = 4096, 1e-2
    th0 = synth.theta0(n, block=42)
    g = synth.grad16(n, step=1, block=42)
    r = oracle.Range.fresh(th0)
    oracle.adam_range(r, g, oracle.hparams(step=1, weight_decay=wd, mode=oracle.ADAM_L2))
    gp = _g(g) + wd * th0.astype(np.float64)          # the L2-augmented gradient
    assert close(r.m_bar, (1 - B1) * np.abs(gp), REL)
    exp = np.abs(th0.astype(np.float64)) + LR * np.abs(gp) / (np.abs(gp) + EPS)   # no decoupled decay
    assert close(r.theta_bar, exp, 2.0 ** -21)


def test_scales_apply_wd_off_has_no_decay():
    n = 1024
    th0 = synth.theta0(n, block=43)
    g = synth.grad16(n, step=1, block=43)
    r = oracle.Range.fresh(th0, apply_wd=0)
    oracle.adam_range(r, g, oracle.hparams(step=1, weight_decay=0.1))
    gd = _g(g)
    assert close(r.theta_bar, np.abs(th0.astype(np.float64)) + LR * np.abs(gd) / (np.abs(gd) + EPS), 2.0 ** -21)
    assert close(r.m_bar, (1 - B1) * np.abs(gd), REL)


# ------------------------------------------------------- constant gradient
@pytest.mark.parametrize("b1", [0.9, 0.5])
def test_scales_constant_grad_closed_form(b1):
    vals = np.array([2.0 ** -10, -(2.0 ** -20), 3 * 2.0 ** -15, -(2.0 ** -8), 2.0 ** -27, -(2.0 ** -26)], np.float32)
    g = g_bits(vals)
    th0 = np.array([0.01, -0.02, 0.03, 0.0, -0.004, 0.0], np.float32)
    c = vals.astype(np.float64)
    r = oracle.Range.fresh(th0)
    for t in range(1, 11):
        oracle.adam_range(r, g, oracle.hparams(step=t, beta1=b1, weight_decay=0.0))
        assert close(r.m_bar, np.abs(c) * (1 - b1 ** t), 8 * 2.0 ** -52), t
        exp = np.abs(th0.astype(np.float64)) + t * LR * np.abs(c) / (np.abs(c) + EPS)
        # each |delta| sees m, v after up to t fp32 roundings (relative t * 2^-24 each)
        assert close(r.theta_bar, exp, 4 * t * 2.0 ** -24), t


def test_scales_zero_grad_decay():
    n, wd, T = 1000, 1e-2, 10
    th0 = synth.theta0(n, block=44)
    r = oracle.Range.fresh(th0)
    for t in range(1, T + 1):
        oracle.adam_range(r, np.zeros(n, np.uint16), oracle.hparams(step=t, weight_decay=wd))
    assert not r.m_bar.any()
    assert close(r.theta_bar, np.abs(th0.astype(np.float64)) * (1 - LR * wd) ** T, 4 * T * 2.0 ** -52)


# ----------------------------------------------------------------- invariants
@pytest.mark.parametrize("mode", [oracle.ADAMW, oracle.ADAM_L2])
def test_scales_bound_the_state_and_the_step(mode):
    """|theta_t| <= theta_bar_t and |m_t| <= m_bar_t (triangle inequality
    through the recursions; fp32 storage adds <= t half-ulps), equality
    of |m| and m_bar where the gradient never changes sign, and every
    per-step growth |delta_t| <= lr (1-b1)/sqrt(1-b2) * sqrt(bc2)/bc1
    (|m_hat|/sqrt(v_hat) is bounded by Cauchy-Schwarz over the EMA weights)."""
    n, T, wd = 20_000, 10, 1e-2
    th0 = synth.theta0(n, block=45)
    r = oracle.Range.fresh(th0)
    prev = r.theta_bar.copy()
    for t in range(1, T + 1):
        g = synth.grad16(n, step=t, block=45)
        oracle.adam_range(r, g, oracle.hparams(step=t, weight_decay=wd, mode=mode))
        slack = 1 + t * 2.0 ** -23
        assert np.all(np.abs(r.p32.astype(np.float64)) <= r.theta_bar * slack), t
        assert np.all(np.abs(r.m32.astype(np.float64)) <= r.m_bar * slack + 1e-300), t
        d = (1 - LR * wd) if mode == oracle.ADAMW else 1.0
        bc1, bc2 = 1 - B1 ** t, 1 - B2 ** t
        # |m_hat|/sqrt(v_hat) <= sqrt(sum_k w1_k^2 / w2_k) * sqrt(bc2)/bc1, w1_k = (1-b1) b1^(t-k),
        # w2_k = (1-b2) b2^(t-k): the sum is (1-b1)^2/(1-b2) * sum (b1^2/b2)^j
        q = B1 * B1 / B2
        cs = math.sqrt((1 - B1) ** 2 / (1 - B2) * sum(q ** j for j in range(t))) * math.sqrt(bc2) / bc1
        growth = r.theta_bar - d * prev
        assert np.all(growth >= -4 * 2.0 ** -52 * r.theta_bar), t
        assert np.all(growth <= LR * cs * (1 + 2.0 ** -20)), (t, growth.max(), LR * cs)
        prev = r.theta_bar.copy()
    # a gradient of one sign: m_bar equals |m| up to fp32 storage of m
    vals = np.full(64, 2.0 ** -12, np.float32) * np.arange(1, 65, dtype=np.float32)
    r = oracle.Range.fresh(np.zeros(64, np.float32))
    for t in range(1, 6):
        gb = g_bits(-(vals * (t % 3 + 1)).astype(np.float32))
        oracle.adam_range(r, gb, oracle.hparams(step=t, weight_decay=0.0))
    assert close(np.abs(r.m32), r.m_bar, 6 * 2.0 ** -24)


# ---------------------------------------------------------------- brute force
@pytest.mark.parametrize("mode", [oracle.ADAMW, oracle.ADAM_L2])
def test_scales_mpmath_trace(mode):
    """50-digit trace: every step starts from the oracle's stored fp32
    (theta, m, v) and recomputes that step's update; theta_bar and m_bar are
    tracked by the trace itself from theta_bar_0 = |theta_0|, m_bar_0 = 0 over
    all 10 steps and compared with the oracle's at every step."""
    mp = pytest.importorskip("mpmath")
    mp.mp.dps = 50
    n, T, wd = 16, 10, 1e-2
    th0 = synth.theta0(n, block=46)
    r = oracle.Range.fresh(th0)
    L, Bt1, Bt2, E, W = (mp.mpf(x) for x in (LR, B1, B2, EPS, wd))
    TB = [abs(mp.mpf(float(x))) for x in th0]
    MB = [mp.mpf(0)] * n
    for t in range(1, T + 1):
        g = synth.grad16(n, step=t, block=46)
        P0, M0, V0 = r.p32.copy(), r.m32.copy(), r.v32.copy()
        oracle.adam_range(r, g, oracle.hparams(step=t, weight_decay=wd, mode=mode))
        for i in range(n):
            gi = mp.mpf(float(_g(g)[i]))
            th = mp.mpf(float(P0[i]))
            if mode == oracle.ADAMW:
                th = th * (1 - L * W)
                d = 1 - L * W
            else:
                gi = gi + W * th
                d = mp.mpf(1)
            m = Bt1 * mp.mpf(float(M0[i])) + (1 - Bt1) * gi
            v = Bt2 * mp.mpf(float(V0[i])) + (1 - Bt2) * gi * gi
            delta = L * (m / (1 - Bt1 ** t)) / (mp.sqrt(v / (1 - Bt2 ** t)) + E)
            MB[i] = Bt1 * MB[i] + (1 - Bt1) * abs(gi)
            TB[i] = d * TB[i] + abs(delta)
            assert abs(r.m_bar[i] - float(MB[i])) <= 1e-13 * float(MB[i]) + 1e-300, (t, i)
            assert abs(r.theta_bar[i] - float(TB[i])) <= 1e-13 * float(TB[i]), (t, i)
            # this step's stored fp32 results: within one fp32 rounding of the exact value
            for got, ex in ((r.p32[i], th - delta), (r.m32[i], m), (r.v32[i], v)):
                ex = float(ex)
                assert abs(float(got) - ex) <= 0.5 * float(np.spacing(np.float32(abs(ex)))) * (1 + 1e-6) + 1e-300, \
                    (t, i, float(got), ex)


def test_scales_step1_with_clip_use_the_clipped_gradient():
    """With the global-norm clip the update sees g' = coef * g (R9, torch's
    clip_grad_norm_), so the scales are built from it: m_bar_1 = (1-b1)|g'|,
    theta_bar_1 = d|theta_0| + lr|g'|/(|g'|+eps), coef from the float64 norm."""
    import torch
    n, max_norm = 4096, 1e-4
    th0 = synth.theta0(n, block=47)
    g = synth.grad16(n, step=1, block=47)
    r = oracle.Range.fresh(th0)
    S, coef = oracle.adam_step([r], [g], oracle.hparams(step=1), max_grad_norm=max_norm)
    norm = float(torch.linalg.vector_norm(torch.from_numpy(_g(g))))
    c = max_norm / (norm + 1e-6)
    assert 0 < c < 1 and abs(coef - c) <= 1e-12 * c
    gp = c * _g(g)
    assert close(r.m_bar, (1 - B1) * np.abs(gp), 1e-12)
    exp = (1 - LR * 1e-2) * np.abs(th0.astype(np.float64)) + LR * np.abs(gp) / (np.abs(gp) + EPS)
    assert close(r.theta_bar, exp, 2.0 ** -21)
