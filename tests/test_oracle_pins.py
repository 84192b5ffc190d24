"""Pins for the CPU oracle against things other than itself (CPU only).

The paper prints no optimizer values, hyperparameters or worked example
(SURVEY §8(c) "Paper values: none"), so the oracle is pinned by
mathematics and by library routines the paper names:
  * step-1 closed form (separates the two eps placements, R2),
  * bias-correction invariant under a constant gradient (R6),
  * zero-gradient decay closed form (R3),
  * beta1 = beta2 = 0 special case (sign-descent),
  * sign / power-of-two scale symmetries (bitwise),
  * torch.optim.AdamW / torch.optim.Adam (float64, foreach=False) -- Fig. 4's
    optimizer, PAPER.md P:L1525, P:L1550 -- with fp32 storage emulated,
  * torch.nn.utils.clip_grad_norm_ for the clip coefficient (R9),
  * a 50-digit mpmath brute-force trace of the double arithmetic,
  * exhaustive bf16 round-to-nearest-even against torch's cast.
"""
import math

import numpy as np
import pytest
import torch

import oracle
import synth
from tests.tolerance import check_range

F32 = np.float32


def f32ulp(x):
    return np.spacing(np.abs(np.float32(x))).astype(np.float64)


def run_steps(theta0, grads, hp_kw, apply_wd=1, steps=None):
    r = oracle.Range.fresh(theta0, apply_wd)
    for t, g in enumerate(grads, start=1):
        oracle.adam_range(r, g, oracle.hparams(step=t, **hp_kw))
    return r


def g_bits(vals):
    """bf16 bit patterns of values that are exactly representable in bf16."""
    a = np.asarray(vals, np.float32)
    bits = (a.view(np.uint32) >> 16).astype(np.uint16)
    assert np.array_equal(synth.bf16_bits_to_f32(bits), a)
    return bits


# ---------------------------------------------------------------- closed forms
@pytest.mark.parametrize("wd", [0.0, 1e-2])
def test_step1_closed_form_adamw(wd):
    n = 4096
    th0 = synth.theta0(n, block=3)
    g = synth.grad16(n, step=1, block=3)
    lr, eps = 1e-3, 1e-8
    r = run_steps(th0, [g], dict(lr=lr, eps=eps, weight_decay=wd))
    gd = synth.bf16_bits_to_f32(g).astype(np.float64)
    # m1=(1-b1)g, v1=(1-b2)g^2 -> m_hat=g, v_hat=g^2 -> theta1 = theta0(1-lr wd) - lr g/(|g|+eps)
    exp = th0.astype(np.float64) * (1 - lr * wd) - lr * gd / (np.abs(gd) + eps)
    assert np.all(np.abs(r.p32 - exp) <= f32ulp(exp)), "theta1 != closed form"
    assert np.all(np.abs(r.m32 - 0.1 * gd) <= f32ulp(0.1 * gd))
    assert np.all(np.abs(r.v32 - 0.001 * gd * gd) <= f32ulp(0.001 * gd * gd))


def test_step1_eps_placement_separates_readings():
    """|g| ~ eps: torch/Kingma-Alg.1 (eps outside sqrt(v_hat)) vs Kingma's
    'efficient' form (eps/sqrt(1-b2) effectively).  theta0 = 0, wd = 0, so
    theta1 = -delta at full relative precision."""
    eps, lr = 1e-8, 1e-3
    vals = np.array([2.0 ** -27, -(2.0 ** -26), 2.0 ** -25, 1.5 * 2.0 ** -27], np.float32)
    g = g_bits(vals)
    r = run_steps(np.zeros(4, F32), [g], dict(lr=lr, eps=eps, weight_decay=0.0))
    gd = vals.astype(np.float64)
    torch_form = -lr * gd / (np.abs(gd) + eps)
    kingma_eff = -lr * gd / (np.abs(gd) + eps / math.sqrt(1 - 0.999))
    assert np.all(np.abs(r.p32 - torch_form) <= f32ulp(torch_form))
    assert np.all(np.abs(r.p32 - kingma_eff) > 100 * f32ulp(kingma_eff))


def test_step1_closed_form_adam_l2():
    n = 2048
    th0 = synth.theta0(n, block=1)
    g = synth.grad16(n, step=1, block=1)
    lr, eps, wd = 1e-3, 1e-8, 1e-2
    r = run_steps(th0, [g], dict(lr=lr, eps=eps, weight_decay=wd, mode=oracle.ADAM_L2))
    gp = synth.bf16_bits_to_f32(g).astype(np.float64) + wd * th0.astype(np.float64)
    exp = th0.astype(np.float64) - lr * gp / (np.abs(gp) + eps)
    assert np.all(np.abs(r.p32 - exp) <= f32ulp(exp))


def test_constant_grad_bias_correction():
    """g == c for all t: m_hat = c, v_hat = c^2 exactly, so with wd = 0
    theta_t = theta0 - t * lr * c / (|c| + eps)."""
    vals = np.array([2.0 ** -10, -(2.0 ** -20), 3 * 2.0 ** -15, -(2.0 ** -8)], np.float32)
    g = g_bits(vals)
    th0 = np.array([0.01, -0.02, 0.03, 0.0], F32)
    lr, eps, T = 1e-3, 1e-8, 10
    r = run_steps(th0, [g] * T, dict(lr=lr, eps=eps, weight_decay=0.0))
    c = vals.astype(np.float64)
    exp = th0.astype(np.float64) - T * lr * c / (np.abs(c) + eps)
    # T roundings of fp32 storage, each <= half an ulp of a value <= |theta0| + T lr
    assert np.all(np.abs(r.p32 - exp) <= T * f32ulp(np.abs(th0) + T * lr))
    m_exp = c * (1 - 0.9 ** T)
    assert np.all(np.abs(r.m32 - m_exp) <= T * f32ulp(m_exp))


def test_zero_grad_decay():
    n = 1000
    th0 = synth.theta0(n, block=7)
    zero = np.zeros(n, np.uint16)
    lr, wd, T = 1e-3, 1e-2, 10
    r = run_steps(th0, [zero] * T, dict(lr=lr, weight_decay=wd))
    exp = th0.astype(np.float64) * (1 - lr * wd) ** T
    assert np.all(r.m32 == 0) and np.all(r.v32 == 0)
    assert np.all(np.abs(r.p32 - exp) <= T * f32ulp(exp))


def test_beta_zero_is_sign_descent():
    n = 512
    lr, eps = 1e-3, 1e-8
    hp = dict(lr=lr, eps=eps, weight_decay=0.0, beta1=0.0, beta2=0.0)
    th = synth.theta0(n, block=2)
    r = oracle.Range.fresh(th, 1)
    for t in range(1, 6):
        g = synth.grad16(n, step=t, block=2)
        prev = r.p32.astype(np.float64)
        oracle.adam_range(r, g, oracle.hparams(step=t, **hp))
        gd = synth.bf16_bits_to_f32(g).astype(np.float64)
        exp = prev - lr * gd / (np.abs(gd) + eps)
        assert np.all(np.abs(r.p32 - exp) <= f32ulp(exp))


def test_sign_and_scale_symmetry():
    n = 4096
    th0 = np.zeros(n, F32)
    gs = [synth.grad16(n, step=t, block=5) for t in range(1, 6)]
    neg = [g ^ np.uint16(0x8000) for g in gs]
    sc = [(g.astype(np.int32) + np.where((g & 0x7FFF) != 0, 3 << 7, 0)).astype(np.uint16) for g in gs]
    base = run_steps(th0, gs, dict(weight_decay=0.0))
    rn = run_steps(th0, neg, dict(weight_decay=0.0))
    assert np.array_equal(rn.p32, -base.p32)
    # x8 scale (exponent + 3) with eps = 0 leaves every update unchanged
    b0 = run_steps(th0, gs, dict(weight_decay=0.0, eps=0.0))
    b8 = run_steps(th0, sc, dict(weight_decay=0.0, eps=0.0))
    nz = ~np.isnan(b0.p32)
    assert np.array_equal(b0.p32[nz], b8.p32[nz])


# ----------------------------------------------------------- library routines
def _torch_run(th0, grads, mode, lr=1e-3, wd=1e-2, eps=1e-8, betas=(0.9, 0.999),
               clip=0.0):
    p = torch.nn.Parameter(torch.from_numpy(th0.astype(np.float64)))
    cls = torch.optim.AdamW if mode == oracle.ADAMW else torch.optim.Adam
    opt = cls([p], lr=lr, betas=betas, eps=eps, weight_decay=wd, foreach=False)
    coefs = []
    for g in grads:
        p.grad = torch.from_numpy(synth.bf16_bits_to_f32(g).astype(np.float64))
        if clip > 0:
            tn = torch.nn.utils.clip_grad_norm_([p], clip, foreach=False)
            coefs.append(float(tn))
        opt.step()
        with torch.no_grad():  # emulate fp32 storage of P32 / OS32
            p.copy_(p.float().double())
            st = opt.state[p]
            st["exp_avg"].copy_(st["exp_avg"].float().double())
            st["exp_avg_sq"].copy_(st["exp_avg_sq"].float().double())
    st = opt.state[p]
    return (p.detach().float().numpy(), st["exp_avg"].float().numpy(),
            st["exp_avg_sq"].float().numpy(), coefs)


@pytest.mark.parametrize("mode", [oracle.ADAMW, oracle.ADAM_L2])
def test_vs_torch_optim_float64(mode):
    n, T = 200_000, 10
    th0 = synth.theta0(n, block=11)
    grads = [synth.grad16(n, step=t, block=11) for t in range(1, T + 1)]
    r = run_steps(th0, grads, dict(mode=mode))
    tp, tm, tv, _ = _torch_run(th0, grads, mode)
    got = dict(p32=tp, m32=tm, v32=tv, p16=oracle.bf16_rne(tp))
    rep = check_range(got, r, tol=1e-6, what="torch")
    assert rep["v_rel"] < 1e-6


def test_vs_torch_gaussian_grads():
    n, T = 100_000, 10
    th0 = synth.theta0(n, block=12)
    grads = [synth.grad16_normal(n, 1e-3, seed=100 + t) for t in range(T)]
    r = run_steps(th0, grads, {})
    tp, tm, tv, _ = _torch_run(th0, grads, oracle.ADAMW)
    check_range(dict(p32=tp, m32=tm, v32=tv, p16=oracle.bf16_rne(tp)), r, tol=1e-6)


def test_clip_vs_torch_clip_grad_norm():
    n, T, max_norm = 50_000, 4, 1e-3
    th0 = synth.theta0(n, block=13)
    grads = [synth.grad16(n, step=t, block=13) for t in range(1, T + 1)]
    r = oracle.Range.fresh(th0)
    for t, g in enumerate(grads, start=1):
        S, coef = oracle.adam_step([r], [g], oracle.hparams(step=t), max_grad_norm=max_norm)
        tn = torch.linalg.vector_norm(torch.from_numpy(synth.bf16_bits_to_f32(g).astype(np.float64)))
        # both sums are double; orders differ (torch is blocked): bound n * 2^-53
        assert abs(math.sqrt(S) - float(tn)) <= n * 2.0 ** -53 * float(tn)
        assert coef < 1.0
    tp, tm, tv, norms = _torch_run(th0, grads, oracle.ADAMW, clip=max_norm)
    check_range(dict(p32=tp, m32=tm, v32=tv, p16=oracle.bf16_rne(tp)), r, tol=1e-6)


def test_clip_coef_definition():
    assert oracle.clip_coef(4.0, 1.0) == pytest.approx(1.0 / (2.0 + 1e-6), rel=1e-15)
    assert oracle.clip_coef(1e-12, 1.0) == 1.0          # clamped at 1
    assert oracle.clip_coef(0.0, 1.0) == 1.0
    assert math.isnan(oracle.clip_coef(float("nan"), 1.0))


def test_sumsq_exact_small():
    from fractions import Fraction
    g = synth.grad16(3000, step=4, block=9)
    exact = sum(Fraction(float(x)) ** 2 for x in synth.bf16_bits_to_f32(g))
    S = oracle.grad_sumsq(g)
    assert abs(Fraction(S) - exact) <= Fraction(1, 10 ** 15) * exact
    # continuing a running sum == sum over the concatenation
    assert oracle.grad_sumsq(g[1000:], oracle.grad_sumsq(g[:1000])) == S


# ------------------------------------------------------------------ brute force
def test_mpmath_trace():
    mp = pytest.importorskip("mpmath")
    mp.mp.dps = 50
    n, T = 12, 10
    lr, b1, b2, eps, wd = 1e-3, 0.9, 0.999, 1e-8, 1e-2
    th = synth.theta0(n, block=21).astype(np.float64)
    grads = [synth.bf16_bits_to_f32(synth.grad16(n, step=t, block=21)).astype(np.float64)
             for t in range(1, T + 1)]
    p, m, v = th.copy(), np.zeros(n), np.zeros(n)
    P = [mp.mpf(float(x)) for x in th]
    M = [mp.mpf(0)] * n
    V = [mp.mpf(0)] * n
    Mbar = [mp.mpf(0)] * n
    L, B1, B2, E, W = (mp.mpf(x) for x in (lr, b1, b2, eps, wd))
    for t in range(1, T + 1):
        oracle.adam_range_f64(p, m, v, grads[t - 1], oracle.hparams(step=t))
        for i in range(n):
            gi = mp.mpf(float(grads[t - 1][i]))
            P[i] = P[i] * (1 - L * W)
            M[i] = B1 * M[i] + (1 - B1) * gi
            Mbar[i] = B1 * Mbar[i] + (1 - B1) * abs(gi)
            V[i] = B2 * V[i] + (1 - B2) * gi * gi
            mh = M[i] / (1 - B1 ** t)
            vh = V[i] / (1 - B2 ** t)
            P[i] = P[i] - L * mh / (mp.sqrt(vh) + E)
        for i in range(n):
            scale = abs(float(th[i])) + t * lr
            assert abs(p[i] - float(P[i])) <= 1e-14 * scale
            assert abs(m[i] - float(M[i])) <= 1e-14 * float(Mbar[i])
            assert abs(v[i] - float(V[i])) <= 1e-14 * float(V[i]) + 1e-300


# ---------------------------------------------------------------- bf16 rounding
def test_bf16_rne_special_values():
    cases = [(1.0, 0x3F80), (-2.0, 0xC000), (0.0, 0x0000), (-0.0, 0x8000),
             (float("inf"), 0x7F80), (float("-inf"), 0xFF80),
             (3.3895313892515355e38, 0x7F7F),           # largest finite bf16
             (3.4028234663852886e38, 0x7F80)]           # FLT_MAX rounds up to Inf
    for x, b in cases:
        assert int(oracle.bf16_rne(np.array([x], F32))[0]) == b, x
    # ties: 1 + 2^-8 (exactly halfway between 1 and 1+2^-7) -> even (1.0)
    t = np.array([1 + 2.0 ** -8, 1 + 3 * 2.0 ** -8], F32)
    assert list(oracle.bf16_rne(t)) == [0x3F80, 0x3F82]
    nan = oracle.bf16_rne(np.array([float("nan"), -float("nan")], F32))
    assert list(nan) == [0x7FC0, 0xFFC0]


@pytest.mark.slow
def test_bf16_rne_exhaustive_vs_torch():
    """All 2^32 fp32 patterns: oracle RNE == torch's CPU cast (NaN: both NaN)."""
    chunk = 1 << 26
    for start in range(0, 1 << 32, chunk):
        u = np.arange(start, start + chunk, dtype=np.uint64).astype(np.uint32)
        x = u.view(np.float32)
        mine = oracle.bf16_rne(x)
        ref = torch.from_numpy(x).to(torch.bfloat16).view(torch.int16).numpy().view(np.uint16)
        isn = np.isnan(x)
        if not np.array_equal(mine[~isn], ref[~isn]):
            bad = np.flatnonzero(mine != ref)[0]
            raise AssertionError(f"pattern {u[bad]:#010x}: {mine[bad]:#06x} vs {ref[bad]:#06x}")
        assert np.all((mine[isn] & 0x7FFF) > 0x7F80)


def test_oracle_regression_digests():
    """The oracle's C1 outputs are unchanged since tests/golden/ was written
    (tests/golden/make_golden.py; regenerate only with a cited reason)."""
    import json
    import os
    import importlib.util
    here = os.path.join(os.path.dirname(os.path.abspath(__file__)), "golden")
    spec = importlib.util.spec_from_file_location("make_golden", os.path.join(here, "make_golden.py"))
    mg = importlib.util.module_from_spec(spec)
    spec.loader.exec_module(mg)
    gold = json.load(open(os.path.join(here, "oracle_digests.json")))
    assert mg.digests() == gold["sha256"]
    assert mg.scale_digests() == gold["sha256_scales"]   # theta_bar / m_bar (R13)


# ------------------------------------- data-parallel gradient reduction (R17)
def _rank_grads(n, N, step=1, block=21):
    return [synth.grad16(n, step=step, block=block + 100 * q) for q in range(N)]


@pytest.mark.parametrize("N,scale", [(2, 0.5), (4, 0.25), (3, 1.0 / 3.0), (8, 1.0)])
def test_dp_reduce_is_the_exact_sum(N, scale):
    """scale * sum_q g_q: for these inputs (exponents within 24 binades) the
    double sum is exact, so it must equal math.fsum (the correctly rounded
    sum) times scale, element by element."""
    n = 3000
    gq = _rank_grads(n, N)
    got = oracle.reduce_grads(gq, scale)
    vals = np.stack([synth.bf16_bits_to_f32(g).astype(np.float64) for g in gq])
    exp = np.array([math.fsum(vals[:, i]) for i in range(n)]) * scale
    assert np.array_equal(got, exp)


@pytest.mark.parametrize("N", [1, 2, 4, 8])
def test_dp_identical_replicas_reduce_to_the_plain_step(N):
    """N identical replicas averaged (scale 1/N, exact) give exactly the
    single-gradient update -- the special case that is the pinned step."""
    n, T = 5000, 3
    th0 = synth.theta0(n, block=22)
    a = oracle.Range.fresh(th0)
    b = oracle.Range.fresh(th0)
    for t in range(1, T + 1):
        g = synth.grad16(n, step=t, block=22)
        hp = oracle.hparams(step=t)
        oracle.adam_range(a, g, hp)
        oracle.adam_range_gd(b, oracle.reduce_grads([g] * N, 1.0 / N), hp)
    for k in ("p32", "m32", "v32", "p16", "theta_bar", "m_bar"):
        assert np.array_equal(getattr(a, k), getattr(b, k)), k


@pytest.mark.parametrize("clip", [0.0, 1e-3])
def test_dp_vs_torch_mean_of_replica_grads(clip):
    """torch.optim.AdamW (float64, fp32 storage emulated) on p.grad = the
    mean of N ranks' grads (what DDP hands the optimizer), optionally
    clip_grad_norm_ on that mean: R13 bound 1e-6."""
    n, T, N = 20_000, 5, 4
    th0 = synth.theta0(n, block=23)
    steps = [_rank_grads(n, N, step=t, block=23) for t in range(1, T + 1)]
    r = oracle.Range.fresh(th0)
    p = torch.nn.Parameter(torch.from_numpy(th0.astype(np.float64)))
    opt = torch.optim.AdamW([p], lr=1e-3, weight_decay=1e-2, foreach=False)
    for t, gq in enumerate(steps, start=1):
        S, coef = oracle.adam_step_dp([r], [gq], 1.0 / N, oracle.hparams(step=t), max_grad_norm=clip)
        mean = sum(torch.from_numpy(synth.bf16_bits_to_f32(g).astype(np.float64)) for g in gq) / N
        p.grad = mean
        if clip > 0:
            tn = float(torch.nn.utils.clip_grad_norm_([p], clip, foreach=False))
            assert abs(math.sqrt(S) - tn) <= n * 2.0 ** -53 * tn
            assert coef < 1.0
        opt.step()
        with torch.no_grad():
            p.copy_(p.float().double())
            st = opt.state[p]
            st["exp_avg"].copy_(st["exp_avg"].float().double())
            st["exp_avg_sq"].copy_(st["exp_avg_sq"].float().double())
    st = opt.state[p]
    tp = p.detach().float().numpy()
    check_range(dict(p32=tp, m32=st["exp_avg"].float().numpy(), v32=st["exp_avg_sq"].float().numpy(),
                     p16=oracle.bf16_rne(tp)), r, tol=1e-6, what="dp torch")


def test_dp_sumsq_exact_small():
    from fractions import Fraction
    gd = oracle.reduce_grads(_rank_grads(2000, 3, block=24), 1.0 / 3.0)
    exact = sum(Fraction(float(x)) ** 2 for x in gd)
    # each square and each partial sum rounds once: |err| <= 2n * 2^-53 * S
    assert abs(Fraction(oracle.grad_sumsq_d(gd)) - exact) <= Fraction(2 * gd.size, 2 ** 53) * exact
