"""Mutation check of the oracle's pins (CPU).

Each mutant is ratel_oracle.c with ONE plausible mistake (a dropped term, a
wrong sign, a wrong index/power, a transposed operand, the other eps reading,
truncating instead of rounding), compiled to a temp dir.  The pins of
tests/test_oracle_pins.py are re-run against it in a compact form: every
mutant must be caught by at least one pin, otherwise the pins would not be
pinning that part of the oracle.
"""
import ctypes
import math
import os
import subprocess

import numpy as np
import pytest
import torch

import oracle
import synth

SRC = os.path.join(os.path.dirname(oracle.__file__), "ratel_oracle.c")

MUTANTS = {
    "eps_inside_sqrt": ("(sqrt(vv / bc2) + hp->eps)", "sqrt(vv / bc2 + hp->eps)"),
    "kingma_efficient_eps": ("(sqrt(vv / bc2) + hp->eps)", "(sqrt(vv / bc2) + hp->eps / sqrt(1.0 - hp->beta2))"),
    "bias1_uses_t_minus_1": ("double bc1 = 1.0 - pow(hp->beta1, t);", "double bc1 = 1.0 - pow(hp->beta1, t - 1.0 + 1e-300);"),
    "no_bias2": ("double bc2 = 1.0 - pow(hp->beta2, t);", "double bc2 = 1.0;"),
    "beta2_swapped": ("double vv = hp->beta2 * (*v) + (1.0 - hp->beta2) * g * g;",
                      "double vv = (1.0 - hp->beta2) * (*v) + hp->beta2 * g * g;"),
    "m_drops_1_minus_beta1": ("(1.0 - hp->beta1) * g;", "g;"),
    "wd_sign": ("th = th * (1.0 - hp->lr * hp->weight_decay);", "th = th * (1.0 + hp->lr * hp->weight_decay);"),
    "wd_without_lr": ("th = th * (1.0 - hp->lr * hp->weight_decay);", "th = th * (1.0 - hp->weight_decay);"),
    "l2_sign": ("g = g + hp->weight_decay * th;", "g = g - hp->weight_decay * th;"),
    "update_sign": ("th = th - delta;", "th = th + delta;"),
    "bf16_truncates": ("if (rem > 0x8000u) return (uint16_t)(lo + 1);", "if (rem > 0xFFFFu) return (uint16_t)(lo + 1);"),
    "bf16_ties_away": ("return (lo & 1u) ? (uint16_t)(lo + 1) : lo;", "return (uint16_t)(lo + 1);"),
    "p16_from_wrong_array": ("p16[i] = oracle_bf16_rne(p32[i]);", "p16[i] = oracle_bf16_rne(m32[i]);"),
    "clip_not_clamped": ("return (c < 1.0 || isnan(c)) ? c : 1.0;", "return c;"),
    "clip_norm_squared": ("double c = max_norm / (sqrt(sumsq) + 1e-6);", "double c = max_norm / (sumsq + 1e-6);"),
    "sumsq_abs": ("s += g * g;", "s += fabs(g);"),
    # data-parallel gradient reduction (R17)
    "dp_no_scale": ("out[i] = scale * s;", "out[i] = s;"),
    "dp_first_rank_only": ("for (int q = 0; q < nq; ++q)", "for (int q = 0; q < 1; ++q)"),
    "dp_drops_last_rank": ("for (int q = 0; q < nq; ++q)", "for (int q = 0; q < nq - 1; ++q)"),
    "dp_ignores_clip_coef": ("double g = gd[i] * coef;", "double g = gd[i];"),
    "dp_sumsq_abs": ("s += g[i] * g[i];", "s += fabs(g[i]);"),
    # tolerance scales theta_bar / m_bar (R13): every parity bound divides by them
    "theta_bar_x2": ("theta_bar[i] = d * theta_bar[i] + absdelta;",
                     "theta_bar[i] = 2.0 * (d * theta_bar[i] + absdelta);"),
    "theta_bar_x100_delta": ("theta_bar[i] = d * theta_bar[i] + absdelta;",
                             "theta_bar[i] = d * theta_bar[i] + 100.0 * absdelta;"),
    "theta_bar_no_decay": ("double d = (apply_wd && hp->mode == ORACLE_ADAMW) ? (1.0 - hp->lr * hp->weight_decay) : 1.0;",
                           "double d = 1.0;"),
    "theta_bar_decay_in_l2_mode": ("double d = (apply_wd && hp->mode == ORACLE_ADAMW) ? (1.0 - hp->lr * hp->weight_decay) : 1.0;",
                                   "double d = apply_wd ? (1.0 - hp->lr * hp->weight_decay) : 1.0;"),
    "theta_bar_drops_delta": ("theta_bar[i] = d * theta_bar[i] + absdelta;", "theta_bar[i] = d * theta_bar[i];"),
    "theta_bar_signed_delta": ("return fabs(delta);", "return delta;"),
    "m_bar_no_beta1_decay": ("m_bar[i] = hp->beta1 * m_bar[i] + (1.0 - hp->beta1) * fabs(g_used);",
                             "m_bar[i] = m_bar[i] + (1.0 - hp->beta1) * fabs(g_used);"),
    "m_bar_signed_g": ("(1.0 - hp->beta1) * fabs(g_used);", "(1.0 - hp->beta1) * g_used;"),
    "m_bar_drops_1_minus_beta1": ("(1.0 - hp->beta1) * fabs(g_used);", "fabs(g_used);"),
    "m_bar_uses_beta2": ("m_bar[i] = hp->beta1 * m_bar[i] + (1.0 - hp->beta1) * fabs(g_used);",
                         "m_bar[i] = hp->beta2 * m_bar[i] + (1.0 - hp->beta2) * fabs(g_used);"),
    "scales_ignore_clip": ("update_scales(i, gu, ad, apply_wd, hp, theta_bar, m_bar);\n  }\n}\n\n/* Same update",
                           "update_scales(i, gu / coef, ad, apply_wd, hp, theta_bar, m_bar);\n  }\n}\n\n/* Same update"),
    "m_bar_l2_from_raw_grad": [("double th = *theta;", "double th = *theta;\n  *g_used = g;"),
                               ("  *g_used = g;\n  return fabs(delta);", "  return fabs(delta);")],
}


def _build_mutant(tmp_path, name, edits):
    """edits: one (old, new) pair or a list of them, applied in order."""
    src = open(SRC).read()
    for old, new in ([edits] if isinstance(edits, tuple) else edits):
        assert src.count(old) >= 1, (name, old)  # every occurrence is mutated
        src = src.replace(old, new)
    path = tmp_path / f"{name}.c"
    path.write_text(src)
    so = tmp_path / f"lib{name}.so"
    subprocess.check_call(["gcc", "-O2", "-ffp-contract=off", "-fopenmp", "-fPIC", "-shared", "-std=c11",
                           "-o", str(so), str(path), "-lm"])
    return str(so)


def _with_lib(path):
    """Point the oracle wrapper at another build for the duration of a check."""
    saved = oracle._lib
    oracle._lib = None
    real_build = oracle.build
    oracle.build = lambda force=False: path
    try:
        oracle.lib()
    finally:
        oracle.build = real_build
    return saved


def _pins_pass():
    """Compact versions of the oracle pins; True iff all hold."""
    f32ulp = lambda x: np.spacing(np.abs(np.float32(x))).astype(np.float64)
    lr, eps = 1e-3, 1e-8
    try:
        # step-1 closed form, AdamW with decay, and the eps separator
        n = 2048
        th0 = synth.theta0(n, block=3)
        g = synth.grad16(n, step=1, block=3)
        for wd in (0.0, 1e-2):
            r = oracle.Range.fresh(th0)
            oracle.adam_range(r, g, oracle.hparams(step=1, weight_decay=wd))
            gd = synth.bf16_bits_to_f32(g).astype(np.float64)
            exp = th0.astype(np.float64) * (1 - lr * wd) - lr * gd / (np.abs(gd) + eps)
            if not np.all(np.abs(r.p32 - exp) <= f32ulp(exp)):
                return False
        # Adam-L2 step 1
        r = oracle.Range.fresh(th0)
        oracle.adam_range(r, g, oracle.hparams(step=1, mode=oracle.ADAM_L2))
        gp = synth.bf16_bits_to_f32(g).astype(np.float64) + 1e-2 * th0.astype(np.float64)
        exp = th0.astype(np.float64) - lr * gp / (np.abs(gp) + eps)
        if not np.all(np.abs(r.p32 - exp) <= f32ulp(exp)):
            return False
        # constant gradient over 10 steps (bias corrections at every t)
        vals = np.array([2.0 ** -10, -(2.0 ** -20), 3 * 2.0 ** -15, -(2.0 ** -8)], np.float32)
        cb = (vals.view(np.uint32) >> 16).astype(np.uint16)
        r = oracle.Range.fresh(np.array([0.01, -0.02, 0.03, 0.0], np.float32))
        for t in range(1, 11):
            oracle.adam_range(r, cb, oracle.hparams(step=t, weight_decay=0.0))
        exp = np.array([0.01, -0.02, 0.03, 0.0]) - 10 * lr * vals / (np.abs(vals.astype(np.float64)) + eps)
        if not np.all(np.abs(r.p32 - exp) <= 10 * f32ulp(np.abs(exp) + 10 * lr)):
            return False
        # tolerance scales (tests/test_oracle_scale_pins.py): step-1 closed forms, AdamW and Adam-L2
        for mode, wd in ((oracle.ADAMW, 1e-2), (oracle.ADAM_L2, 1e-2)):
            r = oracle.Range.fresh(th0)
            oracle.adam_range(r, g, oracle.hparams(step=1, weight_decay=wd, mode=mode))
            gu = synth.bf16_bits_to_f32(g).astype(np.float64)
            d = 1 - lr * wd
            if mode == oracle.ADAM_L2:
                gu, d = gu + wd * th0.astype(np.float64), 1.0
            if not np.all(np.abs(r.m_bar - 0.1 * np.abs(gu)) <= 1e-15 * np.abs(gu)):
                return False
            exp = d * np.abs(th0.astype(np.float64)) + lr * np.abs(gu) / (np.abs(gu) + eps)
            if not np.all(np.abs(r.theta_bar - exp) <= 2.0 ** -21 * exp):
                return False
        # scales under a constant gradient: m_bar = |c|(1-b1^t), theta_bar = |theta0| + t lr |c|/(|c|+eps)
        vals = np.array([2.0 ** -10, -(2.0 ** -20), 3 * 2.0 ** -15, -(2.0 ** -8)], np.float32)
        cb = (vals.view(np.uint32) >> 16).astype(np.uint16)
        r = oracle.Range.fresh(np.array([0.01, -0.02, 0.03, 0.0], np.float32))
        for t in range(1, 6):
            oracle.adam_range(r, cb, oracle.hparams(step=t, weight_decay=0.0))
        c = np.abs(vals.astype(np.float64))
        if not np.all(np.abs(r.m_bar - c * (1 - 0.9 ** 5)) <= 1e-14 * c):
            return False
        exp = np.array([0.01, 0.02, 0.03, 0.0], np.float32).astype(np.float64) + 5 * lr * c / (c + eps)
        if not np.all(np.abs(r.theta_bar - exp) <= 2.0 ** -18 * exp):
            return False
        # scales under the clip: built from the clipped gradient coef * g
        r = oracle.Range.fresh(th0)
        _, coef = oracle.adam_step([r], [g], oracle.hparams(step=1), max_grad_norm=1e-4)
        gp = coef * synth.bf16_bits_to_f32(g).astype(np.float64)
        if not (coef < 1 and np.all(np.abs(r.m_bar - 0.1 * np.abs(gp)) <= 1e-12 * np.abs(gp))):
            return False
        # torch.optim.AdamW, 10 steps, fp32 storage emulated (R13 bound 1e-6)
        from tests.tolerance import check_range
        from tests.test_oracle_pins import _torch_run
        n, T = 20_000, 6
        th0 = synth.theta0(n, block=11)
        grads = [synth.grad16(n, step=t, block=11) for t in range(1, T + 1)]
        r = oracle.Range.fresh(th0)
        for t, gg in enumerate(grads, start=1):
            oracle.adam_range(r, gg, oracle.hparams(step=t))
        tp, tm, tv, _ = _torch_run(th0, grads, oracle.ADAMW)
        check_range(dict(p32=tp, m32=tm, v32=tv, p16=oracle.bf16_rne(tp)), r, tol=1e-6)
        # clip vs torch clip_grad_norm_
        S = oracle.grad_sumsq(grads[0])
        tn = float(torch.linalg.vector_norm(torch.from_numpy(synth.bf16_bits_to_f32(grads[0]).astype(np.float64))))
        if abs(math.sqrt(S) - tn) > 1e-12 * tn:
            return False
        if oracle.clip_coef(1e-12, 1.0) != 1.0 or abs(oracle.clip_coef(4.0, 1.0) - 1 / (2 + 1e-6)) > 1e-15:
            return False
        # bf16 rounding against torch's cast on random patterns + all ties
        u = np.random.default_rng(0).integers(0, 2 ** 32, 1 << 18, dtype=np.uint64).astype(np.uint32)
        ties = ((np.arange(1 << 16, dtype=np.uint32) << 16) | 0x8000).astype(np.uint32)
        x = np.concatenate([u, ties]).view(np.float32)
        x = x[np.isfinite(x)]
        mine = oracle.bf16_rne(x)
        ref = torch.from_numpy(x).to(torch.bfloat16).view(torch.int16).numpy().view(np.uint16)
        if not np.array_equal(mine, ref):
            return False
        # no staleness: P16 == bf16_rne(stored P32)
        if not np.array_equal(r.p16, oracle.bf16_rne(r.p32)):
            return False
        # data-parallel reduction: exact sum x scale, then torch AdamW + clip on the mean
        N, n = 3, 4000
        gq = [synth.grad16(n, step=1, block=31 + 100 * q) for q in range(N)]
        vals = np.stack([synth.bf16_bits_to_f32(g).astype(np.float64) for g in gq])
        if not np.array_equal(oracle.reduce_grads(gq, 0.5), np.array([math.fsum(vals[:, i]) for i in range(n)]) * 0.5):
            return False
        th0 = synth.theta0(n, block=31)
        r = oracle.Range.fresh(th0)
        p = torch.nn.Parameter(torch.from_numpy(th0.astype(np.float64)))
        opt = torch.optim.AdamW([p], lr=lr, weight_decay=1e-2, foreach=False)
        for t in (1, 2):
            gq = [synth.grad16(n, step=t, block=31 + 100 * q) for q in range(N)]
            S, _ = oracle.adam_step_dp([r], [gq], 1.0 / N, oracle.hparams(step=t), max_grad_norm=1e-4)
            p.grad = sum(torch.from_numpy(synth.bf16_bits_to_f32(g).astype(np.float64)) for g in gq) / N
            tn = float(torch.nn.utils.clip_grad_norm_([p], 1e-4, foreach=False))
            if abs(math.sqrt(S) - tn) > n * 2.0 ** -53 * tn:
                return False
            opt.step()
            with torch.no_grad():
                p.copy_(p.float().double())
                st = opt.state[p]
                st["exp_avg"].copy_(st["exp_avg"].float().double())
                st["exp_avg_sq"].copy_(st["exp_avg_sq"].float().double())
        st = opt.state[p]
        tp = p.detach().float().numpy()
        check_range(dict(p32=tp, m32=st["exp_avg"].float().numpy(), v32=st["exp_avg_sq"].float().numpy(),
                         p16=oracle.bf16_rne(tp)), r, tol=1e-6)
    except AssertionError:
        return False
    return True


def test_unmutated_oracle_passes_the_compact_pins():
    assert _pins_pass()


@pytest.mark.parametrize("name", sorted(MUTANTS))
def test_every_mutant_is_caught(tmp_path, name):
    so = _build_mutant(tmp_path, name, MUTANTS[name])
    saved = _with_lib(so)
    try:
        assert not _pins_pass(), f"mutant {name} survived the pins"
    finally:
        oracle._lib = saved
