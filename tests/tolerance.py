"""Condition-aware parity bounds (reading R13).

BASELINE.json's north star asks for "max relative error 1e-5" on the fp32
states and "bf16 within 1 ulp".  Literally these cannot hold where theta or m
cross zero by cancellation, so every bound is taken relative to the scale the
oracle tracks in double beside its result:

  |m - m_ref|         <= tol * m_bar
  |theta - theta_ref| <= tol * theta_bar
  |v - v_ref|         <= tol * v_ref                (v has no cancellation)
  |val(p) - val(p_ref)| <= one bf16 ulp at theta_bar  (2^(floor(log2 theta_bar) - 7))
  and p == bf16_rne(own fp32 theta) bit for bit (self-consistency).

Where |ref| ~ scale these reduce to the literal criteria.  NaN must match NaN.
"""
from __future__ import annotations

import numpy as np

TOL = 1e-5


def bf16_to_f64(bits: np.ndarray) -> np.ndarray:
    return (np.asarray(bits, np.uint16).astype(np.uint32) << np.uint32(16)).view(np.float32).astype(np.float64)


def bf16_ulp_at(scale: np.ndarray) -> np.ndarray:
    s = np.maximum(np.asarray(scale, np.float64), np.finfo(np.float64).tiny)
    return np.exp2(np.floor(np.log2(s)) - 7.0)


def _nan_ok(a, b):
    an, bn = np.isnan(a), np.isnan(b)
    assert np.array_equal(an, bn), f"NaN pattern differs at {np.flatnonzero(an != bn)[:8]}"
    return ~an


def _absdiff(a, b):
    """|a - b| in float64, 0 where the values are equal (so matching
    infinities compare as equal instead of producing inf - inf = NaN)."""
    a, b = np.asarray(a, np.float64), np.asarray(b, np.float64)
    with np.errstate(invalid="ignore"):
        return np.where(a == b, 0.0, np.abs(a - b))


def check_range(got: dict, ref, tol: float = TOL, own_rne=None, what: str = "") -> dict:
    """got: dict with p32, m32, v32 (float32) and p16 (uint16) from the GPU.
    ref: oracle.Range after the same steps (carries theta_bar and m_bar).
    own_rne: callable float32 -> uint16 bf16 RNE (the oracle's), for the
    self-consistency check.  Returns a report of the worst errors."""
    th, m, v, p = (np.asarray(got[k]) for k in ("p32", "m32", "v32", "p16"))
    th_r, m_r, v_r, p_r = ref.p32, ref.m32, ref.v32, ref.p16
    tbar, mbar = ref.theta_bar, ref.m_bar
    rep = {}

    ok = _nan_ok(th, th_r)
    e_th = _absdiff(th[ok], th_r[ok])
    lim = tol * tbar[ok]
    bad = e_th > lim
    assert not bad.any(), (f"{what} theta: {bad.sum()} elements out of bound; worst "
                           f"{(e_th / np.maximum(tbar[ok], 1e-300)).max():.3e}")
    rep["theta_scaled"] = float((e_th / np.maximum(tbar[ok], 1e-300)).max(initial=0.0))

    ok = _nan_ok(m, m_r)
    e_m = _absdiff(m[ok], m_r[ok])
    bad = e_m > tol * mbar[ok]
    assert not bad.any(), (f"{what} m: {bad.sum()} elements out of bound; worst abs "
                           f"{e_m[bad].max():.3e}")
    rep["m_scaled"] = float((e_m / np.maximum(mbar[ok], 1e-300)).max(initial=0.0))

    ok = _nan_ok(v, v_r)
    e_v = _absdiff(v[ok], v_r[ok])
    bad = e_v > tol * np.abs(v_r[ok].astype(np.float64))
    assert not bad.any(), f"{what} v: {bad.sum()} elements out of bound"
    rep["v_rel"] = float((e_v / np.maximum(np.abs(v_r[ok].astype(np.float64)), 1e-300)).max(initial=0.0))

    pv, pv_r = bf16_to_f64(p), bf16_to_f64(p_r)
    ok = _nan_ok(pv, pv_r)
    e_p = _absdiff(pv[ok], pv_r[ok])
    bad = e_p > bf16_ulp_at(tbar[ok])
    assert not bad.any(), f"{what} p16: {bad.sum()} elements beyond 1 bf16 ulp at scale"
    rep["p16_ulps_at_scale"] = float((e_p / bf16_ulp_at(tbar[ok])).max(initial=0.0))
    rep["p16_bits_differ"] = int((p != p_r).sum())
    if own_rne is not None:
        mine = own_rne(th.astype(np.float32))
        nn = ~np.isnan(th)
        assert np.array_equal(mine[nn], p[nn]), f"{what} p16 != bf16_rne(own theta)"

    # literal criteria over well-conditioned elements (|ref| >= 0.1 * scale)
    wc = np.abs(th_r.astype(np.float64)) >= 0.1 * tbar
    if wc.any():
        rep["theta_literal_rel_wc"] = float((np.abs(th[wc].astype(np.float64) - th_r[wc])
                                             / np.abs(th_r[wc].astype(np.float64))).max())
    rep["excluded_theta"] = int((~wc).sum())
    return rep
