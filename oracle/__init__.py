"""CPU oracle for the Ratel AGO AdamW step -- TEST INFRASTRUCTURE ONLY.

Only tests/, __graft_entry__.smoke() and bench.py's cpu_baseline leg (and
`bench.py --impl reference`) may import this package.  The product library
(paper_conf_icde_liaosyxcyww25_b200) never imports it and never links it.

Thin ctypes wrapper over ``ratel_oracle.c`` (see that file's header for the
update it computes and the PAPER.md passages it follows).  The wrapper only
marshals numpy arrays; every step of the arithmetic is in the C file.
"""
from __future__ import annotations

import ctypes
import os
import subprocess
from dataclasses import dataclass, field

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SRC = os.path.join(_HERE, "ratel_oracle.c")
_LIB = os.path.join(_HERE, "liboracle.so")

ADAMW = 0
ADAM_L2 = 1


class HParams(ctypes.Structure):
    _fields_ = [
        ("lr", ctypes.c_double),
        ("beta1", ctypes.c_double),
        ("beta2", ctypes.c_double),
        ("eps", ctypes.c_double),
        ("weight_decay", ctypes.c_double),
        ("step", ctypes.c_int64),
        ("mode", ctypes.c_int),
    ]


def build(force: bool = False) -> str:
    """Compile the oracle with gcc (-O2, no FMA contraction, no fast-math)."""
    if force or not os.path.exists(_LIB) or os.path.getmtime(_LIB) < os.path.getmtime(_SRC):
        tmp = _LIB + f".tmp{os.getpid()}"
        subprocess.check_call(
            ["gcc", "-O2", "-ffp-contract=off", "-fno-fast-math", "-fopenmp", "-fPIC",
             "-shared", "-std=c11", "-o", tmp, _SRC, "-lm"])
        os.replace(tmp, _LIB)
    return _LIB


_lib = None


def lib():
    global _lib
    if _lib is None:
        _lib = ctypes.CDLL(build())
        P = ctypes.c_void_p
        _lib.oracle_bf16_to_double.argtypes = [ctypes.c_uint16]
        _lib.oracle_bf16_to_double.restype = ctypes.c_double
        _lib.oracle_bf16_rne.argtypes = [ctypes.c_float]
        _lib.oracle_bf16_rne.restype = ctypes.c_uint16
        _lib.oracle_bf16_rne_array.argtypes = [P, P, ctypes.c_size_t]
        _lib.oracle_adam_range.argtypes = [ctypes.c_size_t, P, ctypes.c_double, ctypes.c_int,
                                           ctypes.POINTER(HParams), P, P, P, P, P, P, ctypes.c_int]
        _lib.oracle_adam_range_f64.argtypes = [ctypes.c_size_t, P, ctypes.c_double, ctypes.c_int,
                                               ctypes.POINTER(HParams), P, P, P]
        _lib.oracle_grad_sumsq.argtypes = [P, ctypes.c_size_t, ctypes.c_double]
        _lib.oracle_grad_sumsq.restype = ctypes.c_double
        _lib.oracle_clip_coef.argtypes = [ctypes.c_double, ctypes.c_double]
        _lib.oracle_clip_coef.restype = ctypes.c_double
        _lib.oracle_reduce_grads.argtypes = [ctypes.c_size_t, P, ctypes.c_int, ctypes.c_double, P]
        _lib.oracle_adam_range_gd.argtypes = [ctypes.c_size_t, P, ctypes.c_double, ctypes.c_int,
                                              ctypes.POINTER(HParams), P, P, P, P, P, P]
        _lib.oracle_grad_sumsq_d.argtypes = [P, ctypes.c_size_t, ctypes.c_double]
        _lib.oracle_grad_sumsq_d.restype = ctypes.c_double
    return _lib


def _ptr(a):
    return None if a is None else a.ctypes.data_as(ctypes.c_void_p)


def _check(a, dtype, n):
    assert a.dtype == dtype and a.flags.c_contiguous and a.size == n, (a.dtype, a.size, n)


def bf16_rne(x: np.ndarray) -> np.ndarray:
    x = np.ascontiguousarray(x, dtype=np.float32)
    out = np.empty(x.shape, dtype=np.uint16)
    lib().oracle_bf16_rne_array(_ptr(x), _ptr(out), x.size)
    return out


def grad_sumsq(g16: np.ndarray, s0: float = 0.0) -> float:
    g16 = np.ascontiguousarray(g16, dtype=np.uint16)
    return lib().oracle_grad_sumsq(_ptr(g16), g16.size, s0)


def clip_coef(sumsq: float, max_norm: float) -> float:
    return lib().oracle_clip_coef(sumsq, max_norm)


def hparams(lr=1e-3, beta1=0.9, beta2=0.999, eps=1e-8, weight_decay=1e-2, step=1, mode=ADAMW):
    return HParams(lr, beta1, beta2, eps, weight_decay, step, mode)


@dataclass
class Range:
    """One contiguous parameter range: fp32 states, bf16 working copy, scales."""
    p32: np.ndarray
    m32: np.ndarray
    v32: np.ndarray
    p16: np.ndarray
    apply_wd: int = 1
    theta_bar: np.ndarray = field(default=None)
    m_bar: np.ndarray = field(default=None)

    @staticmethod
    def fresh(theta0: np.ndarray, apply_wd: int = 1) -> "Range":
        theta0 = np.ascontiguousarray(theta0, dtype=np.float32)
        n = theta0.size
        return Range(theta0.copy(), np.zeros(n, np.float32), np.zeros(n, np.float32),
                     bf16_rne(theta0), apply_wd, np.abs(theta0.astype(np.float64)),
                     np.zeros(n, np.float64))

    def copy(self) -> "Range":
        return Range(self.p32.copy(), self.m32.copy(), self.v32.copy(), self.p16.copy(),
                     self.apply_wd, None if self.theta_bar is None else self.theta_bar.copy(),
                     None if self.m_bar is None else self.m_bar.copy())


def adam_range(r: Range, g16: np.ndarray, hp: HParams, coef: float = 1.0, threads: int = 1) -> None:
    """In-place update of one range (fp32 storage semantics)."""
    n = r.p32.size
    g16 = np.ascontiguousarray(g16, dtype=np.uint16)
    for a, dt in ((r.p32, np.float32), (r.m32, np.float32), (r.v32, np.float32),
                  (r.p16, np.uint16), (g16, np.uint16)):
        _check(a, dt, n)
    for a in (r.theta_bar, r.m_bar):
        if a is not None:
            _check(a, np.float64, n)
    lib().oracle_adam_range(n, _ptr(g16), coef, r.apply_wd, ctypes.byref(hp), _ptr(r.p32),
                            _ptr(r.m32), _ptr(r.v32), _ptr(r.p16), _ptr(r.theta_bar),
                            _ptr(r.m_bar), threads)


def adam_step(ranges, grads, hp: HParams, max_grad_norm: float = 0.0, threads: int = 1):
    """One synchronous step over every range (all blocks): optional global
    clip over all grads (R9), then the per-element update.  Returns
    (sumsq, coef); sumsq is None when clipping is off."""
    S = None
    coef = 1.0
    if max_grad_norm > 0:
        S = 0.0
        for g in grads:  # index order over the concatenation of all ranges
            S = grad_sumsq(g, S)
        coef = clip_coef(S, max_grad_norm)
    for r, g in zip(ranges, grads):
        adam_range(r, g, hp, coef, threads)
    return S, coef


def reduce_grads(g16s, scale: float) -> np.ndarray:
    """Data-parallel gradient of a range: scale * sum over ranks (R17), double."""
    gs = [np.ascontiguousarray(g, dtype=np.uint16) for g in g16s]
    n = gs[0].size
    for g in gs:
        _check(g, np.uint16, n)
    ptrs = (ctypes.c_void_p * len(gs))(*[g.ctypes.data for g in gs])
    out = np.empty(n, np.float64)
    lib().oracle_reduce_grads(n, ptrs, len(gs), scale, _ptr(out))
    return out


def adam_range_gd(r: Range, gd: np.ndarray, hp: HParams, coef: float = 1.0) -> None:
    """In-place update of one range from a double gradient (fp32 storage)."""
    n = r.p32.size
    gd = np.ascontiguousarray(gd, dtype=np.float64)
    _check(gd, np.float64, n)
    lib().oracle_adam_range_gd(n, _ptr(gd), coef, r.apply_wd, ctypes.byref(hp), _ptr(r.p32),
                               _ptr(r.m32), _ptr(r.v32), _ptr(r.p16), _ptr(r.theta_bar), _ptr(r.m_bar))


def grad_sumsq_d(gd: np.ndarray, s0: float = 0.0) -> float:
    gd = np.ascontiguousarray(gd, dtype=np.float64)
    return lib().oracle_grad_sumsq_d(_ptr(gd), gd.size, s0)


def adam_step_dp(ranges, rank_grads, scale: float, hp: HParams, max_grad_norm: float = 0.0):
    """One synchronous step with the data-parallel gradient reduction (R17):
    rank_grads[k] is the list of every rank's bf16 grad of range k.  Returns
    (sumsq, coef) like adam_step."""
    gds = [reduce_grads(gq, scale) for gq in rank_grads]
    S = None
    coef = 1.0
    if max_grad_norm > 0:
        S = 0.0
        for gd in gds:
            S = grad_sumsq_d(gd, S)
        coef = clip_coef(S, max_grad_norm)
    for r, gd in zip(ranges, gds):
        adam_range_gd(r, gd, hp, coef)
    return S, coef


def adam_range_f64(p, m, v, g, hp: HParams, coef: float = 1.0, apply_wd: int = 1):
    """Double-state variant (pins the arithmetic; no fp32 storage)."""
    for a in (p, m, v, g):
        assert a.dtype == np.float64 and a.flags.c_contiguous
    lib().oracle_adam_range_f64(p.size, _ptr(g), coef, apply_wd, ctypes.byref(hp),
                                _ptr(p), _ptr(m), _ptr(v))
