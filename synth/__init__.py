"""Seeded synthetic inputs shared by the oracle side and the CUDA side.

This module holds NONE of the method's arithmetic (no Adam, no bf16 rounding,
no norms). It only turns (seed, tag, step, block, index) into bit patterns.
The CUDA library implements the same counter-based generator in
`paper_conf_icde_liaosyxcyww25_b200/csrc/ratel_gen.cu` (declared in
`include/ratel_gen.h`) so that multi-GB device runs see bit-identical inputs
without a host round trip; `tests/test_gen_gpu.py` checks the two agree bit
for bit.  The recipe is DESIGN.md §"Input recipe" (SURVEY §8(d) "Synthetic
inputs"):

* theta0 (P32 at t=0): uniform in [-0.05, 0.05) built from a 24-bit integer,
  ``float32(u24 - 2^23) * float32(0.05 * 2^-23)`` (one IEEE single multiply),
  the paper "randomly initialize[s] model parameters".
* G16 (bf16 gradients): sign random; 1 % +0, 0.1 % -0; otherwise an exponent
  uniform over [2^-30, 2^-7] and 7 random mantissa bits, i.e. magnitudes
  log-uniform over [2^-30, 2^-6).  About 1/6 of the non-zero magnitudes fall
  at or below eps = 1e-8, exercising the eps term.

Counter-based generator (splitmix64, Steele et al.; constants are the public
splitmix64 ones):

    mix64(z)   = splitmix64 finaliser
    key(seed, tag, step, block) = mix64(mix64(mix64(seed ^ tag*G) ^ step) ^ block)
    draw(key, i) = mix64(key + (i + 1) * G)          # i-th splitmix64 output

with G = 0x9E3779B97F4A7C15 and all arithmetic modulo 2^64.
"""
from __future__ import annotations

import numpy as np

SEED = 0x5EED5EED
GOLDEN = 0x9E3779B97F4A7C15
M1 = 0xBF58476D1CE4E5B9
M2 = 0x94D049BB133111EB
MASK64 = (1 << 64) - 1

TAG_THETA = 1
TAG_GRAD = 2

# 0.05 * 2^-23 as float32: float32(0.05) scaled by an exact power of two.
THETA_SCALE = np.float32(np.float32(0.05) * np.float32(2.0 ** -23))

_CHUNK = 1 << 24


def mix64_int(z: int) -> int:
    """splitmix64 finaliser on a Python int (reference for the vector form)."""
    z &= MASK64
    z = ((z ^ (z >> 30)) * M1) & MASK64
    z = ((z ^ (z >> 27)) * M2) & MASK64
    return z ^ (z >> 31)


def stream_key(seed: int, tag: int, step: int, block: int) -> int:
    k = mix64_int((seed ^ ((tag * GOLDEN) & MASK64)) & MASK64)
    k = mix64_int(k ^ (step & MASK64))
    return mix64_int(k ^ (block & MASK64))


def _mix64_vec(z: np.ndarray) -> np.ndarray:
    z = (z ^ (z >> np.uint64(30))) * np.uint64(M1)
    z = (z ^ (z >> np.uint64(27))) * np.uint64(M2)
    return z ^ (z >> np.uint64(31))


def draws(key: int, idx: np.ndarray) -> np.ndarray:
    """splitmix64 outputs number idx (0-based) of a stream whose state is `key`."""
    idx = np.asarray(idx, dtype=np.uint64)
    with np.errstate(over="ignore"):
        z = np.uint64(key) + (idx + np.uint64(1)) * np.uint64(GOLDEN)
        return _mix64_vec(z)


def _theta_from_draws(r: np.ndarray) -> np.ndarray:
    u = (r >> np.uint64(40)).astype(np.int64) - (1 << 23)
    return u.astype(np.float32) * THETA_SCALE


def _grad_from_draws(r: np.ndarray) -> np.ndarray:
    sel = ((r >> np.uint64(32)) & np.uint64(0xFFFFFFFF)) % np.uint64(1000)
    sign = ((r >> np.uint64(31)) & np.uint64(1)).astype(np.uint16)
    e = (((r >> np.uint64(8)) & np.uint64(0xFF)) % np.uint64(24)).astype(np.uint16)
    mant = (r & np.uint64(0x7F)).astype(np.uint16)
    bits = (sign << np.uint16(15)) | ((np.uint16(97) + e) << np.uint16(7)) | mant
    bits = np.where(sel < 10, np.uint16(0x0000), bits)
    bits = np.where(sel == 10, np.uint16(0x8000), bits)
    return bits.astype(np.uint16)


def _chunked(fn, key: int, start: int, n: int, dtype) -> np.ndarray:
    out = np.empty(n, dtype=dtype)
    for off in range(0, n, _CHUNK):
        m = min(_CHUNK, n - off)
        idx = np.arange(start + off, start + off + m, dtype=np.uint64)
        out[off:off + m] = fn(draws(key, idx))
    return out


def theta0(n: int, block: int = 0, start: int = 0, seed: int = SEED) -> np.ndarray:
    """fp32 initial master weights for elements [start, start+n) of `block`."""
    return _chunked(_theta_from_draws, stream_key(seed, TAG_THETA, 0, block), start, n, np.float32)


def grad16(n: int, step: int, block: int = 0, start: int = 0, seed: int = SEED) -> np.ndarray:
    """bf16 gradient bit patterns (uint16) for elements [start, start+n) of `block` at `step`."""
    return _chunked(_grad_from_draws, stream_key(seed, TAG_GRAD, step, block), start, n, np.uint16)


def theta0_at(idx: np.ndarray, block: int = 0, seed: int = SEED) -> np.ndarray:
    """theta0 at arbitrary (sampled) element indices of `block`."""
    return _theta_from_draws(draws(stream_key(seed, TAG_THETA, 0, block), idx))


def grad16_at(idx: np.ndarray, step: int, block: int = 0, seed: int = SEED) -> np.ndarray:
    """G16 at arbitrary (sampled) element indices of `block` at `step`."""
    return _grad_from_draws(draws(stream_key(seed, TAG_GRAD, step, block), idx))


def bf16_bits_to_f32(bits: np.ndarray) -> np.ndarray:
    """Exact widening bf16 -> fp32 (a bit shift; used only to build inputs)."""
    return (np.asarray(bits, dtype=np.uint16).astype(np.uint32) << np.uint32(16)).view(np.float32)


def grad16_normal(n: int, std: float, seed: int) -> np.ndarray:
    """Gaussian-shaped bf16 grads (numpy RNG, truncated to bf16 bits).

    Host-only variant used by the tolerance tests (SURVEY §8(c) "Tolerance
    evidence", g ~ N(0, 1e-3^2)); generated here and copied to the device.
    Truncation (not rounding) keeps this free of the method's arithmetic.
    """
    x = np.random.default_rng(seed).normal(0.0, std, size=n).astype(np.float32)
    return (x.view(np.uint32) >> np.uint32(16)).astype(np.uint16)
