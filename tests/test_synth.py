"""The seeded input generator (synth/) -- CPU checks.

Known-answer values: splitmix64 with state 0 yields 0xE220A8397B1DCDAF,
0x6E789E6AA1B965F4, 0x06C45D188009454F (the published splitmix64 sequence).
"""
import numpy as np

import synth


def test_splitmix64_known_answer():
    r = synth.draws(0, np.arange(3))
    assert [int(x) for x in r] == [0xE220A8397B1DCDAF, 0x6E789E6AA1B965F4, 0x06C45D188009454F]
    # vector and scalar finaliser agree
    z = np.array([1, 2, 0xFFFFFFFFFFFFFFFF], dtype=np.uint64)
    assert [int(x) for x in synth._mix64_vec(z)] == [synth.mix64_int(int(x)) for x in z]


def test_theta0_range_and_resolution():
    th = synth.theta0(1 << 20, block=0)
    assert th.dtype == np.float32
    assert th.min() >= -0.05 and th.max() < 0.05
    assert abs(float(th.mean())) < 1e-3
    # uniform: std = 0.1/sqrt(12)
    assert abs(float(th.std()) - 0.1 / np.sqrt(12)) < 1e-3


def test_grad_distribution():
    g = synth.grad16(1 << 20, step=1, block=0)
    zp = np.mean(g == 0x0000)
    zn = np.mean(g == 0x8000)
    assert 0.008 < zp < 0.012 and 0.0006 < zn < 0.0014
    nz = g[(g & 0x7FFF) != 0]
    e = ((nz >> 7) & 0xFF).astype(int) - 127
    assert e.min() == -30 and e.max() == -7
    counts = np.bincount(e + 30)
    assert counts.min() > 0.9 * counts.mean()
    assert 0.45 < np.mean(nz >> 15) < 0.55
    f = np.abs(synth.bf16_bits_to_f32(nz))
    assert f.max() < 2.0 ** -6 and f.min() >= 2.0 ** -30


def test_streams_independent_and_sampled_access():
    a = synth.grad16(5000, step=1, block=3)
    b = synth.grad16(5000, step=2, block=3)
    c = synth.grad16(5000, step=1, block=4)
    assert np.mean(a == b) < 0.05 and np.mean(a == c) < 0.05
    idx = np.array([0, 17, 4999, 123], dtype=np.uint64)
    assert np.array_equal(synth.grad16_at(idx, step=1, block=3), a[idx.astype(int)])
    th = synth.theta0(5000, block=3)
    assert np.array_equal(synth.theta0_at(idx, block=3), th[idx.astype(int)])
    # offset windows equal slices of the full stream
    assert np.array_equal(synth.grad16(100, step=1, block=3, start=200), a[200:300])
