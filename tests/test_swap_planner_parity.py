"""Parity of the native activation-swap planner (libratel.so,
include/ratel_plan.h) with the CPU oracle (oracle/swap_planner.py), PAPER.md
§IV-D Eq. 1-8 and Algorithm 1.

The planner is host code (no CUDA), so these run in the CPU suite through the
C ABI.  Both sides evaluate the same equations in IEEE double in the paper's
order without FMA contraction; the layer order and the swap decision are
integer results (compared exactly) and the reported times are compared
bitwise (R18-R22 pin the readings both follow).
"""
import math
import random

import pytest

import paper_conf_icde_liaosyxcyww25_b200 as R
from oracle import swap_planner as SP
from tests.test_swap_planner_pins import HAND, HAND_LAYERS, rand_layers, rand_model


def cmodel(m: SP.Model) -> R.ratel_swap_model:
    return R.ratel_swap_model(m.thp_g, m.bw_g, m.bw_s2m, m.bw_m2s, m.mem_m_avail, m.params, m.flop_f)


def pairs(layers):
    return [(l.act, l.flop) for l in layers]


def check_plan(layers, m, floor):
    ref = SP.algorithm1(layers, m, floor)
    swap, order, plan = R.ratel_plan_activation_swap(pairs(layers), cmodel(m), floor)
    assert order == SP.sort_by_offloading_benefit(layers)
    assert swap == ref.swap
    assert plan.n_swap == len(ref.swap)
    assert (plan.a_g2m, plan.flop_r, plan.t_iter, plan.t_min) == (ref.a_g2m, ref.flop_r, ref.t_iter, ref.t_min)
    assert (plan.t_f, plan.t_b) == (SP.t_forward(ref.a_g2m, m), SP.t_backward(ref.a_g2m, ref.flop_r, m))
    return swap, plan


def test_hand_example():
    swap, plan = check_plan(HAND_LAYERS, HAND, 0.0)
    assert swap == [1, 0, 2] and plan.t_iter == 19.5
    swap, _ = check_plan(HAND_LAYERS, HAND, 80.0)
    assert swap == [1, 0, 2, 3]


@pytest.mark.parametrize("seed", range(200))
def test_random_plans(seed):
    rng = random.Random(10_000 + seed)
    layers = rand_layers(rng, rng.randint(0, 40))
    m = rand_model(rng, sum(l.flop for l in layers) * rng.uniform(1.0, 1.3))
    floor = rng.choice([0.0, sum(l.act for l in layers) * rng.uniform(0, 1.2)])
    check_plan(layers, m, floor)


@pytest.mark.parametrize("seed", range(50))
def test_iter_time_and_eq7(seed):
    rng = random.Random(20_000 + seed)
    layers = rand_layers(rng, rng.randint(1, 30))
    flop_f = sum(l.flop for l in layers)
    m = rand_model(rng, flop_f)
    srt = [layers[i] for i in SP.sort_by_offloading_benefit(layers)]
    total = sum(l.act for l in layers)
    pts = [0.0, total, 2 * total, m.mem_m_avail] + [rng.uniform(0, total) for _ in range(20)]
    acc = 0.0
    for l in srt:          # exact prefix boundaries (the binary search's edge cases)
        acc += l.act
        pts.append(acc)
    for a in pts:
        fr = R.ratel_swap_recompute_flop(pairs(layers), flop_f, a)
        assert fr == SP.flop_r_interp(a, srt, flop_f), a
        assert R.ratel_swap_iter_time(cmodel(m), a, fr) == (SP.t_forward(a, m), SP.t_backward(a, fr, m))


def test_ties_keep_input_order():
    """R20: equal OB (including OB = 0) keep the caller's order."""
    layers = [SP.Layer(2.0, 4.0), SP.Layer(1.0, 0.0), SP.Layer(1.0, 2.0), SP.Layer(3.0, 0.0),
              SP.Layer(4.0, 8.0)]
    m = SP.Model(1.0, 1.0, 1.0, 1.0, 0.0, 1.0, 14.0)
    _, order, _ = R.ratel_plan_activation_swap(pairs(layers), cmodel(m), 0.0)
    assert order == [0, 2, 4, 1, 3]
    check_plan(layers, m, 0.0)


def test_empty_and_degenerate():
    check_plan([], HAND, 0.0)
    check_plan([], HAND, 1e9)
    one = [SP.Layer(5.0, 7.0)]
    check_plan(one, HAND, 0.0)
    check_plan(one, HAND, 1e9)               # floor above everything: swap all
    zero_p = SP.Model(1e12, 1e9, 1e9, 1e9, 0.0, 0.0, 0.0)   # P = 0, FLOP_f = 0
    check_plan([SP.Layer(1e6, 0.0)] * 3, zero_p, 0.0)


def test_gpt_shaped_layer_lists():
    """The tool's GPT layer recipe (tools/plan_swap.py) on Table IV shapes."""
    from tools.plan_swap import gpt_layers, gpt_model
    for shape in ("13B", "70B", "175B"):
        for bsz in (1, 8, 32):
            layers, a_inter, flop_f, params = gpt_layers(shape, bsz)
            for bw_ssd in (6e9, 25e9):
                m = gpt_model(params, flop_f, thp_g=1.3428e15, bw_g=55e9, bw_s2m=bw_ssd, bw_m2s=bw_ssd,
                              mem_m_avail=100e9)
                check_plan([SP.Layer(a, f) for a, f in layers], m, a_inter)


@pytest.mark.parametrize("bad", [
    dict(thp_g=0.0), dict(bw_g=-1.0), dict(bw_s2m=math.inf), dict(bw_m2s=math.nan),
    dict(mem_m_avail=-1.0), dict(params=-2.0), dict(flop_f=math.nan)])
def test_invalid_model_rejected(bad):
    kw = dict(thp_g=1.0, bw_g=1.0, bw_s2m=1.0, bw_m2s=1.0, mem_m_avail=0.0, params=1.0, flop_f=1.0)
    kw.update(bad)
    with pytest.raises(R.RatelError) as e:
        R.ratel_plan_activation_swap([(1.0, 1.0)], R.ratel_swap_model(**kw), 0.0)
    assert e.value.code == R.RATEL_EINVAL and "swap planner" in str(e.value)
    with pytest.raises(R.RatelError):
        R.ratel_swap_iter_time(R.ratel_swap_model(**kw), 0.0, 0.0)


@pytest.mark.parametrize("layers,floor", [([(0.0, 1.0)], 0.0), ([(-1.0, 1.0)], 0.0), ([(1.0, -1.0)], 0.0),
                                          ([(math.inf, 1.0)], 0.0), ([(1.0, math.nan)], 0.0),
                                          ([(1.0, 1.0)], -1.0), ([(1.0, 1.0)], math.nan)])
def test_invalid_layers_rejected(layers, floor):
    with pytest.raises(R.RatelError) as e:
        R.ratel_plan_activation_swap(layers, cmodel(HAND), floor)
    assert e.value.code == R.RATEL_EINVAL


def test_null_pointers_rejected():
    lib = R.lib()
    plan = R.ratel_swap_plan()
    assert lib.ratel_plan_activation_swap(None, 1, None, 0.0, None, None) == R.RATEL_EINVAL
    arr = (R.ratel_swap_layer * 1)(R.ratel_swap_layer(1.0, 1.0))
    m = cmodel(HAND)
    import ctypes
    assert lib.ratel_plan_activation_swap(arr, 1, ctypes.byref(m), 0.0, None, ctypes.byref(plan)) == R.RATEL_EINVAL
    assert lib.ratel_plan_activation_swap(arr, -1, ctypes.byref(m), 0.0, None, ctypes.byref(plan)) == R.RATEL_EINVAL
    assert lib.ratel_swap_recompute_flop(arr, 1, 1.0, 0.0, None) == R.RATEL_EINVAL
