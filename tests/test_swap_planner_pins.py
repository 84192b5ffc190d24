"""Pins for the activation-swap planner oracle (oracle/swap_planner.py,
PAPER.md §IV-D) against things other than itself (CPU only).

The paper prints no planner inputs or outputs, so the oracle is pinned by
  * a worked example computed by hand (below, every term written out),
  * the paper's own theorems: T_iter convex in A_G2M, Eq. 8's
    slope dFLOP_r/dA_G2M = -OB_{i+1}, Eq. 7's end points,
  * fractional-knapsack optimality of the OB order (brute force over every
    subset of small layer lists: no subset saves more recomputation than the
    Eq. 7 curve at the same A_G2M -- which is why the paper sorts by OB),
  * Cases 1-3 on inputs built to fall in each case, and
    Algorithm 1's result vs a brute-force scan of every prefix.
"""
import itertools
import random

import pytest

from oracle import swap_planner as SP

# ---------------------------------------------------------------- worked example
# THP_G 100 FLOP/s, BW_G 10 B/s, BW_S2M 20 B/s, BW_M2S 10 B/s, MEM_M^avail 30 B,
# P = 5 params, FLOP_f = 600.
#   T_f = max(600/100 = 6, A/10, 2*5/10 = 1, 10/20 + alpha/10)          (Eq. 4)
#   T_b = max((1200 + FLOP_r)/100, 1, (10 + A)/10, (70 + alpha)/20 + 7) (Eq. 5)
# Layers (act, flop): L0 (20, 100) OB 5; L1 (10, 300) OB 30; L2 (40, 200) OB 5;
# L3 (30, 0) OB 0.  OB order (descending, stable): L1, L0, L2, L3.
#   prefix L1          A=10  FLOP_r=300 alpha=0  T_f=6   T_b=15   T=21
#   prefix L1 L0       A=30  FLOP_r=200 alpha=0  T_f=6   T_b=14   T=20
#   prefix L1 L0 L2    A=70  FLOP_r=0   alpha=40 T_f=7   T_b=12.5 T=19.5
#   prefix all         A=100 FLOP_r=0   alpha=70 T_f=10  T_b=14   T=24
HAND = SP.Model(thp_g=100.0, bw_g=10.0, bw_s2m=20.0, bw_m2s=10.0, mem_m_avail=30.0,
                params=5.0, flop_f=600.0)
HAND_LAYERS = [SP.Layer(20, 100), SP.Layer(10, 300), SP.Layer(40, 200), SP.Layer(30, 0)]


@pytest.mark.parametrize("a,flop_r,tf,tb", [(10, 300, 6, 15), (30, 200, 6, 14), (70, 0, 7, 12.5),
                                            (100, 0, 10, 14), (0, 600, 6, 18)])
def test_hand_example_times(a, flop_r, tf, tb):
    assert SP.t_forward(a, HAND) == tf
    assert SP.t_backward(a, flop_r, HAND) == tb
    assert SP.t_iter(a, flop_r, HAND) == tf + tb


def test_hand_example_alpha_never_negative():
    """R18: below MEM_M^avail nothing spills (a negative alpha would shorten
    the SSD terms)."""
    assert SP.alpha_a_g2m(10, HAND) == 0.0
    assert SP.alpha_a_g2m(30, HAND) == 0.0
    assert SP.alpha_a_g2m(70, HAND) == 40.0


def test_hand_example_order_and_eq7():
    assert SP.sort_by_offloading_benefit(HAND_LAYERS) == [1, 0, 2, 3]
    srt = [HAND_LAYERS[i] for i in [1, 0, 2, 3]]
    assert SP.flop_r_interp(0, srt, 600) == 600
    assert SP.flop_r_interp(10, srt, 600) == 300
    assert SP.flop_r_interp(20, srt, 600) == 250      # half of L0: 600-300-50
    assert SP.flop_r_interp(50, srt, 600) == 100      # half of L2: 600-300-100-100
    assert SP.flop_r_interp(100, srt, 600) == 0
    assert SP.flop_r_interp(1e9, srt, 600) == 0       # R19


def test_hand_example_algorithm1():
    p = SP.algorithm1(HAND_LAYERS, HAND, a_inter_block=0.0)
    assert (p.swap, p.a_g2m, p.flop_r, p.t_iter, p.t_min) == ([1, 0, 2], 70, 0, 19.5, 19.5)


def test_hand_example_oom_guard_reading():
    """R21: with A_interBlock = 80 the list (70 B) is below the floor when L3
    raises T, so L3 is still swapped (the literal test on 70+30 would stop at
    70 B < A_interBlock)."""
    p = SP.algorithm1(HAND_LAYERS, HAND, a_inter_block=80.0)
    assert (p.swap, p.a_g2m, p.t_iter, p.t_min) == ([1, 0, 2, 3], 100, 24, 19.5)
    p = SP.algorithm1(HAND_LAYERS, HAND, a_inter_block=70.0)
    assert p.swap == [1, 0, 2]


def test_empty_layer_list():
    p = SP.algorithm1([], HAND, 0.0)
    assert (p.swap, p.a_g2m, p.flop_r, p.t_iter) == ([], 0.0, 600.0, 24.0)


# ---------------------------------------------------------------- random inputs
def rand_model(rng, flop_f):
    return SP.Model(thp_g=10 ** rng.uniform(12, 16), bw_g=10 ** rng.uniform(9, 11.5),
                    bw_s2m=10 ** rng.uniform(8.5, 10.5), bw_m2s=10 ** rng.uniform(8.5, 10.5),
                    mem_m_avail=10 ** rng.uniform(8, 12), params=10 ** rng.uniform(8, 11),
                    flop_f=flop_f)


def rand_layers(rng, n):
    return [SP.Layer(10 ** rng.uniform(6, 10), rng.choice([0.0, 10 ** rng.uniform(8, 13)]))
            for _ in range(n)]


@pytest.mark.parametrize("seed", range(40))
def test_t_iter_convex_in_a_g2m(seed):
    """§IV-D 'Proving Convexity': with FLOP_r from Eq. 7 over the
    OB order, T_iter is convex in A_G2M -- slopes between consecutive grid
    points never decrease."""
    rng = random.Random(seed)
    layers = rand_layers(rng, rng.randint(1, 12))
    srt = [layers[i] for i in SP.sort_by_offloading_benefit(layers)]
    flop_f = sum(l.flop for l in layers) * rng.uniform(1.0, 1.5)
    m = rand_model(rng, flop_f)
    total = sum(l.act for l in layers)
    pts = sorted({total * k / 400 for k in range(401)} |
                 set(itertools.accumulate(l.act for l in srt)) | {m.mem_m_avail})
    pts = [a for a in pts if 0 <= a <= total]
    ts = [SP.t_iter(a, SP.flop_r_interp(a, srt, flop_f), m) for a in pts]
    keep = [0] + [i for i in range(1, len(pts)) if pts[i] - pts[i - 1] > total * 1e-9]
    pts, ts = [pts[i] for i in keep], [ts[i] for i in keep]
    da = [pts[i + 1] - pts[i] for i in range(len(pts) - 1)]
    slopes = [(ts[i + 1] - ts[i]) / da[i] for i in range(len(da))]
    tmax = max(ts)
    for i in range(len(slopes) - 1):   # rounding of T (~1e-16 relative) over the spacing
        assert slopes[i + 1] >= slopes[i] - 1e-13 * tmax / min(da[i], da[i + 1])


@pytest.mark.parametrize("seed", range(20))
def test_eq8_slope_is_minus_ob(seed):
    """Eq. 8: inside segment i+1, dFLOP_r/dA_G2M = -OB_{i+1}."""
    rng = random.Random(100 + seed)
    layers = rand_layers(rng, rng.randint(1, 10))
    srt = [layers[i] for i in SP.sort_by_offloading_benefit(layers)]
    flop_f = sum(l.flop for l in layers)
    start = 0.0
    for l in srt:
        a0, a1 = start + 0.25 * l.act, start + 0.75 * l.act
        slope = (SP.flop_r_interp(a1, srt, flop_f) - SP.flop_r_interp(a0, srt, flop_f)) / (a1 - a0)
        assert slope == pytest.approx(-l.flop / l.act, rel=1e-9, abs=1e-9 * flop_f / l.act)
        start += l.act
    # and the OB order makes those slopes non-decreasing (FLOP_r convex)
    obs = [-l.flop / l.act for l in srt]
    assert obs == sorted(obs)


@pytest.mark.parametrize("seed", range(30))
def test_ob_order_is_optimal_fractional_knapsack(seed):
    """Brute force over all 2^n subsets: no set of whole layers with total
    activation A saves more recomputation than Eq. 7's OB-ordered curve at A
    (the greedy OB order solves the fractional knapsack)."""
    rng = random.Random(200 + seed)
    layers = rand_layers(rng, rng.randint(1, 9))
    srt = [layers[i] for i in SP.sort_by_offloading_benefit(layers)]
    flop_f = sum(l.flop for l in layers)
    for r in range(len(layers) + 1):
        for sub in itertools.combinations(range(len(layers)), r):
            a = sum(layers[i].act for i in sub)
            fr = flop_f - sum(layers[i].flop for i in sub)
            assert fr >= SP.flop_r_interp(a, srt, flop_f) - 1e-9 * flop_f


def brute_force_prefix(layers, m, floor):
    """Every prefix k >= 1 of the OB order: the smallest k that reaches the
    floor (or all layers), then the first minimum of T over k >= that."""
    order = SP.sort_by_offloading_benefit(layers)
    ts, acts = [], []
    a, fr = 0.0, m.flop_f
    for i in order:
        a, fr = a + layers[i].act, fr - layers[i].flop
        ts.append(SP.t_iter(a, fr, m))
        acts.append(a)
    prev = [0.0] + acts[:-1]
    kf = next((k for k in range(len(order)) if prev[k] >= floor), len(order))
    kf = max(kf, 1)     # Algorithm 1 always swaps the first layer (T < Tmin = inf)
    cands = range(kf, len(order) + 1)
    best = min(ts[k - 1] for k in cands)
    kstar = next(k for k in cands if ts[k - 1] == best)
    return order[:kstar]


@pytest.mark.parametrize("seed", range(60))
def test_algorithm1_equals_prefix_brute_force(seed):
    """Convexity makes T over OB prefixes unimodal, so Algorithm 1's first
    non-improving layer marks the best prefix that satisfies the OOM floor."""
    rng = random.Random(300 + seed)
    layers = rand_layers(rng, rng.randint(1, 14))
    m = rand_model(rng, sum(l.flop for l in layers) * rng.uniform(1.0, 1.3))
    floor = rng.choice([0.0, sum(l.act for l in layers) * rng.uniform(0, 1.2)])
    p = SP.algorithm1(layers, m, floor)
    assert p.swap == brute_force_prefix(layers, m, floor)
    assert p.a_g2m == pytest.approx(sum(layers[i].act for i in p.swap), rel=1e-12)


def test_case2_gpu_bound_swaps_everything():
    """Case 2: T decreases with A_G2M -> A_G2M = A_all."""
    rng = random.Random(7)
    layers = [SP.Layer(10 ** rng.uniform(6, 8), 10 ** rng.uniform(10, 12)) for _ in range(10)]
    m = SP.Model(thp_g=1e9, bw_g=1e12, bw_s2m=1e12, bw_m2s=1e12, mem_m_avail=1e15, params=1e6,
                 flop_f=sum(l.flop for l in layers))
    p = SP.algorithm1(layers, m, 0.0)
    assert sorted(p.swap) == list(range(10))
    assert p.a_g2m == pytest.approx(sum(l.act for l in layers))


@pytest.mark.parametrize("floor_frac", [0.0, 0.3, 0.75])
def test_case1_pcie_bound_stops_at_the_floor(floor_frac):
    """Case 1: T increases with A_G2M -> the smallest safe amount
    (the shortest OB prefix whose activations reach A_interBlock)."""
    rng = random.Random(8)
    layers = [SP.Layer(10 ** rng.uniform(8, 9), 10 ** rng.uniform(6, 7)) for _ in range(10)]
    m = SP.Model(thp_g=1e18, bw_g=1e6, bw_s2m=1e12, bw_m2s=1e12, mem_m_avail=1e15, params=1e3,
                 flop_f=sum(l.flop for l in layers))
    floor = floor_frac * sum(l.act for l in layers)
    p = SP.algorithm1(layers, m, floor)
    order = SP.sort_by_offloading_benefit(layers)
    acc, k = 0.0, 0
    while k == 0 or acc < floor:
        acc += layers[order[k]].act
        k += 1
    assert p.swap == order[:k]


def test_case3_interior_optimum():
    """Case 3: recomputation-bound at small A_G2M, PCIe-bound at
    large A_G2M -> an interior optimum.  Ten identical 1 GB layers of 1 TFLOP:
    T_b's GPU term is (2F + FLOP_r)/THP, its link term (2P + A)/BW_G; they cross
    at A = 5 GB here, so exactly 5 layers are swapped."""
    layers = [SP.Layer(1e9, 1e12) for _ in range(10)]
    # F = 1e13; T_b GPU term = (2e13 + 1e13 - k e12)/1e12 = 30 - k s;
    # link term = (2P + k e9)/1e9 = 20 + k s with P = 1e10 -> cross at k = 5.
    m = SP.Model(thp_g=1e12, bw_g=1e9, bw_s2m=1e15, bw_m2s=1e15, mem_m_avail=1e15, params=1e10,
                 flop_f=1e13)
    # T_f = max(10, k, 20, ~0) = 20 for every k <= 10; T_b = max(30-k, 20, 20+k, ~0)
    p = SP.algorithm1(layers, m, 0.0)
    assert p.swap == [0, 1, 2, 3, 4]
    assert p.t_iter == pytest.approx(20 + 25)


# ---------------------------------------------------------------- the pins pin
MUTANTS = [
    ("key=lambda i: -offloading_benefit(layers[i])", "key=lambda i: offloading_benefit(layers[i])"),
    ("return max(0.0, a_g2m - m.mem_m_avail)", "return a_g2m - m.mem_m_avail"),
    ("return max(0.0, a_g2m - m.mem_m_avail)", "return a_g2m"),
    ("if a_g2m >= a_inter_block:", "if a_next >= a_inter_block:"),
    ("t_g = (2.0 * m.flop_f + flop_r) / m.thp_g", "t_g = (m.flop_f + flop_r) / m.thp_g"),
    ("t_s = (14.0 * m.params + alpha_a_g2m(a_g2m, m)) / m.bw_s2m + 14.0 * m.params / m.bw_m2s",
     "t_s = (14.0 * m.params + alpha_a_g2m(a_g2m, m)) / m.bw_s2m"),
    ("t_m2g = (2.0 * m.params + a_g2m) / m.bw_g", "t_m2g = 2.0 * m.params / m.bw_g"),
    ("t_g2m = a_g2m / m.bw_g", "t_g2m = 0.0"),
    ("return t_forward(a_g2m, m) + t_backward(a_g2m, flop_r, m)",
     "return max(t_forward(a_g2m, m), t_backward(a_g2m, flop_r, m))"),
    ("flop_r -= layer.flop * (a_g2m - covered) / layer.act", "flop_r -= layer.flop"),
    ("if t >= t_min:", "if t > t_min:"),
    ("t_min = t                          # line 16", "pass"),
    ("        a_g2m, flop_r = a_next, flop_r_next\n", "        a_g2m = a_next\n"),
]


def _pins(mod, monkeypatch):
    """Run every deterministic pin above against module `mod`; True if all pass."""
    import sys
    me = sys.modules[__name__]
    monkeypatch.setattr(me, "SP", mod)
    checks = [lambda: [test_hand_example_times(*a) for a in
                       [(10, 300, 6, 15), (30, 200, 6, 14), (70, 0, 7, 12.5), (100, 0, 10, 14), (0, 600, 6, 18)]],
              test_hand_example_alpha_never_negative, test_hand_example_order_and_eq7,
              test_hand_example_algorithm1, test_hand_example_oom_guard_reading, test_empty_layer_list,
              test_case2_gpu_bound_swaps_everything, test_case3_interior_optimum,
              lambda: [test_case1_pcie_bound_stops_at_the_floor(f) for f in (0.0, 0.3, 0.75)]]
    checks += [lambda s=s: test_t_iter_convex_in_a_g2m(s) for s in range(10)]
    checks += [lambda s=s: test_algorithm1_equals_prefix_brute_force(s) for s in range(20)]
    checks += [lambda s=s: test_ob_order_is_optimal_fractional_knapsack(s) for s in range(5)]
    for c in checks:
        try:
            c()
        except (AssertionError, ZeroDivisionError, TypeError, ValueError):
            return False
    return True


@pytest.mark.parametrize("k", range(len(MUTANTS)))
def test_every_planner_mutant_fails_a_pin(k, monkeypatch, tmp_path):
    import importlib.util
    src = open(SP.__file__).read()
    old, new = MUTANTS[k]
    assert src.count(old) == 1, old
    path = tmp_path / f"swap_planner_mut{k}.py"
    path.write_text(src.replace(old, new))
    spec = importlib.util.spec_from_file_location(f"swap_planner_mut{k}", path)
    mod = importlib.util.module_from_spec(spec)
    import sys
    sys.modules[spec.name] = mod      # dataclasses look the module up by name
    spec.loader.exec_module(mod)
    # the HAND model/layers are objects of the original module's classes; rebuild
    monkeypatch.setattr(sys.modules[__name__], "HAND", mod.Model(**vars(HAND)))
    monkeypatch.setattr(sys.modules[__name__], "HAND_LAYERS", [mod.Layer(l.act, l.flop) for l in HAND_LAYERS])
    assert not _pins(mod, monkeypatch), f"mutant {k} survives: {new!r}"


def test_unmutated_oracle_passes_the_pin_runner(monkeypatch):
    assert _pins(SP, monkeypatch)
