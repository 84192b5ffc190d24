"""CPU oracle for Ratel's holistic traffic-aware activation swapping planner
(§IV-D) -- TEST INFRASTRUCTURE ONLY.

Only tests/ may import this module; the product library never imports or
links it.  Plain Python floats (IEEE double), one function per equation, in
the paper's order and notation (Table I).  Units: bytes, FLOP,
seconds, bytes/s, FLOP/s; P is a parameter count (2P = bytes of a 16-bit copy).

Readings (R18-R22):
  R18  Eq. 3/4: MEM_CPU^avail in Eq. 4 is Table I's MEM_M^avail,
       and alpha*A_G2M = max(0, A_G2M - MEM_M^avail) (activations that do not
       fit in main memory go to the SSDs; never negative).
  R19  Eq. 7: A_G2M beyond sum(A) clamps to the last layer
       (FLOP_r = FLOP_f - sum(FLOP)); below 0 is not defined.
  R20  Algorithm 1 line 6: "sortByOffloadingBenefit" sorts by OB
       (Eq. 6) DESCENDING -- "higher offloading benefits have higher priority
       in swapping" -- stable, so equal OB keep list order.
  R21  Algorithm 1 lines 11-13: the OOM guard compares the
       amount already in the swap list (A_G2M before adding this layer) with
       A_interBlock.  The literal test on A_G2M after adding the layer can
       break with a swap list smaller than A_interBlock, contradicting the
       line-13 comment "Ensure A_G2M >= A_interBlock" and Case 1's "choose
       A_interBlock as the minimum safe swapped activation amount".
  R22  The planner's result is the swap list of Algorithm 1; A_G2M, FLOP_r and
       T_iter reported with it are those of that list (Eq. 1/4/5 at the list's
       totals), not of the layer that triggered the break.
"""
from __future__ import annotations

from dataclasses import dataclass


@dataclass
class Model:
    """Table I quantities that do not depend on the swap decision."""
    thp_g: float          # THP_G: measured peak GPU throughput, FLOP/s
    bw_g: float           # BW_G: max unidirectional GPU<->main PCIe bandwidth, B/s
    bw_s2m: float         # BW_S2M: SSD -> main bandwidth, B/s
    bw_m2s: float         # BW_M2S: main -> SSD bandwidth, B/s
    mem_m_avail: float    # MEM_M^avail: minimum unallocated main memory, bytes
    params: float         # P: number of parameters
    flop_f: float         # FLOP_f: forward FLOPs (backward is 2 FLOP_f, Table I)


@dataclass
class Layer:
    act: float            # A_i: activation bytes of the layer
    flop: float           # FLOP_i: FLOPs to recompute the layer


def alpha_a_g2m(a_g2m: float, m: Model) -> float:
    """Eq. 3 with R18: activations that spill to the SSDs."""
    return max(0.0, a_g2m - m.mem_m_avail)


def t_forward(a_g2m: float, m: Model) -> float:
    """Eq. 2 / Eq. 4: the forward stage is the slowest of GPU
    compute, GPU->main activations, main->GPU 16-bit params, and SSD I/O
    (params read plus spilled activations written; the SSD is simplex)."""
    t_g = m.flop_f / m.thp_g
    t_g2m = a_g2m / m.bw_g
    t_m2g = 2.0 * m.params / m.bw_g
    t_s = 2.0 * m.params / m.bw_s2m + alpha_a_g2m(a_g2m, m) / m.bw_m2s
    return max(t_g, t_g2m, t_m2g, t_s)


def t_backward(a_g2m: float, flop_r: float, m: Model) -> float:
    """Eq. 5: backward is the slowest of GPU compute (2 FLOP_f
    + recomputation), GPU->main 16-bit grads, main->GPU params + swapped-back
    activations, and SSD I/O (14P of states and spilled activations read,
    14P written).  The CPU Adam is not a term."""
    t_g = (2.0 * m.flop_f + flop_r) / m.thp_g
    t_g2m = 2.0 * m.params / m.bw_g
    t_m2g = (2.0 * m.params + a_g2m) / m.bw_g
    t_s = (14.0 * m.params + alpha_a_g2m(a_g2m, m)) / m.bw_s2m + 14.0 * m.params / m.bw_m2s
    return max(t_g, t_g2m, t_m2g, t_s)


def t_iter(a_g2m: float, flop_r: float, m: Model) -> float:
    """Eq. 1: T_iter = T_f + T_b (computeIterTime, Alg. 1 line 10)."""
    return t_forward(a_g2m, m) + t_backward(a_g2m, flop_r, m)


def offloading_benefit(layer: Layer) -> float:
    """Eq. 6: OB = FLOP_layer / A_layer."""
    return layer.flop / layer.act


def sort_by_offloading_benefit(layers: list[Layer]) -> list[int]:
    """Algorithm 1 line 6 with R20: indices by OB descending, stable."""
    return sorted(range(len(layers)), key=lambda i: -offloading_benefit(layers[i]))


def flop_r_interp(a_g2m: float, sorted_layers: list[Layer], flop_f: float) -> float:
    """Eq. 7: recomputation FLOPs when A_G2M covers the first i
    layers (in OB order) and the fraction (A_G2M - sum_{n<=i} A_n)/A_{i+1} of
    layer i+1 (the interpolation assumption of footnote 5)."""
    flop_r = flop_f
    covered = 0.0
    for layer in sorted_layers:
        if a_g2m >= covered + layer.act:
            flop_r -= layer.flop
            covered += layer.act
        else:
            flop_r -= layer.flop * (a_g2m - covered) / layer.act
            return flop_r
    return flop_r  # R19: beyond sum(A) every layer is swapped


@dataclass
class Plan:
    swap: list[int]       # swapped layers (indices into the input list), in OB order
    a_g2m: float          # sum of their activation bytes
    flop_r: float         # FLOP_f minus their recompute FLOPs
    t_iter: float         # Eq. 1 at (a_g2m, flop_r)
    t_min: float          # Algorithm 1's Tmin when it stopped


def algorithm1(layers: list[Layer], m: Model, a_inter_block: float) -> Plan:
    """Algorithm 1, line by line, with R20-R22."""
    swap_list: list[int] = []                  # line 1
    t_min = float("inf")                       # line 2
    a_g2m = 0.0                                # line 3
    flop_r = m.flop_f                          # line 4: full recomputation
    order = sort_by_offloading_benefit(layers)  # line 6
    for i in order:                            # line 7
        layer = layers[i]
        a_next = a_g2m + layer.act             # line 8
        flop_r_next = flop_r - layer.flop      # line 9
        t = t_iter(a_next, flop_r_next, m)     # line 10
        if t >= t_min:                         # line 11
            if a_g2m >= a_inter_block:         # line 12 (R21: the list before this layer)
                break                          # line 13 (R22: the list's totals stay)
        else:
            t_min = t                          # line 16
        swap_list.append(i)                    # line 18
        a_g2m, flop_r = a_next, flop_r_next
    return Plan(swap_list, a_g2m, flop_r, t_iter(a_g2m, flop_r, m), t_min)
