"""Ratel's activation-swap plan (§IV-D, Algorithm 1) for the Table IV
GPT shapes on a measured B200 box, through the library's C ABI
(include/ratel_plan.h).

    python tools/plan_swap.py [--box profiles/r01_box.json] [--shapes 13B,70B,175B]
                              [--bsz 1,8,32] [--bw-ssd GB/s ...] [--mem-avail-gb X]

Layer recipe (synthetic; the paper profiles real layers): each
transformer block of hidden h, heads a, sequence s = 1024 and batch
b is split into the operators whose inputs backward needs, with bf16
activations -- the standard per-layer accounting of 34·s·b·h + 5·a·s²·b bytes
(Korthikanti et al., "Reducing Activation Recomputation in Large Transformer
Models", 2022; outside the paper) -- and each operator's recompute FLOPs are
its forward FLOPs (2 per multiply-add for the GEMMs).  A_interBlock = the
block inputs, 2·s·b·h bytes per block.  FLOP_f = the sum over all layers
(Algorithm 1 line 4: FLOP_r starts at FLOP_f, full recomputation).

Machine (Table I): THP_G = MEASURED_PEAKS.json bf16_tflops_sustained;
BW_G = min(H2D, D2H) pinned bandwidth from the box probe (unidirectional);
BW_S2M / BW_M2S = the SSD read/write bandwidth (the box probe's direct-I/O
file numbers when present, else the --bw-ssd values); MEM_M^avail = host RAM
minus the pinned model states the AGO step needs (16 B/param: P32 + m + v +
P16 staging), floored at 0, unless --mem-avail-gb is given.
"""
from __future__ import annotations

import argparse
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
if ROOT not in sys.path:
    sys.path.insert(0, ROOT)

SEQ = 1024
VOCAB = 50257
# Table IV: layers, heads, hidden
SHAPES = {"6B": (28, 32, 4096), "13B": (40, 40, 5120), "30B": (48, 56, 7168), "70B": (80, 64, 8192),
          "135B": (88, 88, 11264), "175B": (96, 96, 12288), "276B": (112, 112, 14336),
          "412B": (128, 128, 16384)}


def block_ops(h: int, a: int, b: int, s: int = SEQ):
    """(name, activation bytes, recompute FLOPs) per operator of one block."""
    sbh = s * b * h
    as2b = a * s * s * b
    return [
        ("ln1", 2 * sbh, 5 * sbh),
        ("qkv", 2 * sbh, 2 * sbh * 3 * h),
        ("qk^T", 4 * sbh, 2 * b * s * s * h),
        ("softmax", 2 * as2b, 5 * as2b),
        ("attn_dropout", as2b, as2b),
        ("attn_v", 2 * as2b + 2 * sbh, 2 * b * s * s * h),
        ("proj", 2 * sbh, 2 * sbh * h),
        ("dropout1", sbh, sbh),
        ("ln2", 2 * sbh, 5 * sbh),
        ("fc1", 2 * sbh, 2 * sbh * 4 * h),
        ("gelu", 8 * sbh, 8 * 4 * sbh),
        ("fc2", 8 * sbh, 2 * sbh * 4 * h),
        ("dropout2", sbh, sbh),
    ]


def gpt_layers(shape: str, bsz: int):
    """-> ([(act_bytes, flop)] over every block, A_interBlock, FLOP_f, P)."""
    L, a, h = SHAPES[shape]
    ops = block_ops(h, a, bsz)
    layers = [(float(act), float(fl)) for _ in range(L) for _, act, fl in ops]
    a_inter = float(L * 2 * SEQ * bsz * h)
    flop_f = sum(f for _, f in layers)
    params = float(L * (12 * h * h + 13 * h) + VOCAB * h + SEQ * h + 2 * h)
    return layers, a_inter, flop_f, params


def gpt_model(params, flop_f, *, thp_g, bw_g, bw_s2m, bw_m2s, mem_m_avail):
    from paper_conf_icde_liaosyxcyww25_b200 import ratel_swap_model
    return ratel_swap_model(thp_g=thp_g, bw_g=bw_g, bw_s2m=bw_s2m, bw_m2s=bw_m2s,
                            mem_m_avail=mem_m_avail, params=params, flop_f=flop_f)


def plan(shape, bsz, *, thp_g, bw_g, bw_s2m, bw_m2s, ram_bytes, mem_avail=None):
    import paper_conf_icde_liaosyxcyww25_b200 as R
    layers, a_inter, flop_f, params = gpt_layers(shape, bsz)
    mem = mem_avail if mem_avail is not None else max(0.0, ram_bytes - 16.0 * params)
    m = gpt_model(params, flop_f, thp_g=thp_g, bw_g=bw_g, bw_s2m=bw_s2m, bw_m2s=bw_m2s, mem_m_avail=mem)
    swap, order, p = R.ratel_plan_activation_swap(layers, m, a_inter)
    a_all = sum(x for x, _ in layers)
    _, heads, hidden = SHAPES[shape]
    names = [n for n, _, _ in block_ops(hidden, heads, bsz)]
    n_ops = len(names)
    swapped_ops = sorted({names[i % n_ops] for i in swap})
    # the two baselines of Fig. 1: inter-block checkpoints only (ZeRO-Infinity) vs swap everything
    inter_idx = [i for i in range(len(layers)) if names[i % n_ops] == "ln1"]
    fr = flop_f - sum(layers[i][1] for i in inter_idx)
    t_ckpt = sum(R.ratel_swap_iter_time(m, a_inter, fr))
    t_all = sum(R.ratel_swap_iter_time(m, a_all, flop_f - sum(f for _, f in layers)))
    return {"shape": shape, "bsz": bsz, "tokens": bsz * SEQ, "params": params, "layers": len(layers),
            "a_all_gb": a_all / 1e9, "a_inter_block_gb": a_inter / 1e9,
            "swapped_layers": p.n_swap, "swapped_ops": swapped_ops,
            "a_g2m_gb": p.a_g2m / 1e9, "recompute_tflop": p.flop_r / 1e12, "flop_f_tflop": flop_f / 1e12,
            "t_f_s": p.t_f, "t_b_s": p.t_b, "t_iter_s": p.t_iter,
            "t_iter_interblock_only_s": t_ckpt, "t_iter_swap_all_s": t_all,
            "machine": {"thp_g_tflops": thp_g / 1e12, "bw_g_gbs": bw_g / 1e9, "bw_s2m_gbs": bw_s2m / 1e9,
                        "bw_m2s_gbs": bw_m2s / 1e9, "mem_m_avail_gb": mem / 1e9}}


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--box", default=os.path.join(ROOT, "profiles", "r01_box.json"))
    ap.add_argument("--peaks", default=os.path.join(ROOT, "MEASURED_PEAKS.json"))
    ap.add_argument("--shapes", default="13B,70B,175B")
    ap.add_argument("--bsz", default="1,8,32")
    ap.add_argument("--bw-ssd", type=float, nargs="*", default=None, help="GB/s; overrides the probe")
    ap.add_argument("--mem-avail-gb", type=float, default=None)
    args = ap.parse_args()
    box = json.load(open(args.box)) if os.path.exists(args.box) else {}
    try:
        thp = float(json.load(open(args.peaks))["bf16_tflops_sustained"]) * 1e12
    except Exception:
        thp = 1.3428e15
    bw_g = min(box.get("h2d_gbs", 55.0), box.get("d2h_gbs", 55.0)) * 1e9
    ram = 0.0
    for line in box.get("meminfo", "").splitlines():
        if line.startswith("MemTotal:"):
            ram = float(line.split()[1]) * 1024
    ssd = []
    if args.bw_ssd:
        ssd = [(g * 1e9, g * 1e9) for g in args.bw_ssd]
    elif "ssd_read_gbs" in box:
        ssd = [(box["ssd_read_gbs"] * 1e9, box["ssd_write_gbs"] * 1e9)]
    else:
        ssd = [(6e9, 4e9), (25e9, 20e9)]
    mem = args.mem_avail_gb * 1e9 if args.mem_avail_gb is not None else None
    for shape in args.shapes.split(","):
        for b in (int(x) for x in args.bsz.split(",")):
            for r, w in ssd:
                print(json.dumps(plan(shape, b, thp_g=thp, bw_g=bw_g, bw_s2m=r, bw_m2s=w, ram_bytes=ram,
                                      mem_avail=mem)))


if __name__ == "__main__":
    main()
