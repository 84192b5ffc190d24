"""Per-rank work of an N-GPU step, measured as rank 0 of a simulated world N on
ONE B200 (tools, not product).  --residency host does the same for the
pinned-host path (BASELINE configs[4], C5): the rank streams only its 1/N slices
of theta/m/v over its host link.

BASELINE configs[2] (30B states sharded across 8 GPUs, grad-norm clip
allreduce + bf16 all-gather) cannot run here: every gpurun call has one GPU.
What one rank of it does on its own HBM can: this registers every block of
the shape with a full-range bf16 P16 and G16 and this rank's 1/N slice of
theta/m/v (ratel_rank_slice), RATEL_COMM_NONE (no NCCL: the clip norm is
then the rank-local one and the all-gather is not run), and times the step
(K2 partials at each hand-off, K3, K1 on the slices) with CUDA events.

Printed per (shape, N): the rank's own params/s, K1's achieved HBM GB/s at
28 B/param, and the slice size.  The NVLink all-gather (2(N-1)/N B/param) and
the 8-byte allreduce are NOT in these numbers.

  python tools/rank_sim.py --shape 30B --worlds 1 2 4 8 --clip 1.0
"""
import argparse
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import torch  # noqa: E402

import bench  # noqa: E402
import paper_conf_icde_liaosyxcyww25_b200 as R  # noqa: E402


def run(shape, world, clip, steps, warmup, blocks, residency="device"):
    dev = torch.device("cuda:0")
    sizes = bench.model_blocks(shape)
    if blocks:
        sizes = sizes[:blocks]
    cfg = R.ratel_default_config()
    cfg.timing = 1
    cfg.max_grad_norm = clip
    cfg.comm = R.RATEL_COMM_NONE
    R.ratel_init(0, 0, world, None, cfg)
    try:
        model = bench.Model(R, torch, dev, sizes, world, 0, residency)
        for b in range(len(sizes)):
            R.ratel_register_block(b, [model.ranges[b]],
                                   R.RATEL_DEVICE if residency == "device" else R.RATEL_PINNED_HOST)
        s = torch.cuda.Stream(device=dev)
        order = list(reversed(range(len(sizes))))
        t = 1
        for _ in range(warmup):
            bench.step_once(R, t, order, s)
            t += 1
        torch.cuda.synchronize()
        R.ratel_kernel_timing(reset=True)
        ms = bench.timed_steps(R, torch, order, s, t, steps)
        k1_ms, k1_n = R.ratel_kernel_timing(reset=True)
        own = sum(e - b for (b, e) in model.slices)
        extra = {}
        if residency != "device":   # the rank's theta/m/v cross its host link: 12 B/param each way
            extra = {"host_link_gbs": 24 * own * steps / (ms / 1e3) / 1e9,
                     "host_link_probe": bench.host_link_probe(torch, dev)}
        del model
        return {"shape": shape, "world": world, "rank": 0, "residency": residency, **extra,
                "blocks": len(sizes), "params": sum(sizes),
                "own_params": own, "clip": clip, "steps": steps, "ms_per_step": ms / steps,
                "own_params_per_s": own * steps / (ms / 1e3),
                "k1_gbs": 28 * own * steps / (k1_ms / 1e3) / 1e9 if k1_ms > 0 else None,
                "k1_share_of_step": k1_ms / ms, "k1_launches_per_step": k1_n / steps,
                "not_included": "NCCL bf16 all-gather (2(N-1)/N B/param over NVLink) and the 8-byte norm allreduce"}
    finally:
        R.ratel_finalize()
        torch.cuda.empty_cache()


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--shape", default="30B")
    ap.add_argument("--worlds", type=int, nargs="+", default=[1, 2, 4, 8])
    ap.add_argument("--clip", type=float, default=1.0)
    ap.add_argument("--steps", type=int, default=10)
    ap.add_argument("--warmup", type=int, default=3)
    ap.add_argument("--blocks", type=int, default=0, help="first N blocks only (N = 1 of 30B does not fit)")
    ap.add_argument("--residency", default="device", choices=["device", "host"],
                    help="host: the rank's slices of theta/m/v in pinned host memory (C5's path)")
    a = ap.parse_args()
    for w in a.worlds:
        print(json.dumps(run(a.shape, w, a.clip, a.steps, a.warmup, a.blocks, a.residency)), flush=True)


if __name__ == "__main__":
    main()
