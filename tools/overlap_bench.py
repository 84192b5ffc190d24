"""Overlap of the AGO optimizer step with a synthetic backward (Fig. 7 analog).

SURVEY §8(d) C2: 13B device-resident states; the synthetic backward runs, per
block in decreasing order, the two GEMMs of each of the block's four linears
(dX = dY.W and dW = dY^T.X, 4.P_blk.T FLOPs, T tokens, bf16 on cuBLAS via
torch -- harness, not product) writing dW into a small ring of gradient
buffers, then hands the block off (ratel_offload_grad_chunk).  Before a ring
slot is rewritten the backward stream waits for the update that consumed it
(ratel_block_wait).

Schedules (§V-E, Fig. 7):
  bwd      backward alone (no optimizer)                       -> T_bwd
  opt      optimizer alone (all hand-offs, then arm)           -> T_opt
  ago      arm first, hand off each block as produced (Optimized AGO)
  deferred backward, then arm after the last hand-off ("Ratel+ZeRO")
  naive    like ago but the backward waits for each block's update before
           continuing (the handler is not overlapped, Fig. 3a)
Reported per token count: step ms, exposed optimizer ms = T - T_bwd, and the
update kernel's own time.  One JSON line per (tokens, schedule, max_ctas).

Memory: the grad ring replaces full-model G16 (25.7 GB for 13B), which would
not fit next to 180 GB of states -- the AGO memory effect.
"""
import argparse
import json
import os
import sys
import time

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import torch  # noqa: E402

import bench  # noqa: E402
import paper_conf_icde_liaosyxcyww25_b200 as R  # noqa: E402


from bench import SynthBackward, linears  # noqa: E402,F401


def run(args):
    dev = torch.device("cuda:0")
    torch.cuda.set_device(dev)
    L, h = bench.SHAPES[args.shape]
    sizes = bench.model_blocks(args.shape)[:args.blocks] if args.blocks else bench.model_blocks(args.shape)
    cfg = R.ratel_default_config()
    cfg.timing = 1
    cfg.max_ctas = 0
    R.ratel_init(0, 0, 1, None, cfg)
    if args.ring <= 0:
        args.ring = len(sizes)          # full-model G16 (only fits for a block subset)
    model = bench.Model(R, torch, dev, sizes, 1, 0, "device", grad_ring=args.ring)
    ring = model.grad_ring
    for b in range(len(sizes)):
        R.ratel_register_block(b, [model.ranges[b]], R.RATEL_DEVICE)
    # registered ranges point at ring[b % R]; the backward writes dW there
    vocab = bench.VOCAB if len(sizes) == L + 1 else 0
    hi = torch.cuda.Stream(priority=-2)
    order = list(reversed(range(len(sizes))))
    t_state = {"t": 1}
    results = []

    def arm():
        R.ratel_adam_step(1e-3, 0.9, 0.999, 1e-8, 1e-2, t_state["t"])
        t_state["t"] += 1

    def one(schedule, bw):
        with torch.cuda.stream(hi):
            if schedule == "opt":
                for b in order:
                    R.ratel_offload_grad_chunk(b, hi)
                arm()
            elif schedule == "bwd":
                for b in order:
                    bw.block(b, b % args.ring)
            else:
                if schedule in ("ago", "naive"):
                    arm()
                for j, b in enumerate(order):
                    slot = b % args.ring
                    if schedule != "deferred" and j >= args.ring:
                        R.ratel_block_wait(b + args.ring, hi)   # ring slot free
                    bw.block(b, slot)
                    R.ratel_offload_grad_chunk(b, hi)
                    if schedule == "naive":
                        R.ratel_block_wait(b, hi)               # handler not overlapped
                if schedule == "deferred":
                    arm()
            if schedule != "bwd":
                R.ratel_sync(hi)

    for tokens in args.tokens:
        bw = SynthBackward(dev, h, tokens, model.p16, ring, vocab)
        for mc in args.max_ctas:
            R.ratel_finalize()
            cfg.max_ctas = mc
            R.ratel_init(0, 0, 1, None, cfg)
            for b in range(len(sizes)):
                R.ratel_register_block(b, [model.ranges[b]], R.RATEL_DEVICE)
            t_state["t"] = 1
            scheds = ["bwd", "opt", "ago", "deferred", "naive"]
            times = {}
            for sch in scheds:
                if sch == "deferred" and args.ring < len(sizes):
                    # deferred needs every block's grad alive until the arm
                    times[sch] = None
                    continue
                for _ in range(args.warmup):
                    one(sch, bw)
                torch.cuda.synchronize()
                R.ratel_kernel_timing(reset=True)
                e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
                e0.record(hi)
                for _ in range(args.steps):
                    one(sch, bw)
                e1.record(hi)
                e1.synchronize()
                k1_ms, k1_n = R.ratel_kernel_timing(reset=True)
                times[sch] = (e0.elapsed_time(e1) / args.steps, k1_ms / args.steps)
            tb = times["bwd"][0]
            row = {"tokens": tokens, "max_ctas": mc, "blocks": len(sizes), "params": sum(sizes),
                   "bwd_ms": tb, "opt_ms": times["opt"][0],
                   "bwd_tflops": 4 * sum(sizes) * tokens / (tb / 1e3) / 1e12}
            for sch in ("ago", "deferred", "naive"):
                if times.get(sch):
                    row[f"{sch}_ms"] = times[sch][0]
                    row[f"{sch}_exposed_ms"] = times[sch][0] - tb
                    row[f"{sch}_k1_ms"] = times[sch][1]
            print(json.dumps(row), flush=True)
            results.append(row)
        del bw
        torch.cuda.empty_cache()
    R.ratel_finalize()
    return results


if __name__ == "__main__":
    ap = argparse.ArgumentParser()
    ap.add_argument("--shape", default="13B")
    ap.add_argument("--blocks", type=int, default=0)
    ap.add_argument("--tokens", type=int, nargs="+", default=[2048, 8192, 32768])
    ap.add_argument("--max-ctas", type=int, nargs="+", default=[0, 32])
    ap.add_argument("--ring", type=int, default=3)
    ap.add_argument("--steps", type=int, default=3)
    ap.add_argument("--warmup", type=int, default=1)
    run(ap.parse_args())
