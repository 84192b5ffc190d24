"""Overlap of the AGO optimizer step with a synthetic backward (Fig. 7 analog).

SURVEY §8(d) C2/C4: the synthetic backward runs, per block in decreasing
order, the two GEMMs of each of the block's four linears (dX = dY.W and
dW = dY^T.X, 4.P_blk.T FLOPs, T tokens, bf16 cuBLAS via torch -- harness, not
product), writes dW into a ring of gradient buffers and hands the block off.
Before a ring slot is rewritten the backward stream waits for the update that
consumed it (ratel_block_wait).

Schedules (§V-E, Fig. 7; Fig. 3):
  bwd       backward alone                                   -> T_bwd
  opt       optimizer alone (all hand-offs, then arm)        -> T_opt
  ago       arm first, hand off each block as produced (optimized AGO;
            pinned-host: pipelined tile ring, Fig. 3b)
  naive     pinned-host: AGO with the SERIALIZED tile schedule (Fig. 3a);
            device: the backward waits for each block's update
  deferred  backward, then arm after the last hand-off ("Ratel+ZeRO";
            needs every block's grad alive: --ring 0)
One JSON line per (tokens, max_ctas): times and exposed = T - T_bwd.
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
from bench import SynthBackward  # noqa: E402
import paper_conf_icde_liaosyxcyww25_b200 as R  # noqa: E402


def run(args):
    dev = torch.device("cuda:0")
    torch.cuda.set_device(dev)
    L, h = bench.SHAPES[args.shape]
    sizes = bench.model_blocks(args.shape)
    if args.blocks:
        sizes = sizes[:args.blocks]
    if args.ring <= 0:
        args.ring = len(sizes)          # full-model G16 (only fits for a block subset)
    cfg = R.ratel_default_config()
    cfg.timing = 1
    R.ratel_init(0, 0, 1, None, cfg)
    model = bench.Model(R, torch, dev, sizes, 1, 0, "device" if args.residency == "device" else "host",
                        grad_ring=args.ring)
    R.ratel_finalize()
    ring = model.grad_ring
    res_code = {"host": R.RATEL_PINNED_HOST, "hostcompute": R.RATEL_HOST_COMPUTE}.get(args.residency, R.RATEL_DEVICE)
    hybrid = args.residency == "hybrid"
    vocab = bench.VOCAB if len(sizes) == L + 1 else 0
    hi = torch.cuda.Stream(priority=args.bwd_priority)
    order = list(reversed(range(len(sizes))))
    # --granularity tensor: every linear of a block (its weights; the last one
    # also carries the block's 13h biases/LN) is its own registered unit,
    # handed off right after its dW GEMM -- the paper's per-tensor hand-off
    # (P:L1038-1041).  Unit id = b*K + j, j = linear index (qkv 0 .. fc2 3).
    K = 4 if args.granularity == "tensor" else 1
    units = {}            # block -> [ratel_range per unit]
    for b, n in enumerate(sizes):
        if K == 1 or (vocab and b == len(sizes) - 1):
            units[b] = [model.ranges[b]]
            continue
        r0, offs, off = model.ranges[b], [], 0
        for (o, i) in bench.linears(h):
            offs.append((off, o * i))
            off += o * i
        offs[-1] = (offs[-1][0], offs[-1][1] + (n - off))   # biases / LN with fc2
        units[b] = [R.ratel_range(r0.param_bf16 + 2 * o, r0.grad_bf16 + 2 * o, 0, r0.master + 4 * o,
                                  r0.exp_avg + 4 * o, r0.exp_avg_sq + 4 * o, ln, 1) for (o, ln) in offs]

    # Registered library blocks per unit: one, or with --residency hybrid the
    # unit's first hybrid_gpu_frac GPU-streamed (PINNED_HOST) and the rest on
    # the CPU handler (HOST_COMPUTE), handed off together.
    lib = {}
    nxt = 0
    for b in range(len(sizes)):
        for j, r in enumerate(units[b]):
            parts = [(r, res_code)]
            if hybrid:
                k = min(r.numel, int(round(args.hybrid_gpu_frac * r.numel / 8)) * 8)
                tail = R.ratel_range(r.param_bf16 + 2 * k, r.grad_bf16 + 2 * k, 0, r.master + 4 * k,
                                     r.exp_avg + 4 * k, r.exp_avg_sq + 4 * k, r.numel - k, r.apply_weight_decay)
                head = R.ratel_range(r.param_bf16, r.grad_bf16, 0, r.master, r.exp_avg, r.exp_avg_sq, k,
                                     r.apply_weight_decay)
                parts = [(x, c) for x, c, n in ((head, R.RATEL_PINNED_HOST, k),
                                                (tail, R.RATEL_HOST_COMPUTE, r.numel - k)) if n > 0]
            lib[(b, j)] = []
            for x, c in parts:
                lib[(b, j)].append((nxt, x, c))
                nxt += 1

    def handoff_unit(b, j, stream):
        for i, _, _ in lib[(b, j)]:
            R.ratel_offload_grad_chunk(i, stream)

    def handoff_all(b, stream):
        for j in range(len(units[b])):
            handoff_unit(b, j, stream)

    def wait_all(b, stream):
        for j in range(len(units[b])):
            for i, _, _ in lib[(b, j)]:
                R.ratel_block_wait(i, stream)
    t_state = {"t": 1}

    def arm():
        R.ratel_adam_step(1e-3, 0.9, 0.999, 1e-8, 1e-2, t_state["t"])
        t_state["t"] += 1

    side = torch.cuda.Stream()
    tl = {}

    def one(schedule, bw, timeline=False):
        if timeline:
            tl["t0"] = torch.cuda.Event(enable_timing=True)
            tl["t0"].record(hi)
            tl["g"], tl["d"] = {}, {}
        with torch.cuda.stream(hi):
            if schedule == "opt":
                for b in order:
                    handoff_all(b, hi)
                arm()
            elif schedule == "bwd":
                for b in order:
                    bw.block(b, b % args.ring)
            else:
                if schedule != "deferred":
                    arm()
                held = []                                       # --group: blocks not yet handed off
                for j, b in enumerate(order):
                    if schedule != "deferred" and j >= args.ring:
                        wait_all(b + args.ring, hi)             # ring slot free
                    if len(units[b]) > 1:                       # per-tensor hand-off
                        bw.block(b, b % args.ring, on_linear=lambda k, b=b: handoff_unit(b, k, hi))
                    else:
                        bw.block(b, b % args.ring)
                        held.append(b)
                        if len(held) >= args.group or j == len(order) - 1:
                            for x in held:                      # a burst of hand-offs: one update phase
                                handoff_unit(x, 0, hi)
                            held = []
                    if timeline:
                        tl["g"][b] = torch.cuda.Event(enable_timing=True)
                        tl["g"][b].record(hi)
                        if schedule != "deferred":
                            wait_all(b, side)
                            tl["d"][b] = torch.cuda.Event(enable_timing=True)
                            tl["d"][b].record(side)
                    if schedule == "naive" and args.residency == "device":
                        wait_all(b, hi)                         # handler not overlapped
                if schedule == "deferred":
                    arm()
            if schedule != "bwd":
                R.ratel_sync(hi)

    def init(mc, staging):
        cfg.max_ctas = mc
        cfg.host_threads = args.host_threads
        cfg.cta_tiles = args.cta_tiles
        cfg.k1_kernel = args.k1_kernel
        if args.tile_elems:
            cfg.tile_elems = args.tile_elems
        cfg.staging = staging
        R.ratel_init(0, 0, 1, None, cfg)
        for parts in lib.values():
            for i, x, c in parts:
                R.ratel_register_block(i, [x], c)
        t_state["t"] = 1

    for tokens in args.tokens:
        bw = SynthBackward(dev, h, tokens, model.p16, ring, vocab)
        for mc in args.max_ctas:
            # cuBLAS SM carve-out: the backward GEMMs size their grids for
            # SMs - mc, leaving mc SMs to the update kernel (max_ctas = mc)
            if args.carveout:
                torch._C._set_sm_carveout_experimental(mc if mc > 0 else None)
            times = {}
            # the backward alone is timed again after the optimizer schedules: its speed
            # drifts once the optimizer has run (power management), so the baseline is the mean
            scheds = list(args.schedules) + (["bwd_after"] if "bwd" in args.schedules else [])
            for sch in scheds:
                if sch == "deferred" and args.ring < len(sizes):
                    continue
                staging = R.RATEL_STAGING_SERIALIZED if (sch == "naive" and args.residency == "host") \
                    else (R.RATEL_STAGING_ZERO_COPY if args.zero_copy else R.RATEL_STAGING_PIPELINED)
                init(mc, staging)
                run_sch = "bwd" if sch == "bwd_after" else sch
                for _ in range(args.warmup):
                    one(run_sch, bw)
                torch.cuda.synchronize()
                R.ratel_kernel_timing(reset=True)
                sampler = bench.ClockSampler(bench.gpu_uuid(torch, dev))
                time.sleep(0.6)
                w0 = time.time()
                e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
                e0.record(hi)
                for _ in range(args.steps):
                    one(run_sch, bw)
                e1.record(hi)
                e1.synchronize()
                sampler.mark(w0, time.time())
                clk = sampler.stop() or {}
                k1_ms, _ = R.ratel_kernel_timing(reset=True)
                if args.timeline and sch in ("ago", "naive"):
                    one(sch, bw, timeline=True)
                    torch.cuda.synchronize()
                    t0 = tl["t0"]
                    print(json.dumps({"timeline": sch, "tokens": tokens,
                                      "grad_ready_ms": {b: round(t0.elapsed_time(e), 1) for b, e in tl["g"].items()},
                                      "update_done_ms": {b: round(t0.elapsed_time(e), 1) for b, e in tl["d"].items()}}),
                          flush=True)
                times[sch] = (e0.elapsed_time(e1) / args.steps, k1_ms / args.steps, clk.get("sm_mhz"),
                              clk.get("power_w"))
                R.ratel_finalize()
            tb = times["bwd"][0] if "bwd_after" not in times else 0.5 * (times["bwd"][0] + times["bwd_after"][0])
            row = {"residency": args.residency + (f" {args.hybrid_gpu_frac}" if hybrid else ""),
                   "host_threads": args.host_threads, "granularity": args.granularity, "cta_tiles": args.cta_tiles,
                   "k1_kernel": args.k1_kernel, "bwd_priority": args.bwd_priority, "ring": args.ring,
                   "group": args.group,
                   "tile_elems": args.tile_elems, "zero_copy": bool(args.zero_copy),
                   "tokens": tokens, "max_ctas": mc,
                   "carveout": bool(args.carveout),
                   "blocks": len(sizes),
                   "params": sum(sizes), "bwd_ms": tb,
                   "bwd_ms_before_after": [times["bwd"][0], times["bwd_after"][0]] if "bwd_after" in times else None, "bwd_tflops": 4 * sum(sizes) * tokens / (tb / 1e3) / 1e12}
            for sch, v in times.items():
                row[f"{sch}_sm_mhz"], row[f"{sch}_power_w"] = v[2], v[3]
            if "opt" in times:
                row["opt_ms"] = times["opt"][0]
                if args.residency == "host":
                    row["opt_host_link_gbs"] = 24 * sum(sizes) / (times["opt"][0] / 1e3) / 1e9
            for sch in ("ago", "deferred", "naive"):
                if sch in times:
                    row[f"{sch}_ms"] = times[sch][0]
                    row[f"{sch}_exposed_ms"] = times[sch][0] - tb
                    row[f"{sch}_k1_ms"] = times[sch][1]
            print(json.dumps(row), flush=True)
        del bw
        torch.cuda.empty_cache()


if __name__ == "__main__":
    ap = argparse.ArgumentParser()
    ap.add_argument("--shape", default="13B")
    ap.add_argument("--blocks", type=int, default=0)
    ap.add_argument("--residency", default="device", choices=["device", "host", "hostcompute", "hybrid"])
    ap.add_argument("--host-threads", type=int, default=0, help="cfg.host_threads (CPU handler threads, 0 = default)")
    ap.add_argument("--hybrid-gpu-frac", type=float, default=0.3,
                    help="hybrid: fraction of each unit GPU-streamed; the rest goes to the CPU handler")
    ap.add_argument("--tokens", type=int, nargs="+", default=[2048, 8192, 32768])
    ap.add_argument("--max-ctas", type=int, nargs="+", default=[0, 32])
    ap.add_argument("--schedules", nargs="+", default=["bwd", "opt", "ago", "deferred", "naive"])
    ap.add_argument("--ring", type=int, default=3)
    ap.add_argument("--group", type=int, default=1,
                    help="hand blocks off in bursts of this many (fewer GEMM/update interleave points; "
                         "needs --ring >= 2 * group)")
    ap.add_argument("--steps", type=int, default=3)
    ap.add_argument("--warmup", type=int, default=1)
    ap.add_argument("--timeline", action="store_true", help="per-block grad-ready / update-done times")
    ap.add_argument("--carveout", action="store_true", help="cuBLAS SM carve-out = max_ctas for the backward")
    ap.add_argument("--cta-tiles", type=int, default=0, help="cfg.cta_tiles (0 = persistent update grid)")
    ap.add_argument("--k1-kernel", type=int, default=0, help="cfg.k1_kernel: 0 TMA, 1 LDG, 2 LDG_LITE")
    ap.add_argument("--tile-elems", type=int, default=0, help="cfg.tile_elems (pinned-host tile ring)")
    ap.add_argument("--zero-copy", action="store_true", help="pinned-host: RATEL_STAGING_ZERO_COPY")
    ap.add_argument("--bwd-priority", type=int, default=-2,
                    help="torch stream priority of the synthetic backward (0 = default streams = the optimizer's)")
    ap.add_argument("--granularity", default="block", choices=["block", "tensor"],
                    help="hand-off unit: a transformer block, or each of its four linears")
    run(ap.parse_args())
