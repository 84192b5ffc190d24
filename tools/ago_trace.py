"""Kernel-level timeline of one AGO step overlapped with the synthetic backward
(device-resident), from CUPTI via torch.profiler -- where does the exposed
optimizer time come from?

    python tools/ago_trace.py [--blocks 8] [--tokens 8192] [--k1-kernel 0] [--cta-tiles 0]

Runs the backward alone and the AGO step (arm, then per block: GEMMs, hand-off)
under the profiler and prints one JSON line with, per schedule: the step's
span, the summed duration of the backward GEMM kernels, the summed duration of
the update kernels, and the time during which both kinds ran at once.  The
GEMM slowdown under overlap is (sum of GEMM time in AGO) / (sum alone).
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


def intervals(events, pred):
    return sorted((e["ts"], e["ts"] + e["dur"]) for e in events if pred(e["name"]))


def union(iv):
    tot, cur = 0.0, None
    for a, b in iv:
        if cur is None or a > cur[1]:
            if cur:
                tot += cur[1] - cur[0]
            cur = [a, b]
        else:
            cur[1] = max(cur[1], b)
    if cur:
        tot += cur[1] - cur[0]
    return tot


def overlap(iv1, iv2):
    """Time (us) during which some interval of iv1 and some of iv2 are both active."""
    pts = sorted([(a, 0, +1) for a, _ in iv1] + [(b, 0, -1) for _, b in iv1] +
                 [(a, 1, +1) for a, _ in iv2] + [(b, 1, -1) for _, b in iv2])
    c = [0, 0]
    last, tot = None, 0.0
    for t, k, d in pts:
        if last is not None and c[0] > 0 and c[1] > 0:
            tot += t - last
        c[k] += d
        last = t
    return tot


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--blocks", type=int, default=8)
    ap.add_argument("--tokens", type=int, default=8192)
    ap.add_argument("--k1-kernel", type=int, default=0)
    ap.add_argument("--cta-tiles", type=int, default=0)
    ap.add_argument("--trace", default="")
    args = ap.parse_args()
    dev = torch.device("cuda:0")
    L, h = bench.SHAPES["13B"]
    sizes = bench.model_blocks("13B")[:args.blocks]
    cfg = R.ratel_default_config()
    R.ratel_init(0, 0, 1, None, cfg)
    model = bench.Model(R, torch, dev, sizes, 1, 0, "device", grad_ring=3)
    R.ratel_finalize()
    cfg.k1_kernel, cfg.cta_tiles = args.k1_kernel, args.cta_tiles
    R.ratel_init(0, 0, 1, None, cfg)
    for b in range(len(sizes)):
        R.ratel_register_block(b, [model.ranges[b]], R.RATEL_DEVICE)
    bw = bench.SynthBackward(dev, h, args.tokens, model.p16, model.grad_ring, 0)
    s = torch.cuda.Stream(priority=-2)
    order = list(reversed(range(len(sizes))))
    t = [1]

    def bwd():
        with torch.cuda.stream(s):
            for b in order:
                bw.block(b, b % 3)

    def ago():
        R.ratel_adam_step(1e-3, 0.9, 0.999, 1e-8, 1e-2, t[0])
        t[0] += 1
        with torch.cuda.stream(s):
            for j, b in enumerate(order):
                if j >= 3:
                    R.ratel_block_wait(b + 3, s)
                bw.block(b, b % 3)
                R.ratel_offload_grad_chunk(b, s)
        R.ratel_sync(s)

    flush = torch.empty(256 << 20, dtype=torch.uint8, device=dev)

    def bwd_flush():
        """backward with a 256 MB memset (> L2) after every block: the L2
        disturbance of an update without its HBM time or power"""
        with torch.cuda.stream(s):
            for b in order:
                bw.block(b, b % 3)
                flush.fill_(b & 1)

    def opt():
        R.ratel_adam_step(1e-3, 0.9, 0.999, 1e-8, 1e-2, t[0])
        t[0] += 1
        for b in order:
            R.ratel_offload_grad_chunk(b, s)
        R.ratel_sync(s)

    out = {"blocks": len(sizes), "tokens": args.tokens, "k1_kernel": args.k1_kernel, "cta_tiles": args.cta_tiles}
    for name, fn in (("bwd", bwd), ("bwd_flush", bwd_flush), ("opt", opt), ("ago", ago)):
        for _ in range(2):
            fn()
        torch.cuda.synchronize()
        with torch.profiler.profile(activities=[torch.profiler.ProfilerActivity.CUDA]) as prof:
            fn()
            torch.cuda.synchronize()
        path = args.trace or f"/tmp/ago_trace_{name}.json"
        prof.export_chrome_trace(path)
        ev = [e for e in json.load(open(path))["traceEvents"] if e.get("ph") == "X" and e.get("cat") == "kernel"]
        is_upd = lambda n: "adam_update" in n
        is_gemm = lambda n: not is_upd(n) and "elementwise" not in n and "fill" not in n.lower()
        g, u = intervals(ev, is_gemm), intervals(ev, is_upd)
        span = (max(e["ts"] + e["dur"] for e in ev) - min(e["ts"] for e in ev)) if ev else 0.0
        out[name] = {"span_ms": span / 1e3, "gemm_sum_ms": sum(b - a for a, b in g) / 1e3,
                     "gemm_union_ms": union(g) / 1e3, "update_sum_ms": sum(b - a for a, b in u) / 1e3,
                     "update_union_ms": union(u) / 1e3, "both_active_ms": overlap(g, u) / 1e3,
                     "gemm_kernels": len(g), "update_kernels": len(u)}
    out["gemm_slowdown"] = out["ago"]["gemm_sum_ms"] / out["bwd"]["gemm_sum_ms"]
    out["gemm_slowdown_l2_flush"] = out["bwd_flush"]["gemm_sum_ms"] / out["bwd"]["gemm_sum_ms"]
    out["update_slowdown"] = out["ago"]["update_sum_ms"] / max(out["opt"]["update_sum_ms"], 1e-9)
    print(json.dumps(out), flush=True)
    R.ratel_finalize()


if __name__ == "__main__":
    main()
