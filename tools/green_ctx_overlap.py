"""Device-resident AGO with a green-context SM partition.

The synthetic backward's GEMMs run in a CUDA green context holding
148 - k SMs (torch.cuda.GreenContext, cuBLAS inside it); the library stays in
the primary context with its update kernel capped at k CTAs (cfg.max_ctas),
so the update has k SMs the GEMMs can never take -- a hard spatial
partition, unlike round 1's cuBLAS SM carve-out (which only sizes the GEMM
grids).  Events do not cross contexts for recording, so every hand-off goes
through a primary-context relay stream that waits on an event recorded in
the green context; ring recycling goes the other way (ratel_block_wait on a
primary stream, the green stream waits on its event).

    python tools/green_ctx_overlap.py [--blocks 8] [--tokens 8192 32768] [--sms 8 16 32]

One JSON line per (tokens, k): backward alone (green), optimizer alone, AGO
step, exposed = AGO - backward; plus the same with no partition (k = 0).
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


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--blocks", type=int, default=8)
    ap.add_argument("--tokens", type=int, nargs="+", default=[8192, 32768])
    ap.add_argument("--sms", type=int, nargs="+", default=[8, 16, 32])
    ap.add_argument("--reps", type=int, default=3)
    ap.add_argument("--residency", default="device", choices=["device", "host"],
                    help="host: pinned-host states, per-tensor hand-off (the tile updates capped at k CTAs)")
    args = ap.parse_args()
    from torch.cuda.green_contexts import SUPPORTED, GreenContext
    if not SUPPORTED:
        print(json.dumps({"error": "torch built without green context support"}))
        return
    dev = torch.device("cuda:0")
    torch.cuda.set_device(dev)
    nsm = torch.cuda.get_device_properties(dev).multi_processor_count
    L, h = bench.SHAPES["13B"]
    sizes = bench.model_blocks("13B", with_embedding=False)[:args.blocks]
    cfg = R.ratel_default_config()
    R.ratel_init(0, 0, 1, None, cfg)
    model = bench.Model(R, torch, dev, sizes, 1, 0, args.residency, grad_ring=3)
    R.ratel_finalize()
    host = args.residency == "host"
    K = 4 if host else 1                # per-tensor units for the pinned-host path
    units = {}
    for b, n in enumerate(sizes):
        if not host:
            units[b] = [model.ranges[b]]
            continue
        r0, offs, off = model.ranges[b], [], 0
        for (o, i) in bench.linears(h):
            offs.append([off, o * i])
            off += o * i
        offs[-1][1] += n - off
        units[b] = [R.ratel_range(r0.param_bf16 + 2 * o, r0.grad_bf16 + 2 * o, 0, r0.master + 4 * o,
                                  r0.exp_avg + 4 * o, r0.exp_avg_sq + 4 * o, ln, 1) for o, ln in offs]
    order = list(reversed(range(len(sizes))))
    nr = 3
    relay = torch.cuda.Stream()         # primary-context hand-off stream
    relay2 = torch.cuda.Stream()        # primary-context ring-recycling stream
    out = []
    for T in args.tokens:
        bw = bench.SynthBackward(dev, h, T, model.p16, model.grad_ring, 0, chunk=65536 if host else 16384)
        for k in [0] + list(args.sms):
            gc = GreenContext.create(nsm - k, 0) if k > 0 else None
            cfg = R.ratel_default_config()
            cfg.max_ctas = k
            R.ratel_init(0, 0, 1, None, cfg)
            try:
                for b in range(len(sizes)):
                    for j, r in enumerate(units[b]):
                        R.ratel_register_block(b * K + j, [r], R.RATEL_PINNED_HOST if host else R.RATEL_DEVICE)
                t = [1]

                def arm():
                    R.ratel_adam_step(1e-3, 0.9, 0.999, 1e-8, 1e-2, t[0])
                    t[0] += 1

                def in_green(fn):
                    if gc is None:
                        return fn(torch.cuda.current_stream())
                    gc.set_context()
                    try:
                        return fn(gc.Stream())
                    finally:
                        gc.pop_context()

                def bwd_only():
                    def f(s):
                        with torch.cuda.stream(s):
                            for b in order:
                                bw.block(b, b % nr)
                        ev = torch.cuda.Event()
                        ev.record(s)
                        return ev
                    relay.wait_event(in_green(f))

                def ago():
                    arm()
                    for j, b in enumerate(order):
                        if j >= nr:                       # the ring slot's previous update ran
                            for q in range(K):
                                R.ratel_block_wait((b + nr) * K + q, relay2)
                            ev_free = torch.cuda.Event()
                            ev_free.record(relay2)
                        else:
                            ev_free = None

                        def f(s, b=b, ev_free=ev_free):
                            # every library call happens after the context is popped: the
                            # per-linear events are collected here and relayed below (the
                            # GEMMs are already enqueued, so the GPU timeline is the same)
                            if ev_free is not None:
                                s.wait_event(ev_free)
                            evs = []

                            def on_linear(q, s=s, b=b):
                                ev = torch.cuda.Event()
                                ev.record(s)
                                evs.append((b * K + q, ev))
                            with torch.cuda.stream(s):
                                bw.block(b, b % nr, on_linear=on_linear if host else None)
                            ev = torch.cuda.Event()
                            ev.record(s)
                            return evs or [(b, ev)]
                        for uid, ev in in_green(f):
                            relay.wait_event(ev)
                            R.ratel_offload_grad_chunk(uid, relay)
                    R.ratel_sync(relay)

                def opt():
                    arm()
                    for b in order:
                        for q in range(K):
                            R.ratel_offload_grad_chunk(b * K + q, relay)
                    R.ratel_sync(relay)

                def timed(fn):
                    torch.cuda.synchronize()
                    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
                    e0.record(relay)
                    fn()
                    e1.record(relay)
                    e1.synchronize()
                    torch.cuda.synchronize()
                    return e0.elapsed_time(e1)

                bwd_only()
                ago()
                opt()
                t_opt = min(timed(opt) for _ in range(2))
                b_runs, a_runs = [timed(bwd_only)], []
                for _ in range(args.reps):
                    a_runs.append(timed(ago))
                    b_runs.append(timed(bwd_only))
                base = [0.5 * (b_runs[i] + b_runs[i + 1]) for i in range(args.reps)]
                exp = sorted(a - b for a, b in zip(a_runs, base))
                row = {"residency": args.residency, "tokens": T, "green_sms_backward": nsm - k if k else nsm,
                       "update_ctas": k or "all",
                       "blocks": len(sizes), "backward_ms": sorted(base)[len(base) // 2], "optimizer_alone_ms": t_opt,
                       "ago_ms": sorted(a_runs)[len(a_runs) // 2], "exposed_ms": exp[len(exp) // 2],
                       "exposed_ms_spread": [exp[0], exp[-1]], "backward_ms_runs": b_runs}
                print(json.dumps(row), flush=True)
                out.append(row)
            finally:
                R.ratel_finalize()
        del bw
        torch.cuda.empty_cache()


if __name__ == "__main__":
    main()
