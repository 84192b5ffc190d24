#!/usr/bin/env python
"""bench.py -- params updated/sec of the AGO AdamW step on B200.

One "step" = one pass of the whole hot path over the model
states: ratel_adam_step(t), one ratel_offload_grad_chunk per block in
decreasing block order (the order backward produces them, PAPER.md
P:L1038-1041), ratel_sync.  Default workload at N=1: BASELINE.json
configs[1], the 13B GPT model states of Table IV resident in
HBM.  With N>1 (torchrun) the same 13B states are range-sharded over the
ranks (strong scaling) with the per-block bf16 all-gather over NCCL.

Printed: ONE JSON line on rank 0.
  value      params/s over the timed region (device clock, max over ranks)
  e2e        same metric through the C ABI with HOST buffers: states in
             pinned host memory streamed by the library's tile ring, grads
             H2D from pinned host and P16 D2H, all inside the timed region
  roofline   the update kernel K1: 28 algorithmic B/param / its event-timed
             launch durations vs MEASURED_PEAKS.json hbm_gbs (pinned-host
             states: 24 B/param over the host link vs this run's duplex
             probe; HOST_COMPUTE: 32 B/param of host DRAM vs this run's
             host_stream probe -- K1's numbers then under roofline.k1)
  cpu_baseline  the CPU oracle on a whole 13B block per pass, on this host's cores
  overlap    (N=1) device-resident C2 sweep, 1K-64K tokens: AGO vs deferred vs
             backward alone, 3 bracketed repetitions, NVML energy
  overlap_host / overlap_hostcompute  (N=1) pinned-host states of 16 x 13B
             blocks, per-tensor hand-off, 32K-192K tokens, 3 bracketed reps
  multi_gpu  (N>1) NCCL all-gather busbw at the C3 / workload slices, the 8-byte
             allreduce latency, all-rank host-link probe, all-rank P16 equality,
             NCCL init log summary; roofline.nvlink and roofline.step_bounds_ms
`--impl reference` times the oracle as the reference arm.  `--gpus N` outside
torchrun re-launches this script under torch.distributed.run (N ranks).
"""
from __future__ import annotations

import argparse
import datetime
import json
import math
import os
import subprocess
import sys
import threading
import time

ROOT = os.path.dirname(os.path.abspath(__file__))
if ROOT not in sys.path:
    sys.path.insert(0, ROOT)

METRIC = "params updated/sec (Adam step) and % of HBM / host-link roofline at 1/2/4/8 B200"
UNIT = "params/s"
VOCAB, SEQ = 50257, 1024
# Table IV: name -> (layers, hidden)
SHAPES = {"c1": (1, 256), "13B": (40, 5120), "30B": (48, 7168), "70B": (80, 8192), "175B": (96, 12288)}
HP = dict(lr=1e-3, beta1=0.9, beta2=0.999, eps=1e-8, weight_decay=1e-2)   # torch defaults (R14)
BYTES_PER_PARAM = 28                        # g 2 + theta/m/v 12 read; theta/m/v 12 + p 2 write


def block_params(h: int) -> int:
    return 12 * h * h + 13 * h


def embed_params(h: int) -> int:
    return VOCAB * h + SEQ * h + 2 * h


def model_blocks(shape: str, with_embedding: bool = True):
    L, h = SHAPES[shape]
    sizes = [block_params(h)] * L
    if with_embedding and shape != "c1":
        sizes.append(embed_params(h))      # handed off last (R10)
    return sizes


# --------------------------------------------------------------- helpers
def peaks():
    try:
        with open(os.path.join(ROOT, "MEASURED_PEAKS.json")) as f:
            p = json.load(f)
        return float(p["hbm_gbs"]), "measured"
    except Exception:
        return 6650.0, "fallback"


def ncu_summary():
    """K1's committed ncu --set full summary (profiles/k1_ncu_summary.json), if any."""
    try:
        with open(os.path.join(ROOT, "profiles", "k1_ncu_summary.json")) as f:
            return json.load(f)
    except Exception:
        return {}


def ncu_traffic_per_param():
    """dram bytes per param of K1 from the committed ncu summary, if any."""
    v = ncu_summary().get("dram_bytes_per_param")
    return float(v) if v is not None else None


class ClockSampler:
    """nvidia-smi clocks / throttle reasons sampled during the timed region."""
    Q = ("clocks.sm,clocks.max.sm,power.draw,clocks_event_reasons.hw_slowdown,"
         "clocks_event_reasons.hw_thermal_slowdown,clocks_event_reasons.sw_thermal_slowdown,"
         "clocks_event_reasons.sw_power_cap")
    NAMES = ["hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown", "sw_power_cap"]

    def __init__(self, gpu_id: str):
        self.samples = []
        self.window = None
        try:
            self.p = subprocess.Popen(["nvidia-smi", f"--query-gpu={self.Q}", "--format=csv,noheader,nounits",
                                       "-i", gpu_id, "-lms", "100"], stdout=subprocess.PIPE,
                                      stderr=subprocess.DEVNULL, text=True)
            self.t = threading.Thread(target=self._read, daemon=True)
            self.t.start()
        except Exception:
            self.p = None

    def _read(self):
        for line in self.p.stdout:
            self.samples.append((time.time(), [x.strip() for x in line.split(",")]))

    def mark(self, t0, t1):
        self.window = (t0, t1)

    BAD = ("hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown")

    def stop(self):
        if self.p is None:
            return None
        time.sleep(0.25)
        self.p.terminate()
        try:
            self.p.wait(timeout=5)
        except Exception:
            self.p.kill()
        return self.stats()

    def stats(self, window=None):
        """Clock summary of the samples inside `window` (default: the marked one)."""
        if self.p is None:
            return None
        t0, t1 = window or self.window or (0, 1e30)
        rows = [r for (t, r) in self.samples if t0 - 0.05 <= t <= t1 + 0.15 and len(r) >= 7]
        if not rows:
            rows = [r for (_, r) in self.samples if len(r) >= 7][-3:]
        if not rows:
            return None
        sm = sorted(float(r[0]) for r in rows if r[0].replace(".", "").isdigit())
        pw = sorted(float(r[2]) for r in rows if r[2].replace(".", "").isdigit())
        reasons = sorted({self.NAMES[i] for r in rows for i in range(4) if r[3 + i].lower() == "active"})
        return {"sm_mhz": sm[len(sm) // 2] if sm else None, "sm_max_mhz": float(rows[0][1]),
                "power_w": pw[len(pw) // 2] if pw else None, "reasons": reasons, "samples": len(rows)}


def gpu_uuid(torch, dev):
    try:
        return "GPU-" + str(torch.cuda.get_device_properties(dev).uuid)
    except Exception:
        return str(dev)


# ------------------------------------------------------ reference arm (oracle)
def cpu_facts():
    """Host CPU model, socket and NUMA-node counts (the oracle's machine)."""
    model, sockets = None, set()
    try:
        with open("/proc/cpuinfo") as f:
            for line in f:
                k, _, v = line.partition(":")
                k = k.strip()
                if k == "model name" and model is None:
                    model = v.strip()
                elif k == "physical id":
                    sockets.add(v.strip())
    except OSError:
        pass
    try:
        numa = len([d for d in os.listdir("/sys/devices/system/node") if d.startswith("node") and d[4:].isdigit()])
    except OSError:
        numa = None
    return {"cpu_model": model, "sockets": len(sockets) or None, "numa_nodes": numa, "nproc": os.cpu_count()}


_ORACLE_INPUTS = {}


def oracle_inputs(n: int):
    """theta0 and two bf16 gradient draws of an n-element sample of block 0
    (synth/, the seeded recipe).  Large samples repeat a 2^25-element draw
    (the generator is numpy: ~1 s per 2^25 draws, so drawing a whole 13B
    block would take longer than timing it); only the update is timed."""
    if n not in _ORACLE_INPUTS:
        import numpy as np
        import synth
        k = min(n, 1 << 25)
        th = synth.theta0(k, block=0)
        gs = [synth.grad16(k, step=t, block=0) for t in (1, 2)]
        if n > k:
            reps = -(-n // k)
            th = np.tile(th, reps)[:n]
            gs = [np.tile(g, reps)[:n] for g in gs]
        _ORACLE_INPUTS.clear()
        _ORACLE_INPUTS[n] = (th, gs)
    return _ORACLE_INPUTS[n]


def oracle_sample_rate(n: int, steps: int, threads: int, min_seconds: float = 0.0, warmup: int = 1):
    """Time the CPU oracle's update (oracle/, as it stands) over an n-element
    sample of block 0 of the workload: `warmup` untimed passes (first touch),
    then at least `steps` timed passes and `min_seconds`.  Returns
    (params/s, passes, seconds)."""
    import oracle
    th, gs = oracle_inputs(n)
    r = oracle.Range.fresh(th)
    r.theta_bar = r.m_bar = None          # the product's 28 B/param, no tolerance scales
    t = 1
    for _ in range(warmup):
        oracle.adam_range(r, gs[t % 2], oracle.hparams(step=t), threads=threads)
        t += 1
    done, t0 = 0, time.perf_counter()
    while done < steps or (time.perf_counter() - t0) < min_seconds:
        oracle.adam_range(r, gs[t % 2], oracle.hparams(step=t), threads=threads)
        done += 1
        t += 1
    dt = time.perf_counter() - t0
    return n * done / dt, done, dt


def host_threads():
    try:
        return len(os.sched_getaffinity(0))
    except Exception:
        return os.cpu_count() or 1


def oracle_baseline(n: int, steps: int, warmup: int, threads: int, min_seconds: float = 0.0):
    """cpu_baseline object: the oracle on an n-element sample at `threads`
    threads, with the host facts and the DRAM rate its 28 B/param imply."""
    v, done, dt = oracle_sample_rate(n, steps, threads, min_seconds=min_seconds, warmup=warmup)
    out = {"value": v, "unit": UNIT, "cores": threads, "kind": "oracle",
           "sample": f"{n:,} params of block 0 (one 13B block = 314,639,360), {done} timed passes in {dt:.2f} s "
                     f"after {warmup} untimed, OpenMP {threads} threads",
           "sample_params": n, "sample_passes": done, "sample_ms_per_pass": 1e3 * dt / done,
           "dram_gbs_at_28B_per_param": 28 * v / 1e9}
    out.update(cpu_facts())
    return out


def run_reference(args, rank, world):
    """The reference arm: the oracle as it stands on this host's cores.  One
    step = one oracle pass over a bounded sample of the workload (default
    one whole 13B block); ms_per_step is that pass, as timed."""
    if rank != 0:
        return                               # under torchrun rank 0 alone runs and prints
    n = args.oracle_sample
    threads = host_threads()
    cb = oracle_baseline(n, args.steps, args.warmup, threads)
    v = cb["value"]
    cfg = workload_config(args, world)
    print(json.dumps({
        "impl": "reference", "metric": METRIC, "value": v, "unit": UNIT, "n_gpus": world,
        "steps": cb["sample_passes"], "warmup": args.warmup, "ms_per_step": cb["sample_ms_per_pass"],
        "higher_is_better": True, "scaling": "strong", "vs_baseline": None,
        "dtype": "f64", "data": "synthetic", "config": cfg,
        "step": f"one oracle pass over a {n:,}-param sample of the workload ({cfg['params']:,} params)",
        "full_workload_ms_per_step_extrapolated": 1e3 * cfg["params"] / v,
        "cpu_baseline": cb,
        "e2e": {"value": v, "unit": UNIT, "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0},
    }), flush=True)


# --------------------------------------------------------------- workload
def workload_config(args, world):
    shape = args.shape
    sizes = model_blocks(shape)
    if args.blocks:
        sizes = sizes[:args.blocks]
    P = sum(sizes)
    resid = {"host": "pinned-host", "hostcompute": "pinned-host, CPU handler (HOST_COMPUTE)",
             "hybrid": f"pinned-host, {args.hybrid_gpu_frac:.2f} of each block GPU-streamed + the rest by the CPU "
                       f"handler"}.get(args.residency, "device")
    name = {"13B": "13B", "30B": "30B", "70B": "70B (Table IV shape, 64.9B)", "175B": "175B",
            "c1": "C1 tiny block"}[shape]
    leff = (f", L_eff = {len(sizes)} of {len(model_blocks(shape))} blocks sized to this box"
            if getattr(args, "blocks_auto", False) else "")
    return {"workload": f"{name} GPT model states ({len(sizes)} blocks), {resid}-resident, AdamW, "
                        f"per-block AGO hand-off" + (", clip" if args.clip > 0 else "") + leff,
            "params": P, "blocks": len(sizes), "block_params": sizes[0], "residency": resid,
            "parallelism": (f"range-sharded x{world}" + (" (fused peer-store all-gather)" if args.fused_allgather else
                                                          " (NCCL all-gather)")
                            + (" [test mode: all ranks on cuda:0, NCCL over loopback sockets]" if args.share_gpu
                               else "")
                            + (" [test mode: all ranks on one GPU, no NCCL, P16 slices not exchanged]"
                               if args.sim_comm_none else "")) if world > 1 else "single GPU",
            "l2": "inputs larger than L2 (working set >> 126 MB)", "hyperparameters": HP,
            "max_grad_norm": args.clip, "update_streams": args.update_streams, "cta_tiles": args.cta_tiles,
            **({"clip_schedule": "K2 (sum of g^2 partials, 2 B/param) at every hand-off, overlapping backward; "
                                 "K3 + the norm allreduce and K1 of EVERY block only after the last hand-off "
                                 "(the global norm needs all gradients): the update cannot overlap backward"}
               if args.clip > 0 else {}),
            "k1_kernel": ["tma", "ldg", "ldg_lite"][args.k1_kernel], "staging": args.staging}


class PinnedArena:
    """One exact-size page-locked host buffer from ratel_alloc_pinned
    (cudaHostAlloc): torch's pinned allocator rounds large blocks up, which
    would not fit 100+ GB of host states into the box's RAM."""

    def __init__(self, torch, nfloats):
        import paper_conf_icde_liaosyxcyww25_b200 as R
        self.torch = torch
        self.owner = R.pinned_tensor(max(nfloats, 8))
        self.t = self.owner.tensor
        self.t.zero_()
        self.off = 0

    def take(self, n):
        v = self.t[self.off:self.off + n]
        self.off += (n + 7) // 8 * 8          # keep every slice 32-byte aligned
        return v

    def close(self):
        if self.t is not None:
            self.torch.cuda.synchronize()
            self.t = None
            self.owner = None   # ratel_free_pinned

    __del__ = close


class Model:
    """Synthetic model states of one rank: per block one flat range.
    symm=True allocates P16 in memory every rank maps, for the fused update +
    all-gather (ratel_register_peer_params): torch symmetric memory, or with
    peer_memory="ipc" plain allocations opened through CUDA IPC handles (ranks
    sharing a GPU, where symmetric memory refuses)."""

    def __init__(self, R, torch, dev, sizes, world, rank, residency, grad_ring=2, pin_grads=False, symm=False,
                 peer_memory="symm"):
        self.sizes = sizes
        self.ranges = []
        self.keep = []
        self.slices = []
        cap_max = max(R.ratel_padded_numel(n, world) for n in sizes)
        self.grad_ring = [torch.empty(cap_max, dtype=torch.bfloat16, device=dev) for _ in range(grad_ring)]
        for i, g in enumerate(self.grad_ring):
            key = R.ratel_gen_stream_key(0x5EED5EED, 2, 1, i)
            R.ratel_gen_grad16(g.data_ptr(), cap_max, 0, key)
        self.p16 = []
        self.peer_ptrs = []
        self.arenas = []
        if residency != "device":
            own_total = 0
            for n in sizes:
                beg, end = R.ratel_rank_slice(n, world, rank)
                own_total += (max(end - beg, 8) + 7) // 8 * 8
            self.arenas = [PinnedArena(torch, own_total) for _ in range(3)]
        for b, n in enumerate(sizes):
            cap = R.ratel_padded_numel(n, world)
            beg, end = R.ratel_rank_slice(n, world, rank)
            s = max(end - beg, 8)
            if symm and peer_memory == "ipc":
                import torch.distributed as dist
                from torch.multiprocessing.reductions import reduce_tensor
                p = torch.zeros(cap, dtype=torch.bfloat16, device=dev)
                torch.cuda.synchronize()
                allh = [None] * world
                dist.all_gather_object(allh, reduce_tensor(p))
                ptrs = []
                for q, h in enumerate(allh):
                    t = p if q == rank else h[0](*h[1])
                    self.keep.append(t)            # the peer mappings live as long as the model
                    ptrs.append(t.data_ptr())
                self.peer_ptrs.append(ptrs)
            elif symm:
                import torch.distributed as dist
                import torch.distributed._symmetric_memory as symm_mem
                p = symm_mem.empty(cap, dtype=torch.bfloat16, device=dev)
                p.zero_()
                hdl = symm_mem.rendezvous(p, dist.group.WORLD.group_name)
                self.keep.append(hdl)          # the peer mappings live as long as the model
                self.peer_ptrs.append(list(hdl.buffer_ptrs))
            else:
                p = torch.zeros(cap, dtype=torch.bfloat16, device=dev)
            if residency == "device":
                th = torch.empty(s, dtype=torch.float32, device=dev)
                m = torch.zeros(s, dtype=torch.float32, device=dev)
                v = torch.zeros(s, dtype=torch.float32, device=dev)
                R.ratel_gen_theta0(th.data_ptr(), end - beg, beg, R.ratel_gen_stream_key(0x5EED5EED, 1, 0, b))
            else:
                tmp = torch.empty(s, dtype=torch.float32, device=dev)
                R.ratel_gen_theta0(tmp.data_ptr(), end - beg, beg, R.ratel_gen_stream_key(0x5EED5EED, 1, 0, b))
                th, m, v = (a.take(s) for a in self.arenas)
                th.copy_(tmp)
                del tmp
            g = self.grad_ring[b % grad_ring]
            self.ranges.append(R.make_range(p, g, th, m, v, n))
            self.keep.append((p, th, m, v))
            self.p16.append(p)
            self.slices.append((beg, end))
        torch.cuda.synchronize()


def linears(h):
    # (out, in) of QKV, proj, fc1, fc2 in the block's flat P16 buffer
    return [(3 * h, h), (h, h), (4 * h, h), (h, 4 * h)]


class SynthBackward:
    """Synthetic backward for the overlap measurement (harness, cuBLAS via
    torch): per block the dX and dW GEMMs of its four linears (4*P_blk*T
    FLOPs), dW written into the block's grad-ring slot.  `chunk`: at most this
    many tokens per GEMM (dW accumulated over chunks, like micro-batches), so
    large T fits beside 13B device-resident states; None = one chunk."""
    def __init__(self, dev, h, tokens, p16_views, grad_ring, vocab_rows, chunk=None):
        import torch
        self.h, self.T = h, tokens
        self.C = min(tokens, chunk) if chunk else tokens
        self.dev = dev
        g = torch.Generator(device=dev)
        g.manual_seed(1)
        mk = lambda *s: (torch.randn(*s, device=dev, dtype=torch.bfloat16, generator=g) * 0.01)
        C = self.C
        self.X = {1: mk(C, h), 4: mk(C, 4 * h)}
        self.dY = {3: mk(C, 3 * h), 1: mk(C, h), 4: mk(C, 4 * h)}
        self.dX = torch.empty(C, 4 * h, device=dev, dtype=torch.bfloat16)
        self.p16 = p16_views
        self.ring = grad_ring
        self.vocab_rows = vocab_rows
        self.dYv = mk(2048, vocab_rows) if vocab_rows else None

    def block(self, b, slot, on_linear=None):
        """GEMMs of block b; dW into ring slot `slot` (flat, same layout as P16).
        The linears run in backward order (fc2, fc1, proj, qkv); on_linear(j)
        is called after linear j's dW (per-tensor hand-off)."""
        import torch
        h, T, C = self.h, self.T, self.C
        P = self.p16[b]
        G = self.ring[slot]
        if b == len(self.p16) - 1 and self.vocab_rows:
            # embedding block (tied token embedding / LM head): dW[V, h] =
            # dY^T X accumulated over 2048-token chunks of the logits grad
            V = self.vocab_rows
            out = G[:V * h].view(V, h)
            X = self.X[1]
            out.zero_()
            for t0 in range(0, T, 2048):
                t1 = min(T, t0 + 2048)
                c0 = t0 % C
                c1 = c0 + (t1 - t0)
                if c1 > C:
                    c0, c1 = 0, t1 - t0
                out.addmm_(self.dYv[:t1 - t0].t(), X[c0:c1])
            return
        offs, off = [], 0
        for (o, i) in linears(h):
            offs.append(off)
            off += o * i
        for j in reversed(range(len(offs))):
            (o, i), off = linears(h)[j], offs[j]
            W = P[off:off + o * i].view(o, i)
            X = self.X[i // h]
            dY = self.dY[o // h]
            dW = G[off:off + o * i].view(o, i)
            for t0 in range(0, T, C):
                c = min(C, T - t0)
                torch.mm(dY[:c], W, out=self.dX[:c, :i])                    # dX = dY W
                if t0 == 0:
                    torch.mm(dY[:c].t(), X[:c], out=dW)                      # dW = dY^T X
                else:
                    dW.addmm_(dY[:c].t(), X[:c])                             # dW += dY^T X (next chunk)
            if on_linear is not None:
                on_linear(j)


class Energy:
    """GPU energy counter (NVML total energy, mJ) of the bench's device."""

    def __init__(self, uuid):
        self.h = None
        try:
            import pynvml
            pynvml.nvmlInit()
            self.nv = pynvml
            self.h = pynvml.nvmlDeviceGetHandleByUUID(uuid)
            self.nv.nvmlDeviceGetTotalEnergyConsumption(self.h)
        except Exception:
            self.h = None

    def joules(self):
        if self.h is None:
            return None
        return self.nv.nvmlDeviceGetTotalEnergyConsumption(self.h) / 1e3


def _med(xs):
    xs = sorted(x for x in xs if x is not None)
    if not xs:
        return None
    k = len(xs)
    return xs[k // 2] if k % 2 else 0.5 * (xs[k // 2 - 1] + xs[k // 2])


def _spread(xs):
    xs = [x for x in xs if x is not None]
    return [min(xs), max(xs)] if xs else None


def timed_run(torch, s, fn, energy=None):
    """One run of fn on stream s: (CUDA-event ms on s, joules or None)."""
    torch.cuda.synchronize()
    j0 = energy.joules() if energy else None
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record(s)
    fn()
    e1.record(s)
    e1.synchronize()
    torch.cuda.synchronize()
    j1 = energy.joules() if energy else None
    return e0.elapsed_time(e1), (j1 - j0 if j0 is not None and j1 is not None else None)


SIM_COMM_NONE = False   # --sim-comm-none: N ranks on ONE GPU, gloo group, no NCCL (test mode)


def init_lib(R, torch, dev_index, rank, world, cfg):
    uid = None
    if world > 1 and SIM_COMM_NONE:
        cfg.comm = R.RATEL_COMM_NONE   # P16 slices are not exchanged: a plumbing test, not a result
    elif world > 1:
        import torch.distributed as dist
        buf = torch.zeros(128, dtype=torch.uint8, device=f"cuda:{dev_index}")
        if rank == 0:
            buf.copy_(torch.frombuffer(bytearray(R.ratel_get_nccl_unique_id()), dtype=torch.uint8))
        dist.broadcast(buf, 0)
        uid = bytes(buf.cpu().numpy().tobytes())
    R.ratel_init(dev_index, rank, world, uid, cfg)


ARM_AFTER = False   # --arm after: the deferred "Ratel+ZeRO" order


def step_once(R, t, order, stream):
    if not ARM_AFTER:
        R.ratel_adam_step(HP["lr"], HP["beta1"], HP["beta2"], HP["eps"], HP["weight_decay"], t)
    for b in order:
        R.ratel_offload_grad_chunk(b, stream)
    if ARM_AFTER:
        R.ratel_adam_step(HP["lr"], HP["beta1"], HP["beta2"], HP["eps"], HP["weight_decay"], t)
    R.ratel_sync(stream)


def overlap_probe(args, R, torch, dev, model, sizes, order, t0, opt_ms, energy=None):
    """C2 batch sweep (the Fig. 7 analog): for
    each token count T the synthetic backward of the whole model alone, the
    AGO step (armed first, every block's update enqueued at its hand-off,
    grad ring recycled with ratel_block_wait) and the deferred "Ratel+ZeRO"
    step (backward, then the whole optimizer step), alternated
    `reps` times with the backward-alone baseline bracketing every repetition
    (mean of the runs before and after).  Per run: CUDA-event time on the
    backward stream and NVML energy.  Reported: medians and [min, max] over
    repetitions of exposed optimizer ms, backward slowdown % and J per step."""
    L, h = SHAPES[args.shape]
    ring = model.grad_ring
    vocab = VOCAB if len(sizes) == L + 1 else 0
    s = torch.cuda.Stream(device=dev, priority=-2)
    nr = len(ring)
    t = [t0]
    points = []
    for T in args.overlap_sweep:
        bw = SynthBackward(dev, h, T, model.p16, ring, vocab, chunk=16384)

        def bwd_only():
            with torch.cuda.stream(s):
                for b in order:
                    bw.block(b, b % nr)

        def arm():
            R.ratel_adam_step(HP["lr"], HP["beta1"], HP["beta2"], HP["eps"], HP["weight_decay"], t[0])
            t[0] += 1

        def ago():
            arm()
            with torch.cuda.stream(s):
                for j, b in enumerate(order):
                    if j >= nr:
                        R.ratel_block_wait(b + nr, s)       # ring slot consumed
                    bw.block(b, b % nr)
                    R.ratel_offload_grad_chunk(b, s)
            R.ratel_sync(s)

        def deferred():
            bwd_only()
            arm()
            for b in order:                                  # every update after the whole backward
                R.ratel_offload_grad_chunk(b, s)
            R.ratel_sync(s)

        bwd_only()                                           # warm-up (cuBLAS heuristics, clocks)
        ago()
        runs = {"bwd": [timed_run(torch, s, bwd_only, energy)], "ago": [], "deferred": []}
        for _ in range(args.overlap_reps):
            runs["ago"].append(timed_run(torch, s, ago, energy))
            runs["deferred"].append(timed_run(torch, s, deferred, energy))
            runs["bwd"].append(timed_run(torch, s, bwd_only, energy))
        base = [0.5 * (runs["bwd"][i][0] + runs["bwd"][i + 1][0]) for i in range(args.overlap_reps)]
        ebase = [0.5 * (runs["bwd"][i][1] + runs["bwd"][i + 1][1]) if runs["bwd"][i][1] is not None else None
                 for i in range(args.overlap_reps)]
        pt = {"tokens": T, "reps": args.overlap_reps, "backward_ms": _med(base), "backward_ms_spread": _spread(base),
              "backward_ms_runs": [r[0] for r in runs["bwd"]], "optimizer_alone_ms": opt_ms}
        for k in ("ago", "deferred"):
            exp = [runs[k][i][0] - base[i] for i in range(args.overlap_reps)]
            pt[f"{k}_step_ms"] = _med([r[0] for r in runs[k]])
            pt[f"{k}_exposed_ms"] = _med(exp)
            pt[f"{k}_exposed_ms_spread"] = _spread(exp)
            pt[f"{k}_backward_slowdown_pct"] = _med([100 * e / b for e, b in zip(exp, base)])
            pt[f"{k}_hidden_fraction"] = _med([1 - e / opt_ms for e in exp])
            if runs[k][0][1] is not None:
                pt[f"{k}_joules_per_step"] = _med([r[1] for r in runs[k]])
                pt[f"{k}_extra_joules_over_backward"] = _med([r[1] - e for r, e in zip(runs[k], ebase)])
        if runs["bwd"][0][1] is not None:
            pt["backward_joules"] = _med(ebase)
        points.append(pt)
        del bw
        torch.cuda.empty_cache()
    return points, t[0]


HOST_ENQUEUE_MS = []   # host time to issue one step (arm + hand-offs + stream sync)


def overlap_host_probe(args, R, torch, dev, dev_index, energy=None):
    """The north star's host-resident overlap target (Fig. 7 analog): pinned-host
    states of `--overlap-host-blocks` 13B blocks, each of a block's four linears
    registered as its own unit and handed off right after its dW GEMM (the
    paper's per-tensor hand-off), with a synthetic backward of T
    tokens for every T of `--overlap-host-sweep`.  Per T: `reps` alternating
    (AGO, backward-alone) runs after a backward-alone run, so every AGO run has
    a baseline right before and right after it (their mean: the GPU's power
    state drifts over the probe).  Exposed = AGO - baseline; hidden = 1 -
    exposed / optimizer alone.  Medians and [min, max] over repetitions.
    Measured for the GPU-streamed residency (the north star's path) and, on the
    same states and backward, the paper's own CPU handler (HOST_COMPUTE).
    Returns {residency: result}."""
    L, h = SHAPES[args.shape]
    sizes = model_blocks(args.shape, with_embedding=False)[:args.overlap_host_blocks]
    cfg = R.ratel_default_config()
    R.ratel_init(dev_index, 0, 1, None, cfg)
    model = Model(R, torch, dev, sizes, 1, 0, "host", grad_ring=3)
    R.ratel_finalize()
    units = []
    for b, n in enumerate(sizes):
        r0, offs, off = model.ranges[b], [], 0
        for (o, i) in linears(h):
            offs.append([off, o * i])
            off += o * i
        offs[-1][1] += n - off            # biases / LN ride with fc2
        units.append([R.ratel_range(r0.param_bf16 + 2 * o, r0.grad_bf16 + 2 * o, 0, r0.master + 4 * o,
                                    r0.exp_avg + 4 * o, r0.exp_avg_sq + 4 * o, ln, 1) for o, ln in offs])
    K = 4
    s = torch.cuda.Stream(device=dev, priority=-2)
    order = list(reversed(range(len(sizes))))
    P = sum(sizes)
    out = {}
    bw0 = None
    # one set of activations (<= 64K tokens per GEMM chunk) serves every T of the sweep
    bw0 = SynthBackward(dev, h, max(args.overlap_host_sweep), model.p16, model.grad_ring, 0, chunk=65536)
    # settle the GPU at its thermal/power operating point first: measured, the same
    # backward runs ~10 % faster for the first several seconds of load
    w0 = time.time()
    while time.time() - w0 < 15.0:
        with torch.cuda.stream(s):
            for b in order:
                bw0.block(b, b % 3)
        torch.cuda.synchronize()
    try:
        for resname, code in (("pinned-host", R.RATEL_PINNED_HOST), ("hostcompute", R.RATEL_HOST_COMPUTE)):
            R.ratel_init(dev_index, 0, 1, None, cfg)
            try:
                for b in range(len(sizes)):
                    for j, r in enumerate(units[b]):
                        R.ratel_register_block(b * K + j, [r], code)
                t = [1]

                def opt():
                    R.ratel_adam_step(HP["lr"], HP["beta1"], HP["beta2"], HP["eps"], HP["weight_decay"], t[0])
                    t[0] += 1
                    for b in order:
                        for j in range(K):
                            R.ratel_offload_grad_chunk(b * K + j, s)
                    R.ratel_sync(s)

                opt()
                opt_runs = [timed_run(torch, s, opt, energy) for _ in range(2)]
                opt_ms = _med([r[0] for r in opt_runs])
                pts = []
                for T in args.overlap_host_sweep:
                    bw = bw0
                    bw.T = T

                    def bwd():
                        with torch.cuda.stream(s):
                            for b in order:
                                bw.block(b, b % 3)

                    def ago():
                        R.ratel_adam_step(HP["lr"], HP["beta1"], HP["beta2"], HP["eps"], HP["weight_decay"], t[0])
                        t[0] += 1
                        with torch.cuda.stream(s):
                            for jb, b in enumerate(order):
                                if jb >= 3:
                                    for j in range(K):
                                        R.ratel_block_wait((b + 3) * K + j, s)   # ring slot consumed
                                bw.block(b, b % 3, on_linear=lambda j, b=b: R.ratel_offload_grad_chunk(b * K + j, s))
                        R.ratel_sync(s)

                    ago()                                    # warm-up at this T
                    runs_b = [timed_run(torch, s, bwd, energy)]
                    runs_a = []
                    for _ in range(args.overlap_reps):
                        runs_a.append(timed_run(torch, s, ago, energy))
                        runs_b.append(timed_run(torch, s, bwd, energy))
                    base = [0.5 * (runs_b[i][0] + runs_b[i + 1][0]) for i in range(args.overlap_reps)]
                    exp = [a[0] - b for a, b in zip(runs_a, base)]
                    hid = [1 - e / opt_ms for e in exp]
                    pt = {"tokens": T, "reps": args.overlap_reps, "backward_ms": _med(base),
                          "backward_ms_runs": [r[0] for r in runs_b], "ago_step_ms": _med([a[0] for a in runs_a]),
                          "exposed_optimizer_ms": _med(exp), "exposed_ms_spread": _spread(exp),
                          "hidden_fraction": _med(hid), "hidden_fraction_spread": _spread(hid)}
                    if runs_a[0][1] is not None:
                        eb = [0.5 * (runs_b[i][1] + runs_b[i + 1][1]) for i in range(args.overlap_reps)]
                        pt["backward_joules"] = _med(eb)
                        pt["ago_extra_joules_over_backward"] = _med([a[1] - e for a, e in zip(runs_a, eb)])
                    pts.append(pt)
                r = {"blocks": len(sizes), "params": P, "residency": resname,
                     "handoff": "per tensor (4 linears per block)", "optimizer_alone_ms": opt_ms,
                     "backward": "synthetic: dX and dW GEMMs of each block's 4 linears (cuBLAS bf16)",
                     "points": pts}
                if code == R.RATEL_PINNED_HOST:
                    r["host_link_gbs_optimizer_alone"] = 24 * P / (opt_ms / 1e3) / 1e9
                else:
                    r["handler"] = "the paper's CPU AdamW (HOST_COMPUTE): G16 D2H, CPU update, P16 H2D"
                if opt_runs[0][1] is not None:
                    r["optimizer_alone_joules"] = _med([x[1] for x in opt_runs])
                out[resname] = r
            finally:
                R.ratel_finalize()
        return out
    finally:
        del bw0
        del model
        torch.cuda.empty_cache()


def timed_steps(R, torch, order, stream, t0, K, pre_step=None, post_step=None):
    ev0, ev1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    ev0.record(stream)
    for k in range(K):
        if pre_step:
            pre_step(k)
        h0 = time.perf_counter()
        step_once(R, t0 + k, order, stream)
        HOST_ENQUEUE_MS.append(1e3 * (time.perf_counter() - h0))
        if post_step:
            post_step(k)
    ev1.record(stream)
    ev1.synchronize()
    return ev0.elapsed_time(ev1)


def max_over_ranks(torch, x, world, dev):
    if world == 1:
        return x
    import torch.distributed as dist
    t = torch.tensor([x], dtype=torch.float64, device=dev if dist.get_backend() == "nccl" else "cpu")
    dist.all_reduce(t, op=dist.ReduceOp.MAX)
    return float(t.item())


def barrier(torch, world):
    torch.cuda.synchronize()
    if world > 1:
        import torch.distributed as dist
        dist.barrier()
    torch.cuda.synchronize()


# ------------------------------------------------------------ N > 1 probes
C3_SLICE_N8 = 77_081_984          # 30B block (616,655,872 params) / 8 ranks: SURVEY §8(a) C3


def nccl_allgather_probe(torch, dev, world, counts, reps=5):
    """NCCL bf16 all-gather bus bandwidth at the given per-rank counts
    (torch.distributed on the same NCCL): busbw = (N-1)/N * N*count*2 B / t,
    median of `reps` after one warm-up, CUDA events, max over ranks.  The
    denominator of roofline.nvlink (SURVEY §8(d) roofline probe 4)."""
    import torch.distributed as dist
    out = {}
    for name, c in counts.items():
        send = torch.empty(c, dtype=torch.bfloat16, device=dev).fill_(1.0)
        recv = torch.empty(c * world, dtype=torch.bfloat16, device=dev)
        dist.all_gather_into_tensor(recv, send)
        torch.cuda.synchronize()
        ts = []
        for _ in range(reps):
            dist.barrier()
            e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            e0.record()
            dist.all_gather_into_tensor(recv, send)
            e1.record()
            e1.synchronize()
            ts.append(max_over_ranks(torch, e0.elapsed_time(e1), world, dev))
        t = sorted(ts)[len(ts) // 2]
        out[name] = {"count_per_rank": c, "bytes_per_rank": 2 * c, "ms": t,
                     "busbw_gbs": (world - 1) / world * world * 2 * c / (t / 1e3) / 1e9,
                     "algbw_gbs": world * 2 * c / (t / 1e3) / 1e9}
        del send, recv
    torch.cuda.empty_cache()
    return out


def nccl_allreduce_latency_us(torch, dev, world, reps=50):
    """Latency of the clip's 8-byte fp64 allreduce (X1) on this world:
    median of `reps` back-to-back single calls, CUDA events, max over ranks."""
    import torch.distributed as dist
    x = torch.zeros(1, dtype=torch.float64, device=dev)
    for _ in range(5):
        dist.all_reduce(x)
    torch.cuda.synchronize()
    ts = []
    for _ in range(reps):
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record()
        dist.all_reduce(x)
        e1.record()
        e1.synchronize()
        ts.append(e0.elapsed_time(e1) * 1e3)
    return max_over_ranks(torch, sorted(ts)[len(ts) // 2], world, dev)


def p16_identical_across_ranks(torch, dev, world, p16s) -> bool:
    """Every rank holds the same gathered P16 (bitwise
    equality of all ranks' bf16): two position-weighted int64 checksums over
    every block's P16 words, compared across ranks."""
    import torch.distributed as dist
    C = 1 << 24
    w = (torch.arange(C, device=dev, dtype=torch.int64) % 65521) + 1
    acc = torch.zeros(2, dtype=torch.int64, device=dev)
    for p in p16s:
        words = p.view(torch.int16)
        for k in range(0, words.numel(), C):
            x = words[k:k + C].to(torch.int64)
            acc[0] += x.sum()
            acc[1] += (x * w[:x.numel()]).sum()
    allv = [torch.zeros_like(acc) for _ in range(world)]
    dist.all_gather(allv, acc)
    return all(torch.equal(allv[0], v) for v in allv[1:])


def host_link_probe_all_ranks(torch, dev, world):
    """The duplex host-link probe run in every rank at once (started behind a
    barrier): per-rank and aggregate GB/s -- the pinned-host roofline at this
    N, where ranks may share PCIe switches and host DRAM (SURVEY §8(d) probe 3)."""
    import torch.distributed as dist
    barrier(torch, world)
    mine = host_link_probe(torch, dev)
    vals = torch.tensor([mine["h2d"], mine["d2h"], mine["duplex"]], dtype=torch.float64,
                        device=dev if dist.get_backend() == "nccl" else "cpu")
    allv = [torch.zeros_like(vals) for _ in range(world)]
    dist.all_gather(allv, vals)
    per = [[float(x) for x in v.cpu()] for v in allv]
    return {"per_rank": [{"h2d": a, "d2h": b, "duplex": c} for a, b, c in per],
            "aggregate_duplex_gbs": sum(r[2] for r in per), "min_rank_duplex_gbs": min(r[2] for r in per),
            "note": "every rank's pinned H2D || D2H probe concurrently"}


# ------------------------------------------------------------------- e2e
def run_e2e_device(args, R, torch, dev, model, sizes, order, t, world):
    """e2e on the SAME workload as `value`: every step the gradients come
    from pinned host memory (H2D before each block's hand-off) and the
    updated P16 goes back to pinned host memory (D2H as soon as each block's
    update ran), through the C ABI; the states stay resident."""
    ring = model.grad_ring
    nr = len(ring)
    g_host = torch.empty(ring[0].numel(), dtype=torch.bfloat16, pin_memory=True)
    g_host.copy_(ring[0])
    p_host = [torch.empty(e - b, dtype=torch.bfloat16, pin_memory=True) for (b, e) in model.slices]
    s_in = torch.cuda.Stream(device=dev)
    s_out = torch.cuda.Stream(device=dev)
    tt = [t]

    def one():
        R.ratel_adam_step(HP["lr"], HP["beta1"], HP["beta2"], HP["eps"], HP["weight_decay"], tt[0])
        tt[0] += 1
        with torch.cuda.stream(s_in):
            for j, b in enumerate(order):
                if j >= nr:
                    R.ratel_block_wait(order[j - nr], s_in)   # ring slot consumed
                beg, end = model.slices[b]
                ring[b % nr][beg:end].copy_(g_host[beg:end], non_blocking=True)   # G16 host -> device
                R.ratel_offload_grad_chunk(b, s_in)
        with torch.cuda.stream(s_out):
            for b in order:
                R.ratel_block_wait(b, s_out)
                beg, end = model.slices[b]
                p_host[b].copy_(model.p16[b][beg:end], non_blocking=True)      # P16 device -> host
        s_in.wait_stream(s_out)
        R.ratel_sync(s_in)

    one()
    barrier(torch, world)
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    K = args.e2e_steps
    e0.record(s_in)
    for _ in range(K):
        one()
    e1.record(s_in)
    e1.synchronize()
    ms = max_over_ranks(torch, e0.elapsed_time(e1), world, dev)
    own = sum(e - b for (b, e) in model.slices)
    P = sum(sizes)
    host_link_probe(torch, dev)
    link = best_link()
    moved = 4 * own   # 2 B/param in, 2 B/param out, this rank
    achieved = moved / (ms / K / 1e3) / 1e9
    return {"value": P * K / (ms / 1e3), "unit": UNIT, "h2d_bytes_per_step": int(2 * own * world),
            "d2h_bytes_per_step": int(2 * own * world), "ms_per_step": ms / K, "steps": K,
            "workload": "the value's workload (all blocks, states resident); G16 in from pinned host, "
                        "P16 out to pinned host, every step",
            "host_link_gbs": achieved, "host_link_peak_gbs": link["duplex"],
            "host_link_frac": achieved / link["duplex"], "host_link_probe": link}, tt[0]


K1_NAME = {0: "adam_update_tma_kernel (K1)", 1: "adam_update_kernel (K1, LDG)", 2: "adam_update_kernel (K1, LDG_LITE)"}


def host_dram_probe():
    """Host DRAM ceiling for the CPU handler: tools/host_stream.c (OpenMP, all
    cores) built with gcc into build/ and run; its 5-read/4-write pattern moves
    the handler's 28 B/param."""
    src = os.path.join(ROOT, "tools", "host_stream.c")
    exe = os.path.join(ROOT, "build", "host_stream")
    if not os.path.exists(exe) or os.path.getmtime(exe) < os.path.getmtime(src):
        os.makedirs(os.path.dirname(exe), exist_ok=True)
        subprocess.run(["gcc", "-O3", "-march=native", "-fopenmp", "-o", exe, src], check=True,
                       capture_output=True)
    out = subprocess.run([exe], check=True, capture_output=True, text=True, timeout=300).stdout
    return json.loads(out.strip().splitlines()[-1])


def offdevice_roofline(args, torch, dev, own_params_per_s, k1_roof):
    """roofline for a step whose states live off the device.
    A fraction f of the params is GPU-streamed (pinned-host tile ring: 12 B/param
    H2D + 12 B/param D2H over the host link, the same 24 B/param through host
    DRAM by DMA), the rest goes to the CPU handler (HOST_COMPUTE: 28 B/param of
    CPU traffic + 4 B/param of G16/P16 DMA in host DRAM, 4 B/param on the link);
    f = 1 for --residency host, 0 for hostcompute.  Each resource's achieved
    bytes are set against this run's probe of it (duplex link probe,
    tools/host_stream.c); the bound is the one closer to its peak.  The tile
    kernel's HBM numbers stay under "k1"."""
    f = {"host": 1.0, "hostcompute": 0.0}.get(args.residency, args.hybrid_gpu_frac)
    k1 = {k: v for k, v in k1_roof.items() if k not in ("traffic", "ncu_dram_pct_of_peak")}
    legs = {}
    if f > 0:
        host_link_probe(torch, dev)
        link = best_link()
        bpp = 24 * f + 4 * (1 - f)
        a = bpp * own_params_per_s / 1e9
        legs["host_link"] = {"achieved": a, "peak": link["duplex"], "frac": a / link["duplex"],
                             "algorithmic_bytes_per_param": bpp, "probe": link,
                             "peak_source": "best of this run's pinned H2D || D2H probes on two streams "
                                            "(start-up and after the measurement)", "probes": list(LINK_PROBES)}
    if f < 1:
        probe = host_dram_probe()
        bpp = 24 * f + 32 * (1 - f)
        a = bpp * own_params_per_s / 1e9
        legs["host_dram"] = {"achieved": a, "peak": probe["adam_pattern_gbs"], "frac": a / probe["adam_pattern_gbs"],
                             "algorithmic_bytes_per_param": bpp, "probe": probe,
                             "peak_source": f"this run's tools/host_stream.c 5-read/4-write pattern, "
                                            f"{probe['threads']} threads"}
    bound = max(legs, key=lambda k: legs[k]["frac"])
    b = legs[bound]
    kernel = {1.0: "pinned-host tile ring (H2D theta/m/v, K1 on the tile, D2H)",
              0.0: "CPU AdamW handler (HOST_COMPUTE) + G16/P16 DMA"}.get(
        f, f"{f:.2f} pinned-host tile ring + {1 - f:.2f} CPU handler")
    return {"bound": bound, "kernel": kernel, "achieved": b["achieved"], "peak": b["peak"], "unit": "GB/s",
            "frac": b["frac"], "traffic": None, "algorithmic_bytes_per_param": b["algorithmic_bytes_per_param"],
            "peak_source": b["peak_source"], **legs, "k1": k1}


LINK_PROBES = []   # every host_link_probe of this run (the roofline peak is their best)


def best_link():
    """Element-wise best of every host-link probe taken in this run (one at
    start-up, one beside each measurement): the duplex probe of a single run
    varied 79-100 GB/s on one box, so the peak is the best observed."""
    return {k: max(p[k] for p in LINK_PROBES) for k in ("h2d", "d2h", "duplex")}


def host_link_probe(torch, dev, nbytes=1 << 30, reps=5):
    """Measured duplex host-link bandwidth on this box (pinned H2D and D2H
    concurrently on two streams): the e2e roofline denominator."""
    n = nbytes // 4
    h1 = torch.empty(n, dtype=torch.float32, pin_memory=True)
    h2 = torch.empty(n, dtype=torch.float32, pin_memory=True)
    d1 = torch.empty(n, dtype=torch.float32, device=dev)
    d2 = torch.empty(n, dtype=torch.float32, device=dev)
    s1, s2 = torch.cuda.Stream(device=dev), torch.cuda.Stream(device=dev)
    best = {}
    for name in ("h2d", "d2h", "duplex"):
        ts = []
        for _ in range(reps):
            torch.cuda.synchronize()
            e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            e0.record()
            s1.wait_stream(torch.cuda.current_stream())
            s2.wait_stream(torch.cuda.current_stream())
            if name in ("h2d", "duplex"):
                with torch.cuda.stream(s1):
                    d1.copy_(h1, non_blocking=True)
            if name in ("d2h", "duplex"):
                with torch.cuda.stream(s2):
                    h2.copy_(d2, non_blocking=True)
            torch.cuda.current_stream().wait_stream(s1)
            torch.cuda.current_stream().wait_stream(s2)
            e1.record()
            e1.synchronize()
            ts.append(e0.elapsed_time(e1))
        moved = nbytes * (2 if name == "duplex" else 1)
        best[name] = moved / (min(ts) / 1e3) / 1e9
    del h1, h2, d1, d2
    LINK_PROBES.append(dict(best))
    return best


def run_e2e(args, R, torch, dev, dev_index, rank, world):
    """Pinned-host residency through the C ABI: theta/m/v stream H2D/D2H via
    the library's tile ring; grads H2D from pinned host before each block's
    hand-off; P16 D2H after the sync -- all inside the timed region."""
    L, h = SHAPES[args.shape]
    n_blk = args.e2e_blocks
    sizes = [block_params(h)] * n_blk
    cfg = R.ratel_default_config()
    cfg.timing = 0
    cfg.pipeline_depth = args.e2e_depth
    init_lib(R, torch, dev_index, rank, world, cfg)
    try:
        model = Model(R, torch, dev, sizes, world, rank, "host", grad_ring=1)
        # host-side grads (one pinned buffer, re-sent for every block) and P16 out
        cap = model.grad_ring[0].numel()
        g_host = torch.empty(cap, dtype=torch.bfloat16, pin_memory=True)
        g_host.copy_(model.grad_ring[0])
        g_dev = [torch.empty(cap, dtype=torch.bfloat16, device=dev) for _ in range(n_blk)]
        for b in range(n_blk):
            model.ranges[b].grad_bf16 = g_dev[b].data_ptr()
        model.grad_ring = None
        p_host = [torch.empty(R.ratel_padded_numel(n, world), dtype=torch.bfloat16, pin_memory=True)
                  for n in sizes]
        for b in range(n_blk):
            R.ratel_register_block(b, [model.ranges[b]], R.RATEL_PINNED_HOST)
        s = torch.cuda.Stream(device=dev)
        order = list(reversed(range(n_blk)))

        s_out = torch.cuda.Stream(device=dev)

        def one_safe(t):
            R.ratel_adam_step(HP["lr"], HP["beta1"], HP["beta2"], HP["eps"], HP["weight_decay"], t)
            with torch.cuda.stream(s):
                for b in order:
                    beg, end = model.slices[b]                         # G16 host -> device
                    g_dev[b][beg:end].copy_(g_host[beg:end], non_blocking=True)
                    R.ratel_offload_grad_chunk(b, s)
            with torch.cuda.stream(s_out):
                for b in order:                                        # P16 device -> host, per block
                    R.ratel_block_wait(b, s_out)                       # as soon as its update ran
                    beg, end = model.slices[b]
                    p_host[b][beg:end].copy_(model.p16[b][beg:end], non_blocking=True)
            s.wait_stream(s_out)
            R.ratel_sync(s)
        t = 1
        for _ in range(max(1, min(args.warmup, 2))):
            one_safe(t)
            t += 1
        barrier(torch, world)
        ev0, ev1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        ev0.record(s)
        K = args.e2e_steps
        for _ in range(K):
            one_safe(t)
            t += 1
        ev1.record(s)
        ev1.synchronize()
        ms = max_over_ranks(torch, ev0.elapsed_time(ev1), world, dev)
        barrier(torch, world)
        P = sum(sizes)
        own = sum(e - b for (b, e) in model.slices)
        h2d = (12 * own + 2 * own) * world            # states in + grads in (all ranks)
        d2h = (12 * own + 2 * own) * world            # states out + this rank's P16 slice (all ranks)
        val = P * K / (ms / 1e3)
        host_link_probe(torch, dev)
        link = best_link()
        achieved = (h2d + d2h) / world / (ms / K / 1e3) / 1e9
        res = {"value": val, "unit": UNIT, "h2d_bytes_per_step": int(h2d), "d2h_bytes_per_step": int(d2h),
               "ms_per_step": ms / K, "steps": K, "params": P, "blocks": n_blk,
               "host_link_gbs": achieved, "host_link_peak_gbs": link["duplex"],
               "host_link_frac": achieved / link["duplex"], "host_link_probe": link,
               "workload": f"{n_blk} of the {args.shape} model's blocks ({sizes[0]:,} params each), "
                           "pinned-host states through the same C ABI",
               "path": "pinned-host states (tile ring depth %d, %d-elem tiles)" % (cfg.pipeline_depth,
                                                                                   cfg.tile_elems)}
        del model
        return res
    finally:
        R.ratel_finalize()


# ------------------------------------------------------------------- main
def token_list(x: str):
    """--overlap-sweep / --overlap-host-sweep: comma-separated token counts;
    '', '0' or 'none' disables the probe."""
    x = x.strip().strip("'\"")
    if x.lower() in ("", "0", "none"):
        return []
    return [int(v) for v in x.split(",") if v]


def free_port() -> int:
    import socket
    with socket.socket() as so:
        so.bind(("127.0.0.1", 0))
        return so.getsockname()[1]


def relaunch_or_world(args) -> int:
    """World size of this run.  `--gpus N` (N > 1) outside torchrun re-executes
    this script under torch.distributed.run with N ranks on this node (master
    127.0.0.1) and exits with its return code, so `python bench.py --gpus 8`
    can never silently measure one GPU; under torchrun WORLD_SIZE must equal
    --gpus (rc 2 otherwise)."""
    env_world = os.environ.get("WORLD_SIZE")
    if env_world is None:
        n = args.gpus or 1
        if n > 1:
            cmd = [sys.executable, "-m", "torch.distributed.run", "--nnodes=1", f"--nproc-per-node={n}",
                   "--master-addr", "127.0.0.1", f"--master-port={free_port()}",
                   os.path.abspath(__file__)] + sys.argv[1:]
            print(f"bench.py: --gpus {n}: re-launching under torch.distributed.run ({n} ranks)",
                  file=sys.stderr, flush=True)
            sys.stdout.flush()
            rc = subprocess.call(cmd)
            raise SystemExit(rc)
        return 1
    world = int(env_world)
    if args.gpus is not None and args.gpus != world:
        print(f"bench.py: --gpus {args.gpus} but WORLD_SIZE={world}: refusing to measure a different "
              f"number of GPUs than asked", file=sys.stderr, flush=True)
        raise SystemExit(2)
    return world


def mem_available_bytes() -> int:
    with open("/proc/meminfo") as f:
        for line in f:
            if line.startswith("MemAvailable:"):
                return int(line.split()[1]) * 1024
    raise RuntimeError("no MemAvailable in /proc/meminfo")


def auto_blocks(args, world: int) -> int:
    """L_eff: the most leading blocks of the shape whose
    states fit the box.  Host residencies: the fp32 theta/m/v of ALL ranks'
    slices (12 B/param in total) within 85 % of MemAvailable; every rank also
    keeps the full bf16 P16 of its blocks in HBM (2 B/param), capped at 60 %
    of a 180 GB GPU.  Device residency: (12/N + 2) B/param within 95 % of HBM."""
    sizes = model_blocks(args.shape)
    if args.residency == "device":
        budget = 0.95 * 183_359 * 2 ** 20
        per = lambda n: (12.0 / world + 2.0) * n
    else:
        host = 0.85 * mem_available_bytes()
        dev = 0.60 * 183_359 * 2 ** 20
        per = lambda n: max(12.0 * n / host, 2.0 * n / dev)
        budget = 1.0
    used, k = 0.0, 0
    for n in sizes:
        if used + per(n) > budget:
            break
        used += per(n)
        k += 1
    if k == 0:
        raise SystemExit("--blocks auto: not even one block of this shape fits the box")
    return k


NCCL_LOG_DIR = os.path.join(ROOT, "build", "nccl_logs")


def nccl_log_env() -> None:
    """Keep NCCL's communicator-init log (transports, channels, NVLS) without
    letting N ranks' INFO lines interleave with rank 0's JSON line on stdout:
    NCCL_DEBUG=INFO (INIT, GRAPH, NVLS) into one file per process; rank 0
    summarises its own file in multi_gpu.nccl_init and on stderr."""
    if os.environ.get("NCCL_DEBUG_FILE"):
        return                                   # the caller routes NCCL's log already
    os.makedirs(NCCL_LOG_DIR, exist_ok=True)
    os.environ["NCCL_DEBUG"] = "INFO"
    os.environ.setdefault("NCCL_DEBUG_SUBSYS", "INIT,GRAPH,NVLS,ENV")
    os.environ["NCCL_DEBUG_FILE"] = os.path.join(NCCL_LOG_DIR, "nccl.%h.%p.log")


def nccl_init_summary() -> dict | None:
    """Key lines of this process's NCCL log: version, transports per peer,
    NVLS / CollNet state, ring/tree channel counts, communicator sizes."""
    path = os.environ.get("NCCL_DEBUG_FILE", "")
    if not path:
        return None
    path = path.replace("%p", str(os.getpid()))
    import glob
    import socket
    cands = glob.glob(path.replace("%h", "*"))
    if not cands:
        return {"log": path, "lines": []}
    keys = ("NCCL version", "via P2P", "via NET", "via SHM", "NVLS", "nvls", "CollNet", "Channel 00",
            "Init COMPLETE", "comm 0x", "Connected all rings", "Connected all trees", "NCCL_")
    out = []
    with open(cands[0], errors="replace") as f:
        for line in f:
            if any(k in line for k in keys):
                out.append(line.strip()[:200])
            if len(out) >= 40:
                break
    for line in out[:12]:
        print("nccl:", line, file=sys.stderr)
    return {"log": cands[0], "host": socket.gethostname(), "lines": out}


def share_gpu_nccl_env(rank: int) -> None:
    """--share-gpu: NCCL refuses two ranks on one device of one host ("Duplicate
    GPU"); giving each rank its own NCCL host id makes them peers on different
    "hosts" that talk over loopback sockets, so the real NCCL data path (the
    library's all-gather / allreduce, torch's process group) runs with N ranks
    on the one GPU a gpurun box has.  Set before any communicator exists."""
    os.environ["NCCL_HOSTID"] = f"ratel-bench-rank{rank}"
    os.environ.setdefault("NCCL_SOCKET_IFNAME", "lo")
    os.environ.setdefault("NCCL_IB_DISABLE", "1")


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=None,
                    help="N GPUs of this node; N > 1 without torchrun re-launches this script under "
                         "torch.distributed.run (one rank per GPU); under torchrun it must equal WORLD_SIZE")
    ap.add_argument("--steps", type=int, default=20)
    ap.add_argument("--warmup", type=int, default=3)
    ap.add_argument("--impl", default="ratel", choices=["ratel", "reference"])
    ap.add_argument("--shape", default="13B", choices=list(SHAPES))
    ap.add_argument("--blocks", default="0",
                    help="use only the first N blocks; 'auto' = L_eff, the most blocks whose states fit this box "
                         "(host residencies: 85 %% of MemAvailable shared by all ranks; device: 95 %% of HBM)")
    ap.add_argument("--residency", default="device", choices=["device", "host", "hostcompute", "hybrid"])
    ap.add_argument("--hybrid-gpu-frac", type=float, default=0.3,
                    help="hybrid residency: fraction of each block streamed through the GPU (pinned-host tile "
                         "ring); the rest is updated by the CPU handler (HOST_COMPUTE)")
    ap.add_argument("--host-threads", type=int, default=0)
    ap.add_argument("--clip", type=float, default=0.0)
    ap.add_argument("--max-ctas", type=int, default=0)
    ap.add_argument("--e2e-blocks", type=int, default=4)
    ap.add_argument("--e2e-steps", type=int, default=3)
    ap.add_argument("--e2e-depth", type=int, default=8)
    ap.add_argument("--fused-allgather", action="store_true",
                    help="N>1: P16 in torch symmetric memory, all-gather fused into the update kernel")
    ap.add_argument("--sim-comm-none", action="store_true",
                    help="test mode: N ranks may share one GPU; gloo process group, library without NCCL")
    ap.add_argument("--no-e2e", action="store_true")
    ap.add_argument("--no-cpu-baseline", action="store_true")
    ap.add_argument("--oracle-sample", type=int, default=314_639_360,
                    help="params per oracle pass (reference arm and cpu_baseline); default one whole 13B block")
    ap.add_argument("--share-gpu", action="store_true",
                    help="test mode: every rank on cuda:0 with real NCCL (each rank its own NCCL host id, "
                         "loopback sockets); numbers are plumbing, not a scaling result")
    ap.add_argument("--overlap-sweep", type=token_list, default=[1024, 2048, 8192, 32768, 65536],
                    help="device-resident AGO vs deferred overlap sweep: tokens per step, comma-separated "
                         "(0 disables)")
    ap.add_argument("--overlap-reps", type=int, default=3, help="alternating repetitions per overlap point")
    ap.add_argument("--overlap-host-sweep", type=token_list,
                    default=[32768, 65536, 98304, 131072, 196608],
                    help="pinned-host per-tensor AGO overlap probe: tokens per step, comma-separated (0 disables)")
    ap.add_argument("--overlap-host-blocks", type=int, default=16,
                    help="13B-shape blocks of pinned-host states in the host overlap probe (16 = 5.0B params, 60 GB)")
    ap.add_argument("--arm", default="before", choices=["before", "after"],
                    help="arm before the hand-offs (AGO) or after the last one (deferred)")
    ap.add_argument("--cta-tiles", type=int, default=0, help="cfg.cta_tiles (0 = persistent update grid)")
    ap.add_argument("--staging", default="pipelined", choices=["pipelined", "serialized", "zero_copy"],
                    help="pinned-host residency: tile ring (Fig. 3b / 3a) or in-place over the link")
    ap.add_argument("--k1-kernel", type=int, default=0, choices=[0, 1, 2], help="cfg.k1_kernel: 0 TMA, 1 LDG, 2 LDG_LITE")
    ap.add_argument("--tile-elems", type=int, default=0)
    ap.add_argument("--depth", type=int, default=0)
    ap.add_argument("--update-streams", type=int, default=2, choices=[1, 2],
                    help="device-residency update kernels alternate over this many streams")
    args = ap.parse_args()
    global ARM_AFTER
    ARM_AFTER = args.arm == "after"
    if args.steps < 1 or args.warmup < 0:
        raise SystemExit("need --steps >= 1")
    world = relaunch_or_world(args)
    args.blocks_auto = args.blocks == "auto"
    args.blocks = auto_blocks(args, world) if args.blocks_auto else int(args.blocks)
    rank = int(os.environ.get("RANK", "0"))
    local = int(os.environ.get("LOCAL_RANK", "0"))

    if args.impl == "reference":
        run_reference(args, rank, world)
        return
    if args.share_gpu and world > 1:
        share_gpu_nccl_env(rank)
    if world > 1 and not args.sim_comm_none:
        nccl_log_env()

    import torch
    import paper_conf_icde_liaosyxcyww25_b200 as R
    global SIM_COMM_NONE
    SIM_COMM_NONE = args.sim_comm_none
    if SIM_COMM_NONE or args.share_gpu:
        local = local % torch.cuda.device_count()
    torch.cuda.set_device(local)
    dev = torch.device(f"cuda:{local}")
    if world > 1:
        import torch.distributed as dist
        if SIM_COMM_NONE:
            dist.init_process_group("gloo")
        else:
            dist.init_process_group("nccl", device_id=dev)

    cfgd = workload_config(args, world)
    sizes = model_blocks(args.shape)
    if args.blocks:
        sizes = sizes[:args.blocks]
    cfg = R.ratel_default_config()
    cfg.timing = 1
    cfg.max_ctas = args.max_ctas
    cfg.max_grad_norm = args.clip
    if args.tile_elems:
        cfg.tile_elems = args.tile_elems
    if args.depth:
        cfg.pipeline_depth = args.depth
    cfg.host_threads = args.host_threads
    cfg.update_streams = args.update_streams
    cfg.cta_tiles = args.cta_tiles
    cfg.staging = {"pipelined": R.RATEL_STAGING_PIPELINED, "serialized": R.RATEL_STAGING_SERIALIZED,
                   "zero_copy": R.RATEL_STAGING_ZERO_COPY}[args.staging]
    cfg.k1_kernel = args.k1_kernel
    if not args.no_e2e or args.residency != "device":
        host_link_probe(torch, dev)          # start-up probe, before 100+ GB of states are pinned
    init_lib(R, torch, local, rank, world, cfg)
    sampler = ClockSampler(gpu_uuid(torch, dev)) if rank == 0 else None
    try:
        fused = args.fused_allgather and world > 1 and not SIM_COMM_NONE
        model = Model(R, torch, dev, sizes, world, rank, "device" if args.residency == "device" else "host",
                      symm=fused, peer_memory="ipc" if args.share_gpu else "symm")
        res = {"host": R.RATEL_PINNED_HOST, "hostcompute": R.RATEL_HOST_COMPUTE}.get(args.residency, R.RATEL_DEVICE)
        hybrid = args.residency == "hybrid"
        if hybrid and world > 1:
            raise SystemExit("--residency hybrid is single-rank")
        for b in range(len(sizes)):
            if hybrid:   # block b = GPU-streamed head (id b) + CPU-handler tail (id b + L), handed off together
                r = model.ranges[b]
                k = min(sizes[b], int(round(args.hybrid_gpu_frac * sizes[b] / 8)) * 8)
                head = R.make_range(r.param_bf16, r.grad_bf16, r.master, r.exp_avg, r.exp_avg_sq, k)
                tail = R.make_range(r.param_bf16 + 2 * k, r.grad_bf16 + 2 * k, r.master + 4 * k, r.exp_avg + 4 * k,
                                    r.exp_avg_sq + 4 * k, sizes[b] - k)
                if k > 0:
                    R.ratel_register_block(b, [head], R.RATEL_PINNED_HOST)
                if k < sizes[b]:
                    R.ratel_register_block(b + len(sizes), [tail], R.RATEL_HOST_COMPUTE)
                continue
            R.ratel_register_block(b, [model.ranges[b]], res)
            if fused:   # update kernel stores P16 into every peer over NVLink; no NCCL all-gather
                R.ratel_register_peer_params(b, 0, model.peer_ptrs[b])
        s = torch.cuda.Stream(device=dev)
        order = list(reversed(range(len(sizes))))          # decreasing index
        if hybrid:
            order = [x for b in order for x, on in ((b, args.hybrid_gpu_frac > 0),
                                                    (b + len(sizes), args.hybrid_gpu_frac < 1)) if on]
        t = 1
        for _ in range(args.warmup):
            step_once(R, t, order, s)
            t += 1
        barrier(torch, world)
        remeasured = False
        for attempt in range(2):
            R.ratel_kernel_timing(reset=True)
            l0 = R.ratel_launch_count()
            w0 = time.time()
            ms = timed_steps(R, torch, order, s, t, args.steps)
            t += args.steps
            w1 = time.time()
            launches = R.ratel_launch_count() - l0
            k1_ms, k1_n = R.ratel_kernel_timing(reset=True)
            bad = 0.0
            if sampler:
                sampler.mark(w0, w1)
                time.sleep(0.3)   # let the sampler deliver the window's last rows
                st = sampler.stats() or {}
                bad = 1.0 if any(r in ClockSampler.BAD for r in st.get("reasons", [])) else 0.0
                if st.get("sm_mhz") and st.get("sm_max_mhz") and not st.get("reasons") \
                        and st["sm_mhz"] < 0.6 * st["sm_max_mhz"]:
                    bad = 1.0     # clocks stuck low with no reason: a leftover clock lock
            if world > 1:        # every rank re-measures together
                import torch.distributed as dist
                flag = torch.tensor([bad], dtype=torch.float64,
                                    device=dev if dist.get_backend() == "nccl" else "cpu")
                dist.all_reduce(flag, op=dist.ReduceOp.MAX)
                bad = float(flag.item())
            if bad == 0.0 or attempt == 1:
                break
            remeasured = True     # throttled window (hw/thermal slowdown): measure once more
        ms = max_over_ranks(torch, ms, world, dev)
        barrier(torch, world)
        own = sum(e - b for (b, e) in model.slices)
        P = sum(sizes)
        value = P * args.steps / (ms / 1e3)
        peak, peak_kind = peaks()
        k1_bytes = BYTES_PER_PARAM * own * args.steps
        achieved = k1_bytes / (k1_ms / 1e3) / 1e9 if k1_ms > 0 else None
        tpp = ncu_traffic_per_param()
        per_launch = own * args.steps / max(k1_n, 1)
        roof = {"bound": "hbm", "kernel": K1_NAME.get(args.k1_kernel, "K1"), "achieved": achieved, "peak": peak,
                "unit": "GB/s", "frac": (achieved / peak) if achieved else None,
                "traffic": (tpp * per_launch) if tpp else None,
                "algorithmic_bytes_per_launch": BYTES_PER_PARAM * per_launch,
                "launches": k1_n, "avg_launch_ms": k1_ms / max(k1_n, 1),
                "k1_share_of_step": (k1_ms / args.steps) / (ms / args.steps),
                "peak_source": f"MEASURED_PEAKS.json hbm_gbs ({peak_kind}): a torch copy, whose grid-stride "
                               "loop splits work statically; K1 schedules tiles dynamically and can exceed it",
                "ncu_dram_pct_of_peak": ncu_summary().get("ncu_dram_pct_of_peak_sustained")}
        overlap = None
        if args.overlap_sweep and world == 1 and args.residency == "device" and args.clip == 0:
            try:
                pts, t = overlap_probe(args, R, torch, dev, model, sizes, order, t, ms / args.steps,
                                       Energy(gpu_uuid(torch, dev)))
                overlap = {"backward": "synthetic: dX and dW GEMMs of each block's 4 linears (cuBLAS bf16), "
                                       "<= 16K tokens per GEMM chunk", "grad_ring": len(model.grad_ring),
                           "schedules": "ago = armed before backward, per-block hand-off; deferred = whole "
                                        "backward, then the whole step (Ratel+ZeRO)",
                           "energy": "NVML total-energy counter around each run", "points": pts}
            except Exception as ex:
                overlap = {"error": repr(ex)[:300]}
        multi = None
        if world > 1 and not SIM_COMM_NONE:
            try:
                own_max = max(e - b for (b, e) in model.slices)
                probes = nccl_allgather_probe(torch, dev, world, {
                    "c3_block_slice_n8": C3_SLICE_N8,
                    "this_workload_block_slice": R.ratel_padded_numel(max(sizes), world) // world})
                bw = probes["this_workload_block_slice"]["busbw_gbs"]
                nv_bytes = 2.0 * (world - 1) / world * P          # bf16 P16 received per GPU per step
                step_s = ms / args.steps / 1e3
                t_hbm = BYTES_PER_PARAM * (P / world) / (peak * 1e9)
                t_nv = nv_bytes / (bw * 1e9)
                roof["nvlink"] = {"bound": "nvlink", "collective": "per-block bf16 all-gather (X2)",
                                  "algorithmic_bytes_per_gpu_per_step": nv_bytes,
                                  "achieved": nv_bytes / step_s / 1e9, "peak": bw, "unit": "GB/s",
                                  "frac": nv_bytes / step_s / 1e9 / bw,
                                  "peak_source": "this run's NCCL all-gather busbw at the workload's per-rank "
                                                 "block slice", "spec_gbs_per_direction": 900.0}
                roof["step_bounds_ms"] = {"hbm": 1e3 * t_hbm, "nvlink": 1e3 * t_nv,
                                          "max": 1e3 * max(t_hbm, t_nv),
                                          "step_over_max_bound": (ms / args.steps) / (1e3 * max(t_hbm, t_nv))}
                multi = {"nccl_allgather": probes, "host_link": host_link_probe_all_ranks(torch, dev, world),
                         "nccl_allreduce_8B_latency_us": nccl_allreduce_latency_us(torch, dev, world),
                         "p16_identical_across_ranks": p16_identical_across_ranks(torch, dev, world, model.p16),
                         "own_params_max_rank": own_max,
                         "nccl_init": nccl_init_summary() if rank == 0 else None,
                         "transport": ("loopback sockets, all ranks on one GPU (--share-gpu test mode)"
                                       if args.share_gpu else "NCCL over NVLink/NVSwitch")}
            except Exception as ex:  # report, do not hide
                multi = {"error": repr(ex)[:300]}
        e2e = None
        if not args.no_e2e and args.residency == "device":
            try:
                e2e, t = run_e2e_device(args, R, torch, dev, model, sizes, order, t, world)
            except Exception as ex:  # report, do not hide
                e2e = {"value": None, "unit": UNIT, "error": repr(ex)[:300],
                       "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0}
        del model
        R.ratel_finalize()
        torch.cuda.empty_cache()
        clocks = sampler.stop() if sampler else None

        e2e_host = None
        if not args.no_e2e:
            try:
                e2e_host = run_e2e(args, R, torch, dev, local, rank, world)
            except Exception as ex:  # report, do not hide
                e2e_host = {"value": None, "unit": UNIT, "error": repr(ex)[:300],
                            "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0}
            torch.cuda.empty_cache()
        if e2e is None:
            e2e = e2e_host
        if args.residency != "device":      # the bound is off-device: report that roofline, K1 beside it
            try:
                nv = {k: roof[k] for k in ("nvlink", "step_bounds_ms") if k in roof}
                roof = dict(offdevice_roofline(args, torch, dev, own * args.steps / (ms / 1e3), roof), **nv)
            except Exception as ex:  # report, do not hide
                roof = dict(roof, offdevice_error=repr(ex)[:300])

        overlap_host = overlap_hostcompute = None
        if args.overlap_host_sweep and world == 1 and args.residency == "device":
            try:
                oh = overlap_host_probe(args, R, torch, dev, local, Energy(gpu_uuid(torch, dev)))
                overlap_host, overlap_hostcompute = oh.get("pinned-host"), oh.get("hostcompute")
            except Exception as ex:  # report, do not hide
                overlap_host = {"error": repr(ex)[:300]}
            torch.cuda.empty_cache()

        cpu = None
        if rank == 0 and world == 1 and not args.no_cpu_baseline:
            # the oracle as it stands on this host: a whole 13B block per pass at
            # every core (>= 8 s), and one pass of the same block on one core
            threads = host_threads()
            n = args.oracle_sample
            try:
                cpu = oracle_baseline(n, 2, 1, threads, min_seconds=8.0)
                one = oracle_baseline(n, 1, 0 if n >= (1 << 27) else 1, 1)
                cpu["single_thread"] = {k: one[k] for k in ("value", "unit", "cores", "sample",
                                                            "sample_ms_per_pass", "dram_gbs_at_28B_per_param")}
            except Exception as ex:  # report, do not hide
                cpu = {"value": None, "unit": UNIT, "cores": threads, "kind": "oracle", "error": repr(ex)[:300]}

        if rank == 0:
            line = {"metric": METRIC, "value": value, "unit": UNIT, "n_gpus": world, "steps": args.steps,
                    "warmup": args.warmup, "ms_per_step": ms / args.steps, "higher_is_better": True,
                    "scaling": "strong", "vs_baseline": None, "dtype": "f32", "data": "synthetic",
                    "config": cfgd, "roofline": roof, "cpu_baseline": cpu, "e2e": e2e,
                    "e2e_host_states": e2e_host,
                    "clocks": dict(clocks or {}, remeasured=remeasured), "gpu_launches": launches,
                    # first timed step: issued into a drained launch queue, so this is the
                    # host cost of a step (later ones wait on queue back-pressure)
                    "host_enqueue_ms_first_step": HOST_ENQUEUE_MS[0] if HOST_ENQUEUE_MS else None,
                    "overlap": overlap, "overlap_host": overlap_host, "overlap_hostcompute": overlap_hostcompute,
                    "hbm_gbs_step": BYTES_PER_PARAM * P / (ms / args.steps / 1e3) / 1e9 / world}
            if multi is not None:
                line["multi_gpu"] = multi
            print(json.dumps(line), flush=True)
    finally:
        try:
            R.ratel_finalize()
        except Exception:
            pass
        if world > 1:
            import torch.distributed as dist
            dist.destroy_process_group()


if __name__ == "__main__":
    main()
