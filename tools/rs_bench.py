"""Throughput of the fused-reduction update kernel (K1-RS, R17) on
ONE B200 (tools, not product).

Rank 0 of a simulated world N (RATEL_COMM_NONE) owns the slice n/N of one
13B-shaped block (n = 314,639,360) and reduces the N ranks' full-range G16,
all resident in this GPU's HBM (on a real NVSwitch system N-1 of them are
peers' and are read over NVLink).  Per slice element the kernel moves
2N B of gradients + 12 B of states in and 12 + 2 B out, so HBM GB/s =
slice x (2N + 26) / t.  Compared with the plain (TMA) K1 on the same slice,
which reads one already-reduced G16 (28 B/param).

  python tools/rs_bench.py [--steps 20]        # one JSON line per N
"""
import argparse
import ctypes
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import torch  # noqa: E402

import paper_conf_icde_liaosyxcyww25_b200 as R  # noqa: E402

N_BLOCK = 314_639_360
PEAK = 6554.6   # MEASURED_PEAKS.json hbm_gbs


def run(world, steps, rs=True, k1_kernel=0):
    dev = torch.device("cuda:0")
    cap = R.ratel_padded_numel(N_BLOCK, world)
    beg, end = R.ratel_rank_slice(N_BLOCK, world, 0)
    s = end - beg
    p16 = torch.zeros(cap, dtype=torch.bfloat16, device=dev)
    grads = [torch.empty(cap, dtype=torch.bfloat16, device=dev) for _ in range(world if rs else 1)]
    for q, g in enumerate(grads):
        R.ratel_gen_grad16(g.data_ptr(), cap, 0, R.ratel_gen_stream_key(0x5EED5EED, 1, q, 0))
    th = torch.empty(s, device=dev)
    R.ratel_gen_theta0(th.data_ptr(), s, 0, R.ratel_gen_stream_key(0x5EED5EED, 0, 0, 0))
    m = torch.zeros(s, device=dev)
    v = torch.zeros(s, device=dev)
    cfg = R.ratel_default_config()
    cfg.comm = R.RATEL_COMM_NONE
    cfg.timing = 1
    cfg.k1_kernel = k1_kernel          # 0: TMA-staged kernels, 1: register-staged (LDG)
    R.ratel_init(0, 0, world, None, cfg)
    try:
        R.ratel_register_block(0, [R.make_range(p16, grads[0], th, m, v, N_BLOCK, 1)])
        if rs:
            R.ratel_register_peer_grads(0, 0, grads, 1.0 / world)
        for t in range(1, steps + 4):
            if t == 4:
                torch.cuda.synchronize()
                R.ratel_kernel_timing(reset=True)
            R.ratel_adam_step(1e-3, 0.9, 0.999, 1e-8, 1e-2, t)
            R.ratel_offload_grad_chunk(0, None)
            R.ratel_sync(None)
        ms, n = R.ratel_kernel_timing(reset=True)
    finally:
        R.ratel_finalize()
    per = ms / n
    bpp = (2 * world + 26) if rs else 28
    name = ("adam_update_rs_tma_kernel" if k1_kernel == 0 else "adam_update_rs_kernel") if rs else \
        ("adam_update_tma_kernel" if k1_kernel == 0 else "adam_update_kernel")
    return dict(world=world, kernel=name,
                slice=s, ms=round(per, 4), params_per_s=s / (per / 1e3),
                bytes_per_param=bpp, hbm_gbs=round(s * bpp / (per / 1e3) / 1e9, 1),
                frac=round(s * bpp / (per / 1e3) / 1e9 / PEAK, 4))


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--steps", type=int, default=20)
    ap.add_argument("--worlds", type=int, nargs="*", default=[1, 2, 4, 8])
    a = ap.parse_args()
    for w in a.worlds:
        print(json.dumps(run(w, a.steps, rs=False)), flush=True)
        print(json.dumps(run(w, a.steps, rs=True)), flush=True)            # TMA-staged K1-RS (default)
        print(json.dumps(run(w, a.steps, rs=True, k1_kernel=1)), flush=True)  # register-staged K1-RS


if __name__ == "__main__":
    main()
