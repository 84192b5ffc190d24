"""How far does the fp32 GPU path drift from the double oracle over many steps?
(R13's 1e-5 is the north star's "after 10 steps" bound.)

One 1M-element range (13B-block-like values: theta0 from the recipe, fresh
log-uniform bf16 gradients every step), AdamW with torch defaults, device
residency through the C ABI; the oracle steps the same range on the host (all
cores).  At each checkpoint step prints the worst |theta - theta_ref| /
theta_bar, |m - m_ref| / m_bar and |v - v_ref| / v_ref over ALL elements, and
the bf16 distance in ulps at scale.

    python tools/long_run_drift.py [--n 1048576] [--steps 5000]
"""
import argparse
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import numpy as np  # noqa: E402
import torch  # noqa: E402

import oracle  # noqa: E402
import synth  # noqa: E402
import paper_conf_icde_liaosyxcyww25_b200 as R  # noqa: E402
from tests.harness import torch_to_u16, u16_to_torch  # noqa: E402
from tests.tolerance import _absdiff, bf16_to_f64, bf16_ulp_at  # noqa: E402


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--n", type=int, default=1 << 20)
    ap.add_argument("--steps", type=int, default=5000)
    ap.add_argument("--checkpoints", type=int, nargs="+", default=[10, 30, 100, 300, 1000, 2000, 5000])
    args = ap.parse_args()
    dev = torch.device("cuda:0")
    n = args.n
    th0 = synth.theta0(n, block=0)
    ref = oracle.Range.fresh(th0)
    th = torch.from_numpy(th0.copy()).to(dev)
    m = torch.zeros(n, device=dev)
    v = torch.zeros(n, device=dev)
    p = torch.zeros(R.ratel_padded_numel(n, 1), dtype=torch.bfloat16, device=dev)
    g = torch.zeros(R.ratel_padded_numel(n, 1), dtype=torch.bfloat16, device=dev)
    threads = len(os.sched_getaffinity(0))
    cfg = R.ratel_default_config()
    R.ratel_init(0, 0, 1, None, cfg)
    try:
        R.ratel_register_block(0, [R.make_range(p, g, th, m, v, n)], R.RATEL_DEVICE)
        for t in range(1, args.steps + 1):
            gb = synth.grad16(n, step=t, block=0)
            g[:n].copy_(u16_to_torch(gb, dev))
            R.ratel_adam_step(1e-3, 0.9, 0.999, 1e-8, 1e-2, t)
            R.ratel_offload_grad_chunk(0, None)
            R.ratel_sync(None)
            oracle.adam_range(ref, gb, oracle.hparams(step=t), threads=threads)
            if t in args.checkpoints:
                P32, M32, V32 = th.cpu().numpy(), m.cpu().numpy(), v.cpu().numpy()
                P16 = torch_to_u16(p[:n])
                e_th = _absdiff(P32, ref.p32) / np.maximum(ref.theta_bar, 1e-300)
                e_m = _absdiff(M32, ref.m32) / np.maximum(ref.m_bar, 1e-300)
                e_v = _absdiff(V32, ref.v32) / np.maximum(np.abs(ref.v32.astype(np.float64)), 1e-300)
                e_p = _absdiff(bf16_to_f64(P16), bf16_to_f64(ref.p16)) / bf16_ulp_at(ref.theta_bar)
                print(json.dumps({"step": t, "n": n, "theta_over_theta_bar": float(e_th.max()),
                                  "m_over_m_bar": float(e_m.max()), "v_rel": float(e_v.max()),
                                  "p16_ulps_at_scale": float(e_p.max()),
                                  "theta_p999": float(np.quantile(e_th, 0.999)),
                                  "within_1e-5": bool(e_th.max() <= 1e-5 and e_m.max() <= 1e-5 and e_v.max() <= 1e-5)}),
                      flush=True)
    finally:
        R.ratel_finalize()


if __name__ == "__main__":
    main()
