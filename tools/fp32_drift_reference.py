"""The same long run as tools/long_run_drift.py with torch's own fp32 AdamW
(CPU, foreach=False, fp32 parameter and states) in place of the GPU path:
how far does ANY fp32-master AdamW drift from the double oracle?  (Context
for R13's "after 10 steps": the GPU path's drift is that of fp32 storage.)

    python tools/fp32_drift_reference.py [--n 1048576] [--steps 1000]
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
from tests.tolerance import _absdiff  # noqa: E402


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--n", type=int, default=1 << 20)
    ap.add_argument("--steps", type=int, default=1000)
    ap.add_argument("--checkpoints", type=int, nargs="+", default=[10, 30, 100, 300, 1000, 2000])
    args = ap.parse_args()
    n = args.n
    th0 = synth.theta0(n, block=0)
    ref = oracle.Range.fresh(th0)
    p = torch.nn.Parameter(torch.from_numpy(th0.copy()))
    opt = torch.optim.AdamW([p], lr=1e-3, betas=(0.9, 0.999), eps=1e-8, weight_decay=1e-2, foreach=False)
    threads = len(os.sched_getaffinity(0))
    for t in range(1, args.steps + 1):
        gb = synth.grad16(n, step=t, block=0)
        p.grad = torch.from_numpy(synth.bf16_bits_to_f32(gb))
        opt.step()
        oracle.adam_range(ref, gb, oracle.hparams(step=t), threads=threads)
        if t in args.checkpoints:
            st = opt.state[p]
            e_th = _absdiff(p.detach().numpy(), ref.p32) / np.maximum(ref.theta_bar, 1e-300)
            e_m = _absdiff(st["exp_avg"].numpy(), ref.m32) / np.maximum(ref.m_bar, 1e-300)
            e_v = _absdiff(st["exp_avg_sq"].numpy(), ref.v32) / np.maximum(np.abs(ref.v32.astype(np.float64)), 1e-300)
            print(json.dumps({"impl": "torch.optim.AdamW fp32 (CPU, foreach=False)", "step": t, "n": n,
                              "theta_over_theta_bar": float(e_th.max()), "m_over_m_bar": float(e_m.max()),
                              "v_rel": float(e_v.max()), "theta_p999": float(np.quantile(e_th, 0.999))}), flush=True)


if __name__ == "__main__":
    main()
