"""Writes tests/golden/oracle_digests.json: SHA-256 digests of the CPU
oracle's fp32/bf16 outputs on the C1 workload (BASELINE.json configs[0]) after
10 steps.  Calls only oracle/ and synth/ (no CUDA path).  These are regression
fixtures for the oracle itself -- the paper prints no worked example -- so a
change to the oracle's arithmetic shows up as a digest change that the commit
must justify (DESIGN.md R-readings).

    python tests/golden/make_golden.py      # regenerate (review the diff!)
"""
import hashlib
import json
import os
import sys

HERE = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, os.path.dirname(os.path.dirname(HERE)))

import numpy as np  # noqa: E402

import oracle  # noqa: E402
import synth  # noqa: E402

H = 256
C1_SIZES = [H, H, 3 * H * H, 3 * H, H * H, H, H, H, 4 * H * H, 4 * H, 4 * H * H, H]
C1_WD = [0, 0, 1, 0, 1, 0, 0, 0, 1, 0, 1, 0]


def run(case, scales=False):
    """Digest of the fp32/bf16 outputs, or (scales=True) of the tolerance
    scales theta_bar / m_bar the oracle tracks beside them (R13)."""
    n = sum(C1_SIZES)
    th0 = synth.theta0(n, block=0)
    offs = np.concatenate([[0], np.cumsum(C1_SIZES)])
    if case["ranges"] == "flat":
        ranges = [oracle.Range.fresh(th0)]
        cuts = [(0, n)]
    else:
        ranges = [oracle.Range.fresh(th0[offs[i]:offs[i + 1]], C1_WD[i]) for i in range(len(C1_SIZES))]
        cuts = [(offs[i], offs[i + 1]) for i in range(len(C1_SIZES))]
    for t in range(1, 11):
        g = synth.grad16(n, step=t, block=0)
        oracle.adam_step(ranges, [g[a:b] for a, b in cuts], oracle.hparams(step=t, mode=case["mode"]),
                         max_grad_norm=case["clip"])
    h = hashlib.sha256()
    for r in ranges:
        for a in ((r.theta_bar, r.m_bar) if scales else (r.p32, r.m32, r.v32, r.p16)):
            h.update(np.ascontiguousarray(a).tobytes())
    return h.hexdigest()


CASES = {
    "c1_flat_adamw": dict(ranges="flat", mode=oracle.ADAMW, clip=0.0),
    "c1_12ranges_adamw": dict(ranges="split", mode=oracle.ADAMW, clip=0.0),
    "c1_12ranges_adam_l2": dict(ranges="split", mode=oracle.ADAM_L2, clip=0.0),
    "c1_flat_adamw_clip1e-3": dict(ranges="flat", mode=oracle.ADAMW, clip=1e-3),
}


def digests():
    return {k: run(v) for k, v in CASES.items()}


def scale_digests():
    return {k: run(v, scales=True) for k, v in CASES.items()}


if __name__ == "__main__":
    out = {"source": "tests/golden/make_golden.py (oracle/ + synth/ only)",
           "workload": "C1: one GPT block h=256 (789,760 params), 10 steps, torch-default hyperparameters",
           "sha256": digests(),
           "sha256_scales": scale_digests()}
    with open(os.path.join(HERE, "oracle_digests.json"), "w") as f:
        json.dump(out, f, indent=1)
    print(json.dumps(out, indent=1))
