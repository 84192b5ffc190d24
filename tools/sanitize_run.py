"""Small AGO steps through the C ABI for compute-sanitizer (memcheck,
racecheck, synccheck): C1-sized ragged blocks, a capped grid so every CTA
cycles the TMA stage ring, clip mode, a pinned-host block, the register-staged
LDG / LDG_LITE kernels, a non-persistent grid (cta_tiles), zero-copy staging
and the fused-reduction kernels (K1-RS, K2-RS) at world 1; every run ends with
ratel_refresh_params (refresh_p16_kernel over device and pinned-host masters)."""
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import torch  # noqa: E402

import paper_conf_icde_liaosyxcyww25_b200 as R  # noqa: E402
from tests.harness import GpuBlock, ratel_lib  # noqa: E402


def run(max_ctas, clip, pinned, rs_scale=None, **cfg):
    dev = torch.device("cuda:0")
    blocks = [GpuBlock(0, [789_760 + 3], dev, pinned=pinned), GpuBlock(1, [40_001, 17], dev)]
    with ratel_lib(max_ctas=max_ctas, max_grad_norm=clip, tile_elems=65_536, **cfg):
        for b in blocks:
            b.register()
            if rs_scale is not None:
                for i in range(len(b.sizes)):
                    R.ratel_register_peer_grads(b.id, i, [None], rs_scale)
        for t in (1, 2):
            for b in blocks:
                b.load_grads(t)
            torch.cuda.synchronize()
            R.ratel_adam_step(1e-3, 0.9, 0.999, 1e-8, 1e-2, t)
            for b in reversed(blocks):
                R.ratel_offload_grad_chunk(b.id, None)
            R.ratel_sync(None)
        for b in blocks:                       # P16 rebuilt from the masters (refresh_p16_kernel)
            R.ratel_refresh_params(b.id, None)


if __name__ == "__main__":
    run(4, 0.0, False)
    run(0, 1.0, False)
    run(2, 0.0, True)
    run(8, 0.0, False, k1_kernel=R.RATEL_UPDATE_LDG)
    run(0, 1.0, False, k1_kernel=R.RATEL_UPDATE_LDG_LITE)
    run(0, 0.0, False, cta_tiles=4)
    run(16, 0.0, True, staging=R.RATEL_STAGING_ZERO_COPY)
    run(0, 0.0, False, rs_scale=0.5)
    run(4, 1.0, True, rs_scale=0.5)
    print("sanitize_run: done")
