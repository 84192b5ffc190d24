"""ratel_refresh_params (checkpoint resume): P16 rebuilt in the library from
the registered masters -- the update's own RNE conversion (P:L1108-1110,
"produces a 16-bit parameter copy") -- for every residency, including SSD
masters read back from the state file; refused while a step is in flight.
(N = 2 with the all-gather: tests/test_nccl_ranks_gpu.py.)"""
import numpy as np
import pytest
import torch

import oracle
import paper_conf_icde_liaosyxcyww25_b200 as R
from tests.harness import GpuBlock, SsdBlock, ratel_lib, torch_to_u16
from tests.test_parity_gpu import run

pytestmark = pytest.mark.gpu

SIZES = [300_001, 65_560, 7]


def _blocks(kind, dev, tmp_path):
    if kind == "ssd":
        out, base = [], 0
        for i, n in enumerate(SIZES):
            b = SsdBlock(i, [n, 24], dev, tmp_path / "s.bin", base=base)
            base = b.file_bytes
            out.append(b)
        return out
    return [GpuBlock(i, [n, 24], dev, pinned=kind == "pinned", host_compute=kind == "hostcompute")
            for i, n in enumerate(SIZES)]


@pytest.mark.parametrize("kind", ["device", "pinned", "hostcompute", "ssd"])
def test_refresh_rebuilds_p16_from_masters(cuda_dev, tmp_path, kind):
    blocks = _blocks(kind, cuda_dev, tmp_path)
    run(blocks, 2, tile_elems=1 << 16)                     # two checked steps -> masters != theta0
    with ratel_lib(tile_elems=1 << 16):
        for b in blocks:
            b.register()
        masters = [[b.gpu_state(j)["p32"] for j in range(len(b.sizes))] for b in blocks]
        for b in blocks:                                   # scramble the working copies
            for p in b.p16:
                p.fill_(5.0)
        torch.cuda.synchronize()
        s = torch.cuda.Stream()
        for b in blocks:
            R.ratel_refresh_params(b.id, s)
        s.synchronize()
        for b, ms in zip(blocks, masters):
            for j, (n, m) in enumerate(zip(b.sizes, ms)):
                assert np.array_equal(torch_to_u16(b.p16[j][:n]), oracle.bf16_rne(m)), (kind, b.id, j)
        # between steps only
        R.ratel_adam_step(1e-3, 0.9, 0.999, 1e-8, 0.0, 1)
        with pytest.raises(R.RatelError) as e:
            R.ratel_refresh_params(blocks[0].id, None)
        assert e.value.code == R.RATEL_ESTATE
        for b in reversed(blocks):
            R.ratel_offload_grad_chunk(b.id, None)
        R.ratel_sync(None)
        R.ratel_refresh_params(blocks[0].id, None)          # host-blocking form
        with pytest.raises(R.RatelError) as e:
            R.ratel_refresh_params(999, None)
        assert e.value.code == R.RATEL_ESTATE
    if kind == "ssd":
        for b in blocks:
            b.close()
