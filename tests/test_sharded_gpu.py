"""Range-sharded (N > 1) path on ONE GPU.

gpurun gives one GPU and NCCL refuses two ranks on one device, so:
1. N = 2, 4, 8 ranks are simulated in one process with N separately loaded
   copies of libratel.so (independent library state), each `ratel_init(rank
   r, world N)` with RATEL_COMM_NONE; the test plays the bf16 all-gather (X2)
   with device copies.  The gathered P16 and the concatenated fp32 slices
   must equal the single-rank run bit for bit (R16): this checks the C
   runtime's slicing, rank offsets of grad/param pointers, padding and the
   kernels on ragged slices.
2. A one-rank NCCL communicator (RATEL_COMM_NCCL) runs the real NCCL calls
   (in-place all-gather per block, fp64 allreduce of the clip norm, async
   error query, destroy) and must not change a single bit.
"""
import ctypes
import os
import shutil

import numpy as np
import pytest
import torch

import synth
import paper_conf_icde_liaosyxcyww25_b200 as R
from tests.harness import GpuBlock, ratel_lib

pytestmark = pytest.mark.gpu

SIZES = [300_001, 65_560, 1_000_003, 24]


def _single_rank(dev, steps, **cfg_kw):
    blocks = [GpuBlock(i, [n], dev) for i, n in enumerate(SIZES)]
    with ratel_lib(**cfg_kw):
        for b in blocks:
            b.register()
        for t in range(1, steps + 1):
            for b in blocks:
                b.load_grads(t)
            torch.cuda.synchronize()
            R.ratel_adam_step(1e-3, 0.9, 0.999, 1e-8, 1e-2, t)
            for b in reversed(blocks):
                R.ratel_offload_grad_chunk(b.id, None)
            R.ratel_sync(None)
    return blocks


@pytest.mark.parametrize("world", [2, 4, 8])
def test_ranks_simulated_bitwise_equal_single_rank(cuda_dev, tmp_path, world):
    steps = 3
    ref = _single_rank(cuda_dev, steps)
    libs = [R.lib()]
    for r in range(1, world):
        lib_copy = tmp_path / f"libratel_rank{r}.so"
        shutil.copy(R.LIB_PATH, lib_copy)
        libs.append(R.load_library(str(lib_copy)))
    ranks = [[GpuBlock(i, [n], cuda_dev, world=world, rank=r) for i, n in enumerate(SIZES)]
             for r in range(world)]
    for r, L in enumerate(libs):
        cfg = R.ratel_config()
        L.ratel_default_config(ctypes.byref(cfg))
        cfg.comm = R.RATEL_COMM_NONE
        assert L.ratel_init(0, r, world, None, ctypes.byref(cfg)) == 0, L.ratel_last_error()
        for b in ranks[r]:
            rr = (R.ratel_range * 1)(*b.ranges())
            assert L.ratel_register_block(b.id, rr, 1, R.RATEL_DEVICE) == 0, L.ratel_last_error()
    try:
        for t in range(1, steps + 1):
            for r in range(world):
                for b in ranks[r]:
                    b.load_grads(t)   # full-range grads; each rank reads its slice
            torch.cuda.synchronize()
            for L, blocks in zip(libs, ranks):
                assert L.ratel_adam_step(1e-3, 0.9, 0.999, 1e-8, 1e-2, t) == 0
                for b in reversed(blocks):
                    assert L.ratel_offload_grad_chunk(b.id, None) == 0
                assert L.ratel_sync(None) == 0
            # X2 by hand: every rank receives the other rank's P16 slice
            for i, n in enumerate(SIZES):
                s = R.ratel_padded_numel(n, world) // world
                for src in range(world):
                    for dst in range(world):
                        if src != dst:
                            ranks[dst][i].p16[0][src * s:(src + 1) * s].copy_(
                                ranks[src][i].p16[0][src * s:(src + 1) * s])
            torch.cuda.synchronize()
        for i, n in enumerate(SIZES):
            want = ref[i].gpu_state(0)
            cap = R.ratel_padded_numel(n, world)
            for r in range(world):
                p = ranks[r][i].p16[0]
                assert torch.equal(p[:n].view(torch.int16).cpu(),
                                   torch.from_numpy(want["p16"].view(np.int16)))
                assert torch.count_nonzero(p[n:cap].view(torch.int16)) == 0     # pads stay zero
            for k, attr in (("p32", "master"), ("m32", "m"), ("v32", "v")):
                parts = []
                for r in range(world):
                    beg, end = R.ratel_rank_slice(n, world, r)
                    if end > beg:
                        parts.append(getattr(ranks[r][i], attr)[0][:end - beg].cpu().numpy())
                got = np.concatenate(parts)
                assert np.array_equal(got.view(np.uint32), want[k].view(np.uint32)), (i, k)
    finally:
        for L in libs:
            L.ratel_finalize()


@pytest.mark.parametrize("clip", [0.0, 1e-3])
def test_one_rank_nccl_communicator_is_bit_neutral(cuda_dev, clip):
    a = _single_rank(cuda_dev, 2, max_grad_norm=clip)
    b = _single_rank(cuda_dev, 2, max_grad_norm=clip, comm=R.RATEL_COMM_NCCL)
    for x, y in zip(a, b):
        sx, sy = x.gpu_state(0), y.gpu_state(0)
        for k in ("p32", "m32", "v32"):
            assert np.array_equal(sx[k].view(np.uint32), sy[k].view(np.uint32)), k
        assert np.array_equal(sx["p16"], sy["p16"])
