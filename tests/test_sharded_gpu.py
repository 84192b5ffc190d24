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


def _single_rank(dev, steps, self_peer=False, **cfg_kw):
    blocks = [GpuBlock(i, [n], dev) for i, n in enumerate(SIZES)]
    with ratel_lib(**cfg_kw):
        for b in blocks:
            b.register()
            if self_peer:   # the fused all-gather path with a one-rank world: barrier only
                R.ratel_register_peer_params(b.id, 0, [b.p16[0]])
        for t in range(1, steps + 1):
            for b in blocks:
                b.load_grads(t)
            torch.cuda.synchronize()
            R.ratel_adam_step(1e-3, 0.9, 0.999, 1e-8, 1e-2, t)
            for b in reversed(blocks):
                R.ratel_offload_grad_chunk(b.id, None)
            R.ratel_sync(None)
    return blocks


@pytest.mark.parametrize("world,fused", [(2, False), (4, False), (8, False), (2, True), (4, True), (8, True)])
def test_ranks_simulated_bitwise_equal_single_rank(cuda_dev, tmp_path, world, fused):
    """fused=True: ratel_register_peer_params -- each rank's update kernel
    stores its P16 slice straight into the other ranks' buffers (here all on
    one GPU), so no exchange is played by the test."""
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
            if fused:
                ptrs = (ctypes.c_void_p * world)(*[ranks[q][b.id].p16[0].data_ptr() for q in range(world)])
                assert L.ratel_register_peer_params(b.id, 0, ptrs, world) == 0, L.ratel_last_error()
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
            for i, n in enumerate(SIZES if not fused else []):
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


@pytest.mark.parametrize("clip,self_peer", [(0.0, False), (1e-3, False), (0.0, True)])
def test_one_rank_nccl_communicator_is_bit_neutral(cuda_dev, clip, self_peer):
    a = _single_rank(cuda_dev, 2, max_grad_norm=clip)
    b = _single_rank(cuda_dev, 2, self_peer=self_peer, max_grad_norm=clip, comm=R.RATEL_COMM_NCCL)
    for x, y in zip(a, b):
        sx, sy = x.gpu_state(0), y.gpu_state(0)
        for k in ("p32", "m32", "v32"):
            assert np.array_equal(sx[k].view(np.uint32), sy[k].view(np.uint32)), k
        assert np.array_equal(sx["p16"], sy["p16"])


def test_symmetric_memory_peer_pointers_one_rank(cuda_dev):
    """The bench's --fused-allgather plumbing on one GPU: P16 allocated in
    torch symmetric memory, peer pointers from rendezvous, registered with
    ratel_register_peer_params under a one-rank NCCL communicator."""
    import torch.distributed as dist
    try:
        import torch.distributed._symmetric_memory as symm_mem
    except ImportError:
        pytest.skip("torch symmetric memory unavailable")
    import socket
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    port = s.getsockname()[1]
    s.close()
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    dist.init_process_group("nccl", rank=0, world_size=1, device_id=cuda_dev)
    try:
        ref = _single_rank(cuda_dev, 2)
        n = SIZES[0]
        b = GpuBlock(0, [n], cuda_dev)
        p = symm_mem.empty(R.ratel_padded_numel(n, 1), dtype=torch.bfloat16, device=cuda_dev)
        p.zero_()
        hdl = symm_mem.rendezvous(p, dist.group.WORLD.group_name)
        ptrs = list(hdl.buffer_ptrs)
        assert len(ptrs) == 1 and ptrs[0] == p.data_ptr()
        b.p16[0] = p
        with ratel_lib(comm=R.RATEL_COMM_NCCL):
            b.register()
            R.ratel_register_peer_params(0, 0, ptrs)
            for t in (1, 2):
                b.load_grads(t)
                torch.cuda.synchronize()
                R.ratel_adam_step(1e-3, 0.9, 0.999, 1e-8, 1e-2, t)
                R.ratel_offload_grad_chunk(0, None)
                R.ratel_sync(None)
        got, want = b.gpu_state(0), ref[0].gpu_state(0)
        assert np.array_equal(got["p16"], want["p16"])
        assert np.array_equal(got["p32"].view(np.uint32), want["p32"].view(np.uint32))
    finally:
        dist.destroy_process_group()
