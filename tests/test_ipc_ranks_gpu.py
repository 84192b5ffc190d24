"""Fused reduce-scatter + update + all-gather across real PROCESSES (SURVEY
NEXT N1, R17, §8(e)).

tests/test_reduce_gpu.py simulates N ranks inside one process (N copies of
libratel.so sharing one address space).  Here every rank is its own process,
as under torchrun: each allocates its own G16 / P16 / states, the peers'
G16 and P16 buffers reach it through CUDA IPC (torch.multiprocessing tensor
sharing = cudaIpcGetMemHandle / cudaIpcOpenMemHandle), and it registers
those mapped pointers with ratel_register_peer_grads / _peer_params -- the
same calls a multi-GPU job makes with NVLink peer mappings.  gpurun gives one
GPU, so all ranks share cuda:0; ordering between ranks is a gloo barrier
(RATEL_COMM_NONE: no NCCL, which refuses two ranks on one GPU).  Every rank's
slice and every rank's gathered P16 are checked against the oracle's
data-parallel step (oracle.adam_step_dp) under the R13 bounds.
"""
import numpy as np
import pytest
import torch

import oracle
from tests.tolerance import check_range
from tests.test_reduce_gpu import SIZES, _oracle_refs, rank_grad

pytestmark = pytest.mark.gpu

STEPS = 3


def _rank_main(rank, world, init_file, chans, res_q, fused, pinned):
    import torch.distributed as dist

    import paper_conf_icde_liaosyxcyww25_b200 as R
    from tests.harness import HP, GpuBlock, torch_to_u16, u16_to_torch

    dist.init_process_group("gloo", init_method=f"file://{init_file}", rank=rank, world_size=world)
    torch.cuda.set_device(0)
    dev = torch.device("cuda", 0)
    blocks = [GpuBlock(i, [n], dev, pinned=pinned, world=world, rank=rank) for i, n in enumerate(SIZES)]
    mine = [(b.g16[0], b.p16[0]) for b in blocks]
    for q in range(world):                         # publish this rank's buffers (CUDA IPC handles)
        if q != rank:
            chans[(rank, q)].put(mine)
    peers = {rank: mine}
    for q in range(world):                         # map every peer's buffers into this process
        if q != rank:
            peers[q] = chans[(q, rank)].get()
    torch.cuda.synchronize()

    cfg = R.ratel_default_config()
    cfg.comm = R.RATEL_COMM_NONE
    cfg.tile_elems = 1 << 17
    R.ratel_init(0, rank, world, None, cfg)
    try:
        for b in blocks:
            b.register()
            R.ratel_register_peer_grads(b.id, 0, [peers[q][b.id][0].data_ptr() for q in range(world)], 1.0 / world)
            if fused:
                R.ratel_register_peer_params(b.id, 0, [peers[q][b.id][1].data_ptr() for q in range(world)])
        for t in range(1, STEPS + 1):
            for b in blocks:                       # this rank's backward
                n = b.sizes[0]
                b.g16[0][:n].copy_(u16_to_torch(rank_grad(n, t, b.id, rank), dev))
            torch.cuda.synchronize()
            dist.barrier()                         # every rank's G16 complete (the per-block ready barrier)
            R.ratel_adam_step(HP["lr"], HP["beta1"], HP["beta2"], HP["eps"], HP["weight_decay"], t)
            for b in reversed(blocks):
                R.ratel_offload_grad_chunk(b.id, None)
            R.ratel_sync(None)                     # host-blocking: this rank's updates (and peer stores) done
            dist.barrier()                         # nobody overwrites a G16 another rank still reads
            if not fused:                          # X2 played through the IPC mappings
                for b in blocks:
                    s = R.ratel_padded_numel(b.sizes[0], world) // world
                    for q in range(world):
                        if q != rank:
                            b.p16[0][q * s:(q + 1) * s].copy_(peers[q][b.id][1][q * s:(q + 1) * s])
                torch.cuda.synchronize()
                dist.barrier()
        out = []
        for b in blocks:
            n = b.sizes[0]
            beg, end = R.ratel_rank_slice(n, world, rank)
            k = end - beg
            cap = R.ratel_padded_numel(n, world)
            out.append(dict(p32=b.master[0][:k].cpu().numpy(), m32=b.m[0][:k].cpu().numpy(),
                            v32=b.v[0][:k].cpu().numpy(), p16=torch_to_u16(b.p16[0][:n]),
                            pad_nonzero=int(torch.count_nonzero(b.p16[0][n:cap].view(torch.int16)))))
        res_q.put((rank, out))
    finally:
        R.ratel_finalize()
        dist.barrier()                             # keep exported buffers alive until every rank is done
        dist.destroy_process_group()


@pytest.mark.parametrize("world,fused,pinned", [(2, True, False), (3, True, True), (2, False, False)])
def test_fused_reduction_across_processes_vs_oracle(cuda_dev, tmp_path, world, fused, pinned):
    ctx = torch.multiprocessing.get_context("spawn")
    chans = {(a, b): ctx.Queue() for a in range(world) for b in range(world) if a != b}
    res_q = ctx.Queue()
    init_file = tmp_path / "gloo_init"
    procs = [ctx.Process(target=_rank_main, args=(r, world, str(init_file), chans, res_q, fused, pinned))
             for r in range(world)]
    for p in procs:
        p.start()
    results = {}
    try:
        for _ in range(world):
            r, out = res_q.get(timeout=600)
            results[r] = out
    finally:
        for p in procs:
            p.join(timeout=120)
            if p.is_alive():
                p.kill()
    assert all(p.exitcode == 0 for p in procs), [p.exitcode for p in procs]

    refs = _oracle_refs(STEPS, world, 1.0 / world)
    for i, n in enumerate(SIZES):
        got = {k: np.concatenate([results[r][i][k] for r in range(world)]) for k in ("p32", "m32", "v32")}
        got["p16"] = results[0][i]["p16"]
        check_range(got, refs[i], own_rne=oracle.bf16_rne, what=f"ipc N={world} fused={fused} block {i}")
        for r in range(world):                     # every process holds the same gathered P16, pads zero
            assert np.array_equal(results[r][i]["p16"], results[0][i]["p16"]), (i, r)
            assert results[r][i]["pad_nonzero"] == 0, (i, r)
