"""N > 1 ranks on a REAL NCCL communicator (NEXT N1).

Every rank is its own process, as under torchrun; torch.distributed runs on
NCCL and the library's communicator is bootstrapped through it exactly as in
production (paper_conf_icde_liaosyxcyww25_b200.dist.init_distributed: rank 0's
ratel_get_nccl_unique_id broadcast over the torch group).  What runs:

  * the per-block in-place bf16 all-gather X2 (device and pinned-host states);
  * the clip: per-rank K2 partials, K3, the 8-byte fp64 allreduce X1 -> one
    global coefficient on every rank (the global norm over all ranks' slices);
  * the fused data-parallel path (ratel_register_peer_grads + _peer_params:
    every rank's update kernel reduces the N local G16 of its slice and stores
    its P16 slice into every rank's buffer) with the library's own NCCL
    barriers (hand-off ready barrier, sync barrier) and no test-side ordering;
  * ratel_refresh_params (checkpoint resume): P16 rebuilt from the masters and
    all-gathered (NCCL and peer stores).

With >= 2 GPUs: one GPU per rank (up to 8).  With one GPU (gpurun): 2 ranks
share cuda:0 -- NCCL refuses two ranks on one device of one host, so each rank
gets its own NCCL host id (NCCL_HOSTID) and they talk over loopback sockets;
the data path (collective calls, buffers, counts, ordering) is the real one,
only the transport differs.  Results are checked against the oracle's
unsharded step (plain) or data-parallel step (fused) under the R13 bounds,
and every rank's gathered P16 must be identical.
"""
import os
import socket

import numpy as np
import pytest
import torch

import oracle
import synth
from tests.tolerance import check_range

pytestmark = pytest.mark.gpu

SIZES = [300_001, 65_560, 1_000_003, 24]
BLOCKS = [[n] for n in SIZES]                         # one range per block
BLOCKS_MULTI = [[300_001, 24, 4_104], [65_560, 1_000_003]]   # several ranges per block (weights + biases)
STEPS = 3
HPK = dict(lr=1e-3, beta1=0.9, beta2=0.999, eps=1e-8, weight_decay=1e-2)


def _plan(world=None):
    """(world, shared): one GPU per rank when the box has them, else every
    rank on cuda:0 with its own NCCL host id."""
    n = torch.cuda.device_count()
    if world is None:
        return (min(n, 8), False) if n >= 2 else (2, True)
    return world, n < world


def rank_grad(n, step, block, q):
    return synth.grad16(n, step=step, block=block + 1000 * q)


def _free_port():
    with socket.socket() as s:
        s.bind(("127.0.0.1", 0))
        return s.getsockname()[1]


def _split(g, sizes):
    offs = np.concatenate([[0], np.cumsum(sizes)]).astype(int)
    return [g[offs[j]:offs[j + 1]] for j in range(len(sizes))]


def _rank_main(rank, world, shared, port, mode, pinned, clip, chans, res_q, blocks_spec=BLOCKS):
    if shared:   # distinct NCCL "hosts" on one GPU, loopback sockets (set before any communicator)
        os.environ["NCCL_HOSTID"] = f"ratel-test-rank{rank}"
        os.environ["NCCL_SOCKET_IFNAME"] = "lo"
        os.environ["NCCL_IB_DISABLE"] = "1"
    import torch.distributed as dist

    import paper_conf_icde_liaosyxcyww25_b200 as R
    from paper_conf_icde_liaosyxcyww25_b200 import dist as rdist
    from tests.harness import GpuBlock, torch_to_u16, u16_to_torch

    dev_i = 0 if shared else rank
    torch.cuda.set_device(dev_i)
    dev = torch.device("cuda", dev_i)
    dist.init_process_group("nccl", init_method=f"tcp://127.0.0.1:{port}", rank=rank, world_size=world,
                            device_id=dev)
    cfg = R.ratel_default_config()
    cfg.max_grad_norm = clip
    cfg.tile_elems = 1 << 17                        # pinned: several ring tiles per slice
    try:
        got_rank, got_world = rdist.init_distributed(dev_i, cfg)
        assert (got_rank, got_world) == (rank, world)
        blocks = [GpuBlock(i, sz, dev, pinned=pinned, world=world, rank=rank) for i, sz in enumerate(blocks_spec)]
        fused = mode == "fused"
        if fused:                                   # every rank's G16 / P16 mapped here (CUDA IPC)
            mine = [[(b.g16[j], b.p16[j]) for j in range(len(b.sizes))] for b in blocks]
            for q in range(world):
                if q != rank:
                    chans[(rank, q)].put(mine)
            peers = {rank: mine}
            for q in range(world):
                if q != rank:
                    peers[q] = chans[(q, rank)].get()
            torch.cuda.synchronize()
        for b in blocks:
            b.register()
            if fused:
                for j in range(len(b.sizes)):
                    R.ratel_register_peer_grads(b.id, j, [peers[q][b.id][j][0].data_ptr() for q in range(world)],
                                                1.0 / world)
                    R.ratel_register_peer_params(b.id, j, [peers[q][b.id][j][1].data_ptr() for q in range(world)])
        s = torch.cuda.Stream(device=dev)
        norms = []
        for t in range(1, STEPS + 1):
            with torch.cuda.stream(s):              # this rank's "backward"
                for b in blocks:
                    g = rank_grad(b.total, t, b.id, rank) if fused else synth.grad16(b.total, step=t, block=b.id)
                    for j, gj in enumerate(_split(g, b.sizes)):
                        b.g16[j][:b.sizes[j]].copy_(u16_to_torch(gj, dev))
            R.ratel_adam_step(HPK["lr"], HPK["beta1"], HPK["beta2"], HPK["eps"], HPK["weight_decay"], t)
            for b in reversed(blocks):              # decreasing index, as backward produces them
                R.ratel_offload_grad_chunk(b.id, s)
            R.ratel_sync(s)
            s.synchronize()
            if clip > 0:
                norms.append(R.ratel_get_grad_sumsq())
        out = []
        for b in blocks:
            for j, n in enumerate(b.sizes):
                beg, end = R.ratel_rank_slice(n, world, rank)
                k = end - beg
                cap = R.ratel_padded_numel(n, world)
                out.append(dict(p32=b.master[j][:k].cpu().numpy(), m32=b.m[j][:k].cpu().numpy(),
                                v32=b.v[j][:k].cpu().numpy(), p16=torch_to_u16(b.p16[j][:n]),
                                pad_nonzero=int(torch.count_nonzero(b.p16[j][n:cap].view(torch.int16)))))
        # checkpoint resume: scramble P16, refresh from the masters, all-gathered
        for b in blocks:
            for p16 in b.p16:
                p16.fill_(7.0)
        torch.cuda.synchronize()
        dist.barrier()                              # nobody's refresh may land before a peer scrambled
        for b in blocks:
            R.ratel_refresh_params(b.id, s)
        s.synchronize()
        refreshed = [torch_to_u16(b.p16[j][:n]) for b in blocks for j, n in enumerate(b.sizes)]
        res_q.put((rank, out, norms, refreshed))
    except BaseException as e:  # report, then let the parent fail
        res_q.put((rank, repr(e), None, None))
        raise
    finally:
        try:
            R.ratel_finalize()
        except Exception:
            pass
        try:
            dist.barrier()                          # keep exported IPC buffers alive until all are done
            dist.destroy_process_group()
        except Exception:
            pass


def _run(mode, pinned, clip, blocks_spec=BLOCKS, world=None):
    world, shared = _plan(world)
    ctx = torch.multiprocessing.get_context("spawn")
    chans = {(a, b): ctx.Queue() for a in range(world) for b in range(world) if a != b}
    res_q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_rank_main, args=(r, world, shared, port, mode, pinned, clip, chans, res_q,
                                                              blocks_spec))
             for r in range(world)]
    for p in procs:
        p.start()
    results = {}
    try:
        for _ in range(world):
            r, out, norms, refreshed = res_q.get(timeout=600)
            assert not isinstance(out, str), f"rank {r}: {out}"
            results[r] = (out, norms, refreshed)
    finally:
        for p in procs:
            p.join(timeout=120)
            if p.is_alive():
                p.kill()
    assert all(p.exitcode == 0 for p in procs), [p.exitcode for p in procs]
    return world, results


def _refs(world, fused, clip, blocks_spec=BLOCKS):
    """Oracle ranges in (block, range) order; the inputs exactly as the
    GpuBlocks draw them (one synth stream per block, split by range)."""
    refs = [oracle.Range.fresh(t) for i, sz in enumerate(blocks_spec)
            for t in _split(synth.theta0(sum(sz), block=i), sz)]
    sums = []
    for t in range(1, STEPS + 1):
        hp = oracle.hparams(step=t, **HPK)
        if fused:
            per_rank = [[g for i, sz in enumerate(blocks_spec) for g in _split(rank_grad(sum(sz), t, i, q), sz)]
                        for q in range(world)]
            S, _ = oracle.adam_step_dp(refs, [[per_rank[q][k] for q in range(world)] for k in range(len(refs))],
                                       1.0 / world, hp, max_grad_norm=clip)
        else:
            S, _ = oracle.adam_step(refs, [g for i, sz in enumerate(blocks_spec)
                                           for g in _split(synth.grad16(sum(sz), step=t, block=i), sz)], hp,
                                    max_grad_norm=clip)
        sums.append(S)
    return refs, sums


def _check(world, results, refs, sums, what):
    n_all = sum(r.p32.size for r in refs)
    for i in range(len(refs)):
        got = {k: np.concatenate([results[r][0][i][k] for r in range(world)]) for k in ("p32", "m32", "v32")}
        got["p16"] = results[0][0][i]["p16"]
        check_range(got, refs[i], own_rne=oracle.bf16_rne, what=f"{what} block {i}")
        for r in range(world):   # every rank holds the same gathered P16; pads stay zero
            assert np.array_equal(results[r][0][i]["p16"], results[0][0][i]["p16"]), (what, i, r)
            assert results[r][0][i]["pad_nonzero"] == 0, (what, i, r)
            # refresh: bf16_rne(master) of every rank's slice, gathered everywhere
            assert np.array_equal(results[r][2][i], oracle.bf16_rne(got["p32"])), (what, "refresh", i, r)
    if sums[0] is not None:
        for r in range(world):   # the clip allreduce: one global norm on every rank (all ranks' slices)
            for t, S in enumerate(sums):
                # both double sums of exact squares, in different orders: n * 2^-53 relative
                assert abs(results[r][1][t] - S) <= n_all * 2.0 ** -53 * S, (what, r, t, results[r][1][t], S)
            assert results[r][1] == results[0][1]


@pytest.mark.parametrize("pinned,clip", [(False, 0.0), (False, 1e-3), (True, 0.0), (True, 1e-3)])
def test_nccl_allgather_and_clip_vs_oracle(cuda_dev, pinned, clip):
    world, results = _run("plain", pinned, clip)
    refs, sums = _refs(world, False, clip)
    _check(world, results, refs, sums, f"nccl N={world} pinned={pinned} clip={clip}")


@pytest.mark.parametrize("pinned,clip,multi", [(False, 0.0, False), (True, 1e-3, False), (False, 0.0, True),
                                               (True, 1e-3, True)])
def test_nccl_fused_reduce_scatter_and_allgather_vs_oracle(cuda_dev, pinned, clip, multi):
    spec = BLOCKS_MULTI if multi else BLOCKS
    world, results = _run("fused", pinned, clip, spec)
    refs, sums = _refs(world, True, clip, spec)
    _check(world, results, refs, sums, f"fused N={world} pinned={pinned} clip={clip} multi={multi}")


@pytest.mark.parametrize("world", [4, 8])
def test_nccl_allgather_and_fused_at_4_and_8_ranks(cuda_dev, world):
    """N = 4 and 8 ranks: slices padded to 8N elements (ragged tails, a
    24-element range with empty slices on most ranks), the in-place NCCL
    all-gather with clip, then the fused path, all on a real communicator."""
    for mode, clip in (("plain", 1e-3), ("fused", 0.0)):
        w, results = _run(mode, False, clip, BLOCKS, world=world)
        refs, sums = _refs(w, mode == "fused", clip, BLOCKS)
        _check(w, results, refs, sums, f"{mode} N={w} clip={clip}")


def test_nccl_allgather_multirange_vs_oracle(cuda_dev):
    world, results = _run("plain", False, 1e-3, BLOCKS_MULTI)
    refs, sums = _refs(world, False, 1e-3, BLOCKS_MULTI)
    _check(world, results, refs, sums, f"nccl N={world} multi-range clip")
