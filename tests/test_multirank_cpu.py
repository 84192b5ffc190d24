"""World-size-2 host logic over gloo (CPU): the N>1 path minus the GPU.

1. The NCCL unique-id bootstrap (dist.broadcast_unique_id) delivers rank 0's
   bytes to every rank.
2. The range partition (ratel_rank_slice, the C library's function) plus the
   two collectives the library issues -- the 8-byte sum-of-squares allreduce
   (X1) and the per-range bf16 all-gather (X2), played here by gloo -- turn
   per-rank oracle updates of the owned slices into exactly the unsharded
   step: bitwise without clipping (elementwise independence, R16), within
   the R13 bounds with clipping (only the order of the norm's sum changes).
"""
import os
import socket

import numpy as np
import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp

import oracle
import synth
import paper_conf_icde_liaosyxcyww25_b200 as R
from paper_conf_icde_liaosyxcyww25_b200 import dist as rdist

SIZES = [1, 9, 4097, 100_003, 789_760]
WORLD = 2


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _sharded_steps(rank, world, steps, max_norm):
    """Each rank updates only its slices; results gathered on every rank."""
    hp = dict(lr=1e-3, beta1=0.9, beta2=0.999, eps=1e-8, weight_decay=1e-2)
    shards = []
    for b, n in enumerate(SIZES):
        beg, end = R.ratel_rank_slice(n, world, rank)
        th = synth.theta0(n, block=b)[beg:end]
        shards.append((beg, end, oracle.Range.fresh(th) if end > beg else None))
    for t in range(1, steps + 1):
        grads = [synth.grad16(n, step=t, block=b) for b, n in enumerate(SIZES)]
        coef = 1.0
        if max_norm > 0:
            local = 0.0
            for (beg, end, _), g in zip(shards, grads):
                local = oracle.grad_sumsq(g[beg:end], local)
            S = torch.tensor([local], dtype=torch.float64)
            dist.all_reduce(S)                                     # X1
            coef = oracle.clip_coef(float(S.item()), max_norm)
        for (beg, end, r), g in zip(shards, grads):
            if r is not None:
                oracle.adam_range(r, g[beg:end], oracle.hparams(step=t, **hp), coef)
    out = []
    for b, n in enumerate(SIZES):
        cap = R.ratel_padded_numel(n, world)
        s = cap // world
        beg, end, r = shards[b]
        mine = np.zeros(s, np.uint16)
        if r is not None:
            mine[:end - beg] = r.p16
        full = torch.zeros(cap, dtype=torch.int32)  # gloo has no 16-bit ints: widen
        dist.all_gather_into_tensor(full, torch.from_numpy(mine.astype(np.int32)))  # X2
        st = {}
        for k in ("p32", "m32", "v32"):
            part = np.zeros(s, np.float32)
            if r is not None:
                part[:end - beg] = getattr(r, k)
            allp = torch.zeros(cap, dtype=torch.float32)
            dist.all_gather_into_tensor(allp, torch.from_numpy(part))
            st[k] = allp.numpy()[:n]
        st["p16"] = full.numpy().astype(np.uint16)[:n]
        st["pad"] = full.numpy().astype(np.uint16)[n:]
        out.append(st)
    return out


def _worker(rank, world, port, steps, max_norm, q):
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        uid = rdist.broadcast_unique_id(getter=lambda: bytes(range(128)))
        assert uid == bytes(range(128))
        res = _sharded_steps(rank, world, steps, max_norm)
        q.put((rank, res))
    except Exception as e:  # report instead of leaving the parent waiting
        q.put((rank, repr(e)))
        raise
    finally:
        dist.destroy_process_group()


def _run(steps, max_norm):
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    ps = [ctx.Process(target=_worker, args=(r, WORLD, port, steps, max_norm, q)) for r in range(WORLD)]
    for p in ps:
        p.start()
    res = dict(q.get(timeout=120) for _ in ps)
    for r, v in res.items():
        assert not isinstance(v, str), f"rank {r}: {v}"
    for p in ps:
        p.join(timeout=60)
        assert p.exitcode == 0
    return res


def _unsharded(steps, max_norm):
    hp = dict(lr=1e-3, beta1=0.9, beta2=0.999, eps=1e-8, weight_decay=1e-2)
    rs = [oracle.Range.fresh(synth.theta0(n, block=b)) for b, n in enumerate(SIZES)]
    for t in range(1, steps + 1):
        grads = [synth.grad16(n, step=t, block=b) for b, n in enumerate(SIZES)]
        oracle.adam_step(rs, grads, oracle.hparams(step=t, **hp), max_grad_norm=max_norm)
    return rs


def test_sharded_step_bitwise_equals_unsharded():
    res = _run(3, 0.0)
    ref = _unsharded(3, 0.0)
    for rank in range(WORLD):
        for st, r in zip(res[rank], ref):
            assert np.array_equal(st["p16"], r.p16)
            assert np.all(st["pad"] == 0)
            for k in ("p32", "m32", "v32"):
                assert np.array_equal(st[k].view(np.uint32), getattr(r, k).view(np.uint32))


def test_sharded_clip_within_bounds():
    from tests.tolerance import check_range
    res = _run(3, 1e-3)
    ref = _unsharded(3, 1e-3)
    for st, r in zip(res[0], ref):
        check_range(st, r, own_rne=oracle.bf16_rne)
    # every rank holds the same gathered P16
    for a, b in zip(res[0], res[1]):
        assert np.array_equal(a["p16"], b["p16"])
