"""Fused data-parallel gradient reduction (R17).

`ratel_register_peer_grads` hands the update kernel every rank's local
full-range G16; each rank's kernel reduces (fp64 sum in rank order, x scale,
one rounding) and updates its own slice -- the reduce-scatter folded into K1.
gpurun gives one GPU, so N ranks are simulated in one process with N
separately loaded copies of libratel.so on the same device (RATEL_COMM_NONE;
the test orders the ranks' backward before any hand-off, and plays or fuses
the all-gather).  Every rank's slice and the gathered P16 are checked against
the oracle's data-parallel step (oracle.adam_step_dp) under the R13 bounds.
A one-rank NCCL communicator exercises the barrier allreduces.
"""
import ctypes
import shutil

import numpy as np
import pytest
import torch

import oracle
import synth
import paper_conf_icde_liaosyxcyww25_b200 as R
from tests.harness import HP, GpuBlock, ratel_lib, torch_to_u16, u16_to_torch
from tests.tolerance import check_range

pytestmark = pytest.mark.gpu

SIZES = [300_001, 65_560, 1_000_003, 24]


def rank_grad(n, step, block, q):
    """Rank q's local bf16 gradient of block `block` at `step`."""
    return synth.grad16(n, step=step, block=block + 1000 * q)


_copies = [0]


def _libs(tmp_path, world):
    """Rank 0 = the package library; ranks 1.. = fresh copies (never reuse a
    file name: overwriting a loaded .so would crash the process)."""
    libs = [R.lib()]
    for r in range(1, world):
        _copies[0] += 1
        p = tmp_path / f"libratel_rs{r}_{_copies[0]}.so"
        shutil.copy(R.LIB_PATH, p)
        libs.append(R.load_library(str(p)))
    return libs


def _oracle_refs(steps, world, scale, clip=0.0, sizes=SIZES):
    refs = [oracle.Range.fresh(synth.theta0(n, block=i)) for i, n in enumerate(sizes)]
    for t in range(1, steps + 1):
        oracle.adam_step_dp(refs, [[rank_grad(n, t, i, q) for q in range(world)] for i, n in enumerate(sizes)],
                            scale, oracle.hparams(step=t, **HP), max_grad_norm=clip)
    return refs


def _simulate(dev, tmp_path, world, steps, pinned=False, fused=False, scale=None, k1_kernel=None):
    """N ranks on one GPU; returns (ranks' GpuBlocks)."""
    scale = 1.0 / world if scale is None else scale
    libs = _libs(tmp_path, world)
    ranks = [[GpuBlock(i, [n], dev, pinned=pinned, world=world, rank=r) for i, n in enumerate(SIZES)]
             for r in range(world)]
    for r, L in enumerate(libs):
        cfg = R.ratel_config()
        L.ratel_default_config(ctypes.byref(cfg))
        cfg.comm = R.RATEL_COMM_NONE
        cfg.tile_elems = 1 << 17       # pinned: several ring tiles per slice
        if k1_kernel is not None:
            cfg.k1_kernel = k1_kernel
        assert L.ratel_init(0, r, world, None, ctypes.byref(cfg)) == 0, L.ratel_last_error()
        for b in ranks[r]:
            rr = (R.ratel_range * 1)(*b.ranges())
            res = R.RATEL_PINNED_HOST if pinned else R.RATEL_DEVICE
            assert L.ratel_register_block(b.id, rr, 1, res) == 0, L.ratel_last_error()
            gptrs = (ctypes.c_void_p * world)(*[ranks[q][b.id].g16[0].data_ptr() for q in range(world)])
            assert L.ratel_register_peer_grads(b.id, 0, gptrs, world, scale) == 0, L.ratel_last_error()
            if fused:
                pptrs = (ctypes.c_void_p * world)(*[ranks[q][b.id].p16[0].data_ptr() for q in range(world)])
                assert L.ratel_register_peer_params(b.id, 0, pptrs, world) == 0, L.ratel_last_error()
    try:
        for t in range(1, steps + 1):
            for r in range(world):       # every rank's backward, before any hand-off
                for b in ranks[r]:
                    n = b.sizes[0]
                    b.g16[0][:n].copy_(u16_to_torch(rank_grad(n, t, b.id, r), dev))
            torch.cuda.synchronize()
            for L, blocks in zip(libs, ranks):
                assert L.ratel_adam_step(HP["lr"], HP["beta1"], HP["beta2"], HP["eps"], HP["weight_decay"], t) == 0
                for b in reversed(blocks):
                    assert L.ratel_offload_grad_chunk(b.id, None) == 0, L.ratel_last_error()
            for L in libs:
                assert L.ratel_sync(None) == 0, L.ratel_last_error()
            if not fused:                 # X2 played by the test
                for i, n in enumerate(SIZES):
                    s = R.ratel_padded_numel(n, world) // world
                    for src in range(world):
                        for dst in range(world):
                            if src != dst:
                                ranks[dst][i].p16[0][src * s:(src + 1) * s].copy_(
                                    ranks[src][i].p16[0][src * s:(src + 1) * s])
            torch.cuda.synchronize()
    finally:
        for L in libs:
            L.ratel_finalize()
    return ranks


def _gathered(ranks, i, n, world):
    parts = {k: [] for k in ("p32", "m32", "v32")}
    for r in range(world):
        beg, end = R.ratel_rank_slice(n, world, r)
        if end > beg:
            b = ranks[r][i]
            parts["p32"].append(b.master[0][:end - beg].cpu().numpy())
            parts["m32"].append(b.m[0][:end - beg].cpu().numpy())
            parts["v32"].append(b.v[0][:end - beg].cpu().numpy())
    got = {k: np.concatenate(v) for k, v in parts.items()}
    got["p16"] = torch_to_u16(ranks[0][i].p16[0][:n])
    return got


@pytest.mark.parametrize("world,pinned,fused", [(2, False, False), (4, False, False), (8, False, False),
                                                (4, True, False), (8, False, True), (3, True, True)])
def test_fused_reduction_simulated_ranks_vs_oracle(cuda_dev, tmp_path, world, pinned, fused):
    steps = 3
    ranks = _simulate(cuda_dev, tmp_path, world, steps, pinned=pinned, fused=fused)
    refs = _oracle_refs(steps, world, 1.0 / world)
    for i, n in enumerate(SIZES):
        got = _gathered(ranks, i, n, world)
        check_range(got, refs[i], own_rne=oracle.bf16_rne, what=f"rs N={world} block {i}")
        for r in range(1, world):      # every rank holds the same gathered P16
            assert torch.equal(ranks[r][i].p16[0][:n].view(torch.int16), ranks[0][i].p16[0][:n].view(torch.int16))
        cap = R.ratel_padded_numel(n, world)
        for r in range(world):
            assert torch.count_nonzero(ranks[r][i].p16[0][n:cap].view(torch.int16)) == 0


@pytest.mark.parametrize("world,pinned,fused", [(4, False, False), (8, False, True), (3, True, True)])
def test_fused_reduction_tma_kernel_equals_ldg_kernel_bitwise(cuda_dev, tmp_path, world, pinned, fused):
    """The TMA-staged K1-RS (default) and the register-staged one reduce in
    the same fp64 rank order and run the same adam_update(): same bits."""
    a = _simulate(cuda_dev, tmp_path, world, 2, pinned=pinned, fused=fused, k1_kernel=R.RATEL_UPDATE_TMA)
    b = _simulate(cuda_dev, tmp_path, world, 2, pinned=pinned, fused=fused, k1_kernel=R.RATEL_UPDATE_LDG)
    for i, n in enumerate(SIZES):
        ga, gb = _gathered(a, i, n, world), _gathered(b, i, n, world)
        for k in ("p32", "m32", "v32"):
            assert np.array_equal(ga[k].view(np.uint32), gb[k].view(np.uint32)), (i, k)
        assert np.array_equal(ga["p16"], gb["p16"])


def test_fused_reduction_residency_bitwise(cuda_dev, tmp_path):
    """Device vs pinned-host states under the fused reduction: same bits."""
    a = _simulate(cuda_dev, tmp_path, 4, 2, pinned=False)
    b = _simulate(cuda_dev, tmp_path, 4, 2, pinned=True)
    for i, n in enumerate(SIZES):
        ga, gb = _gathered(a, i, n, 4), _gathered(b, i, n, 4)
        for k in ("p32", "m32", "v32"):
            assert np.array_equal(ga[k].view(np.uint32), gb[k].view(np.uint32)), (i, k)
        assert np.array_equal(ga["p16"], gb["p16"])


def _one_rank(dev, steps, scale=None, clip=0.0, pinned=False, comm=R.RATEL_COMM_NONE, block_wait=False):
    blocks = [GpuBlock(i, [n], dev, pinned=pinned) for i, n in enumerate(SIZES)]
    with ratel_lib(max_grad_norm=clip, comm=comm, tile_elems=1 << 17):
        for b in blocks:
            b.register()
            if scale is not None:
                R.ratel_register_peer_grads(b.id, 0, [None], scale)
        for t in range(1, steps + 1):
            for b in blocks:
                n = b.sizes[0]
                b.g16[0][:n].copy_(u16_to_torch(rank_grad(n, t, b.id, 0), dev))
            torch.cuda.synchronize()
            R.ratel_adam_step(HP["lr"], HP["beta1"], HP["beta2"], HP["eps"], HP["weight_decay"], t)
            for b in reversed(blocks):
                R.ratel_offload_grad_chunk(b.id, None)
                if block_wait:
                    R.ratel_block_wait(b.id, torch.cuda.current_stream().cuda_stream)
            R.ratel_sync(None)
    return blocks


@pytest.mark.parametrize("scale,clip,pinned", [(0.5, 0.0, False), (0.5, 1e-3, False), (3.0, 0.0, True),
                                               (0.25, 1e-3, True)])
def test_fused_reduction_one_rank_scale_and_clip(cuda_dev, scale, clip, pinned):
    """World 1: g = fp32(scale * g16); with clip, the norm is of that g (K2-RS)."""
    steps = 3
    blocks = _one_rank(cuda_dev, steps, scale=scale, clip=clip, pinned=pinned)
    refs = _oracle_refs(steps, 1, scale, clip=clip)
    for i, b in enumerate(blocks):
        check_range(b.gpu_state(0), refs[i], own_rne=oracle.bf16_rne, what=f"rs1 block {i}")


def test_fused_reduction_n1_scale1_is_the_plain_path_bitwise(cuda_dev):
    """One rank, scale 1: fp32(1.0 * bf16) == bf16, so the RS kernel must give
    the TMA kernel's bits exactly (same adam_update, R16)."""
    a = _one_rank(cuda_dev, 3)
    b = _one_rank(cuda_dev, 3, scale=1.0)
    for x, y in zip(a, b):
        sx, sy = x.gpu_state(0), y.gpu_state(0)
        for k in ("p32", "m32", "v32"):
            assert np.array_equal(sx[k].view(np.uint32), sy[k].view(np.uint32)), k
        assert np.array_equal(sx["p16"], sy["p16"])


@pytest.mark.parametrize("clip,block_wait", [(0.0, False), (1e-3, False), (0.0, True)])
def test_fused_reduction_one_rank_nccl_barriers_bit_neutral(cuda_dev, clip, block_wait):
    """A one-rank NCCL communicator runs the per-block ready barrier, the
    collective block_wait release and the sync barrier: no bit changes."""
    a = _one_rank(cuda_dev, 2, scale=0.5, clip=clip)
    b = _one_rank(cuda_dev, 2, scale=0.5, clip=clip, comm=R.RATEL_COMM_NCCL, block_wait=block_wait)
    for x, y in zip(a, b):
        sx, sy = x.gpu_state(0), y.gpu_state(0)
        for k in ("p32", "m32", "v32"):
            assert np.array_equal(sx[k].view(np.uint32), sy[k].view(np.uint32)), k
        assert np.array_equal(sx["p16"], sy["p16"])


def test_fused_reduction_mixed_ranges_in_one_block(cuda_dev, tmp_path):
    """A 2-range block where only range 1 registers peer grads (world 2):
    range 0 takes this rank's own full-range grad, range 1 the mean."""
    world, steps, sizes = 2, 2, [40_003, 70_001]
    libs = _libs(tmp_path, world)
    ranks = [GpuBlock(0, sizes, cuda_dev, world=world, rank=r) for r in range(world)]
    for r, L in enumerate(libs):
        cfg = R.ratel_config()
        L.ratel_default_config(ctypes.byref(cfg))
        cfg.comm = R.RATEL_COMM_NONE
        assert L.ratel_init(0, r, world, None, ctypes.byref(cfg)) == 0
        rr = (R.ratel_range * 2)(*ranks[r].ranges())
        assert L.ratel_register_block(0, rr, 2, R.RATEL_DEVICE) == 0
        g = (ctypes.c_void_p * world)(*[ranks[q].g16[1].data_ptr() for q in range(world)])
        assert L.ratel_register_peer_grads(0, 1, g, world, 0.5) == 0, L.ratel_last_error()
    th0 = synth.theta0(sum(sizes), block=0)
    ref0 = [oracle.Range.fresh(th0[:sizes[0]]) for _ in range(world)]   # per-rank plain reference for range 0
    ref1 = oracle.Range.fresh(th0[sizes[0]:])
    try:
        for t in range(1, steps + 1):
            g0 = [rank_grad(sizes[0], t, 7, q) for q in range(world)]
            g1 = [rank_grad(sizes[1], t, 8, q) for q in range(world)]
            for q in range(world):
                ranks[q].g16[0][:sizes[0]].copy_(u16_to_torch(g0[q], cuda_dev))
                ranks[q].g16[1][:sizes[1]].copy_(u16_to_torch(g1[q], cuda_dev))
            torch.cuda.synchronize()
            for L in libs:
                assert L.ratel_adam_step(HP["lr"], HP["beta1"], HP["beta2"], HP["eps"], HP["weight_decay"], t) == 0
                assert L.ratel_offload_grad_chunk(0, None) == 0
            for L in libs:
                assert L.ratel_sync(None) == 0
            hp = oracle.hparams(step=t, **HP)
            for q in range(world):
                oracle.adam_range(ref0[q], g0[q], hp)
            oracle.adam_range_gd(ref1, oracle.reduce_grads(g1, 0.5), hp)
    finally:
        for L in libs:
            L.ratel_finalize()
    # range 1: the slices together are the data-parallel step
    parts = {k: [] for k in ("p32", "m32", "v32")}
    for q in range(world):
        beg, end = R.ratel_rank_slice(sizes[1], world, q)
        parts["p32"].append(ranks[q].master[1][:end - beg].cpu().numpy())
        parts["m32"].append(ranks[q].m[1][:end - beg].cpu().numpy())
        parts["v32"].append(ranks[q].v[1][:end - beg].cpu().numpy())
    got = {k: np.concatenate(v) for k, v in parts.items()}
    p16 = np.concatenate([torch_to_u16(ranks[q].p16[1][R.ratel_rank_slice(sizes[1], world, q)[0]:
                                                       R.ratel_rank_slice(sizes[1], world, q)[1]])
                          for q in range(world)])
    got["p16"] = p16
    check_range(got, ref1, own_rne=oracle.bf16_rne, what="mixed range 1")
    # range 0: rank q's slice is rank q's own plain step on its own grad
    for q in range(world):
        beg, end = R.ratel_rank_slice(sizes[0], world, q)
        sub = ref0[q]
        ref = oracle.Range(sub.p32[beg:end].copy(), sub.m32[beg:end].copy(), sub.v32[beg:end].copy(),
                           sub.p16[beg:end].copy(), 1, sub.theta_bar[beg:end].copy(), sub.m_bar[beg:end].copy())
        got0 = dict(p32=ranks[q].master[0][:end - beg].cpu().numpy(), m32=ranks[q].m[0][:end - beg].cpu().numpy(),
                    v32=ranks[q].v[0][:end - beg].cpu().numpy(), p16=torch_to_u16(ranks[q].p16[0][beg:end]))
        check_range(got0, ref, own_rne=oracle.bf16_rne, what=f"mixed range 0 rank {q}")


def test_register_peer_grads_errors(cuda_dev):
    b = GpuBlock(0, [1000], cuda_dev)
    hc = GpuBlock(1, [1000], cuda_dev, host_compute=True)
    with ratel_lib():
        b.register()
        hc.register()
        for args, code in [((0, 0, [None, None], 0.5), R.RATEL_EINVAL),    # n != world
                           ((0, 0, [None], 0.0), R.RATEL_EINVAL),           # scale must be > 0
                           ((0, 0, [None], float("inf")), R.RATEL_EINVAL),
                           ((0, 1, [None], 1.0), R.RATEL_EINVAL),           # range out of range
                           ((5, 0, [None], 1.0), R.RATEL_EINVAL),           # not registered
                           ((1, 0, [None], 1.0), R.RATEL_EINVAL)]:          # HOST_COMPUTE
            with pytest.raises(R.RatelError) as e:
                R.ratel_register_peer_grads(*args)
            assert e.value.code == code, args
        R.ratel_adam_step(1e-3, 0.9, 0.999, 1e-8, 0.0, 1)
        with pytest.raises(R.RatelError) as e:                              # step in flight
            R.ratel_register_peer_grads(0, 0, [None], 1.0)
        assert e.value.code == R.RATEL_ESTATE
    sl = GpuBlock(2, [1000], cuda_dev)
    with ratel_lib():
        rng = sl.ranges()[0]
        rng.grad_is_rank_slice = 1
        R.ratel_register_block(2, [rng])
        with pytest.raises(R.RatelError) as e:                              # needs a full-range grad
            R.ratel_register_peer_grads(2, 0, [None], 1.0)
        assert e.value.code == R.RATEL_EINVAL


@pytest.mark.parametrize("k1_kernel", [R.RATEL_UPDATE_TMA, R.RATEL_UPDATE_LDG])
def test_fused_reduction_slice_beyond_2pow32_sampled_vs_oracle(cuda_dev, k1_kernel):
    """Maximum sizes for the fused reduction: rank 0 of a simulated world 2
    owns a slice of 2^32 + 4104 elements of one range (both ranks' full-range
    G16 resident here, ~103 GB in all), so the TMA-staged kernel's tile offsets
    and the peer-grad pointers cross 2^31 and 2^32 and the slice ends in a
    scalar tail.  Two steps; sampled elements around both boundaries and the
    end of the slice vs the oracle's data-parallel step (R17)."""
    n = 2 * ((1 << 32) + 4099)
    world, scale = 2, 0.5
    beg, end = R.ratel_rank_slice(n, world, 0)
    s = end - beg
    assert beg == 0 and s > (1 << 32)
    picks = [np.arange(0, 32), np.arange((1 << 31) - 40, (1 << 31) + 40), np.arange((1 << 32) - 40, (1 << 32) + 40),
             np.arange(s - 40, s), np.random.default_rng(6).integers(0, s, 50_000)]
    idx = np.unique(np.concatenate(picks)).astype(np.uint64)
    cfg = R.ratel_default_config()
    cfg.comm = R.RATEL_COMM_NONE
    cfg.k1_kernel = k1_kernel
    R.ratel_init(0, 0, world, None, cfg)
    try:
        cap = R.ratel_padded_numel(n, world)
        gq = [torch.empty(cap, dtype=torch.bfloat16, device=cuda_dev) for _ in range(world)]
        th = torch.empty(s, dtype=torch.float32, device=cuda_dev)
        R.ratel_gen_theta0(th.data_ptr(), s, 0, R.ratel_gen_stream_key(synth.SEED, synth.TAG_THETA, 0, 0))
        m, v = torch.zeros(s, device=cuda_dev), torch.zeros(s, device=cuda_dev)
        p = torch.zeros(cap, dtype=torch.bfloat16, device=cuda_dev)
        R.ratel_register_block(0, [R.make_range(p, gq[0], th, m, v, n)], R.RATEL_DEVICE)
        R.ratel_register_peer_grads(0, 0, gq, scale)
        ref = oracle.Range.fresh(synth.theta0_at(idx, block=0))
        for t in (1, 2):
            for q in range(world):
                R.ratel_gen_grad16(gq[q].data_ptr(), n, 0, R.ratel_gen_stream_key(synth.SEED, synth.TAG_GRAD, t, 1000 * q))
            torch.cuda.synchronize()
            R.ratel_adam_step(HP["lr"], HP["beta1"], HP["beta2"], HP["eps"], HP["weight_decay"], t)
            R.ratel_offload_grad_chunk(0, None)
            R.ratel_sync(None)
            gd = oracle.reduce_grads([synth.grad16_at(idx, step=t, block=1000 * q) for q in range(world)], scale)
            oracle.adam_range_gd(ref, gd, oracle.hparams(step=t, **HP))
        ii = torch.from_numpy(idx.astype(np.int64)).to(cuda_dev)
        got = dict(p32=th[ii].cpu().numpy(), m32=m[ii].cpu().numpy(), v32=v[ii].cpu().numpy(),
                   p16=torch_to_u16(p[ii]))
        check_range(got, ref, own_rne=oracle.bf16_rne, what=f"RS slice 2^32+ (k1_kernel {k1_kernel})")
        assert np.array_equal(got["p16"], oracle.bf16_rne(got["p32"]))
    finally:
        R.ratel_finalize()
        del gq, th, m, v, p
        torch.cuda.empty_cache()
