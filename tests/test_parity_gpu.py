"""GPU parity: the CUDA path through the C ABI vs the CPU oracle.

Bounds: DESIGN.md R13 (tests/tolerance.py) at tol 1e-5 -- BASELINE.json's
"max relative error 1e-5" and "bf16 within 1 ulp" read against the scale the
oracle tracks.  Self-consistency claims (R16) are bitwise.
"""
import math
import numpy as np
import pytest
import torch

import oracle
import synth
import paper_conf_icde_liaosyxcyww25_b200 as R
from tests.harness import HP, GpuBlock, ratel_lib, torch_to_u16, u16_to_torch
from tests.tolerance import check_range

pytestmark = pytest.mark.gpu

# C1 (BASELINE.json configs[0]): one GPT block, h = 256 -> 12h^2 + 13h params,
# the 12 tensors of SURVEY §8(d): ln1 w/b, qkv W/b, proj W/b, ln2 w/b, fc1 W/b, fc2 W/b.
H = 256
C1_SIZES = [H, H, 3 * H * H, 3 * H, H * H, H, H, H, 4 * H * H, 4 * H, 4 * H * H, H]
C1_WD = [0, 0, 1, 0, 1, 0, 0, 0, 1, 0, 1, 0]
assert sum(C1_SIZES) == 789_760


def oracle_step(blocks, step, grads, mode=oracle.ADAMW, max_norm=0.0, **hp):
    h = dict(HP, **hp)
    rs, gs = [], []
    for b in blocks:
        rs += b.oracle
        gs += grads[b.id]
    return oracle.adam_step(rs, gs, oracle.hparams(step=step, mode=mode, **h), max_grad_norm=max_norm)


def run(blocks, steps, mode=oracle.ADAMW, max_norm=0.0, order="decreasing", arm="before",
        check_every=True, tol=1e-5, hp_sched=None, **cfg_kw):
    """Drive `steps` optimizer steps through the ABI and the oracle; check."""
    dev = blocks[0].dev
    reports = []
    with ratel_lib(mode=mode, max_grad_norm=max_norm, **cfg_kw):
        for b in blocks:
            b.register()
        bwd = torch.cuda.Stream()
        rng = np.random.default_rng(7)
        for t in range(1, steps + 1):
            h = dict(HP)
            if hp_sched:
                h.update(hp_sched(t))
            grads = {}
            for b in blocks:
                grads[b.id] = b.load_grads(t)
            torch.cuda.synchronize()
            ids = [b.id for b in blocks]
            if order == "decreasing":
                ids = sorted(ids, reverse=True)
            elif order == "random":
                ids = list(rng.permutation(ids))
            if arm == "before":
                R.ratel_adam_step(h["lr"], h["beta1"], h["beta2"], h["eps"], h["weight_decay"], t)
            for i in ids:
                R.ratel_offload_grad_chunk(int(i), bwd)
            if arm == "after":
                R.ratel_adam_step(h["lr"], h["beta1"], h["beta2"], h["eps"], h["weight_decay"], t)
            R.ratel_sync(None)
            S, coef = oracle_step(blocks, t, grads, mode=mode, max_norm=max_norm, **h)
            if max_norm > 0:
                got = R.ratel_get_grad_sumsq()
                n_all = sum(sum(b.sizes) for b in blocks)  # positive terms: |err| <= n u S
                assert abs(got - S) <= n_all * 2.0 ** -53 * S, (got, S)
            if check_every or t == steps:
                for b in blocks:
                    for i in range(len(b.sizes)):
                        reports.append(check_range(b.gpu_state(i), b.oracle[i], tol=tol,
                                                   own_rne=oracle.bf16_rne,
                                                   what=f"step {t} block {b.id} range {i}"))
    return reports


def snapshot(blocks):
    return [[b.gpu_state(i) for i in range(len(b.sizes))] for b in blocks]


def assert_bitwise(sa, sb):
    for xa, xb in zip(sa, sb):
        for ra, rb in zip(xa, xb):
            for k in ("p32", "m32", "v32", "p16"):
                assert np.array_equal(ra[k].view(np.uint32) if ra[k].dtype == np.float32 else ra[k],
                                      rb[k].view(np.uint32) if rb[k].dtype == np.float32 else rb[k]), k


# ------------------------------------------------------------------ C1 parity
def test_c1_flat_range_10_steps(cuda_dev):
    b = GpuBlock(0, [sum(C1_SIZES)], cuda_dev)
    reps = run([b], 10)
    worst = max(r["theta_scaled"] for r in reps)
    assert worst < 1e-5
    print("C1 flat worst scaled errors:", {k: max(r[k] for r in reps)
                                           for k in ("theta_scaled", "m_scaled", "v_rel", "p16_ulps_at_scale")})


def test_c1_twelve_ranges_wd_exempt(cuda_dev):
    b = GpuBlock(0, C1_SIZES, cuda_dev, wd_flags=C1_WD)
    run([b], 10)


def test_c1_adam_l2_mode(cuda_dev):
    b = GpuBlock(0, C1_SIZES, cuda_dev, wd_flags=C1_WD)
    run([b], 10, mode=oracle.ADAM_L2)


def test_lr_schedule_flows_per_step(cuda_dev):
    b = GpuBlock(3, [100_003], cuda_dev)
    run([b], 6, hp_sched=lambda t: dict(lr=1e-3 * (0.5 ** t), weight_decay=0.1 * t))


@pytest.mark.parametrize("max_norm", [1e-3, 1e6])
def test_clip_global_norm(cuda_dev, max_norm):
    blocks = [GpuBlock(i, [50_000 + 13 * i, 777], cuda_dev) for i in range(3)]
    run(blocks, 5, max_norm=max_norm)


def test_ragged_sizes_many_blocks(cuda_dev):
    sizes = [[1], [7], [8], [9], [15, 17], [1023], [1_000_003], [4096 * 3 + 5, 1]]
    blocks = [GpuBlock(i, s, cuda_dev) for i, s in enumerate(sizes)]
    run(blocks, 4, order="random")


def test_special_values_propagate(cuda_dev):
    """Non-finite grads propagate (torch default, R8); eps, zeros handled."""
    b = GpuBlock(0, [64], cuda_dev)
    with ratel_lib():
        b.register()
        g = b.grads_np(1)[0].copy()
        g[:6] = [0x7F80, 0xFF80, 0x7FC0, 0x0000, 0x8000, 0x0001]  # +inf -inf nan +0 -0 denormal
        b.g16[0][:64].copy_(u16_to_torch(g, cuda_dev))
        torch.cuda.synchronize()
        R.ratel_adam_step(1e-3, 0.9, 0.999, 1e-8, 1e-2, 1)
        R.ratel_offload_grad_chunk(0, None)
        R.ratel_sync(None)
        oracle.adam_range(b.oracle[0], g, oracle.hparams(step=1))
        check_range(b.gpu_state(0), b.oracle[0], own_rne=oracle.bf16_rne)


# ------------------------------------------------ self-consistency (R16)
def _fresh(sizes_list, dev, **kw):
    return [GpuBlock(i, s, dev, **kw) for i, s in enumerate(sizes_list)]


SIZES = [[300_001], [65_536 + 24], [4_000, 12, 999]]


def test_bitwise_handoff_order_and_deferred(cuda_dev):
    a = _fresh(SIZES, cuda_dev)
    run(a, 3, order="decreasing", arm="before", check_every=False)
    b = _fresh(SIZES, cuda_dev)
    run(b, 3, order="random", arm="before", check_every=False)
    c = _fresh(SIZES, cuda_dev)
    run(c, 3, order="decreasing", arm="after", check_every=False)  # "Ratel+ZeRO" deferred
    sa = snapshot(a)
    assert_bitwise(sa, snapshot(b))
    assert_bitwise(sa, snapshot(c))


@pytest.mark.parametrize("depth,staging,tile", [(2, 0, 4096), (3, 0, 65_536), (3, 1, 8192), (2, 0, 1 << 24),
                                                (2, 2, 4096)])
def test_pinned_host_bitwise_equals_device(cuda_dev, depth, staging, tile):
    a = _fresh(SIZES, cuda_dev)
    run(a, 3, check_every=False)
    b = _fresh(SIZES, cuda_dev, pinned=True)
    run(b, 3, check_every=False, pipeline_depth=depth, staging=staging, tile_elems=tile)
    assert_bitwise(snapshot(a), snapshot(b))


@pytest.mark.parametrize("max_ctas", [1, 3, 37])
def test_max_ctas_cap_bitwise(cuda_dev, max_ctas):
    """A capped grid makes every CTA cycle its shared-memory stage ring many
    times (the TMA pipeline's phase/release logic); results must not move."""
    a = _fresh(SIZES, cuda_dev)
    run(a, 2, check_every=False)
    b = _fresh(SIZES, cuda_dev)
    run(b, 2, check_every=False, max_ctas=max_ctas)
    assert_bitwise(snapshot(a), snapshot(b))


@pytest.mark.parametrize("cta_tiles,clip", [(1, 0.0), (3, 0.0), (8, 0.05), (1000, 0.0)])
def test_cta_tiles_nonpersistent_grid_bitwise(cuda_dev, cta_tiles, clip):
    """cfg.cta_tiles > 0: a non-persistent grid whose CTAs retire after
    cta_tiles tiles (ragged last CTA, tiles crossing range boundaries, one CTA
    covering everything at 1000) must update every element exactly as the
    persistent grid does, also in clip mode, and match the oracle."""
    a = _fresh(SIZES, cuda_dev)
    run(a, 2, check_every=False, max_norm=clip)
    b = _fresh(SIZES, cuda_dev)
    run(b, 2, max_norm=clip, cta_tiles=cta_tiles)
    assert_bitwise(snapshot(a), snapshot(b))


@pytest.mark.parametrize("kernel,max_ctas", [(1, 0), (2, 0), (2, 5)])
def test_k1_kernel_variants_bitwise(cuda_dev, kernel, max_ctas):
    """cfg.k1_kernel = LDG / LDG_LITE (register-staged, no shared memory)
    gives the TMA kernel's bits and matches the oracle (also capped)."""
    a = _fresh(SIZES, cuda_dev)
    run(a, 2, check_every=False)
    b = _fresh(SIZES, cuda_dev)
    run(b, 2, k1_kernel=kernel, max_ctas=max_ctas)
    assert_bitwise(snapshot(a), snapshot(b))


@pytest.mark.parametrize("mode,max_norm,max_ctas", [(oracle.ADAMW, 0.0, 0), (oracle.ADAM_L2, 0.05, 0),
                                                     (oracle.ADAMW, 0.05, 3)])
def test_zero_copy_staging_vs_oracle(cuda_dev, mode, max_norm, max_ctas):
    """RATEL_STAGING_ZERO_COPY: the update kernel reads/writes the pinned
    host states in place over the link; oracle parity (clip, Adam-L2, a
    3-CTA grid cycling many times) and bitwise = device residency."""
    a = _fresh(SIZES, cuda_dev)
    run(a, 3, mode=mode, max_norm=max_norm, check_every=False)
    b = _fresh(SIZES, cuda_dev, pinned=True)
    run(b, 3, mode=mode, max_norm=max_norm, staging=2, max_ctas=max_ctas)
    assert_bitwise(snapshot(a), snapshot(b))


def test_cta_tiles_pinned_host_bitwise(cuda_dev):
    a = _fresh(SIZES, cuda_dev)
    run(a, 2, check_every=False)
    b = _fresh(SIZES, cuda_dev, pinned=True)
    run(b, 2, check_every=False, tile_elems=65_536, cta_tiles=2)
    assert_bitwise(snapshot(a), snapshot(b))


def test_large_block_ring_wraps_vs_oracle(cuda_dev):
    """20M + 5 elements, two ranges: ~33 tiles per CTA at the full grid."""
    b = GpuBlock(0, [20_000_005, 4_096 * 7 + 3], cuda_dev)
    run([b], 3)


def test_overlapped_with_backward_stream(cuda_dev):
    """Grads are produced on a side stream right before each hand-off (the
    AGO pattern); a busy GEMM keeps that stream occupied so K1 must wait on
    the event, not on host order."""
    blocks = _fresh([[200_000], [150_000], [99_999]], cuda_dev)
    with ratel_lib():
        for b in blocks:
            b.register()
        bwd = torch.cuda.Stream()
        x = torch.randn(4096, 4096, device=cuda_dev, dtype=torch.bfloat16)
        for t in (1, 2, 3):
            grads = {b.id: b.grads_np(t) for b in blocks}
            host = {b.id: [u16_to_torch(g, "cpu").pin_memory() for g in grads[b.id]] for b in blocks}
            torch.cuda.synchronize()
            R.ratel_adam_step(1e-3, 0.9, 0.999, 1e-8, 1e-2, t)
            with torch.cuda.stream(bwd):
                for b in sorted(blocks, key=lambda b: -b.id):
                    for _ in range(4):
                        x = (x @ x).clamp_(-1, 1)          # "backward" work
                    for i, hg in enumerate(host[b.id]):
                        b.g16[i][:hg.numel()].copy_(hg, non_blocking=True)
                    R.ratel_offload_grad_chunk(b.id, bwd)
            R.ratel_sync(torch.cuda.current_stream())
            torch.cuda.synchronize()
            oracle_step(blocks, t, grads)
            for b in blocks:
                check_range(b.gpu_state(0), b.oracle[0], own_rne=oracle.bf16_rne)


def test_no_staleness_after_stream_sync(cuda_dev):
    """ratel_sync(stream): work queued on `stream` afterwards sees the updated
    P16, which equals bf16_rne(P32) bit for bit (footnote 4)."""
    b = GpuBlock(0, [1 << 20], cuda_dev)
    with ratel_lib():
        b.register()
        s = torch.cuda.Stream()
        for t in (1, 2):
            b.load_grads(t)
            torch.cuda.synchronize()
            R.ratel_adam_step(1e-3, 0.9, 0.999, 1e-8, 1e-2, t)
            R.ratel_offload_grad_chunk(0, None)
            R.ratel_sync(s)
            with torch.cuda.stream(s):
                snap = b.p16[0].clone()
                want = b.master[0].to(torch.bfloat16)  # torch's RNE cast, independent of K1
            s.synchronize()
            assert torch.equal(snap.view(torch.int16), want.view(torch.int16))


# --------------------------------------------------------- protocol errors
def test_protocol_errors(cuda_dev):
    b = GpuBlock(0, [1000], cuda_dev)
    c = GpuBlock(1, [1000], cuda_dev)
    with ratel_lib():
        b.register()
        c.register()
        with pytest.raises(R.RatelError) as e:
            b.register()
        assert e.value.code == R.RATEL_EINVAL
        R.ratel_adam_step(1e-3, 0.9, 0.999, 1e-8, 0.0, 1)
        with pytest.raises(R.RatelError) as e:
            R.ratel_adam_step(1e-3, 0.9, 0.999, 1e-8, 0.0, 2)  # already armed
        assert e.value.code == R.RATEL_ESTATE
        R.ratel_offload_grad_chunk(0, None)
        with pytest.raises(R.RatelError) as e:
            R.ratel_offload_grad_chunk(0, None)
        assert e.value.code == R.RATEL_ESTATE
        with pytest.raises(R.RatelError) as e:
            R.ratel_sync(None)  # block 1 missing
        assert e.value.code == R.RATEL_ESTATE
        with pytest.raises(R.RatelError) as e:
            R.ratel_offload_grad_chunk(7, None)
        assert e.value.code == R.RATEL_ESTATE
        R.ratel_offload_grad_chunk(1, None)
        R.ratel_sync(None)
        with pytest.raises(R.RatelError) as e:
            R.ratel_adam_step(1e-3, 0.9, 0.999, 1e-8, 0.0, 1)  # step must increase
        assert e.value.code == R.RATEL_ESTATE
        with pytest.raises(R.RatelError) as e:
            R.ratel_adam_step(1e-3, 1.0, 0.999, 1e-8, 0.0, 5)
        assert e.value.code == R.RATEL_EINVAL
        # pointer validation: pageable host memory, misalignment, wrong kind
        pageable = torch.zeros(1000, dtype=torch.float32)
        bad = R.make_range(b.p16[0], b.g16[0], pageable, pageable, pageable, 1000)
        with pytest.raises(R.RatelError) as e:
            R.ratel_register_block(5, [bad], R.RATEL_PINNED_HOST)
        assert e.value.code == R.RATEL_EINVAL
        with pytest.raises(R.RatelError) as e:
            R.ratel_register_block(5, [bad], R.RATEL_DEVICE)
        assert e.value.code == R.RATEL_EINVAL
        mis = R.make_range(b.p16[0].data_ptr() + 2, b.g16[0], b.master[0], b.m[0], b.v[0], 100)
        with pytest.raises(R.RatelError) as e:
            R.ratel_register_block(5, [mis], R.RATEL_DEVICE)
        assert e.value.code == R.RATEL_EINVAL
        # still healthy (EINVAL/ESTATE are not sticky)
        R.ratel_adam_step(1e-3, 0.9, 0.999, 1e-8, 0.0, 9)
        R.ratel_offload_grad_chunk(1, None)
        R.ratel_offload_grad_chunk(0, None)
        R.ratel_sync(None)
    with pytest.raises(R.RatelError) as e:
        R.ratel_sync(None)
    assert e.value.code == R.RATEL_ESTATE


@pytest.mark.parametrize("residency", ["device", "host_compute"])
def test_nonfinite_norm_reported(cuda_dev, residency):
    """A NaN gradient under clipping: the blocking sync reports RATEL_ENONFINITE
    and the NaN coefficient propagates (torch), also when only the CPU handler
    updates (no kernel sees the norm)."""
    b = GpuBlock(0, [4096], cuda_dev, host_compute=(residency == "host_compute"))
    with ratel_lib(max_grad_norm=1.0):
        b.register()
        g = b.grads_np(1)[0].copy()
        g[5] = 0x7FC0
        b.g16[0][:4096].copy_(u16_to_torch(g, cuda_dev))
        torch.cuda.synchronize()
        R.ratel_adam_step(1e-3, 0.9, 0.999, 1e-8, 1e-2, 1)
        R.ratel_offload_grad_chunk(0, None)
        with pytest.raises(R.RatelError) as e:
            R.ratel_sync(None)
        assert e.value.code == R.RATEL_ENONFINITE
        assert np.isnan(b.gpu_state(0)["p32"]).all()  # NaN coef propagates like torch


# -------------------------------------------------------- conversions / inputs
def test_gpu_bf16_rne_exhaustive(cuda_dev):
    """The device P16 conversion == the oracle's RNE for all 2^32 fp32 patterns
    (NaN: both NaN)."""
    chunk = 1 << 28
    out = torch.empty(chunk, dtype=torch.int16, device=cuda_dev)
    for start in range(0, 1 << 32, chunk):
        u = torch.arange(start, start + chunk, dtype=torch.int64, device=cuda_dev).to(torch.int32)
        x = u.view(torch.float32)
        R.ratel_test_bf16_rne(x.data_ptr(), out.data_ptr(), chunk)
        got = out.cpu().numpy().view(np.uint16)
        xs = x.cpu().numpy()
        ref = oracle.bf16_rne(xs)
        isn = np.isnan(xs)
        assert np.array_equal(got[~isn], ref[~isn]), start
        assert np.all((got[isn] & 0x7FFF) > 0x7F80)


def test_device_generator_matches_synth(cuda_dev):
    n, start = 3_000_017, 123_456_789
    for blk, step in ((0, 1), (5, 9)):
        kg = R.ratel_gen_stream_key(synth.SEED, synth.TAG_GRAD, step, blk)
        kt = R.ratel_gen_stream_key(synth.SEED, synth.TAG_THETA, 0, blk)
        assert kg == synth.stream_key(synth.SEED, synth.TAG_GRAD, step, blk)
        g = torch.empty(n, dtype=torch.int16, device=cuda_dev)
        th = torch.empty(n, dtype=torch.float32, device=cuda_dev)
        R.ratel_gen_grad16(g.data_ptr(), n, start, kg)
        R.ratel_gen_theta0(th.data_ptr(), n, start, kt)
        assert np.array_equal(g.cpu().numpy().view(np.uint16), synth.grad16(n, step, blk, start=start))
        assert np.array_equal(th.cpu().numpy().view(np.uint32),
                              synth.theta0(n, blk, start=start).view(np.uint32))


def test_grad_ring_recycling_with_block_wait(cuda_dev):
    """5 blocks share a ring of 2 gradient buffers: the backward stream waits
    (ratel_block_wait) for the update that consumed a slot before writing the
    next block's gradient into it -- the AGO memory pattern."""
    sizes = [70_001, 65_536, 40_000, 33_333, 8]
    blocks = _fresh([[n] for n in sizes], cuda_dev)
    cap = max(R.ratel_padded_numel(n, 1) for n in sizes)
    ring = [torch.zeros(cap, dtype=torch.bfloat16, device=cuda_dev) for _ in range(2)]
    for b in blocks:
        b.g16 = [ring[b.id % 2]]
    with ratel_lib():
        for b in blocks:
            b.register()
        bwd = torch.cuda.Stream()
        for t in (1, 2, 3):
            grads = {b.id: b.grads_np(t) for b in blocks}
            host = {b.id: u16_to_torch(grads[b.id][0], "cpu").pin_memory() for b in blocks}
            R.ratel_adam_step(1e-3, 0.9, 0.999, 1e-8, 1e-2, t)
            with torch.cuda.stream(bwd):
                order = sorted(blocks, key=lambda b: -b.id)
                for j, b in enumerate(order):
                    if j >= 2:
                        R.ratel_block_wait(b.id + 2, bwd)      # slot's previous block consumed
                    slot = ring[b.id % 2]
                    slot[:host[b.id].numel()].copy_(host[b.id], non_blocking=True)
                    R.ratel_offload_grad_chunk(b.id, bwd)
            R.ratel_sync(torch.cuda.current_stream())
            torch.cuda.synchronize()
            oracle_step(blocks, t, grads)
            for b in blocks:
                check_range(b.gpu_state(0), b.oracle[0], own_rne=oracle.bf16_rne, what=f"t{t} b{b.id}")
        # deferred arming: the update is not enqueued yet -> waiting is refused
        R.ratel_offload_grad_chunk(0, None)
        with pytest.raises(R.RatelError) as e:
            R.ratel_block_wait(0, None)
        assert e.value.code == R.RATEL_ESTATE
        R.ratel_adam_step(1e-3, 0.9, 0.999, 1e-8, 1e-2, 4)
        R.ratel_block_wait(0, None)
        for b in blocks[1:]:
            R.ratel_offload_grad_chunk(b.id, None)
        R.ratel_sync(None)


def test_fullsize_13b_blocks_sampled_vs_oracle(cuda_dev):
    """BASELINE configs[1] block size (314,639,360 params, h = 5120) in the
    bench's launch configuration, inputs from the device generator: sampled
    elements vs the oracle computed one by one; no-staleness on every element."""
    h = 5120
    n = 12 * h * h + 13 * h
    nblk, steps = 2, 3
    idx = np.unique(np.concatenate([np.arange(0, 64), np.arange(n - 64, n),
                                    np.random.default_rng(3).integers(0, n, 200_000)])).astype(np.uint64)
    state = []
    with ratel_lib():
        g = torch.empty(n, dtype=torch.bfloat16, device=cuda_dev)
        for b in range(nblk):
            th = torch.empty(n, dtype=torch.float32, device=cuda_dev)
            R.ratel_gen_theta0(th.data_ptr(), n, 0, R.ratel_gen_stream_key(synth.SEED, synth.TAG_THETA, 0, b))
            m = torch.zeros(n, device=cuda_dev)
            v = torch.zeros(n, device=cuda_dev)
            p = torch.zeros(n, dtype=torch.bfloat16, device=cuda_dev)
            state.append((p, th, m, v))
            R.ratel_register_block(b, [R.make_range(p, g, th, m, v, n)], R.RATEL_DEVICE)
        refs = [oracle.Range.fresh(synth.theta0_at(idx, block=b)) for b in range(nblk)]
        for t in range(1, steps + 1):
            R.ratel_adam_step(1e-3, 0.9, 0.999, 1e-8, 1e-2, t)
            for b in reversed(range(nblk)):
                # the single grad buffer is rewritten per block: wait for the previous consumer
                if b < nblk - 1:
                    R.ratel_block_wait(b + 1, None)
                R.ratel_gen_grad16(g.data_ptr(), n, 0, R.ratel_gen_stream_key(synth.SEED, synth.TAG_GRAD, t, b))
                R.ratel_offload_grad_chunk(b, None)
            R.ratel_sync(None)
            for b in range(nblk):
                oracle.adam_range(refs[b], synth.grad16_at(idx, step=t, block=b), oracle.hparams(step=t))
        ii = torch.from_numpy(idx.astype(np.int64)).to(cuda_dev)
        for b in range(nblk):
            p, th, m, v = state[b]
            got = dict(p32=th[ii].cpu().numpy(), m32=m[ii].cpu().numpy(), v32=v[ii].cpu().numpy(),
                       p16=torch_to_u16(p[ii]))
            check_range(got, refs[b], own_rne=oracle.bf16_rne, what=f"13B block {b}")
            assert torch.equal(p.view(torch.int16), th.to(torch.bfloat16).view(torch.int16))


def test_range_beyond_2pow32_elements_sampled_vs_oracle(cuda_dev):
    """Maximum sizes: one range of 2^32 + 4099 elements (69 GB of states and
    grads in HBM), so tile indices, element offsets and the generator's
    counters cross 2^31 and 2^32 (64-bit indexing everywhere) and the range
    ends in a ragged scalar tail.  Two steps; sampled elements around both
    boundaries and the tail vs the oracle; P16 == bf16(P32) on the samples."""
    n = (1 << 32) + 4099
    picks = [np.arange(0, 32), np.arange((1 << 31) - 40, (1 << 31) + 40), np.arange((1 << 32) - 40, (1 << 32) + 40),
             np.arange(n - 40, n), np.random.default_rng(5).integers(0, n, 50_000)]
    idx = np.unique(np.concatenate(picks)).astype(np.uint64)
    with ratel_lib():
        th = torch.empty(n, dtype=torch.float32, device=cuda_dev)
        R.ratel_gen_theta0(th.data_ptr(), n, 0, R.ratel_gen_stream_key(synth.SEED, synth.TAG_THETA, 0, 0))
        m = torch.zeros(n, device=cuda_dev)
        v = torch.zeros(n, device=cuda_dev)
        p = torch.zeros(R.ratel_padded_numel(n, 1), dtype=torch.bfloat16, device=cuda_dev)
        g = torch.empty(R.ratel_padded_numel(n, 1), dtype=torch.bfloat16, device=cuda_dev)
        R.ratel_register_block(0, [R.make_range(p, g, th, m, v, n)], R.RATEL_DEVICE)
        ref = oracle.Range.fresh(synth.theta0_at(idx, block=0))
        for t in (1, 2):
            R.ratel_gen_grad16(g.data_ptr(), n, 0, R.ratel_gen_stream_key(synth.SEED, synth.TAG_GRAD, t, 0))
            R.ratel_adam_step(1e-3, 0.9, 0.999, 1e-8, 1e-2, t)
            R.ratel_offload_grad_chunk(0, None)
            R.ratel_sync(None)
            oracle.adam_range(ref, synth.grad16_at(idx, step=t, block=0), oracle.hparams(step=t))
        ii = torch.from_numpy(idx.astype(np.int64)).to(cuda_dev)
        got = dict(p32=th[ii].cpu().numpy(), m32=m[ii].cpu().numpy(), v32=v[ii].cpu().numpy(),
                   p16=torch_to_u16(p[ii]))
        check_range(got, ref, own_rne=oracle.bf16_rne, what="2^32+ range")
        assert np.array_equal(got["p16"], oracle.bf16_rne(got["p32"]))
        # the P16 refresh (64-bit grid-stride indexing) over the same 2^32+ range
        p.fill_(2.0)
        R.ratel_refresh_params(0, None)
        assert np.array_equal(torch_to_u16(p[ii]), got["p16"])
    del th, m, v, p, g
    torch.cuda.empty_cache()


def test_fullsize_30b_blocks_clip_sampled_vs_oracle(cuda_dev):
    """BASELINE configs[2] block shape (616,655,872 params, h = 7168) with the
    global grad-norm clip (max_norm 1.0) in the bench's launch configuration:
    that block plus a small ragged one, two steps, device-generated inputs.  The oracle's norm runs
    over every element of both blocks (synth's grads, fp64 in index order) and
    must agree with the library's K2/K3 sum; sampled elements vs the oracle
    with that coefficient; P16 == bf16(P32) everywhere."""
    h = 7168
    ns = [12 * h * h + 13 * h, 1_000_003]     # a full block and a small ragged one share the norm
    nblk = 2
    idxs = [np.unique(np.concatenate([np.arange(0, 64), np.arange(n - 64, n),
                                      np.random.default_rng(4).integers(0, n, 100_000)])).astype(np.uint64)
            for n in ns]
    state = []
    with ratel_lib(max_grad_norm=1.0):
        gs = [torch.empty(n, dtype=torch.bfloat16, device=cuda_dev) for n in ns]
        for b in range(nblk):
            n = ns[b]
            th = torch.empty(n, dtype=torch.float32, device=cuda_dev)
            R.ratel_gen_theta0(th.data_ptr(), n, 0, R.ratel_gen_stream_key(synth.SEED, synth.TAG_THETA, 0, b))
            m, v = torch.zeros(n, device=cuda_dev), torch.zeros(n, device=cuda_dev)
            p = torch.zeros(n, dtype=torch.bfloat16, device=cuda_dev)
            state.append((p, th, m, v))
            R.ratel_register_block(b, [R.make_range(p, gs[b], th, m, v, n)], R.RATEL_DEVICE)
        refs = [oracle.Range.fresh(synth.theta0_at(idxs[b], block=b)) for b in range(nblk)]
        for t in (1, 2):
            S, parts = 0.0, []
            for b in range(nblk):
                n = ns[b]
                R.ratel_gen_grad16(gs[b].data_ptr(), n, 0, R.ratel_gen_stream_key(synth.SEED, synth.TAG_GRAD, t, b))
                g16 = synth.grad16(n, step=t, block=b)
                S = oracle.grad_sumsq(g16, S)
                for c in range(0, n, 1 << 24):   # squares of bf16 values are exact in fp64; pairwise sums
                    x = synth.bf16_bits_to_f32(g16[c:c + (1 << 24)]).astype(np.float64)
                    parts.append(float(np.sum(x * x)))
            S_acc = math.fsum(parts)             # accurate to ~1e-15 relative
            R.ratel_adam_step(1e-3, 0.9, 0.999, 1e-8, 1e-2, t)
            for b in reversed(range(nblk)):
                R.ratel_offload_grad_chunk(b, None)
            R.ratel_sync(None)
            s_gpu = R.ratel_get_grad_sumsq()
            # the library's fp64 tree of per-CTA partials is accurate; the oracle's plain
            # index-order recursion is within its textbook bound (n-1)*u*S (u = 2^-53)
            assert abs(s_gpu - S_acc) <= 1e-12 * S_acc, (s_gpu, S_acc)
            assert abs(S - S_acc) <= sum(ns) * 2.0 ** -53 * S_acc, (S, S_acc)
            coef = oracle.clip_coef(S, 1.0)
            assert coef < 1.0                     # the clip is active at this size
            for b in range(nblk):
                oracle.adam_range(refs[b], synth.grad16_at(idxs[b], step=t, block=b), oracle.hparams(step=t),
                                  coef=coef)
        for b in range(nblk):
            ii = torch.from_numpy(idxs[b].astype(np.int64)).to(cuda_dev)
            p, th, m, v = state[b]
            got = dict(p32=th[ii].cpu().numpy(), m32=m[ii].cpu().numpy(), v32=v[ii].cpu().numpy(),
                       p16=torch_to_u16(p[ii]))
            check_range(got, refs[b], own_rne=oracle.bf16_rne, what=f"30B block {b} (clip)")
            assert torch.equal(p.view(torch.int16), th.to(torch.bfloat16).view(torch.int16))
    del state, gs
    torch.cuda.empty_cache()


@pytest.mark.parametrize("h", [8192, 12288])
def test_fullsize_70b_block_pinned_host_sampled_vs_oracle(cuda_dev, h):
    """BASELINE configs[3] / configs[4] block shapes (70B: 805,412,864 params,
    h = 8192; 175B: 1,812,099,072 params, h = 12288) with theta/m/v in
    exact-size pinned host memory, streamed through the default tile ring (the
    bench's host configuration): two steps, sampled elements vs the oracle,
    P16 == bf16(P32) on every element."""
    n = 12 * h * h + 13 * h
    idx = np.unique(np.concatenate([np.arange(0, 64), np.arange(n - 64, n),
                                    np.random.default_rng(6).integers(0, n, 100_000)])).astype(np.uint64)
    owners = [R.pinned_tensor(n) for _ in range(3)]
    th, m, v = (o.tensor for o in owners)
    chunk = 1 << 26
    tmp = torch.empty(chunk, dtype=torch.float32, device=cuda_dev)
    for beg in range(0, n, chunk):
        k = min(chunk, n - beg)
        R.ratel_gen_theta0(tmp.data_ptr(), k, beg, R.ratel_gen_stream_key(synth.SEED, synth.TAG_THETA, 0, 0))
        th[beg:beg + k].copy_(tmp[:k])
    del tmp
    m.zero_()
    v.zero_()
    with ratel_lib():
        p = torch.zeros(n, dtype=torch.bfloat16, device=cuda_dev)
        g = torch.empty(n, dtype=torch.bfloat16, device=cuda_dev)
        R.ratel_register_block(0, [R.make_range(p, g, th, m, v, n)], R.RATEL_PINNED_HOST)
        ref = oracle.Range.fresh(synth.theta0_at(idx, block=0))
        for t in (1, 2):
            R.ratel_gen_grad16(g.data_ptr(), n, 0, R.ratel_gen_stream_key(synth.SEED, synth.TAG_GRAD, t, 0))
            R.ratel_adam_step(1e-3, 0.9, 0.999, 1e-8, 1e-2, t)
            R.ratel_offload_grad_chunk(0, None)
            R.ratel_sync(None)
            oracle.adam_range(ref, synth.grad16_at(idx, step=t, block=0), oracle.hparams(step=t))
        ii = torch.from_numpy(idx.astype(np.int64))
        got = dict(p32=th[ii].numpy().copy(), m32=m[ii].numpy().copy(), v32=v[ii].numpy().copy(),
                   p16=torch_to_u16(p[ii.to(cuda_dev)]))
        check_range(got, ref, own_rne=oracle.bf16_rne, what=f"h={h} block (pinned host)")
        for beg in range(0, n, chunk):     # no staleness on every element
            k = min(chunk, n - beg)
            assert torch.equal(p[beg:beg + k].view(torch.int16),
                               th[beg:beg + k].to(cuda_dev).to(torch.bfloat16).view(torch.int16))
        del p, g
    del th, m, v, owners
    torch.cuda.empty_cache()


def test_max_ranges_and_block_ids(cuda_dev):
    """A block with RATEL_MAX_RANGES_PER_BLOCK ranges (sizes 1..., mixed wd
    flags) under the largest block id, next to a one-range block; and the
    33rd range is rejected."""
    n_r = R.RATEL_MAX_RANGES_PER_BLOCK
    sizes = [1 + 37 * i for i in range(n_r)]
    big = GpuBlock(R.RATEL_MAX_BLOCKS - 1, sizes, cuda_dev, wd_flags=[i % 2 for i in range(n_r)])
    small = GpuBlock(0, [4096 * 3 + 1], cuda_dev)
    run([big, small], 3)
    with ratel_lib():
        b = GpuBlock(5, [8] * (n_r + 1), cuda_dev)
        with pytest.raises(R.RatelError) as e:
            R.ratel_register_block(5, b.ranges(), R.RATEL_DEVICE)
        assert e.value.code == R.RATEL_EINVAL
        with pytest.raises(R.RatelError) as e:
            R.ratel_register_block(R.RATEL_MAX_BLOCKS, b.ranges()[:1], R.RATEL_DEVICE)
        assert e.value.code == R.RATEL_EINVAL


def test_clip_adam_l2_pinned_host(cuda_dev):
    """Clip + Adam-L2 + pinned-host residency together, multi-range."""
    blocks = [GpuBlock(i, [30_011 + i, 515], cuda_dev, pinned=True, wd_flags=[1, 0]) for i in range(3)]
    run(blocks, 4, mode=oracle.ADAM_L2, max_norm=1e-3, tile_elems=4096)


# ------------------------------------------- HOST_COMPUTE (the paper's CPU handler)
@pytest.mark.parametrize("mode,max_norm", [(oracle.ADAMW, 0.0), (oracle.ADAM_L2, 0.0), (oracle.ADAMW, 1e-3)])
def test_host_compute_vs_oracle(cuda_dev, mode, max_norm):
    """RATEL_HOST_COMPUTE: G16 D2H, CPU AdamW (fp32, SIMD) on the pinned states,
    P16 H2D (§IV-C) -- ragged multi-range blocks, 5 steps."""
    blocks = [GpuBlock(0, [789_760 + 3, 256], cuda_dev, host_compute=True, wd_flags=[1, 0]),
              GpuBlock(1, [65_537], cuda_dev, host_compute=True)]
    run(blocks, 5, mode=mode, max_norm=max_norm, host_threads=4)


def test_mixed_residencies_in_one_step(cuda_dev):
    """Device, pinned-host and host-compute blocks handed off in one step,
    AGO order and random order, with clipping across all of them."""
    blocks = [GpuBlock(0, [100_003], cuda_dev),
              GpuBlock(1, [70_001, 9], cuda_dev, pinned=True),
              GpuBlock(2, [50_000], cuda_dev, host_compute=True),
              GpuBlock(3, [12_345], cuda_dev)]
    run(blocks, 3, order="random", max_norm=5e-3, tile_elems=8192)


@pytest.mark.parametrize("residency", ["device", "pinned", "host_compute"])
def test_grad_freed_after_record_stream_then_reused(cuda_dev, residency):
    """The ownership contract of ratel.h: a grad tensor freed right after its
    hand-off with grad.record_stream(ratel_optimizer_stream()) must not be
    recycled by torch's caching allocator before the update has read it --
    here the freed memory is immediately reallocated and overwritten."""
    n = 1_000_003
    b = GpuBlock(0, [n], cuda_dev, pinned=(residency == "pinned"), host_compute=(residency == "host_compute"))
    opt_stream = None
    with ratel_lib():
        b.register()
        opt_stream = torch.cuda.ExternalStream(R.ratel_optimizer_stream())
        for t in (1, 2, 3):
            g = b.grads_np(t)[0]
            gt = torch.empty(R.ratel_padded_numel(n, 1), dtype=torch.bfloat16, device=cuda_dev)
            gt[:n].copy_(u16_to_torch(g, cuda_dev))
            rng = R.make_range(b.p16[0], gt, b.master[0], b.m[0], b.v[0], n)
            # re-register the block's grad pointer each step (fresh tensor) --
            # registration is only allowed between steps, so finalize/init
            R.ratel_finalize()
            R.ratel_init(0, 0, 1, None, R.ratel_default_config())
            R.ratel_register_block(0, [rng], {"device": R.RATEL_DEVICE, "pinned": R.RATEL_PINNED_HOST,
                                              "host_compute": R.RATEL_HOST_COMPUTE}[residency])
            opt_stream = torch.cuda.ExternalStream(R.ratel_optimizer_stream())
            torch.cuda.synchronize()
            R.ratel_adam_step(1e-3, 0.9, 0.999, 1e-8, 1e-2, t)
            torch.cuda._sleep(2_000_000)                 # keep the current stream busy
            R.ratel_offload_grad_chunk(0, torch.cuda.current_stream())
            gt.record_stream(opt_stream)
            del gt
            junk = torch.empty(R.ratel_padded_numel(n, 1), dtype=torch.bfloat16, device=cuda_dev)
            junk.fill_(float("nan"))                     # would poison the update if reused too early
            R.ratel_sync(torch.cuda.current_stream())
            torch.cuda.synchronize()
            del junk
            oracle.adam_range(b.oracle[0], g, oracle.hparams(step=t))
            check_range(b.gpu_state(0), b.oracle[0], own_rne=oracle.bf16_rne, what=f"{residency} t{t}")
        del opt_stream


def test_back_to_back_steps_without_host_sync(cuda_dev):
    """Five steps enqueued back to back with only stream-ordered syncs
    (ratel_sync(stream)) -- grads rewritten on that stream each step -- over
    device, pinned-host and host-compute blocks: cross-step ordering of the
    library's internal streams, tile ring and host staging."""
    blocks = [GpuBlock(0, [200_003], cuda_dev),
              GpuBlock(1, [150_001], cuda_dev, pinned=True),
              GpuBlock(2, [90_000, 13], cuda_dev, host_compute=True)]
    steps = 5
    host_grads = {t: {b.id: [u16_to_torch(g, "cpu").pin_memory() for g in b.grads_np(t)] for b in blocks}
                  for t in range(1, steps + 1)}
    s = torch.cuda.Stream()
    with ratel_lib(tile_elems=16_384, pipeline_depth=2):
        for b in blocks:
            b.register()
        torch.cuda.synchronize()
        with torch.cuda.stream(s):
            for t in range(1, steps + 1):
                R.ratel_adam_step(1e-3, 0.9, 0.999, 1e-8, 1e-2, t)
                for b in reversed(blocks):
                    for i, hg in enumerate(host_grads[t][b.id]):
                        b.g16[i][:hg.numel()].copy_(hg, non_blocking=True)
                    R.ratel_offload_grad_chunk(b.id, s)
                R.ratel_sync(s)
        s.synchronize()
        for t in range(1, steps + 1):
            oracle_step(blocks, t, {b.id: b.grads_np(t) for b in blocks})
        for b in blocks:
            for i in range(len(b.sizes)):
                check_range(b.gpu_state(i), b.oracle[i], own_rne=oracle.bf16_rne, what=f"b{b.id} r{i}")


def test_checkpoint_resume_bitwise(cuda_dev):
    """Checkpoint/resume: states are caller-owned tensors.  Ten continuous
    steps == five steps, copy P32/m/v/P16 out (torch.save-able), finalize,
    re-init, register the restored copies and continue at t = 6..10."""
    a = _fresh(SIZES, cuda_dev)
    run(a, 10, check_every=False)
    b = _fresh(SIZES, cuda_dev)
    run(b, 5, check_every=False)
    ckpt = [[(x.clone(), y.clone(), z.clone(), p.clone()) for x, y, z, p in zip(bl.master, bl.m, bl.v, bl.p16)]
            for bl in b]
    c = _fresh(SIZES, cuda_dev)
    for bl, saved in zip(c, ckpt):
        for i, (x, y, z, p) in enumerate(saved):
            bl.master[i].copy_(x)
            bl.m[i].copy_(y)
            bl.v[i].copy_(z)
            bl.p16[i].copy_(p)
    with ratel_lib():
        for bl in c:
            bl.register()
        for t in range(6, 11):
            for bl in c:
                bl.load_grads(t)
            torch.cuda.synchronize()
            R.ratel_adam_step(1e-3, 0.9, 0.999, 1e-8, 1e-2, t)
            for bl in reversed(c):
                R.ratel_offload_grad_chunk(bl.id, None)
            R.ratel_sync(None)
    assert_bitwise(snapshot(a), snapshot(c))


def test_randomized_protocol_no_side_effects(cuda_dev):
    """Randomised call sequences: arming before/after/between hand-offs,
    random hand-off order, and injected out-of-protocol calls (double
    hand-off, early sync, non-increasing step, unknown block, bad
    hyperparameters) that must fail with RATEL_ESTATE/EINVAL and change
    nothing.  The final states equal a canonical run bit for bit."""
    rng = np.random.default_rng(2024)
    sizes = [[40_001], [8_192, 5], [100_000], [17]]
    canon = _fresh(sizes, cuda_dev)
    run(canon, 6, check_every=False)
    blocks = _fresh(sizes, cuda_dev)
    with ratel_lib():
        for b in blocks:
            b.register()
        for t in range(1, 7):
            for b in blocks:
                b.load_grads(t)
            torch.cuda.synchronize()
            ids = list(rng.permutation([b.id for b in blocks]))
            arm_at = int(rng.integers(0, len(ids) + 1))     # arm after this many hand-offs
            handed = []
            for j in range(len(ids) + 1):
                if j == arm_at:
                    R.ratel_adam_step(1e-3, 0.9, 0.999, 1e-8, 1e-2, t)
                if rng.random() < 0.5:   # inject an invalid call
                    kind = int(rng.integers(0, 5))
                    with pytest.raises(R.RatelError) as e:
                        if kind == 0 and handed:
                            R.ratel_offload_grad_chunk(int(handed[0]), None)
                        elif kind == 1 and j < len(ids):
                            R.ratel_sync(None)          # missing hand-offs
                        elif kind == 1:
                            R.ratel_offload_grad_chunk(-1, None)
                        elif kind == 2:
                            R.ratel_adam_step(1e-3, 0.9, 0.999, 1e-8, 1e-2, t - 1 if t > 1 else 0)
                        elif kind == 3:
                            R.ratel_offload_grad_chunk(999, None)
                        else:
                            R.ratel_adam_step(-1.0, 0.9, 0.999, 1e-8, 1e-2, t + 100)
                    assert e.value.code in (R.RATEL_ESTATE, R.RATEL_EINVAL)
                if j < len(ids):
                    R.ratel_offload_grad_chunk(int(ids[j]), None)
                    handed.append(ids[j])
            R.ratel_sync(None)
    assert_bitwise(snapshot(canon), snapshot(blocks))


def test_fullsize_13b_model_sampled_vs_oracle(cuda_dev):
    """The whole BASELINE configs[1] model (13B GPT states: 40 x 314,639,360 +
    262,568,960 params, 180 GB resident) in bench.py's launch configuration
    (one flat range per block, AGO order, 2-slot gradient ring recycled with
    ratel_block_wait), 3 steps with device-generated inputs; 4096 sampled
    elements per block vs the oracle computed one by one, plus the first and
    last 8 elements of every block (tails)."""
    import bench
    sizes = bench.model_blocks("13B")
    assert sum(sizes) == 12_848_143_360
    steps = 3
    rng = np.random.default_rng(11)
    samples = [np.unique(np.concatenate([np.arange(8), np.arange(n - 8, n),
                                         rng.integers(0, n, 4096)])).astype(np.uint64) for n in sizes]
    refs = [oracle.Range.fresh(synth.theta0_at(idx, block=b)) for b, idx in enumerate(samples)]
    cap = max(sizes)
    ring = [torch.empty(cap, dtype=torch.bfloat16, device=cuda_dev) for _ in range(2)]
    states = []
    with ratel_lib():
        for b, n in enumerate(sizes):
            th = torch.empty(n, dtype=torch.float32, device=cuda_dev)
            R.ratel_gen_theta0(th.data_ptr(), n, 0, R.ratel_gen_stream_key(synth.SEED, synth.TAG_THETA, 0, b))
            m = torch.zeros(n, device=cuda_dev)
            v = torch.zeros(n, device=cuda_dev)
            p = torch.zeros(n, dtype=torch.bfloat16, device=cuda_dev)
            states.append((p, th, m, v))
            R.ratel_register_block(b, [R.make_range(p, ring[b % 2], th, m, v, n)], R.RATEL_DEVICE)
        s = torch.cuda.Stream()
        order = list(reversed(range(len(sizes))))
        for t in range(1, steps + 1):
            R.ratel_adam_step(1e-3, 0.9, 0.999, 1e-8, 1e-2, t)
            for j, b in enumerate(order):
                if j >= 2:
                    R.ratel_block_wait(order[j - 2], s)              # ring slot consumed
                R.ratel_gen_grad16(ring[b % 2].data_ptr(), sizes[b], 0,
                                   R.ratel_gen_stream_key(synth.SEED, synth.TAG_GRAD, t, b), s)
                R.ratel_offload_grad_chunk(b, s)
            R.ratel_sync(None)
            for b, idx in enumerate(samples):
                oracle.adam_range(refs[b], synth.grad16_at(idx, step=t, block=b), oracle.hparams(step=t))
        for b, idx in enumerate(samples):
            p, th, m, v = states[b]
            ii = torch.from_numpy(idx.astype(np.int64)).to(cuda_dev)
            got = dict(p32=th[ii].cpu().numpy(), m32=m[ii].cpu().numpy(), v32=v[ii].cpu().numpy(),
                       p16=torch_to_u16(p[ii]))
            check_range(got, refs[b], own_rne=oracle.bf16_rne, what=f"13B block {b}")
            assert torch.equal(p.view(torch.int16), th.to(torch.bfloat16).view(torch.int16))
        del states


def test_alloc_pinned_states(cuda_dev):
    """ratel_alloc_pinned: exact-size page-locked host memory accepted as
    RATEL_PINNED_HOST / RATEL_HOST_COMPUTE states; results equal the device
    residency bit for bit."""
    n = 300_001
    ref = _fresh([[n]], cuda_dev)
    run(ref, 2, check_every=False)
    for residency in (R.RATEL_PINNED_HOST, R.RATEL_HOST_COMPUTE):
        b = GpuBlock(0, [n], cuda_dev)
        owners = [R.pinned_tensor(n) for _ in range(3)]
        for o, src in zip(owners, (b.master[0], b.m[0], b.v[0])):
            o.tensor.copy_(src.cpu())
        b.master[0], b.m[0], b.v[0] = (o.tensor for o in owners)
        with ratel_lib():
            R.ratel_register_block(0, b.ranges(), residency)
            for t in (1, 2):
                b.load_grads(t)
                torch.cuda.synchronize()
                R.ratel_adam_step(1e-3, 0.9, 0.999, 1e-8, 1e-2, t)
                R.ratel_offload_grad_chunk(0, None)
                R.ratel_sync(None)
        got, want = b.gpu_state(0), ref[0].gpu_state(0)
        if residency == R.RATEL_PINNED_HOST:   # same kernel: bitwise
            assert np.array_equal(got["p32"].view(np.uint32), want["p32"].view(np.uint32))
            assert np.array_equal(got["p16"], want["p16"])
        else:                                   # CPU handler: within the R13 bounds
            check_range(got, ref[0].oracle[0], own_rne=oracle.bf16_rne)
        del owners


@pytest.mark.filterwarnings("ignore:The CUDA Graph is empty")
def test_graph_capture_is_refused_without_side_effects(cuda_dev):
    """A caller stream under CUDA-graph capture is refused (RATEL_EINVAL)
    before anything is enqueued; the step then completes normally and matches
    the oracle."""
    b = GpuBlock(0, [50_003], cuda_dev)
    with ratel_lib():
        b.register()
        gs = b.load_grads(1)
        torch.cuda.synchronize()
        R.ratel_adam_step(HP["lr"], HP["beta1"], HP["beta2"], HP["eps"], HP["weight_decay"], 1)
        s = torch.cuda.Stream(device=cuda_dev)
        g = torch.cuda.CUDAGraph()
        codes = []
        with torch.cuda.graph(g, stream=s):
            for call in (lambda: R.ratel_offload_grad_chunk(0, s.cuda_stream),
                         lambda: R.ratel_block_wait(0, s.cuda_stream),
                         lambda: R.ratel_sync(s.cuda_stream)):
                try:
                    call()
                    codes.append(0)
                except R.RatelError as e:
                    codes.append(e.code)
        assert codes == [R.RATEL_EINVAL] * 3, codes
        R.ratel_offload_grad_chunk(0, None)     # not handed off by the refused call
        R.ratel_sync(None)
    oracle.adam_step(b.oracle, gs, oracle.hparams(step=1, **HP))
    check_range(b.gpu_state(0), b.oracle[0], own_rne=oracle.bf16_rne, what="after refused capture")


def test_long_run_300_steps_with_schedule_sampled_vs_oracle(cuda_dev):
    """A long run: one 13B-shaped block, 300 AGO steps with a warm-up + cosine
    lr schedule and weight decay, a fresh device-generated gradient every
    step.  Rounding errors must not accumulate past R13: sampled elements vs
    the oracle after steps 10, 100 and 300 (the oracle runs the same 300
    steps on the samples); P16 == bf16(P32) everywhere at the end."""
    h = 5120
    n = 12 * h * h + 13 * h
    idx = np.unique(np.concatenate([np.arange(0, 64), np.arange(n - 64, n),
                                    np.random.default_rng(8).integers(0, n, 50_000)])).astype(np.uint64)

    def lr_at(t, peak=3e-4, warm=30, total=300):
        if t <= warm:
            return peak * t / warm
        return 0.5 * peak * (1 + math.cos(math.pi * (t - warm) / (total - warm))) + 1e-6

    ii = torch.from_numpy(idx.astype(np.int64)).to(cuda_dev)
    with ratel_lib():
        g = torch.empty(n, dtype=torch.bfloat16, device=cuda_dev)
        th = torch.empty(n, dtype=torch.float32, device=cuda_dev)
        R.ratel_gen_theta0(th.data_ptr(), n, 0, R.ratel_gen_stream_key(synth.SEED, synth.TAG_THETA, 0, 0))
        m, v = torch.zeros(n, device=cuda_dev), torch.zeros(n, device=cuda_dev)
        p = torch.zeros(n, dtype=torch.bfloat16, device=cuda_dev)
        R.ratel_register_block(0, [R.make_range(p, g, th, m, v, n)], R.RATEL_DEVICE)
        ref = oracle.Range.fresh(synth.theta0_at(idx, block=0))
        for t in range(1, 301):
            lr = lr_at(t)
            R.ratel_adam_step(lr, 0.9, 0.95, 1e-8, 0.1, t)
            R.ratel_block_wait(0, None)   # the grad buffer is rewritten every step
            R.ratel_gen_grad16(g.data_ptr(), n, 0, R.ratel_gen_stream_key(synth.SEED, synth.TAG_GRAD, t, 0))
            R.ratel_offload_grad_chunk(0, None)
            R.ratel_sync(None)
            oracle.adam_range(ref, synth.grad16_at(idx, step=t, block=0),
                              oracle.hparams(lr=lr, beta1=0.9, beta2=0.95, eps=1e-8, weight_decay=0.1, step=t))
            if t in (10, 100, 300):
                got = dict(p32=th[ii].cpu().numpy(), m32=m[ii].cpu().numpy(), v32=v[ii].cpu().numpy(),
                           p16=torch_to_u16(p[ii]))
                rep = check_range(got, ref, own_rne=oracle.bf16_rne, what=f"long run step {t}")
                print(f"long run step {t}: {rep}")
        assert torch.equal(p.view(torch.int16), th.to(torch.bfloat16).view(torch.int16))
