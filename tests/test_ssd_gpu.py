"""SSD residency (RATEL_SSD): states in a file, streamed by
the library's reader/writer threads through pinned staging and device tiles
around the same update kernel (the paper's Fig. 3b pipeline with the SSD as
the link).  Checked against the oracle (R13) and bitwise
against device residency (R16: the staging does not change a bit)."""
import os

import numpy as np
import pytest
import torch

import oracle
import paper_conf_icde_liaosyxcyww25_b200 as R
from tests.harness import HP, GpuBlock, SsdBlock, ratel_lib
from tests.test_parity_gpu import assert_bitwise, run, snapshot

pytestmark = pytest.mark.gpu

SIZES = [300_001, 65_560, 1_000_003]
TILE = 1 << 16   # several tiles per range, ragged last tiles


def _ssd_blocks(dev, tmp_path, sizes=SIZES, one_file=False):
    if one_file:
        blocks, base = [], 0
        for i, n in enumerate(sizes):
            b = SsdBlock(i, [n], dev, tmp_path / "states.bin", base=base)
            base = b.file_bytes
            blocks.append(b)
        return blocks
    return [SsdBlock(i, [n], dev, tmp_path / f"block{i}.bin") for i, n in enumerate(sizes)]


@pytest.mark.parametrize("arm,depth", [("before", 3), ("after", 2), ("before", 8)])
def test_ssd_vs_oracle_and_bitwise_device(cuda_dev, tmp_path, arm, depth):
    ssd = _ssd_blocks(cuda_dev, tmp_path, one_file=(depth == 8))
    run(ssd, 3, arm=arm, tile_elems=TILE, pipeline_depth=depth)
    dev = [GpuBlock(i, [n], cuda_dev) for i, n in enumerate(SIZES)]
    run(dev, 3, arm=arm)
    assert_bitwise(snapshot(ssd), snapshot(dev))
    for b in ssd:
        b.close()


def test_ssd_clip_and_multirange(cuda_dev, tmp_path):
    sizes = [40_003, 7, 250_000]
    ssd = [SsdBlock(0, sizes, cuda_dev, tmp_path / "a.bin", wd_flags=[1, 0, 1]),
           SsdBlock(1, [123_457], cuda_dev, tmp_path / "b.bin")]
    run(ssd, 3, max_norm=1e-3, tile_elems=TILE)
    dev = [GpuBlock(0, sizes, cuda_dev, wd_flags=[1, 0, 1]), GpuBlock(1, [123_457], cuda_dev)]
    run(dev, 3, max_norm=1e-3)
    assert_bitwise(snapshot(ssd), snapshot(dev))
    for b in ssd:
        b.close()


@pytest.mark.parametrize("max_norm,mode", [(0.0, oracle.ADAMW), (1e-3, oracle.ADAMW), (0.0, oracle.ADAM_L2)])
def test_ssd_host_compute_vs_oracle_and_bitwise_host_compute(cuda_dev, tmp_path, max_norm, mode):
    """RATEL_SSD_HOST_COMPUTE (the paper's full pipeline: states in the file,
    G16 to host, the CPU handler on each staged tile, P16 back): within R13 of
    the oracle at every step, and bitwise equal to HOST_COMPUTE on the same
    inputs (same handler, same arithmetic)."""
    sizes = [40_003, 7, 250_000]
    ssd = [SsdBlock(0, sizes, cuda_dev, tmp_path / "a.bin", wd_flags=[1, 0, 1], cpu=True),
           SsdBlock(1, [123_457], cuda_dev, tmp_path / "b.bin", cpu=True)]
    run(ssd, 3, mode=mode, max_norm=max_norm, tile_elems=TILE, host_threads=4)
    hc = [GpuBlock(0, sizes, cuda_dev, wd_flags=[1, 0, 1], host_compute=True),
          GpuBlock(1, [123_457], cuda_dev, host_compute=True)]
    run(hc, 3, mode=mode, max_norm=max_norm, host_threads=4)
    assert_bitwise(snapshot(ssd), snapshot(hc))
    for b in ssd:
        b.close()


def test_ssd_host_compute_mixed_residencies(cuda_dev, tmp_path):
    """SSD + CPU handler beside GPU-updated SSD, device and pinned-host blocks in one step (random order)."""
    blocks = [GpuBlock(0, [200_000], cuda_dev), SsdBlock(1, [300_000], cuda_dev, tmp_path / "s.bin", cpu=True),
              SsdBlock(2, [100_003], cuda_dev, tmp_path / "t.bin"), GpuBlock(3, [100_000], cuda_dev, pinned=True)]
    run(blocks, 3, order="random", max_norm=5e-3, tile_elems=TILE)
    for b in blocks[1:3]:
        b.close()


def test_ssd_mixed_with_device_and_pinned(cuda_dev, tmp_path):
    blocks = [GpuBlock(0, [200_000], cuda_dev), SsdBlock(1, [300_000], cuda_dev, tmp_path / "s.bin"),
              GpuBlock(2, [100_000], cuda_dev, pinned=True)]
    run(blocks, 3, tile_elems=TILE)
    blocks[1].close()


def test_ssd_block_wait_recycles_grad(cuda_dev, tmp_path):
    """ratel_block_wait on an SSD block: once it returns (stream-ordered), the
    grad buffer may be overwritten without changing the step's result."""
    a = SsdBlock(0, [500_000], cuda_dev, tmp_path / "a.bin")
    ref = SsdBlock(0, [500_000], cuda_dev, tmp_path / "r.bin")
    s = torch.cuda.Stream()
    for blk, clobber in ((a, True), (ref, False)):
        with ratel_lib(tile_elems=TILE):
            blk.register()
            for t in (1, 2):
                blk.load_grads(t)
                torch.cuda.synchronize()
                R.ratel_adam_step(HP["lr"], HP["beta1"], HP["beta2"], HP["eps"], HP["weight_decay"], t)
                R.ratel_offload_grad_chunk(0, s)
                R.ratel_block_wait(0, s)
                if clobber:
                    with torch.cuda.stream(s):
                        blk.g16[0].fill_(float("nan"))
                R.ratel_sync(None)
    sa, sr = a.gpu_state(0), ref.gpu_state(0)
    for k in ("p32", "m32", "v32"):
        assert np.array_equal(sa[k].view(np.uint32), sr[k].view(np.uint32)), k
    a.close()
    ref.close()


def test_ssd_registration_errors(cuda_dev, tmp_path):
    b = SsdBlock(0, [10_000], cuda_dev, tmp_path / "x.bin")
    with ratel_lib(tile_elems=TILE):
        R.ratel_register_block(0, b.ranges(), R.RATEL_SSD)
        for args in [(0, 0, b.fd, 100),                 # offset not 4096-aligned
                     (0, 0, b.fd, 1 << 20),             # file too short for that offset
                     (0, 0, -1, 0),                     # not an fd
                     (0, 1, b.fd, 0)]:                  # range out of range
            with pytest.raises(R.RatelError) as e:
                R.ratel_register_ssd(*args)
            assert e.value.code == R.RATEL_EINVAL, args
        ro = os.open(b.path, os.O_RDONLY)
        with pytest.raises(R.RatelError) as e:          # must be O_RDWR
            R.ratel_register_ssd(0, 0, ro, 0)
        assert e.value.code == R.RATEL_EINVAL
        os.close(ro)
        R.ratel_adam_step(1e-3, 0.9, 0.999, 1e-8, 0.0, 1)
        with pytest.raises(R.RatelError) as e:          # no file attached yet
            R.ratel_offload_grad_chunk(0, None)
        assert e.value.code == R.RATEL_ESTATE
    dev = GpuBlock(1, [10_000], cuda_dev)
    with ratel_lib(tile_elems=TILE):
        R.ratel_register_block(1, dev.ranges(), R.RATEL_DEVICE)
        with pytest.raises(R.RatelError) as e:          # not an SSD block
            R.ratel_register_ssd(1, 0, b.fd, 0)
        assert e.value.code == R.RATEL_EINVAL
    with ratel_lib(tile_elems=1000 * 8):                # tile not a multiple of 1024
        with pytest.raises(R.RatelError) as e:
            R.ratel_register_block(0, b.ranges(), R.RATEL_SSD)
        assert e.value.code == R.RATEL_EINVAL
    with ratel_lib(tile_elems=TILE, comm=R.RATEL_COMM_NCCL):
        with pytest.raises(R.RatelError) as e:          # single rank, no NCCL
            R.ratel_register_block(0, b.ranges(), R.RATEL_SSD)
        assert e.value.code == R.RATEL_EINVAL
    b.close()


def test_ssd_io_error_is_sticky(cuda_dev, tmp_path):
    """A state file that shrinks under the library: the reader's pread hits
    end of file -> RATEL_EIO from ratel_sync, sticky until finalize."""
    b = SsdBlock(0, [300_000], cuda_dev, tmp_path / "t.bin")
    with ratel_lib(tile_elems=TILE):
        b.register()
        b.load_grads(1)
        torch.cuda.synchronize()
        os.ftruncate(b.fd_check, 0)
        R.ratel_adam_step(1e-3, 0.9, 0.999, 1e-8, 0.0, 1)
        R.ratel_offload_grad_chunk(0, None)
        with pytest.raises(R.RatelError) as e:
            R.ratel_sync(None)
        assert e.value.code == R.RATEL_EIO
        with pytest.raises(R.RatelError) as e:
            R.ratel_adam_step(1e-3, 0.9, 0.999, 1e-8, 0.0, 2)
        assert e.value.code == R.RATEL_EIO
    with ratel_lib(tile_elems=TILE):                    # finalize cleared it
        pass
    b.close()


def test_ssd_host_compute_nonfinite_norm_reported(cuda_dev, tmp_path):
    """SSD + CPU handler under clipping with a NaN gradient: RATEL_ENONFINITE
    from the blocking sync, NaN propagated into the file's states."""
    b = SsdBlock(0, [70_000], cuda_dev, tmp_path / "n.bin", cpu=True)
    with ratel_lib(max_grad_norm=1.0, tile_elems=TILE):
        b.register()
        g = b.grads_np(1)[0].copy()
        g[5] = 0x7FC0
        b.g16[0][:70_000].copy_(torch.from_numpy(g.view(np.int16)).to(cuda_dev).view(torch.bfloat16))
        torch.cuda.synchronize()
        R.ratel_adam_step(1e-3, 0.9, 0.999, 1e-8, 1e-2, 1)
        R.ratel_offload_grad_chunk(0, None)
        with pytest.raises(R.RatelError) as e:
            R.ratel_sync(None)
        assert e.value.code == R.RATEL_ENONFINITE
    assert np.isnan(b.gpu_state(0)["p32"]).all()
    b.close()


@pytest.mark.parametrize("cpu", [False, True])
def test_ssd_simplex_schedule_bitwise(cuda_dev, tmp_path, cpu):
    """cfg.ssd_schedule = RATEL_SSD_SIMPLEX (the paper's simplex order, Fig. 3b
    P:L1128-1131: one transfer at a time, write-back of tile k after the read of
    tile k+1) changes only when the file is touched: bitwise the device /
    HOST_COMPUTE result, with clipping and one state file for all blocks."""
    base, ssd = 0, []
    for i, n in enumerate(SIZES):
        b = SsdBlock(i, [n], cuda_dev, tmp_path / "states.bin", base=base, cpu=cpu)
        base = b.file_bytes
        ssd.append(b)
    run(ssd, 3, max_norm=1e-3, tile_elems=TILE, pipeline_depth=2, ssd_schedule=R.RATEL_SSD_SIMPLEX,
        host_threads=4)
    ref = [GpuBlock(i, [n], cuda_dev, host_compute=cpu) for i, n in enumerate(SIZES)]
    run(ref, 3, max_norm=1e-3, host_threads=4)
    assert_bitwise(snapshot(ssd), snapshot(ref))
    for b in ssd:
        b.close()


@pytest.mark.parametrize("cpu,schedule", [(False, 0), (True, 0), (False, 1)])
def test_ssd_io_uring_bitwise(cuda_dev, tmp_path, cpu, schedule):
    """cfg.ssd_io = RATEL_SSD_IO_URING (each I/O thread keeps up to 32 requests
    of <= 4 MiB in flight through its own io_uring) moves the same bytes as
    pread/pwrite: bitwise the device / HOST_COMPUTE result, with clipping, the
    simplex schedule and one state file for all blocks."""
    base, ssd = 0, []
    for i, n in enumerate(SIZES):
        b = SsdBlock(i, [n], cuda_dev, tmp_path / "states.bin", base=base, cpu=cpu)
        base = b.file_bytes
        ssd.append(b)
    run(ssd, 3, max_norm=1e-3, tile_elems=TILE, pipeline_depth=3, ssd_io=R.RATEL_SSD_IO_URING,
        ssd_schedule=schedule, host_threads=4)
    ref = [GpuBlock(i, [n], cuda_dev, host_compute=cpu) for i, n in enumerate(SIZES)]
    run(ref, 3, max_norm=1e-3, host_threads=4)
    assert_bitwise(snapshot(ssd), snapshot(ref))
    for b in ssd:
        b.close()
