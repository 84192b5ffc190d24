"""Test harness: seeded GPU model states mirrored by oracle states.

Only marshals data (numpy <-> torch, synth inputs); no optimizer arithmetic.
"""
from __future__ import annotations

import contextlib

import numpy as np
import torch

import oracle
import synth
import paper_conf_icde_liaosyxcyww25_b200 as R

HP = dict(lr=1e-3, beta1=0.9, beta2=0.999, eps=1e-8, weight_decay=1e-2)


def u16_to_torch(a: np.ndarray, device) -> torch.Tensor:
    return torch.from_numpy(np.ascontiguousarray(a).view(np.int16)).to(device).view(torch.bfloat16)


def torch_to_u16(t: torch.Tensor) -> np.ndarray:
    return t.detach().view(torch.int16).cpu().numpy().view(np.uint16)


@contextlib.contextmanager
def ratel_lib(device=0, **cfg_kw):
    cfg = R.ratel_default_config()
    for k, v in cfg_kw.items():
        setattr(cfg, k, v)
    R.ratel_init(device, 0, 1, None, cfg)
    try:
        yield cfg
    finally:
        R.ratel_finalize()


class GpuBlock:
    """One block made of ranges of the given sizes (element j of range i is
    block element off_i + j for the generator).  States on the device or in
    pinned host memory; P16 and grads on the device."""

    def __init__(self, block_id: int, sizes, device, pinned: bool = False, wd_flags=None,
                 world: int = 1, rank: int = 0, host_compute: bool = False):
        self.id = block_id
        self.sizes = list(sizes)
        self.offs = np.concatenate([[0], np.cumsum(self.sizes)]).astype(int)
        self.total = int(self.offs[-1])
        self.dev = device
        self.pinned = pinned or host_compute
        self.host_compute = host_compute
        self.wd = list(wd_flags) if wd_flags is not None else [1] * len(self.sizes)
        th0 = synth.theta0(self.total, block=block_id)
        self.p16, self.g16, self.master, self.m, self.v = [], [], [], [], []
        self.oracle = []
        for i, n in enumerate(self.sizes):
            t = th0[self.offs[i]:self.offs[i + 1]]
            cap = R.ratel_padded_numel(n, world)
            b, e = R.ratel_rank_slice(n, world, rank)
            p = torch.zeros(cap, dtype=torch.bfloat16, device=device)
            ref = oracle.Range.fresh(t, self.wd[i])
            self.p16.append(p)
            self.g16.append(torch.zeros(cap, dtype=torch.bfloat16, device=device))
            if self.pinned:
                mk = lambda x: torch.from_numpy(np.ascontiguousarray(x)).pin_memory()
            else:
                mk = lambda x: torch.from_numpy(np.ascontiguousarray(x)).to(device)
            self.master.append(mk(t[b:e].copy() if e > b else np.zeros(8, np.float32)))
            self.m.append(mk(np.zeros(max(e - b, 8), np.float32)))
            self.v.append(mk(np.zeros(max(e - b, 8), np.float32)))
            self.oracle.append(ref)

    def ranges(self):
        return [R.make_range(self.p16[i], self.g16[i], self.master[i], self.m[i], self.v[i],
                             n, self.wd[i]) for i, n in enumerate(self.sizes)]

    def register(self):
        R.ratel_register_block(self.id, self.ranges(),
                               R.RATEL_HOST_COMPUTE if self.host_compute else
                               (R.RATEL_PINNED_HOST if self.pinned else R.RATEL_DEVICE))

    def grads_np(self, step: int):
        g = synth.grad16(self.total, step=step, block=self.id)
        return [g[self.offs[i]:self.offs[i + 1]] for i in range(len(self.sizes))]

    def load_grads(self, step: int, stream=None):
        gs = self.grads_np(step)
        with torch.cuda.stream(stream) if stream is not None else contextlib.nullcontext():
            for i, g in enumerate(gs):
                self.g16[i][:len(g)].copy_(u16_to_torch(g, self.dev), non_blocking=False)
        return gs

    def gpu_state(self, i: int) -> dict:
        n = self.sizes[i]
        return dict(p32=self.master[i][:n].cpu().numpy(), m32=self.m[i][:n].cpu().numpy(),
                    v32=self.v[i][:n].cpu().numpy(), p16=torch_to_u16(self.p16[i][:n]))


class SsdBlock(GpuBlock):
    """A RATEL_SSD block: P16 and grads on the device, theta/m/v in a state
    file (layout of ratel_ssd_range_bytes; the test writes theta0 and zeros
    through a buffered fd, the library gets an O_DIRECT fd)."""

    def __init__(self, block_id: int, sizes, device, path, wd_flags=None, direct: bool = True, base: int = 0,
                 cpu: bool = False):
        super().__init__(block_id, sizes, device, wd_flags=wd_flags)
        self.cpu = cpu   # RATEL_SSD_HOST_COMPUTE: the CPU handler updates the tiles
        import os
        self.path = str(path)
        self.offs_file = []
        off = base
        for n in self.sizes:
            self.offs_file.append(off)
            off += R.ratel_ssd_range_bytes(n, 1, 0)
        self.file_bytes = off
        self.strides = [R.ratel_ssd_range_bytes(n, 1, 0) // 3 for n in self.sizes]
        fdw = os.open(self.path, os.O_RDWR | os.O_CREAT, 0o600)
        os.ftruncate(fdw, max(os.fstat(fdw).st_size, off))
        for i, n in enumerate(self.sizes):
            th = self.master[i][:n].cpu().numpy()
            os.pwrite(fdw, th.tobytes(), self.offs_file[i])
            z = np.zeros(n, np.float32).tobytes()
            os.pwrite(fdw, z, self.offs_file[i] + self.strides[i])
            os.pwrite(fdw, z, self.offs_file[i] + 2 * self.strides[i])
        os.fsync(fdw)
        self.fd_check = fdw
        self.fd = os.open(self.path, os.O_RDWR | (os.O_DIRECT if direct else 0))
        # the device states of the base class are not used
        self.master = self.m = self.v = None

    def ranges(self):
        return [R.make_range(self.p16[i], self.g16[i], None, None, None, n, self.wd[i])
                for i, n in enumerate(self.sizes)]

    def register(self):
        R.ratel_register_block(self.id, self.ranges(), R.RATEL_SSD_HOST_COMPUTE if self.cpu else R.RATEL_SSD)
        for i in range(len(self.sizes)):
            R.ratel_register_ssd(self.id, i, self.fd, self.offs_file[i])

    def gpu_state(self, i: int) -> dict:
        import os
        n = self.sizes[i]
        rd = lambda k: np.frombuffer(os.pread(self.fd_check, 4 * n, self.offs_file[i] + k * self.strides[i]),
                                     dtype=np.float32).copy()
        return dict(p32=rd(0), m32=rd(1), v32=rd(2), p16=torch_to_u16(self.p16[i][:n]))

    def close(self):
        import os
        os.close(self.fd)
        os.close(self.fd_check)
