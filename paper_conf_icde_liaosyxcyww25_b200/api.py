"""PyTorch-facing wrappers named after the paper's user API.

PAPER.md Fig. 4 and §IV-E: the user wraps setup
in ``with Ratel_init():``, calls ``Ratel_hook(model)``, wraps the optimizer
with ``Ratel_Optimizer(...)`` and drops ``optimizer.step()`` -- each block's
update runs when its gradient is complete.  Here:

    with Ratel_init():                                   # ratel_init / finalize
        opt = Ratel_Optimizer(blocks, lr=1e-3, ...)      # flat buffers + register
        Ratel_hook(opt)                                  # per-block hand-off hooks
        for x in data:
            opt.begin_step()            # arm step t (AGO: before backward)
            loss = model(x); loss.backward()   # blocks handed off as grads complete
            opt.end_step()              # hand off stragglers, ratel_sync(stream)

`blocks` is a list of parameter lists, one per transformer block, in forward
order (backward produces them in reverse).  The wrapper owns one
flat bf16 P16 buffer, one flat bf16 G16 buffer and fp32 master/m/v per range
(a block has a weight-decay range and a no-decay range for biases/norms); the
model's parameters become bf16 views of P16 and their ``.grad`` views of G16,
so autograd accumulates straight into the buffers the library reads.  The
hand-off is a post-accumulate-grad hook with a per-block countdown.  All
arithmetic is in libratel.so; this module only arranges memory and calls.
Gradient accumulation: begin_step(micro_batches=k) hands units off during the
k-th backward.
"""
from __future__ import annotations

import contextlib

import torch

from . import ratel as R


@contextlib.contextmanager
def Ratel_init(device: int | None = None, **cfg_kw):
    """Initialise the library for this process (multi-GPU: torch.distributed
    must be initialised; the NCCL id is broadcast over it)."""
    from . import dist as rdist
    dev = torch.cuda.current_device() if device is None else device
    cfg = R.ratel_default_config()
    for k, v in cfg_kw.items():
        setattr(cfg, k, v)
    rdist.init_distributed(dev, cfg)
    try:
        yield cfg
    finally:
        torch.cuda.synchronize()
        R.ratel_finalize()


class _SsdFile:
    """One state file for every SSD range of an optimizer: ranges are laid out
    back to back (ratel_ssd_range_bytes each).  Written through a buffered fd
    (theta0, zeros), handed to the library as an O_DIRECT fd."""

    def __init__(self, path):
        import os
        self.path = path
        self.size = 0
        self.fd_buf = os.open(path, os.O_RDWR | os.O_CREAT | os.O_TRUNC, 0o600)
        self.fd = None

    def add(self, numel, world, rank):
        off = self.size
        self.size += R.ratel_ssd_range_bytes(numel, world, rank)
        return off

    def open_direct(self):
        import os
        os.ftruncate(self.fd_buf, self.size)
        os.fsync(self.fd_buf)
        self.fd = os.open(self.path, os.O_RDWR | getattr(os, "O_DIRECT", 0))
        return self.fd

    def close(self):
        import os
        for fd in (self.fd, self.fd_buf):
            if fd is not None:
                os.close(fd)
        self.fd = self.fd_buf = None


class _PeerArena:
    """Data-parallel buffers for world > 1: every range's P16 and G16 carved
    out of two flat allocations that every rank maps, so each rank holds the
    peer pointers the fused reduce-scatter (ratel_register_peer_grads) and the
    fused all-gather (ratel_register_peer_params) need.
      peer_memory="symm": torch symmetric memory (one rendezvous per buffer;
        one GPU per rank, NVLink peer mappings);
      peer_memory="ipc": plain CUDA allocations exported as CUDA IPC handles
        and opened by every rank of this node (torch's tensor-sharing
        reduction, handles exchanged with all_gather_object) -- also works
        when ranks share a GPU, which symmetric memory refuses."""

    def __init__(self, caps, dev, peer_memory="symm"):
        import torch.distributed as dist
        self.offs, off = [], 0
        for c in caps:
            self.offs.append(off)
            off += (c + 7) // 8 * 8          # 16-byte aligned views
        n = max(off, 8)
        if peer_memory == "symm":
            import torch.distributed._symmetric_memory as symm_mem
            self.p16 = symm_mem.empty(n, dtype=torch.bfloat16, device=dev)
            self.g16 = symm_mem.empty(n, dtype=torch.bfloat16, device=dev)
            self.p16.zero_()
            self.g16.zero_()
            group = dist.group.WORLD.group_name
            self.handles = (symm_mem.rendezvous(self.p16, group), symm_mem.rendezvous(self.g16, group))
            self.bases_p = list(self.handles[0].buffer_ptrs)   # the handles stay referenced with the arena
            self.bases_g = list(self.handles[1].buffer_ptrs)
        elif peer_memory == "ipc":
            from torch.multiprocessing.reductions import reduce_tensor
            self.p16 = torch.zeros(n, dtype=torch.bfloat16, device=dev)
            self.g16 = torch.zeros(n, dtype=torch.bfloat16, device=dev)
            torch.cuda.synchronize()
            mine = (reduce_tensor(self.p16), reduce_tensor(self.g16))
            allh = [None] * dist.get_world_size()
            dist.all_gather_object(allh, mine)
            me = dist.get_rank()
            self.mapped = []                 # peers' tensors, kept open until this arena dies
            self.bases_p, self.bases_g = [], []
            for q, (hp, hg) in enumerate(allh):
                if q == me:
                    tp, tg = self.p16, self.g16
                else:
                    tp, tg = hp[0](*hp[1]), hg[0](*hg[1])
                    self.mapped += [tp, tg]
                self.bases_p.append(tp.data_ptr())
                self.bases_g.append(tg.data_ptr())
        else:
            raise ValueError(f"peer_memory must be 'symm' or 'ipc', not {peer_memory!r}")
        self.next = 0

    def take(self, cap):
        k = self.next
        self.next += 1
        o = self.offs[k]
        return (self.p16[o:o + cap], self.g16[o:o + cap],
                [b + 2 * o for b in self.bases_p], [b + 2 * o for b in self.bases_g])


class _Range:
    def __init__(self, params, apply_wd, world, rank, dev, residency, ssd=None, arena=None):
        self.params = params
        self.numel = sum(p.numel() for p in params)
        cap = R.ratel_padded_numel(self.numel, world)
        beg, end = R.ratel_rank_slice(self.numel, world, rank)
        self.peer_p16 = self.peer_g16 = None
        if arena is not None:   # world > 1, data parallel: memory every rank maps
            self.p16, self.g16, self.peer_p16, self.peer_g16 = arena.take(cap)
        else:
            self.p16 = torch.zeros(cap, dtype=torch.bfloat16, device=dev)
            self.g16 = torch.zeros(cap, dtype=torch.bfloat16, device=dev)
        flat32 = torch.cat([p.detach().reshape(-1).to(torch.float32) for p in params]).to(dev)
        s = max(end - beg, 8)
        self.ssd, self.ssd_off = ssd, None
        if residency in ("ssd", "ssd_hostcompute"):
            # theta0 and zero moments go to the file; no state tensors are kept
            import os
            self.ssd_off = ssd.add(self.numel, world, rank)
            self.ssd_stride = R.ratel_ssd_range_bytes(self.numel, world, rank) // 3
            if end > beg:
                os.pwrite(ssd.fd_buf, flat32[beg:end].cpu().numpy().tobytes(), self.ssd_off)
            self.master = self.m = self.v = None
        else:
            if residency == "device":
                mk = lambda: torch.zeros(s, dtype=torch.float32, device=dev)
            else:
                mk = lambda: torch.zeros(s, dtype=torch.float32).pin_memory()
            self.master, self.m, self.v = mk(), mk(), mk()
            if end > beg:
                self.master[:end - beg].copy_(flat32[beg:end])
        off = 0                     # P16 is built from the masters by the library (ratel_refresh_params)
        for p in params:  # parameters become views of the flat buffers
            k = p.numel()
            p.data = self.p16[off:off + k].view(p.shape)
            p.grad = self.g16[off:off + k].view(p.shape)
            off += k
        self.apply_wd = apply_wd
        self.slice = (beg, end)

    def ratel_range(self):
        return R.make_range(self.p16, self.g16, self.master, self.m, self.v, self.numel, int(self.apply_wd))

    def split_ranges(self, frac):
        """(head, tail) library ranges for the hybrid residency (single rank):
        elements [0, k) and [k, numel), k = frac * numel rounded to a multiple
        of 8 (16-byte alignment); None for an empty part."""
        k = min(self.numel, max(0, int(round(frac * self.numel / 8)) * 8))
        wd = int(self.apply_wd)
        ptr = lambda t, off, size: t.data_ptr() + off * size
        head = R.make_range(self.p16, self.g16, self.master, self.m, self.v, k, wd) if k > 0 else None
        tail = (R.make_range(ptr(self.p16, k, 2), ptr(self.g16, k, 2), ptr(self.master, k, 4), ptr(self.m, k, 4),
                             ptr(self.v, k, 4), self.numel - k, wd) if k < self.numel else None)
        return head, tail

    def states(self):
        """(master, exp_avg, exp_avg_sq) of this rank's slice as CPU/device
        tensors (SSD: read back from the state file)."""
        if self.ssd is None:
            return self.master, self.m, self.v
        import os
        import numpy as np
        n = self.slice[1] - self.slice[0]
        rd = lambda k: torch.from_numpy(np.frombuffer(os.pread(self.ssd.fd_buf, 4 * n, self.ssd_off + k * self.ssd_stride),
                                                      dtype=np.float32).copy())
        return rd(0), rd(1), rd(2)

    def load_states(self, master, m, v):
        if self.ssd is None:
            self.master.copy_(master)
            self.m.copy_(m)
            self.v.copy_(v)
            return
        import os
        n = self.slice[1] - self.slice[0]
        for k, t in enumerate((master, m, v)):
            os.pwrite(self.ssd.fd_buf, t[:n].to(torch.float32).contiguous().numpy().tobytes(),
                      self.ssd_off + k * self.ssd_stride)
        os.fsync(self.ssd.fd_buf)


class Ratel_Optimizer:
    """AdamW (or Adam-L2) over flat per-block buffers, driven by hand-offs.

    residency: "device" (states in HBM), "host" (pinned host, GPU-streamed),
    "hostcompute" (pinned host, the paper's CPU handler), "hybrid" (pinned host;
    the first `hybrid_gpu_frac` of every range GPU-streamed, the rest updated
    by the CPU handler -- two library blocks per unit, handed off together, so
    the host link and the host's cores work on one block at the same time;
    single rank; unit j uses library block ids first_block_id + j and
    first_block_id + len(units) + j), "ssd_hostcompute" (the paper's full pipeline: the same state
    file, each staged tile updated by the CPU handler, no state crossing the
    host link) or "ssd" (a state file at `ssd_path`, streamed by the
    library's reader/writer threads; the paper's storage tier, single rank).

    granularity: "block" hands a transformer block off when its last gradient
    has accumulated; "tensor" registers every weight matrix of a block as its
    own unit (and the block's no-decay parameters as one more), each handed
    off as soon as its own gradient is complete -- the paper's per-tensor
    handler.  Finer units shorten the update tail after the
    last gradient (a block's update done 12-13 ms after its last gradient instead
    of ~70 ms, profiles/r01_overlap_granularity.jsonl); the result is bitwise the same.
    `blocks`/`block_ids`/`state(i)` then index units.

    Data parallelism (torch.distributed initialised, world > 1; one process
    per GPU): every rank runs its own micro-batch and each hook hands off the
    rank's LOCAL gradient.  data_parallel="fused" (default) allocates P16 and
    G16 in torch symmetric memory and registers every rank's buffers with the
    library, so each rank's update kernel reduces the N local gradients of its
    slice (mean, fp64, R17) and stores its P16 slice into every
    rank's copy (fused reduce-scatter + all-gather over NVLink; residency
    "device" or "host"; peer_memory="ipc" maps plain allocations through CUDA
    IPC instead, e.g. when ranks share a GPU).  data_parallel="reduced" is for callers whose
    gradients are already identical on every rank when the hook fires (the
    library then only all-gathers P16 over NCCL, R11).  Both sides of a step
    are collective: every rank hands off the same units in the same order."""

    def __init__(self, blocks, lr=1e-3, betas=(0.9, 0.999), eps=1e-8, weight_decay=1e-2,
                 residency="device", no_decay=None, first_block_id=0, granularity="block", ssd_path=None,
                 hybrid_gpu_frac=0.3, data_parallel="fused", peer_memory="symm"):
        import torch.distributed as dist
        distributed = dist.is_available() and dist.is_initialized()
        world = dist.get_world_size() if distributed else 1
        rank = dist.get_rank() if distributed else 0
        dev = torch.device("cuda", torch.cuda.current_device())
        no_decay = no_decay or (lambda p: p.ndim <= 1)
        self.lr, self.betas, self.eps, self.weight_decay = lr, betas, eps, weight_decay
        self.t = 0
        self.blocks = []
        self.block_ids = []
        if granularity not in ("block", "tensor"):
            raise ValueError(f"granularity must be 'block' or 'tensor', not {granularity!r}")
        units = []            # each unit: [(params, apply_wd)] -> one registered block
        for params in blocks:
            params = [p for p in params if p.requires_grad]
            decay = [p for p in params if not no_decay(p)]
            nodecay = [p for p in params if no_decay(p)]
            if granularity == "block":
                groups = [(ps, wd) for ps, wd in ((decay, True), (nodecay, False)) if ps]
                if groups:
                    units.append(groups)
            else:
                units += [[([p], True)] for p in decay]
                if nodecay:
                    units.append([(nodecay, False)])
        if residency == "hybrid" and world > 1:
            raise ValueError('residency="hybrid" is single-rank')
        if data_parallel not in ("fused", "reduced"):
            raise ValueError(f"data_parallel must be 'fused' or 'reduced', not {data_parallel!r}")
        fused_dp = world > 1 and data_parallel == "fused"
        if fused_dp and residency not in ("device", "host"):
            raise ValueError(f'data_parallel="fused" needs residency "device" or "host", not {residency!r} '
                             f'(the fused reduction reads peer gradients inside the update kernel)')
        arena = None
        if fused_dp:
            caps = [R.ratel_padded_numel(sum(p.numel() for p in ps), world) for groups in units for ps, _ in groups]
            arena = _PeerArena(caps, dev, peer_memory)
        self._arena = arena                  # keeps the peer mappings open for the optimizer's lifetime
        ssd = residency in ("ssd", "ssd_hostcompute")
        if ssd and not ssd_path:
            raise ValueError(f'residency="{residency}" needs ssd_path (the state file to create)')
        self.ssd = _SsdFile(ssd_path) if ssd else None
        for j, groups in enumerate(units):
            ranges = [_Range(ps, wd, world, rank, dev, "host" if residency == "hybrid" else residency, self.ssd,
                             arena) for ps, wd in groups]
            self.blocks.append(ranges)
            self.block_ids.append(first_block_id + j)
        if self.ssd is not None:
            self.ssd.open_direct()
        self._lib_ids = {}   # unit id -> the library blocks handed off for it
        for bid, ranges in zip(self.block_ids, self.blocks):
            if residency == "hybrid":
                tail_id = bid + len(units)
                head, tail = zip(*[r.split_ranges(hybrid_gpu_frac) for r in ranges])
                head, tail = [x for x in head if x is not None], [x for x in tail if x is not None]
                self._lib_ids[bid] = []
                if head:
                    R.ratel_register_block(bid, head, R.RATEL_PINNED_HOST)
                    self._lib_ids[bid].append(bid)
                if tail:
                    R.ratel_register_block(tail_id, tail, R.RATEL_HOST_COMPUTE)
                    self._lib_ids[bid].append(tail_id)
                continue
            self._lib_ids[bid] = [bid]
            R.ratel_register_block(bid, [r.ratel_range() for r in ranges],
                                   {"device": R.RATEL_DEVICE, "host": R.RATEL_PINNED_HOST,
                                    "hostcompute": R.RATEL_HOST_COMPUTE, "ssd": R.RATEL_SSD,
                                    "ssd_hostcompute": R.RATEL_SSD_HOST_COMPUTE}[residency])
            if self.ssd is not None:
                for i, r in enumerate(ranges):
                    R.ratel_register_ssd(bid, i, self.ssd.fd, r.ssd_off)
            if fused_dp:
                for i, r in enumerate(ranges):
                    R.ratel_register_peer_grads(bid, i, r.peer_g16, 1.0 / world)
                    R.ratel_register_peer_params(bid, i, r.peer_p16)
        # the working copy P16 = bf16_rne(master), built by the library (the
        # update's own conversion) and all-gathered across ranks -- collective
        s = torch.cuda.current_stream()
        for bid in self.block_ids:
            for lid in self._lib_ids[bid]:
                R.ratel_refresh_params(lid, s)
        torch.cuda.synchronize()
        self._pending = {}
        self._handed = set()
        self._hooks = []
        self._micro = 1

    # ------------------------------------------------------------ Ratel_hook
    def install_hooks(self):
        for bid, ranges in zip(self.block_ids, self.blocks):
            params = [p for r in ranges for p in r.params]
            for p in params:
                self._hooks.append(p.register_post_accumulate_grad_hook(self._make_hook(bid, len(params))))

    def _make_hook(self, bid, count):
        def hook(_p):
            left = self._pending.get(bid, count * self._micro) - 1
            self._pending[bid] = left
            if left == 0 and bid not in self._handed:
                self._handed.add(bid)
                # the active message: gradient complete on the stream backward used
                for lid in self._lib_ids[bid]:
                    R.ratel_offload_grad_chunk(lid, torch.cuda.current_stream())
        return hook

    # ------------------------------------------------------------- a step
    def begin_step(self, lr=None, weight_decay=None, micro_batches=1):
        """Zero the grad buffers and arm step t (before backward = AGO).
        micro_batches > 1: gradient accumulation -- the step's gradients are
        the sum over that many backward passes, and each unit is handed off
        when its last parameter's gradient of the LAST micro-batch has
        accumulated (only that backward overlaps the update)."""
        if micro_batches < 1:
            raise ValueError("micro_batches must be >= 1")
        self._micro = int(micro_batches)
        for ranges in self.blocks:
            for r in ranges:
                r.g16.zero_()
                for p in r.params:  # autograd must keep accumulating into our views
                    assert p.grad is not None and p.grad.data_ptr() >= r.g16.data_ptr()
        self.t += 1
        if lr is not None:
            self.lr = lr
        if weight_decay is not None:
            self.weight_decay = weight_decay
        self._pending.clear()
        self._handed.clear()
        R.ratel_adam_step(self.lr, self.betas[0], self.betas[1], self.eps, self.weight_decay, self.t)

    def end_step(self):
        """Hand off blocks whose hooks did not fire (unused params) and order
        the current stream after every update (no staleness)."""
        s = torch.cuda.current_stream()
        for bid in self.block_ids:
            if bid not in self._handed:
                self._handed.add(bid)
                for lid in self._lib_ids[bid]:
                    R.ratel_offload_grad_chunk(lid, s)
        R.ratel_sync(s)

    def state_dict(self) -> dict:
        """Step counter and copies of every range's fp32 master/exp_avg/
        exp_avg_sq (this rank's slices).  Call between steps."""
        torch.cuda.synchronize()
        out = []
        for ranges in self.blocks:
            out.append([])
            for r in ranges:
                master, m, v = r.states()
                out[-1].append({"master": master.detach().cpu().clone(), "exp_avg": m.detach().cpu().clone(),
                                "exp_avg_sq": v.detach().cpu().clone()})
        return {"t": self.t, "lr": self.lr, "betas": self.betas, "eps": self.eps,
                "weight_decay": self.weight_decay, "ranges": out}

    def load_state_dict(self, sd: dict) -> None:
        """Restore states saved by state_dict() (same block/range layout; this
        rank's slices) and rebuild the model's P16 from the restored masters in
        the library (ratel_refresh_params: bf16 RNE of the rank slice, then the
        all-gather across ranks); the step counter continues from sd["t"].
        Call between steps, on every rank."""
        assert len(sd["ranges"]) == len(self.blocks)
        for ranges, saved in zip(self.blocks, sd["ranges"]):
            assert len(ranges) == len(saved)
            for r, s in zip(ranges, saved):
                r.load_states(s["master"], s["exp_avg"], s["exp_avg_sq"])
        torch.cuda.synchronize()   # pinned-host / file states written before the library reads them
        s = torch.cuda.current_stream()
        for bid in self.block_ids:
            for lid in self._lib_ids[bid]:
                R.ratel_refresh_params(lid, s)
        self.t = int(sd["t"])
        self.lr, self.betas, self.eps, self.weight_decay = sd["lr"], tuple(sd["betas"]), sd["eps"], sd["weight_decay"]
        torch.cuda.synchronize()

    def state(self, block_index: int):
        """(master, exp_avg, exp_avg_sq, p16, g16) flat views of each range of a
        block (SSD: the states are copies read back from the file)."""
        return [(*r.states(), r.p16, r.g16) for r in self.blocks[block_index]]

    def remove_hooks(self):
        for h in self._hooks:
            h.remove()
        self._hooks.clear()

    def close(self):
        """Release the SSD state file (after ratel_finalize / Ratel_init exit)."""
        if self.ssd is not None:
            self.ssd.close()


def Ratel_hook(optimizer: Ratel_Optimizer) -> Ratel_Optimizer:
    """Install the per-block hand-off hooks (Fig. 4's `Ratel_hook(model)`)."""
    optimizer.install_hooks()
    return optimizer
