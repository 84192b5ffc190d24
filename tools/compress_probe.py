"""Does L2 compression touch K1's traffic?  (tools, not product)

ncu's full capture of K1 lists every byte the kernel reads as "sent to the L2
compression unit" with 0 % compressed.  This probe times K1 (the in-tree
library, 8 x 13B-shaped blocks, two update streams) on states allocated three
ways: torch (cudaMalloc via the caching allocator), cuMemCreate without
compression, and cuMemCreate with CU_MEM_ALLOCATION_COMP_GENERIC -- same
bytes, same launches.  One JSON line per (allocation, round).

  python tools/compress_probe.py [rounds]
"""
import ctypes
import json
import sys
import os

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import torch  # noqa: E402
from cuda.bindings import driver as d  # noqa: E402

import paper_conf_icde_liaosyxcyww25_b200 as R  # noqa: E402

N = 12 * 5120 * 5120 + 13 * 5120
NB = 8


def ck(res):
    err = res[0] if isinstance(res, tuple) else res
    if err != d.CUresult.CUDA_SUCCESS:
        raise RuntimeError(str(err))
    return res[1] if isinstance(res, tuple) and len(res) > 1 else None


class VmmPool:
    """One cuMemCreate allocation per array (compression on or off)."""

    def __init__(self, comp):
        self.comp = comp
        self.allocs = []

    def alloc(self, nbytes):
        prop = d.CUmemAllocationProp()
        prop.type = d.CUmemAllocationType.CU_MEM_ALLOCATION_TYPE_PINNED
        prop.location.type = d.CUmemLocationType.CU_MEM_LOCATION_TYPE_DEVICE
        prop.location.id = 0
        if self.comp:
            prop.allocFlags.compressionType = d.CUmemAllocationCompType.CU_MEM_ALLOCATION_COMP_GENERIC
        gran = ck(d.cuMemGetAllocationGranularity(prop, d.CUmemAllocationGranularity_flags.CU_MEM_ALLOC_GRANULARITY_RECOMMENDED))
        size = (nbytes + gran - 1) // gran * gran
        h = ck(d.cuMemCreate(size, prop, 0))
        ptr = ck(d.cuMemAddressReserve(size, gran, 0, 0))
        ck(d.cuMemMap(ptr, size, 0, h, 0))
        acc = d.CUmemAccessDesc()
        acc.location.type = d.CUmemLocationType.CU_MEM_LOCATION_TYPE_DEVICE
        acc.location.id = 0
        acc.flags = d.CUmemAccess_flags.CU_MEM_ACCESS_FLAGS_PROT_READWRITE
        ck(d.cuMemSetAccess(ptr, size, [acc], 1))
        granted = None
        if self.comp:
            p2 = ck(d.cuMemGetAllocationPropertiesFromHandle(h))
            granted = int(p2.allocFlags.compressionType)
        self.allocs.append((ptr, size, h))
        return int(ptr), granted

    def free(self):
        for ptr, size, h in self.allocs:
            ck(d.cuMemUnmap(ptr, size))
            ck(d.cuMemAddressFree(ptr, size))
            ck(d.cuMemRelease(h))
        self.allocs = []


def time_k1(ptrs, g_ptr, steps=10, warmup=3):
    cfg = R.ratel_default_config()
    cfg.timing = 1
    R.ratel_init(0, 0, 1, None, cfg)
    try:
        for b, (p, th, m, v) in enumerate(ptrs):
            R.ratel_register_block(b, [R.make_range(p, g_ptr, th, m, v, N)], R.RATEL_DEVICE)
        s = torch.cuda.Stream()
        t = 1
        for k in range(warmup + steps):
            if k == warmup:
                torch.cuda.synchronize()
                R.ratel_kernel_timing(reset=True)
            R.ratel_adam_step(1e-3, 0.9, 0.999, 1e-8, 1e-2, t)
            for b in reversed(range(NB)):
                R.ratel_offload_grad_chunk(b, s)
            R.ratel_sync(s)
            t += 1
        torch.cuda.synchronize()
        ms, n = R.ratel_kernel_timing(reset=True)
    finally:
        R.ratel_finalize()
    return 28 * N * NB * steps / (ms / 1e3) / 1e9


def states(alloc):
    out, granted = [], set()
    for b in range(NB):
        arrs = []
        for nbytes in (2 * N, 4 * N, 4 * N, 4 * N):
            ptr, gr = alloc(nbytes)
            granted.add(gr)
            arrs.append(ptr)
        p, th, m, v = arrs
        R.ratel_gen_theta0(th, N, 0, R.ratel_gen_stream_key(0x5EED5EED, 1, 0, b))
        torch.cuda.synchronize()
        for x, nb in ((m, 4 * N), (v, 4 * N)):
            ck(d.cuMemsetD8(x, 0, nb))
        out.append((p, th, m, v))
    return out, granted


def main():
    rounds = int(sys.argv[1]) if len(sys.argv) > 1 else 3
    torch.cuda.init()
    dev = torch.device("cuda:0")
    g = torch.empty(N, dtype=torch.bfloat16, device=dev)
    R.ratel_gen_grad16(g.data_ptr(), N, 0, R.ratel_gen_stream_key(0x5EED5EED, 2, 1, 0))
    torch.cuda.synchronize()
    for rnd in range(rounds):
        for kind in ("torch", "vmm", "vmm_comp"):
            keep, pool, granted = [], None, {None}
            if kind == "torch":
                for b in range(NB):
                    th = torch.empty(N, device=dev)
                    R.ratel_gen_theta0(th.data_ptr(), N, 0, R.ratel_gen_stream_key(0x5EED5EED, 1, 0, b))
                    keep.append((torch.zeros(N, dtype=torch.bfloat16, device=dev), th, torch.zeros(N, device=dev),
                                 torch.zeros(N, device=dev)))
                ptrs = [tuple(x.data_ptr() for x in t4) for t4 in keep]
            else:
                pool = VmmPool(kind == "vmm_comp")
                ptrs, granted = states(pool.alloc)
            gbs = time_k1(ptrs, g.data_ptr())
            print(json.dumps({"round": rnd, "alloc": kind, "k1_gbs": round(gbs, 1),
                              "compression_granted": sorted(x for x in granted if x is not None) or None}),
                  flush=True)
            del keep
            if pool:
                pool.free()
            torch.cuda.empty_cache()


if __name__ == "__main__":
    main()
