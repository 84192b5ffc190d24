"""Roofline probes on the GPU box (SURVEY §8(d) "Roofline probe protocol"):
box facts, pinned host-link bandwidth (H2D, D2H, duplex) and a same-pattern
HBM stream ceiling.  Writes gpurun_out/box.json."""
import json
import os
import subprocess
import time

import torch


def sh(cmd):
    try:
        return subprocess.run(cmd, shell=True, capture_output=True, text=True, timeout=60).stdout
    except Exception as e:
        return repr(e)


def bw_copy(dst, src, reps=10, stream=None):
    s = stream or torch.cuda.current_stream()
    ts = []
    for _ in range(reps):
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record(s)
        with torch.cuda.stream(s):
            dst.copy_(src, non_blocking=True)
        e1.record(s)
        e1.synchronize()
        ts.append(e0.elapsed_time(e1))
    ts.sort()
    return src.numel() * src.element_size() / (ts[len(ts) // 2] / 1e3) / 1e9


def main():
    out = {}
    out["nproc"] = os.cpu_count()
    out["affinity"] = len(os.sched_getaffinity(0))
    out["lscpu"] = sh("lscpu | egrep 'Model name|Socket|NUMA node|Thread|Core'")
    out["meminfo"] = sh("egrep 'MemTotal|MemAvailable|Hugepagesize|HugePages_Total' /proc/meminfo")
    out["topo"] = sh("nvidia-smi topo -m")
    out["smi"] = sh("nvidia-smi --query-gpu=name,memory.total,clocks.max.sm,pcie.link.gen.max,pcie.link.width.max --format=csv")
    free, total = torch.cuda.mem_get_info()
    p = torch.cuda.get_device_properties(0)
    out["device"] = dict(name=p.name, sms=p.multi_processor_count, total=total, free=free,
                         l2=getattr(p, "L2_cache_size", None))
    n = 1 << 28  # 1 GiB of fp32
    t0 = time.time()
    h = torch.empty(n, dtype=torch.float32, pin_memory=True)
    h2 = torch.empty(n, dtype=torch.float32, pin_memory=True)
    out["pin_2GiB_s"] = time.time() - t0
    d = torch.empty(n, dtype=torch.float32, device="cuda")
    d2 = torch.empty(n, dtype=torch.float32, device="cuda")
    h.fill_(1.0)
    out["h2d_gbs"] = bw_copy(d, h)
    out["d2h_gbs"] = bw_copy(h, d)
    s1, s2 = torch.cuda.Stream(), torch.cuda.Stream()
    torch.cuda.synchronize()
    e0 = torch.cuda.Event(enable_timing=True)
    e1 = torch.cuda.Event(enable_timing=True)
    reps = 5
    e0.record()
    s1.wait_stream(torch.cuda.current_stream())
    s2.wait_stream(torch.cuda.current_stream())
    for _ in range(reps):
        with torch.cuda.stream(s1):
            d.copy_(h, non_blocking=True)
        with torch.cuda.stream(s2):
            h2.copy_(d2, non_blocking=True)
    torch.cuda.current_stream().wait_stream(s1)
    torch.cuda.current_stream().wait_stream(s2)
    e1.record()
    e1.synchronize()
    out["duplex_gbs_each_way"] = n * 4 * reps / (e0.elapsed_time(e1) / 1e3) / 1e9
    # HBM copy reference (same as MEASURED_PEAKS's method)
    a = torch.empty(1 << 30, dtype=torch.bfloat16, device="cuda")
    b = torch.empty_like(a)
    best = 1e9
    for _ in range(10):
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record()
        b.copy_(a)
        e1.record()
        e1.synchronize()
        best = min(best, e0.elapsed_time(e1))
    out["hbm_copy_gbs"] = 2 * a.numel() * 2 / (best / 1e3) / 1e9
    os.makedirs("gpurun_out", exist_ok=True)
    with open("gpurun_out/box.json", "w") as f:
        json.dump(out, f, indent=1)
    print(json.dumps({k: v for k, v in out.items() if k not in ("topo", "lscpu", "meminfo")}))
    print(out["lscpu"], out["meminfo"], out["topo"])


if __name__ == "__main__":
    main()
