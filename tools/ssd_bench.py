"""SSD residency (RATEL_SSD) throughput on the GPU box, with
the box's own storage probe in the same run.

    python tools/ssd_bench.py [--dir D] [--shape 13B] [--blocks 2] [--steps 3] [--warmup 3]
                              [--depths 2,4,8] [--tile-elems N]

A step = ratel_adam_step + one hand-off per block (decreasing index) +
ratel_sync(NULL) over blocks whose theta/m/v live in one state file opened
with O_DIRECT (the page cache is bypassed: every byte crosses the device).
The library's reader thread streams each tile file -> pinned staging ->
device, the update kernel runs, the writer thread writes it back: 12 B/param
read + 12 B/param written per step (the paper's Eq. 5 "14P/BW_S2M +
14P/BW_M2S" minus the G16/P16 that stay on the GPU here).

Probe: single-thread O_DIRECT sequential write then read of a probe file
(64 MiB requests, the library's pattern), then read and write concurrently
(two threads, two files) -- the SSD link is shared by the reads and the
write-backs, so the roofline of a step is 24 B/param over the larger of the
concurrent read+write bandwidth and the simplex time-sharing model
2/(1/read + 1/write) (reported as `roofline_gbs`).
Prints one JSON line per pipeline depth; writes nothing but the state/probe
files (deleted at the end).
"""
from __future__ import annotations

import argparse
import json
import mmap
import os
import sys
import threading
import time

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
if ROOT not in sys.path:
    sys.path.insert(0, ROOT)

CHUNK = 64 << 20


def _aligned(nbytes):
    return mmap.mmap(-1, nbytes)   # page-aligned anonymous buffer (O_DIRECT needs 4 KiB alignment)


def probe_file(path, nbytes, write: bool):
    fd = os.open(path, os.O_RDWR | os.O_CREAT | os.O_DIRECT, 0o600)
    buf = _aligned(CHUNK)
    buf.write(os.urandom(4096) * (CHUNK // 4096))
    mv = memoryview(buf)
    t0 = time.perf_counter()
    off = 0
    while off < nbytes:
        if write:
            os.pwritev(fd, [mv], off)
        else:
            os.preadv(fd, [mv], off)
        off += CHUNK
    dt = time.perf_counter() - t0     # O_DIRECT: no page cache; no fsync, like the library's writer
    os.close(fd)
    return nbytes / dt / 1e9


def storage_probe(d, nbytes=8 << 30):
    a, b = os.path.join(d, "ratel_probe_a.bin"), os.path.join(d, "ratel_probe_b.bin")
    out = {"dir": d, "probe_bytes": nbytes}
    try:
        out["write_gbs"] = probe_file(a, nbytes, True)
        out["read_gbs"] = probe_file(a, nbytes, False)
        probe_file(b, nbytes, True)
        res = {}
        th = [threading.Thread(target=lambda: res.__setitem__("r", probe_file(a, nbytes, False))),
              threading.Thread(target=lambda: res.__setitem__("w", probe_file(b, nbytes, True)))]
        t0 = time.perf_counter()
        for t in th:
            t.start()
        for t in th:
            t.join()
        dt = time.perf_counter() - t0
        out["concurrent_read_gbs"], out["concurrent_write_gbs"] = res["r"], res["w"]
        out["concurrent_total_gbs"] = 2 * nbytes / dt / 1e9
        # a simplex link time-shared between the reads and the write-backs (the paper's SSD model,
        # P:L1200-1203): equal bytes each way -> 2 / (1/read + 1/write)
        out["simplex_model_gbs"] = 2.0 / (1.0 / out["read_gbs"] + 1.0 / out["write_gbs"])
        out["roofline_gbs"] = max(out["concurrent_total_gbs"], out["simplex_model_gbs"])
    finally:
        for p in (a, b):
            try:
                os.unlink(p)
            except OSError:
                pass
    return out


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--dir", default=os.environ.get("GRAFT_REPO_ROOT", ROOT))
    ap.add_argument("--shape", default="13B")
    ap.add_argument("--blocks", type=int, default=2)
    ap.add_argument("--steps", type=int, default=3)
    ap.add_argument("--warmup", type=int, default=3)
    ap.add_argument("--depths", default="2,4,8")
    ap.add_argument("--tile-elems", type=int, default=0)
    ap.add_argument("--probe-gb", type=float, default=8.0)
    ap.add_argument("--handlers", default="gpu,cpu",
                    help="gpu: RATEL_SSD (tile kernel); cpu: RATEL_SSD_HOST_COMPUTE (the paper's CPU handler)")
    ap.add_argument("--schedules", default="duplex,simplex",
                    help="cfg.ssd_schedule: duplex (reader and writer free) and/or simplex (the paper's Fig. 3b "
                         "order: one transfer at a time, write-back of tile k after the read of tile k+1)")
    ap.add_argument("--io", default="pread",
                    help="cfg.ssd_io: pread (one blocking request at a time) and/or uring (io_uring, up to 32 "
                         "requests of 4 MiB in flight per I/O thread)")
    args = ap.parse_args()

    import torch
    import paper_conf_icde_liaosyxcyww25_b200 as R
    from bench import model_blocks, HP

    probe = storage_probe(args.dir, int(args.probe_gb * (1 << 30)) // CHUNK * CHUNK)
    print(json.dumps({"probe": probe}), flush=True)
    dev = torch.device("cuda:0")
    sizes = model_blocks(args.shape)[:args.blocks]
    path = os.path.join(args.dir, "ratel_ssd_states.bin")
    runs = [(d, h, sc, io) for h in args.handlers.split(",") for d in (int(x) for x in args.depths.split(","))
            for sc in args.schedules.split(",") for io in args.io.split(",")]
    for depth, handler, sched, io in runs:
        cfg = R.ratel_default_config()
        cfg.pipeline_depth = depth
        cfg.ssd_schedule = {"duplex": R.RATEL_SSD_DUPLEX, "simplex": R.RATEL_SSD_SIMPLEX}[sched]
        cfg.ssd_io = {"pread": R.RATEL_SSD_IO_PREAD, "uring": R.RATEL_SSD_IO_URING}[io]
        if args.tile_elems:
            cfg.tile_elems = args.tile_elems
        R.ratel_init(0, 0, 1, None, cfg)
        fds = []
        try:
            offs, off = [], 0
            for n in sizes:
                offs.append(off)
                off += R.ratel_ssd_range_bytes(n, 1, 0)
            fdw = os.open(path, os.O_RDWR | os.O_CREAT | os.O_TRUNC, 0o600)
            os.ftruncate(fdw, off)
            fds.append(fdw)
            p16, g16 = [], []
            chunk = 1 << 26
            tmp = torch.empty(chunk, dtype=torch.float32, device=dev)
            for b, n in enumerate(sizes):      # theta0 from the device generator, m = v = 0 (written by warm-up)
                key = R.ratel_gen_stream_key(0x5EED5EED, 1, 0, b)
                for beg in range(0, n, chunk):
                    k = min(chunk, n - beg)
                    R.ratel_gen_theta0(tmp.data_ptr(), k, beg, key)
                    os.pwrite(fdw, tmp[:k].cpu().numpy().tobytes(), offs[b] + 4 * beg)
                p16.append(torch.zeros(R.ratel_padded_numel(n, 1), dtype=torch.bfloat16, device=dev))
                g = torch.empty(R.ratel_padded_numel(n, 1), dtype=torch.bfloat16, device=dev)
                R.ratel_gen_grad16(g.data_ptr(), n, 0, R.ratel_gen_stream_key(0x5EED5EED, 2, 1, b))
                g16.append(g)
            os.fsync(fdw)
            del tmp
            fd = os.open(path, os.O_RDWR | os.O_DIRECT)
            fds.append(fd)
            for b, n in enumerate(sizes):
                R.ratel_register_block(b, [R.make_range(p16[b], g16[b], None, None, None, n)],
                                       R.RATEL_SSD_HOST_COMPUTE if handler == "cpu" else R.RATEL_SSD)
                R.ratel_register_ssd(b, 0, fd, offs[b])
            s = torch.cuda.Stream(device=dev)
            order = list(reversed(range(len(sizes))))
            hp = (HP["lr"], HP["beta1"], HP["beta2"], HP["eps"], HP["weight_decay"])

            def step(t):
                R.ratel_adam_step(*hp, t)
                for b in order:
                    R.ratel_offload_grad_chunk(b, s)
                R.ratel_sync(None)

            t = 1
            for _ in range(args.warmup):
                step(t)
                t += 1
            torch.cuda.synchronize()
            w0 = time.perf_counter()
            for _ in range(args.steps):
                step(t)
                t += 1
            torch.cuda.synchronize()
            dt = (time.perf_counter() - w0) / args.steps
            P = sum(sizes)
            gbs = 24.0 * P / dt / 1e9
            print(json.dumps({
                "residency": "ssd" if handler == "gpu" else "ssd_host_compute", "shape": args.shape, "blocks": len(sizes), "params": P,
                "pipeline_depth": depth, "schedule": sched, "io": io, "tile_elems": int(cfg.tile_elems), "steps": args.steps,
                "warmup": args.warmup, "ms_per_step": dt * 1e3, "params_per_s": P / dt,
                "ssd_gbs_24B_per_param": gbs, "roofline_gbs": probe.get("roofline_gbs"),
                "frac": gbs / probe["roofline_gbs"] if probe.get("roofline_gbs") else None,
                "timing": "host wall clock around ratel_sync(NULL) (the reader/writer threads are host I/O)",
                "file": "one state file, O_DIRECT"}), flush=True)
        finally:
            R.ratel_finalize()
            for f in fds:
                os.close(f)
            try:
                os.unlink(path)
            except OSError:
                pass
            torch.cuda.empty_cache()


if __name__ == "__main__":
    main()
