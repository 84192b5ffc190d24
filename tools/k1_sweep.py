"""K1 build-variant sweep on the B200 (tools, not product).

  python tools/k1_sweep.py build          # here: nvcc variants -> build/variants/
  python tools/k1_sweep.py run [blocks]   # on the GPU: time every variant on the
                                          # same 13B-shaped device states
Each variant is a separate libratel.so (own static cudart + state), loaded
side by side with ctypes; states are allocated once by torch and registered
with each library in turn.  Prints one JSON line per variant.
"""
import ctypes
import glob
import itertools
import json
import os
import sys
from concurrent.futures import ThreadPoolExecutor

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
VDIR = os.path.join(ROOT, "build", "variants")

GRID = {"LDST": [0, 1, 2], "UNROLL": [1, 2, 4], "MINB": [1, 2, 3]}


def build():
    from paper_conf_icde_liaosyxcyww25_b200 import _build
    os.makedirs(VDIR, exist_ok=True)
    jobs = []
    for ldst, un, mb in itertools.product(GRID["LDST"], GRID["UNROLL"], GRID["MINB"]):
        name = f"ldst{ldst}_u{un}_mb{mb}"
        jobs.append((name, [f"RATEL_K1_LDST={ldst}", f"RATEL_K1_UNROLL={un}", f"RATEL_K1_MINB={mb}"]))
    with ThreadPoolExecutor(8) as ex:
        for name, path in zip([j[0] for j in jobs], ex.map(
                lambda j: _build.build(out=os.path.join(VDIR, f"libratel_{j[0]}.so"), defines=j[1]), jobs)):
            print(name, path)


TMA_GRID = [  # (consumer warps, stages, CTAs per SM, evict-first) -- dynamic tile scheduling
    (16, 3, 1, 0), (8, 6, 1, 0), (8, 8, 1, 0), (12, 5, 1, 0), (8, 4, 2, 0), (16, 2, 2, 0), (4, 7, 2, 0),
    (16, 4, 1, 1), (8, 8, 1, 1)]
if os.environ.get("RATEL_TMA_GRID"):   # e.g. "8,6,1,0;8,7,1,0"
    TMA_GRID = [tuple(int(x) for x in g.split(",")) for g in os.environ["RATEL_TMA_GRID"].split(";")]


def build_tma():
    """TMA K1 geometry variants (the default is 16 warps x 4 stages x 1 CTA/SM)."""
    from paper_conf_icde_liaosyxcyww25_b200 import _build
    os.makedirs(VDIR, exist_ok=True)
    for f in glob.glob(os.path.join(VDIR, "libratel_*.so")):
        os.remove(f)
    jobs = []
    for w, st, c, ef in TMA_GRID:
        name = f"tma_w{w}s{st}c{c}" + ("_ef" if ef else "")
        jobs.append((name, [f"RATEL_TMA_CONSUMER_WARPS={w}", f"RATEL_TMA_STAGES={st}",
                            f"RATEL_TMA_CTAS_PER_SM={c}", f"RATEL_TMA_EVICT_FIRST={ef}"]))
    with ThreadPoolExecutor(8) as ex:
        for name, path in zip([j[0] for j in jobs], ex.map(
                lambda j: _build.build(out=os.path.join(VDIR, f"libratel_{j[0]}.so"), defines=j[1]), jobs)):
            print(name, path)


def copy_gbs(torch):
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
    del a, b
    return 4 * (1 << 30) / (best / 1e3) / 1e9


def check_variant(torch, R, L, base_out=None):
    """2 steps on a small ragged block; returns (theta, m, v, p) bytes."""
    dev = torch.device("cuda:0")
    n = 1_000_003
    base = R.lib()
    th = torch.empty(n + 5, dtype=torch.float32, device=dev)
    base.ratel_gen_theta0(th.data_ptr(), n, 0, base.ratel_gen_stream_key(0x5EED5EED, 1, 0, 9), None)
    m = torch.zeros(n + 5, device=dev)
    v = torch.zeros(n + 5, device=dev)
    p = torch.zeros(n + 5, dtype=torch.bfloat16, device=dev)
    g = torch.empty(n + 5, dtype=torch.bfloat16, device=dev)
    cfg = R.ratel_config()
    L.ratel_default_config(ctypes.byref(cfg))
    assert L.ratel_init(0, 0, 1, None, ctypes.byref(cfg)) == 0, L.ratel_last_error()
    arr = (R.ratel_range * 1)(R.make_range(p, g, th, m, v, n))
    assert L.ratel_register_block(0, arr, 1, 0) == 0
    for t in (1, 2):
        base.ratel_gen_grad16(g.data_ptr(), n, 0, base.ratel_gen_stream_key(0x5EED5EED, 2, t, 9), None)
        torch.cuda.synchronize()
        assert L.ratel_adam_step(1e-3, 0.9, 0.999, 1e-8, 1e-2, t) == 0
        assert L.ratel_offload_grad_chunk(0, None) == 0
        assert L.ratel_sync(None) == 0
    assert L.ratel_finalize() == 0
    out = [x[:n].view(torch.int32 if x.dtype == torch.float32 else torch.int16).clone() for x in (th, m, v, p)]
    if base_out is not None:
        return all(torch.equal(a, b) for a, b in zip(out, base_out))
    return out


def run(nblocks=8, steps=10, warmup=3, rounds=int(os.environ.get("RATEL_SWEEP_ROUNDS", "3"))):
    import torch
    from paper_conf_icde_liaosyxcyww25_b200 import ratel as R
    dev = torch.device("cuda:0")
    n = 12 * 5120 * 5120 + 13 * 5120
    base = R.lib()
    blocks = []
    for b in range(nblocks):
        th = torch.empty(n, dtype=torch.float32, device=dev)
        base.ratel_gen_theta0(th.data_ptr(), n, 0, base.ratel_gen_stream_key(0x5EED5EED, 1, 0, b), None)
        m = torch.zeros(n, device=dev)
        v = torch.zeros(n, device=dev)
        p = torch.zeros(n, dtype=torch.bfloat16, device=dev)
        blocks.append((p, th, m, v))
    g = torch.empty(n, dtype=torch.bfloat16, device=dev)
    base.ratel_gen_grad16(g.data_ptr(), n, 0, base.ratel_gen_stream_key(0x5EED5EED, 2, 1, 0), None)
    torch.cuda.synchronize()
    libs = sorted(glob.glob(os.path.join(VDIR, "libratel_*.so")))
    libs = [R.LIB_PATH] + libs
    results = {}
    print(json.dumps({"torch_copy_gbs": copy_gbs(torch)}), flush=True)
    ref = check_variant(torch, R, R.load_library(R.LIB_PATH))
    for path in libs:
        ok = check_variant(torch, R, R.load_library(path, strict=False), ref)
        print(json.dumps({"variant": os.path.basename(path), "bitwise_equal_to_intree": ok}), flush=True)
    uss = [int(x) for x in os.environ.get("RATEL_SWEEP_US", "1").split(",")]
    for rnd, path, us in [(r, p, u) for r in range(rounds) for p in libs for u in uss]:
        L = R.load_library(path, strict=False)
        cfg = R.ratel_config()
        L.ratel_default_config(ctypes.byref(cfg))
        cfg.timing = 1
        cfg.update_streams = us
        assert L.ratel_init(0, 0, 1, None, ctypes.byref(cfg)) == 0, L.ratel_last_error()
        for b, (p, th, m, v) in enumerate(blocks):
            rr = R.make_range(p, g, th, m, v, n)
            arr = (R.ratel_range * 1)(rr)
            assert L.ratel_register_block(b, arr, 1, 0) == 0, L.ratel_last_error()
        s = torch.cuda.Stream()
        t = 1
        def step(t):
            assert L.ratel_adam_step(1e-3, 0.9, 0.999, 1e-8, 1e-2, t) == 0
            for b in reversed(range(nblocks)):
                assert L.ratel_offload_grad_chunk(b, ctypes.c_void_p(s.cuda_stream)) == 0
            assert L.ratel_sync(ctypes.c_void_p(s.cuda_stream)) == 0
        for _ in range(warmup):
            step(t); t += 1
        torch.cuda.synchronize()
        ms, cnt = ctypes.c_double(), ctypes.c_int64()
        L.ratel_kernel_timing(ctypes.byref(ms), ctypes.byref(cnt), 1)
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record(s)
        for _ in range(steps):
            step(t); t += 1
        e1.record(s)
        e1.synchronize()
        L.ratel_kernel_timing(ctypes.byref(ms), ctypes.byref(cnt), 1)
        step_ms = e0.elapsed_time(e1) / steps
        bytes_ = 28 * n * nblocks * steps
        k1 = bytes_ / (ms.value / 1e3) / 1e9
        name = os.path.basename(path) + f"/us{us}"
        results.setdefault(name, []).append(k1)
        print(json.dumps({"round": rnd, "variant": name, "k1_gbs": k1,
                          "step_gbs": 28 * n * nblocks / (step_ms / 1e3) / 1e9,
                          "avg_launch_ms": ms.value / cnt.value}), flush=True)
        assert L.ratel_finalize() == 0
    print(json.dumps({"torch_copy_gbs": copy_gbs(torch)}), flush=True)
    for k, v in sorted(results.items(), key=lambda kv: sorted(kv[1])[len(kv[1]) // 2]):
        print(json.dumps({"variant": k, "median_k1_gbs": sorted(v)[len(v) // 2], "all": v}), flush=True)


if __name__ == "__main__":
    if sys.argv[1] == "build":
        build()
    elif sys.argv[1] == "build_tma":
        build_tma()
    else:
        run(int(sys.argv[2]) if len(sys.argv) > 2 else 8)
