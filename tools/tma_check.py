"""Bitwise check of K1 build variants vs the LDG build with a tiny grid
(max_ctas) so every CTA wraps the TMA stage ring many times."""
import ctypes, glob, json, os, sys
ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import torch
from paper_conf_icde_liaosyxcyww25_b200 import ratel as R

def run(L, n, max_ctas, steps=3):
    dev = torch.device("cuda:0"); base = R.lib()
    th = torch.empty(n + 8, dtype=torch.float32, device=dev)
    base.ratel_gen_theta0(th.data_ptr(), n, 0, base.ratel_gen_stream_key(0x5EED5EED, 1, 0, 9), None)
    m = torch.zeros(n + 8, device=dev); v = torch.zeros(n + 8, device=dev)
    p = torch.zeros(n + 8, dtype=torch.bfloat16, device=dev); g = torch.empty(n + 8, dtype=torch.bfloat16, device=dev)
    cfg = R.ratel_config(); L.ratel_default_config(ctypes.byref(cfg)); cfg.max_ctas = max_ctas
    assert L.ratel_init(0, 0, 1, None, ctypes.byref(cfg)) == 0
    arr = (R.ratel_range * 1)(R.make_range(p, g, th, m, v, n))
    assert L.ratel_register_block(0, arr, 1, 0) == 0
    for t in range(1, steps + 1):
        base.ratel_gen_grad16(g.data_ptr(), n, 0, base.ratel_gen_stream_key(0x5EED5EED, 2, t, 9), None)
        torch.cuda.synchronize()
        assert L.ratel_adam_step(1e-3, 0.9, 0.999, 1e-8, 1e-2, t) == 0
        assert L.ratel_offload_grad_chunk(0, None) == 0
        assert L.ratel_sync(None) == 0
    assert L.ratel_finalize() == 0
    return [x[:n].clone() for x in (th, m, v, p.view(torch.int16))]

vdir = os.path.join(ROOT, "build", "variants")
ref = {}
for n, mc in ((300_001, 3), (1_000_003, 1), (5_000_000, 7), (20_000_000, 0)):
    ref = run(R.load_library(os.path.join(vdir, "libratel_ldg_fm.so")), n, mc)
    for path in sorted(glob.glob(os.path.join(vdir, "libratel_tma*.so"))):
        out = run(R.load_library(path), n, mc)
        bad = [int((a.view(torch.int32) != b.view(torch.int32)).sum()) if a.dtype == torch.float32 else int((a != b).sum()) for a, b in zip(out, ref)]
        print(json.dumps({"variant": os.path.basename(path), "n": n, "max_ctas": mc, "mismatches": bad}), flush=True)
