"""C-ABI library checks that need no GPU: it loads, exports every symbol the
headers declare, its host-only functions (partition, generator keys) are
right, and every stateful call fails cleanly without a device."""
import ctypes
import os
import re

import numpy as np
import pytest

import synth
import paper_conf_icde_liaosyxcyww25_b200 as R

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def declared_functions():
    names = []
    for h in ("ratel.h", "ratel_gen.h", "ratel_plan.h"):
        src = open(os.path.join(ROOT, "include", h)).read()
        src = re.sub(r"/\*.*?\*/", "", src, flags=re.S)
        names += re.findall(r"^[A-Za-z_][\w\s\*]*?\b(ratel_\w+)\s*\(", src, flags=re.M)
    return sorted(set(names))


def test_exports_every_declared_symbol():
    names = declared_functions()
    assert len(names) >= 20, names
    lib = ctypes.CDLL(R.LIB_PATH)
    missing = [n for n in names if not hasattr(lib, n)]
    assert not missing, missing


def test_built_for_sm100a_only():
    out = os.popen(f"cuobjdump -lelf {R.LIB_PATH} 2>/dev/null").read()
    if not out:
        pytest.skip("cuobjdump unavailable")
    archs = set(re.findall(r"sm_(\d+a?)", out))
    assert archs == {"100a"}, archs


def test_stateful_calls_without_init_are_estate():
    for f in (lambda: R.ratel_adam_step(1e-3, 0.9, 0.999, 1e-8, 0.0, 1),
              lambda: R.ratel_offload_grad_chunk(0, None),
              lambda: R.ratel_sync(None),
              lambda: R.ratel_finalize(),
              lambda: R.ratel_get_grad_sumsq()):
        with pytest.raises(R.RatelError) as e:
            f()
        assert e.value.code == R.RATEL_ESTATE
    assert R.ratel_optimizer_stream() is None
    assert R.ratel_launch_count() == 0


def test_init_without_gpu_fails_cleanly():
    import torch
    if torch.cuda.is_available():
        pytest.skip("a GPU is present: this checks the no-device failure path")
    with pytest.raises(R.RatelError) as e:
        R.ratel_init(0)
    assert e.value.code in (R.RATEL_ECUDA, R.RATEL_EINVAL)
    assert "device" in R.ratel_last_error() or "CUDA" in R.ratel_last_error()
    # bad arguments are rejected before touching CUDA
    with pytest.raises(R.RatelError) as e:
        R.ratel_init(0, 2, 2, None)
    assert e.value.code == R.RATEL_EINVAL
    with pytest.raises(R.RatelError) as e:
        R.ratel_init(0, 1, 2, None)  # world > 1 needs a unique id
    assert e.value.code == R.RATEL_EINVAL
    cfg = R.ratel_default_config()
    cfg.pipeline_depth = 17
    with pytest.raises(R.RatelError) as e:
        R.ratel_init(0, 0, 1, None, cfg)
    assert e.value.code == R.RATEL_EINVAL


def test_default_config():
    c = R.ratel_default_config()
    assert (c.mode, c.max_grad_norm, c.pipeline_depth, c.staging, c.tile_elems, c.max_ctas, c.timing, c.comm,
            c.host_threads, c.update_streams, c.cta_tiles, c.k1_kernel) == \
        (R.RATEL_ADAMW, 0.0, 4, R.RATEL_STAGING_PIPELINED, 1 << 24, 0, 0, R.RATEL_COMM_AUTO, 0, 2, 0, R.RATEL_UPDATE_TMA)


@pytest.mark.parametrize("world", [1, 2, 3, 4, 8])
def test_partition_covers_range_exactly(world):
    """Slices of every rank tile [0, n) in order, disjointly; each slice
    starts at a multiple of 8 elements (16-byte aligned for bf16 and fp32);
    all ranks own ceil-equal shares."""
    rng = np.random.default_rng(world)
    ns = [1, 7, 8, 9, 63, 64, 65, 8 * world, 8 * world + 1, 789_760, 314_639_360, 1_812_099_072]
    ns += [int(x) for x in rng.integers(1, 10 ** 7, 50)]
    for n in ns:
        cap = R.ratel_padded_numel(n, world)
        assert cap >= n and cap % (8 * world) == 0 and cap - n < 8 * world
        s = cap // world
        prev = 0
        for r in range(world):
            b, e = R.ratel_rank_slice(n, world, r)
            assert b == min(n, r * s) and e == min(n, b + s)
            assert b == prev or b == n
            assert b % 8 == 0 or b == n
            prev = e
        assert prev == n


def test_rank_slice_rejects_bad_args():
    with pytest.raises(R.RatelError):
        R.ratel_rank_slice(10, 2, 2)
    with pytest.raises(R.RatelError):
        R.ratel_rank_slice(10, 0, 0)
    assert R.ratel_padded_numel(10, 0) == 0


def test_generator_keys_match_synth():
    for args in [(synth.SEED, 1, 0, 0), (synth.SEED, 2, 7, 40), (0, 0, 0, 0), (2 ** 64 - 1, 5, 2 ** 40, 3)]:
        assert R.ratel_gen_stream_key(*args) == synth.stream_key(*args)


def test_struct_layouts_match_header():
    # ratel_config: int, double, int, int, uint64, int x 9 -> 68 bytes, padded to 72 (double alignment)
    assert ctypes.sizeof(R.ratel_config) == 72
    assert R.ratel_config.k1_kernel.offset == 56
    assert R.ratel_config.ssd_schedule.offset == 60 and R.ratel_config.ssd_io.offset == 64
    assert R.ratel_config.update_streams.offset == 48
    assert R.ratel_config.tile_elems.offset == 24
    # ratel_range: 2 ptrs, int, 3 ptrs, uint64, int -> 64 bytes
    assert ctypes.sizeof(R.ratel_range) == 64
    assert R.ratel_range.master.offset == 24 and R.ratel_range.numel.offset == 48


def test_ssd_range_bytes():
    """3 fp32 arrays of the rank slice, each padded to 4096 bytes (pure host)."""
    for n, world, rank in [(1, 1, 0), (1024, 1, 0), (1025, 1, 0), (300_001, 1, 0), (300_001, 4, 3), (16, 4, 3)]:
        b, e = R.ratel_rank_slice(n, world, rank)
        want = 3 * ((4 * (e - b) + 4095) // 4096 * 4096)
        assert R.ratel_ssd_range_bytes(n, world, rank) == want
    assert R.ratel_ssd_range_bytes(10, 0, 0) == 0


def test_struct_layouts_match_the_c_compiler(tmp_path):
    """ratel.py's ctypes structs against what a C compiler makes of
    include/ratel.h (sizeof / offsetof of every field)."""
    import subprocess
    fields = {"ratel_config": [f[0] for f in R.ratel_config._fields_],
              "ratel_range": [f[0] for f in R.ratel_range._fields_]}
    src = ["#include <stdio.h>", "#include <stddef.h>", '#include "ratel.h"', "int main(void) {"]
    for st, fs in fields.items():
        src.append(f'  printf("{st} size %zu\\n", sizeof({st}));')
        for f in fs:
            src.append(f'  printf("{st} {f} %zu\\n", offsetof({st}, {f}));')
    src += ["  return 0;", "}"]
    c = tmp_path / "layout.c"
    c.write_text("\n".join(src))
    exe = tmp_path / "layout"
    subprocess.check_call(["gcc", "-I", os.path.join(ROOT, "include"), "-o", str(exe), str(c)])
    out = subprocess.run([str(exe)], capture_output=True, text=True, check=True).stdout.split("\n")
    got = {tuple(line.split()[:2]): int(line.split()[2]) for line in out if line.strip()}
    for st, fs in fields.items():
        cls = getattr(R, st)
        assert got[(st, "size")] == ctypes.sizeof(cls), st
        for f in fs:
            assert got[(st, f)] == getattr(cls, f).offset, (st, f)
