"""bench.py's reference arm on CPU (the oracle timed as the reference, SURVEY
§8(d)): one JSON line with the contract's keys, on rank 0 only under torchrun
(the other ranks exit 0 without output)."""
import json
import os
import socket
import subprocess
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
KEYS = {"impl", "metric", "value", "unit", "n_gpus", "steps", "warmup", "ms_per_step", "higher_is_better",
        "scaling", "vs_baseline", "dtype", "data", "config", "cpu_baseline", "e2e"}


def _lines(out: str):
    return [json.loads(l) for l in out.splitlines() if l.startswith("{")]


def _check(line, n_gpus):
    assert KEYS <= set(line), KEYS - set(line)
    assert line["impl"] == "reference" and line["n_gpus"] == n_gpus
    assert line["value"] > 0 and line["unit"] == "params/s" and line["higher_is_better"] is True
    assert line["cpu_baseline"]["kind"] == "oracle" and line["cpu_baseline"]["value"] == line["value"]
    assert line["cpu_baseline"]["cores"] >= 1
    assert line["e2e"] == {"value": line["value"], "unit": "params/s", "h2d_bytes_per_step": 0,
                           "d2h_bytes_per_step": 0}
    assert line["config"]["params"] == 12_848_143_360     # C2, the bench workload


def _env():
    env = dict(os.environ, OMP_NUM_THREADS="2")
    env.pop("CUDA_VISIBLE_DEVICES", None)
    return env


def test_reference_arm_single_process():
    r = subprocess.run([sys.executable, "bench.py", "--impl", "reference", "--steps", "2", "--warmup", "1",
                        "--oracle-sample", "65536"], cwd=ROOT, capture_output=True, text=True, timeout=300,
                       env=_env())
    assert r.returncode == 0, r.stderr[-2000:]
    lines = _lines(r.stdout)
    assert len(lines) == 1, r.stdout
    _check(lines[0], 1)


def test_reference_arm_under_torchrun_prints_once():
    with socket.socket() as s:
        s.bind(("127.0.0.1", 0))
        port = s.getsockname()[1]
    r = subprocess.run([sys.executable, "-m", "torch.distributed.run", "--nnodes=1", "--nproc-per-node", "2",
                        "--master-addr", "127.0.0.1", "--master-port", str(port), "bench.py", "--impl",
                        "reference", "--gpus", "2", "--steps", "1", "--warmup", "1", "--oracle-sample", "65536"],
                       cwd=ROOT, capture_output=True, text=True, timeout=300, env=_env())
    assert r.returncode == 0, r.stderr[-2000:]
    lines = _lines(r.stdout)
    assert len(lines) == 1, r.stdout
    _check(lines[0], 2)


def test_gpus_flag_relaunches_under_torchrun():
    """`bench.py --gpus 2` outside torchrun re-launches itself with 2 ranks
    (the flag was parsed and ignored, so an 8-GPU run would
    have measured one GPU)."""
    env = _env()
    for k in ("WORLD_SIZE", "RANK", "LOCAL_RANK"):
        env.pop(k, None)
    r = subprocess.run([sys.executable, "bench.py", "--impl", "reference", "--gpus", "2", "--steps", "1",
                        "--warmup", "1", "--oracle-sample", "65536"], cwd=ROOT, capture_output=True, text=True,
                       timeout=300, env=env)
    assert r.returncode == 0, r.stderr[-2000:]
    lines = _lines(r.stdout)
    assert len(lines) == 1, r.stdout
    _check(lines[0], 2)
    assert lines[0]["config"]["parallelism"].startswith("range-sharded x2")


def test_world_size_mismatch_is_refused():
    env = dict(_env(), WORLD_SIZE="2", RANK="0", LOCAL_RANK="0")
    r = subprocess.run([sys.executable, "bench.py", "--impl", "reference", "--gpus", "4", "--steps", "1",
                        "--oracle-sample", "65536"], cwd=ROOT, capture_output=True, text=True, timeout=120, env=env)
    assert r.returncode == 2 and not _lines(r.stdout), (r.returncode, r.stdout)
    assert "WORLD_SIZE=2" in r.stderr


def test_reference_arm_reports_the_sample_it_timed():
    """ms_per_step x steps must be time that actually ran (the driver's
    consistency check): the step is one pass over the sample, with the host
    facts and the implied DRAM rate in cpu_baseline."""
    import time
    t0 = time.time()
    r = subprocess.run([sys.executable, "bench.py", "--impl", "reference", "--steps", "3", "--warmup", "1",
                        "--oracle-sample", "200000"], cwd=ROOT, capture_output=True, text=True, timeout=300,
                       env=_env())
    wall = time.time() - t0
    assert r.returncode == 0, r.stderr[-2000:]
    (line,) = _lines(r.stdout)
    assert line["steps"] * line["ms_per_step"] / 1e3 <= wall
    cb = line["cpu_baseline"]
    assert cb["sample_params"] == 200000 and cb["sample_passes"] == line["steps"]
    assert abs(line["value"] - 200000 / (line["ms_per_step"] / 1e3)) <= 1e-6 * line["value"]
    assert abs(cb["dram_gbs_at_28B_per_param"] - 28 * line["value"] / 1e9) <= 1e-9 * cb["dram_gbs_at_28B_per_param"]
    for k in ("cpu_model", "numa_nodes", "sockets"):
        assert k in cb
    assert line["full_workload_ms_per_step_extrapolated"] > line["ms_per_step"]


def test_auto_blocks_sizes_l_eff_to_the_box(monkeypatch):
    """--blocks auto: host residencies keep all ranks' fp32 states within
    85 % of MemAvailable (and P16 within 60 % of HBM); device residency fits
    (12/N + 2) B/param into 95 % of HBM.  C2 at N=1 is the whole model."""
    import argparse
    sys.path.insert(0, ROOT)
    import bench
    monkeypatch.setattr(bench, "mem_available_bytes", lambda: 196 * 10 ** 9)
    a = lambda shape, res: argparse.Namespace(shape=shape, residency=res)
    assert bench.auto_blocks(a("13B", "device"), 1) == 41          # the whole C2 model (12.85B params)
    assert bench.auto_blocks(a("70B", "host"), 1) == 17             # 0.85 * 196 GB / 9.66 GB per block
    assert bench.auto_blocks(a("175B", "host"), 1) == 7             # 21.75 GB per block
    assert bench.auto_blocks(a("70B", "host"), 8) == 17             # host RAM is shared by the ranks
    n = bench.auto_blocks(a("30B", "device"), 8)
    assert n == len(bench.model_blocks("30B"))                      # C3 fits at N = 8
    for shape, res, w in (("70B", "host", 1), ("13B", "device", 1)):
        k = bench.auto_blocks(a(shape, res), w)
        sizes = bench.model_blocks(shape)[:k]
        if res == "host":
            assert 12 * sum(sizes) <= 0.85 * 196e9 < 12 * sum(bench.model_blocks(shape)[:k + 1])


def test_nccl_log_summary(tmp_path, monkeypatch):
    sys.path.insert(0, ROOT)
    import bench
    log = tmp_path / f"nccl.host.{os.getpid()}.log"
    log.write_text("x NCCL INFO NCCL version 2.28.9+cuda12.9\nx NCCL INFO Channel 00/0 : 0[0] -> 1[1] via P2P/CUMEM\n"
                   "irrelevant\nx NCCL INFO NVLS multicast support is available on dev 0\n")
    monkeypatch.setenv("NCCL_DEBUG_FILE", str(tmp_path / "nccl.%h.%p.log"))
    out = bench.nccl_init_summary()
    assert out["log"] == str(log) and len(out["lines"]) == 3
    assert any("via P2P" in line for line in out["lines"]) and any("NVLS" in line for line in out["lines"])


def test_bench_host_helpers(monkeypatch, tmp_path):
    """Host-side helpers added for N > 1 and the reference arm: the sweep
    parser, the WORLD_SIZE / --gpus reconciliation, the NCCL log routing and
    the CPU facts reported with the oracle."""
    import argparse
    sys.path.insert(0, ROOT)
    import bench
    for k in ("NCCL_SOCKET_IFNAME", "NCCL_IB_DISABLE", "NCCL_DEBUG_SUBSYS", "NCCL_DEBUG", "NCCL_DEBUG_FILE"):
        monkeypatch.delenv(k, raising=False)          # whatever the helpers set is undone after the test
    assert bench.token_list("0") == [] and bench.token_list("") == [] and bench.token_list("none") == []
    assert bench.token_list("1024,2048") == [1024, 2048]
    monkeypatch.setenv("WORLD_SIZE", "4")
    assert bench.relaunch_or_world(argparse.Namespace(gpus=None)) == 4
    assert bench.relaunch_or_world(argparse.Namespace(gpus=4)) == 4
    try:
        bench.relaunch_or_world(argparse.Namespace(gpus=2))
        raise AssertionError("a --gpus / WORLD_SIZE mismatch must exit")
    except SystemExit as e:
        assert e.code == 2
    monkeypatch.delenv("WORLD_SIZE")
    assert bench.relaunch_or_world(argparse.Namespace(gpus=None)) == 1
    assert bench.relaunch_or_world(argparse.Namespace(gpus=1)) == 1
    monkeypatch.setattr(bench, "NCCL_LOG_DIR", str(tmp_path / "logs"))
    bench.nccl_log_env()
    assert os.environ["NCCL_DEBUG"] == "INFO" and "%p" in os.environ["NCCL_DEBUG_FILE"]
    assert os.path.isdir(tmp_path / "logs")
    facts = bench.cpu_facts()
    assert {"cpu_model", "sockets", "numa_nodes", "nproc"} <= set(facts) and facts["nproc"] >= 1
    monkeypatch.setenv("NCCL_HOSTID", "x")
    bench.share_gpu_nccl_env(3)
    assert os.environ["NCCL_HOSTID"] == "ratel-bench-rank3"
