"""The SSD tier's io_uring path (csrc/ratel_uring.h, cfg.ssd_io =
RATEL_SSD_IO_URING) on the CPU: a native check writes three arrays through
the ring (more 4 MiB requests than the queue depth, a ragged tail), reads
them back, compares, and expects an error for a read past the end of file."""
import os
import subprocess

import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def test_uring_roundtrip_and_eof(tmp_path):
    exe = tmp_path / "uring_check"
    subprocess.check_call(["g++", "-O2", "-std=c++17", "-I", os.path.join(ROOT, "paper_conf_icde_liaosyxcyww25_b200",
                                                                           "csrc"),
                           "-o", str(exe), os.path.join(ROOT, "tests", "native", "uring_check.cpp")])
    r = subprocess.run([str(exe), str(tmp_path / "f.bin")], capture_output=True, text=True, timeout=120)
    if r.returncode == 77:
        pytest.skip(r.stdout.strip())
    assert r.returncode == 0, (r.returncode, r.stdout, r.stderr)
    assert r.stdout.startswith("ok depth=")
