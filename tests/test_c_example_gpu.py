"""The C ABI from plain C (examples/c_api_step.c): no Python, no torch on the
calling side -- builds with nvcc against libratel.so and runs three AGO steps."""
import os
import subprocess

import pytest

import paper_conf_icde_liaosyxcyww25_b200 as R

pytestmark = pytest.mark.gpu
ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def test_c_program_uses_the_abi(cuda_dev, tmp_path):
    exe = tmp_path / "c_api_step"
    libdir = os.path.dirname(R.LIB_PATH)
    subprocess.check_call(["nvcc", "-o", str(exe), os.path.join(ROOT, "examples", "c_api_step.c"),
                           "-I", os.path.join(ROOT, "include"), "-L", libdir, "-lratel",
                           "-Xlinker", f"-rpath={libdir}"])
    r = subprocess.run([str(exe)], capture_output=True, text=True, timeout=120)
    assert r.returncode == 0, r.stdout + r.stderr
    assert "launches=3 p16_matches_master=1" in r.stdout, r.stdout
