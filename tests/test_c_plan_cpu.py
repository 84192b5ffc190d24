"""The planner's C ABI from plain C (examples/c_plan_swap.c): gcc against
libratel.so, no Python on the calling side, no GPU (host code)."""
import os
import subprocess

import paper_conf_icde_liaosyxcyww25_b200 as R

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def test_c_program_plans_the_hand_example(tmp_path):
    exe = tmp_path / "c_plan_swap"
    libdir = os.path.dirname(R.LIB_PATH)
    subprocess.check_call(["gcc", "-std=c11", "-Wall", "-Werror", "-o", str(exe),
                           os.path.join(ROOT, "examples", "c_plan_swap.c"), "-I", os.path.join(ROOT, "include"),
                           "-L", libdir, "-lratel", f"-Wl,-rpath,{libdir}"])
    r = subprocess.run([str(exe)], capture_output=True, text=True, timeout=60)
    assert r.returncode == 0, r.stdout + r.stderr
    assert "order=1,0,2,3 n_swap=3 a_g2m=70 flop_r=0 t_f=7 t_b=12.5 t_iter=19.5" in r.stdout, r.stdout
    assert "bad_layer_rc=-1 msg=ratel swap planner: invalid layer act_bytes" in r.stdout, r.stdout
