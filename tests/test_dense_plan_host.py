"""Host logic of the dense-block planner (csrc/dense_plan.cpp, DESIGN §6 "Dense blocks"):
compiled with g++ against a small C++ driver (tests/cpp/dense_plan_check.cpp) and checked
without a GPU: blocks + residual reproduce the tile exactly (the split of the stage sum
C_i (+)= A_ij H_j of P:705-720 into two parts loses no entry and adds none)."""
import os
import subprocess

import pytest

HERE = os.path.dirname(os.path.abspath(__file__))
ROOT = os.path.dirname(HERE)
CSRC = os.path.join(ROOT, "paper_conf_icpp_balinsc22_b200", "csrc")


@pytest.fixture(scope="module")
def exe(tmp_path_factory):
    out = str(tmp_path_factory.mktemp("dp") / "dense_plan_check")
    subprocess.check_call(["g++", "-O2", "-std=c++17", "-I", CSRC, "-I", os.path.join(ROOT, "include"),
                           os.path.join(HERE, "cpp", "dense_plan_check.cpp"), os.path.join(CSRC, "dense_plan.cpp"),
                           "-o", out])
    return out


@pytest.mark.parametrize("thr,seed", [("0.05", 1), ("0.01", 2), ("0.2", 3), ("0.5", 4)])
def test_blocks_plus_residual_reproduce_tile(exe, thr, seed):
    r = subprocess.run([exe, thr, str(seed)], capture_output=True, text=True, timeout=120)
    assert r.returncode == 0, r.stdout + r.stderr
    assert "max err 0" in r.stdout
    # a 30 %-dense core fills 128 x 32 blocks above every threshold up to ~0.3, none at 0.5
    assert ("active 1" in r.stdout) == (float(thr) < 0.3), r.stdout
