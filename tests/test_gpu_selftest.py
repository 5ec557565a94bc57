"""The sm_100a building blocks (TMA SW128/SW32, tcgen05.mma kind::tf32 and kind::i8 u8 x s8,
TMEM loads) against a CPU int64 reference on integer data (exact)."""
import os
import subprocess

import pytest

HERE = os.path.dirname(os.path.abspath(__file__))
ROOT = os.path.dirname(HERE)


def _build():
    exe = os.path.join(HERE, "cuda", "umma_selftest")
    src = exe + ".cu"
    if not os.path.exists(exe) or os.path.getmtime(exe) < os.path.getmtime(src):
        subprocess.check_call(["/usr/local/cuda/bin/nvcc", "-gencode", "arch=compute_100a,code=sm_100a", "-O2",
                               "-std=c++17", "-I", os.path.join(ROOT, "paper_conf_sigmod_wangygjxlwglxyy21_b200", "csrc"),
                               "-I", os.path.join(ROOT, "include"), "-o", exe, src])
    return exe


def test_selftest_builds():
    assert os.path.exists(_build())


@pytest.mark.gpu
def test_umma_selftest():
    r = subprocess.run([_build()], capture_output=True, text=True, timeout=120)
    assert r.returncode == 0 and "SELFTEST PASS" in r.stdout, r.stdout + r.stderr
