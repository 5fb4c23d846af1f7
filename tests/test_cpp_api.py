"""include/pagoda.hpp: the paper-named C++ API (Table 1) over the C ABI.
tests/cpp/paper_api.cpp is compiled against the header and libpagoda.so and run:
without a GPU every call must fail loudly; on a B200 it spawns, checks, waits."""
import os
import subprocess

import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
PKG = os.path.join(ROOT, "paper_conf_ppopp_yehsser17_b200")


def _build(tmp_path):
    from paper_conf_ppopp_yehsser17_b200 import build as B
    B.build()
    exe = str(tmp_path / "paper_api")
    subprocess.check_call(["/usr/local/cuda/bin/nvcc", "-std=c++17", "-I" + os.path.join(ROOT, "include"),
                           os.path.join(ROOT, "tests", "cpp", "paper_api.cpp"), "-o", exe,
                           "-L" + PKG, "-lpagoda", "-Xlinker", "-rpath=" + PKG])
    return exe


def _has_gpu():
    import torch
    return torch.cuda.is_available()


def test_paper_api_without_gpu(tmp_path):
    if _has_gpu():
        pytest.skip("GPU present: covered by test_paper_api_on_gpu")
    r = subprocess.run([_build(tmp_path)], capture_output=True, text=True, timeout=120)
    assert r.returncode == 0, r.stderr
    assert r.stdout.strip() == "nodev"


@pytest.mark.gpu
def test_paper_api_on_gpu(tmp_path):
    r = subprocess.run([_build(tmp_path)], capture_output=True, text=True, timeout=300)
    assert r.returncode == 0, r.stdout + r.stderr
    assert r.stdout.strip() == "ok"
