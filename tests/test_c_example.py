"""The C ABI is usable from plain C: examples/c_api_example.c compiles and
links against libkde.so (CPU), and runs end to end on a GPU."""
import os
import subprocess

import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
LIBDIR = os.path.join(ROOT, "paper_conf_sigmod_heimelkm15_b200")


def _build(tmp_path):
    exe = str(tmp_path / "c_api_example")
    subprocess.check_call(["gcc", "-O2", "-std=c99", "-Wall", "-I", os.path.join(ROOT, "include"),
                           os.path.join(ROOT, "examples", "c_api_example.c"), "-L", LIBDIR, "-l:libkde.so",
                           "-Wl,-rpath," + LIBDIR, "-lm", "-o", exe])
    return exe


def test_c_example_compiles_and_links(tmp_path):
    assert os.path.exists(_build(tmp_path))


@pytest.mark.gpu
def test_c_example_runs(tmp_path):
    import torch
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    r = subprocess.run([_build(tmp_path)], capture_output=True, text=True, timeout=300)
    assert r.returncode == 0, r.stdout + r.stderr
    assert "p_hat after replacement" in r.stdout
