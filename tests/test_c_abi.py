"""librap.so from plain C (tests/c_abi_smoke.c): compiled here on CPU, run on the GPU."""
import glob
import os
import subprocess

import pytest

from conftest import ROOT


def _build(tmp_path):
    exe = str(tmp_path / "c_abi_smoke")
    subprocess.check_call(["gcc", "-O2", "-std=c99", "-D_GNU_SOURCE", "-Wall", "-I", os.path.join(ROOT, "include"),
                           os.path.join(ROOT, "tests", "c_abi_smoke.c"), "-o", exe, "-ldl"])
    return exe


def _cudart():
    import torch
    cands = glob.glob(os.path.join(os.path.dirname(torch.__file__), "..", "nvidia", "cuda_runtime", "lib",
                                   "libcudart.so*"))
    cands += glob.glob("/usr/local/cuda/lib64/libcudart.so*")
    return sorted(cands)[-1] if cands else "libcudart.so"


def test_c_program_compiles_against_header(tmp_path):
    assert os.path.exists(_build(tmp_path))


@pytest.mark.gpu
def test_c_program_runs(tmp_path):
    from paper_conf_icppw_nakanomi14_b200 import build
    lib = build.build()
    out = subprocess.run([_build(tmp_path), lib, _cudart()], capture_output=True, text=True, timeout=300)
    assert out.returncode == 0, out.stderr
    assert "c_abi_smoke ok" in out.stdout
