"""The C-ABI is usable from plain C: examples/adder_c_abi.c compiles and links against
libgsim.so with gcc (CPU); on a GPU it runs and checks a+b on all 65,536 input pairs."""
import os
import subprocess

import pytest

from tests._build import ensure_built

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
ensure_built()


def _compile():
    os.makedirs(os.path.join(ROOT, "build_examples"), exist_ok=True)
    exe = os.path.join(ROOT, "build_examples", "adder_c_abi")
    pkg = os.path.join(ROOT, "paper_conf_ipps_gavierrprs23_b200")
    subprocess.check_call(["gcc", "-O2", "-std=c11", "-Wall", "-Werror", "-I" + os.path.join(ROOT, "include"),
                           "-I/usr/local/cuda/include", os.path.join(ROOT, "examples", "adder_c_abi.c"),
                           "-L" + pkg, "-l:libgsim.so", "-L/usr/local/cuda/lib64", "-lcudart",
                           "-Wl,-rpath," + pkg, "-o", exe])
    return exe


def test_c_example_compiles_and_links():
    assert os.path.exists(_compile())


@pytest.mark.gpu
def test_c_example_runs_on_gpu():
    r = subprocess.run([_compile()], capture_output=True, text=True, timeout=300)
    assert r.returncode == 0, r.stdout + r.stderr
    assert "0 mismatches" in r.stdout
