"""The boundary from plain C99 (tests/c/abi_smoke.c): compiled with gcc against
include/ddt.h and libddt.so, no Python or torch in the process."""
import os
import subprocess

import pytest

pytestmark = pytest.mark.gpu
ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def test_c99_consumer():
    from paper_conf_cluster_chukzsp20_b200.build import build
    build()
    exe = os.path.join(ROOT, "build", "abi_smoke")
    libdir = os.path.join(ROOT, "paper_conf_cluster_chukzsp20_b200")
    subprocess.check_call(["gcc", "-std=c99", "-O2", "-I", os.path.join(ROOT, "include"), "-I",
                           "/usr/local/cuda/include", os.path.join(ROOT, "tests", "c", "abi_smoke.c"), "-o", exe,
                           "-L", libdir, "-l:libddt.so", f"-Wl,-rpath,{libdir}", "-L", "/usr/local/cuda/lib64",
                           "-lcudart"])
    out = subprocess.run([exe], capture_output=True, text=True, timeout=120)
    assert out.returncode == 0, out.stdout + out.stderr
    assert out.stdout.startswith("OK"), out.stdout
