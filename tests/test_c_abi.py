"""The C ABI used from plain C (tests/c/stitch_c_demo.c): it compiles and links against
include/stitch.h and libstitch_b200.so with gcc alone (CPU); on a B200 it runs steps 1-7, the
bounded mode and an error path without Python or torch in the process (GPU)."""
import os
import subprocess

import pytest

import __graft_entry__

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
PKG = os.path.join(ROOT, "paper_conf_icpp_blattnerkcsbz14_b200")


def build_demo(tmp_path):
    __graft_entry__.build()
    exe = str(tmp_path / "stitch_c_demo")
    subprocess.check_call(["gcc", "-O2", "-std=c11", "-I", os.path.join(ROOT, "include"),
                           os.path.join(ROOT, "tests", "c", "stitch_c_demo.c"), "-L", PKG,
                           "-lstitch_b200", "-Wl,-rpath," + PKG, "-lm", "-o", exe])
    return exe


def test_c_demo_compiles_and_links(tmp_path):
    exe = build_demo(tmp_path)
    assert os.path.exists(exe)


@pytest.mark.gpu
def test_c_demo_runs(tmp_path):
    exe = build_demo(tmp_path)
    out = subprocess.run([exe], capture_output=True, text=True, timeout=300)
    print(out.stdout)
    assert out.returncode == 0, out.stdout + out.stderr
    assert "0 mismatches" in out.stdout
