"""The C ABI used by a pure-C client (examples/tmm_protect.c: no Python, no torch): protected bf16 TMM,
a simulated crash of one region, validate -> exactly that region, recover -> the golden bytes."""
from __future__ import annotations

import os
import subprocess

import pytest

pytestmark = pytest.mark.gpu

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def test_c_client_end_to_end():
    exe = os.path.join(ROOT, "examples", "tmm_protect")
    if not os.path.exists(exe):
        subprocess.check_call(["make", "-C", ROOT, "examples/tmm_protect"])
    r = subprocess.run([exe], capture_output=True, text=True, timeout=120)
    assert r.returncode == 0, r.stdout + r.stderr
    assert r.stdout.strip().splitlines()[-1] == "OK"
    assert "1 failed region(s), first = 9 (expected 9)" in r.stdout
