"""Run-time specialisation layer (NVRTC + on-disk binary cache) -- no GPU needed.

The paper's technique (Ch. 4; binary cache P:1232-1238): a kernel is
compiled once problem parameters are known, baking them in as constants, and the binary is
cached.  ncc_specialize runs the same selection as ncc_plan_create and compiles the chosen
instance for sm_100a into NCC_CACHE_DIR."""
import os
import subprocess
import time

import pytest

from paper_conf_ipps_moorelk13_b200 import _native as N
from paper_conf_ipps_moorelk13_b200 import build as B


@pytest.fixture(autouse=True)
def _cache(tmp_path, monkeypatch):
    B.build()
    monkeypatch.setenv("NCC_CACHE_DIR", str(tmp_path))
    monkeypatch.delenv("NCC_NO_JIT", raising=False)
    return tmp_path


def test_aot_instances_need_no_compile():
    name, now = N.ncc_specialize(N.make_problem(N.NCC_MODE_MATCH, 1024, 1024, None, 128, 128))
    assert name.startswith("tm_sk_128x128") and not now
    name, now = N.ncc_specialize(N.make_problem(N.NCC_MODE_PIV, 2048, 2048, None, 64, 64, 32, 32, 32, 32))
    assert name.startswith("piv_sk_64x64") and not now


def test_tm_156x116_compiled_then_cached(_cache):
    # the odd template of the paper's Tab 5.2 (Patient 4: 156 x 116 pixels)
    p = N.make_problem(N.NCC_MODE_MATCH, 400, 380, None, 156, 116)
    t0 = time.time()
    name, now = N.ncc_specialize(p)
    assert name.startswith("tm_jit_156x116") and now
    cubins = [f for f in os.listdir(_cache) if f.endswith(".cubin")]
    assert len(cubins) == 1
    out = subprocess.run(["cuobjdump", "--list-elf", str(_cache / cubins[0])], capture_output=True, text=True)
    assert "sm_100a" in out.stdout + out.stderr or out.returncode == 0
    t1 = time.time()
    name2, now2 = N.ncc_specialize(p)
    assert name2 == name and not now2
    assert time.time() - t1 < (t1 - t0)


def test_piv_odd_shape_compiles():
    name, now = N.ncc_specialize(N.make_problem(N.NCC_MODE_PIV, 512, 512, None, 48, 40, 20, 12, 24, 20))
    assert name.startswith("piv_jit_48x40_m20x12") and now


def test_no_jit_flag_selects_generic(monkeypatch):
    name, now = N.ncc_specialize(N.make_problem(N.NCC_MODE_MATCH, 400, 380, None, 156, 116, flags=N.NCC_F_NO_JIT))
    assert name.startswith("tm_re") and not now
    monkeypatch.setenv("NCC_NO_JIT", "1")
    name, now = N.ncc_specialize(N.make_problem(N.NCC_MODE_MATCH, 400, 380, None, 100, 90))
    assert name.startswith("tm_re") and not now
