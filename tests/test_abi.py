"""C-ABI library checks that need no GPU: it loads, exports every symbol include/ncc.h
declares, struct layouts match, and argument validation runs before any device work."""
import ctypes
import os
import re

import pytest

from paper_conf_ipps_moorelk13_b200 import _native as N
from paper_conf_ipps_moorelk13_b200 import build as B

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


@pytest.fixture(scope="module")
def L():
    B.build()
    return N.lib()


def declared_functions():
    src = open(os.path.join(ROOT, "include", "ncc.h")).read()
    src = re.sub(r"/\*.*?\*/", "", src, flags=re.S)
    return sorted(set(re.findall(r"^\s*(?:ncc_status|const char\*|int32_t)\s+(\w+)\s*\(", src, flags=re.M)))


def test_exports_every_declared_symbol(L):
    names = declared_functions()
    assert len(names) >= 12
    for n in names:
        assert hasattr(L, n), n
    assert set(names) == set(N.EXPORTS)


def test_build_arch(L):
    assert L.ncc_build_arch() == 100


def test_struct_sizes():
    assert ctypes.sizeof(N.NccPeak) == 16
    assert ctypes.sizeof(N.PivVector) == 24
    assert ctypes.sizeof(N.NccProblem) == 88  # 5 x i32, pad, i64, 13 x 32-bit (+pad)


def test_sm100a_cubin_in_library(L):
    import subprocess
    out = subprocess.run(["cuobjdump", "--list-elf", N.LIB_PATH], capture_output=True, text=True).stdout
    assert "sm_100a" in out


def test_status_strings(L):
    for k, v in N.STATUS.items():
        assert N.ncc_status_string(k) == v


def _create(**kw):
    base = dict(mode=N.NCC_MODE_MATCH, image_h=64, image_w=64, tmpl_h=16, tmpl_w=16)
    base.update(kw)
    p = N.make_problem(**base)
    h = ctypes.c_void_p()
    return N.lib().ncc_plan_create(ctypes.byref(p), 0, ctypes.byref(h)), h.value


@pytest.mark.parametrize("kw", [
    dict(tmpl_h=65), dict(tmpl_w=0), dict(image_h=0), dict(image_pitch=10), dict(batch=0),
    dict(shard_count=0), dict(shard_rank=2, shard_count=2), dict(search_y=3),
    dict(mode=N.NCC_MODE_PIV, search_y=-1, search_x=2, step_y=4, step_x=4),
    dict(mode=N.NCC_MODE_PIV, search_y=40, search_x=2, step_y=4, step_x=4),
    dict(mode=N.NCC_MODE_PIV, search_y=2, search_x=2, step_y=0, step_x=4),
    dict(mode=N.NCC_MODE_PIV, search_y=2, search_x=2, step_y=4, step_x=4, shard_count=2),
    dict(mode=7), dict(shard_count=50, shard_rank=0),
])
def test_invalid_arguments_rejected_before_device(L, kw):
    st, h = _create(**kw)
    assert st == 1 and not h  # NCC_ERR_INVALID_ARGUMENT, *out == NULL


def test_bad_score_rejected(L):
    st, h = _create(score=5)
    assert st == 1 and not h


def test_null_arguments(L):
    assert L.ncc_plan_create(None, 0, None) == 1
    assert L.ncc_plan_destroy(None) == 0
    assert L.ncc_match(None, None, None, 16, None, None, None) == 1
    assert L.piv_correlate(None, None, None, None, None) == 1
    assert L.ncc_plan_query(None, None, 0) == 1


def test_product_package_does_not_import_oracle():
    pkg = os.path.join(ROOT, "paper_conf_ipps_moorelk13_b200")
    for dp, _, fs in os.walk(pkg):
        for f in fs:
            if f.endswith((".py", ".cu", ".cuh", ".h")):
                txt = open(os.path.join(dp, f)).read()
                assert "import oracle" not in txt and "from oracle" not in txt and "ncc_oracle" not in txt, f


def test_c_example_compiles_against_the_header(tmp_path):
    """The C ABI is usable from plain C (gcc, no CUDA headers): examples/ncc_example.c."""
    import subprocess
    exe = tmp_path / "ncc_example"
    r = subprocess.run(["gcc", "-O2", "-I", os.path.join(ROOT, "include"), os.path.join(ROOT, "examples", "ncc_example.c"),
                        "-o", str(exe), "-L", os.path.dirname(N.LIB_PATH), "-lncc_b200",
                        "-Wl,-rpath," + os.path.dirname(N.LIB_PATH)], capture_output=True, text=True)
    assert r.returncode == 0, r.stderr


def test_experiments_tables_match_the_committed_sweep(tmp_path):
    """EXPERIMENTS.md's tables are generated from profiles/r02_paper_sweeps.jsonl
    (tools/experiments_md.py): regenerating them from the committed measurements changes
    nothing, and every sweep run was correct against its planted input."""
    import json
    import shutil
    import subprocess
    import sys
    root = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
    src = os.path.join(root, "profiles", "r02_paper_sweeps.jsonl")
    md = tmp_path / "EXPERIMENTS.md"
    shutil.copy(os.path.join(root, "EXPERIMENTS.md"), md)
    subprocess.run([sys.executable, os.path.join(root, "tools", "experiments_md.py"), src, str(md)], check=True)
    assert md.read_text() == open(os.path.join(root, "EXPERIMENTS.md")).read()
    rows = [json.loads(l) for l in open(src) if l.strip().startswith("{")]
    assert rows and all(r["correct"] in (True, None) for r in rows)


def test_python_binding_validates_buffers_before_the_c_abi():
    """wrong dtype / device / shape / contiguity / size raise ValueError
    in the binding instead of reaching the C ABI as raw pointers (checked on host tensors)."""
    import torch
    from paper_conf_ipps_moorelk13_b200.api import _check_tensor, _check_template
    ok = torch.zeros((2, 8, 10), dtype=torch.float32)
    _check_tensor(ok, "images", torch.float32, None, 2 * 8 * 10, last_dims=(8, 10))
    bad = [
        (ok.double(), dict(dtype=torch.float32)),                          # dtype
        (ok[:, :, :5], dict(last_dims=(8, 10))),                            # trailing shape
        (ok.transpose(1, 2), dict()),                                       # not contiguous
        (ok[:1], dict()),                                                   # too small
    ]
    for t, kw in bad:
        args = dict(dtype=torch.float32, device=None, min_numel=2 * 8 * 10, last_dims=None)
        args.update(kw)
        with pytest.raises(ValueError):
            _check_tensor(t, "x", args["dtype"], args["device"], args["min_numel"], last_dims=args["last_dims"])
    with pytest.raises(ValueError):  # a device tensor where host memory is required is caught too
        _check_tensor(ok, "x", torch.float32, torch.device("cuda", 0), 1)
    # templates: (h, >= w) with unit column stride; a padded row pitch is fine
    big = torch.zeros((6, 12), dtype=torch.float32)
    _check_template(big[:, :7], "tmpl", 6, 7, None)
    with pytest.raises(ValueError):
        _check_template(big[:, ::2], "tmpl", 6, 6, None)  # column stride 2
    with pytest.raises(ValueError):
        _check_template(big, "tmpl", 7, 7, None)  # too few rows


def test_sensitivity_surfaces_match_the_committed_sweep(tmp_path):
    """EXPERIMENTS.md's Tab 6.21 / 6.22 surfaces are generated from profiles/r02_sensitivity.jsonl
    (tools/sensitivity_md.py): regenerating them changes nothing; every built point was correct."""
    import json
    import shutil
    import subprocess
    import sys
    root = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
    src = os.path.join(root, "profiles", "r02_sensitivity.jsonl")
    md = tmp_path / "EXPERIMENTS.md"
    shutil.copy(os.path.join(root, "EXPERIMENTS.md"), md)
    subprocess.run([sys.executable, os.path.join(root, "tools", "sensitivity_md.py"), src, str(md)], check=True)
    assert md.read_text() == open(os.path.join(root, "EXPERIMENTS.md")).read()
    rows = [json.loads(l) for l in open(src) if l.strip().startswith("{")]
    built = [r for r in rows if "tflops" in r]
    assert len(built) >= 40 and all(r["correct"] for r in built)
    assert {r["table"] for r in built} == {"6.21", "6.22"}
