"""C-ABI boundary checks that run without a GPU: the library builds, loads, exports every
symbol include/pt.h declares, and fails loudly (no CPU fallback) without a device."""
from __future__ import annotations

import ctypes
import os
import re
import subprocess

import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def _declared():
    hdr = open(os.path.join(ROOT, "include", "pt.h")).read()
    hdr = re.sub(r"/\*.*?\*/", "", hdr, flags=re.S)
    return sorted(set(re.findall(r"\b(pt_[a-z_]+)\s*\(", hdr)))


@pytest.fixture(scope="module")
def ptlib():
    import paper_conf_ipps_xuzwrwxgxy12_b200 as pt
    pt.build()
    return pt


def test_header_declarations_match_binding(ptlib):
    assert _declared() == sorted(ptlib.EXPORTS)


def test_library_exports_every_declared_symbol(ptlib):
    L = ctypes.CDLL(ptlib.LIB)
    for name in _declared():
        assert hasattr(L, name), name
    out = subprocess.run(["nm", "-D", "--defined-only", ptlib.LIB], capture_output=True, text=True).stdout
    exported = set(re.findall(r"\bT (pt_[a-z_]+)$", out, flags=re.M))
    assert set(_declared()) <= exported


def test_library_is_sm100a(ptlib):
    out = subprocess.run(["cuobjdump", "--list-elf", ptlib.LIB], capture_output=True, text=True).stdout
    assert "sm_100a" in out


def test_no_fma_in_stepping_code(ptlib):
    """R15: the library is compiled with -fmad=false; no FFMA may appear in the tracking
    kernels (a contracted a*b+c would change rounding vs the oracle)."""
    sass = subprocess.run(["cuobjdump", "-sass", ptlib.LIB], capture_output=True, text=True).stdout
    assert "track_kernel" in sass
    funcs = re.split(r"\n\s*Function : ", sass)
    tracking = [f for f in funcs if f.split("\n", 1)[0].find("track") >= 0]
    # per (F, precision): 2 bench-path layouts, outputs, 4 variant / unique-map, 2 no-refill
    assert len(tracking) >= 6 * 11
    for f in tracking:
        assert "FFMA" not in f, f.split("\n", 1)[0]


def test_record_bytes(ptlib):
    assert [ptlib.pt_record_bytes(F, ptlib.PT_F32) for F in (1, 2, 3)] == [16, 32, 64]
    assert [ptlib.pt_record_bytes(F, ptlib.PT_F16) for F in (1, 2, 3)] == [8, 16, 32]
    assert ptlib.pt_record_bytes(4, ptlib.PT_F32) == 0
    assert ptlib.pt_record_bytes(2, 7) == 0


def test_no_cpu_fallback_without_device(ptlib):
    import torch
    if torch.cuda.is_available():
        pytest.skip("a GPU is present")
    with pytest.raises(ptlib.PtError) as e:
        ptlib.pt_create(0)
    assert e.value.status in (ptlib.PT_ERR_CUDA, ptlib.PT_ERR_ARG)
    assert "pt_create" in ptlib.pt_last_error(None)


def test_product_path_does_not_import_oracle():
    """The product package never imports the oracle (nor the reverse)."""
    pkg = os.path.join(ROOT, "paper_conf_ipps_xuzwrwxgxy12_b200")
    for dirpath, _, files in os.walk(pkg):
        for fn in files:
            if fn.endswith((".py", ".cu", ".cuh", ".h", ".cpp")):
                src = open(os.path.join(dirpath, fn)).read()
                assert "oracle" not in re.sub(r"#.*|//.*", "", src).replace("the oracle", ""), fn
    for fn in os.listdir(os.path.join(ROOT, "oracle")):
        if fn.endswith((".py", ".c", ".h")):
            src = open(os.path.join(ROOT, "oracle", fn)).read()
            assert "import paper_conf" not in src and "pt.h" not in src.replace("include/pt.h", ""), fn
