"""CPU-side checks of the boundary: the library builds, loads and exports every
symbol that include/arbalest.h declares; argument validation needs no GPU."""
import ctypes
import os
import re
import subprocess

import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
HEADER = os.path.join(ROOT, "include", "arbalest.h")


def declared_functions():
    src = open(HEADER).read()
    return sorted(set(re.findall(r"^\s*(?:int|const char\*)\s+(arb_\w+)\s*\(", src, re.M)))


@pytest.fixture(scope="module")
def lib():
    from paper_conf_ipps_yuphs21_b200 import build, binding
    build.build()
    return binding.load()


def test_header_declares_the_survey_calls():
    names = declared_functions()
    for f in ("arb_init", "arb_submit_events", "arb_flush", "arb_get_reports", "arb_destroy"):
        assert f in names


def test_library_exports_every_declared_symbol(lib):
    from paper_conf_ipps_yuphs21_b200.binding import EXPORTS, LIB_PATH
    out = subprocess.check_output(["nm", "-D", "--defined-only", LIB_PATH]).decode()
    exported = set(re.findall(r"\bT (arb_\w+)", out))
    assert set(declared_functions()) <= exported
    assert set(EXPORTS) == set(declared_functions())
    for name in declared_functions():
        assert getattr(lib, name) is not None


def test_sm100a_cubin_present(lib):
    from paper_conf_ipps_yuphs21_b200.binding import LIB_PATH
    out = subprocess.check_output(["/usr/local/cuda/bin/cuobjdump", "--list-elf", LIB_PATH]).decode()
    assert "sm_100a" in out


def test_argument_validation_without_gpu(lib):
    from paper_conf_ipps_yuphs21_b200.binding import arb_config, ARB_EINVAL
    h = ctypes.c_void_p()
    # misaligned range, zero size, bad world/rank: rejected before touching the GPU
    for cfg in (arb_config(3, 64, 0, 0, 1, None, 0, 0, 0), arb_config(0, 0, 0, 0, 1, None, 0, 0, 0),
                arb_config(0, 64, 0, 2, 2, None, 0, 0, 0), arb_config(0, 64, 0, 0, 0, None, 0, 0, 0)):
        assert lib.arb_init(ctypes.byref(cfg), ctypes.byref(h)) == ARB_EINVAL
        assert not h.value
    assert lib.arb_init(None, ctypes.byref(h)) == ARB_EINVAL
    assert lib.arb_destroy(None) == 0
    assert lib.arb_last_error(None) == b"null context"
    assert lib.arb_flush(None, None, None, None) == ARB_EINVAL


def test_product_does_not_import_oracle():
    pkg = os.path.join(ROOT, "paper_conf_ipps_yuphs21_b200")
    for dp, _, files in os.walk(pkg):
        for f in files:
            if f.endswith((".py", ".cu", ".cpp", ".h")):
                txt = open(os.path.join(dp, f)).read()
                assert "import oracle" not in txt and "from oracle" not in txt and "arb_oracle" not in txt, f
