"""Host-side checks of the C ABI: the libraries load and export every declared symbol.
No compute calls (this container has no GPU)."""
import ctypes
import os
import re
import subprocess

import pytest

import paper_conf_hpdc_jaiganeshb18_b200 as ecl
from paper_conf_hpdc_jaiganeshb18_b200 import build as b

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
HEADER = os.path.join(ROOT, "include", "ecl_cc.h")


def declared_symbols():
    text = open(HEADER).read()
    return sorted(set(re.findall(r"ECL_CC_API\s+[^;(]*?\b(ecl_cc_\w+)\s*\(", text)))


@pytest.fixture(scope="module", autouse=True)
def built():
    b.build()


def test_header_declares_the_north_star_calls():
    syms = declared_symbols()
    for s in ("ecl_cc_create", "ecl_cc_run", "ecl_cc_destroy", "ecl_cc_run_i64",
              "ecl_cc_run_rows", "ecl_cc_merge", "ecl_cc_finalize", "ecl_cc_run_host"):
        assert s in syms


@pytest.mark.parametrize("stats", [False, True])
def test_library_exports_every_declared_symbol(stats):
    path = ecl.library_path(stats)
    assert os.path.exists(path)
    lib = ctypes.CDLL(path)
    for s in declared_symbols():
        assert hasattr(lib, s), s
    out = subprocess.run(["nm", "-D", "--defined-only", path], capture_output=True, text=True).stdout
    exported = set(re.findall(r"\b(ecl_cc_\w+)\b", out))
    assert exported == set(declared_symbols()), exported ^ set(declared_symbols())


def test_library_is_sm100a_native():
    out = subprocess.run(["/usr/local/cuda/bin/cuobjdump", "--list-elf", ecl.library_path()],
                         capture_output=True, text=True).stdout
    assert "sm_100a" in out


def test_host_only_calls():
    lib = ecl._load()
    assert lib.ecl_cc_version().decode().startswith("ecl_cc")
    assert lib.ecl_cc_status_string(1) == b"invalid argument"
    assert lib.ecl_cc_stats_enabled() == 0
    assert ecl._load(stats=True).ecl_cc_stats_enabled() == 1
    # argument errors are reported before touching the device
    assert lib.ecl_cc_run(None, 10, 0, None, None, None, None) == 1
    assert lib.ecl_cc_destroy(None) == 0
