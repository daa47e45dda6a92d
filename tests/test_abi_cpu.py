"""CPU-only checks of the boundary: libcdd.so loads and exports every function of include/cdd.h."""
import ctypes
import os
import re
import subprocess

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def test_library_exports_every_header_symbol():
    import paper_conf_ipps_awasthillw16_b200 as m

    names = m.header_functions()
    assert len(names) >= 16
    lib = ctypes.CDLL(os.path.join(ROOT, "paper_conf_ipps_awasthillw16_b200", "libcdd.so"))
    for n in names:
        assert hasattr(lib, n), n
    assert m.abi_version() == 5


def test_header_compiles_as_c():
    r = subprocess.run(["gcc", "-std=c99", "-Wall", "-Werror", "-fsyntax-only", "-x", "c",
                        os.path.join(ROOT, "include", "cdd.h")], capture_output=True, text=True)
    assert r.returncode == 0, r.stderr


def test_no_cpu_fallback_and_no_oracle_in_product():
    pkg = os.path.join(ROOT, "paper_conf_ipps_awasthillw16_b200")
    for dirpath, _, files in os.walk(pkg):
        for f in files:
            if f.endswith((".py", ".cu", ".cuh", ".h")):
                txt = open(os.path.join(dirpath, f)).read()
                assert not re.search(r"^\s*(import|from)\s+oracle", txt, re.M), f
                assert "oracle.h" not in txt and "liboracle" not in txt, f


def test_argument_errors_without_gpu():
    import paper_conf_ipps_awasthillw16_b200 as m
    import pytest

    with pytest.raises(m.CddError):
        m.Instance([1, 2], [1, 1], [1, 1], -1)  # d < 0 (or no device): rejected, nothing launched
