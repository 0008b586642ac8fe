"""CPU checks of the boundary: libdda.so builds for sm_100a, loads, and exports
every symbol include/dda.h declares; the product package has no CPU fallback
and shares no code with the oracle.  No compute calls (no GPU here)."""
import os
import re
import subprocess

import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
PKG = os.path.join(ROOT, "paper_conf_ipps_xiaohmxw17_b200")


def _header_symbols():
    txt = open(os.path.join(ROOT, "include", "dda.h")).read()
    return sorted(set(re.findall(r"\b(dda_[a-z_]+)\s*\(", txt)))


@pytest.fixture(scope="module")
def built():
    import __graft_entry__
    __graft_entry__.build()
    import paper_conf_ipps_xiaohmxw17_b200 as dda
    return dda


def test_header_symbols_exported(built):
    syms = _header_symbols()
    assert len(syms) >= 12
    L = built.lib()
    for s in syms:
        assert hasattr(L, s), s
    assert set(syms) == set(built.ABI_SYMBOLS)
    out = subprocess.check_output(["nm", "-D", "--defined-only", built.LIB_PATH]).decode()
    for s in syms:
        assert re.search(rf" T {s}$", out, re.M), s


def test_library_is_sm100a(built):
    out = subprocess.check_output(["cuobjdump", "--list-elf", built.LIB_PATH]).decode()
    assert "sm_100a" in out


def test_256bit_loads_in_sass(built):
    # the BSR6 chunk loads are single 256-bit LDGs (ld.global.nc.v4.f64)
    sass = subprocess.check_output(["cuobjdump", "-sass", built.LIB_PATH]).decode()
    assert re.search(r"LDG\.E\S*\.256", sass)


def test_status_strings_without_gpu(built):
    L = built.lib()
    assert L.dda_status_string(0) == b"DDA_OK"
    assert L.dda_status_string(6) == b"DDA_ERR_NO_CONVERGENCE"


def test_no_oracle_in_product_and_vice_versa():
    for dirpath, _, files in os.walk(PKG):
        for f in files:
            if f.endswith((".py", ".cu", ".cuh", ".h")):
                txt = open(os.path.join(dirpath, f)).read()
                for bad in ("import oracle", "from oracle", "orc_", "liboracle", "oracle.c"):
                    assert bad not in txt, (f, bad)
    for f in os.listdir(os.path.join(ROOT, "oracle")):
        if f.endswith((".py", ".c", ".h")):
            txt = open(os.path.join(ROOT, "oracle", f)).read()
            for bad in ("import paper_conf", "from paper_conf", "libdda", "dda.h", "#include \"", "dda_"):
                assert bad not in txt, (f, bad)


def test_synth_has_no_method_arithmetic():
    txt = open(os.path.join(ROOT, "synth", "slope.py")).read()
    assert "import oracle" not in txt and "paper_conf_ipps_xiaohmxw17_b200" not in txt


def test_missing_library_fails_loudly(tmp_path, monkeypatch):
    import paper_conf_ipps_xiaohmxw17_b200 as dda
    monkeypatch.setattr(dda, "LIB_PATH", str(tmp_path / "nope.so"))
    monkeypatch.setattr(dda, "_lib", None)
    with pytest.raises(ImportError):
        dda.lib()
