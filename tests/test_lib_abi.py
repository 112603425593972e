"""The C-ABI library loads (no GPU needed) and exports every entry point
include/betty.h declares; the Python binding declares the same names."""
import ctypes
import os
import re
import subprocess

import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
HEADER = os.path.join(ROOT, "include", "betty.h")


def declared():
    src = open(HEADER).read()
    src = re.sub(r"/\*.*?\*/", "", src, flags=re.S)
    return sorted(set(re.findall(r"\b(betty_[a-z0-9_]+)\s*\(", src)))


def test_header_declares_the_boundary():
    names = declared()
    for must in ["betty_reg_build", "betty_extract_blocks", "betty_sage_fwd", "betty_sage_bwd", "betty_step",
                 "betty_plan_create", "betty_adam"]:
        assert must in names


def test_library_exports_every_symbol():
    from paper_conf_asplos_yangzd023_b200 import _lib
    assert os.path.exists(_lib.LIB_PATH), "libbetty.so missing: run __graft_entry__.build()"
    L = ctypes.CDLL(_lib.LIB_PATH)
    for name in declared():
        assert hasattr(L, name), name
    out = subprocess.run(["nm", "-D", "--defined-only", _lib.LIB_PATH], capture_output=True, text=True).stdout
    exported = set(re.findall(r"\bT (betty_[a-z0-9_]+)", out))
    assert set(declared()) <= exported
    assert set(_lib.EXPORTED) == set(declared())


def test_binding_loads_and_reports_version():
    import paper_conf_asplos_yangzd023_b200 as B
    assert "sm_100a" in B.betty_version()


def test_binding_has_no_fallback(monkeypatch, tmp_path):
    from paper_conf_asplos_yangzd023_b200 import _lib
    monkeypatch.setattr(_lib, "LIB_PATH", str(tmp_path / "missing.so"))
    monkeypatch.setattr(_lib, "_lib", None)
    with pytest.raises(RuntimeError, match="no fallback"):
        _lib.lib()
