"""The C-ABI libraries load and export every symbol include/deepum_b200.h and
include/deepum_hook.h declare (no compute calls: CPU only)."""
import ctypes
import os
import re

import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
HDR = os.path.join(ROOT, "include", "deepum_b200.h")
HOOK_HDR = os.path.join(ROOT, "include", "deepum_hook.h")


def _declared(hdr=HDR):
    txt = open(hdr).read()
    txt = re.sub(r"/\*.*?\*/", "", txt, flags=re.S)
    return sorted(set(re.findall(r"\b(dum_[a-z_0-9]+)\s*\(", txt)))


def test_header_declares_the_five_calls():
    names = _declared()
    for n in ("dum_record_faults", "dum_build_tables", "dum_predict_prefetch", "dum_select_evictions",
              "dum_migrate_blocks"):
        assert n in names


def test_library_exports_every_declared_symbol():
    from paper_conf_asplos_jungkl23_b200 import build as bld
    so = bld.build()
    lib = ctypes.CDLL(so)
    missing = [n for n in _declared() if not hasattr(lib, n)]
    assert not missing, missing


def test_hook_library_exports_every_declared_symbol():
    from paper_conf_asplos_jungkl23_b200 import build as bld
    bld.build()
    import torch  # noqa: F401  (libc10 / libc10_cuda)
    lib = ctypes.CDLL(bld.build_hook())
    names = _declared(HOOK_HDR)
    assert "dum_hook_flush" in names
    missing = [n for n in names if not hasattr(lib, n)]
    assert not missing, missing


def test_binding_refuses_without_library(tmp_path, monkeypatch):
    from paper_conf_asplos_jungkl23_b200 import binding
    monkeypatch.setattr(binding, "_LIBPATH", str(tmp_path / "missing.so"))
    monkeypatch.setattr(binding, "_LIB", None)
    with pytest.raises(ImportError):
        binding.load_library()
