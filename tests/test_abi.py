"""CPU-side checks of the boundary: the C-ABI library builds, loads without a
GPU and exports every symbol include/proteus.h declares; the binding refuses
to run without it (no fallback)."""

import ctypes
import os
import re

import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def _declared():
    src = open(os.path.join(ROOT, "include", "proteus.h")).read()
    src = re.sub(r"/\*.*?\*/", "", src, flags=re.S)
    return sorted(set(re.findall(r"\b(proteus_[a-z_]+)\s*\(", src)))


def test_header_declares_the_path():
    names = _declared()
    for must in ("proteus_load_profiles", "proteus_solve", "proteus_replay"):
        assert must in names


def test_library_exports_every_declared_symbol():
    from paper_conf_asplos_ahmadgfwsw24_b200 import build
    lib = ctypes.CDLL(build.build())
    for name in _declared():
        assert hasattr(lib, name), name
    from paper_conf_asplos_ahmadgfwsw24_b200 import _native
    assert set(_native.EXPORTED) == set(_declared())
    assert lib.proteus_abi_version() == _native.ABI_VERSION == 3


def test_create_without_gpu_fails_cleanly():
    import torch
    if torch.cuda.is_available():
        pytest.skip("a GPU is present")
    from paper_conf_asplos_ahmadgfwsw24_b200 import Proteus, ProteusError
    with pytest.raises(ProteusError):
        Proteus(0)


def test_binding_has_no_fallback(tmp_path):
    from paper_conf_asplos_ahmadgfwsw24_b200 import _native
    with pytest.raises(ImportError):
        saved = _native._lib
        _native._lib = None
        try:
            _native.load(str(tmp_path / "missing.so"))
        finally:
            _native._lib = saved


def test_product_package_does_not_import_oracle():
    pkg = os.path.join(ROOT, "paper_conf_asplos_ahmadgfwsw24_b200")
    for dirpath, _, files in os.walk(pkg):
        for f in files:
            if f.endswith((".py", ".cu", ".cuh", ".h")):
                txt = open(os.path.join(dirpath, f)).read()
                assert not re.search(r"^\s*(import|from)\s+oracle", txt, re.M), f
                assert "liboracle" not in txt and "oracle.c" not in txt, f
