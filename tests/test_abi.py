"""The C-ABI library loads on a GPU-less host and exports every symbol include/*.h declares.

No compute call is made here (there is no GPU); calls that need no device are
exercised: error strings, the not-initialised state, argument validation that
happens before any CUDA call.
"""
import ctypes
import os
import re

import pytest

import paper_conf_isca_muthukrishnannl21_b200 as proact
from paper_conf_isca_muthukrishnannl21_b200 import _lib

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
HEADERS = ["proact.h", "proact_workloads.h"]


def _declared():
    names = set()
    for h in HEADERS:
        src = open(os.path.join(ROOT, "include", h)).read()
        src = re.sub(r"/\*.*?\*/", "", src, flags=re.S)
        for m in re.finditer(r"^\s*(?:[A-Za-z_][\w\s\*]*?)\b(proact_\w+)\s*\(", src, flags=re.M):
            names.add(m.group(1))
    return names


def test_every_declared_symbol_is_exported():
    L = proact.load()
    names = _declared()
    assert len(names) >= 25, names
    for n in sorted(names):
        assert hasattr(L, n), f"libproact.so does not export {n}"
    # and the binding declares a signature for every one of them
    missing = names - set(_lib.EXPORTED)
    assert not missing, f"binding lacks signatures for {sorted(missing)}"


def test_error_strings_and_uninitialised_state():
    L = proact.load()
    for code, name in [(0, b"PROACT_OK"), (-1, b"PROACT_ERR_INVALID"), (-5, b"PROACT_ERR_TIMEOUT"),
                       (-6, b"PROACT_ERR_PROTOCOL"), (-99, b"PROACT_ERR_UNKNOWN")]:
        assert L.proact_error_string(code) == name
    assert L.proact_rank() == -1 and L.proact_world() == 0
    assert L.proact_finalize() == _lib.ERR_STATE
    assert L.proact_phase_sync(None, 0) == _lib.ERR_STATE
    assert L.proact_check() == _lib.ERR_STATE
    assert L.proact_register_region(None, 0, 4096, 1) == _lib.ERR_STATE
    # argument validation before any CUDA call
    assert L.proact_init_ex(0, 0, b"x") == _lib.ERR_INVALID
    assert L.proact_init_ex(17, 0, b"x") == _lib.ERR_INVALID
    assert L.proact_init_ex(2, 2, b"x") == _lib.ERR_INVALID


def test_binding_fails_loudly_without_library(monkeypatch, tmp_path):
    monkeypatch.setattr(_lib, "_lib", None)
    monkeypatch.setattr(_lib, "LIB_PATH", str(tmp_path / "missing.so"))
    with pytest.raises(ImportError):
        _lib.load()


def test_struct_layouts_match_header():
    # proact_config: 10 x 4-byte fields; proact_region_info: see include/proact.h
    assert ctypes.sizeof(_lib.Config) == 40
    assert ctypes.sizeof(_lib.RegionInfo) == 8 + 8 * 4 + 4 * 4 + 8 + 8 * (_lib.MAX_RANKS + 1)
