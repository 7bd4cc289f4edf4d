"""CPU-side checks of the C-ABI boundary: the library loads, exports every symbol that
include/*.h declares, and rejects bad arguments before touching the device.  Also checks
the product/oracle separation (no shared code, no oracle import in the product path)."""
import ctypes
import glob
import os
import re

import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
PKG = os.path.join(ROOT, "paper_conf_ipps_dieguezadnm18_b200")


def _declared():
    names = set()
    for h in glob.glob(os.path.join(ROOT, "include", "*.h")):
        src = open(h).read()
        src = re.sub(r"/\*.*?\*/", "", src, flags=re.S)
        for m in re.finditer(r"^\s*(?:const\s+)?[A-Za-z_][A-Za-z0-9_\s\*]*?\b(scan_[a-z0-9_]+)\s*\(", src, re.M):
            names.add(m.group(1))
    return names


def test_library_exports_every_declared_symbol():
    from paper_conf_ipps_dieguezadnm18_b200 import _lib
    declared = _declared()
    assert {"scan_batch", "scan_batch_ex", "scan_shard_totals", "scan_shard_scan"} <= declared
    for name in declared:
        assert hasattr(_lib.lib, name), name
    assert set(_lib.EXPORTS) == declared
    assert _lib.lib.scan_abi_version() == 3


def test_status_strings():
    from paper_conf_ipps_dieguezadnm18_b200 import _lib
    for code, name in _lib.STATUS.items():
        assert _lib.lib.scan_status_string(code).decode() == name


def test_argument_checks_before_any_launch():
    from paper_conf_ipps_dieguezadnm18_b200 import _lib
    L = _lib.lib
    p = ctypes.c_void_p(0x1000)
    # negative sizes
    assert L.scan_batch(p, p, -1, 1, 0, 0, 0, None) == 1
    assert L.scan_batch(p, p, 1, -1, 0, 0, 0, None) == 1
    # bad enums
    assert L.scan_batch(p, p, 10, 1, 7, 0, 0, None) == 1
    assert L.scan_batch(p, p, 10, 1, 0, 9, 0, None) == 1
    assert L.scan_batch(p, p, 10, 1, 0, 0, 5, None) == 1
    assert L.scan_batch_ex(p, p, 10, 1, 0, 0, 0, 99, 0, None, 0, None) == 2
    # empty problems are a successful no-op (no device needed)
    assert L.scan_batch(None, None, 0, 5, 0, 0, 0, None) == 0
    assert L.scan_batch(None, None, 5, 0, 0, 0, 0, None) == 0
    assert L.scan_batch_host(None, None, 0, 0, 0, 0, 0) == 0
    # overflowing N*G
    assert L.scan_batch(p, p, 1 << 40, 1 << 30, 0, 0, 0, None) == 1
    # sharded: bad rank / ngpu
    assert L.scan_shard_scan(p, p, 10, 1, 0, 0, 0, p, 3, 2, None, 0, None) == 1
    assert L.scan_shard_scan(p, p, 10, 1, 0, 0, 0, p, 0, 0, None, 0, None) == 1
    assert L.scan_shard_totals(p, 10, 0, 0, 0, p, None, 0, None) == 0


def test_workspace_sizes_monotone():
    from paper_conf_ipps_dieguezadnm18_b200 import _lib
    L = _lib.lib
    a = L.scan_workspace_bytes(1 << 20, 1, 0, 0, 1, 0)
    b = L.scan_workspace_bytes(1 << 24, 1, 0, 0, 1, 0)
    assert 256 < a < b
    assert L.scan_workspace_bytes(0, 1, 0, 0, 1, 0) == 256
    assert L.scan_shard_workspace_bytes(1 << 20, 4) > 256


def test_product_does_not_touch_oracle():
    # the product path shares no code with oracle/ and never imports it
    for path in glob.glob(os.path.join(PKG, "**", "*"), recursive=True):
        if os.path.isdir(path) or path.endswith((".so", ".pyc", ".o")):
            continue
        src = open(path, errors="ignore").read()
        assert not re.search(r"\boracle\b\s*(import|\.)|import\s+oracle|from\s+oracle|liboracle|oracle_scan",
                             src), path


def test_binding_fails_loudly_without_library(tmp_path, monkeypatch):
    import importlib.util
    spec = importlib.util.spec_from_file_location("_lib_copy", os.path.join(PKG, "_lib.py"))
    mod = importlib.util.module_from_spec(spec)
    monkeypatch.setattr(os.path, "exists", lambda p: False if p.endswith("libscanb200.so") else True)
    with pytest.raises(ImportError):
        spec.loader.exec_module(mod)


def test_lookback_variants_match_library():
    # the binding, the library source and tests/test_gpu_parity.py::test_lookback_variants
    # must agree on which look-back variants exist
    import re
    from paper_conf_ipps_dieguezadnm18_b200 import _lib
    src = open(os.path.join(PKG, "csrc", "scan_lookback.cu")).read()
    body = re.search(r"bool lookback_variant_valid\(int variant\) \{\s*return ([^;]*);", src).group(1)
    valid = tuple(sorted(int(v) for v in re.findall(r"variant == (\d+)", body)))
    assert _lib.LOOKBACK_VARIANTS == valid
    par = open(os.path.join(os.path.dirname(__file__), "test_gpu_parity.py")).read()
    assert '@pytest.mark.parametrize("variant", _lib.LOOKBACK_VARIANTS)\ndef test_lookback_variants' in par


def test_binding_enums_match_header():
    # the ctypes binding's enum tables are the header's values (ops, kinds, algos, statuses)
    from paper_conf_ipps_dieguezadnm18_b200 import _lib
    src = open(os.path.join(ROOT, "include", "scan_b200.h")).read()
    vals = {m.group(1): int(m.group(2)) for m in re.finditer(r"\b(SCAN_[A-Z0-9_]+)\s*=\s*(\d+)", src)}
    assert {k: vals["SCAN_ALGO_" + k.upper()] for k in _lib.ALGOS} == _lib.ALGOS
    assert {k: vals["SCAN_OP_" + k.upper()] for k in _lib.OPS} == _lib.OPS
    assert {k: vals["SCAN_" + k.upper()] for k in _lib.KINDS} == _lib.KINDS
    assert {vals[name]: name for name in _lib.STATUS.values()} == _lib.STATUS
    assert len([k for k in vals if k.startswith("SCAN_ALGO_")]) == len(_lib.ALGOS)
