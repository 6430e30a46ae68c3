"""CPU-side checks of the C-ABI boundary (no compute calls: no GPU here).

* libksel.so loads and exports every symbol include/ksel.h declares;
* argument validation happens on the host, before any device call, with the
  documented status codes;
* the product package never imports or references the oracle.
"""
import ctypes
import os
import re
import subprocess
import sys

import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
HEADER = os.path.join(ROOT, "include", "ksel.h")
PKG = os.path.join(ROOT, "paper_conf_ipps_tang0emg15_b200")


def _declared():
    txt = open(HEADER).read()
    return sorted(set(re.findall(r"KSEL_API\s+[\w\s\*]+?\b(\w+)\s*\(", txt)))


@pytest.fixture(scope="module")
def lib():
    from paper_conf_ipps_tang0emg15_b200 import build
    path = build.build()
    return ctypes.CDLL(path)


def test_header_declares_entry_points():
    names = _declared()
    for n in ("ksel_select", "ksel_merge", "knn_search", "ksel_strerror", "ksel_select_host"):
        assert n in names


def test_exports_every_declared_symbol(lib):
    for name in _declared():
        assert hasattr(lib, name), name
    # and nothing else leaks from the C++ implementation (hidden visibility)
    out = subprocess.run(["nm", "-D", "--defined-only", os.path.join(PKG, "libksel.so")],
                         capture_output=True, text=True).stdout
    exported = {l.split()[-1] for l in out.splitlines() if " T " in l}
    assert set(_declared()) <= exported
    assert not [s for s in exported if s.startswith("_ZN4ksel")]


def test_binding_export_list_matches_header():
    import paper_conf_ipps_tang0emg15_b200 as k
    assert sorted(k.EXPORTS) == _declared()


def test_strerror_and_version(lib):
    lib.ksel_strerror.restype = ctypes.c_char_p
    for s in range(0, 6):
        assert lib.ksel_strerror(s)
    assert lib.ksel_version() >= 100


def test_select_argument_validation_is_host_side(lib):
    f = lib.ksel_select
    p, i64, i32 = ctypes.c_void_p, ctypes.c_int64, ctypes.c_int
    f.argtypes = [p, i64, i64, i32, p, p, p]
    A, B, C = 1 << 20, 2 << 20, 3 << 20  # fake, never dereferenced
    assert f(None, 4, 100, 5, B, C, None) == 1          # null
    assert f(A, 0, 100, 5, B, C, None) == 1             # Q < 1
    assert f(A, 4, 0, 1, B, C, None) == 1               # N < 1
    assert f(A, 4, 100, 0, B, C, None) == 1             # k < 1
    assert f(A, 4, 100, 101, B, C, None) == 1           # k > N
    assert f(A + 2, 4, 100, 5, B, C, None) == 1         # misaligned
    assert f(A, 4, 1 << 31, 5, B, C, None) == 1         # N >= 2^31
    assert f(A, 4, 5000, 1025, B, C, None) == 2         # k > 1024: unsupported
    assert f(A, 4, 100, 5, A + 64, C, None) == 1        # out overlaps input


def test_merge_argument_validation_is_host_side(lib):
    f = lib.ksel_merge
    p, i64, i32 = ctypes.c_void_p, ctypes.c_int64, ctypes.c_int
    f.argtypes = [p, p, i64, i32, i32, i32, p, p, p]
    A, B, C, D = 1 << 20, 2 << 20, 3 << 20, 4 << 20
    assert f(A, B, 8, 0, 4, 4, C, D, None) == 1         # S < 1
    assert f(A, B, 8, 2, 4, 9, C, D, None) == 1         # k > S*kin
    assert f(A, B, 8, 2, 2000, 4, C, D, None) == 2      # kin > 1024
    assert f(None, B, 8, 2, 4, 4, C, D, None) == 1


def test_product_path_does_not_touch_oracle():
    for dirpath, _, files in os.walk(PKG):
        for fn in files:
            if fn.endswith((".py", ".cu", ".cuh", ".h", ".cpp")):
                txt = open(os.path.join(dirpath, fn)).read()
                assert "import oracle" not in txt and "from oracle" not in txt, fn
                assert "ksel_oracle" not in txt and "liboracle" not in txt, fn
    code = ("import sys; import paper_conf_ipps_tang0emg15_b200 as k; "
            "assert 'oracle' not in sys.modules; print('ok')")
    r = subprocess.run([sys.executable, "-c", code], cwd=ROOT, capture_output=True, text=True)
    assert r.returncode == 0 and "ok" in r.stdout, r.stderr


def test_package_fails_loudly_without_library(tmp_path):
    # copy the binding without the .so: import must raise, never fall back
    import shutil
    dst = tmp_path / "paper_conf_ipps_tang0emg15_b200"
    dst.mkdir()
    shutil.copy(os.path.join(PKG, "__init__.py"), dst / "__init__.py")
    r = subprocess.run([sys.executable, "-c", "import paper_conf_ipps_tang0emg15_b200"],
                       cwd=str(tmp_path), capture_output=True, text=True)
    assert r.returncode != 0 and "libksel.so is not built" in r.stderr
