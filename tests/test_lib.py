"""CPU-side checks of the C ABI boundary: libdts.so builds for sm_100a, loads,
and exports every function include/dts.h declares.  No compute call is made
here (there is no GPU in the CPU suite)."""
import ctypes
import os
import re
import subprocess

import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


@pytest.fixture(scope="module")
def lib():
    from paper_conf_ipps_gowanlockc15_b200 import build
    path = build.build()
    return ctypes.CDLL(path), path


def declared_functions():
    src = open(os.path.join(ROOT, "include", "dts.h")).read()
    src = re.sub(r"/\*.*?\*/", "", src, flags=re.S)
    return sorted(set(re.findall(r"\b(dts_[a-z_]+)\s*\(", src)))


def test_header_declares_the_boundary():
    names = declared_functions()
    for required in ("dts_build_index", "dts_search", "dts_free_results", "dts_free_index",
                     "dts_last_error"):
        assert required in names


def test_every_declared_symbol_is_exported(lib):
    cdll, path = lib
    for name in declared_functions():
        assert hasattr(cdll, name), f"{name} declared in dts.h but not exported by {path}"
    import paper_conf_ipps_gowanlockc15_b200 as dts
    assert set(dts.EXPORTED_SYMBOLS) == set(declared_functions())


def test_exports_are_extern_c(lib):
    _, path = lib
    out = subprocess.run(["nm", "-D", "--defined-only", path], capture_output=True, text=True).stdout
    exported = set(re.findall(r"\bT (dts_\w+)", out))
    assert set(declared_functions()) <= exported


def test_cubin_is_sm100a(lib):
    _, path = lib
    out = subprocess.run(["/usr/local/cuda/bin/cuobjdump", "--list-elf", path],
                         capture_output=True, text=True).stdout
    assert "sm_100a" in out


def test_version_and_error_string_without_gpu(lib):
    import paper_conf_ipps_gowanlockc15_b200 as dts
    lib_ = dts.load()
    assert b"sm_100a" in lib_.dts_version()
    assert lib_.dts_last_error() is not None


def test_binding_refuses_without_library(tmp_path, monkeypatch):
    import paper_conf_ipps_gowanlockc15_b200 as dts
    monkeypatch.setattr(dts, "_LIB_PATH", str(tmp_path / "missing.so"))
    monkeypatch.setattr(dts, "_lib", None)
    with pytest.raises(ImportError):
        dts.load()


def test_product_package_does_not_import_oracle():
    pkg = os.path.join(ROOT, "paper_conf_ipps_gowanlockc15_b200")
    for dirpath, _, files in os.walk(pkg):
        for f in files:
            if f.endswith((".py", ".cu", ".cuh", ".h", ".cpp")):
                txt = open(os.path.join(dirpath, f)).read()
                assert not re.search(r"^\s*(import|from)\s+oracle", txt, flags=re.M), f
                assert not re.search(r"#include\s*[<\"].*oracle", txt), f
                assert "liboracle" not in txt, f
