"""The C-ABI library loads and exports every symbol include/hsort.h declares (CPU, no compute)."""
import os
import re
import subprocess

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
HEADER = os.path.join(ROOT, "include", "hsort.h")


def declared_functions():
    src = open(HEADER).read()
    src = re.sub(r"/\*.*?\*/", "", src, flags=re.S)
    return sorted(set(re.findall(r"\b(hsort_[a-z0-9_]+)\s*\(", src)))


def test_header_declares_the_boundary():
    names = declared_functions()
    for must in ["hsort_init", "hsort_sort", "hsort_finalize", "hsort_sort_device",
                 "hsort_device_merge", "hsort_host_merge", "hsort_plan"]:
        assert must in names


def test_library_exports_every_declared_symbol(hs):
    out = subprocess.run(["nm", "-D", "--defined-only", hs.LIB_PATH], capture_output=True,
                         text=True).stdout
    exported = set(re.findall(r"\b[TW] (hsort_[a-z0-9_]+)$", out, flags=re.M))
    missing = [n for n in declared_functions() if n not in exported]
    assert not missing, missing


def test_binding_covers_every_declared_symbol(hs):
    assert set(declared_functions()) == set(hs.SIGNATURES)
    for name in hs.SIGNATURES:
        assert callable(getattr(hs.lib(), name))
        assert hasattr(hs, name), name


def test_library_is_sm100a(hs):
    out = subprocess.run(["cuobjdump", "--list-elf", hs.LIB_PATH], capture_output=True, text=True)
    assert "sm_100a" in out.stdout


def test_product_package_does_not_touch_the_oracle():
    pkg = os.path.join(ROOT, "paper_conf_ipps_gowanlockk18a_b200")
    for dirpath, _, files in os.walk(pkg):
        for f in files:
            if f.endswith((".py", ".cpp", ".cu", ".h")) or f == "Makefile":
                text = open(os.path.join(dirpath, f), errors="ignore").read().lower()
                assert "import oracle" not in text and "liboracle" not in text, f
                assert "oracle_" not in text, f
