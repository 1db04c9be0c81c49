"""Host-side checks of the C-ABI library (no GPU needed): it builds, loads, and exports
every entry point include/neo.h declares; the Python binding names match."""
import ctypes
import os
import re

from paper_conf_isca_jiaodwfcm0z25_b200 import build as nbuild
from paper_conf_isca_jiaodwfcm0z25_b200 import neo

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def _declared():
    src = open(os.path.join(ROOT, "include", "neo.h")).read()
    src = re.sub(r"/\*.*?\*/", "", src, flags=re.S)
    return sorted(set(re.findall(r"\b(neo_[a-z_0-9]+)\s*\(", src)))


def test_library_exports_every_declared_symbol():
    path = nbuild.build()
    lib = ctypes.CDLL(path)
    declared = _declared()
    assert len(declared) >= 17
    for name in declared:
        assert hasattr(lib, name), name


def test_binding_covers_header():
    assert sorted(neo.EXPORTED) == _declared()


def test_no_oracle_in_product_path():
    """The product package never references the oracle (it must fail loudly, not fall back)."""
    pkg = os.path.join(ROOT, "paper_conf_isca_jiaodwfcm0z25_b200")
    for dirpath, _, files in os.walk(pkg):
        for f in files:
            if f.endswith((".py", ".cu", ".cuh", ".h", ".cpp")):
                text = open(os.path.join(dirpath, f)).read()
                assert not re.search(r"(^|\n)\s*(from|import)\s+oracle|liboracle|oracle_core", text), f


def test_sass_uses_sm100a():
    """The fatbin carries sm_100a SASS (cuobjdump lists the arch)."""
    import subprocess
    out = subprocess.run(["/usr/local/cuda/bin/cuobjdump", "--list-elf", nbuild.build()],
                         capture_output=True, text=True).stdout
    assert "sm_100a" in out
