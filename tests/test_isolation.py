"""The product path and the oracle share no code: the package never imports oracle/, the
library is not linked against the oracle, and the oracle never includes product headers."""
import glob
import os
import re
import subprocess
import sys

from conftest import ROOT

PKG = os.path.join(ROOT, "paper_conf_ipps_sundaramrc09_b200")


def test_product_sources_never_reference_oracle():
    pat = re.compile(r"(^\s*(import|from)\s+oracle\b|#\s*include\s*[<\"].*oracle|liboracle|\borc_\w+\s*\()", re.M)
    for path in glob.glob(os.path.join(PKG, "**", "*.*"), recursive=True):
        if path.endswith((".py", ".cu", ".cpp", ".h", ".cuh")):
            assert not pat.search(open(path, errors="ignore").read()), path


def test_oracle_never_includes_product():
    for path in glob.glob(os.path.join(ROOT, "oracle", "*.*")):
        if path.endswith((".c", ".h", ".py")):
            src = open(path).read()
            assert not re.search(r"^\s*(import|from)\s+paper_conf_ipps_sundaramrc09_b200", src, re.M), path
            assert not re.search(r"#\s*include\s*[<\"].*(tg\.h|tg_internal|kernels\.h)", src), path


def test_importing_package_does_not_load_oracle():
    code = ("import sys; sys.path.insert(0, %r); import paper_conf_ipps_sundaramrc09_b200 as p; "
            "print(any(m == 'oracle' or m.startswith('oracle.') for m in sys.modules))" % ROOT)
    out = subprocess.check_output([sys.executable, "-c", code], text=True).strip()
    assert out == "False"


def test_library_not_linked_to_oracle():
    lib = os.path.join(PKG, "libtg.so")
    out = subprocess.check_output(["nm", "-D", "--defined-only", lib], text=True)
    assert "orc_" not in out
