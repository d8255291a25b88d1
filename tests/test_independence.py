"""The oracle and the CUDA path share no code (tier rule ③): neither side's sources name the
other, libsr.so does not link liboracle.so, and the binding fails loudly without libsr.so."""
import os
import re
import subprocess
import sys

import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
PKG = os.path.join(ROOT, "paper_conf_ppopp_jiangha20_b200")
ORACLE = os.path.join(ROOT, "oracle")


def _sources(d, exts):
    for dp, _, fs in os.walk(d):
        for f in fs:
            if f.endswith(exts):
                yield os.path.join(dp, f)


def test_product_sources_do_not_name_the_oracle():
    # code references only (imports, includes, library loads); comments may say "shares nothing"
    pat = re.compile(r"^\s*(import\s+oracle|from\s+oracle|#\s*include\s*[<\"].*oracle)|liboracle|"
                     r"CDLL\(.*oracle|sys\.path.*oracle")
    for p in list(_sources(PKG, (".py", ".cu", ".cpp", ".h"))) + list(_sources(os.path.join(ROOT, "include"), (".h",))):
        for i, line in enumerate(open(p, encoding="utf-8"), 1):
            assert not pat.search(line), f"{p}:{i} references the oracle: {line.strip()}"


def test_oracle_sources_do_not_name_the_product():
    pat = re.compile(r"^\s*(import\s+paper_conf|from\s+paper_conf|#\s*include\s*[<\"].*(sr\.h|internal\.h))|"
                     r"libsr\.so|CDLL\(.*sr")
    for p in _sources(ORACLE, (".py", ".cpp", ".c", ".h")):
        for i, line in enumerate(open(p, encoding="utf-8"), 1):
            assert not pat.search(line), f"{p}:{i} references the CUDA path: {line.strip()}"


def test_libsr_does_not_link_the_oracle():
    so = os.path.join(PKG, "libsr.so")
    if not os.path.exists(so):
        pytest.skip("libsr.so not built")
    out = subprocess.run(["ldd", so], capture_output=True, text=True).stdout
    assert "oracle" not in out


def test_binding_fails_loudly_without_libsr(tmp_path):
    # a copy of the binding's Python files without libsr.so must raise, not fall back
    import shutil
    dst = tmp_path / "paper_conf_ppopp_jiangha20_b200"
    dst.mkdir()
    for f in os.listdir(PKG):
        if f.endswith(".py"):
            shutil.copy(os.path.join(PKG, f), dst / f)
    code = "import paper_conf_ppopp_jiangha20_b200 as m; m.lib()"
    r = subprocess.run([sys.executable, "-c", code], cwd=tmp_path, capture_output=True, text=True)
    assert r.returncode != 0 and "libsr.so is missing" in r.stderr
