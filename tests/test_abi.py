"""CPU-side checks of the C-ABI library: it builds for sm_100a, loads, and
exports every symbol include/bf.h declares.  No compute calls (no GPU here)."""
from __future__ import annotations

import os
import re
import subprocess

import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def _declared_symbols():
    src = open(os.path.join(ROOT, "include", "bf.h")).read()
    src = re.sub(r"/\*.*?\*/", "", src, flags=re.S)
    names = set(re.findall(r"\b(bf_[a-z0-9_]+)\s*\(", src))
    return sorted(n for n in names if not n.endswith("_fn"))


def test_header_declares_the_boundary():
    names = _declared_symbols()
    for n in ("bf_fit", "bf_predict", "bf_oob_importance", "bf_importance_finalize", "bf_pca", "bf_forest_export",
              "bf_forest_import", "bf_forest_free", "bf_last_error", "bf_set_allocator"):
        assert n in names


def test_library_exports_every_declared_symbol():
    from paper_conf_ipps_madougouvln16_b200 import build
    path = build.build()
    out = subprocess.check_output(["nm", "-D", "--defined-only", path]).decode()
    exported = set(re.findall(r" T (bf_[a-z0-9_]+)$", out, flags=re.M))
    missing = [n for n in _declared_symbols() if n not in exported]
    assert not missing, missing


def test_library_loads_and_reports_version():
    import paper_conf_ipps_madougouvln16_b200 as bf
    L = bf.lib()
    assert b"sm_100a" in L.bf_version()
    for n in bf.exported_symbols():
        assert hasattr(L, n)


def test_sass_is_sm100a():
    from paper_conf_ipps_madougouvln16_b200 import build
    path = build.build()
    out = subprocess.check_output(["cuobjdump", "--list-elf", path]).decode()
    assert "sm_100a" in out


def test_params_struct_layout_matches_header():
    import ctypes as C
    import paper_conf_ipps_madougouvln16_b200 as bf
    # int32 x4, int64, uint64, int32 x4 -> 48 bytes, natural alignment
    assert C.sizeof(bf.Params) == 48
    assert C.sizeof(bf.Info) == 64
    assert C.sizeof(bf.Accum) == 48


def test_product_does_not_import_oracle():
    """The product path never imports, links or calls the oracle."""
    pkg = os.path.join(ROOT, "paper_conf_ipps_madougouvln16_b200")
    bad = re.compile(r"^\s*(import\s+oracle|from\s+oracle|from\s+\.\.oracle)|bfo_|libbfo|bfo\.h", re.M)
    for dirpath, _, files in os.walk(pkg):
        for f in files:
            if f.endswith((".py", ".cu", ".cuh", ".h", ".cpp")):
                txt = open(os.path.join(dirpath, f)).read()
                assert not bad.search(txt), f


def test_torch_allocator_hooks_build_and_export():
    """libbf_torch_alloc.so (the bf_set_allocator hooks over torch's CUDA caching allocator) builds against the
    installed torch and exports the two hook functions the binding passes to bf_set_allocator."""
    from paper_conf_ipps_madougouvln16_b200 import build
    path = build.build_torch_alloc()
    out = subprocess.check_output(["nm", "-D", "--defined-only", path]).decode()
    assert re.search(r" T bf_torch_alloc$", out, flags=re.M) and re.search(r" T bf_torch_free$", out, flags=re.M)
    import ctypes as C
    C.CDLL(path)  # resolves libc10_cuda / libc10 through its rpath
