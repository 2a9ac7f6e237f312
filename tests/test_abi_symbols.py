"""CPU-side checks of the boundary: libvpic.so builds for sm_100a, loads
without a GPU, and exports every function include/vpic.h declares; the
binding mirrors the same names; the product package never imports oracle/."""
import ast
import ctypes
import os
import re
import subprocess

import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
HEADER = os.path.join(ROOT, "include", "vpic.h")
PKG = os.path.join(ROOT, "paper_conf_sc_tanlta25_b200")


def declared_functions():
    src = open(HEADER).read()
    src = re.sub(r"/\*.*?\*/", "", src, flags=re.S)
    names = re.findall(r"^\s*(?:const\s+)?[a-z_0-9]+\s*\**\s*(vpic_[a-z_0-9]+)\s*\(", src, flags=re.M)
    return sorted(set(names))


@pytest.fixture(scope="module")
def lib():
    from paper_conf_sc_tanlta25_b200 import _build
    path = _build.build()
    return ctypes.CDLL(path), path


def test_header_declares_the_five_calls():
    names = declared_functions()
    for n in ["vpic_sort_particles", "vpic_load_interpolator", "vpic_advance_p",
              "vpic_unload_accumulator", "vpic_migrate_particles"]:
        assert n in names


def test_exports_every_declared_symbol(lib):
    so, path = lib
    out = subprocess.run(["nm", "-D", "--defined-only", path], capture_output=True, text=True).stdout
    exported = set(re.findall(r" T (vpic_\w+)", out))
    for n in declared_functions():
        assert n in exported, n
        assert hasattr(so, n)


def test_binding_names_match_header():
    from paper_conf_sc_tanlta25_b200 import vpic
    assert sorted(vpic.EXPORTS) == declared_functions()
    for n in declared_functions():
        if n.startswith("vpic_ctx_"):
            continue  # methods of vpic.Context
        assert hasattr(vpic, n) or n in ("vpic_status_string",), n


def test_sm100a_sass(lib):
    _, path = lib
    out = subprocess.run(["cuobjdump", "--list-elf", path], capture_output=True, text=True).stdout
    assert "sm_100a" in out
    assert "sm_90" not in out


def test_status_string_without_gpu(lib):
    so, _ = lib
    so.vpic_status_string.restype = ctypes.c_char_p
    assert so.vpic_status_string(0) == b"ok"
    assert so.vpic_status_string(-5).startswith(b"unsupported")


def test_ctx_create_fails_loudly_without_gpu(lib):
    """No GPU here: the product refuses (no CPU fallback)."""
    import torch
    if torch.cuda.is_available():
        pytest.skip("GPU present")
    from paper_conf_sc_tanlta25_b200 import inputs, vpic
    with pytest.raises(Exception):
        vpic.Context(inputs.GridSpec(4, 4, 4), device=0)


def test_product_does_not_import_oracle():
    for dirpath, _, files in os.walk(PKG):
        for f in files:
            if f.endswith(".py"):
                tree = ast.parse(open(os.path.join(dirpath, f)).read())
                for node in ast.walk(tree):
                    if isinstance(node, ast.Import):
                        assert not any(a.name.split(".")[0] == "oracle" for a in node.names), f
                    if isinstance(node, ast.ImportFrom):
                        assert (node.module or "").split(".")[0] != "oracle", f
            if f.endswith((".cu", ".cuh", ".h", ".cpp")):
                assert "vpic_oracle" not in open(os.path.join(dirpath, f)).read(), f
