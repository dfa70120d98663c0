"""CPU checks of the boundary: the C-ABI library builds, loads and exports every
symbol include/ad.h declares; the binding mirrors the header; the product
package never touches the oracle (no shared code, no fallback)."""
import ctypes
import os
import re
import subprocess

import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
HEADER = os.path.join(ROOT, "include", "ad.h")
PKG = os.path.join(ROOT, "paper_conf_sc_solis_vasquezts25_b200")


def _declared():
    src = open(HEADER).read()
    src = re.sub(r"/\*.*?\*/", "", src, flags=re.S)
    return sorted(set(re.findall(r"^\s*(?:const\s+)?\w+\s*\*?\s*(ad_\w+)\s*\(", src, flags=re.M)))


@pytest.fixture(scope="module")
def libad():
    from paper_conf_sc_solis_vasquezts25_b200 import build
    path = build.build()
    return ctypes.CDLL(path), path


def test_header_declares_the_north_star_entry_points():
    names = _declared()
    for n in ("ad_upload_grids", "ad_upload_ligand", "ad_score_poses", "ad_local_search"):
        assert n in names


def test_library_exports_every_declared_symbol(libad):
    lib, path = libad
    out = subprocess.check_output(["nm", "-D", "--defined-only", path], text=True)
    exported = set(re.findall(r"\bT (ad_\w+)", out))
    for n in _declared():
        assert n in exported, n
        getattr(lib, n)


def test_binding_mirrors_header():
    from paper_conf_sc_solis_vasquezts25_b200 import ad
    assert sorted(ad.EXPORTS) == _declared()


def test_library_is_sm100a(libad):
    _, path = libad
    out = subprocess.check_output(["cuobjdump", "--list-elf", path], text=True)
    assert "sm_100a" in out


def test_host_only_calls_without_gpu(libad):
    lib, _ = libad
    lib.ad_version.restype = ctypes.c_int32
    assert lib.ad_version() == 1
    lib.ad_last_error.restype = ctypes.c_char_p
    h = ctypes.c_void_p()
    rc = lib.ad_context_create(0, ctypes.byref(h))
    import torch
    if not torch.cuda.is_available():
        assert rc in (-1, -3) and not h.value          # error code, no crash, no handle
        assert lib.ad_last_error()
    else:
        assert rc == 0
        lib.ad_context_destroy(h)
    assert lib.ad_context_destroy(None) == 0
    assert lib.ad_context_create(0, None) == -1       # null out pointer


def test_product_code_never_touches_the_oracle():
    for dirpath, _, files in os.walk(PKG):
        for f in files:
            if f.endswith((".py", ".cu", ".cuh", ".h", ".cpp")):
                src = open(os.path.join(dirpath, f)).read()
                assert not re.search(r"(from|import)\s+oracle|libad_oracle|ad_oracle\.|\bado_", src), \
                    f"{f} imports/links the oracle"


def test_oracle_header_marks_test_infrastructure():
    src = open(os.path.join(ROOT, "oracle", "ad_oracle.c")).read()
    assert "TEST INFRASTRUCTURE ONLY" in src
