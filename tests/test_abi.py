"""CPU-side checks of the boundary: the C-ABI library builds for sm_100a, loads, and
exports every symbol include/bgpq.h declares; without a GPU it fails loudly (no CPU
fallback).  No compute calls are made here."""
import ctypes
import os
import re

import pytest

import paper_conf_icpp_chenhjz21_b200 as pkg

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def _declared_functions(header="bgpq.h"):
    src = open(os.path.join(ROOT, "include", header)).read()
    src = re.sub(r"/\*.*?\*/", "", src, flags=re.S)
    return sorted(set(re.findall(r"\b(bgpq_[a-z_]+)\s*\(", src)))


def test_library_builds_and_exports_header_symbols():
    path = pkg.build()
    L = ctypes.CDLL(path)
    declared = _declared_functions()
    assert len(declared) >= 15
    missing = [f for f in declared if not hasattr(L, f)]
    assert not missing, missing
    assert set(declared) == set(pkg.EXPORTS)
    apps_declared = _declared_functions("bgpq_apps.h")
    assert set(apps_declared) == set(pkg.APP_EXPORTS)
    assert not [f for f in apps_declared if not hasattr(L, f)]


def test_library_is_sm100a():
    import subprocess
    out = subprocess.run(["cuobjdump", "--list-elf", pkg.build()], capture_output=True, text=True).stdout
    assert "sm_100a" in out


def test_sass_uses_bulk_copy_and_acquire_cas():
    import subprocess
    sass = subprocess.run(["cuobjdump", "-sass", pkg.build()], capture_output=True, text=True).stdout
    assert "UBLKCP" in sass          # cp.async.bulk (TMA bulk copy engine)
    assert "ATOMG" in sass or "ATOM" in sass
    assert "SHFL.BFLY" in sass       # __shfl_xor_sync bitonic sort


def test_no_gpu_fails_loudly():
    torch = pytest.importorskip("torch")
    if torch.cuda.is_available():
        pytest.skip("GPU present")
    with pytest.raises(pkg.BGPQError):
        pkg.BGPQ(capacity=1024, K=64)
    assert pkg.lib().bgpq_last_error() == pkg.BGPQ_ECUDA


def test_invalid_K_rejected():
    with pytest.raises(ValueError):
        pkg.BGPQ(capacity=1024, K=100)
    h = pkg.lib().bgpq_create_ex(1024, 100, 0)
    assert not h and pkg.lib().bgpq_last_error() == pkg.BGPQ_EINVAL


def test_strerror():
    assert b"capacity" in pkg.lib().bgpq_strerror(pkg.BGPQ_EFULL)


def test_product_does_not_import_oracle():
    pdir = os.path.join(ROOT, "paper_conf_icpp_chenhjz21_b200")
    for dirpath, _, files in os.walk(pdir):
        for f in files:
            if f.endswith((".py", ".cu", ".cuh", ".h", ".cpp")):
                txt = open(os.path.join(dirpath, f)).read()
                assert "import oracle" not in txt and "from oracle" not in txt
                assert "bgpq_oracle" not in txt and "liboracle" not in txt
