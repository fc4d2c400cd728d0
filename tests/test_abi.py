"""CPU checks of the C-ABI library: it loads, exports every symbol include/xs.h declares,
validates arguments before touching a device, and has no CPU fallback."""
import ctypes
import os
import re
import subprocess

import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
LIB = os.path.join(ROOT, "paper_conf_cgo_murtovigplls24_b200", "libxs.so")
HEADER = os.path.join(ROOT, "include", "xs.h")


@pytest.fixture(scope="module")
def xs():
    import importlib.util
    # by path: the package's __init__ refuses to import before libxs.so exists
    spec = importlib.util.spec_from_file_location(
        "_xs_build", os.path.join(ROOT, "paper_conf_cgo_murtovigplls24_b200", "build.py"))
    build = importlib.util.module_from_spec(spec)
    spec.loader.exec_module(build)
    build.build()
    import paper_conf_cgo_murtovigplls24_b200 as pkg
    return pkg


def _declared():
    text = open(HEADER).read()
    text = re.sub(r"/\*.*?\*/", "", text, flags=re.S)
    return sorted(set(re.findall(r"\b(xs_[a-z_]+)\s*\(", text)))


def test_header_declares_the_north_star_entry_points():
    names = _declared()
    for n in ("xs_grid_create", "xs_lookup_batch", "xs_grid_destroy", "xs_last_error",
              "xs_lookup_range", "xs_lookup_indices", "xs_grid_checksum"):
        assert n in names


def test_library_exports_every_declared_symbol(xs):
    lib = ctypes.CDLL(LIB)
    for n in _declared():
        assert hasattr(lib, n), n
    out = subprocess.run(["nm", "-D", "--defined-only", LIB], capture_output=True, text=True).stdout
    exported = set(re.findall(r" T (xs_[a-z_]+)$", out, flags=re.M))
    assert set(_declared()) <= exported


def test_library_is_sm100a_only(xs):
    out = subprocess.run(["/usr/local/cuda/bin/cuobjdump", "--list-elf", LIB], capture_output=True, text=True).stdout
    archs = set(re.findall(r"sm_(\d+a?)", out))
    assert archs == {"100a"}, archs


@pytest.mark.parametrize("args,frag", [
    ((100, 1000, 1, 42), "n_nuclides"),
    ((68, 1, 1, 42), "n_gridpoints"),
    ((68, 1000, 7, 42), "grid_type"),
    ((355, 2 ** 30, 1, 42), "2^31"),
])
def test_create_validates_before_device(xs, args, frag):
    with pytest.raises(xs.XSError) as e:
        xs.xs_grid_create(*args)
    assert frag in str(e.value)
    assert frag in xs.xs_last_error()


def test_null_grid_is_einval(xs):
    with pytest.raises(xs.XSError) as e:
        xs.xs_lookup_range(0, 0, 10, 1070)
    assert e.value.code == xs.XS_EINVAL
    xs.xs_grid_destroy(0)  # NULL-safe


def test_no_cpu_fallback_without_gpu(xs):
    import torch
    if torch.cuda.is_available():
        pytest.skip("a GPU is present")
    with pytest.raises(xs.XSError) as e:
        xs.xs_grid_create(68, 1000, 1, 42)
    assert "CUDA" in str(e.value)


def test_binding_fails_loudly_when_library_missing(tmp_path):
    # import the binding from a copy of the package that has no libxs.so
    import shutil
    import sys
    pkg = os.path.join(ROOT, "paper_conf_cgo_murtovigplls24_b200")
    dst = tmp_path / "paper_conf_cgo_murtovigplls24_b200"
    shutil.copytree(pkg, dst, ignore=shutil.ignore_patterns("*.so", "_build", "__pycache__"))
    code = ("import sys; sys.path.insert(0, %r)\n"
            "try:\n import paper_conf_cgo_murtovigplls24_b200\nexcept ImportError as e:\n print('LOUD', e)\n"
            "else:\n print('SILENT')" % str(tmp_path))
    r = subprocess.run([sys.executable, "-c", code], capture_output=True, text=True)
    assert "LOUD" in r.stdout and "no CPU fallback" in r.stdout


def test_product_never_imports_oracle():
    pkg = os.path.join(ROOT, "paper_conf_cgo_murtovigplls24_b200")
    for dirpath, _, files in os.walk(pkg):
        for f in files:
            if f.endswith((".py", ".cu", ".cuh", ".h")):
                text = open(os.path.join(dirpath, f)).read()
                assert "oracle" not in re.sub(r"#.*|//.*", "", text).lower().replace("oracle/", ""), f
