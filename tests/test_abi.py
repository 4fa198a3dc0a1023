"""C-ABI library: builds, loads, exports every symbol include/mdnorm.h declares, and validates
arguments before touching the GPU (no compute calls here; runs on the CPU-only box)."""
import ctypes as C
import os
import subprocess

import numpy as np
import pytest

from paper_conf_sc_hahnfgmmshvvs24_b200 import _native, build


@pytest.fixture(scope="module")
def lib():
    build.build()
    return _native.load()


def test_header_symbols_exported(lib):
    names = _native.header_functions()
    assert len(names) == 31
    for n in names:
        assert hasattr(lib, n), f"{n} declared in include/mdnorm.h but not exported"
        assert n in _native.SIGNATURES, f"{n} missing from the Python binding"
    # and nothing the binding expects is missing from the header
    assert set(_native.SIGNATURES) == set(names)


def test_exports_are_extern_c(lib):
    out = subprocess.check_output(["nm", "-D", "--defined-only", _native.LIB_PATH], text=True)
    syms = {line.split()[-1] for line in out.splitlines() if " T " in line}
    for n in _native.header_functions():
        assert n in syms, f"{n} not exported with C linkage"


def test_sm100a_code_present():
    out = subprocess.check_output(["/usr/local/cuda/bin/cuobjdump", "--list-elf", _native.LIB_PATH], text=True)
    assert "sm_100a" in out


def test_version_and_last_error(lib):
    assert lib.mdn_version().decode().startswith("mdnorm sm_100a")
    assert isinstance(lib.mdn_last_error(), bytes)


def _create(lib, lo=(0, 0, 0), hi=(1, 1, 1), n=(2, 2, 2), W=np.eye(3), acc=1):
    lo = np.asarray(lo, np.float64)
    hi = np.asarray(hi, np.float64)
    n = np.asarray(n, np.int64)
    W = np.ascontiguousarray(W, np.float64)
    h = C.c_void_p()
    st = lib.mdnorm_create_grid(0, lo.ctypes.data, hi.ctypes.data, n.ctypes.data, W.ctypes.data, acc,
                                C.byref(h))
    return st, h


@pytest.mark.parametrize("kw,frag", [
    (dict(lo=(0, 0, 1), hi=(1, 1, 1)), "lo < hi"),
    (dict(lo=(0, np.nan, 0)), "lo < hi"),
    (dict(n=(2, 0, 2)), "nbins"),
    (dict(W=np.zeros((3, 3))), "W"),
    (dict(acc=7), "accumulation mode"),
])
def test_create_grid_validation_precedes_cuda(lib, kw, frag):
    st, h = _create(lib, **kw)
    assert st == _native.MDN_EINVAL
    assert h.value is None
    assert frag in lib.mdn_last_error().decode()


def test_null_handles_are_einval(lib):
    z = np.zeros(9)
    assert lib.mdnorm_set_flux(None, 2, z.ctypes.data, z.ctypes.data) == _native.MDN_EINVAL
    assert lib.mdnorm_set_instrument(None, 1, z.ctypes.data, z.ctypes.data) == _native.MDN_EINVAL
    assert lib.mdnorm_accumulate(None, z.ctypes.data, z.ctypes.data, 1, z.ctypes.data, 1.0, 2.0, 1.0, 0,
                                 -1, 1, None) == _native.MDN_EINVAL
    assert lib.mdnorm_cross_section(None, z.ctypes.data, None) == _native.MDN_EINVAL
    assert lib.mdnorm_reset(None, None) == _native.MDN_EINVAL
    assert lib.mdnorm_destroy(None) == _native.MDN_OK
    assert lib.mdnorm_set_privatization(None, 0) == _native.MDN_EINVAL
    assert lib.mdnorm_accumulation_paths(None, np.zeros(2, np.int32).ctypes.data) == _native.MDN_EINVAL


def test_no_gpu_is_reported_not_crashing(lib):
    import torch
    if torch.cuda.is_available():
        pytest.skip("GPU present")
    st, h = _create(lib)
    assert st == _native.MDN_ECUDA
    assert lib.mdn_last_error().decode()


def test_binding_fails_loudly_without_library(monkeypatch, tmp_path):
    monkeypatch.setattr(_native, "LIB_PATH", str(tmp_path / "missing.so"))
    monkeypatch.setattr(_native, "_lib", None)
    with pytest.raises(RuntimeError, match="no CPU fallback"):
        _native.load()


def test_product_package_never_imports_oracle():
    pkg = os.path.dirname(_native.__file__)
    for root, _, files in os.walk(pkg):
        for f in files:
            if f.endswith((".py", ".cu", ".cuh", ".h", ".cpp")):
                src = open(os.path.join(root, f)).read()
                assert "import oracle" not in src and "from oracle" not in src, f
                assert "liboracle" not in src and "oracle.h" not in src, f


def test_divide_validates_before_cuda(lib):
    x = np.zeros(4)
    p = x.ctypes.data
    assert lib.mdn_divide(0, p, p, p, -1, None) == _native.MDN_EINVAL
    assert lib.mdn_divide(0, None, p, p, 4, None) == _native.MDN_EINVAL
    assert lib.mdn_divide(0, p, p, p, 0, None) == _native.MDN_OK  # empty shard: nothing to do
