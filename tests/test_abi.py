"""Host-side checks of the C ABI library (no GPU needed): it loads, exports every symbol include/sesa.h
declares, and reports errors without a device instead of falling back to anything."""
import ctypes
import os
import re

import numpy as np
import pytest

from paper_conf_sc_lilg14_b200 import sesa as S

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def header_functions():
    text = open(os.path.join(ROOT, "include", "sesa.h")).read()
    text = re.sub(r"/\*.*?\*/", "", text, flags=re.S)
    return sorted(set(re.findall(r"\b(sesa_[a-z_0-9]+)\s*\(", text)))


def test_library_exports_every_declared_symbol():
    lib = S.load()
    names = header_functions()
    assert "sesa_race_check" in names and "sesa_expand" in names
    for name in names:
        assert hasattr(lib, name), name
    assert set(names) == set(S.EXPORTS)


def test_abi_version_and_status_strings():
    lib = S.load()
    assert lib.sesa_abi_version() == 1
    assert lib.sesa_status_str(S.SESA_EINVAL) == b"SESA_EINVAL"
    assert lib.sesa_status_str(S.SESA_ETRUNC) == b"SESA_ETRUNC"


def test_struct_layouts_match_generators_and_oracle():
    import sesagen
    from oracle import oracle as O
    assert S.ACCESS_DTYPE == sesagen.REC_DTYPE == O.REC_DTYPE
    assert S.RACE_DTYPE == sesagen.RACE_DTYPE == O.RACE_DTYPE
    assert S.FLOW_DTYPE == sesagen.FLOW_DTYPE == O.FLOW_DTYPE
    assert ctypes.sizeof(S.sesa_config) == 16
    assert S.REGION_DTYPE.itemsize == 24 and ctypes.sizeof(S.sesa_oob_report) == 48
    assert S.REGION_DTYPE == sesagen.f6_regions().dtype


def test_bad_config_rejected_before_device():
    lib = S.load()
    h = ctypes.c_void_p()
    for cfg in ((0, 0, 4, 0), (32, 2, 4, 0), (32, 0, 3, 0), (32, 0, 8192, 0), (32, 0, 4, 2), (32, 0, 4, 0x80)):
        c = S.sesa_config(*cfg)
        assert lib.sesa_trace_create(ctypes.byref(c), ctypes.byref(h)) == S.SESA_EINVAL
        assert not h.value


def test_null_handle_calls():
    lib = S.load()
    n = ctypes.c_uint64()
    assert lib.sesa_races_get(None, None, 0, ctypes.byref(n)) == S.SESA_EINVAL
    assert lib.sesa_race_check(None, None, 0, 0, None) == S.SESA_EINVAL
    assert lib.sesa_trace_set_regions(None, None, 0) == S.SESA_EINVAL
    assert lib.sesa_oob_get(None, None) == S.SESA_EINVAL
    lib.sesa_trace_destroy(None)  # NULL-safe
    assert lib.sesa_last_error(None) == b""


def test_no_cpu_fallback_without_device():
    torch = pytest.importorskip("torch")
    if torch.cuda.is_available():
        pytest.skip("a GPU is present")
    lib = S.load()
    h = ctypes.c_void_p()
    c = S.sesa_config(32, 0, 4, 0)
    assert lib.sesa_trace_create(ctypes.byref(c), ctypes.byref(h)) == S.SESA_ECUDA
    with pytest.raises(S.SesaError):
        S.Trace()


def test_product_path_independent_of_oracle():
    """The product (package + CUDA sources + generators) never names the oracle, and the oracle never names the
    product: the two share no code (task rule ③)."""
    pkg = os.path.join(ROOT, "paper_conf_sc_lilg14_b200")
    product = [os.path.join(d, f) for d, _, fs in os.walk(pkg) for f in fs
               if f.endswith((".py", ".cu", ".cuh", ".h", ".cpp"))]
    product += [os.path.join(ROOT, "include", f) for f in os.listdir(os.path.join(ROOT, "include"))]
    assert len(product) > 10
    for path in product:
        text = open(path).read()
        assert not re.search(r"^\s*(from|import)\s+oracle\b|#include\s*[<\"][^>\"]*oracle|sesa_oracle|oracle/_build",
                             text, flags=re.M), path
    odir = os.path.join(ROOT, "oracle")
    for f in os.listdir(odir):
        if f.endswith((".py", ".c", ".h")):
            text = open(os.path.join(odir, f)).read()
            assert not re.search(r"^\s*(from|import)\s+paper_conf_sc_lilg14_b200|#include\s*[<\"]sesa|libsesa\.so",
                                 text, flags=re.M), f
