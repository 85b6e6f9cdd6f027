"""CPU-only checks of the C-ABI boundary: the library loads, exports every symbol include/bmr.h
declares, and fails loudly (no CPU fallback) when no CUDA device is present."""
import ctypes as C
import re

import pytest

import paper_conf_ipps_jim11_b200 as bmr


def declared():
    src = open("include/bmr.h").read()
    return sorted(set(re.findall(r"^\s*(?:mr_status|const char\*)\s+(mr_\w+)\(", src, re.M)))


def test_header_declares_the_abi():
    d = declared()
    for name in ("mr_job_create", "mr_map", "mr_group", "mr_reduce", "mr_fetch", "mr_job_destroy"):
        assert name in d
    assert set(d) == set(bmr.EXPORTS)


def test_library_exports_every_declared_symbol():
    L = bmr.lib()
    for name in declared():
        assert hasattr(L, name), name


def test_status_strings():
    L = bmr.lib()
    assert L.mr_status_string(0) == b"MR_OK"
    assert L.mr_status_string(4) == b"MR_ERR_OVERFLOW"


def test_invalid_arguments_are_rejected_without_device():
    L = bmr.lib()
    h = C.c_void_p()
    assert L.mr_job_create(None, C.byref(h)) == 1
    cfg = bmr.Config()
    cfg.abi_version = 99
    cfg.workload = 1
    assert L.mr_job_create(C.byref(cfg), C.byref(h)) == 1          # abi_version mismatch
    cfg.abi_version = 1
    cfg.workload = 3                                               # KM without params
    cfg.record_stride = 32
    assert L.mr_job_create(C.byref(cfg), C.byref(h)) == 1
    assert L.mr_job_destroy(None) == 0


def test_no_cpu_fallback():
    torch = pytest.importorskip("torch")
    if torch.cuda.is_available():
        pytest.skip("GPU present")
    with pytest.raises(bmr.MRError) as e:
        bmr.Job("wc", stream=0)
    assert e.value.status == 5  # MR_ERR_CUDA
