"""CPU-side checks of the C-ABI library: it loads, exports every symbol include/msm.h
declares, and its size/error entry points behave without a GPU."""
import ctypes
import os
import re

import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
HDR = os.path.join(ROOT, "include", "msm.h")
LIB = os.path.join(ROOT, "paper_conf_asplos_ji0x024_b200", "libmsm.so")


def declared_functions():
    src = open(HDR).read()
    src = re.sub(r"/\*.*?\*/", "", src, flags=re.S)
    names = re.findall(r"^\s*[A-Za-z_][\w\s\*]*?\b(msm_\w+)\s*\(", src, flags=re.M)
    return sorted(set(names))


def test_header_declares_the_boundary():
    names = declared_functions()
    for must in ("msm_context_create", "msm_run", "msm_context_destroy", "msm_run_partial", "msm_finalize"):
        assert must in names


@pytest.mark.skipif(not os.path.exists(LIB), reason="libmsm.so not built")
def test_library_exports_every_declared_symbol():
    L = ctypes.CDLL(LIB)
    missing = [n for n in declared_functions() if not hasattr(L, n)]
    assert not missing, missing


@pytest.mark.skipif(not os.path.exists(LIB), reason="libmsm.so not built")
def test_sizes_and_errors_without_gpu():
    from paper_conf_asplos_ji0x024_b200 import msm
    assert [msm.field_words(c) for c in ("bn254", "bls12_377", "bls12_381", "mnt4_753")] == [8, 12, 12, 24]
    assert [msm.scalar_words(c) for c in ("bn254", "bls12_377", "bls12_381", "mnt4_753")] == [8, 8, 8, 24]
    L = msm.lib()
    assert [L.msm_scalar_bits(i) for i in range(4)] == [254, 253, 255, 753]
    assert L.msm_field_words(7) == -2
    assert L.msm_error_string(-7) == b"scalar >= r"
    assert msm.partial_words("bls12_381") == 4 * 13
    if msm.device_count() == 0:
        with pytest.raises(msm.MSMError) as e:
            msm.Context("bn254", None, n=0)
        assert e.value.code == -9
