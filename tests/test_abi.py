"""CPU-side checks of the boundary: the shared library loads, exports every symbol that
include/fmmfft.h declares, and rejects invalid plans before touching a device."""
import ctypes
import os
import re

import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


@pytest.fixture(scope="module")
def L():
    from paper_conf_sc_cecka17_b200 import build
    build.build()
    from paper_conf_sc_cecka17_b200 import _lib
    return _lib


def header_symbols():
    src = open(os.path.join(ROOT, "include", "fmmfft.h")).read()
    return sorted(set(re.findall(r"FMMFFT_API\s+[\w\s\*]+?\b(fmmfft_\w+)\s*\(", src)))


def test_header_declares_symbols():
    syms = header_symbols()
    assert "fmmfft_plan" in syms and "fmmfft_execute" in syms and "fmmfft_destroy" in syms
    assert len(syms) >= 12


def test_library_exports_every_header_symbol(L):
    lib = ctypes.CDLL(L.LIB_PATH)
    for s in header_symbols():
        assert hasattr(lib, s), s
    assert sorted(header_symbols()) == sorted(L.EXPORTS)


def test_version_and_last_error(L):
    assert b"sm_100a" in L.lib.fmmfft_version()
    assert isinstance(L.lib.fmmfft_last_error(), bytes)


@pytest.mark.parametrize("args,frag", [
    ((1 << 20, 63, 1, 2, 16, 0, 64, 0), b"powers of two"),      # P not a power of two
    ((1 << 20, 64, 3, 2, 16, 0, 64, 0), b"G must be"),          # G = 3
    ((1 << 20, 64, 1, 1, 16, 0, 64, 0), b"L >= B >= 2"),        # B < 2
    ((1 << 12, 16, 1, 3, 16, 0, 64, 0), b"L >= B >= 2"),        # L = 2 < B = 3
    ((1 << 20, 64, 1, 2, 1, 0, 64, 0), b"Q <= 32"),             # Q = 1
    ((1 << 20, 64, 1, 2, 40, 0, 64, 0), b"Q <= 32"),            # Q = 40
    ((1 << 20, 64, 1, 2, 16, 7, 64, 0), b"precision"),
    ((1 << 20, 64, 1, 2, 16, 0, 8, 0), b"M_L"),                 # M_L = 8 < 16
    ((1 << 20, 4, 8, 2, 16, 0, 64, 1), b"P % G"),               # P % G != 0
    ((1 << 20, 64, 2, 2, 16, 0, 64, 0), b"fmmfft_comm_init"),   # G > 1 without a communicator
    ((1001, 16, 1, 2, 16, 0, 64, 32), b"even"),                 # FMMFFT_FLAG_REAL with odd N
])
def test_invalid_plans_rejected(L, args, frag):
    h = ctypes.c_void_p()
    st = L.lib.fmmfft_plan_ex(ctypes.byref(h), *args)
    assert st in (L.INVALID_VALUE, L.NOT_INITIALIZED)
    assert frag in L.lib.fmmfft_last_error()
    assert not h.value


def test_null_arguments(L):
    assert L.lib.fmmfft_plan_ex(None, 1 << 20, 64, 1, 2, 16, 0, 64, 0) == L.INVALID_VALUE
    assert L.lib.fmmfft_execute(None, None, None, None) == L.INVALID_VALUE
    assert L.lib.fmmfft_destroy(None) == L.SUCCESS
    assert L.lib.fmmfft_get_unique_id(None) == L.INVALID_VALUE
    assert L.lib.fmmfft_comm_init(0, 2, None) == L.INVALID_VALUE


def test_stage_names(L):
    names = [L.lib.fmmfft_stage_name(i).decode() for i in range(10)]
    assert names == ["comm_S", "s2m", "m2m", "comm_M", "top", "down", "post_pfft", "a2a", "mfft", "s2t"]
    assert L.lib.fmmfft_stage_name(99) == b""


def test_package_has_no_cpu_fallback():
    """The product package never imports the oracle or numpy FFTs."""
    pkg = os.path.join(ROOT, "paper_conf_sc_cecka17_b200")
    for f in os.listdir(pkg):
        if f.endswith(".py"):
            src = open(os.path.join(pkg, f)).read()
            assert "oracle" not in src.replace("oracle/", ""), f
            assert "numpy.fft" not in src and "np.fft" not in src and "torch.fft" not in src, f


# ------------------------------------------------------------------ autotuner model mode (host only)
def test_autotune_model_host_only():
    from paper_conf_sc_cecka17_b200 import autotune
    from paper_conf_sc_cecka17_b200._lib import FmmfftError
    t = autotune(1 << 26, G=8, precision="c64", tol=1e-5, measure=False)
    assert t["Q"] == 8 and t["M_L"] == 64 and t["P"] % 8 == 0 and 2 <= t["B"] <= 4
    L = (26 - (t["P"].bit_length() - 1) - 6)
    assert L >= t["B"] and (1 << L) % 8 == 0 and t["candidates"] > 3 and t["error"] * 4 <= 1e-5
    t = autotune(1 << 28, G=8, precision="c128", tol=1e-11, measure=False)
    assert t["Q"] == 16
    with pytest.raises(FmmfftError):
        autotune(1 << 20, precision="c64", tol=1e-8, measure=False)      # below the fp32 floor
    with pytest.raises(FmmfftError):
        autotune(1 << 20, G=2, precision="c64", measure=True)           # measuring is G = 1 only


def test_flag_values_match_header(L):
    src = open(os.path.join(ROOT, "include", "fmmfft.h")).read()
    hdr = {m[0]: int(m[1]) for m in re.findall(r"#define FMMFFT_FLAG_(\w+)\s+(\d+)u", src)}
    assert hdr == {"VIRTUAL": L.FLAG_VIRTUAL, "PROFILE": L.FLAG_PROFILE, "DEBUG": L.FLAG_DEBUG,
                   "INVERSE": L.FLAG_INVERSE, "DIRECT": L.FLAG_DIRECT, "REAL": L.FLAG_REAL,
                   "VIRTUAL_NCCL": L.FLAG_VIRTUAL_NCCL}


def test_real_rejects_odd_length(L):
    # FMMFFT_FLAG_REAL (any G, incl. G > 1 since round 2) needs an even real length: rejected before
    # any device or communicator is touched
    h = ctypes.c_void_p()
    st = L.lib.fmmfft_plan_ex(ctypes.byref(h), (1 << 21) + 1, 64, 2, 2, 16, 0, 64, 32 | 1)
    assert st == L.INVALID_VALUE and b"even" in L.lib.fmmfft_last_error() and not h.value
