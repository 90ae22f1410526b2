"""The C-ABI library loads and exports every symbol include/feves_me.h declares (CPU only)."""
import ctypes
import os
import re
import subprocess

import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
HDR = os.path.join(ROOT, "include", "feves_me.h")


@pytest.fixture(scope="module")
def feves_lib():
    import __graft_entry__ as g
    g.build()
    import paper_conf_icpp_ilicmrs14_b200 as pkg
    return pkg.lib()


def declared_functions():
    src = open(HDR).read()
    src = re.sub(r"/\*.*?\*/", "", src, flags=re.S)
    names = re.findall(r"^[A-Za-z_][\w\s\*]*?\b(\w+)\s*\([^;]*\)\s*;", src, flags=re.M)
    return sorted(set(names))


def test_header_declares_the_boundary():
    names = declared_functions()
    for n in ("me_create", "me_destroy", "me_estimate", "int_interpolate", "sme_refine",
              "me_set_rows", "me_set_stream", "me_get_layout", "me_strerror", "me_last_error",
              "me_encode_frame", "me_last_launch_count"):
        assert n in names, n


def test_library_exports_every_declared_symbol(feves_lib):
    lib_path = feves_lib._name
    out = subprocess.check_output(["nm", "-D", "--defined-only", lib_path], text=True)
    exported = {line.split()[-1] for line in out.splitlines() if line.strip()}
    for n in declared_functions():
        assert n in exported, n
        assert getattr(feves_lib, n) is not None


@pytest.mark.parametrize("args", [(0, 16, 16, 1), (16, -1, 16, 1), (64, 64, 2, 1), (64, 64, 15, 1),
                                  (64, 64, 130, 1), (64, 64, 16, 0), (64, 64, 16, 17)])
def test_create_rejects_bad_arguments(feves_lib, args):
    # argument validation happens before any CUDA call, so this runs without a GPU
    assert not feves_lib.me_create(*args)
    assert feves_lib.me_last_error() == -1


def test_strerror_and_null_safety(feves_lib):
    assert feves_lib.me_strerror(0) == b"ok"
    assert feves_lib.me_strerror(-1) == b"invalid argument"
    feves_lib.me_destroy(None)                       # NULL-safe
    assert feves_lib.me_set_rows(None, 0, 1) == -1
    assert feves_lib.me_estimate(None, None, None, None, None) == -1


def test_no_oracle_in_product_path():
    pkg = os.path.join(ROOT, "paper_conf_icpp_ilicmrs14_b200")
    for dirpath, _, files in os.walk(pkg):
        for f in files:
            if f.endswith((".py", ".cu", ".cuh", ".h", ".cpp")):
                txt = open(os.path.join(dirpath, f)).read()
                assert "import oracle" not in txt and "from oracle" not in txt and "liboracle" not in txt, f


@pytest.mark.parametrize("args", [(64, 64, 16, 1, -1), (64, 64, 16, 1, 257), (256, 256, 128, 1, 4)])
def test_create_pmv_rejects_bad_arguments(feves_lib, args):
    # G21: max_pmv in 0..256, and not with the S = 128 quadrant kernel; checked before any CUDA call
    feves_lib.me_create_pmv.restype = ctypes.c_void_p
    assert not feves_lib.me_create_pmv(*args)
    assert feves_lib.me_last_error() == -1
    assert feves_lib.me_set_pmv(None, None) == -1


@pytest.mark.parametrize("S,inc,lmax", [(128, 0, 1731), (128, 1, 1731), (64, 0, 1935), (64, 1, 1935),
                                        (32, 0, 2000), (4, 0, 2000)])
def test_lambda_limit_keeps_the_key_exact(feves_lib, S, inc, lmax):
    """the ME key J * 2^15 + rank is 32 bits, so J = SAD + lambda * R must stay
    below 2^17.  Hand-derived bounds: max R = 2 * se(4 * 64) = 2 * 19 bits at S = 128 (and for
    the inclusive +64), 2 * se(4 * 32) = 2 * 17 at S = 64: 65280 + 1731 * 38 = 131058 < 131072 <
    65280 + 1732 * 38; 65280 + 1935 * 34 = 131070 < 131072.  Smaller SAs stay at the API cap 2000."""
    Sc = S + inc
    ka = (ctypes.c_uint32 * (Sc * ((Sc + 3) & ~3)))()
    inv = (ctypes.c_uint32 * ((S + 1) ** 2))()
    glob = (ctypes.c_uint32 * (4 * 4096))()
    assert feves_lib.me_key_tables(S, inc, lmax, ka, inv, glob) == 0
    assert feves_lib.me_key_tables(S, inc, lmax + 1, ka, inv, glob) == -1
