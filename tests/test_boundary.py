"""CPU-side checks of the C-ABI boundary (no GPU needed): the library builds for
sm_100a, loads, and exports every symbol include/ftgehrd.h declares; the ctypes
structures match the header's layout; argument validation happens before any
device work."""
import ctypes
import os
import re
import subprocess

import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
HEADER = os.path.join(ROOT, "include", "ftgehrd.h")


@pytest.fixture(scope="module")
def ft():
    import paper_conf_ipps_jiald16_b200 as ft
    ft.build()
    return ft


def declared_functions():
    src = open(HEADER).read()
    return sorted(set(re.findall(r"^\s*(?:const\s+)?[a-z_0-9]+\s*\*?\s*(ft_[a-z_0-9]+)\s*\(", src, re.M)))


def test_header_declares_the_boundary():
    names = declared_functions()
    for f in ["ft_dgehrd", "ft_dgehrd_host", "ft_dorghr", "ft_dgehrd_mgpu", "ft_mgpu_setup", "ft_mgpu_connect",
              "ft_dgehrd_vranks", "ft_mgpu_finalize", "ft_strerror", "ft_finalize",
              "ft_opts_default", "ft_version", "ft_launch_count"]:
        assert f in names


def test_library_exports_every_declared_symbol(ft):
    out = subprocess.run(["nm", "-D", "--defined-only", ft.ftgehrd.LIB_PATH], capture_output=True, text=True).stdout
    exported = set(re.findall(r" T (ft_[a-z_0-9]+)", out))
    missing = [f for f in declared_functions() if f not in exported]
    assert not missing, missing
    L = ft.lib()
    for f in declared_functions():
        getattr(L, f)


def test_library_is_sm100a_native(ft):
    out = subprocess.run(["cuobjdump", "-lelf", ft.ftgehrd.LIB_PATH], capture_output=True, text=True).stdout
    assert "sm_100a" in out
    sass = subprocess.run(["cuobjdump", "-sass", ft.ftgehrd.LIB_PATH], capture_output=True, text=True).stdout
    assert "DMMA" in sass  # the block-reflector updates run on the FP64 tensor pipe


def test_struct_layouts_match_header(ft):
    m = ft.ftgehrd
    assert ctypes.sizeof(m.Fault) == 4 * 4 + 2 * 8
    assert ctypes.sizeof(m.Event) == 2 * 4 + 3 * 8
    assert ctypes.sizeof(m.Report) == 6 * 4 + 8 + 8 * 8 + 256 * ctypes.sizeof(m.Event)
    o = m.Opts()
    ft.lib().ft_opts_default(ctypes.byref(o))
    assert o.abft == 1 and o.nb == 0 and o.c_thr == 2.0 and o.stop_after_panel == -1 and o.weighted == 0


@pytest.mark.parametrize("args,expect", [
    ((-1, 1, 0, 8, 1, 8), -1),      # n < 0
    ((4, 0, 4, 8, 4, 8), -2),       # ilo < 1
    ((4, 3, 2, 8, 4, 8), -3),       # ihi < ilo
    ((4, 1, 5, 8, 4, 8), -3),       # ihi > n
    ((4, 1, 4, 0, 4, 8), -4),       # A null
    ((4, 1, 4, 8, 3, 8), -5),       # lda < n
    ((4, 1, 4, 8, 4, 0), -6),       # tau null
])
def test_argument_validation_without_gpu(ft, args, expect):
    n, ilo, ihi, a, lda, t = args
    info = ft.lib().ft_dgehrd(n, ilo, ihi, ctypes.c_void_p(a), lda, ctypes.c_void_p(t), None)
    assert info == expect


def test_bad_opts_rejected_without_gpu(ft):
    m = ft.ftgehrd
    o = m.Opts()
    ft.lib().ft_opts_default(ctypes.byref(o))
    o.nb = 65
    assert ft.lib().ft_dgehrd(4, 1, 4, ctypes.c_void_p(8), 4, ctypes.c_void_p(8), ctypes.byref(o)) == -7
    o.nb = 0
    o.weighted = 2  # 0 or 1
    assert ft.lib().ft_dgehrd(4, 1, 4, ctypes.c_void_p(8), 4, ctypes.c_void_p(8), ctypes.byref(o)) == -7
    o.weighted = 1
    o.abft = 0  # the weighted pair (NEXT-1) needs the checksums
    assert ft.lib().ft_dgehrd(4, 1, 4, ctypes.c_void_p(8), 4, ctypes.c_void_p(8), ctypes.byref(o)) == -7
    o.weighted = 0
    o.abft = 1
    o.timing = 3
    assert ft.lib().ft_dgehrd(4, 1, 4, ctypes.c_void_p(8), 4, ctypes.c_void_p(8), ctypes.byref(o)) == -7


def test_strerror(ft):
    assert "success" in ft.strerror(0)
    assert "argument 5" in ft.strerror(-5)
    assert "uncorrectable" in ft.strerror(1)
    assert "sm_100a" in ft.version()


def test_n0_is_a_noop_without_gpu(ft):
    assert ft.lib().ft_dgehrd(0, 1, 0, None, 1, None, None) == 0


def test_product_package_does_not_import_oracle():
    pkg = os.path.join(ROOT, "paper_conf_ipps_jiald16_b200")
    for dirpath, _, files in os.walk(pkg):
        for f in files:
            if f.endswith((".py", ".cu", ".cuh", ".h", ".cpp")):
                txt = open(os.path.join(dirpath, f)).read()
                assert "import oracle" not in txt and "oracle.h" not in txt and "liboracle" not in txt, f
