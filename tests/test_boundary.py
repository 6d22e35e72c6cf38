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
    assert "UTMALDG" in sass  # their operand tiles arrive by 2-D tensor TMA


def test_struct_layouts_match_header(ft):
    m = ft.ftgehrd
    assert ctypes.sizeof(m.Fault) == 4 * 4 + 2 * 8
    assert ctypes.sizeof(m.Event) == 2 * 4 + 3 * 8
    assert ctypes.sizeof(m.Report) == 6 * 4 + 8 + 8 * 8 + 256 * ctypes.sizeof(m.Event)
    o = m.Opts()
    ft.lib().ft_opts_default(ctypes.byref(o))
    assert o.abft == 1 and o.nb == 0 and o.c_thr == 2.0 and o.stop_after_panel == -1 and o.weighted == 0
    assert o.deterministic == 0 and o.timing == 0


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


def test_right_update_row_splits_partition_each_strip(ft):
    """Host logic of the right update's weighted row splits (ft_gemm.cu): every split of a strip
    gets a contiguous tile range, the ranges cover the strip exactly once, and the weights
    (right-only tiles above the W rows 1, right + W tiles 2) differ by at most one tile."""
    L = ft.lib()
    L.ft_debug_right_split_range.argtypes = [ctypes.c_int] * 4 + [ctypes.POINTER(ctypes.c_int)] * 2
    t0, t1 = ctypes.c_int(), ctypes.c_int()
    for nrt in (1, 2, 3, 17, 64, 256, 257):
        for tw in sorted({0, 1, nrt // 3, nrt // 2, nrt - 1, nrt}):
            if tw < 0 or tw > nrt:
                continue
            for ns in (1, 2, 3, 5, 16, 32):
                ranges = []
                for y in range(ns):
                    L.ft_debug_right_split_range(nrt, tw, ns, y, ctypes.byref(t0), ctypes.byref(t1))
                    ranges.append((t0.value, t1.value))
                assert ranges[0][0] == 0 and ranges[-1][1] == nrt
                assert all(a <= b for a, b in ranges)
                assert all(ranges[i][1] == ranges[i + 1][0] for i in range(ns - 1))
                w = [sum(1 if t < tw else 2 for t in range(a, b)) for a, b in ranges]
                total = tw + 2 * (nrt - tw)
                assert max(w) - min(w) <= 3 and abs(max(w) - total / ns) <= 2.5, (nrt, tw, ns, w)


def test_right_update_split_count_is_bounded(ft):
    L = ft.lib()
    L.ft_debug_right_splits.argtypes = [ctypes.c_int] * 7
    for n in (300, 2048, 16384):
        for e in (64, n // 2, n - 64):
            for wr in (-1, 0, e - 63):
                ns = L.ft_debug_right_splits(0, n, e, n + 1, 148, 1, wr)
                nrt = (n + 63) // 64
                assert 1 <= ns <= min(32, nrt), (n, e, wr, ns)
