"""ctypes binding of the CPU oracle (TEST INFRASTRUCTURE ONLY).

Only tests/, __graft_entry__.smoke() and bench.py's cpu_baseline /
--impl reference legs may import this module.  The product package
(paper_conf_ipps_jiald16_b200) never imports it.
"""
from __future__ import annotations

import ctypes
import os
import subprocess

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_LIB_PATH = os.path.join(_HERE, "liboracle.so")
_lib = None

SITE_A, SITE_R, SITE_C, SITE_K, SITE_QR, SITE_QC, SITE_RW, SITE_CW = range(8)
(EV_INJECT, EV_DETECT, EV_FIX_DATA, EV_FIX_R, EV_FIX_C, EV_FIX_K, EV_FIX_Q,
 EV_FIX_QR, EV_FIX_QC, EV_FIX_QK, EV_UNCORRECTABLE, EV_FIX_RW, EV_FIX_CW, EV_FIX_KW) = range(14)
EV_NAMES = ["INJECT", "DETECT", "FIX_DATA", "FIX_R", "FIX_C", "FIX_K", "FIX_Q",
            "FIX_QR", "FIX_QC", "FIX_QK", "UNCORRECTABLE", "FIX_RW", "FIX_CW", "FIX_KW"]
MAX_EVENTS = 1024


class Fault(ctypes.Structure):
    _fields_ = [("panel", ctypes.c_int32), ("site", ctypes.c_int32),
                ("i", ctypes.c_int64), ("j", ctypes.c_int64),
                ("bit", ctypes.c_int32), ("pad", ctypes.c_int32)]


class Event(ctypes.Structure):
    _fields_ = [("kind", ctypes.c_int32), ("panel", ctypes.c_int32),
                ("i", ctypes.c_int64), ("j", ctypes.c_int64), ("delta", ctypes.c_double)]


class Report(ctypes.Structure):
    _fields_ = [("detected", ctypes.c_int32), ("corrected", ctypes.c_int32),
                ("uncorrectable", ctypes.c_int32), ("nevents", ctypes.c_int32),
                ("max_drift", ctypes.c_double), ("paper_stat_max", ctypes.c_double),
                ("ev", Event * MAX_EVENTS)]

    def events(self):
        return [(EV_NAMES[e.kind], e.panel, e.i, e.j, e.delta)
                for e in self.ev[: min(self.nevents, MAX_EVENTS)]]


def build(force: bool = False) -> str:
    src = os.path.join(_HERE, "ora_hess.c")
    if force or not os.path.exists(_LIB_PATH) or os.path.getmtime(_LIB_PATH) < os.path.getmtime(src):
        subprocess.check_call(["make", "-s", "-C", _HERE, "-B", "liboracle.so"])
    return _LIB_PATH


def lib():
    global _lib
    if _lib is None:
        build()
        L = ctypes.CDLL(_LIB_PATH)
        dp = ctypes.POINTER(ctypes.c_double)
        L.ora_dgehd2.argtypes = [ctypes.c_int, ctypes.c_int, ctypes.c_int, dp, ctypes.c_int, dp]
        L.ora_dorghr.argtypes = [ctypes.c_int, ctypes.c_int, ctypes.c_int, dp, ctypes.c_int, dp,
                                 dp, ctypes.c_int]
        L.ora_ft_dgehd2.argtypes = [ctypes.c_int, ctypes.c_int, ctypes.c_int, dp, ctypes.c_int, dp,
                                    ctypes.c_int, ctypes.c_double, ctypes.POINTER(Fault),
                                    ctypes.c_int, ctypes.POINTER(Report), ctypes.c_int, dp]
        L.ora_ft_dgehd2_ex.argtypes = [ctypes.c_int, ctypes.c_int, ctypes.c_int, dp, ctypes.c_int, dp,
                                       ctypes.c_int, ctypes.c_double, ctypes.c_int, ctypes.POINTER(Fault),
                                       ctypes.c_int, ctypes.POINTER(Report), ctypes.c_int, dp]
        L.ora_decode_w.argtypes = [ctypes.c_int, dp, ctypes.c_int, dp, dp, dp, dp, dp, dp, dp, ctypes.c_double,
                                   ctypes.POINTER(Report), ctypes.c_int]
        L.ora_decode.argtypes = [ctypes.c_int, dp, ctypes.c_int, dp, dp, dp, ctypes.c_double,
                                 ctypes.POINTER(Report), ctypes.c_int, ctypes.c_int]
        L.ora_encode.argtypes = [ctypes.c_int, dp, ctypes.c_int, dp, dp, dp]
        L.ora_flip.argtypes = [dp, ctypes.c_int]
        L.ora_flip.restype = ctypes.c_double
        L.ora_num_threads.restype = ctypes.c_int
        _lib = L
    return _lib


def _dp(a: np.ndarray):
    return a.ctypes.data_as(ctypes.POINTER(ctypes.c_double))


def _fmat(A: np.ndarray) -> np.ndarray:
    return np.array(A, dtype=np.float64, order="F", copy=True)


def dgehd2(A: np.ndarray, ilo: int = 1, ihi: int | None = None):
    """Return (A_out, tau) -- LAPACK DGEHD2 semantics (H and V packed in A_out)."""
    A = _fmat(A)
    n = A.shape[0]
    ihi = n if ihi is None else ihi
    tau = np.zeros(max(n - 1, 1))
    info = lib().ora_dgehd2(n, ilo, ihi, _dp(A), max(n, 1), _dp(tau))
    if info != 0:
        raise ValueError(f"ora_dgehd2 info={info}")
    return A, tau[: max(n - 1, 0)]


def dorghr(Aout: np.ndarray, tau: np.ndarray, ilo: int = 1, ihi: int | None = None) -> np.ndarray:
    A = _fmat(Aout)
    n = A.shape[0]
    ihi = n if ihi is None else ihi
    t = np.zeros(max(n - 1, 1))
    t[: len(tau)] = tau
    Q = np.zeros((n, n), order="F")
    info = lib().ora_dorghr(n, ilo, ihi, _dp(A), max(n, 1), _dp(t), _dp(Q), max(n, 1))
    if info != 0:
        raise ValueError(f"ora_dorghr info={info}")
    return Q


def ft_dgehd2(A: np.ndarray, nb: int, ilo: int = 1, ihi: int | None = None, c_thr: float = 2.0,
              faults=(), stop_after_panel: int = -1, weighted: bool = False):
    """ABFT oracle.  faults: iterable of (panel, site, i, j, bit).
    Returns (info, A_out, tau, report, chk) with chk = [r | c | kappa] when stopping
    (weighted: [r | c | kappa | r_w | c_w | e^T L w | w^T L e])."""
    A = _fmat(A)
    n = A.shape[0]
    ihi = n if ihi is None else ihi
    tau = np.zeros(max(n - 1, 1))
    fl = list(faults)
    farr = (Fault * max(len(fl), 1))()
    for k, (p, s, i, j, b) in enumerate(fl):
        farr[k] = Fault(p, s, i, j, b, 0)
    rep = Report()
    chk = np.zeros(4 * n + 3 if weighted else 2 * n + 1)
    info = lib().ora_ft_dgehd2_ex(n, ilo, ihi, _dp(A), max(n, 1), _dp(tau), nb, c_thr, 1 if weighted else 0,
                                  farr, len(fl), ctypes.byref(rep), stop_after_panel, _dp(chk))
    if info < 0:
        raise ValueError(f"ora_ft_dgehd2 info={info}")
    return info, A, tau[: max(n - 1, 0)], rep, chk


def decode(L: np.ndarray, r: np.ndarray, c: np.ndarray, kappa: float, tau_abs: float, mode: int = 0):
    """Run the R12 decoder. Returns (result, L, r, c, kappa, report); result 0/1/2."""
    L = _fmat(L)
    r = np.array(r, dtype=np.float64)
    c = np.array(c, dtype=np.float64)
    k = np.array([kappa], dtype=np.float64)
    rep = Report()
    n = L.shape[0]
    res = lib().ora_decode(n, _dp(L), max(n, 1), _dp(r), _dp(c), _dp(k), tau_abs, ctypes.byref(rep), 0, mode)
    return res, L, r, c, float(k[0]), rep


def decode_w(L: np.ndarray, r, c, kappa: float, rw, cw, krw: float, kcw: float, tau_abs: float):
    """Run decoder v3 (weighted pair, w_i = i + 1).
    Returns (result, L, r, c, kappa, rw, cw, krw, kcw, report); result 0/1/2."""
    L = _fmat(L)
    r, c, rw, cw = (np.array(x, dtype=np.float64) for x in (r, c, rw, cw))
    k = np.array([kappa, krw, kcw], dtype=np.float64)
    rep = Report()
    n = L.shape[0]
    kp = k.ctypes.data
    res = lib().ora_decode_w(n, _dp(L), max(n, 1), _dp(r), _dp(c), ctypes.cast(kp, ctypes.POINTER(ctypes.c_double)),
                             _dp(rw), _dp(cw), ctypes.cast(kp + 8, ctypes.POINTER(ctypes.c_double)),
                             ctypes.cast(kp + 16, ctypes.POINTER(ctypes.c_double)), tau_abs, ctypes.byref(rep), 0)
    return res, L, r, c, float(k[0]), rw, cw, float(k[1]), float(k[2]), rep


def encode(A: np.ndarray):
    """Return (r, c, kappa) = (A e, e^T A, e^T A e)."""
    A = _fmat(A)
    n = A.shape[0]
    r = np.zeros(max(n, 1))
    c = np.zeros(max(n, 1))
    k = np.zeros(1)
    lib().ora_encode(n, _dp(A), max(n, 1), _dp(r), _dp(c), _dp(k))
    return r[:n], c[:n], float(k[0])


def flip(x: float, bit: int) -> float:
    a = np.array([x], dtype=np.float64)
    lib().ora_flip(_dp(a), bit)
    return float(a[0])


def num_threads() -> int:
    return lib().ora_num_threads()


def unpack(Aout: np.ndarray):
    """Split the packed result into (H, V) with V unit-lower-trapezoidal (n x (n-1))."""
    n = Aout.shape[0]
    H = np.triu(Aout, -1)
    return H
