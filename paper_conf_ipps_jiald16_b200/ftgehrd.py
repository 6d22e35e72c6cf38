"""Thin ctypes binding of libftgehrd.so (include/ftgehrd.h).

Argument marshalling only: every step of the reduction runs in the library's
CUDA kernels.  torch supplies device memory and streams.  If the shared
library is missing this module raises -- there is no CPU fallback.
"""
from __future__ import annotations

import ctypes
import os
import subprocess
from dataclasses import dataclass, field

_HERE = os.path.dirname(os.path.abspath(__file__))
LIB_PATH = os.path.join(_HERE, "libftgehrd.so")
CSRC = os.path.join(_HERE, "csrc")
_lib = None

FT_E_UNCORRECTABLE, FT_E_CUDA, FT_E_NCCL, FT_E_NOMEM = 1, 2, 3, 4
PHASE_BEFORE_PANEL, PHASE_AFTER_PANEL, PHASE_AFTER_RIGHT, PHASE_AFTER_UPDATE, PHASE_AT_END = range(5)
SITE_A, SITE_R, SITE_C, SITE_K, SITE_Y, SITE_V, SITE_T, SITE_RW, SITE_CW = range(9)
EV_NAMES = ["INJECT", "DETECT", "FIX_DATA", "FIX_R", "FIX_C", "FIX_K", "FIX_Q", "FIX_QR", "FIX_QC",
            "FIX_QK", "UNCORRECTABLE", "ROLLBACK", "PANEL_REDO", "FIX_RW", "FIX_CW", "FIX_KW"]
POLICY_EAGER, POLICY_PAPER = 0, 1
MAX_EVENTS = 256


class Fault(ctypes.Structure):
    _fields_ = [("panel", ctypes.c_int32), ("phase", ctypes.c_int32), ("site", ctypes.c_int32),
                ("bit", ctypes.c_int32), ("i", ctypes.c_int64), ("j", ctypes.c_int64)]


class Event(ctypes.Structure):
    _fields_ = [("kind", ctypes.c_int32), ("panel", ctypes.c_int32), ("i", ctypes.c_int64),
                ("j", ctypes.c_int64), ("delta", ctypes.c_double)]


class Report(ctypes.Structure):
    _fields_ = [("detected", ctypes.c_int32), ("corrected", ctypes.c_int32), ("rollbacks", ctypes.c_int32),
                ("panel_redos", ctypes.c_int32), ("uncorrectable", ctypes.c_int32), ("nevents", ctypes.c_int32),
                ("max_drift_rel", ctypes.c_double), ("ms", ctypes.c_double * 8),
                ("events", Event * MAX_EVENTS)]

    def event_list(self):
        return [(EV_NAMES[e.kind], e.panel, e.i, e.j, e.delta)
                for e in self.events[: min(self.nevents, MAX_EVENTS)]]


class IpcHandle(ctypes.Structure):
    _fields_ = [("bytes", ctypes.c_char * 64)]


class Opts(ctypes.Structure):
    _fields_ = [("nb", ctypes.c_int32), ("abft", ctypes.c_int32), ("weighted", ctypes.c_int32),
                ("policy", ctypes.c_int32), ("c_thr", ctypes.c_double),
                ("faults", ctypes.POINTER(Fault)), ("nfaults", ctypes.c_int32),
                ("report", ctypes.POINTER(Report)), ("stop_after_panel", ctypes.c_int32),
                ("dchk_out", ctypes.c_void_p), ("stream", ctypes.c_void_p), ("timing", ctypes.c_int32),
                ("deterministic", ctypes.c_int32)]


def build(force: bool = False) -> str:
    """Compile libftgehrd.so for sm_100a (nvcc cross-compiles without a GPU)."""
    cmd = ["make", "-s", "-C", CSRC]
    if force:
        cmd.append("-B")
    subprocess.check_call(cmd)
    return LIB_PATH


def lib():
    global _lib
    if _lib is None:
        if not os.path.exists(LIB_PATH):
            raise RuntimeError(f"{LIB_PATH} is missing: run __graft_entry__.build() (no CPU fallback exists)")
        L = ctypes.CDLL(LIB_PATH)
        vp, i32 = ctypes.c_void_p, ctypes.c_int
        L.ft_opts_default.argtypes = [ctypes.POINTER(Opts)]
        L.ft_dgehrd.argtypes = [i32, i32, i32, vp, i32, vp, ctypes.POINTER(Opts)]
        L.ft_dgehrd_host.argtypes = [i32, i32, i32, vp, i32, vp, ctypes.POINTER(Opts)]
        L.ft_dorghr.argtypes = [i32, i32, i32, vp, i32, vp, vp, i32, ctypes.POINTER(Opts)]
        L.ft_dsytrd.argtypes = [i32, vp, i32, vp, vp, vp, ctypes.POINTER(Opts)]
        L.ft_dgehrd_mgpu.argtypes = [i32, i32, i32, vp, i32, vp, i32, i32, ctypes.POINTER(Opts)]
        L.ft_mgpu_setup.argtypes = [i32, i32, i32, ctypes.POINTER(IpcHandle)]
        L.ft_mgpu_connect.argtypes = [ctypes.POINTER(IpcHandle), i32, i32]
        L.ft_dgehrd_vranks.argtypes = [i32, i32, i32, ctypes.POINTER(vp), i32, ctypes.POINTER(vp), i32,
                                       ctypes.POINTER(Opts)]
        L.ft_mgpu_probe_put.argtypes = [ctypes.c_double]
        L.ft_mgpu_probe_get.argtypes = [vp]
        L.ft_strerror.argtypes = [i32]
        L.ft_strerror.restype = ctypes.c_char_p
        L.ft_version.restype = ctypes.c_char_p
        L.ft_launch_count.argtypes = [i32]
        L.ft_launch_count.restype = ctypes.c_int64
        _lib = L
    return _lib


EXPORTS = ["ft_opts_default", "ft_dgehrd", "ft_dgehrd_host", "ft_dorghr", "ft_dsytrd", "ft_dgehrd_mgpu",
           "ft_mgpu_setup", "ft_mgpu_connect", "ft_dgehrd_vranks", "ft_mgpu_finalize",
           "ft_mgpu_probe_put", "ft_mgpu_probe_get",
           "ft_strerror", "ft_finalize", "ft_version", "ft_launch_count"]


@dataclass
class Result:
    info: int
    report: Report | None = None
    events: list = field(default_factory=list)


def _stream_ptr(stream):
    if stream is None:
        import torch
        return ctypes.c_void_p(torch.cuda.current_stream().cuda_stream)
    return ctypes.c_void_p(getattr(stream, "cuda_stream", stream))


def _check_fortran(A, name="A"):
    import torch
    if not isinstance(A, torch.Tensor) or A.dtype != torch.float64 or not A.is_cuda:
        raise TypeError(f"{name} must be a CUDA float64 tensor")
    if A.dim() != 2 or A.shape[0] != A.shape[1]:
        raise ValueError(f"{name} must be square")
    n = A.shape[0]
    if n > 1 and A.stride(0) != 1:
        raise ValueError(f"{name} must be column-major (stride(0) == 1); use fortran()")
    return n, (A.stride(1) if n > 1 else max(n, 1))


def fortran(x):
    """Column-major copy of a 2-D tensor (same values, Fortran layout)."""
    return x.t().contiguous().t()


def make_opts(nb=0, abft=True, policy=POLICY_EAGER, c_thr=2.0, faults=(), report=None,
              stop_after_panel=-1, dchk_out=None, stream=None, timing=False, weighted=False, deterministic=False):
    o = Opts()
    lib().ft_opts_default(ctypes.byref(o))
    o.nb = nb
    o.abft = 1 if abft else 0
    o.weighted = 1 if weighted else 0
    o.policy = policy
    o.c_thr = c_thr
    fl = list(faults)
    farr = (Fault * max(len(fl), 1))()
    for k, f in enumerate(fl):
        if isinstance(f, Fault):
            farr[k] = f
        else:
            panel, phase, site, i, j, bit = f
            farr[k] = Fault(panel, phase, site, bit, i, j)
    o.faults = ctypes.cast(farr, ctypes.POINTER(Fault))
    o.nfaults = len(fl)
    o.report = ctypes.pointer(report) if report is not None else None
    o.stop_after_panel = stop_after_panel
    o.dchk_out = ctypes.c_void_p(dchk_out.data_ptr()) if dchk_out is not None else None
    o.stream = _stream_ptr(stream)
    o.timing = 1 if timing else 0
    o.deterministic = 1 if deterministic else 0
    o._keep = farr  # keep the fault array alive
    return o


def dgehrd(A, tau=None, ilo=1, ihi=None, **kw):
    """In-place ABFT Hessenberg reduction of the column-major CUDA float64 matrix A.

    faults: iterable of (panel, phase, site, i, j, bit).  Returns (tau, Result)."""
    import torch
    n, lda = _check_fortran(A)
    ihi = n if ihi is None else ihi
    if tau is None:
        tau = torch.zeros(max(n - 1, 1), dtype=torch.float64, device=A.device)
    rep = Report()
    o = make_opts(report=rep, **kw)
    info = lib().ft_dgehrd(n, ilo, ihi, ctypes.c_void_p(A.data_ptr()), lda, ctypes.c_void_p(tau.data_ptr()),
                           ctypes.byref(o))
    return tau, Result(info, rep, rep.event_list())


def dsytrd(A, **kw):
    """Symmetric tridiagonal reduction (DSYTRD, uplo 'L') of the column-major CUDA float64 matrix A
    (lower triangle read; NEXT-4 on the protected path).  Returns (d, e, tau, Result)."""
    import torch
    n, lda = _check_fortran(A)
    d = torch.zeros(max(n, 1), dtype=torch.float64, device=A.device)
    e = torch.zeros(max(n - 1, 1), dtype=torch.float64, device=A.device)
    tau = torch.zeros(max(n - 1, 1), dtype=torch.float64, device=A.device)
    rep = Report()
    o = make_opts(report=rep, **kw)
    info = lib().ft_dsytrd(n, ctypes.c_void_p(A.data_ptr()), lda, ctypes.c_void_p(d.data_ptr()),
                           ctypes.c_void_p(e.data_ptr()), ctypes.c_void_p(tau.data_ptr()), ctypes.byref(o))
    return d[:n], e[: max(n - 1, 0)], tau[: max(n - 1, 0)], Result(info, rep, rep.event_list())


def dgehrd_host(A_np, ilo=1, ihi=None, **kw):
    """End-to-end entry with host buffers (numpy float64, Fortran order, modified in place)."""
    import numpy as np
    if not (A_np.flags["F_CONTIGUOUS"] and A_np.dtype == np.float64):
        raise ValueError("A must be a Fortran-ordered float64 numpy array")
    n = A_np.shape[0]
    ihi = n if ihi is None else ihi
    tau = np.zeros(max(n - 1, 1))
    rep = Report()
    o = make_opts(report=rep, **kw)
    info = lib().ft_dgehrd_host(n, ilo, ihi, ctypes.c_void_p(A_np.ctypes.data), max(n, 1),
                                ctypes.c_void_p(tau.ctypes.data), ctypes.byref(o))
    return tau[: max(n - 1, 0)], Result(info, rep, rep.event_list())


def dorghr(A, tau, ilo=1, ihi=None, Q=None, nb=0, stream=None, abft=True, faults=(), c_thr=2.0, timing=False,
           full=False):
    """Explicit Q from ft_dgehrd's output (DORGHR semantics).  abft: checksum-protected accumulation
    (NEXT-3); faults: (panel, phase, site, i, j, bit) on Q (sites A, R, C, K; phases BEFORE_PANEL /
    AFTER_UPDATE of panel t, AT_END).  Returns (Q, info), or (Q, Result) with full=True."""
    import torch
    n, lda = _check_fortran(A)
    ihi = n if ihi is None else ihi
    if Q is None:
        Q = fortran(torch.empty((n, n), dtype=torch.float64, device=A.device))
    _, ldq = _check_fortran(Q, "Q")
    rep = Report()
    o = make_opts(nb=nb, stream=stream, abft=abft, faults=faults, c_thr=c_thr, report=rep, timing=timing)
    info = lib().ft_dorghr(n, ilo, ihi, ctypes.c_void_p(A.data_ptr()), lda, ctypes.c_void_p(tau.data_ptr()),
                           ctypes.c_void_p(Q.data_ptr()), ldq, ctypes.byref(o))
    if full:
        return Q, Result(info, rep, rep.event_list())
    return Q, info


def strerror(info: int) -> str:
    return lib().ft_strerror(info).decode()


def version() -> str:
    return lib().ft_version().decode()


def launch_count(reset: bool = False) -> int:
    return int(lib().ft_launch_count(1 if reset else 0))


def finalize() -> None:
    lib().ft_finalize()


# ---------------------------------------------------------------------------------------
# Multi-GPU: 1-D block-column cyclic layout, block = nb.  Host-side layout
# logic is plain Python (tested with gloo on CPU); the reduction runs in the library.
# ---------------------------------------------------------------------------------------
def default_nb(n: int) -> int:
    """Panel width the library picks for opts.nb = 0 (reading R4)."""
    return 32 if n < 4096 else 64


def cyclic_columns(n: int, nb: int, rank: int, nranks: int) -> list:
    """Global columns of `rank`, in local order: J lives on rank (J // nb) % nranks at local
    column (J // (nb * nranks)) * nb + J % nb (include/ftgehrd.h)."""
    cols = []
    for b in range(rank, (n + nb - 1) // nb, nranks):
        cols.extend(range(b * nb, min(n, (b + 1) * nb)))
    return cols


def global_to_local(J: int, nb: int, nranks: int) -> tuple:
    """(rank, local column) of global column J."""
    return (J // nb) % nranks, (J // (nb * nranks)) * nb + J % nb


def shard(A, nb: int, nranks: int) -> list:
    """Split an n x n matrix (torch or numpy) into the ranks' column-major slabs."""
    n = A.shape[0]
    out = []
    for r in range(nranks):
        idx = cyclic_columns(n, nb, r, nranks)
        sl = A[:, idx]
        if hasattr(sl, "is_cuda"):
            sl = fortran(sl)
        else:
            import numpy as np
            sl = np.asfortranarray(sl)
        out.append(sl)
    return out


def unshard(slabs: list, n: int, nb: int):
    """Inverse of shard (returns a torch tensor on the slabs' device, or numpy)."""
    nranks = len(slabs)
    first = slabs[0]
    if hasattr(first, "is_cuda"):
        import torch
        A = torch.empty((n, n), dtype=first.dtype, device=first.device)
    else:
        import numpy as np
        A = np.empty((n, n), dtype=first.dtype)
    for r in range(nranks):
        idx = cyclic_columns(n, nb, r, nranks)
        if len(idx):
            A[:, idx] = slabs[r][:, : len(idx)]
    return A


def _slab_ld(S, n):
    if n > 1 and S.shape[1] > 1 and S.stride(0) != 1:
        raise ValueError("slabs must be column-major (use fortran())")
    return max(S.stride(1) if S.shape[1] > 1 else n, n, 1)


def dgehrd_vranks(slabs: list, nb: int = 0, abft: bool = True, taus=None, stream=None, faults=(), c_thr=2.0,
                  deterministic=False):
    """Sharded reduction with len(slabs) VIRTUAL ranks on the current GPU (ft_dgehrd_vranks).

    slabs: the ranks' n x ncols CUDA float64 column-major slabs (modified in place).
    faults: (panel, phase, site, i, J, bit) with J a GLOBAL column (sites A, C; the owner's word).
    Returns (taus, Result)."""
    import torch
    G = len(slabs)
    n = slabs[0].shape[0]
    nb_eff = nb if nb > 0 else default_nb(n)
    for r, S in enumerate(slabs):
        if S.shape[1] != len(cyclic_columns(n, nb_eff, r, G)):
            raise ValueError(f"slab {r} has {S.shape[1]} columns, layout needs {len(cyclic_columns(n, nb_eff, r, G))}")
    lda = max(_slab_ld(S, n) for S in slabs)
    if any(_slab_ld(S, n) != lda for S in slabs):
        raise ValueError("all slabs must share one leading dimension")
    if taus is None:
        taus = [torch.zeros(max(n - 1, 1), dtype=torch.float64, device=slabs[0].device) for _ in range(G)]
    pa = (ctypes.c_void_p * G)(*[S.data_ptr() for S in slabs])
    pt = (ctypes.c_void_p * G)(*[t.data_ptr() for t in taus])
    rep = Report()
    o = make_opts(nb=nb, abft=abft, report=rep, stream=stream, faults=faults, c_thr=c_thr, deterministic=deterministic)
    info = lib().ft_dgehrd_vranks(n, 1, n, pa, lda, pt, G, ctypes.byref(o))
    return taus, Result(info, rep, rep.event_list())


def exchange_handles(local: bytes, group=None) -> list:
    """All-gather each rank's 64-byte IPC handle over torch.distributed (any backend)."""
    import torch.distributed as dist
    out = [None] * dist.get_world_size(group)
    dist.all_gather_object(out, bytes(local), group=group)
    return out


def mgpu_init(n_max: int, group=None) -> None:
    """Bootstrap of the multi-GPU path for this process's rank (one process per GPU)."""
    import torch.distributed as dist
    rank, nranks = dist.get_rank(group), dist.get_world_size(group)
    h = IpcHandle()
    info = lib().ft_mgpu_setup(n_max, rank, nranks, ctypes.byref(h))
    if info:
        raise RuntimeError(f"ft_mgpu_setup: {strerror(info)}")
    # the raw 64 bytes (ctypes' c_char-array value would stop at the first NUL byte of the handle)
    hs = exchange_handles(ctypes.string_at(ctypes.addressof(h), 64), group)
    arr = (IpcHandle * nranks)()
    for g, b in enumerate(hs):
        ctypes.memmove(ctypes.byref(arr[g]), b, 64)
    info = lib().ft_mgpu_connect(arr, rank, nranks)
    if info:
        raise RuntimeError(f"ft_mgpu_connect: {strerror(info)}")


def dgehrd_mgpu(slab, rank: int, nranks: int, nb: int = 0, abft: bool = True, tau=None, stream=None, faults=(),
                deterministic=False):
    """This rank's part of the sharded reduction (after mgpu_init). Returns (tau, Result)."""
    import torch
    n = slab.shape[0]
    lda = _slab_ld(slab, n)
    if tau is None:
        tau = torch.zeros(max(n - 1, 1), dtype=torch.float64, device=slab.device)
    rep = Report()
    o = make_opts(nb=nb, abft=abft, report=rep, stream=stream, faults=faults, deterministic=deterministic)
    info = lib().ft_dgehrd_mgpu(n, 1, n, ctypes.c_void_p(slab.data_ptr()), lda, ctypes.c_void_p(tau.data_ptr()),
                                rank, nranks, ctypes.byref(o))
    return tau, Result(info, rep, rep.event_list())
