"""The real-rank bootstrap of the multi-GPU path with two PROCESSES (one GPU box suffices): each
process allocates its symmetric region (ft_mgpu_setup), the CUDA IPC handles are all-gathered over
torch.distributed (gloo), every process maps its peer's region (ft_mgpu_connect, cudaIpcOpenMemHandle)
and writes into it through the mapping; after a barrier each reads what its peer wrote.  No persistent
kernel runs here: two processes' kernels are not co-resident on one GPU without MPS, and the exchange
kernels spin on peer flags."""
import ctypes
import os
import socket

import numpy as np
import pytest

pytestmark = pytest.mark.gpu

torch = pytest.importorskip("torch")
if not torch.cuda.is_available():  # pragma: no cover
    pytest.skip("needs a CUDA device", allow_module_level=True)


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _worker(rank, world, port, q):
    try:
        import sys
        sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
        import torch
        import torch.distributed as dist

        import paper_conf_ipps_jiald16_b200 as ft
        os.environ["MASTER_ADDR"] = "127.0.0.1"
        os.environ["MASTER_PORT"] = str(port)
        dist.init_process_group("gloo", rank=rank, world_size=world)
        torch.cuda.set_device(0)
        ft.mgpu_init(64)
        L = ft.lib()
        assert L.ft_mgpu_probe_put(ctypes.c_double(100.0 + rank)) == 0
        dist.barrier()
        out = np.zeros(world)
        assert L.ft_mgpu_probe_get(ctypes.c_void_p(out.ctypes.data)) == 0
        dist.barrier()
        ft.lib().ft_mgpu_finalize()
        dist.destroy_process_group()
        q.put((rank, out.tolist()))
    except Exception as ex:  # pragma: no cover
        q.put((rank, repr(ex)))


def test_two_process_ipc_bootstrap():
    import torch.multiprocessing as mp
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    ps = [ctx.Process(target=_worker, args=(r, 2, port, q)) for r in range(2)]
    for p in ps:
        p.start()
    res = dict(q.get(timeout=300) for _ in ps)
    for p in ps:
        p.join(timeout=60)
    for r in range(2):
        assert isinstance(res[r], list), res[r]
        assert res[r] == [100.0, 101.0], res  # own slot (own write) and the peer's write
