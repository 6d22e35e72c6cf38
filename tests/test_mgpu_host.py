"""Host-side logic of the multi-GPU path (no GPU): the 1-D block-column cyclic layout and the
bootstrap exchange of IPC handles, including a world-size-2 gloo run on 127.0.0.1."""
import os
import socket

import numpy as np
import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp

from paper_conf_ipps_jiald16_b200 import ftgehrd as F


@pytest.mark.parametrize("n,nb,G", [(64, 16, 2), (100, 32, 3), (517, 32, 4), (40000, 64, 8), (5, 16, 8)])
def test_layout_partition(n, nb, G):
    seen = []
    for r in range(G):
        cols = F.cyclic_columns(n, nb, r, G)
        assert cols == sorted(cols)
        for loc, J in enumerate(cols):
            assert F.global_to_local(J, nb, G) == (r, loc)
        seen += cols
    assert sorted(seen) == list(range(n))


def cmap_c(l, G, rank, nb, ncl, n):
    """The device-side map ft_cmap of ft_internal.h, retyped (local column -> global)."""
    if G <= 1:
        return l
    if l == ncl:
        return n
    return (l // nb) * nb * G + rank * nb + l % nb


@pytest.mark.parametrize("n,nb,G", [(130, 16, 2), (517, 32, 3), (2048, 32, 8)])
def test_device_map_agrees(n, nb, G):
    for r in range(G):
        cols = F.cyclic_columns(n, nb, r, G)
        for l, J in enumerate(cols):
            assert cmap_c(l, G, r, nb, len(cols), n) == J
        assert cmap_c(len(cols), G, r, nb, len(cols), n) == n  # the replicated r column


def test_shard_unshard_roundtrip():
    A = np.asfortranarray(np.arange(37 * 37, dtype=np.float64).reshape(37, 37))
    for G in (1, 2, 3, 5):
        sl = F.shard(A, 8, G)
        assert all(s.flags["F_CONTIGUOUS"] for s in sl)
        assert np.array_equal(F.unshard(sl, 37, 8), A)
        assert sum(s.shape[1] for s in sl) == 37


def _free_port():
    with socket.socket() as s:
        s.bind(("127.0.0.1", 0))
        return s.getsockname()[1]


def _worker(rank, world, port, q):
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        # the bootstrap all-gather of 64-byte handles (fake handle bytes on CPU)
        mine = bytes([rank + 1]) * 64
        hs = F.exchange_handles(mine)
        ok = hs == [bytes([g + 1]) * 64 for g in range(world)]
        # each rank's slab of the same seeded matrix; allgather and reassemble
        n, nb = 50, 8
        A = np.asfortranarray(np.random.default_rng(3).standard_normal((n, n)))
        slab = F.shard(A, nb, world)[rank]
        parts = [None] * world
        dist.all_gather_object(parts, slab)
        ok = ok and np.array_equal(F.unshard(parts, n, nb), A)
        q.put((rank, ok))
    finally:
        dist.destroy_process_group()


def test_gloo_world2_bootstrap_and_layout():
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    ps = [ctx.Process(target=_worker, args=(r, 2, port, q)) for r in range(2)]
    for p in ps:
        p.start()
    res = dict(q.get(timeout=120) for _ in ps)
    for p in ps:
        p.join(timeout=60)
    assert res == {0: True, 1: True}
