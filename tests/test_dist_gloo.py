"""The N>1 host path on CPU: world_size 2 over gloo (127.0.0.1).  Each rank
balances its tree shard {t : t mod W == rank} -- here with the
oracle standing in for the device range call, since there is no GPU -- and
graphb.sharded_balance all-reduces the concatenated counters.  The result must
equal the single-process frustration cloud on every rank."""
from __future__ import annotations

import os
import socket

import numpy as np
import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _worker(rank, world, port, T, seed, out):
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        import graphgen
        import oracle
        from paper_conf_sc_alabanditrb21_b200.graphb import sharded_balance
        g = graphgen.chung_lu(3000, 12000, 400, 0.75, 0.3, 2)
        og = oracle.Graph.from_csr(g)
        seen = []

        def range_fn(t_begin, t_end, stride, s):
            seen.append((t_begin, t_end, stride))
            c, a = og.balance(t_end, s, t_begin=t_begin, stride=stride)
            return torch.from_numpy(np.concatenate([c, a]).astype(np.int32))

        cnt, agree = sharded_balance(T, seed, rank, world, range_fn, g.m)
        assert seen == [(rank, T, world)]
        out[rank] = (cnt.numpy().copy(), agree.numpy().copy())
    finally:
        dist.destroy_process_group()


@pytest.mark.parametrize("world", [2])
def test_gloo_sharded_cloud_equals_single_process(world):
    import graphgen
    import oracle
    T, seed = 10, 4
    port = _free_port()
    mgr = mp.get_context("spawn").Manager()
    out = mgr.dict()
    mp.start_processes(_worker, args=(world, port, T, seed, out), nprocs=world, join=True,
                       start_method="spawn")
    g = graphgen.chung_lu(3000, 12000, 400, 0.75, 0.3, 2)
    c, a = oracle.Graph.from_csr(g).balance(T, seed)
    for r in range(world):
        assert np.array_equal(out[r][0].astype(np.uint32), c)
        assert np.array_equal(out[r][1].astype(np.uint32), a)
