"""The multi-GPU path itself: world size 2, each
rank runs graphb.balance() -- gb_balance_range over its tree shard
{t : t mod W == rank} on the GPU, then one all-reduce of the [cnt | agree]
buffer -- and the result must equal the oracle's frustration cloud on every
rank.  NCCL when the box has >= 2 GPUs; otherwise both ranks share cuda:0
and the all-reduce goes through gloo (CUDA tensors)."""
from __future__ import annotations

import os
import socket

import numpy as np
import pytest

pytestmark = pytest.mark.gpu


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _worker(rank, world, port, T, seed, out):
    from datetime import timedelta
    import torch
    import torch.distributed as dist
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    ndev = torch.cuda.device_count()
    torch.cuda.set_device(rank % ndev)
    backend = "nccl" if ndev >= world else "gloo"
    # a rank that dies must not leave the other waiting forever
    if backend == "nccl":
        dist.init_process_group("nccl", rank=rank, world_size=world, timeout=timedelta(seconds=300),
                                device_id=torch.device("cuda", rank % ndev))
    else:
        dist.init_process_group("gloo", rank=rank, world_size=world, timeout=timedelta(seconds=300))
    try:
        import graphgen
        from paper_conf_sc_alabanditrb21_b200 import graphb
        g = graphgen.chung_lu(20000, 90000, 900, 0.75, 0.3, 5)
        graphb.load_graph(g)
        cnt, agree = graphb.balance(T, seed)
        st = graphb.stats()
        out[rank] = (cnt.copy(), agree.copy(), backend, st["trees"])
        graphb.free()
    finally:
        dist.destroy_process_group()


@pytest.mark.parametrize("world,T", [(2, 9), (2, 70)])
def test_sharded_balance_on_gpu_equals_oracle(world, T):
    import torch.multiprocessing as mp
    import graphgen
    import oracle
    seed = 3
    port = _free_port()
    mgr = mp.get_context("spawn").Manager()
    out = mgr.dict()
    mp.start_processes(_worker, args=(world, port, T, seed, out), nprocs=world, join=True,
                       start_method="spawn")
    g = graphgen.chung_lu(20000, 90000, 900, 0.75, 0.3, 5)
    c, a = oracle.Graph.from_csr(g).balance(T, seed)
    for r in range(world):
        cnt, agree, backend, trees = out[r]
        assert cnt.dtype == np.uint32 and agree.dtype == np.uint32
        assert len(cnt) == g.m and len(agree) == g.n
        assert trees == len(range(r, T, world))          # rank r balanced its own shard only
        assert np.array_equal(cnt, c), (r, backend)
        assert np.array_equal(agree, a), (r, backend)
