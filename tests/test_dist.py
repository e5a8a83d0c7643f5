"""World-size-2 gloo test of the multi-GPU host logic on CPU: shards partition the initial
edge tasks, and the single all-reduce of the per-rank counts gives the full count.
The per-rank counts come from the oracle's shard restriction (same round-robin rule
as the kernel's), so this exercises the product's exchange path without
a GPU."""
import os
import socket

import pytest
import torch
import torch.multiprocessing as mp

import oracle as O
import tdfs_inputs as T


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _worker(rank, world, port, out):
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port), RANK=str(rank), WORLD_SIZE=str(world))
    from paper_conf_icde_yuan0ha0024_b200 import dist as D
    D.init_process_group("gloo")
    g = T.rmat(9, 8, 3)
    res = {}
    for name in ["triangle", "diamond", "house"]:
        q = T.query(name)
        local = O.count(g, q, "auto", shard=(rank, world))
        t = torch.tensor([local], dtype=torch.int64)
        D.allreduce_count(t)
        res[name] = int(t.item())
    out[rank] = res
    torch.distributed.destroy_process_group()


@pytest.mark.parametrize("world", [2])
def test_gloo_sharded_allreduce(world):
    port = _free_port()
    mgr = mp.Manager()
    out = mgr.dict()
    mp.spawn(_worker, args=(world, port, out), nprocs=world, join=True)
    g = T.rmat(9, 8, 3)
    for name in ["triangle", "diamond", "house"]:
        ref = O.count(g, T.query(name), "auto")
        assert out[0][name] == out[1][name] == ref


def test_shards_partition_edges():
    from paper_conf_icde_yuan0ha0024_b200 import dist as D
    for nnz in (0, 1, 7, 100):
        for w in (1, 2, 3, 8):
            assert D.ranks_cover_all_edges(nnz, w)
