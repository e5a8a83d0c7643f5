"""The multi-GPU path through the product on one B200: two ranks (processes) on cuda:0 with a
gloo process group over CUDA tensors.  Each rank runs dist.count_sharded (static round-robin or
degree-balanced shards, R31) or dist.count_balanced (both kernels take
edge chunks from one shared cursor in rank 0's memory mapped by CUDA IPC),
and the checked all-reduce must give the oracle's full count on every rank."""
import os
import socket

import pytest
import torch
import torch.multiprocessing as mp

import oracle as O
import tdfs_inputs as T

pytestmark = pytest.mark.gpu

NAMES = ["triangle", "c4", "diamond", "house"]


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _worker(rank, world, port, out):
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port), RANK=str(rank), WORLD_SIZE=str(world))
    import paper_conf_icde_yuan0ha0024_b200 as M
    from paper_conf_icde_yuan0ha0024_b200 import dist as D
    torch.cuda.set_device(0)
    D.init_process_group("gloo")
    g = T.rmat(11, 12, 4)
    h = M.tdfs_load_edges(g.n, g.edges, device=0)
    cur = D.SharedCursorGroup(0)
    res = {}
    for name in NAMES:
        p = M.plan_from_query(T.query(name))
        o = M.default_opts(tau_ms=1.0, chunk=2)
        res[name] = (D.count_sharded(h, p, o), D.count_sharded(h, p, o, policy=M.TDFS_SHARD_DEGREE_BALANCED),
                     D.count_sharded(h, p, o, policy=M.TDFS_SHARD_BLOCKED),
                     D.count_balanced(h, p, cur, o), D.count_balanced(h, p, cur, o))
        assert o.shard_world == 1 and o.shared_cursor is None  # caller's opts untouched
    cur.close()
    out[rank] = res
    torch.distributed.destroy_process_group()


def test_two_ranks_on_one_gpu_sharded_and_shared_cursor():
    world = 2
    port = _free_port()
    mgr = mp.Manager()
    out = mgr.dict()
    mp.spawn(_worker, args=(world, port, out), nprocs=world, join=True)
    g = T.rmat(11, 12, 4)
    for name in NAMES:
        ref = O.count(g, T.query(name), "auto", threads=8)
        for r in range(world):
            assert out[r][name] == (ref,) * 5, (name, r, out[r][name], ref)
