"""Multi-rank host logic on CPU (gloo, world size 2) and the edge partition of SURVEY.md 8(e).

* ``reduce_counts`` (the one exchange of the multi-GPU path): per-rank shard counts of the
  oracle (shard = the same round-robin rule the kernel uses) sum to the full
  count, and one failed rank (TDFS_COUNT_INVALID) makes every rank raise -- never a partial sum.
* ``tdfs_partition_edges`` (host C-ABI, no GPU): round-robin is e mod W; degree-balanced
  assigns every directed edge to exactly one rank, keeps light roots whole, deals heavy roots
  edge by edge, and balances the per-rank root cost on a skewed R-MAT graph.
"""
import os
import socket

import numpy as np
import pytest
import torch
import torch.multiprocessing as mp

import oracle as O
import tdfs_inputs as T
import paper_conf_icde_yuan0ha0024_b200 as M


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


NAMES = ["triangle", "diamond", "house"]


def _worker(rank, world, port, out, fail_rank):
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port), RANK=str(rank), WORLD_SIZE=str(world))
    from paper_conf_icde_yuan0ha0024_b200 import dist as D
    D.init_process_group("gloo")
    g = T.rmat(9, 8, 3)
    local = torch.tensor([O.count(g, T.query(n), "auto", shard=(rank, world)) for n in NAMES], dtype=torch.int64)
    out[rank] = D.reduce_counts(local.clone()).tolist()
    # a failed job on one rank: every rank raises
    bad = local.clone()
    if rank == fail_rank:
        bad[1] = D.COUNT_INVALID_I64
    try:
        D.reduce_counts(bad)
        out[f"raised{rank}"] = False
    except RuntimeError:
        out[f"raised{rank}"] = True
    torch.distributed.destroy_process_group()


def test_gloo_reduce_counts_and_failure_propagation():
    world = 2
    port = _free_port()
    mgr = mp.Manager()
    out = mgr.dict()
    mp.spawn(_worker, args=(world, port, out, 1), nprocs=world, join=True)
    g = T.rmat(9, 8, 3)
    ref = [O.count(g, T.query(n), "auto") for n in NAMES]
    assert out[0] == out[1] == ref
    assert out["raised0"] and out["raised1"]


def _csr(g):
    return T.to_csr(g)


@pytest.mark.parametrize("world", [1, 2, 3, 8])
def test_partition_round_robin_is_e_mod_w(world):
    offs, adj = _csr(T.rmat(8, 6, 2))
    own = M.tdfs_partition_edges(offs, adj, world, M.TDFS_SHARD_ROUND_ROBIN)
    assert np.array_equal(own, np.arange(adj.shape[0]) % world)


@pytest.mark.parametrize("world", [1, 2, 4, 8])
def test_partition_degree_balanced(world):
    g = T.rmat(12, 16, 9)
    offs, adj = _csr(g)
    own = M.tdfs_partition_edges(offs, adj, world, M.TDFS_SHARD_DEGREE_BALANCED)
    assert own.shape == adj.shape and own.min() >= 0 and own.max() < world  # a partition of the edges
    deg = np.diff(offs)
    src = np.repeat(np.arange(g.n), deg)
    cost = np.zeros(g.n, dtype=np.float64)
    np.add.at(cost, src, deg[adj].astype(np.float64))  # c(v) = sum of neighbour degrees
    heavy = cost > cost.sum() / (64 * world)
    # light roots are dealt whole
    light_e = ~heavy[src]
    first = own[offs[src[light_e]]]
    assert np.array_equal(own[light_e], first)
    # heavy roots are dealt edge by edge round-robin over the heavy edges (in CSR order)
    he = np.nonzero(heavy[src])[0]
    assert np.array_equal(own[he], np.arange(he.shape[0]) % world)
    # balance of the cost proxy: every rank within 5% of the mean
    per_edge = deg[adj].astype(np.float64)
    load = np.bincount(own, weights=per_edge, minlength=world)
    assert load.max() <= 1.05 * load.mean(), load


@pytest.mark.parametrize("world", [1, 3, 8])
def test_partition_blocked(world):
    """TDFS_SHARD_BLOCKED: blocks of 1024 consecutive directed edges dealt round-robin (R36)."""
    offs, adj = _csr(T.rmat(11, 8, 2))
    own = M.tdfs_partition_edges(offs, adj, world, M.TDFS_SHARD_BLOCKED)
    assert np.array_equal(own, (np.arange(adj.shape[0]) // M.TDFS_SHARD_BLOCK_EDGES) % world)


def test_partition_errors():
    offs, adj = _csr(T.rmat(6, 4, 1))
    with pytest.raises(M.TdfsError):
        M.tdfs_partition_edges(offs, adj, 0)
    with pytest.raises(M.TdfsError):
        M.tdfs_partition_edges(offs, adj, 2, 7)
