"""Multi-GPU driver: one process per GPU, initial edge tasks sharded across ranks, one
all-reduce of the match count.

The paper assigns initial edges to GPUs round-robin ("the i-th edge is assigned to the
(i mod NUM_GPU)-th GPU") and does no migration among GPUs.
Each rank runs the full single-GPU hot path on its shard (``shard_rank`` /
``shard_world`` in tdfs_run_opts); the only exchange is the sum of the per-rank counts:
one ``torch.distributed.all_reduce`` of an int64 over NCCL (NVLink 5 / NVSwitch) --
latency-bound (8 bytes), so there is no compute to fuse it with.
"""
from __future__ import annotations

import os
from typing import Optional

import torch
import torch.distributed as dist


def env_rank_world():
    return int(os.environ.get("RANK", "0")), int(os.environ.get("WORLD_SIZE", "1")), \
        int(os.environ.get("LOCAL_RANK", os.environ.get("RANK", "0")))


def init_process_group(backend: str = "nccl") -> None:
    if dist.is_initialized():
        return
    rank, world, local = env_rank_world()
    os.environ.setdefault("MASTER_ADDR", "127.0.0.1")
    os.environ.setdefault("MASTER_PORT", "29531")
    if backend == "nccl":
        torch.cuda.set_device(local)
        dist.init_process_group("nccl", rank=rank, world_size=world, device_id=torch.device("cuda", local))
    else:
        dist.init_process_group(backend, rank=rank, world_size=world)


def allreduce_count(local: torch.Tensor, group=None) -> torch.Tensor:
    """Sum a 1-element int64 count over all ranks, in place (NCCL on GPU tensors, gloo on CPU)."""
    assert local.dtype == torch.int64 and local.numel() == 1
    if dist.is_initialized() and dist.get_world_size(group) > 1:
        dist.all_reduce(local, op=dist.ReduceOp.SUM, group=group)
    return local


def count_sharded(graph, plan, opts=None, group=None, workspace=None, stream=None) -> torch.Tensor:
    """This rank's shard of the count on its GPU, then the all-reduce.  Returns the device
    int64 tensor holding the global count (asynchronous until the caller reads it)."""
    import paper_conf_icde_yuan0ha0024_b200 as M

    opts = opts or M.default_opts()
    if dist.is_initialized():
        opts.shard_rank = dist.get_rank(group)
        opts.shard_world = dist.get_world_size(group)
    d_count = torch.zeros(1, dtype=torch.int64, device=f"cuda:{graph.device}")
    M.tdfs_count(graph, plan, opts, workspace=workspace, stream=stream, d_count=d_count, sync=False)
    return allreduce_count(d_count, group)


def shard_edges(nnz: int, rank: int, world: int):
    """Directed-edge indices of a rank's shard (host-side mirror of the kernel's task mapping)."""
    return range(rank, nnz, world)


def ranks_cover_all_edges(nnz: int, world: int) -> bool:
    seen = []
    for r in range(world):
        seen.extend(shard_edges(nnz, r, world))
    return sorted(seen) == list(range(nnz))
