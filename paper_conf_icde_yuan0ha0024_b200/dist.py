"""Multi-GPU driver: one process per GPU, initial edge tasks partitioned across ranks, one
all-reduce of the match count.

The paper assigns initial edges to GPUs round-robin ("the i-th edge is assigned to the
(i mod NUM_GPU)-th GPU") and does no migration among GPUs.
Each rank runs the full single-GPU hot path on its shard (``shard_rank`` / ``shard_world`` /
``shard_policy`` in tdfs_run_opts: round-robin, or degree-balanced roots, R31);
the only exchange is the sum of the per-rank counts: one ``torch.distributed.all_reduce``
over NCCL (NVLink 5 / NVSwitch) of {count, failed} -- latency-bound (16 bytes), so there is
no compute to fuse it with.  A failed rank (its kernel wrote TDFS_COUNT_INVALID, e.g. stack
pool exhausted) makes every rank raise instead of returning a partial sum.

Cross-GPU dynamic balancing: ``count_balanced`` maps one chunk
cursor in rank 0's HBM into every rank (CUDA IPC + peer access over NVLink), and every rank's
persistent kernel takes edge chunks from it with system-scope atomics until all edges are
taken -- a rank that finishes early keeps taking chunks instead of idling.
"""
from __future__ import annotations

import os
from typing import Optional

import torch
import torch.distributed as dist

COUNT_INVALID_I64 = -1  # TDFS_COUNT_INVALID (~0 as uint64) read through an int64 view


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


def reduce_counts(local: torch.Tensor, group=None) -> torch.Tensor:
    """All-reduce per-rank int64 counts (any shape, e.g. one per query) together with a
    per-element failure flag (a local value of TDFS_COUNT_INVALID).  Returns the int64 sums;
    raises RuntimeError on every rank if any rank failed for any element."""
    assert local.dtype == torch.int64
    bad = (local == COUNT_INVALID_I64).to(torch.int64)
    buf = torch.stack([torch.where(bad.bool(), torch.zeros_like(local), local), bad])
    if dist.is_initialized() and dist.get_world_size(group) > 1:
        dist.all_reduce(buf, op=dist.ReduceOp.SUM, group=group)
    if int(buf[1].sum().item()) != 0:
        failed = [i for i, x in enumerate(buf[1].reshape(-1).tolist()) if x]
        raise RuntimeError(f"tdfs: a rank's job failed (TDFS_COUNT_INVALID) for element(s) {failed}; no count")
    return buf[0]


def _copy_opts(opts):
    import paper_conf_icde_yuan0ha0024_b200 as M
    return M.default_opts() if opts is None else M.tdfs_run_opts.from_buffer_copy(opts)


def count_sharded(graph, plan, opts=None, group=None, workspace=None, stream=None, policy: Optional[int] = None) -> int:
    """This rank's shard of the count on its GPU (static partition), then the checked all-reduce.
    The caller's opts are not modified."""
    import paper_conf_icde_yuan0ha0024_b200 as M

    o = _copy_opts(opts)
    if dist.is_initialized():
        o.shard_rank = dist.get_rank(group)
        o.shard_world = dist.get_world_size(group)
    if policy is not None:
        o.shard_policy = policy
    d_count = torch.zeros(1, dtype=torch.int64, device=f"cuda:{graph.device}")
    M.tdfs_count(graph, plan, o, workspace=workspace, stream=stream, d_count=d_count, sync=False)
    return int(reduce_counts(d_count, group).item())


class SharedCursorGroup:
    """Rank 0 creates the cursor, the other ranks open it (IPC handle broadcast over the
    process group).  Reusable across jobs: ``prepare`` zeroes it and fences all ranks."""

    def __init__(self, device: int, group=None):
        import paper_conf_icde_yuan0ha0024_b200 as M

        self.group = group
        self.device = device
        rank = dist.get_rank(group) if dist.is_initialized() else 0
        obj = [None]
        if rank == 0:
            self.cursor = M.SharedCursor(device)
            obj[0] = self.cursor.handle
        if dist.is_initialized():
            dist.broadcast_object_list(obj, src=0, group=group)
        if rank != 0:
            self.cursor = M.SharedCursor(device, obj[0])
        self.rank = rank

    def prepare(self, stream=None):
        """Zero the cursor (rank 0) and make sure every rank sees it zeroed before launching."""
        if self.rank == 0:
            self.cursor.reset(stream)
            torch.cuda.current_stream(self.device).synchronize() if stream is None else stream.synchronize()
        if dist.is_initialized():
            dist.barrier(group=self.group)

    def finish(self):
        """Every rank's job has completed (call after the kernels are done) before the next reset."""
        torch.cuda.synchronize(self.device)
        if dist.is_initialized():
            dist.barrier(group=self.group)

    def close(self):
        self.cursor.close()


def count_balanced(graph, plan, cursors: SharedCursorGroup, opts=None, group=None, workspace=None,
                   stream=None) -> int:
    """Cross-GPU dynamically balanced count (NEXT-3): every rank's kernel takes chunks of ALL
    directed edges from the shared cursor; the per-rank counts are summed by the checked
    all-reduce."""
    import paper_conf_icde_yuan0ha0024_b200 as M

    o = _copy_opts(opts)
    o.shared_cursor = cursors.cursor.ptr
    d_count = torch.zeros(1, dtype=torch.int64, device=f"cuda:{graph.device}")
    cursors.prepare(stream)
    M.tdfs_count(graph, plan, o, workspace=workspace, stream=stream, d_count=d_count, sync=False)
    cursors.finish()
    return int(reduce_counts(d_count, group).item())
