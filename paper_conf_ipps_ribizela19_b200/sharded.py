"""Sharded (multi-GPU) exact selection over torch.distributed.

The level loop, the decisions and the exchanges live in the C++/CUDA library
(``ss_select_sharded``: csrc/sharded.cuh, csrc/dist_kernels.cuh, NCCL through
csrc/comm.cu); this module only creates the communicator: rank 0 of the
process group draws a NCCL unique id, torch.distributed broadcasts it, and
every rank binds it to its context (``ss_comm_init``).

    import torch.distributed as dist, paper_conf_ipps_ribizela19_b200 as ss
    from paper_conf_ipps_ribizela19_b200.sharded import ShardedSelect
    sel = ShardedSelect(ss.Context(local_rank))     # collective
    v = sel.select(shard, k)                        # collective, same k everywhere
"""
from __future__ import annotations

from . import Context, nccl_unique_id


def comm_init_from_process_group(ctx: Context, group=None) -> None:
    """Bind a NCCL communicator spanning `group` (default: the world) to ctx.
    Collective over the group."""
    import torch.distributed as dist
    world = dist.get_world_size(group)
    rank = dist.get_rank(group)
    src = dist.get_global_rank(group, 0) if group is not None else 0
    obj = [nccl_unique_id() if rank == 0 else None]
    dist.broadcast_object_list(obj, src=src, group=group)
    ctx.comm_init(obj[0], world, rank)


class ShardedSelect:
    """Exact selection of a global rank over the union of every rank's shard."""

    def __init__(self, ctx: Context, group=None):
        self.ctx = ctx
        comm_init_from_process_group(ctx, group)

    def select(self, shard, k: int):
        return self.ctx.select_sharded(shard, k)

    def stats(self) -> dict:
        return self.ctx.stats()
