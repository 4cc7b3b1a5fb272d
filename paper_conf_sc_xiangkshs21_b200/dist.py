"""Multi-GPU orchestration: root partition, dynamic root-chunk queue, count reduction.

One process per GPU (torchrun).  The data graph is replicated on every rank
(Alg. 3 gives every rank Q and D); the units of work are level-1
roots — independent sub-tries whose counts add up (|V_D|/nGPU
roots per GPU).  Two ways to hand them out:

* static: rank r takes the cyclic slice p % world == r of the seeded-shuffled
  level-1 list (``static_slice``);
* dynamic (``RootQueue``): the shuffled list is cut into chunks and every rank
  pulls the next chunk index from a shared atomic counter (the torch.distributed
  store's ``add``) until the queue is empty — the free/busy protocol of Alg. 3
   reduced to pull-based work sharing at root granularity.

The only data-path collective is the final sum of counts (``allreduce_count``),
exact for any 128-bit total (four 32-bit limbs summed in int64).
This module holds orchestration only: every count is computed by libcuts.so.
"""
from __future__ import annotations

import torch
import torch.distributed as dist

_LIMB = 32
_NLIMB = 4          # 128-bit counts
_MASK = (1 << _LIMB) - 1


def static_slice(rank: int, world: int):
    """(begin, end, part, nparts) for cuts_set_root_slice: cyclic over the shuffled list."""
    if not (0 <= rank < world):
        raise ValueError("rank out of range")
    return 0, 2**64 - 1, rank, world


def chunk_bounds(chunk: int, chunk_size: int):
    """Shuffled-list positions [begin, end) of a dynamic-queue chunk."""
    return chunk * chunk_size, (chunk + 1) * chunk_size


def n_chunks(level1: int, chunk_size: int) -> int:
    return (level1 + chunk_size - 1) // chunk_size if chunk_size > 0 else 0


def allreduce_count(count: int, group=None, device=None) -> int:
    """Exact sum over ranks of a non-negative integer < 2^128 (limbs of 32 bits in int64)."""
    if count < 0 or count >= 1 << (_LIMB * _NLIMB):
        raise ValueError("count out of range")
    if not dist.is_available() or not dist.is_initialized() or dist.get_world_size(group) == 1:
        return count
    limbs = [(count >> (_LIMB * i)) & _MASK for i in range(_NLIMB)]
    t = torch.tensor(limbs, dtype=torch.int64, device=device if device is not None else "cpu")
    dist.all_reduce(t, op=dist.ReduceOp.SUM, group=group)   # <= world * 2^32 per limb: no overflow
    return sum(int(v) << (_LIMB * i) for i, v in enumerate(t.tolist()))


def allreduce_max(x: float, group=None, device=None) -> float:
    if not dist.is_available() or not dist.is_initialized() or dist.get_world_size(group) == 1:
        return x
    t = torch.tensor([x], dtype=torch.float64, device=device if device is not None else "cpu")
    dist.all_reduce(t, op=dist.ReduceOp.MAX, group=group)
    return float(t.item())


class RootQueue:
    """Shared queue of root chunks: ``next()`` returns a chunk index or None.

    Backed by the process group's store (``add`` is an atomic fetch-and-add on the
    rendezvous server), so any rank that runs out of work keeps pulling chunks a
    busy rank has not started yet.  ``key`` must be unique per (query, pass).
    """

    def __init__(self, store, key: str, total_chunks: int):
        self.store = store
        self.key = key
        self.total = total_chunks

    def next(self):
        if self.total <= 0:
            return None
        c = int(self.store.add(self.key, 1)) - 1
        return c if c < self.total else None


def default_store():
    """The default process group's store (torchrun / init_process_group)."""
    from torch.distributed import distributed_c10d as c10d
    return c10d._get_default_store()
