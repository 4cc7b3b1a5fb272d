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


def allreduce_count(count: int, group=None, device=None, ctx=None) -> int:
    """Exact sum over ranks of a non-negative integer < 2^128.  With a context that
    joined a world (``Cuts.set_dist``) the library's own NCCL all-reduce does it
    (cuts_allreduce_count); otherwise 32-bit limbs in int64 over torch.distributed."""
    if count < 0 or count >= 1 << (_LIMB * _NLIMB):
        raise ValueError("count out of range")
    if ctx is not None and getattr(ctx, "world", 1) > 1:
        return ctx.allreduce_count(count)
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


# ---------------------------------------------------------------------------
# Dynamic redistribution of unfinished trie work (Alg. 3; protocol
# P:1188-1207).  Control plane: the process-group store (atomic add /
# compare_set), standing in for the paper's MPI free/busy messages.  Data plane:
# point-to-point send/recv of flat prefixes (NCCL over NVLink for device tensors,
# gloo for host tensors).  The engine (libcuts via ``CutsEngine``) calls
# ``poll`` at chunk boundaries and ``ship`` with the exported prefixes.
#
# Invariant for termination: ``fin`` counts ranks that are idle AND have no
# donation addressed to them.  An idle rank adds 1; a donor that claims it
# subtracts 1 *before* shipping (the donor is itself not idle, so fin < world
# throughout).  Hence fin == world is stable: nobody holds or is owed work.
class WorkSharing:
    def __init__(self, store, tag: str, rank: int, world: int, engine, *,
                 interval: float = 0.002, transport_device=None, group=None, min_give: int = 1):
        import time
        self.store, self.tag, self.rank, self.world = store, tag, rank, world
        self.engine = engine
        self.interval = interval
        self.dev = transport_device          # None: ship host tensors (gloo)
        self.group = group
        self.min_give = min_give
        self._clock = time.monotonic
        self._last = -1e9
        self._target = None                  # (receiver, epoch) claimed by the last poll
        self.epoch = 0
        self.sent = 0                        # donations made
        self.sent_rows = 0
        self.received = 0
        self._pending = []                   # in-flight isend works (+ their tensors)
        import os
        self._log = open(f"/tmp/ws_trace_{rank}.log", "w") if os.environ.get("CUTS_WS_TRACE") else None

    def _t(self, *a):
        if self._log:
            self._log.write(f"{self._clock():.4f} r{self.rank} " + " ".join(str(x) for x in a) + "\n")
            self._log.flush()

    def _k(self, *parts):
        return "/".join((self.tag,) + tuple(str(p) for p in parts))

    # ------------------------------------------------------------ donor side
    def poll(self, depth: int, remaining: int) -> int:
        """Called by the engine at a chunk boundary: entries of `depth` to give away."""
        # donate half, keep half: a rank never gives away its last
        # unstarted entry, so a piece cannot bounce between idle ranks forever
        if self.world == 1 or remaining < 2 * self.min_give:
            return 0
        now = self._clock()
        if now - self._last < self.interval:
            return 0
        self._last = now
        if int(self.store.add(self._k("nwant"), 0)) <= 0:
            return 0
        for off in range(1, self.world):
            r = (self.rank + off) % self.world
            wk = self._k("want", r)
            if not self.store.check([wk]):
                continue
            e = int(self.store.get(wk))
            if e <= 0:
                continue
            self._nclaim = getattr(self, "_nclaim", 0) + 1
            me = f"{self.rank}.{self._nclaim}".encode()     # unique: a re-read of our own old claim never matches
            got = self.store.compare_set(self._k("claim", r, e), "", me)
            if got != me:
                continue
            # claimed: r is no longer idle; count it busy before shipping
            self.store.add(self._k("nwant"), -1)
            self.store.add(self._k("fin"), -1)
            self._target = (r, e)
            self._t("claim", r, e, "depth", depth, "rem", remaining)
            return remaining // 2
        return 0

    def ship(self, depth: int, rows):
        """Called by the engine with the exported (give, depth) int32 prefix rows."""
        import torch
        import torch.distributed as dist
        r, e = self._target
        self._target = None
        if rows is None or rows.shape[0] == 0:     # the engine could not export: release the claim
            self.store.set(self._k("gift", r, e), f"{self.rank},{depth},0")
            return
        t = rows.contiguous()
        t = t.to(self.dev) if self.dev is not None else t.cpu()
        self.store.set(self._k("gift", r, e), f"{self.rank},{depth},{t.shape[0]}")
        self._t("send", r, e, tuple(t.shape))
        dist.send(t, dst=r, group=self.group)
        self._t("sent", r, e)
        self.sent += 1
        self.sent_rows += t.shape[0]
        del torch

    # ---------------------------------------------------------- receiver side
    def _go_idle(self):
        self.epoch += 1
        self.store.set(self._k("want", self.rank), str(self.epoch))
        self.store.add(self._k("nwant"), 1)
        self.store.add(self._k("fin"), 1)

    def idle_loop(self) -> int:
        """After the local roots ran out: receive donations until global termination."""
        import time
        import torch
        import torch.distributed as dist
        total = 0
        while True:
            self._go_idle()
            gk = self._k("gift", self.rank, self.epoch)
            self._t("idle", self.epoch, "fin", int(self.store.add(self._k("fin"), 0)))
            while True:
                if self.store.check([gk]):
                    src, depth, cnt = (int(x) for x in self.store.get(gk).decode().split(","))
                    if cnt == 0:
                        break
                    buf = torch.empty((cnt, depth), dtype=torch.int32,
                                      device=self.dev if self.dev is not None else "cpu")
                    self._t("recv", src, depth, cnt)
                    dist.recv(buf, src=src, group=self.group)
                    self._t("got", src)
                    self.received += 1
                    total += self.engine.count_prefixes(buf)
                    break
                if int(self.store.add(self._k("fin"), 0)) >= self.world:
                    return total
                time.sleep(self.interval / 2)

    def run(self, queue, chunk_size: int) -> int:
        """This rank's share: pull root chunks, then serve as a receiver (Alg. 3)."""
        total = 0
        self.engine.set_hooks(self.poll, self.ship)
        try:
            while (ch := queue.next()) is not None:
                b, e = chunk_bounds(ch, chunk_size)
                total += self.engine.count_roots(b, e)
            total += self.idle_loop()
        finally:
            self.engine.set_hooks(None, None)
        return total


class CutsEngine:
    """libcuts behind the WorkSharing engine interface (count-only, HYBRID)."""

    def __init__(self, ctx, mode: str = "hybrid"):
        self.ctx = ctx
        self.mode = mode
        self.stats = []

    def set_hooks(self, poll, ship):
        self.ctx.set_donation(poll, ship)

    def count_roots(self, begin: int, end: int) -> int:
        self.ctx.set_prefixes(None)
        self.ctx.set_root_slice(begin, end, 0, 1)
        c = self.ctx.count(self.mode)
        self.stats.append(self.ctx.stats())
        return c

    def count_prefixes(self, rows) -> int:
        rows = rows.to(self.ctx.device)      # set_prefixes orders the library's stream after this copy
        self.ctx.set_prefixes(rows)
        try:
            c = self.ctx.count(self.mode)
            self.stats.append(self.ctx.stats())
        finally:
            self.ctx.set_prefixes(None)
        return c
