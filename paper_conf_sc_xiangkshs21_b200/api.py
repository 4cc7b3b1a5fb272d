"""Thin Python API over the C ABI (argument marshalling only).

PyTorch supplies device memory (the arena, the graph, enumeration output) and
the stream; every step of the search runs in libcuts.so's CUDA kernels.

    ctx = Cuts(device=0)                 # arena = most of the free HBM
    ctx.load_graph(row_ptr, col)         # canonical symmetric CSR (numpy or torch)
    ctx.set_query(q_row_ptr, q_col)      # or ctx.set_query_edges(k, edges)
    n = ctx.count("hybrid")              # ordered non-induced embeddings
    rows = ctx.enumerate("bfs", cap)     # (n, k) uint32 on the device, query-id order
"""
from __future__ import annotations

import ctypes

import numpy as np
import torch

from . import _lib as L


class CutsError(RuntimeError):
    def __init__(self, status: int, message: str):
        super().__init__(f"{L.STATUS_NAMES.get(status, status)}: {message}")
        self.status = status
        self.message = message


_MODES = {"bfs": L.CUTS_BFS, "hybrid": L.CUTS_HYBRID, L.CUTS_BFS: L.CUTS_BFS, L.CUTS_HYBRID: L.CUTS_HYBRID}


def _mode(m) -> int:
    try:
        return _MODES[m.lower() if isinstance(m, str) else m]
    except KeyError:
        raise ValueError(f"mode must be 'bfs' or 'hybrid', got {m!r}") from None


def default_arena_bytes(device: int, reserve: int = 4 << 30, fraction: float = 0.9) -> int:
    free, _ = torch.cuda.mem_get_info(device)
    return max(1 << 20, int(min(free - reserve, free * fraction)) & ~0xFFFF)


class _DevRows:
    """A borrowed (count, depth) int32 device buffer exposed to torch without a copy."""

    def __init__(self, ptr: int, count: int, depth: int):
        self.__cuda_array_interface__ = {"shape": (count, depth), "typestr": "<i4", "data": (ptr, False),
                                         "version": 3, "strides": None, "stream": None}


class Cuts:
    """One context on one device: C-ABI handle + torch-owned arena."""

    def __init__(self, device: int = 0, arena_bytes: int | None = None, seed: int = 0x5EED,
                 stream: torch.cuda.Stream | None = None):
        self.lib = L.load()
        if not torch.cuda.is_available():
            raise RuntimeError("libcuts needs a CUDA device (no CPU fallback)")
        self.device = torch.device("cuda", device)
        self.stream = stream if stream is not None else torch.cuda.current_stream(self.device)
        if arena_bytes is None:
            arena_bytes = default_arena_bytes(device)
        self.arena = torch.empty(int(arena_bytes), dtype=torch.uint8, device=self.device)
        opts = L.cuts_opts(device=device, stream=self.stream.cuda_stream, arena=self.arena.data_ptr(),
                           arena_bytes=int(arena_bytes), seed=seed)
        h = ctypes.c_void_p()
        rc = self.lib.cuts_create(ctypes.byref(h), ctypes.byref(opts))
        if rc != 0:
            raise CutsError(rc, "cuts_create failed")
        self.h = h
        self.k = None
        self._graph = None

    # ----------------------------------------------------------------- utils
    def _check(self, rc: int, allow=()):
        if rc != 0 and rc not in allow:
            raise CutsError(rc, self.lib.cuts_last_error(self.h).decode())
        return rc

    def close(self):
        if getattr(self, "h", None):
            self.lib.cuts_destroy(self.h)
            self.h = None

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass

    # ------------------------------------------------------------------- API
    def load_graph(self, row_ptr, col, validate: bool = False, directed: bool = False):
        rp = torch.as_tensor(np.asarray(row_ptr, dtype=np.uint64).view(np.int64)) if not torch.is_tensor(row_ptr) else row_ptr
        cl = torch.as_tensor(np.asarray(col, dtype=np.uint32).view(np.int32)) if not torch.is_tensor(col) else col
        rp = rp.to(self.device, non_blocking=False).contiguous()
        cl = cl.to(self.device, non_blocking=False).contiguous()
        if cl.numel() == 0:
            cl = torch.zeros(1, dtype=torch.int32, device=self.device)
            nnz = 0
        else:
            nnz = cl.numel()
        assert rp.element_size() == 8 and cl.element_size() == 4
        n = rp.numel() - 1
        if directed:       # 2n rows: out-lists then in-lists (cuts_load_digraph)
            assert n % 2 == 0
            n //= 2
        self._graph = (rp, cl)   # keep the borrowed buffers alive
        load = self.lib.cuts_load_digraph if directed else self.lib.cuts_load_graph
        self._check(load(self.h, n, nnz, rp.data_ptr(), cl.data_ptr(), int(validate)))
        self.n = n
        return self

    def load_csr(self, g, validate: bool = False):
        """Load an ``inputs.CSRGraph``-like object (row_ptr, col attributes)."""
        return self.load_graph(g.row_ptr, g.col, validate)

    def load_digraph(self, g, validate: bool = False):
        """Load an ``inputs.DiGraph``-like object (out/in CSR) as one 2n-row CSR."""
        rp, cl = g.combined()
        return self.load_graph(rp, cl, validate, directed=True)

    def set_query_directed(self, row_ptr, col, order=None):
        """Directed query as out-CSR over 0..k-1 (cuts_set_query_directed)."""
        return self.set_query(row_ptr, col, order, directed=True)

    def set_query_arcs(self, k: int, arcs, order=None):
        adj = [sorted({v for u, v in arcs if u == a}) for a in range(k)]
        rp = np.zeros(k + 1, dtype=np.uint32)
        rp[1:] = np.cumsum([len(x) for x in adj])
        return self.set_query_directed(rp, np.asarray([v for x in adj for v in x], dtype=np.uint32), order)

    def set_query(self, row_ptr, col, order=None, directed: bool = False):
        qr = np.ascontiguousarray(row_ptr, dtype=np.uint32)
        qc = np.ascontiguousarray(col, dtype=np.uint32)
        if qc.size == 0:
            qc = np.zeros(1, dtype=np.uint32)
        k = qr.size - 1
        u32p = ctypes.POINTER(ctypes.c_uint32)
        op = None
        if order is not None:
            o = np.ascontiguousarray(order, dtype=np.uint32)
            op = o.ctypes.data_as(u32p)
        fn = self.lib.cuts_set_query_directed if directed else self.lib.cuts_set_query
        self._check(fn(self.h, k, qr.ctypes.data_as(u32p), qc.ctypes.data_as(u32p), op))
        self.k = k
        return self

    def set_query_edges(self, k: int, edges, order=None):
        adj = [[] for _ in range(k)]
        for u, v in edges:
            adj[u].append(v)
            adj[v].append(u)
        rp = np.zeros(k + 1, dtype=np.uint32)
        col = []
        for i in range(k):
            col += sorted(adj[i])
            rp[i + 1] = len(col)
        return self.set_query(rp, np.asarray(col, dtype=np.uint32), order)

    def set_root_range(self, begin: int = 0, end: int = 2**64 - 1):
        self._check(self.lib.cuts_set_root_range(self.h, begin, end))
        return self

    def set_root_slice(self, begin: int = 0, end: int = 2**64 - 1, part: int = 0, nparts: int = 1):
        self._check(self.lib.cuts_set_root_slice(self.h, begin, end, part, nparts))
        return self

    def set_hub_threshold(self, t: int | None):
        """Bitmap rows for vertices with deg >= t at the next load (None: off, 0: auto)."""
        self._check(self.lib.cuts_set_hub_threshold(self.h, 0xFFFFFFFF if t is None else int(t)))
        return self

    def set_prefixes(self, rows: torch.Tensor | None):
        """Seed the next count/enumerate with flat prefixes: rows (count, depth)
        int32/uint32 device tensor in matching-order positions (None: level 1)."""
        if rows is None:
            self._prefixes = None
            self._check(self.lib.cuts_set_prefixes(self.h, 0, 0, None))
            return self
        assert rows.dim() == 2 and rows.element_size() == 4 and rows.is_cuda
        rows = rows.contiguous()
        # the rows may come from another stream (a recv, a copy): the library reads
        # them on its own stream, so order it after everything queued so far
        torch.cuda.current_stream(self.device).synchronize()
        if rows.device != self.device:
            raise ValueError("prefix rows must live on the context's device")
        self._prefixes = rows                   # borrowed by the library until the next run
        cnt, depth = rows.shape
        self._check(self.lib.cuts_set_prefixes(self.h, depth, cnt, rows.data_ptr() if cnt else None))
        return self

    def set_donation(self, poll=None, ship=None):
        """Donation hooks (cuts_set_donation).  poll(depth, remaining) -> int entries
        to give; ship(depth, rows) receives a (give, depth) int32 device tensor that
        is a COPY (owned by the callee).  None, None: off."""
        if poll is None and ship is None:
            self._cb = None
            self._check(self.lib.cuts_set_donation(self.h, L.POLL_FN(), L.SHIP_FN(), None))
            return self
        dev = self.device

        def _poll(_user, depth, remaining):
            try:
                return int(poll(int(depth), int(remaining)))
            except Exception:   # never unwind through C
                import traceback
                traceback.print_exc()
                return 0

        def _ship(_user, depth, ptr, count):
            try:
                # the library synchronised its stream before the call: copy the
                # borrowed arena rows out (zero-copy view via the CUDA array interface)
                if not count:
                    ship(int(depth), None)
                    return 0
                # clone on the library's stream and wait for it: once ship returns the
                # library reuses that arena scratch for the next kernels on its stream
                with torch.cuda.stream(self.stream):
                    view = torch.as_tensor(_DevRows(ptr, int(count), int(depth)), device=dev)
                    rows = view.clone()
                self.stream.synchronize()
                ship(int(depth), rows)
                return 0
            except Exception:
                import traceback
                traceback.print_exc()
                return 1

        self._cb = (L.POLL_FN(_poll), L.SHIP_FN(_ship))
        self._check(self.lib.cuts_set_donation(self.h, self._cb[0], self._cb[1], None))
        return self

    # ------------------------------------------------------------ multi-GPU
    @staticmethod
    def dist_unique_id() -> bytes:
        """A fresh NCCL unique id (cuts_dist_unique_id): create on one rank, broadcast."""
        lib = L.load()
        buf = ctypes.create_string_buffer(L.DIST_UID_BYTES)
        rc = lib.cuts_dist_unique_id(buf)
        if rc != 0:
            raise CutsError(rc, "cuts_dist_unique_id failed (NCCL not loadable)")
        return buf.raw

    def set_dist(self, rank: int, world: int, uid: bytes | None):
        """cuts_set_dist: join a world (collective over the ranks when uid is given).
        Afterwards every query defaults to this rank's cyclic level-1 slice."""
        ub = None if uid is None else ctypes.create_string_buffer(bytes(uid), L.DIST_UID_BYTES)
        self._check(self.lib.cuts_set_dist(self.h, int(rank), int(world), ub, None))
        self.rank, self.world = int(rank), int(world)
        return self

    def allreduce_count(self, count: int) -> int:
        """cuts_allreduce_count: exact 128-bit sum of `count` over the ranks (NCCL)."""
        if count < 0 or count >= 1 << 128:
            raise ValueError("count out of range")
        lo, hi = ctypes.c_uint64(), ctypes.c_uint64()
        self._check(self.lib.cuts_allreduce_count(self.h, count & (2**64 - 1), count >> 64,
                                                  ctypes.byref(lo), ctypes.byref(hi)))
        return int(lo.value) | (int(hi.value) << 64)

    def set_partition_depth(self, depth: int = 1):
        """cuts_set_partition_depth: the root slice applies to the shuffled level-`depth` list."""
        self._check(self.lib.cuts_set_partition_depth(self.h, int(depth)))
        return self

    def partition_size(self) -> int:
        """|L_depth| over the root range (the list cuts_set_root_slice partitions)."""
        n = ctypes.c_uint64()
        self._check(self.lib.cuts_partition_size(self.h, ctypes.byref(n)))
        return int(n.value)

    def level1_size(self):
        """(canonical level-1 size, size inside the root range) for the current query."""
        a, b = ctypes.c_uint64(), ctypes.c_uint64()
        self._check(self.lib.cuts_level1_size(self.h, ctypes.byref(a), ctypes.byref(b)))
        return int(a.value), int(b.value)

    def set_debug(self, timing: bool = False, bytes_: bool = False, no_reuse: bool = False,
                  no_pack: bool = False, first_source: bool = False, no_fast_count: bool = False,
                  preload_count: bool = False, binned: bool = False, sv: bool = False, no_pairs: bool = False,
                  no_lr: bool = False, groups: bool = False, no_dlr: bool = False,
                  tail_alt: bool = False, tail_split: bool = False,
                  no_cta_tail: bool = False):
        """CUTS_DEBUG_* flags: instrumentation and the NEXT-2 ablations (include/cuts.h)."""
        flags = ((1 if timing else 0) | (2 if bytes_ else 0) | (4 if no_reuse else 0) |
                 (8 if no_pack else 0) | (16 if first_source else 0) | (32 if no_fast_count else 0) |
                 (64 if preload_count else 0) | (128 if binned else 0) | (256 if sv else 0) |
                 (512 if no_pairs else 0) | (1024 if no_lr else 0) | (2048 if groups else 0) |
                 (4096 if no_dlr else 0) | (8192 if tail_alt else 0) |
                 (16384 if tail_split else 0) |
                 (32768 if no_cta_tail else 0))
        self._check(self.lib.cuts_set_debug(self.h, flags))
        return self

    def group_hist(self) -> dict:
        """CUTS_DEBUG_GROUPS: {level: [(bucket, groups, sum m, sum m^2), ...]} of the last count."""
        buf = (ctypes.c_uint64 * L.GROUP_HIST_WORDS)()
        self._check(self.lib.cuts_debug_group_hist(self.h, buf))
        out = {}
        for j in range(9):
            rows = [(b, buf[(j * 16 + b) * 3], buf[(j * 16 + b) * 3 + 1], buf[(j * 16 + b) * 3 + 2])
                    for b in range(16) if buf[(j * 16 + b) * 3]]
            if rows:
                out[j] = rows
        return out

    def count(self, mode="hybrid") -> int:
        """Exact count (Python int; values >= 2^64 are returned in full)."""
        out = ctypes.c_uint64()
        rc = self._check(self.lib.cuts_count(self.h, _mode(mode), ctypes.byref(out)), allow=(L.CUTS_EOVERFLOW,))
        if rc == L.CUTS_EOVERFLOW:
            s = self.stats()
            return s["count"]
        return int(out.value)

    def enumerate(self, mode="hybrid", cap_rows: int | None = None, out: torch.Tensor | None = None):
        """Rows (n_found, k) uint32 (as int32 storage) on the device, query-id order.

        If cap_rows is None a count pass sizes the buffer first."""
        if cap_rows is None:
            cap_rows = self.count(mode)
        if out is None:
            out = torch.empty((max(int(cap_rows), 1), self.k), dtype=torch.int32, device=self.device)
        nf = ctypes.c_uint64()
        rc = self._check(self.lib.cuts_enumerate(self.h, _mode(mode), out.data_ptr(), int(cap_rows), ctypes.byref(nf)),
                         allow=(L.CUTS_ETRUNC,))
        self.truncated = rc == L.CUTS_ETRUNC
        return out[:min(int(nf.value), int(cap_rows))]

    def stats(self) -> dict:
        s = L.cuts_stats()
        self._check(self.lib.cuts_get_stats(self.h, ctypes.byref(s)))
        k = s.k
        return {
            "k": k, "order": list(s.order)[:k], "level_size": list(s.level_size)[:k + 1],
            "count": int(s.count_lo) | (int(s.count_hi) << 64),
            "level1_canonical": s.level1_canonical, "chunks": s.chunks, "windows": s.windows,
            "launches": s.launches, "peak_arena_bytes": s.peak_arena_bytes, "items": s.items,
            "ms_total": s.ms_total, "ms_extend": s.ms_extend, "ms_plan": s.ms_plan,
            "extend_launches": s.extend_launches, "alg_bytes_extend": s.alg_bytes_extend,
            "alg_bytes_plan": s.alg_bytes_plan, "hubs": s.hubs, "hub_threshold": s.hub_threshold,
            "donations": s.donations, "donated_entries": s.donated_entries,
            "alg_bytes_extend_needed": s.alg_bytes_extend_needed, "free_identity": s.free_identity,
            "fused_levels": s.fused_levels, "ms_tail": s.ms_tail, "tail_launches": s.tail_launches,
            "tail_word_ops": s.tail_word_ops,
        }

    def trie_decode(self, ca_levels, pa_levels) -> torch.Tensor:
        """GPU decode of a (CA, PA) trie (Fig. 3C) into root-to-leaf rows."""
        L_ = len(ca_levels)
        cas = [torch.as_tensor(np.asarray(c, dtype=np.uint32).view(np.int32)).to(self.device) for c in ca_levels]
        pas = [torch.as_tensor(np.asarray(p if p is not None else [0], dtype=np.uint32).view(np.int32)).to(self.device)
               for p in pa_levels]
        sizes = np.array([c.numel() for c in cas], dtype=np.uint64)
        out = torch.empty((int(sizes[-1]), L_), dtype=torch.int32, device=self.device)
        PA = ctypes.c_void_p * L_
        ca_arr = PA(*[c.data_ptr() for c in cas])
        pa_arr = PA(*[p.data_ptr() for p in pas])
        self._check(self.lib.cuts_trie_decode(self.h, L_, sizes.ctypes.data_as(ctypes.POINTER(ctypes.c_uint64)),
                                              ca_arr, pa_arr, out.data_ptr()))
        return out
