"""TEST INFRASTRUCTURE ONLY — the CPU oracle for cuTS subgraph-isomorphism search.

Only ``tests/``, ``__graft_entry__.smoke()`` and ``bench.py``'s ``cpu_baseline``
/ ``--impl reference`` legs may import this package.  The product package
(``paper_conf_sc_xiangkshs21_b200``) never imports it and shares no code with it.

Thin ctypes wrapper around ``oracle/cuts_oracle.c`` (plain C, single-threaded;
see its header for the paper citations and DESIGN.md §2 for the readings).
"""
from __future__ import annotations

import ctypes
import os
import subprocess
import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SRC = os.path.join(_HERE, "cuts_oracle.c")
_LIB = os.path.join(_HERE, "liboracle.so")
_lib = None

ORC_OK, ORC_EINVAL, ORC_ENOMEM, ORC_EUNSUPPORTED = 0, -1, -2, -7


class OracleError(RuntimeError):
    def __init__(self, code: int):
        super().__init__(f"oracle returned status {code}")
        self.code = code


def build(force: bool = False) -> str:
    """Compile the oracle with gcc (plain -O2; no tuning)."""
    if force or not os.path.exists(_LIB) or os.path.getmtime(_LIB) < os.path.getmtime(_SRC):
        subprocess.check_call(["gcc", "-O2", "-std=gnu11", "-shared", "-fPIC", "-pthread", "-o", _LIB, _SRC])
    return _LIB


def _load():
    global _lib
    if _lib is None:
        lib = ctypes.CDLL(build())
        u32p = ctypes.POINTER(ctypes.c_uint32)
        u64p = ctypes.POINTER(ctypes.c_uint64)
        lib.oracle_count.argtypes = [ctypes.c_uint32, u64p, u32p, ctypes.c_uint32, u32p, u32p, u32p,
                                     ctypes.c_uint64, ctypes.c_uint64, u64p, u64p, u64p, u64p]
        lib.oracle_enumerate.argtypes = [ctypes.c_uint32, u64p, u32p, ctypes.c_uint32, u32p, u32p, u32p,
                                         ctypes.c_uint64, ctypes.c_uint64, u32p, ctypes.c_uint64, u64p]
        lib.oracle_order.argtypes = [ctypes.c_uint32, u32p, u32p, u32p]
        lib.oracle_validate_graph.argtypes = [ctypes.c_uint32, u64p, u32p]
        lib.oracle_level1_size.argtypes = [ctypes.c_uint32, u64p, ctypes.c_uint32, u64p]
        lib.oracle_trie_decode.argtypes = [ctypes.c_uint32, u64p, ctypes.POINTER(u32p),
                                           ctypes.POINTER(u32p), u32p]
        lib.oracle_di_count.argtypes = [ctypes.c_uint32, u64p, u32p, u64p, u32p, ctypes.c_uint32, u32p, u32p,
                                        u32p, u64p, u64p, u64p, u64p, u32p, ctypes.c_uint64]
        lib.oracle_di_order.argtypes = [ctypes.c_uint32, u32p, u32p, u32p]
        lib.oracle_cross_product.argtypes = [ctypes.c_uint32, ctypes.c_uint32, u32p, ctypes.POINTER(u32p),
                                             ctypes.POINTER(u32p), u64p, u32p, ctypes.c_uint64, u64p, u64p]
        lib.oracle_count_mt.argtypes = [ctypes.c_uint32, ctypes.c_uint32, u64p, u32p, ctypes.c_uint32, u32p, u32p,
                                        u32p, ctypes.c_uint64, ctypes.c_uint64, ctypes.c_uint64, u64p, u64p]
        lib.oracle_cross_product.restype = ctypes.c_int
        lib.oracle_count_mt.restype = ctypes.c_int
        lib.oracle_di_count.restype = ctypes.c_int
        lib.oracle_di_order.restype = ctypes.c_int
        for f in (lib.oracle_count, lib.oracle_enumerate, lib.oracle_order,
                  lib.oracle_validate_graph, lib.oracle_level1_size, lib.oracle_trie_decode):
            f.restype = ctypes.c_int
        _lib = lib
    return _lib


def _p(a, ct):
    return a.ctypes.data_as(ctypes.POINTER(ct))


def _check(rc):
    if rc != ORC_OK:
        raise OracleError(rc)


def _graph_arrays(g):
    rp = np.ascontiguousarray(g.row_ptr, dtype=np.uint64)
    col = np.ascontiguousarray(g.col, dtype=np.uint32)
    if col.size == 0:
        col = np.zeros(1, dtype=np.uint32)
    return rp, col


def _query_arrays(q, order):
    qr, qc = q.csr()
    if qc.size == 0:
        qc = np.zeros(1, dtype=np.uint32)
    o = None if order is None else np.ascontiguousarray(order, dtype=np.uint32)
    return np.ascontiguousarray(qr), np.ascontiguousarray(qc), o


def validate_graph(g) -> bool:
    rp, col = _graph_arrays(g)
    return _load().oracle_validate_graph(g.n, _p(rp, ctypes.c_uint64), _p(col, ctypes.c_uint32)) == ORC_OK


def order(q) -> list:
    """The paper's matching order (readings P5/P6)."""
    qr, qc, _ = _query_arrays(q, None)
    out = np.zeros(q.k, dtype=np.uint32)
    _check(_load().oracle_order(q.k, _p(qr, ctypes.c_uint32), _p(qc, ctypes.c_uint32), _p(out, ctypes.c_uint32)))
    return out.tolist()


# ------------------------------------------------------ disconnected queries
# PAPER.md:544-551 (§4): "If the query graph is not connected ... we split Q
# into a set of connected components, compute sub-graph isomorphism on each of
# these components, and produce the final result as the cross product of
# individual solutions."  Reading P16: an element of the result
# is still a subgraph isomorphism (Def. 4), i.e. injective, so the
# cross product keeps only the combinations whose images are disjoint.

def components(q) -> list:
    """Connected components of Q as sorted vertex lists, ordered by min vertex."""
    adj = [set() for _ in range(q.k)]
    for u, v in q.edges:
        adj[u].add(v)
        adj[v].add(u)
    seen, comps = set(), []
    for s in range(q.k):
        if s in seen:
            continue
        stack, comp = [s], set()
        while stack:
            x = stack.pop()
            if x in comp:
                continue
            comp.add(x)
            stack.extend(adj[x] - comp)
        seen |= comp
        comps.append(sorted(comp))
    return comps


def _sub_query(q, comp):
    """The component as its own query on vertices 0..|comp|-1 (same vertex order)."""
    idx = {v: i for i, v in enumerate(comp)}
    return _SubQuery(len(comp), [(idx[u], idx[v]) for u, v in q.edges if u in idx])


class _SubQuery:
    def __init__(self, k, edges):
        self.k, self.edges = k, edges

    def csr(self):
        adj = [sorted({v for a, v in self.edges if a == u} | {a for a, v in self.edges if v == u})
               for u in range(self.k)]
        row = np.zeros(self.k + 1, dtype=np.uint32)
        row[1:] = np.cumsum([len(a) for a in adj])
        return row, np.asarray([v for a in adj for v in a], dtype=np.uint32)


def _cross_product(g, q, want_rows: bool):
    """P:546-551 step by step: per-component embeddings (the connected oracle
    below, each component as its own query), then their cross product keeping
    injective combinations only — nested loops in C (``oracle_cross_product``),
    nothing materialised but the component rows.  Returns (count, rows|None)."""
    comps = components(q)
    subs = [enumerate_rows(g, _sub_query(q, comp)) for comp in comps]
    nc = len(comps)
    sizes = np.array([len(c) for c in comps], dtype=np.uint32)
    verts = [np.ascontiguousarray(c, dtype=np.uint32) for c in comps]
    crow = [np.ascontiguousarray(s if s.size else np.zeros((1, len(c)), np.uint32), dtype=np.uint32)
            for s, c in zip(subs, comps)]
    ccount = np.array([s.shape[0] for s in subs], dtype=np.uint64)
    u32p = ctypes.POINTER(ctypes.c_uint32)
    va = (u32p * nc)(*[_p(v, ctypes.c_uint32) for v in verts])
    ra = (u32p * nc)(*[_p(r, ctypes.c_uint32) for r in crow])
    lo, hi = np.zeros(1, np.uint64), np.zeros(1, np.uint64)
    lib = _load()

    def call(rows, cap):
        _check(lib.oracle_cross_product(q.k, nc, _p(sizes, ctypes.c_uint32), va, ra, _p(ccount, ctypes.c_uint64),
                                        None if rows is None else _p(rows, ctypes.c_uint32), cap,
                                        _p(lo, ctypes.c_uint64), _p(hi, ctypes.c_uint64)))
        return int(lo[0]) | (int(hi[0]) << 64)

    n = call(None, 0)
    if not want_rows:
        return n, None
    rows = np.zeros((max(n, 1), q.k), dtype=np.uint32)
    call(rows, n)
    return n, rows[:n]


def count(g, q, order=None, root_begin: int = 0, root_end: int = 2**64 - 1, levels: bool = False):
    """Exact number of ordered non-induced embeddings (Python int, 128-bit).

    A disconnected Q goes through the per-component cross product of P:546-551
    (``_cross_product``; no order, root range or level sizes there).

    With ``levels=True`` returns ``(count, [|L_0|, |L_1|, ..., |L_k|])`` where
    |L_j| counts partial paths of j matched vertices (|L_0| is 0).
    """
    if len(components(q)) > 1:
        if order is not None or root_begin != 0 or root_end != 2**64 - 1 or levels:
            raise OracleError(ORC_EUNSUPPORTED)
        return _cross_product(g, q, False)[0]
    rp, col = _graph_arrays(g)
    qr, qc, o = _query_arrays(q, order)
    lo = np.zeros(1, np.uint64)
    hi = np.zeros(1, np.uint64)
    llo = np.zeros(q.k + 1, np.uint64)
    lhi = np.zeros(q.k + 1, np.uint64)
    rc = _load().oracle_count(g.n, _p(rp, ctypes.c_uint64), _p(col, ctypes.c_uint32), q.k,
                              _p(qr, ctypes.c_uint32), _p(qc, ctypes.c_uint32),
                              None if o is None else _p(o, ctypes.c_uint32),
                              root_begin, root_end, _p(lo, ctypes.c_uint64), _p(hi, ctypes.c_uint64),
                              _p(llo, ctypes.c_uint64), _p(lhi, ctypes.c_uint64))
    _check(rc)
    total = int(lo[0]) | (int(hi[0]) << 64)
    if levels:
        return total, [int(a) | (int(b) << 64) for a, b in zip(llo, lhi)]
    return total


def enumerate_rows(g, q, order=None, root_begin: int = 0, root_end: int = 2**64 - 1,
                   cap_rows: int | None = None) -> np.ndarray:
    """All embeddings as a sorted (count, k) uint32 array, row[q] = f(q)."""
    if len(components(q)) > 1:
        if order is not None or root_begin != 0 or root_end != 2**64 - 1:
            raise OracleError(ORC_EUNSUPPORTED)
        rows = _cross_product(g, q, True)[1]
        return rows if cap_rows is None else rows[:cap_rows]
    if cap_rows is None:
        cap_rows = count(g, q, order, root_begin, root_end)
    rp, col = _graph_arrays(g)
    qr, qc, o = _query_arrays(q, order)
    rows = np.zeros((max(cap_rows, 1), q.k), dtype=np.uint32)
    nf = np.zeros(1, np.uint64)
    rc = _load().oracle_enumerate(g.n, _p(rp, ctypes.c_uint64), _p(col, ctypes.c_uint32), q.k,
                                  _p(qr, ctypes.c_uint32), _p(qc, ctypes.c_uint32),
                                  None if o is None else _p(o, ctypes.c_uint32),
                                  root_begin, root_end, _p(rows, ctypes.c_uint32), cap_rows,
                                  _p(nf, ctypes.c_uint64))
    _check(rc)
    return rows[:min(int(nf[0]), cap_rows)]


def count_mt(g, q, threads: int, root_begin: int = 0, root_end: int = 2**64 - 1, grain: int = 1,
             order=None) -> int:
    """Root-parallel driver (``oracle_count_mt``): the same ``rec`` on disjoint
    canonical root ranges pulled by `threads` pthreads, summed.  Used for the
    N-core CPU baseline only; parity pins use ``count``."""
    rp, col = _graph_arrays(g)
    qr, qc, o = _query_arrays(q, order)
    lo, hi = np.zeros(1, np.uint64), np.zeros(1, np.uint64)
    _check(_load().oracle_count_mt(threads, g.n, _p(rp, ctypes.c_uint64), _p(col, ctypes.c_uint32), q.k,
                                   _p(qr, ctypes.c_uint32), _p(qc, ctypes.c_uint32),
                                   None if o is None else _p(o, ctypes.c_uint32), root_begin, root_end, grain,
                                   _p(lo, ctypes.c_uint64), _p(hi, ctypes.c_uint64)))
    return int(lo[0]) | (int(hi[0]) << 64)


def level1_size(g, min_deg: int) -> int:
    rp, _ = _graph_arrays(g)
    out = np.zeros(1, np.uint64)
    _check(_load().oracle_level1_size(g.n, _p(rp, ctypes.c_uint64), min_deg, _p(out, ctypes.c_uint64)))
    return int(out[0])


def trie_decode(ca_levels, pa_levels) -> np.ndarray:
    """Decode a (CA, PA) trie (Fig. 3C) into root-to-leaf rows."""
    L = len(ca_levels)
    cas = [np.ascontiguousarray(c, dtype=np.uint32) for c in ca_levels]
    pas = [np.ascontiguousarray(p if p is not None else np.zeros(1), dtype=np.uint32) for p in pa_levels]
    sizes = np.array([c.size for c in cas], dtype=np.uint64)
    u32p = ctypes.POINTER(ctypes.c_uint32)
    ca_arr = (u32p * L)(*[_p(c, ctypes.c_uint32) for c in cas])
    pa_arr = (u32p * L)(*[_p(p, ctypes.c_uint32) for p in pas])
    out = np.zeros((int(sizes[-1]), L), dtype=np.uint32)
    _check(_load().oracle_trie_decode(L, _p(sizes, ctypes.c_uint64), ca_arr, pa_arr, _p(out, ctypes.c_uint32)))
    return out


# ------------------------------------------------------------ directed (NEXT-1)
def _di_call(g, q, order, rows=None, cap=0, levels=False):
    arrs = [np.ascontiguousarray(a, dtype=t) for a, t in
            ((g.out_row, np.uint64), (g.out_col, np.uint32), (g.in_row, np.uint64), (g.in_col, np.uint32))]
    arrs = [a if a.size else np.zeros(1, a.dtype) for a in arrs]
    qr, qc = q.csr()
    qc = qc if qc.size else np.zeros(1, np.uint32)
    qr, qc = np.ascontiguousarray(qr), np.ascontiguousarray(qc)
    o = None if order is None else np.ascontiguousarray(order, dtype=np.uint32)
    lo, hi = np.zeros(1, np.uint64), np.zeros(1, np.uint64)
    llo, lhi = np.zeros(q.k + 1, np.uint64), np.zeros(q.k + 1, np.uint64)
    _check(_load().oracle_di_count(
        g.n, _p(arrs[0], ctypes.c_uint64), _p(arrs[1], ctypes.c_uint32), _p(arrs[2], ctypes.c_uint64),
        _p(arrs[3], ctypes.c_uint32), q.k, _p(qr, ctypes.c_uint32), _p(qc, ctypes.c_uint32),
        None if o is None else _p(o, ctypes.c_uint32), _p(lo, ctypes.c_uint64), _p(hi, ctypes.c_uint64),
        _p(llo, ctypes.c_uint64), _p(lhi, ctypes.c_uint64),
        None if rows is None else _p(rows, ctypes.c_uint32), cap))
    total = int(lo[0]) | (int(hi[0]) << 64)
    if levels:
        return total, [int(a) | (int(b) << 64) for a, b in zip(llo, lhi)]
    return total


def di_count(g, q, order=None, levels: bool = False):
    """Directed: exact number of injective arc-preserving maps (cuts_oracle.c
    'directed' section: P:207-209, c-/p-intersection of Alg. 2)."""
    return _di_call(g, q, order, levels=levels)


def di_enumerate_rows(g, q, order=None) -> np.ndarray:
    n = _di_call(g, q, order)
    rows = np.zeros((max(n, 1), q.k), dtype=np.uint32)
    _di_call(g, q, order, rows=rows, cap=n)
    return rows[:n]


def di_order(q) -> list:
    qr, qc = q.csr()
    qc = qc if qc.size else np.zeros(1, np.uint32)
    out = np.zeros(q.k, dtype=np.uint32)
    _check(_load().oracle_di_order(q.k, _p(np.ascontiguousarray(qr), ctypes.c_uint32),
                                   _p(np.ascontiguousarray(qc), ctypes.c_uint32), _p(out, ctypes.c_uint32)))
    return out.tolist()
