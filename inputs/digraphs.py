"""Directed data and query graphs.

PAPER.md:207-209 (§2.1): "In this work, we consider directed graphs (edges are
directed)"; the undirected case is the special case with both arcs.  A
directed data graph is stored as out-CSR (children, the paper's D.cs) and
in-CSR (parents, D.ps; Alg. 2 l.33-42), both with strictly ascending rows, no
self loops, no duplicate arcs.  Builders only — no matching arithmetic.

* ``digraph_from_arcs(n, arcs)`` — the given arcs (loops dropped, deduped).
* ``directed_er_graph(n, m, seed)`` — m distinct uniform ordered pairs.
* ``directed_rmat_graph(scale, ef, a, b, c, seed)`` — the R-MAT samples of
  ``rmat_edges`` kept as arcs src -> dst (not symmetrised), relabelled by the
  same seeded permutation as ``rmat_graph``.
"""
from __future__ import annotations

from dataclasses import dataclass
import numpy as np

from .graphs import rmat_edges


def _csr(n, src, dst):
    order = np.lexsort((dst, src))
    src, dst = src[order], dst[order]
    row = np.zeros(n + 1, dtype=np.uint64)
    np.add.at(row, src.astype(np.int64) + 1, 1)
    return np.cumsum(row, dtype=np.uint64), dst.astype(np.uint32)


@dataclass(frozen=True)
class DiGraph:
    n: int
    out_row: np.ndarray   # uint64[n+1]
    out_col: np.ndarray   # uint32[nnz]
    in_row: np.ndarray    # uint64[n+1]
    in_col: np.ndarray    # uint32[nnz]
    name: str = ""

    @property
    def nnz(self) -> int:
        return int(self.out_row[-1])

    def out_degrees(self):
        return np.diff(self.out_row).astype(np.int64)

    def in_degrees(self):
        return np.diff(self.in_row).astype(np.int64)

    def arcs(self):
        src = np.repeat(np.arange(self.n, dtype=np.int64), self.out_degrees())
        return np.stack([src, self.out_col.astype(np.int64)], axis=1)

    def combined(self):
        """One CSR of 2n rows: rows 0..n-1 = out-lists, rows n..2n-1 = in-lists
        (the layout cuts_load_digraph takes)."""
        row = np.concatenate([self.out_row, self.in_row[1:] + self.out_row[-1]]).astype(np.uint64)
        return row, np.concatenate([self.out_col, self.in_col]).astype(np.uint32)


def digraph_from_arcs(n: int, arcs, name: str = "") -> DiGraph:
    a = np.asarray(list(arcs), dtype=np.int64).reshape(-1, 2)
    a = a[a[:, 0] != a[:, 1]]
    a = np.unique(a, axis=0) if a.size else a
    src, dst = a[:, 0].astype(np.uint64), a[:, 1].astype(np.uint64)
    orow, ocol = _csr(n, src, dst)
    irow, icol = _csr(n, dst, src)
    return DiGraph(n, orow, ocol, irow, icol, name)


def directed_er_graph(n: int, m: int, seed: int = 1) -> DiGraph:
    rng = np.random.Generator(np.random.PCG64(seed ^ 0xD1D1))
    seen = set()
    while len(seen) < m:
        u, v = (int(x) for x in rng.integers(0, n, 2))
        if u != v:
            seen.add((u, v))
    return digraph_from_arcs(n, sorted(seen), name=f"der_{n}_{m}_seed{seed}")


def directed_rmat_graph(scale: int, ef: int, a: float = 0.57, b: float = 0.19, c: float = 0.19,
                        seed: int = 1) -> DiGraph:
    n = 1 << scale
    src, dst = rmat_edges(scale, ef, a, b, c, seed)
    perm = np.random.Generator(np.random.PCG64(seed ^ 0xA5A5)).permutation(n).astype(np.int64)
    arcs = np.stack([perm[src.astype(np.int64)], perm[dst.astype(np.int64)]], axis=1)
    return digraph_from_arcs(n, arcs, name=f"drmat_s{scale}_ef{ef}_a{a}_b{b}_c{c}_seed{seed}")


def directed_cycle(n: int) -> DiGraph:
    return digraph_from_arcs(n, [(i, (i + 1) % n) for i in range(n)], name=f"dC{n}")


def transitive_tournament(n: int) -> DiGraph:
    return digraph_from_arcs(n, [(i, j) for i in range(n) for j in range(i + 1, n)], name=f"TT{n}")


def complete_digraph(n: int) -> DiGraph:
    return digraph_from_arcs(n, [(i, j) for i in range(n) for j in range(n) if i != j], name=f"DK{n}")


@dataclass(frozen=True)
class DiQuery:
    k: int
    arcs: tuple   # (u, v): u -> v
    name: str = ""

    def csr(self):
        """Out-CSR (row_ptr u32[k+1], col u32) with ascending rows."""
        adj = [sorted({v for u, v in self.arcs if u == a}) for a in range(self.k)]
        row = np.zeros(self.k + 1, dtype=np.uint32)
        row[1:] = np.cumsum([len(x) for x in adj])
        return row, np.asarray([v for x in adj for v in x], dtype=np.uint32)


def query_from_arcs(k: int, arcs, name: str = "") -> DiQuery:
    s = set()
    for u, v in arcs:
        if u == v or not (0 <= u < k and 0 <= v < k):
            raise ValueError(f"bad query arc {(u, v)}")
        s.add((u, v))
    return DiQuery(k, tuple(sorted(s)), name)


# a small directed query catalogue (weakly connected; no reciprocal arcs)
DIRECTED_QUERIES = {
    "dP3": (3, [(0, 1), (1, 2)]),                   # directed path
    "dC3": (3, [(0, 1), (1, 2), (2, 0)]),           # directed triangle (cycle)
    "TT3": (3, [(0, 1), (0, 2), (1, 2)]),           # feed-forward loop
    "out2": (3, [(0, 1), (0, 2)]),                  # out-star
    "in2": (3, [(1, 0), (2, 0)]),                   # in-star
    "dC4": (4, [(0, 1), (1, 2), (2, 3), (3, 0)]),
    "TT4": (4, [(i, j) for i in range(4) for j in range(i + 1, 4)]),
    "bifan": (4, [(0, 2), (0, 3), (1, 2), (1, 3)]),
    "diamond": (4, [(0, 1), (0, 2), (1, 3), (2, 3)]),
    "TT5": (5, [(i, j) for i in range(5) for j in range(i + 1, 5)]),
    "dC5": (5, [(0, 1), (1, 2), (2, 3), (3, 4), (4, 0)]),
    "TT6-rev": (6, [(j, i) for i in range(6) for j in range(i + 1, 6)]),
}


def named_diquery(name: str) -> DiQuery:
    k, arcs = DIRECTED_QUERIES[name]
    return query_from_arcs(k, arcs, name)
