"""Query graphs: small undirected graphs on vertices 0..k-1 (k <= 8).

Catalog.  The paper's procedure (PAPER.md:1323-1328,
§6.2) takes all N-node graphs sorted by edge count, keeps the top 11 and breaks
ties randomly; this build fixes the tie-break deterministically and keeps only
connected members (reading P16: disconnected Q is NEXT-3):

* ``dense_family(k)`` = K_k − M for M in ``m11(k)`` (k >= 6): the 11 removal
  sets ∅, K2, P3, 2K2, K3, P4, K1,3, P3∪K2, 3K2, C4, P5.
* ``DENSE5`` = K5 − M for M in [∅, K2, P3, 2K2, K3, P4, K1,3, P3∪K2, C4, P5, paw].
* ``SPARSE5`` = the 8 connected 5-vertex graphs with <= 5 edges.
"""
from __future__ import annotations

from dataclasses import dataclass
import numpy as np


@dataclass(frozen=True)
class Query:
    k: int
    edges: tuple  # tuple of (u, v) with u < v
    name: str = ""

    def csr(self):
        """(row_ptr u32[k+1], col u32[2|E|]) symmetric CSR, rows ascending."""
        adj = [[] for _ in range(self.k)]
        for u, v in self.edges:
            adj[u].append(v)
            adj[v].append(u)
        row_ptr = np.zeros(self.k + 1, dtype=np.uint32)
        col = []
        for i in range(self.k):
            nb = sorted(adj[i])
            col.extend(nb)
            row_ptr[i + 1] = row_ptr[i] + len(nb)
        return row_ptr, np.asarray(col, dtype=np.uint32)

    def degrees(self):
        d = [0] * self.k
        for u, v in self.edges:
            d[u] += 1
            d[v] += 1
        return d


def query_from_edges(k: int, edges, name: str = "") -> Query:
    es = set()
    for u, v in edges:
        if u == v or not (0 <= u < k and 0 <= v < k):
            raise ValueError(f"bad query edge {(u, v)}")
        es.add((min(u, v), max(u, v)))
    return Query(k=k, edges=tuple(sorted(es)), name=name)


def _parse(spec: str):
    """'01,12' -> [(0,1),(1,2)]"""
    if not spec:
        return []
    return [(int(t[0]), int(t[1])) for t in spec.split(",")]


def k_minus(k: int, removed, name: str = "") -> Query:
    rem = {(min(u, v), max(u, v)) for u, v in removed}
    edges = [(i, j) for i in range(k) for j in range(i + 1, k) if (i, j) not in rem]
    return query_from_edges(k, edges, name=name)


_M11 = [("", "K"), ("01", "K-K2"), ("01,12", "K-P3"), ("01,23", "K-2K2"),
        ("01,12,02", "K-K3"), ("01,12,23", "K-P4"), ("01,02,03", "K-K13"),
        ("01,12,34", "K-P3uK2"), ("01,23,45", "K-3K2"), ("01,12,23,30", "K-C4"),
        ("01,12,23,34", "K-P5")]

_DENSE5 = [("", "K5"), ("01", "K5-K2"), ("01,12", "K5-P3"), ("01,23", "K5-2K2"),
           ("01,12,02", "K5-K3"), ("01,12,23", "K5-P4"), ("01,02,03", "K5-K13"),
           ("01,12,34", "K5-P3uK2"), ("01,12,23,30", "K5-C4"), ("01,12,23,34", "K5-P5"),
           ("01,12,20,23", "K5-paw")]

_SPARSE5 = [("01,12,23,34", "P5"), ("01,02,03,04", "K1_4"), ("01,12,14,23", "chair"),
            ("01,12,23,34,40", "C5"), ("01,12,23,30,04", "banner"),
            ("01,12,20,03,14", "bull"), ("01,12,20,03,04", "cricket"),
            ("01,12,20,03,34", "tadpole32")]


def m11(k: int):
    if k < 6:
        raise ValueError("M11 needs k >= 6 (3K2 uses 6 vertices)")
    return [(_parse(s), n) for s, n in _M11]


def dense_family(k: int):
    return [k_minus(k, rem, name=f"{n.replace('K', f'K{k}', 1)}") for rem, n in m11(k)]


DENSE5 = [k_minus(5, _parse(s), name=n) for s, n in _DENSE5]
SPARSE5 = [query_from_edges(5, _parse(s), name=n) for s, n in _SPARSE5]


def named_query(name: str) -> Query:
    """Small named queries used by tests: K<k>, C<k>, P<k>, S<s> (star K1,s)."""
    for q in DENSE5 + SPARSE5:
        if q.name == name:
            return q
    kind, num = name[0], int(name[1:])
    if kind == "K":
        return k_minus(num, [], name=name)
    if kind == "C":
        return query_from_edges(num, [(i, (i + 1) % num) for i in range(num)], name=name)
    if kind == "P":  # path on num vertices
        return query_from_edges(num, [(i, i + 1) for i in range(num - 1)], name=name)
    if kind == "S":  # star with num leaves
        return query_from_edges(num + 1, [(0, i) for i in range(1, num + 1)], name=name)
    raise KeyError(name)
