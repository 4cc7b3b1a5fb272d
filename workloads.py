"""Named benchmark workloads (BASELINE.json configs -> concrete seeded inputs).

Holds no matching arithmetic: it only names graphs (generator + parameters)
and query lists from ``inputs``.  Calibration record: DESIGN.md §3 and
profiles/r01_calibration.md.
"""
from __future__ import annotations

from dataclasses import dataclass

from inputs import rmat_graph, rmat_graph_torch, er_graph, named_query, DENSE5, SPARSE5, dense_family


_CACHE: dict = {}


@dataclass(frozen=True)
class GraphSpec:
    kind: str
    params: tuple

    def build(self):
        """The graph (cached per process: tests and bench reuse the same bytes)."""
        g = _CACHE.get(self)
        if g is None:
            g = _CACHE[self] = self._build()
        return g

    def _build(self):
        if self.kind == "rmat":
            return rmat_graph(*self.params)
        if self.kind == "rmat_t":   # same bytes as "rmat" (tests/test_oracle.py), generated with torch
            import torch
            *p, seed = self.params
            return rmat_graph_torch(*p, seed=seed, device="cuda" if torch.cuda.is_available() else "cpu")
        if self.kind == "er":
            return er_graph(*self.params)
        raise KeyError(self.kind)

    @property
    def name(self):
        return f"{self.kind}{self.params}"


@dataclass(frozen=True)
class Workload:
    name: str
    description: str
    parts: tuple          # ((GraphSpec, (Query, ...)), ...)
    mode: str = "hybrid"
    root_range: tuple | None = None   # (a, b, den): canonical level-1 positions [a*R/den, b*R/den)
    min_trie_bytes: float = 0.0       # bench asserts 8 B x (deepest chunk-summed stored level) exceeds this

    def roots(self, l1: int):
        """Canonical root range [begin, end) for a level-1 list of size l1
        (den == 0: a and b are absolute positions)."""
        if self.root_range is None:
            return 0, l1
        a, b, den = self.root_range
        if den == 0:
            return min(a, l1), min(b, l1)
        return a * l1 // den, b * l1 // den


# configs[0]: triangle and 4-cycle on ER(1000, avg degree 8)
C1 = Workload(
    "C1", "K3 + C4 on ER G(1000, 4000) seeds 1..5",
    tuple((GraphSpec("er", (1000, 4000, s)), (named_query("K3"), named_query("C4"))) for s in range(1, 6)))

# configs[1]: 5-vertex sparse/dense query set on R-MAT scale 16, edge factor 16.
# Calibrated (profiles/r01_calibration.md): Graph500 skew (.57/.19/.19) needs
# 1e13-1e15 candidate checks per query (hours); no single ef16 graph makes both
# families finite in seconds, so the dense family runs on a mild power law
# (a=.45, max deg ~3k, SNAP-enron-like skew) and the sparse family on a flatter
# one (a=.35, max deg ~260), both R-MAT(16, 16), seed 1.
C2_DENSE_GRAPH = GraphSpec("rmat", (16, 16, 0.45, 0.22, 0.22, 1))
C2_SPARSE_GRAPH = GraphSpec("rmat", (16, 16, 0.35, 0.22, 0.22, 1))
C2 = Workload(
    "C2", "Dense-5 (11, P:1323-1328) on R-MAT(16,16,.45,.22,.22) + Sparse-5 (8) on R-MAT(16,16,.35,.22,.22); hybrid count",
    ((C2_DENSE_GRAPH, tuple(DENSE5)), (C2_SPARSE_GRAPH, tuple(SPARSE5))))

# configs[2]: 6-8-vertex dense families on a ~1M-vertex, ~10M-edge power-law graph
# (com-youtube-like).  Calibrated (profiles/r01_calibration_c3c4.md): R-MAT(20, 10)
# at a=.50 needs up to 4,600 s for one K8-M query and a=.52 hours; a=.48/.21/.21
# keeps every one of the 33 queries under 180 s on the first kernel, all counts
# non-zero and < 2^64.
C3_GRAPH = GraphSpec("rmat_t", (20, 10, 0.48, 0.21, 0.21, 1))
C3 = Workload(
    "C3", "Dense-6/7/8 (33 queries, K_k - M, P:1323-1328) on R-MAT(20,10,.48,.21,.21); hybrid count",
    ((C3_GRAPH, tuple(dense_family(6) + dense_family(7) + dense_family(8))),))

# configs[3]: 8-vertex dense query on R-MAT scale 22 forcing hybrid BFS/DFS chunking
# beyond 180 GB: K8 on R-MAT(22, 16, .50, .20, .20) (n 4,194,304, 66.9 M edges, CSR
# 547 MB), restricted to the stated canonical level-1 positions [13500, 14400) of
# 1,834,382 (SURVEY §8.d allows a stated root range).  Calibrated in round 2
# (profiles/r02b_c4_calibration.jsonl, r02g): the work sits on the hub roots
# (degree tiers ~45 K, ~21 K, ~9.4 K, ~4 K); this range holds one ~21 K hub
# (position 14341) and one ~9.4 K hub (13997) among 900 roots.  Levels 9.1e4 /
# 2.2e6 / 5.6e7 / 1.5e9 / 3.8e10 / 9.1e11, count 2.02e13: the stored level 6 alone
# is 304 GB of 8 B trie entries (level 7, 7.3 TB, is never stored), so it is cut
# into DFS chunks.  The round-1 range [0, 1/16) holds two ~21 K hubs (1,604 s/pass
# on the round-1 kernel).
C4_GRAPH = GraphSpec("rmat_t", (22, 16, 0.50, 0.20, 0.20, 1))
C4 = Workload(
    "C4", "K8 on R-MAT(22,16,.50,.20,.20), canonical roots [13500, 14400) (a ~21K- and a ~9.4K-degree hub); "
          "hybrid count, stored level > 180 GB",
    ((C4_GRAPH, (dense_family(8)[0],)),), root_range=(13500, 14400, 0), min_trie_bytes=180e9)

WORKLOADS = {"C1": C1, "C2": C2, "C3": C3, "C4": C4}
