"""Named benchmark workloads (BASELINE.json configs -> concrete seeded inputs).

Holds no matching arithmetic: it only names graphs (generator + parameters)
and query lists from ``inputs``.  Calibration record: DESIGN.md §3 and
profiles/r01_calibration.md.
"""
from __future__ import annotations

from dataclasses import dataclass

from inputs import rmat_graph, er_graph, named_query, DENSE5, SPARSE5, dense_family


@dataclass(frozen=True)
class GraphSpec:
    kind: str
    params: tuple

    def build(self):
        if self.kind == "rmat":
            return rmat_graph(*self.params)
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

WORKLOADS = {"C1": C1, "C2": C2}
