"""Seeded synthetic inputs shared by the oracle tests and the CUDA path.

This package only *builds inputs*: graphs as canonical CSR arrays and query
graphs as small edge lists.  It holds none of the matching arithmetic (no
ordering, no intersection, no filtering, no counting), so both sides of every
parity test can take their inputs from here without sharing method code
(task rule ③).  The recipes are stated in DESIGN.md §3.
"""
from .graphs import (CSRGraph, canonical_csr, er_graph, rmat_graph, rmat_graph_torch, cycle_graph,
                     complete_graph, path_graph, star_graph, grid_graph,
                     petersen_graph, hypercube_graph, complete_bipartite_graph,
                     graph_from_edges)
from .digraphs import (DiGraph, DiQuery, digraph_from_arcs, directed_er_graph, directed_rmat_graph,
                       directed_cycle, transitive_tournament, complete_digraph, query_from_arcs,
                       named_diquery, DIRECTED_QUERIES)
from .queries import (Query, query_from_edges, k_minus, DENSE5, SPARSE5, m11,
                      dense_family, named_query)

__all__ = [
    "CSRGraph", "canonical_csr", "er_graph", "rmat_graph", "rmat_graph_torch", "cycle_graph",
    "complete_graph", "path_graph", "star_graph", "grid_graph", "petersen_graph",
    "hypercube_graph", "complete_bipartite_graph", "graph_from_edges",
    "Query", "query_from_edges", "k_minus", "DENSE5", "SPARSE5", "m11",
    "dense_family", "named_query",
    "DiGraph", "DiQuery", "digraph_from_arcs", "directed_er_graph", "directed_rmat_graph",
    "directed_cycle", "transitive_tournament", "complete_digraph", "query_from_arcs",
    "named_diquery", "DIRECTED_QUERIES",
]
