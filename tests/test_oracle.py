"""Pins for the CPU oracle (runs with -m "not gpu").

Every test compares the oracle against something other than itself: closed
forms, brute force over all injective maps, networkx's VF2 monomorphism
enumerator, scipy sparse traces, or values printed in the paper.
"""
import itertools
import json
import math
import os

import numpy as np
import pytest

import oracle
from inputs import (er_graph, rmat_graph, complete_graph, cycle_graph, path_graph, star_graph,
                    grid_graph, petersen_graph, hypercube_graph, complete_bipartite_graph,
                    graph_from_edges, query_from_edges, named_query, DENSE5, SPARSE5,
                    dense_family, k_minus)
from tests import bruteforce

GOLDEN = os.path.join(os.path.dirname(__file__), "golden")


def falling(x, s):
    r = 1
    for i in range(s):
        r *= (x - i)
    return r


# ----------------------------------------------------------------- closed forms
@pytest.mark.parametrize("n", [5, 6, 7])
@pytest.mark.parametrize("qname", ["K3", "C4", "P4", "S3", "K5", "K5-P5", "cricket", "C5", "K1_4"])
def test_complete_host_any_query(n, qname):
    """In K_n every injective map is an embedding: n!/(n-k)!."""
    q = named_query(qname)
    assert oracle.count(complete_graph(n), q) == math.perm(n, q.k)


@pytest.mark.parametrize("n", [3, 4, 5, 8, 11])
def test_cycles_in_cycle(n):
    for k in range(3, 9):
        want = 2 * n if k == n else 0
        assert oracle.count(cycle_graph(n), named_query(f"C{k}")) == want


@pytest.mark.parametrize("n", [4, 6, 9])
def test_paths_in_cycle(n):
    for k in range(2, min(n, 8) + 1):
        assert oracle.count(cycle_graph(n), named_query(f"P{k}")) == 2 * n


@pytest.mark.parametrize("seed", [1, 2, 3])
def test_stars_degree_sequence(seed):
    """K1,s: sum_v d(v)(d(v)-1)...(d(v)-s+1); P3 = K1,2; K2 = 2m; K1 = n."""
    g = er_graph(300, 1500, seed)
    d = g.degrees()
    for s in (1, 2, 3, 4, 5):
        assert oracle.count(g, named_query(f"S{s}")) == sum(falling(int(x), s) for x in d)
    assert oracle.count(g, named_query("P3")) == sum(int(x) * (int(x) - 1) for x in d)
    assert oracle.count(g, named_query("K1")) == g.n
    assert oracle.count(g, named_query("P2")) == 2 * g.m


def _adj_sparse(g):
    import scipy.sparse as sp
    return sp.csr_matrix((np.ones(g.nnz, dtype=np.int64), g.col.astype(np.int64),
                          g.row_ptr.astype(np.int64)), shape=(g.n, g.n))


@pytest.mark.parametrize("seed", [1, 2, 3, 4, 5])
def test_triangle_and_c4_traces_er1000(seed):
    """C1 workload (BASELINE configs[0]): K3 = tr(A^3); C4 = tr(A^4) - 2 sum d^2 + sum d."""
    g = er_graph(1000, 4000, seed)
    A = _adj_sparse(g)
    A2 = A @ A
    tr3 = int((A2.multiply(A)).sum())
    tr4 = int((A2.multiply(A2)).sum())
    d = g.degrees()
    assert oracle.count(g, named_query("K3")) == tr3
    assert oracle.count(g, named_query("C4")) == tr4 - 2 * int((d * d).sum()) + int(d.sum())


def test_traces_rmat12():
    g = rmat_graph(10, 4, 0.57, 0.19, 0.19, seed=3)
    A = _adj_sparse(g)
    A2 = A @ A
    d = g.degrees()
    assert oracle.count(g, named_query("K3")) == int((A2.multiply(A)).sum())
    assert oracle.count(g, named_query("C4")) == int((A2.multiply(A2)).sum()) - 2 * int((d * d).sum()) + int(d.sum())


def test_structured_hosts():
    assert oracle.count(petersen_graph(), named_query("C5")) == 120
    assert oracle.count(petersen_graph(), named_query("K3")) == 0
    assert oracle.count(petersen_graph(), named_query("C4")) == 0
    assert oracle.count(hypercube_graph(3), named_query("C4")) == 48
    for a, b in [(2, 3), (3, 4), (4, 4)]:
        assert oracle.count(complete_bipartite_graph(a, b), named_query("C4")) == 2 * a * (a - 1) * b * (b - 1)
    grid = grid_graph(4, 4)
    assert oracle.count(grid, named_query("P3")) == 104
    assert oracle.count(grid, named_query("P4")) == 232


def test_fig2_mesh_chain_levels():
    """Fig. 2: 4x4 mesh, 4-vertex chain.  The paper prints 16 and 48
    candidates at depths 1 and 2 (exact); its depth-3/4 values 96/192 are
    schematic (reading P19), so depths 3/4 are pinned by brute force instead."""
    g = grid_graph(4, 4)
    q = named_query("P4")
    S = oracle.order(q)
    total, lv = oracle.count(g, q, levels=True)
    assert lv[1] == 16 and lv[2] == 48
    assert lv == bruteforce.level_sizes(g, q, S)
    assert total == lv[4] == 232


# ------------------------------------------------------------------ brute force
def _tiny_graphs():
    gs = [er_graph(8, 14, s) for s in (1, 2, 3)] + [er_graph(9, 20, 4), er_graph(7, 18, 5)]
    gs.append(graph_from_edges(8, [(0, 1), (1, 2), (2, 0), (2, 3), (3, 4), (4, 5), (5, 3), (6, 7)]))
    return gs


@pytest.mark.parametrize("gi", range(6))
def test_bruteforce_all_5vertex_queries(gi):
    g = _tiny_graphs()[gi]
    for q in DENSE5 + SPARSE5:
        want = bruteforce.embeddings(g, q)
        assert oracle.count(g, q) == len(want), q.name
        rows = oracle.enumerate_rows(g, q)
        assert [tuple(r) for r in rows.tolist()] == want, q.name


@pytest.mark.parametrize("gi", range(6))
def test_bruteforce_level_sizes(gi):
    g = _tiny_graphs()[gi]
    for q in [named_query("K3"), named_query("C4"), named_query("P4"), DENSE5[2], SPARSE5[2], SPARSE5[6]]:
        S = oracle.order(q)
        _, lv = oracle.count(g, q, levels=True)
        assert lv == bruteforce.level_sizes(g, q, S), q.name


def test_bruteforce_small_queries_k1_to_4():
    g = er_graph(9, 16, 7)
    for q in [named_query("K1"), named_query("P2"), named_query("P3"), named_query("K3"),
              named_query("S3"), named_query("C4"), named_query("K4"),
              query_from_edges(4, [(0, 1), (1, 2), (2, 0), (2, 3)])]:
        assert oracle.count(g, q) == len(bruteforce.embeddings(g, q)), q.name


# ---------------------------------------------------------------- networkx VF2
def _nx(g):
    import networkx as nx
    G = nx.Graph()
    G.add_nodes_from(range(g.n))
    G.add_edges_from(g.edge_list().tolist())
    return G


@pytest.mark.parametrize("seed", [1, 2])
def test_networkx_vf2_monomorphisms(seed):
    """Library routine: networkx GraphMatcher.subgraph_monomorphisms_iter (VF2)."""
    from networkx.algorithms import isomorphism
    g = er_graph(30, 100, seed)
    G = _nx(g)
    for q in DENSE5[4:] + SPARSE5[:3] + [named_query("C4"), named_query("K4")]:
        Q = _nx(type(g)(n=q.k, row_ptr=q.csr()[0].astype(np.uint64), col=q.csr()[1]))
        gm = isomorphism.GraphMatcher(G, Q)
        # mapping is data->query; convert to rows indexed by query vertex
        rows = sorted(tuple(inv[qv] for qv in range(q.k))
                      for m in gm.subgraph_monomorphisms_iter()
                      for inv in [{v: u for u, v in m.items()}])
        got = [tuple(r) for r in oracle.enumerate_rows(g, q).tolist()]
        assert got == rows, q.name


# ------------------------------------------------------------------- invariants
def _aut(q):
    qe = {(u, v) for u, v in q.edges} | {(v, u) for u, v in q.edges}
    return sum(all((p[u], p[v]) in qe for u, v in q.edges) for p in itertools.permutations(range(q.k)))


def test_automorphism_divides_count():
    g = rmat_graph(8, 4, 0.57, 0.19, 0.19, seed=2)
    for q in DENSE5 + SPARSE5:
        c = oracle.count(g, q)
        assert c % _aut(q) == 0, q.name


def _valid_orders(q):
    qe = {(u, v) for u, v in q.edges} | {(v, u) for u, v in q.edges}
    for p in itertools.permutations(range(q.k)):
        if all(any((p[i], p[j]) in qe for j in range(i)) for i in range(1, q.k)):
            yield list(p)


def test_order_invariance():
    g = er_graph(60, 300, 3)
    for q in [DENSE5[5], SPARSE5[0], SPARSE5[4], named_query("C4")]:
        base = oracle.count(g, q)
        for o in list(_valid_orders(q))[::7]:
            assert oracle.count(g, q, order=o) == base, (q.name, o)


def test_subquery_monotone():
    """Q ⊆ Q' on the same vertices => count(Q') <= count(Q) (down the Dense-5 family)."""
    g = rmat_graph(8, 4, 0.57, 0.19, 0.19, seed=5)
    fam = sorted(DENSE5, key=lambda q: len(q.edges))
    cnt = {q.name: oracle.count(g, q) for q in fam}
    for a in fam:
        for b in fam:
            if set(a.edges) <= set(b.edges):
                assert cnt[b.name] <= cnt[a.name], (a.name, b.name)


def test_root_ranges_partition():
    g = er_graph(200, 1200, 9)
    q = DENSE5[8]
    total = oracle.count(g, q)
    l1 = oracle.level1_size(g, max(q.degrees()))
    cuts = [0, 17, 50, 51, 120, l1]
    assert sum(oracle.count(g, q, root_begin=a, root_end=b) for a, b in zip(cuts, cuts[1:])) == total


def test_clique_levels_table1_structure():
    """Table 1 structure: for a K_k query every level j holds
    j! x (#j-cliques among vertices of degree >= k-1) ordered partial paths."""
    import networkx as nx
    g = rmat_graph(9, 4, 0.57, 0.19, 0.19, seed=4)
    k = 5
    G = _nx(g)
    keep = [v for v in range(g.n) if G.degree(v) >= k - 1]
    H = G.subgraph(keep)
    cl = [0] * (k + 1)
    for c in nx.enumerate_all_cliques(H):
        if len(c) <= k:
            cl[len(c)] += 1
    _, lv = oracle.count(g, named_query("K5"), levels=True)
    for j in range(1, k + 1):
        assert lv[j] == math.factorial(j) * cl[j]


# ---------------------------------------------------------------- order rule
def test_order_rule_paper():
    """P:518-530 with min-id ties (readings P5/P6), derived by hand."""
    assert oracle.order(named_query("cricket")) == [0, 1, 2, 3, 4]          # degs 4,2,2,1,1
    assert oracle.order(named_query("P5")) == [1, 2, 3, 0, 4]               # degs 1,2,2,2,1
    assert oracle.order(named_query("K5-K13")) == [4, 1, 2, 3, 0]           # degs 1,3,3,3,4
    assert oracle.order(named_query("chair")) == [1, 2, 0, 3, 4]            # degs 1,3,2,1,1
    assert oracle.order(named_query("K5-paw")) == [4, 3, 0, 1, 2]           # degs 2,2,1,3,4
    assert oracle.order(query_from_edges(4, [(0, 1), (1, 2), (2, 3), (3, 0)])) == [0, 1, 2, 3]


def test_root_is_min_candidate_set():
    """the max-degree root has the smallest level-1 set."""
    g = rmat_graph(10, 8, seed=2)
    for q in DENSE5 + SPARSE5:
        d = q.degrees()
        root = oracle.order(q)[0]
        assert all(oracle.level1_size(g, d[root]) <= oracle.level1_size(g, d[v]) for v in range(q.k))


# ----------------------------------------------------------------- validation
def test_validation():
    assert oracle.validate_graph(er_graph(50, 100, 1))
    assert oracle.validate_graph(rmat_graph(8, 4, seed=1))
    from inputs import CSRGraph
    bad_asym = CSRGraph(n=3, row_ptr=np.array([0, 1, 1, 1], np.uint64), col=np.array([1], np.uint32))
    bad_loop = CSRGraph(n=2, row_ptr=np.array([0, 1, 1], np.uint64), col=np.array([0], np.uint32))
    bad_sort = CSRGraph(n=3, row_ptr=np.array([0, 2, 3, 4], np.uint64), col=np.array([2, 1, 0, 0], np.uint32))
    for g in (bad_asym, bad_loop, bad_sort):
        assert not oracle.validate_graph(g)
    with pytest.raises(oracle.OracleError):
        oracle.count(er_graph(20, 30, 1), named_query("P4"), order=[0, 2, 1, 3])   # order not connected


# -------------------------------------------------------------- trie (Fig. 3)
def test_fig3_trie_decode_matches_csf():
    """Fig. 3: decoding the cuTS (CA, PA) trie gives the same
    root-to-leaf paths as walking the paper's CSF (nodeid, index) arrays."""
    fx = json.load(open(os.path.join(GOLDEN, "fig3_trie.json")))
    got = [tuple(r) for r in oracle.trie_decode(fx["cuts_CA"], fx["cuts_PA"]).tolist()]
    # independent CSF walk: children of node x at level l are index[l][x]..index[l][x+1]
    nid, idx = fx["csf_nodeid"], fx["csf_index"]
    paths = []

    def walk(level, x, prefix):
        p = prefix + (nid[level][x],)
        if level == len(nid) - 1:
            paths.append(p)
            return
        for y in range(idx[level][x], idx[level][x + 1]):
            walk(level + 1, y, p)
    for x in range(len(nid[0])):
        walk(0, x, ())
    assert got == paths
    assert len(got) == 8 and got[0] == (0, 3, 2, 5) and got[-1] == (1, 2, 3, 4)


def test_rmat_torch_generator_is_byte_identical():
    """The torch R-MAT generator (used for the scale-20/22 configs) must emit the
    same canonical CSR bytes as the numpy reference generator."""
    from inputs import rmat_graph_torch
    for args in [(10, 8, 0.57, 0.19, 0.19, 3), (11, 16, 0.45, 0.22, 0.22, 1), (9, 4, 0.35, 0.22, 0.22, 7)]:
        a, b = rmat_graph(*args), rmat_graph_torch(*args, block=1 << 12)
        assert np.array_equal(a.row_ptr, b.row_ptr) and np.array_equal(a.col, b.col), args


# ------------------------------------------------- disconnected Q
# The oracle composes per-component results by the paper's cross product; these
# pins fix it against the plain definition (injective maps) independently.
DISCONNECTED = {
    "2K1": (2, []), "3K1": (3, []), "K2uK1": (3, [(0, 1)]), "2K2": (4, [(0, 1), (2, 3)]),
    "K3uK1": (4, [(0, 1), (1, 2), (0, 2)]), "P3uK2": (5, [(0, 1), (1, 2), (3, 4)]),
    "K4uK1": (5, [(0, 1), (0, 2), (0, 3), (1, 2), (1, 3), (2, 3)]),   # the P:1325-1327 tie member
    "K2uK1_mid": (3, [(0, 2)]), "K3uK2": (5, [(0, 3), (3, 4), (0, 4), (1, 2)]),
}


@pytest.mark.parametrize("name", sorted(DISCONNECTED))
@pytest.mark.parametrize("gi", [0, 1, 2])
def test_disconnected_bruteforce(name, gi):
    """Cross product of the component results, injective combinations only
    (reading P16) == brute force over every injective vertex map."""
    k, es = DISCONNECTED[name]
    q = query_from_edges(k, es)
    g = [er_graph(8, 12, 5), petersen_graph(), graph_from_edges(7, [(0, 1), (1, 2), (2, 0), (3, 4), (5, 6), (4, 5)])][gi]
    want = bruteforce.embeddings(g, q)
    got = [tuple(r) for r in oracle.enumerate_rows(g, q).tolist()]
    assert got == want
    assert oracle.count(g, q) == len(want)


@pytest.mark.parametrize("seed", [1, 2])
def test_disconnected_closed_forms(seed):
    """kK1: falling(n, k); Q ∪ K1: count(Q) * (n - |Q|) (the isolated query
    vertex takes any unused data vertex); 2K2: 4m^2 - 4 Σ d(v)^2 + 4m
    (ordered edge pairs minus those sharing an endpoint)."""
    g = er_graph(60, 150, seed)
    d = [int(x) for x in g.degrees()]
    m = sum(d) // 2
    for k in (1, 2, 3):
        assert oracle.count(g, query_from_edges(k, [])) == falling(g.n, k)
    for qname in ("K3", "P3", "C4"):
        q = named_query(qname)
        qq = query_from_edges(q.k + 1, q.edges)
        assert oracle.count(g, qq) == oracle.count(g, q) * (g.n - q.k)
    assert oracle.count(g, query_from_edges(4, [(0, 1), (2, 3)])) == 4 * m * m - 4 * sum(x * x for x in d) + 4 * m


def test_disconnected_complete_host():
    """In K_n every injective map is an embedding, connected or not."""
    for k, es in DISCONNECTED.values():
        assert oracle.count(complete_graph(7), query_from_edges(k, es)) == math.perm(7, k)


# ------------------------------------------------------- directed (NEXT-1)
from inputs import (directed_er_graph, directed_rmat_graph, directed_cycle, transitive_tournament,
                    complete_digraph, digraph_from_arcs, query_from_arcs, named_diquery, DIRECTED_QUERIES)


@pytest.mark.parametrize("qname", sorted(DIRECTED_QUERIES))
def test_directed_closed_forms(qname):
    """Complete digraph: every injective map (n!/(n-k)!).  Transitive
    tournament: a query embeds iff it is acyclic, C(n, k) maps for TT_k."""
    q = named_diquery(qname)
    assert oracle.di_count(complete_digraph(7), q) == math.perm(7, q.k)
    if qname.startswith("TT"):
        assert oracle.di_count(transitive_tournament(8), q) == math.comb(8, q.k)
    if qname.startswith("dC"):
        assert oracle.di_count(transitive_tournament(8), q) == 0


@pytest.mark.parametrize("n", [3, 4, 5, 7])
def test_directed_cycles_and_paths(n):
    for k in (3, 4, 5):
        want = n if k == n else 0
        assert oracle.di_count(directed_cycle(n), named_diquery(f"dC{k}")) == want
    assert oracle.di_count(directed_cycle(n), named_diquery("dP3")) == n


@pytest.mark.parametrize("seed", [1, 2])
def test_directed_degree_sequence_forms(seed):
    """out-star: Σ out(out-1); in-star: Σ in(in-1); dP3 a->b->c (a != c):
    Σ_b in(b) out(b) - 2 * #reciprocal pairs."""
    g = directed_er_graph(200, 1500, seed)
    od, idg = g.out_degrees(), g.in_degrees()
    arcs = {(int(a), int(b)) for a, b in g.arcs()}
    recip = sum(1 for a, b in arcs if (b, a) in arcs) // 2
    assert recip > 0
    assert oracle.di_count(g, named_diquery("out2")) == int((od * (od - 1)).sum())
    assert oracle.di_count(g, named_diquery("in2")) == int((idg * (idg - 1)).sum())
    assert oracle.di_count(g, named_diquery("dP3")) == int((od * idg).sum()) - 2 * recip


@pytest.mark.parametrize("gi", [0, 1, 2])
def test_directed_bruteforce(gi):
    g = [directed_er_graph(7, 18, 3), directed_er_graph(8, 25, 4), directed_rmat_graph(3, 4, seed=5)][gi]
    for name in ("dP3", "dC3", "TT3", "out2", "in2", "dC4", "TT4", "bifan", "diamond"):
        q = named_diquery(name)
        want = bruteforce.di_embeddings(g, q)
        assert [tuple(r) for r in oracle.di_enumerate_rows(g, q).tolist()] == want, name
        c, lv = oracle.di_count(g, q, levels=True)
        assert c == len(want)
        assert lv == bruteforce.di_level_sizes(g, q, oracle.di_order(q)), name


def test_directed_reduces_to_undirected():
    """an undirected graph is the digraph with both arcs; with
    symmetric queries (reciprocal arcs) the directed oracle equals the
    undirected one."""
    g = er_graph(40, 120, 7)
    dg = digraph_from_arcs(g.n, [(int(u), int(v)) for u, v in g.edge_list()] +
                           [(int(v), int(u)) for u, v in g.edge_list()])
    for qname in ("K3", "C4", "P4", "K4", "S3"):
        q = named_query(qname)
        dq = query_from_arcs(q.k, list(q.edges) + [(v, u) for u, v in q.edges])
        assert oracle.di_count(dg, dq) == oracle.count(g, q), qname


def test_directed_order_rule():
    """Root = max out-degree, ties min id; then weakly adjacent."""
    assert oracle.di_order(named_diquery("in2")) == [1, 0, 2]
    assert oracle.di_order(named_diquery("out2")) == [0, 1, 2]
    assert oracle.di_order(named_diquery("TT6-rev")) == [5, 4, 3, 2, 1, 0]


def test_root_parallel_driver_matches_single_thread():
    """oracle_count_mt (the N-core CPU baseline) sums
    disjoint root ranges counted by the same rec(): equal to the single-threaded
    count for every thread count / grain and every root range."""
    from inputs import rmat_graph, DENSE5, SPARSE5
    g = rmat_graph(9, 4, seed=2)
    for q in (DENSE5[9], SPARSE5[1], named_query("K3")):
        want = oracle.count(g, q)
        for threads, grain in ((1, 1), (3, 1), (4, 7), (8, 64)):
            assert oracle.count_mt(g, q, threads, grain=grain) == want, (q.name, threads, grain)
        assert oracle.count_mt(g, q, 4, 10, 50, grain=3) == oracle.count(g, q, root_begin=10, root_end=50)
