"""GPU parity for directed graphs: the CUDA path
through cuts_load_digraph / cuts_set_query_directed against the directed
oracle (children lists = c-intersection, parents lists = p-intersection,
Alg. 2 l.19-42).  Bit-exact counts, per-level sizes, sorted rows."""
import math

import numpy as np
import pytest

import oracle
from inputs import (directed_er_graph, directed_rmat_graph, directed_cycle, transitive_tournament,
                    complete_digraph, digraph_from_arcs, query_from_arcs, named_diquery, DIRECTED_QUERIES,
                    er_graph, named_query)

pytestmark = pytest.mark.gpu


@pytest.fixture(scope="module")
def cuts():
    torch = pytest.importorskip("torch")
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    from paper_conf_sc_xiangkshs21_b200 import Cuts
    return Cuts


def _rows(t):
    a = t.cpu().numpy().view(np.uint32)
    return a[np.lexsort(a.T[::-1])] if a.size else a.reshape(0, t.shape[1])


def _set(c, q, order=None):
    qr, qc = q.csr()
    c.set_query_directed(qr, qc, order)


@pytest.mark.parametrize("gname", ["der300", "drmat10", "drmat12"])
def test_directed_queries(cuts, gname):
    g = {"der300": lambda: directed_er_graph(300, 3000, 1),
         "drmat10": lambda: directed_rmat_graph(10, 8, seed=2),
         "drmat12": lambda: directed_rmat_graph(12, 8, 0.45, 0.22, 0.22, seed=3)}[gname]()
    big = cuts(device=0, arena_bytes=1 << 30)
    small = cuts(device=0, arena_bytes=256 << 10)
    big.load_digraph(g, validate=True)
    small.load_digraph(g)
    for name in sorted(DIRECTED_QUERIES):
        q = named_diquery(name)
        want, lv = oracle.di_count(g, q, levels=True)
        _set(big, q)
        _set(small, q)
        assert big.count("bfs") == want, (gname, name)
        st = big.stats()
        assert st["order"] == oracle.di_order(q), name
        assert st["level_size"] == lv, (gname, name, st["level_size"], lv)
        assert big.count("hybrid") == want, (gname, name)
        assert small.count("hybrid") == want, (gname, name)
        if want <= 1_000_000:
            rows = big.enumerate("hybrid", cap_rows=want)
            assert np.array_equal(_rows(rows), oracle.di_enumerate_rows(g, q)), (gname, name)


def test_directed_closed_forms_gpu(cuts):
    c = cuts(device=0, arena_bytes=1 << 28)
    c.load_digraph(complete_digraph(9), validate=True)
    for name in sorted(DIRECTED_QUERIES):
        q = named_diquery(name)
        _set(c, q)
        assert c.count("hybrid") == math.perm(9, q.k), name
    c.load_digraph(transitive_tournament(12), validate=True)
    for name in ("TT3", "TT4", "TT5", "TT6-rev"):
        _set(c, named_diquery(name))
        assert c.count("hybrid") == math.comb(12, named_diquery(name).k), name
    _set(c, named_diquery("dC3"))
    assert c.count("hybrid") == 0
    c.load_digraph(directed_cycle(5), validate=True)
    _set(c, named_diquery("dC5"))
    assert c.count("bfs") == 5


def test_directed_orders_and_errors(cuts):
    from paper_conf_sc_xiangkshs21_b200 import CutsError
    g = directed_er_graph(120, 900, 5)
    c = cuts(device=0, arena_bytes=1 << 28)
    c.load_digraph(g, validate=True)
    q = named_diquery("diamond")
    want = oracle.di_count(g, q)
    for order in ([0, 1, 2, 3], [3, 2, 1, 0], [1, 0, 3, 2], [2, 3, 0, 1]):
        _set(c, q, order)
        assert c.count("hybrid") == want, order
        assert c.stats()["level_size"] == oracle.di_count(g, q, order=order, levels=True)[1], order
    # reciprocal arcs at one position need two lists of one neighbour
    with pytest.raises(CutsError) as ei:
        c.set_query_arcs(2, [(0, 1), (1, 0)])
    assert ei.value.status == -7
    # an undirected query on a directed graph
    qr, qc = named_query("K3").csr()
    c.set_query(qr, qc)
    with pytest.raises(CutsError) as ei:
        c.count("hybrid")
    assert ei.value.status == -1
    # in-rows that are not the transpose of the out-rows
    bad = directed_er_graph(30, 60, 1)
    rp, cl = bad.combined()
    cl = cl.copy()
    cl[-1] = (cl[-1] + 1) % 30 if (cl[-1] + 1) % 30 != 29 else 0
    with pytest.raises(CutsError):
        c.load_graph(rp, cl, validate=True, directed=True)


def test_symmetric_digraph_matches_undirected(cuts):
    """the digraph with both arcs of every edge; an acyclic
    orientation of K4 on it counts what the oracle counts."""
    g = er_graph(400, 3000, 2)
    e = [(int(u), int(v)) for u, v in g.edge_list()]
    dg = digraph_from_arcs(g.n, e + [(v, u) for u, v in e])
    c = cuts(device=0, arena_bytes=1 << 28)
    c.load_digraph(dg, validate=True)
    for name in ("TT4", "dC4", "bifan", "TT5"):
        q = named_diquery(name)
        _set(c, q)
        assert c.count("hybrid") == oracle.di_count(dg, q), name
    # TT_k on a symmetric digraph = ordered K_k embeddings
    _set(c, named_diquery("TT4"))
    assert c.count("hybrid") == oracle.count(g, named_query("K4"))
