"""GPU parity: the CUDA path (through the C ABI) against the CPU oracle.

Integer work, so the bar is bit-exact: counts, per-level trie sizes (same
matching order on both sides) and sorted embedding rows.  Row order inside the
trie is unspecified, so rows are compared after sorting.
"""
import json
import os

import numpy as np
import pytest

import oracle
from inputs import (er_graph, rmat_graph, grid_graph, complete_graph, cycle_graph, star_graph,
                    graph_from_edges, named_query, query_from_edges, DENSE5, SPARSE5, dense_family)

pytestmark = pytest.mark.gpu

GOLDEN = os.path.join(os.path.dirname(__file__), "golden")


@pytest.fixture(scope="module")
def cuts():
    torch = pytest.importorskip("torch")
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    from paper_conf_sc_xiangkshs21_b200 import Cuts
    return Cuts


@pytest.fixture(scope="module")
def ctx(cuts):
    return cuts(device=0, arena_bytes=1 << 30)


def _set(ctx, q, order=None):
    qr, qc = q.csr()
    ctx.set_query(qr, qc, order)


def _sorted_rows(t):
    a = t.cpu().numpy().view(np.uint32)
    if a.size == 0:
        return a.reshape(0, t.shape[1] if t.dim() == 2 else 0)
    return a[np.lexsort(a.T[::-1])]


def _check_full(ctx, g, q, enumerate_=True, modes=("bfs", "hybrid")):
    want, lv = oracle.count(g, q, levels=True)
    _set(ctx, q)
    for mode in modes:
        got = ctx.count(mode)
        assert got == want, (g.name, q.name, mode, got, want)
        st = ctx.stats()
        assert st["level_size"] == lv, (g.name, q.name, mode, st["level_size"], lv)
        assert st["order"] == oracle.order(q)
    if enumerate_:
        rows = ctx.enumerate("hybrid", cap_rows=want)
        assert np.array_equal(_sorted_rows(rows), oracle.enumerate_rows(g, q)), (g.name, q.name)


# ----------------------------------------------------------------- C1 config
@pytest.mark.parametrize("seed", [1, 2, 3, 4, 5])
def test_c1_er1000_triangle_c4(ctx, seed):
    """BASELINE configs[0]: K3 and C4 on ER G(1000, 4000), count + levels + sorted rows."""
    g = er_graph(1000, 4000, seed)
    ctx.load_csr(g, validate=True)
    for q in (named_query("K3"), named_query("C4")):
        _check_full(ctx, g, q)


def test_c1_tiny_arena_hybrid_and_bfs_enomem(cuts):
    """Fault injection: a 64 KiB arena forces many hybrid chunks;
    BFS must report CUTS_ENOMEM where a level does not fit."""
    from paper_conf_sc_xiangkshs21_b200 import CutsError
    g = er_graph(1000, 4000, 1)
    small = cuts(device=0, arena_bytes=64 << 10)
    small.load_csr(g)
    q = named_query("C4")
    want, lv = oracle.count(g, q, levels=True)
    _set(small, q)
    assert small.count("hybrid") == want
    st = small.stats()
    assert st["level_size"] == lv and st["chunks"] > 10
    with pytest.raises(CutsError) as ei:
        small.count("bfs")
    assert ei.value.status == -2


@pytest.mark.parametrize("arena_kib", [64, 96, 256, 1024])
def test_chunk_invariance(cuts, arena_kib):
    g = rmat_graph(9, 4, seed=2)
    c = cuts(device=0, arena_bytes=arena_kib << 10)
    c.load_csr(g)
    for q in (DENSE5[9], SPARSE5[3], named_query("C4")):
        want, lv = oracle.count(g, q, levels=True)
        _set(c, q)
        assert c.count("hybrid") == want, (arena_kib, q.name)
        assert c.stats()["level_size"] == lv


@pytest.mark.parametrize("arena_kib", [64, 128, 512, 4096])
def test_ancestor_reuse_chunked(cuts, arena_kib):
    """HYBRID's ancestor-set source (ordered levels, entry-aligned chunks and the
    oversized-entry fallback at tiny arenas) against the oracle and against the
    same run with the reuse disabled (CUTS_DEBUG_NO_REUSE)."""
    g = rmat_graph(8, 6, a=0.5, b=0.2, c=0.2, seed=3)
    c = cuts(device=0, arena_bytes=arena_kib << 10)
    c.load_csr(g)
    qs = [DENSE5[0], DENSE5[3], DENSE5[5]] + dense_family(6)[::3] + dense_family(7)[::4] + dense_family(8)[::5]
    if arena_kib <= 128:
        qs = qs[::2]
    for q in qs:
        want, lv = oracle.count(g, q, levels=True)
        _set(c, q)
        for flags in (0, 4, 512):        # default (pair-shared last level), no reuse, no pair sharing
            c.lib.cuts_set_debug(c.h, flags)
            assert c.count("hybrid") == want, (arena_kib, q.name, flags)
            assert c.stats()["level_size"] == lv, (arena_kib, q.name, flags)
        c.set_debug()


def test_packed_degree_stream_ablation(cuts):
    """The packed (id | min(deg,31)) candidate stream against the plain col + deg
    gather (CUTS_DEBUG_NO_PACK at load): same counts and level sizes, incl. degree
    thresholds above 1 and hubs with degree >= 31."""
    g = rmat_graph(8, 5, a=0.55, b=0.2, c=0.2, seed=4)
    assert g.degrees().max() > 31
    c = cuts(device=0, arena_bytes=64 << 20)
    for flags in (0, 8):
        c.lib.cuts_set_debug(c.h, flags)
        c.load_csr(g)
        for q in (DENSE5[9], DENSE5[10], SPARSE5[1], SPARSE5[4], named_query("C4"), dense_family(6)[5]):
            want, lv = oracle.count(g, q, levels=True)
            _set(c, q)
            for mode in ("hybrid", "bfs"):
                assert c.count(mode) == want, (flags, q.name, mode)
                assert c.stats()["level_size"] == lv, (flags, q.name, mode)
    c.set_debug()


def test_first_source_ablation(cuts):
    """NEXT-2 ablation: streaming the FIRST backward list (Alg. 2's a1,
    CUTS_DEBUG_FIRST_SOURCE) instead of the shortest gives the same counts,
    level sizes and rows, with and without hubs and reuse."""
    g = rmat_graph(9, 8, a=0.55, b=0.2, c=0.2, seed=6)
    c = cuts(device=0, arena_bytes=4 << 20)
    for hub in (None, 0):
        c.set_hub_threshold(hub)
        c.load_csr(g)
        for q in DENSE5[::3] + SPARSE5[::4] + dense_family(6)[::6]:
            want, lv = oracle.count(g, q, levels=True)
            _set(c, q)
            for kw in ({"first_source": True}, {"first_source": True, "no_reuse": True}):
                c.set_debug(**kw)
                assert c.count("hybrid") == want, (hub, q.name, kw)
                assert c.stats()["level_size"] == lv, (hub, q.name, kw)
        c.set_debug(first_source=True)
        q = DENSE5[5]
        want = oracle.count(g, q)
        _set(c, q)
        if want <= 2_000_000:
            assert np.array_equal(_sorted_rows(c.enumerate("hybrid", cap_rows=want)), oracle.enumerate_rows(g, q))
        c.set_debug()


@pytest.mark.parametrize("arena_kib", [64, 256 << 10])
def test_fast_last_level_count(cuts, arena_kib):
    """Single-list degree-free last level of cuts_count (|list| - path vertices
    found by binary search) against the oracle and against the streamed list
    (CUTS_DEBUG_NO_FAST_COUNT), incl. hybrid chunks that split an entry's list."""
    g = rmat_graph(9, 8, a=0.55, b=0.2, c=0.2, seed=8)
    c = cuts(device=0, arena_bytes=arena_kib << 10)
    c.load_csr(g)
    qs = [q for q in SPARSE5 if q.name in ("P5", "K1_4", "chair", "bull", "cricket")]
    qs += [named_query(x) for x in ("P3", "P4", "S3", "K2")] + [query_from_edges(4, [(0, 1), (1, 2), (0, 2), (2, 3)])]
    if arena_kib == 64:     # thousands of chunks per query: a subset keeps the suite inside its budget
        qs = [q for q in qs if q.name in ("P5", "chair", "P3", "K2")] + qs[-1:]
    for q in qs:
        want, lv = oracle.count(g, q, levels=True)
        _set(c, q)
        for kw in ({}, {"no_fast_count": True}):
            c.set_debug(**kw)
            for mode in ("hybrid", "bfs") if arena_kib > 64 else ("hybrid",):
                assert c.count(mode) == want, (q.name, kw, mode)
                assert c.stats()["level_size"] == lv, (q.name, kw, mode)
    c.set_debug()


def test_ancestor_reuse_enumerate(ctx):
    g = er_graph(40, 420, 7)
    ctx.load_csr(g)
    for q in [DENSE5[0]] + dense_family(6)[:4] + dense_family(7)[:2]:
        _check_full(ctx, g, q, modes=("hybrid",))


# ------------------------------------------------------------ 5-vertex family
@pytest.mark.parametrize("seed", [2, 3])
def test_5vertex_families_rmat9(ctx, seed):
    g = rmat_graph(9, 4, seed=seed)
    ctx.load_csr(g)
    for q in DENSE5 + SPARSE5:
        want, lv = oracle.count(g, q, levels=True)
        _set(ctx, q)
        for mode in ("bfs", "hybrid"):
            assert ctx.count(mode) == want, (q.name, mode)
            assert ctx.stats()["level_size"] == lv, (q.name, mode)


def test_5vertex_enumerate_er(ctx):
    g = er_graph(120, 900, 3)
    ctx.load_csr(g)
    for q in DENSE5 + SPARSE5:
        _check_full(ctx, g, q, modes=("hybrid",))


def test_dense_6_7_8_families(ctx):
    g = er_graph(26, 230, 5)
    ctx.load_csr(g)
    for k in (6, 7, 8):
        for q in dense_family(k):
            want, lv = oracle.count(g, q, levels=True)
            _set(ctx, q)
            assert ctx.count("hybrid") == want, q.name
            assert ctx.stats()["level_size"] == lv, q.name
            assert ctx.count("bfs") == want, q.name


def test_dense8_enumerate(ctx):
    g = complete_graph(10)
    ctx.load_csr(g)
    for q in dense_family(8)[::3]:
        _check_full(ctx, g, q, modes=("hybrid",))


# ------------------------------------------------------------------ structure
def test_closed_forms_on_gpu(ctx):
    g = grid_graph(4, 4)
    ctx.load_csr(g)
    _set(ctx, named_query("P4"))
    assert ctx.count("bfs") == 232
    assert ctx.stats()["level_size"][1:3] == [16, 48]       # Fig. 2
    g = cycle_graph(9)
    ctx.load_csr(g)
    for k in range(3, 9):
        _set(ctx, named_query(f"C{k}"))
        assert ctx.count("hybrid") == (18 if k == 9 else 0)
        _set(ctx, named_query(f"P{k}"))
        assert ctx.count("hybrid") == 18
    g = er_graph(500, 3000, 7)
    ctx.load_csr(g)
    d = g.degrees()
    for s in (1, 2, 3, 4):
        _set(ctx, named_query(f"S{s}"))
        want = sum(int(np.prod([int(x) - i for i in range(s)])) for x in d)
        assert ctx.count("hybrid") == want


def test_order_invariance_gpu(ctx):
    g = er_graph(80, 500, 4)
    ctx.load_csr(g)
    q = DENSE5[5]
    want = oracle.count(g, q)
    qr, qc = q.csr()
    import itertools
    qe = {(u, v) for u, v in q.edges} | {(v, u) for u, v in q.edges}
    valid = [list(p) for p in itertools.permutations(range(q.k))
             if all(any((p[i], p[j]) in qe for j in range(i)) for i in range(1, q.k))]
    assert len(valid) > 20
    for o in valid[::len(valid) // 6]:
        ctx.set_query(qr, qc, o)
        assert ctx.count("hybrid") == want
        _, lv = oracle.count(g, q, order=o, levels=True)
        assert ctx.stats()["level_size"] == lv


def test_root_range_and_slices(ctx):
    g = rmat_graph(9, 4, seed=5)
    ctx.load_csr(g)
    q = DENSE5[8]
    _set(ctx, q)
    total = ctx.count("hybrid")
    assert total == oracle.count(g, q)
    l1 = ctx.stats()["level1_canonical"]
    assert ctx.level1_size() == (l1, l1) == (oracle.level1_size(g, max(q.degrees())),) * 2
    cuts_ = [0, 7, 40, 41, l1 // 2, l1]
    for a, b in zip(cuts_, cuts_[1:]):
        ctx.set_root_range(a, b)
        assert ctx.level1_size() == (l1, b - a)
        assert ctx.count("hybrid") == oracle.count(g, q, root_begin=a, root_end=b)
    ctx.set_root_range()
    for nparts in (2, 3, 8):
        s = 0
        for p in range(nparts):
            ctx.set_root_slice(0, 2**64 - 1, p, nparts)
            s += ctx.count("hybrid")
        assert s == total
    # contiguous chunks of the shuffled list (the dynamic root-queue unit)
    s = 0
    for b in range(0, l1, 13):
        ctx.set_root_slice(b, b + 13, 0, 1)
        s += ctx.count("bfs")
    assert s == total


def test_edge_cases(ctx):
    from paper_conf_sc_xiangkshs21_b200 import CutsError
    # k = 1 and k = 2
    g = er_graph(50, 120, 1)
    ctx.load_csr(g)
    _set(ctx, named_query("K1"))
    assert ctx.count("bfs") == 50
    rows = ctx.enumerate("hybrid", cap_rows=50)
    assert sorted(rows.cpu().numpy().ravel().tolist()) == list(range(50))
    _set(ctx, named_query("P2"))
    assert ctx.count("hybrid") == 240
    # graph without edges, isolated vertices
    e = graph_from_edges(10, [])
    ctx.load_csr(e)
    _set(ctx, named_query("K3"))
    assert ctx.count("hybrid") == 0 and ctx.count("bfs") == 0
    _set(ctx, named_query("K1"))
    assert ctx.count("hybrid") == 10
    # query larger than any possible match
    ctx.load_csr(star_graph(5))
    _set(ctx, named_query("K3"))
    assert ctx.count("hybrid") == 0
    _set(ctx, named_query("S5"))
    assert ctx.count("hybrid") == 120
    # truncated enumeration reports the exact count
    g = complete_graph(6)
    ctx.load_csr(g)
    _set(ctx, named_query("K3"))
    rows = ctx.enumerate("bfs", cap_rows=10)
    assert ctx.truncated and rows.shape[0] == 10 and ctx.stats()["count"] == 120
    # k > 8 / bad order / bad graph
    with pytest.raises(CutsError) as ei:
        ctx.set_query_edges(9, [(i, i + 1) for i in range(8)])
    assert ei.value.status == -7
    with pytest.raises(CutsError) as ei:
        qr, qc = named_query("P4").csr()
        ctx.set_query(qr, qc, [0, 2, 1, 3])
    assert ei.value.status == -1
    from inputs import CSRGraph
    bad = CSRGraph(n=3, row_ptr=np.array([0, 1, 1, 1], np.uint64), col=np.array([1], np.uint32))
    with pytest.raises(CutsError):
        ctx.load_csr(bad, validate=True)
    bad = CSRGraph(n=3, row_ptr=np.array([0, 2, 3, 4], np.uint64), col=np.array([2, 1, 0, 0], np.uint32))
    with pytest.raises(CutsError):
        ctx.load_csr(bad, validate=True)


def test_state_errors(cuts):
    from paper_conf_sc_xiangkshs21_b200 import CutsError
    c = cuts(device=0, arena_bytes=1 << 20)
    with pytest.raises(CutsError) as ei:
        c.count("bfs")
    assert ei.value.status == -6


def test_fig3_trie_decode_gpu(ctx):
    """Fig. 3: GPU decode of the paper's (CA, PA) trie == oracle decode."""
    fx = json.load(open(os.path.join(GOLDEN, "fig3_trie.json")))
    got = ctx.trie_decode(fx["cuts_CA"], fx["cuts_PA"]).cpu().numpy()
    want = oracle.trie_decode(fx["cuts_CA"], fx["cuts_PA"])
    assert np.array_equal(got.view(np.uint32), want)


def test_alg_bytes_instrumentation(ctx):
    """Instrumented run: the §8.d byte model is counted and timing is recorded."""
    g = rmat_graph(9, 4, seed=2)
    ctx.load_csr(g)
    _set(ctx, DENSE5[0])
    ctx.set_debug(timing=True, bytes_=True)
    c = ctx.count("hybrid")
    st = ctx.stats()
    ctx.set_debug()
    assert c == oracle.count(g, DENSE5[0])
    assert st["alg_bytes_extend"] > 0 and st["alg_bytes_plan"] > 0
    assert st["ms_extend"] > 0 and st["extend_launches"] >= 1


@pytest.mark.parametrize("t", [2, 16, None])
def test_hub_bitmaps_parity(cuts, t):
    """SV-style hub rows (cuts_set_hub_threshold) never change a result."""
    c = cuts(device=0, arena_bytes=1 << 30)
    c.set_hub_threshold(t)
    g = rmat_graph(9, 4, seed=3)
    c.load_csr(g)
    for q in DENSE5[::2] + SPARSE5[::3] + [named_query("C4")]:
        want, lv = oracle.count(g, q, levels=True)
        _set(c, q)
        assert c.count("hybrid") == want, (t, q.name)
        st = c.stats()
        assert st["level_size"] == lv
        if t is not None:
            assert st["hubs"] == int((g.degrees() >= t).sum())
        else:
            assert st["hubs"] == 0
    g = er_graph(120, 900, 3)
    c.load_csr(g)
    for q in DENSE5[::3]:
        _check_full(c, g, q, modes=("hybrid",))


# --------------------------------------------- disconnected Q (NEXT-3)
DISCONNECTED = {
    "2K1": (2, []), "3K1": (3, []), "K2uK1": (3, [(0, 1)]), "2K2": (4, [(0, 1), (2, 3)]),
    "K3uK1": (4, [(0, 1), (1, 2), (0, 2)]), "P3uK2": (5, [(0, 1), (1, 2), (3, 4)]),
    "K4uK1": (5, [(0, 1), (0, 2), (0, 3), (1, 2), (1, 3), (2, 3)]),   # the P:1325-1327 tie member
    "K2uK1_mid": (3, [(0, 2)]), "K3uK2": (5, [(0, 3), (3, 4), (0, 4), (1, 2)]),
    "C4uK3": (7, [(0, 1), (1, 2), (2, 3), (0, 3), (4, 5), (5, 6), (4, 6)]),
    "K3u2K1": (5, [(0, 1), (1, 2), (0, 2)]),
}


@pytest.mark.parametrize("gname", ["er60", "petersen", "rmat8", "k7"])
def test_disconnected_queries(cuts, gname):
    """In-trie cross product (a component root extends from the degree-filtered
    vertex list, injectivity against the path) == the oracle's per-component
    cross product; counts in both modes, sorted rows, and a 64 KiB arena."""
    from inputs import petersen_graph
    g = {"er60": lambda: er_graph(60, 150, 3), "petersen": petersen_graph,
         "rmat8": lambda: rmat_graph(8, 4, seed=2), "k7": lambda: complete_graph(7)}[gname]()
    big = cuts(device=0, arena_bytes=1 << 28)
    small = cuts(device=0, arena_bytes=64 << 10)
    big.load_csr(g, validate=True)
    small.load_csr(g)
    for name, (k, es) in DISCONNECTED.items():
        q = query_from_edges(k, es, name)
        want = oracle.count(g, q)
        _set(big, q)
        _set(small, q)
        if want <= 1_000_000:     # BFS holds every level only for the small results
            assert big.count("bfs") == want, (gname, name)
        assert big.count("hybrid") == want, (gname, name)
        if want <= 5_000_000:     # the 64 KiB arena runs thousands of chunks per million embeddings
            assert small.count("hybrid") == want, (gname, name)
        if want <= 2_000_000:
            rows = big.enumerate("hybrid", cap_rows=want)
            assert np.array_equal(_sorted_rows(rows), oracle.enumerate_rows(g, q)), (gname, name)


def test_disconnected_levels_and_orders(ctx):
    """Per-level trie sizes against brute force for the order the library picks
    and for explicit orders (components in either sequence); an order that
    leaves a component before its root is matched is rejected."""
    from tests import bruteforce
    from paper_conf_sc_xiangkshs21_b200 import CutsError
    g = er_graph(9, 16, 4)
    ctx.load_csr(g)
    for name, order in (("2K2", None), ("2K2", [2, 3, 0, 1]), ("P3uK2", None), ("P3uK2", [3, 4, 1, 0, 2]),
                        ("K3uK1", [3, 0, 1, 2]), ("K3u2K1", None)):
        k, es = DISCONNECTED[name]
        q = query_from_edges(k, es, name)
        _set(ctx, q, order)
        got = ctx.count("bfs")
        st = ctx.stats()
        assert got == len(bruteforce.embeddings(g, q)) == oracle.count(g, q)
        assert st["level_size"] == bruteforce.level_sizes(g, q, st["order"]), (name, order)
        if order is not None:
            assert st["order"] == order
    with pytest.raises(CutsError) as ei:
        qr, qc = query_from_edges(5, DISCONNECTED["P3uK2"][1]).csr()
        ctx.set_query(qr, qc, [0, 3, 2, 4, 1])   # vertex 2 has no backward neighbour, 0 already placed
    assert ei.value.status == -1


@pytest.mark.parametrize("arena", [2 << 20, 1 << 30])
def test_disconnected_fullsize_closed_forms(cuts, arena):
    """At the C2 bench graph's full size (R-MAT(16,16,.45,.22,.22)), restricted to
    canonical root ranges: K3 ∪ K1 = count_range(K3) * (n - 3) (oracle-counted K3)
    and 2K2 = sum over root edges (u,v) of (2m - 2d(u) - 2d(v) + 2) (ordered edges
    disjoint from {u,v}).  The 2 MiB arena cannot hold the filtered free lists, so
    the component roots stream the identity list with the in-kernel degree filter."""
    g = rmat_graph(16, 16, 0.45, 0.22, 0.22, seed=1)
    c = cuts(device=0, arena_bytes=arena)
    c.load_csr(g)
    d = np.diff(g.row_ptr.astype(np.int64))
    m = int(d.sum()) // 2
    canon = np.nonzero(d >= 1)[0]
    k3 = named_query("K3")
    for a, b in ((0, 40), (len(canon) // 2, len(canon) // 2 + 25)):
        c.set_query_edges(4, [(0, 1), (1, 2), (0, 2)])
        c.set_root_range(a, b)
        got = c.count("hybrid")
        assert c.stats()["free_identity"] == (1 if arena < (1 << 24) else 0)
        assert got == oracle.count(g, k3, root_begin=a, root_end=b) * (g.n - 3)
        c.set_query_edges(4, [(0, 1), (2, 3)])
        c.set_root_range(a, b)
        want = 0
        for u in canon[a:b].tolist():
            for v in g.neighbors(u).tolist():
                want += 2 * m - 2 * int(d[u]) - 2 * int(d[v]) + 2
        assert c.count("hybrid") == want


def test_count_carry_and_overflow(ctx):
    """CUTS_DEBUG_PRELOAD_COUNT starts the 128-bit counter at 2^64 - 2^20: a count of
    2.19e6 must carry into the high word (add_u128) and cuts_count must return
    CUTS_EOVERFLOW with the full value in cuts_stats (P15)."""
    import ctypes
    g = complete_graph(40)
    ctx.load_csr(g)
    q = named_query("K4")
    want = 40 * 39 * 38 * 37
    _set(ctx, q)
    assert ctx.count("hybrid") == want
    ctx.set_debug(preload_count=True)
    try:
        for mode in (0, 1):
            out = ctypes.c_uint64()
            rc = ctx.lib.cuts_count(ctx.h, mode, ctypes.byref(out))
            assert rc == -4                                   # CUTS_EOVERFLOW
            st = ctx.stats()
            assert st["count"] == want + 2**64 - 2**20
            assert out.value == (want - 2**20) % 2**64
    finally:
        ctx.set_debug()
    assert ctx.count("bfs") == want


@pytest.mark.parametrize("flag", ["binned", "sv"])
def test_next2_binned_and_sv_variants(cuts, flag):
    """NEXT-2 ablations against the oracle: binned virtual warps at the last level
    (CUTS_DEBUG_BINNED) and the per-warp scatter-vector intersection
    (Alg. 2 l.7-17, CUTS_DEBUG_SV): counts and level sizes in both
    modes, at a roomy and at a chunk-forcing arena; rows for the binned variant."""
    g = rmat_graph(9, 6, a=0.55, b=0.2, c=0.2, seed=6)
    for arena in (64 << 20, 1 << 20):
        c = cuts(device=0, arena_bytes=arena)
        c.load_csr(g)
        qs = DENSE5[::2] + SPARSE5[::3] + dense_family(6)[::4] + [named_query("C4"), named_query("K3")]
        for q in (qs if arena > (1 << 20) else qs[::3]):
            want, lv = oracle.count(g, q, levels=True)
            _set(c, q)
            c.set_debug(**{flag: True})
            bfs_fits = arena > (1 << 20) and 8 * max(lv) < arena // 8
            for mode in ("hybrid", "bfs") if bfs_fits else ("hybrid",):
                assert c.count(mode) == want, (flag, arena, q.name, mode)
                assert c.stats()["level_size"] == lv, (flag, arena, q.name, mode)
            if flag == "binned" and want <= 1_000_000 and arena > (1 << 20):
                assert np.array_equal(_sorted_rows(c.enumerate("hybrid", cap_rows=want)), oracle.enumerate_rows(g, q))
            c.set_debug()
        c.close()


def test_local_rows_and_pairs_on_clique_unions(cuts):
    """The clique-tail paths (local 64-bit sibling rows, large-group fallback, pair-
    shared last level) on K70 ∪ K30 ∪ ER: sibling groups of 68 (> 64, fallback) and
    28 members (rows).  Every 5-vertex query Q has n!/(n-5)! embeddings in K_n, so
    count = 70!/65! + 30!/25! + count in the ER part (oracle); level sizes likewise.
    Default, CUTS_DEBUG_NO_LR and CUTS_DEBUG_NO_PAIRS must agree, at two arenas."""
    from math import perm
    er = er_graph(60, 200, 9)
    edges = [(u, v) for u in range(70) for v in range(u + 1, 70)]
    edges += [(70 + u, 70 + v) for u in range(30) for v in range(u + 1, 30)]
    edges += [(100 + int(a), 100 + int(b)) for a, b in er.edge_list()]
    g = graph_from_edges(160, edges)
    for arena in (2 << 30, 96 << 20):
        c = cuts(device=0, arena_bytes=arena)
        c.load_csr(g)
        for q in DENSE5[:3] + DENSE5[8:]:
            qe, qlv = oracle.count(er, q, levels=True)
            want = perm(70, 5) + perm(30, 5) + qe
            order = oracle.order(q)
            qd = q.degrees()
            lv = [0] + [sum(perm(n, j) for n in (70, 30) if all(n - 1 >= qd[order[i]] for i in range(j))) + qlv[j]
                        for j in range(1, 6)]
            _set(c, q)
            for flags in ({}, {"no_lr": True}, {"no_pairs": True}):
                c.set_debug(**flags)
                assert c.count("hybrid") == want, (arena, q.name, flags)
                assert c.stats()["level_size"] == lv, (arena, q.name, flags)
            c.set_debug()
        c.close()


def test_local_rows_group_size_tiers(cuts):
    """Sibling groups of every local-rows tier: two adjacent hubs over a circulant
    C_600(1, 2) give the hub pair a group of 600 leaves (> 512: windowed fallback),
    single hubs give mid-size groups (CTA-per-group shared-memory rows) and the
    leaves small ones (64-bit rows).  Counts and level sizes == oracle, with and
    without local rows."""
    n = 600
    edges = [(0, 1)] + [(h, 2 + i) for h in (0, 1) for i in range(n)]
    edges += [(2 + i, 2 + (i + d) % n) for i in range(n) for d in (1, 2)]
    edges += [(2 + n + i, 2 + (7 * i) % n) for i in range(100)]          # pendant vertices
    g = graph_from_edges(2 + n + 100, edges)
    c = cuts(device=0, arena_bytes=1 << 30)
    c.load_csr(g)
    cheap = ("K5", "K5-K2", "K5-P3", "K5-2K2", "K5-P4", "K5-K13", "K5-P3uK2", "K6", "K6-K2", "K6-P3")
    for q in [q for q in DENSE5 + dense_family(6)[:3] if q.name in cheap]:   # oracle <= 2e7 embeddings each
        want, lv = oracle.count(g, q, levels=True)
        _set(c, q)
        for flags in ({}, {"no_lr": True}):
            c.set_debug(**flags)
            assert c.count("hybrid") == want, (q.name, flags)
            assert c.stats()["level_size"] == lv, (q.name, flags)
        c.set_debug()
    c.close()


def test_deep_local_rows_clique_tiers(cuts):
    """Deep local rows (rows of the level-(k-3) sibling groups carry levels k-2, k-1 and
    the count) on clique unions whose level-(k-3) groups span every row width:
    K6 on K200 ∪ K150 ∪ K70 ∪ K9 (groups of 198 / 148 / 68 / 7 members: 4-, 3-, 2- and
    1-word rows),
    K7 on K70 ∪ K12, K8 on K40 ∪ K11, each plus an ER component (oracle).  In K_n the
    level sizes are n!/(n-j)!.  Default, CUTS_DEBUG_NO_DLR and CUTS_DEBUG_NO_LR agree at
    a large arena and at a 96 MiB one (level k-2 cut into many entry-aligned chunks);
    CUTS_DEBUG_TAIL_ALT (lane per triangle) likewise;
    CUTS_DEBUG_NO_LR only where the windowed pipeline's pair count stays small."""
    from math import perm
    er = er_graph(60, 260, 11)
    cases = ((6, (200, 150, 70, 9)), (7, (70, 12)), (8, (40, 11)))
    for k, sizes in cases:
        edges, base = [], 0
        for n in sizes:
            edges += [(base + u, base + v) for u in range(n) for v in range(u + 1, n)]
            base += n
        edges += [(base + int(a), base + int(b)) for a, b in er.edge_list()]
        g = graph_from_edges(base + er.n, edges)
        q = dense_family(k)[0]
        qe, qlv = oracle.count(er, q, levels=True)
        want = sum(perm(n, k) for n in sizes) + qe
        lv = [0] + [sum(perm(n, j) for n in sizes) + qlv[j] for j in range(1, k + 1)]
        for arena in (8 << 30, 96 << 20):
            c = cuts(device=0, arena_bytes=arena)
            c.load_csr(g)
            _set(c, q)
            # the windowed pipeline (no local rows at all) only where its pair count is small
            slow = perm(max(sizes), k - 1) > 2e9
            # the tail variants (ablations) at the large arena only: the small one re-tests chunking
            variants = ({"no_cta_tail": True}, {"tail_alt": True}, {"tail_split": True}) if arena > (1 << 30) else ()
            for flags in ({}, {"no_dlr": True}) + variants + (() if slow else ({"no_lr": True},)):
                c.set_debug(**flags)
                assert c.count("hybrid") == want, (k, arena, flags)
                st = c.stats()
                assert st["level_size"] == lv, (k, arena, flags)
                if not flags and arena > (1 << 30):
                    assert (st["fused_levels"] >> (k - 1)) & 1, "deep local rows did not run"
            c.set_debug()
            c.close()


def test_deep_local_rows_large_group_fallback(cuts):
    """A level-(k-3) group above the deep-rows limit (1,024 members) goes through the
    windowed pipeline while the rest use rows: two adjacent hubs over a circulant
    C_1100(1, 2, 3) give the hub pair a 1,100-member group at level 3 of K6 / K6-K2.
    Counts and level sizes == oracle, default and CUTS_DEBUG_NO_DLR."""
    n = 1100
    edges = [(0, 1)] + [(h, 2 + i) for h in (0, 1) for i in range(n)]
    edges += [(2 + i, 2 + (i + d) % n) for i in range(n) for d in (1, 2, 3)]
    g = graph_from_edges(2 + n, edges)
    c = cuts(device=0, arena_bytes=1 << 30)
    c.load_csr(g)
    for q in dense_family(6)[:2]:
        want, lv = oracle.count(g, q, levels=True)
        _set(c, q)
        for flags in ({}, {"no_dlr": True}):
            c.set_debug(**flags)
            assert c.count("hybrid") == want, (q.name, flags)
            assert c.stats()["level_size"] == lv, (q.name, flags)
        c.set_debug()
    c.close()
