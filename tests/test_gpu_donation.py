"""GPU parity of the dynamic-redistribution pieces (row e, Alg. 3):
flat-prefix seeding (cuts_set_prefixes), donation export (cuts_set_donation) and
the two-rank work-sharing protocol, all against the CPU oracle's total count."""
import os
import socket

import numpy as np
import pytest

import oracle
from inputs import er_graph, rmat_graph, named_query, DENSE5, SPARSE5

pytestmark = pytest.mark.gpu


@pytest.fixture(scope="module")
def cuts():
    torch = pytest.importorskip("torch")
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    from paper_conf_sc_xiangkshs21_b200 import Cuts
    return Cuts


def _set(ctx, q):
    qr, qc = q.csr()
    ctx.set_query(qr, qc)


def _adj(g):
    return [set(g.neighbors(v).tolist()) for v in range(g.n)]


def _check_prefix_rows(g, adj, q, order, rows):
    """Every shipped row is a partial embedding of Q[S[0..d-1]] passing the degree filter."""
    qd = q.degrees()
    qe = {(a, b) for a, b in q.edges} | {(b, a) for a, b in q.edges}
    deg = g.degrees()
    d = rows.shape[1]
    for row in rows.tolist():
        assert len(set(row)) == d
        for i in range(d):
            assert deg[row[i]] >= qd[order[i]]
            for j in range(i):
                if (order[i], order[j]) in qe:
                    assert row[j] in adj[row[i]]


def test_prefix_seeding_level1_and_level2(cuts):
    """Hand-built level-1 and level-2 prefix sets reproduce the full count."""
    import torch
    ctx = cuts(device=0, arena_bytes=256 << 20)
    g = rmat_graph(9, 4, seed=5)
    ctx.load_csr(g)
    deg = g.degrees()
    el = g.edge_list()
    for q in (DENSE5[8], named_query("C4"), SPARSE5[1], named_query("K3")):
        want = oracle.count(g, q)
        _set(ctx, q)
        order = ctx.stats()["order"] if ctx.count("hybrid") >= 0 else None
        qd = q.degrees()
        l1 = np.nonzero(deg >= qd[order[0]])[0].astype(np.int32).reshape(-1, 1)
        pairs = np.concatenate([el, el[:, ::-1]])
        keep = (deg[pairs[:, 0]] >= qd[order[0]]) & (deg[pairs[:, 1]] >= qd[order[1]])
        l2 = pairs[keep].astype(np.int32)
        for rows in (l1, l2):
            t = torch.from_numpy(np.ascontiguousarray(rows)).to("cuda:0")
            for mode in ("hybrid", "bfs"):
                ctx.set_prefixes(t)
                assert ctx.count(mode) == want, (q.name, rows.shape, mode)
                st = ctx.stats()
                assert st["level_size"][rows.shape[1]] == rows.shape[0]
        ctx.set_prefixes(None)
        assert ctx.count("hybrid") == want
    # depth must be < k; empty prefix sets count 0
    from paper_conf_sc_xiangkshs21_b200 import CutsError
    _set(ctx, named_query("K3"))
    with pytest.raises(CutsError):
        ctx.set_prefixes(torch.zeros((4, 3), dtype=torch.int32, device="cuda:0"))
    ctx.set_prefixes(torch.zeros((0, 2), dtype=torch.int32, device="cuda:0"))
    assert ctx.count("hybrid") == 0


@pytest.mark.parametrize("arena_kib,root_end", [(256, None), (192, 1), (1024, 3)])
def test_donation_simulated_alg3(cuts, arena_kib, root_end):
    """Donate half of the shallowest unfinished level at every chunk boundary,
    process every shipped piece (donating again), and sum: == oracle."""
    g = rmat_graph(10, 8, 0.5, 0.2, 0.2, seed=3)
    adj = _adj(g)
    ctx = cuts(device=0, arena_bytes=arena_kib << 10)
    ctx.load_csr(g)
    for q in (DENSE5[6], named_query("C4"), named_query("P4")):
        _set(ctx, q)
        if root_end is not None:
            # the hub roots: the canonical list is ascending id, pick the max-degree root's position
            ctx.set_root_range(0, 2**64 - 1)
        want_full = oracle.count(g, q)
        ctx.count("hybrid")
        order = ctx.stats()["order"]
        l1 = np.nonzero(g.degrees() >= q.degrees()[order[0]])[0]
        if root_end is not None:
            hub = int(np.argmax(g.degrees()[l1]))
            rb, re_ = hub, min(len(l1), hub + root_end)
            want = oracle.count(g, q, root_begin=rb, root_end=re_)
        else:
            rb, re_, want = 0, 2**64 - 1, want_full
        work, shipped, depths = [], [0], set()

        def poll(depth, remaining):
            return remaining // 2 if shipped[0] < 60 else 0

        def ship(depth, rows):
            shipped[0] += 1
            depths.add(depth)
            _check_prefix_rows(g, adj, q, order, rows.cpu())
            work.append(rows)

        ctx.set_donation(poll, ship)
        try:
            ctx.set_prefixes(None)
            ctx.set_root_range(rb, re_)
            total = ctx.count("hybrid")
            st = ctx.stats()
            assert st["donations"] >= 1 or want == 0
            while work:
                ctx.set_prefixes(work.pop())
                total += ctx.count("hybrid")
        finally:
            ctx.set_donation(None, None)
            ctx.set_prefixes(None)
            ctx.set_root_range()
        assert total == want, (q.name, arena_kib, root_end, total, want, shipped[0], depths)
        if root_end == 1 and want:
            assert max(depths) >= 2      # a single root: donations come from deeper levels


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _ws_gpu_worker(rank, world, port, results):
    import faulthandler
    import torch
    import torch.distributed as dist
    faulthandler.dump_traceback_later(240, exit=True)
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        from paper_conf_sc_xiangkshs21_b200 import Cuts, dist as D
        g = rmat_graph(10, 8, 0.5, 0.2, 0.2, seed=2)
        ctx = Cuts(device=0, arena_bytes=8 << 20)      # small arena: many chunk boundaries
        ctx.load_csr(g)
        out = {}
        store = D.default_store()
        for qi, q in enumerate((DENSE5[6], named_query("C4"), named_query("P4"))):
            qr, qc = q.csr()
            ctx.set_query(qr, qc)
            _, l1 = ctx.level1_size()
            cs = max(1, -(-l1 // (world * 4)))
            queue = D.RootQueue(store, f"q{qi}", D.n_chunks(l1, cs))
            eng = D.CutsEngine(ctx)
            ws = D.WorkSharing(store, f"ws{qi}", rank, world, eng, interval=0.0)
            local = ws.run(queue, cs)
            out[q.name] = (D.allreduce_count(local), ws.sent, ws.received)
        results[rank] = out
        torch.cuda.synchronize()
    finally:
        dist.destroy_process_group()


def test_work_sharing_two_ranks_one_gpu(cuts):
    """The multi-GPU protocol end to end (root queue + donations + reduction),
    two ranks sharing cuda:0 over gloo: every count == oracle."""
    import torch.multiprocessing as mp
    port = _free_port()
    mgr = mp.Manager()
    results = mgr.dict()
    mp.start_processes(_ws_gpu_worker, args=(2, port, results), nprocs=2, join=True, start_method="spawn")
    g = rmat_graph(10, 8, 0.5, 0.2, 0.2, seed=2)
    sent = 0
    for q in (DENSE5[6], named_query("C4"), named_query("P4")):
        want = oracle.count(g, q)
        for r in range(2):
            assert results[r][q.name][0] == want, (q.name, results[r][q.name], want)
        sent += sum(results[r][q.name][1] for r in range(2))
        assert sum(results[r][q.name][1] for r in range(2)) == sum(results[r][q.name][2] for r in range(2))
    assert sent >= 1
