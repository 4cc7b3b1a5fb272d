"""Multi-process host logic of the multi-GPU path on CPU (gloo, world_size 2).

The GPU leg is exercised by bench.py under torchrun; here the partition, the
dynamic root-chunk queue and the exact count reduction are checked with the
oracle standing in for the per-chunk count (the oracle only supports canonical
root ranges, which is all the queue hands out here).
"""
import os
import socket

import pytest
import torch.multiprocessing as mp

WORLD = 2


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _worker(rank, world, port, results):
    import torch.distributed as dist
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        from paper_conf_sc_xiangkshs21_b200 import dist as D
        import oracle
        from inputs import er_graph, DENSE5, named_query
        out = {}
        # 1. exact 128-bit reduction
        big = (1 << 100) + 12345 * (rank + 1) + (1 << 63)
        out["sum"] = D.allreduce_count(big)
        # 2. dynamic queue: disjoint cover of all chunks
        store = D.default_store()
        q = D.RootQueue(store, "t_queue", 37)
        got = []
        while (c := q.next()) is not None:
            got.append(c)
        out["chunks"] = got
        # 3. dynamic root chunks + reduction == total (oracle as the per-chunk counter)
        g = er_graph(300, 2400, 3)
        for query in (DENSE5[8], named_query("C4")):
            l1 = oracle.level1_size(g, max(query.degrees()))
            cs = 9
            rq = D.RootQueue(store, f"t_{query.name}", D.n_chunks(l1, cs))
            local = 0
            while (c := rq.next()) is not None:
                b, e = D.chunk_bounds(c, cs)
                local += oracle.count(g, query, root_begin=b, root_end=e)
            out[query.name] = D.allreduce_count(local)
        # 4. static cyclic slices cover the level exactly once
        out["slice"] = D.static_slice(rank, world)
        results[rank] = out
    finally:
        dist.destroy_process_group()


def test_gloo_world2_queue_and_reduction():
    port = _free_port()
    mgr = mp.Manager()
    results = mgr.dict()
    mp.start_processes(_worker, args=(WORLD, port, results), nprocs=WORLD, join=True, start_method="spawn")
    import oracle
    from inputs import er_graph, DENSE5, named_query
    r0, r1 = results[0], results[1]
    want = sum((1 << 100) + 12345 * (r + 1) + (1 << 63) for r in range(WORLD))
    assert r0["sum"] == r1["sum"] == want
    allc = sorted(r0["chunks"] + r1["chunks"])
    assert allc == list(range(37))
    g = er_graph(300, 2400, 3)
    for query in (DENSE5[8], named_query("C4")):
        assert r0[query.name] == r1[query.name] == oracle.count(g, query)
    assert r0["slice"] == (0, 2**64 - 1, 0, 2) and r1["slice"] == (0, 2**64 - 1, 1, 2)


def test_single_process_helpers():
    from paper_conf_sc_xiangkshs21_b200 import dist as D
    assert D.allreduce_count(5) == 5
    assert D.n_chunks(10, 3) == 4 and D.chunk_bounds(3, 3) == (9, 12)
    with pytest.raises(ValueError):
        D.allreduce_count(-1)
    with pytest.raises(ValueError):
        D.static_slice(2, 2)


def _ws_worker(rank, world, port, results):
    import faulthandler
    import torch.distributed as dist
    faulthandler.dump_traceback_later(45, exit=True)
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        from paper_conf_sc_xiangkshs21_b200 import dist as D
        from tests.mock_engine import MockEngine
        eng = MockEngine()
        store = D.default_store()
        cs = 4
        q = D.RootQueue(store, "ws_q", D.n_chunks(eng.roots, cs))
        ws = D.WorkSharing(store, "ws", rank, world, eng, interval=0.0005)
        local = ws.run(q, cs)
        results[rank] = {"local": local, "total": D.allreduce_count(local), "sent": ws.sent,
                         "recv": ws.received, "serial": eng.serial_total()}
    finally:
        dist.destroy_process_group()


@pytest.mark.parametrize("world", [2, 3])
def test_gloo_work_sharing_donations(world):
    """Alg. 3 protocol: root queue + donation of flat prefixes of the
    shallowest unfinished level to idle ranks; every leaf counted exactly once,
    termination detected, and the hub root's work actually redistributed."""
    port = _free_port()
    mgr = mp.Manager()
    results = mgr.dict()
    mp.start_processes(_ws_worker, args=(world, port, results), nprocs=world, join=True, start_method="spawn")
    res = [results[r] for r in range(world)]
    serial = res[0]["serial"]
    assert serial > 0
    assert all(r["total"] == serial for r in res)
    assert sum(r["local"] for r in res) == serial
    assert sum(r["sent"] for r in res) >= 1
    assert sum(r["sent"] for r in res) == sum(r["recv"] for r in res)


def test_workload_root_ranges():
    """The stated root range of C4 (absolute canonical positions [13500, 14400),
    clamped to the list) and the full range of the other configs."""
    from workloads import WORKLOADS, Workload
    assert WORKLOADS["C4"].roots(1834382) == (13500, 14400)
    assert WORKLOADS["C4"].roots(13600) == (13500, 13600)
    assert WORKLOADS["C4"].min_trie_bytes == 180e9
    assert Workload("x", "", (), root_range=(0, 1, 16)).roots(1600) == (0, 100)
    for name in ("C1", "C2", "C3"):
        assert WORKLOADS[name].roots(1234) == (0, 1234)
    assert len(WORKLOADS["C3"].parts[0][1]) == 33
    assert WORKLOADS["C4"].parts[0][1][0].name == "K8"
