"""Row e through the C ABI: cuts_set_dist / cuts_allreduce_count (the library's
own NCCL communicator, "sum of the counts") and the default
per-rank cyclic root partition, against the oracle."""
import os
import socket

import pytest

import oracle
from inputs import rmat_graph, named_query, DENSE5

pytestmark = pytest.mark.gpu


@pytest.fixture(scope="module")
def cuts():
    torch = pytest.importorskip("torch")
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    from paper_conf_sc_xiangkshs21_b200 import Cuts
    return Cuts


def test_world1_nccl_communicator(cuts):
    """world 1 with a real NCCL communicator: the count, the all-reduced count
    and a > 2^64 value survive the limb reduction exactly."""
    g = rmat_graph(9, 4, seed=2)
    c = cuts(device=0, arena_bytes=64 << 20)
    c.load_csr(g)
    c.set_dist(0, 1, cuts.dist_unique_id())
    for q in (DENSE5[8], named_query("C4")):
        qr, qc = q.csr()
        c.set_query(qr, qc)
        n = c.count("hybrid")
        assert n == oracle.count(g, q)
        assert c.allreduce_count(n) == n
    big = (1 << 100) + (1 << 64) + 12345
    assert c.allreduce_count(big) == big
    from paper_conf_sc_xiangkshs21_b200 import CutsError
    with pytest.raises(CutsError):
        c.set_dist(1, 1, None)          # rank out of range
    c.close()


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _worker(rank, world, port, results):
    import faulthandler
    import torch
    import torch.distributed as dist
    faulthandler.dump_traceback_later(200, exit=True)
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        from paper_conf_sc_xiangkshs21_b200 import Cuts, CutsError
        uid = [Cuts.dist_unique_id() if rank == 0 else None]
        dist.broadcast_object_list(uid, src=0)
        g = rmat_graph(9, 4, seed=2)
        c = Cuts(device=0, arena_bytes=64 << 20)
        c.load_csr(g)
        try:
            c.set_dist(rank, world, uid[0])
        except CutsError as e:
            results[rank] = ("skip", str(e))
            return
        out = {}
        for q in (DENSE5[8], named_query("C4"), named_query("K3")):
            qr, qc = q.csr()
            c.set_query(qr, qc)            # default root slice: p % world == rank
            local = c.count("hybrid")
            out[q.name] = (local, c.allreduce_count(local))
        results[rank] = ("ok", out)
        torch.cuda.synchronize()
    finally:
        dist.destroy_process_group()


def test_world2_through_the_abi_one_gpu(cuts):
    """Two ranks on cuda:0: cuts_set_dist, per-rank default slices, the library's
    NCCL all-reduce.  NCCL refuses two ranks on one device on some versions; the
    test then skips (an 8-GPU box runs the same calls in bench.py)."""
    import torch.multiprocessing as mp
    mgr = mp.Manager()
    results = mgr.dict()
    mp.start_processes(_worker, args=(2, _free_port(), results), nprocs=2, join=True, start_method="spawn")
    if any(results[r][0] == "skip" for r in range(2)):
        pytest.skip("NCCL: " + "; ".join(str(results[r][1]) for r in range(2) if results[r][0] == "skip"))
    g = rmat_graph(9, 4, seed=2)
    for q in (DENSE5[8], named_query("C4"), named_query("K3")):
        want = oracle.count(g, q)
        locals_ = [results[r][1][q.name][0] for r in range(2)]
        assert sum(locals_) == want
        assert all(results[r][1][q.name][1] == want for r in range(2))


@pytest.mark.gpu
@pytest.mark.parametrize("depth", [1, 2, 3])
def test_partition_depth_parts_sum_to_oracle(depth):
    """cuts_set_partition_depth: the cyclic parts (and chunked slices) of the shuffled
    level-D list sum to the oracle count, and their level sizes to the oracle's, in
    HYBRID and BFS, on the DLR (K6), local-rows (K5) and windowed (K5-P3, C4) paths."""
    import oracle
    from inputs import rmat_graph, named_query, DENSE5, dense_family
    from paper_conf_sc_xiangkshs21_b200 import Cuts
    g = rmat_graph(9, 8, 0.50, 0.20, 0.20, seed=3)
    c = Cuts(device=0, arena_bytes=512 << 20)
    c.load_csr(g)
    for q in (dense_family(6)[0], DENSE5[0], DENSE5[2], named_query("C4")):
        want, lv = oracle.count(g, q, levels=True)
        qr, qc = q.csr()
        c.set_query(qr, qc)
        c.set_partition_depth(depth)
        L = c.partition_size()
        assert L == lv[min(depth, q.k - 1) if depth < q.k else 1]
        for nparts in (1, 3):
            for mode in ("hybrid", "bfs"):
                tot, lvs = 0, [0] * (q.k + 1)
                for part in range(nparts):
                    c.set_root_slice(0, 2**64 - 1, part, nparts)
                    tot += c.count(mode)
                    for j, v in enumerate(c.stats()["level_size"]):
                        lvs[j] += v
                assert tot == want, (q.name, depth, nparts, mode)
                assert lvs == lv, (q.name, depth, nparts, mode)
        tot = 0                                      # chunks of the shuffled list (the dynamic queue's unit)
        for b in range(0, L, max(1, L // 4)):
            c.set_root_slice(b, b + max(1, L // 4), 0, 1)
            tot += c.count("hybrid")
        assert tot == want, (q.name, depth, "chunks")
        c.set_root_slice(0, 2**64 - 1, 0, 1)
    c.set_partition_depth(1)
    c.close()
