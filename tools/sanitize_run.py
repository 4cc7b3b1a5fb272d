"""Small workload for compute-sanitizer (memcheck / racecheck / synccheck) over every kernel family.

    compute-sanitizer --tool memcheck python tools/sanitize_run.py

Covers: load + validate, level 1, k_plan / scan / k_extend (BFS and HYBRID on a 1 MiB arena, so
chunking runs), ordered levels (ancestor source), k_pairs, k_lr_rows (groups <= 64), k_lr_group
(groups of 65..512), enumerate (kEnum decode), the set-difference count, and the directed path.
Counts are checked against closed forms or the oracle (tests/ infrastructure, small cases only).
"""
from __future__ import annotations

import os
import sys
from math import perm

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))

import numpy as np  # noqa: E402
import torch  # noqa: E402

import oracle  # noqa: E402
from inputs import er_graph, rmat_graph, complete_graph, named_query, DENSE5, dense_family  # noqa: E402
from paper_conf_sc_xiangkshs21_b200 import Cuts  # noqa: E402


def main():
    ctx = Cuts(device=0, arena_bytes=64 << 20)
    small = Cuts(device=0, arena_bytes=1 << 20)
    cases = [
        (er_graph(300, 1500, seed=3), [named_query("K3"), named_query("C4"), DENSE5[9]]),
        (rmat_graph(9, 8, 0.50, 0.20, 0.20, seed=2), [DENSE5[0], DENSE5[3], dense_family(6)[0]]),
    ]
    for g, qs in cases:
        for c in (ctx, small):
            c.load_csr(g, validate=True)
        for q in qs:
            qr, qc = q.csr()
            want = oracle.count(g, q)
            for c in (ctx, small):
                c.set_query(qr, qc)
                for mode in ("bfs", "hybrid") if c is ctx else ("hybrid",):
                    got = c.count(mode)
                    assert got == want, (g.name, q.name, mode, got, want)
            if want <= 200000:
                rows = ctx.enumerate("hybrid", cap_rows=want).cpu().numpy().view(np.uint32)
                rows = rows[np.lexsort(rows.T[::-1])]
                assert np.array_equal(rows, oracle.enumerate_rows(g, q)), q.name
            print("ok", g.name, q.name, want, flush=True)
    # clique tails: K5 in K40 (groups of 37: k_lr_rows), K4 in K90 (groups of 88: k_lr_group)
    for n, k in ((40, 5), (90, 4), (12, 6)):
        g = complete_graph(n)
        q = dense_family(k)[0] if k >= 6 else (named_query("K3") if k == 3 else None)
        if q is None:
            from inputs import k_minus
            q = k_minus(k, [], name=f"K{k}")
        qr, qc = q.csr()
        for c in (ctx, small):
            c.load_csr(g, validate=True)
            c.set_query(qr, qc)
            for flags in ({}, {"no_lr": True}, {"no_pairs": True, "no_lr": True}):
                c.set_debug(**flags)
                got = c.count("hybrid")
                want = perm(n, k) if q.name.startswith("K") and len(q.name) <= 2 else oracle.count(g, q)
                assert got == want, (n, k, flags, got, want)
            c.set_debug()
        print("ok clique", n, k, flush=True)
    torch.cuda.synchronize()
    print("sanitize workload ok")


if __name__ == "__main__":
    main()
