"""BASELINE configs[3] acceptance run: K8 on R-MAT(22,16,.50,.20,.20), stated root range.

    python tools/c4_run.py [--den 16] [--skip-bfs] [--out gpurun_out/c4_run.json]

1. BFS mode must fail with CUTS_ENOMEM (a level does not fit the arena);
2. HYBRID mode must finish, and the chunk-summed size of its deepest stored
   level times 8 B (one (vertex, parent) trie entry) must exceed the arena —
   i.e. the trie the level-synchronous method would hold is larger than HBM
   and only the DFS-over-chunks schedule makes the query feasible.
Prints and writes one JSON record with level sizes, chunks, peak arena, times.
"""
import argparse
import json
import os
import sys
import time

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import torch  # noqa: E402

from workloads import C4  # noqa: E402
from paper_conf_sc_xiangkshs21_b200 import Cuts, CutsError  # noqa: E402


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--den", type=int, default=0, help="override the root range to [0, 1/den)")
    ap.add_argument("--skip-bfs", action="store_true")
    ap.add_argument("--out", default="")
    args = ap.parse_args()
    spec, (q,) = C4.parts[0]
    t = time.time()
    g = spec.build()
    gen_s = time.time() - t
    ctx = Cuts(device=0)
    rp = torch.from_numpy(g.row_ptr.view("int64")).cuda()
    cl = torch.from_numpy(g.col.view("int32")).cuda()
    ctx.load_graph(rp, cl, validate=True)
    qr, qc = q.csr()
    ctx.set_query(qr, qc)
    l1, _ = ctx.level1_size()
    b, e = C4.roots(l1) if not args.den else (0, l1 // args.den)
    rec = {"graph": spec.name, "n": g.n, "m": g.m, "gen_s": round(gen_s, 1), "query": q.name,
           "level1_canonical": l1, "root_range": [b, e], "arena_bytes": ctx.arena.numel()}
    if not args.skip_bfs:
        ctx.set_query(qr, qc)
        ctx.set_root_range(b, e)
        torch.cuda.synchronize()
        t = time.time()
        try:
            c = ctx.count("bfs")
            rec["bfs"] = {"status": "CUTS_OK", "count": c}
        except CutsError as err:
            rec["bfs"] = {"status": err.status, "message": str(err)}
        rec["bfs"]["s"] = round(time.time() - t, 2)
        rec["bfs"]["level_size"] = ctx.stats()["level_size"]
        print(json.dumps(rec["bfs"]), flush=True)
    ctx.set_query(qr, qc)
    ctx.set_root_range(b, e)
    ctx.set_debug(timing=True)
    torch.cuda.synchronize()
    t = time.time()
    c = ctx.count("hybrid")
    dt = time.time() - t
    st = ctx.stats()
    deepest = max(st["level_size"][1:q.k])
    rec["hybrid"] = {"count": c, "s": round(dt, 2), "emb_per_s": c / dt, "level_size": st["level_size"],
                     "chunks": st["chunks"], "windows": st["windows"], "launches": st["launches"],
                     "peak_arena_bytes": st["peak_arena_bytes"], "items": st["items"],
                     "ms_extend": st["ms_extend"], "ms_plan": st["ms_plan"],
                     "deepest_stored_level_entries": deepest,
                     "bfs_trie_bytes_at_deepest_level": 8 * deepest,
                     "exceeds_arena": 8 * deepest > ctx.arena.numel(),
                     "exceeds_180GB": 8 * deepest > 180e9}
    print(json.dumps(rec), flush=True)
    if args.out:
        with open(args.out, "w") as f:
            json.dump(rec, f, indent=1)


if __name__ == "__main__":
    main()
