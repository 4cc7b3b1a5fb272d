"""C4 calibration: K8 on R-MAT(22,16,.50,.20,.20), HYBRID count over several
canonical root ranges [a/den, b/den) — time, level sizes, chunks — to pick the
bench's stated root sub-range (one step ~10-20 s with a chunk-summed stored
level > 2.25e10 entries, i.e. a BFS trie > 180 GB).

    python tools/c4_sweep.py --ranges 0:1:8192 0:1:4096 0:1:2048 1:2:2048 --out gpurun_out/c4_sweep.jsonl
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
from paper_conf_sc_xiangkshs21_b200 import Cuts  # noqa: E402


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--ranges", nargs="+", default=["0:1:4096", "0:1:2048", "0:1:1024"])
    ap.add_argument("--query", type=int, default=0, help="index into dense_family(8)")
    ap.add_argument("--debug", default="", help="comma list of set_debug flags (ablations)")
    ap.add_argument("--reps", type=int, default=1)
    ap.add_argument("--out", default="")
    args = ap.parse_args()
    from inputs import dense_family
    spec, _ = C4.parts[0]
    q = dense_family(8)[args.query]
    t = time.time()
    g = spec.build()
    gen_s = time.time() - t
    ctx = Cuts(device=0)
    rp = torch.from_numpy(g.row_ptr.view("int64")).cuda()
    cl = torch.from_numpy(g.col.view("int32")).cuda()
    ctx.load_graph(rp, cl)
    qr, qc = q.csr()
    ctx.set_query(qr, qc)
    l1, _ = ctx.level1_size()
    out = open(args.out, "a") if args.out else None
    flags = {f: True for f in args.debug.split(",") if f}
    for r in args.ranges:
        if r.startswith("pos:"):                 # absolute canonical positions pos:a:b
            rb, re = (int(x) for x in r.split(":")[1:])
        else:
            a, b, den = (int(x) for x in r.split(":"))
            rb, re = a * l1 // den, b * l1 // den
        for rep in range(args.reps):
            ctx.set_query(qr, qc)
            ctx.set_root_range(rb, re)
            ctx.set_debug(timing=True, **flags)
            torch.cuda.synchronize()
            t = time.time()
            c = ctx.count("hybrid")
            dt = time.time() - t
            st = ctx.stats()
            stored = [j for j in range(1, q.k) if not (st["fused_levels"] >> j) & 1]
            deepest = max(st["level_size"][j] for j in stored)
            rec = {"graph": spec.name, "gen_s": round(gen_s, 1), "query": q.name, "range": r, "roots": [rb, re],
                   "level1_canonical": l1, "count": c, "s": round(dt, 3), "emb_per_s": c / dt,
                   "level_size": st["level_size"], "deepest_stored": deepest, "stored_levels": stored, "exceeds_180GB": 8 * deepest > 180e9,
                   "chunks": st["chunks"], "windows": st["windows"], "launches": st["launches"],
                   "ms_extend": round(st["ms_extend"], 1), "ms_plan": round(st["ms_plan"], 1),
                   "peak_arena_bytes": st["peak_arena_bytes"], "debug": args.debug, "rep": rep}
            if flags.get("groups"):
                rec["group_hist"] = {j: v for j, v in ctx.group_hist().items()}
            print(json.dumps(rec), flush=True)
            if out:
                out.write(json.dumps(rec) + "\n")
                out.flush()


if __name__ == "__main__":
    main()
