"""Calibrate synthetic workloads (BASELINE configs[1..4]) on the GPU.

For each R-MAT parameter set and query, count embeddings over a random 1/S
sample of the shuffled level-1 roots (an unbiased estimate of the full count
and of the work), extrapolate, and — when the estimate fits the time budget —
run the full query.  Prints one JSON line per (graph, query).

    python tools/calibrate.py --scale 16 --ef 16 --abc 0.57,0.19,0.19 --family c2
"""
import argparse
import json
import os
import sys
import time

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import torch  # noqa: E402

from inputs import rmat_graph_torch, DENSE5, SPARSE5, dense_family  # noqa: E402
from paper_conf_sc_xiangkshs21_b200 import Cuts  # noqa: E402


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--scale", type=int, default=16)
    ap.add_argument("--ef", type=int, default=16)
    ap.add_argument("--abc", action="append", default=[])
    ap.add_argument("--family", default="c2")
    ap.add_argument("--sample", type=int, default=64)
    ap.add_argument("--budget", type=float, default=20.0, help="seconds allowed for a full run")
    ap.add_argument("--seed", type=int, default=1)
    ap.add_argument("--out", default="")
    ap.add_argument("--min-nparts", type=int, default=1)
    ap.add_argument("--max-nparts", type=int, default=4096)
    ap.add_argument("--only", default="", help="comma list of query names to keep")
    args = ap.parse_args()
    if args.family == "c2":
        queries = DENSE5 + SPARSE5
    else:
        queries = [q for k in map(int, args.family.split(",")) for q in dense_family(k)]
    if args.only:
        keep = set(args.only.split(","))
        queries = [q for q in queries if q.name in keep]
    ctx = Cuts(device=0)
    for abc in args.abc or ["0.57,0.19,0.19"]:
        a, b, c = map(float, abc.split(","))
        t = time.time()
        g = rmat_graph_torch(args.scale, args.ef, a, b, c, seed=args.seed, device="cuda")
        gen_s = time.time() - t
        d = g.degrees()
        ctx.load_csr(g)
        line = json.dumps({"graph": g.name, "n": g.n, "m": g.m, "maxdeg": int(d.max()), "gen_s": round(gen_s, 1),
                           "isolated": int((d == 0).sum()), "deg_ge7": int((d >= 7).sum())})
        print(line, flush=True)
        if args.out:
            with open(args.out, "a") as f:
                f.write(line + "\n")
        for q in queries:
            qr, qc = q.csr()
            ctx.set_query(qr, qc)
            rec = {"q": q.name}
            for nparts in [p for p in (32768, 4096, 512, 64, 8, 1) if args.min_nparts <= p <= args.max_nparts]:
                ctx.set_root_slice(0, 2**64 - 1, 0, nparts)
                torch.cuda.synchronize()
                t = time.time()
                cnt = ctx.count("hybrid")
                ts = time.time() - t
                st = ctx.stats()
                rec.update({"nparts": nparts, "count_part": cnt, "est_count": cnt * nparts, "s": round(ts, 4),
                            "est_full_s": round(ts * nparts, 2), "items_part": st["items"],
                            "levels_part": st["level_size"]})
                if nparts == 1:
                    rec["emb_per_s"] = cnt / ts
                    rec["items_per_s"] = st["items"] / ts
                if ts * nparts > args.budget * 1.5:
                    break
            ctx.set_root_slice()
            line = json.dumps(rec)
            print(line, flush=True)
            if args.out:
                with open(args.out, "a") as f:
                    f.write(line + "\n")


if __name__ == "__main__":
    main()
