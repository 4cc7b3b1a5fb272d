"""Per-query timing of a workload (and optional hub-threshold sweep) on one GPU.

    python tools/sweep.py --workload C2 [--hub 0,64,128,256,off] [--reps 2] [--out f.jsonl]

For every (graph, query) prints count, best-of-reps seconds, k_extend / k_plan
milliseconds (CUDA events on the library stream), items and levels.
"""
import argparse
import json
import os
import sys
import time

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import torch  # noqa: E402

from workloads import WORKLOADS  # noqa: E402
from paper_conf_sc_xiangkshs21_b200 import Cuts  # noqa: E402


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--workload", default="C2")
    ap.add_argument("--hub", default="0", help="comma list of hub thresholds (0 = auto, off = none)")
    ap.add_argument("--reps", type=int, default=2)
    ap.add_argument("--query", default="", help="only this query name")
    ap.add_argument("--out", default="")
    args = ap.parse_args()
    wl = WORKLOADS[args.workload]
    ctx = Cuts(device=0)
    for hub in args.hub.split(","):
        ctx.set_hub_threshold(None if hub == "off" else int(hub))
        tot = 0.0
        for spec, qs in wl.parts:
            g = spec.build()
            ctx.load_csr(g)
            for q in qs:
                if args.query and q.name != args.query:
                    continue
                qr, qc = q.csr()
                ctx.set_query(qr, qc)
                ctx.set_debug(timing=True)
                best, st, c = None, None, None
                for _ in range(args.reps):
                    torch.cuda.synchronize()
                    t = time.time()
                    c = ctx.count(wl.mode)
                    dt = time.time() - t
                    if best is None or dt < best:
                        best, st = dt, ctx.stats()
                tot += best
                rec = {"hub": hub, "hubs": st["hubs"], "hub_t": st["hub_threshold"], "graph": spec.name,
                       "query": q.name, "count": c, "s": round(best, 4), "ms_extend": round(st["ms_extend"], 2),
                       "ms_plan": round(st["ms_plan"], 2), "items": st["items"], "levels": st["level_size"],
                       "chunks": st["chunks"], "windows": st["windows"]}
                line = json.dumps(rec)
                print(line, flush=True)
                if args.out:
                    with open(args.out, "a") as f:
                        f.write(line + "\n")
        print(json.dumps({"hub": hub, "total_s": round(tot, 3)}), flush=True)


if __name__ == "__main__":
    main()
