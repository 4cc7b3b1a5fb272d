"""Run one (graph, query) of a workload through the C ABI — a short target for ncu.

    python tools/profile_query.py --workload C2 --part 0 --query K5-K2 [--reps 1] [--stats]
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
    ap.add_argument("--part", type=int, default=0)
    ap.add_argument("--query", default="K5-K2")
    ap.add_argument("--mode", default="hybrid")
    ap.add_argument("--reps", type=int, default=1)
    ap.add_argument("--stats", action="store_true")
    args = ap.parse_args()
    spec, qs = WORKLOADS[args.workload].parts[args.part]
    g = spec.build()
    ctx = Cuts(device=0)
    ctx.load_csr(g)
    q = [x for x in qs if x.name == args.query][0]
    qr, qc = q.csr()
    ctx.set_query(qr, qc)
    ctx.set_debug(timing=args.stats)
    for _ in range(args.reps):
        torch.cuda.synchronize()
        t = time.time()
        c = ctx.count(args.mode)
        dt = time.time() - t
        st = ctx.stats()
        print(json.dumps({"graph": spec.name, "query": q.name, "count": c, "s": dt, "items": st["items"],
                          "items_per_s": st["items"] / dt, "levels": st["level_size"], "chunks": st["chunks"],
                          "windows": st["windows"], "ms_extend": st["ms_extend"], "ms_plan": st["ms_plan"]}))


if __name__ == "__main__":
    main()
