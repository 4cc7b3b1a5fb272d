"""Simulated C5 strong scaling on ONE GPU: for N in (1, 2, 4, 8) run each rank's static
cyclic share (cuts_set_root_slice(0, -, r, N)) of the C4 workload back to back and take
the max over ranks as the N-GPU step time (the ranks share nothing but the final count
sum, so they need not run concurrently).  The dynamic queue and Alg. 3 donations of the
real N > 1 bench can only improve on the static split.

    python tools/scale_sim.py --depths 1 3 [--out gpurun_out/scale_sim.jsonl]
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
    ap.add_argument("--depths", type=int, nargs="+", default=[1, 3])
    ap.add_argument("--ns", type=int, nargs="+", default=[1, 2, 4, 8])
    ap.add_argument("--out", default="")
    args = ap.parse_args()
    spec, qs = C4.parts[0]
    q = qs[0]
    g = spec.build()
    ctx = Cuts(device=0)
    ctx.load_graph(torch.from_numpy(g.row_ptr.view("int64")).cuda(), torch.from_numpy(g.col.view("int32")).cuda())
    qr, qc = q.csr()
    out = open(args.out, "a") if args.out else None
    for depth in args.depths:
        for n in args.ns:
            ctx.set_query(qr, qc)
            ctx.set_root_range(*C4.roots(ctx.level1_size()[0]))
            ctx.set_partition_depth(depth)
            L = ctx.partition_size()
            times, counts = [], []
            for r in range(n):
                ctx.set_root_slice(0, 2**64 - 1, r, n)
                ctx.set_debug(timing=True)
                torch.cuda.synchronize()
                t = time.time()
                counts.append(ctx.count("hybrid"))
                torch.cuda.synchronize()
                times.append(time.time() - t)
            rec = {"workload": "C4", "query": q.name, "partition_depth": depth, "partition_list": L, "n": n,
                   "count": sum(counts), "rank_s": [round(x, 4) for x in times], "max_s": max(times),
                   "sum_s": sum(times), "imbalance": max(times) / (sum(times) / n)}
            print(json.dumps(rec), flush=True)
            if out:
                out.write(json.dumps(rec) + "\n")
    ctx.set_partition_depth(1)


if __name__ == "__main__":
    main()
