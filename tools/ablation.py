"""NEXT-2 intersection-method ablation on one GPU.

    python tools/ablation.py --workload C2 [--reps 2] [--out f.jsonl]

Per (graph, query) and variant, best-of-reps seconds of cuts_count plus the
k_extend milliseconds.  Variants (all give the same counts; checked here):
  paper_c   : the paper's c-intersection (Alg. 2 l.19-31): the FIRST backward
              list a1 is the candidate stream, membership by binary search;
              no hub bitmaps, no packed degree stream, no ancestor source
  short_c   : as paper_c, but the SHORTEST list is the stream (B200 choice)
  sv_hubs   : + SV-style bitmaps for hub lists (Alg. 2 l.7-17)
  packed    : + packed (id | degree) stream (degree filter without a gather)
  reuse     : + ancestor-set source
  fastcount : + set-difference count at a single-list degree-free last level
  pairs     : + pair-shared symmetric last level
  lr        : + local rows of the level-(k-2) sibling groups (round 1)
  full      : + deep local rows of the level-(k-3) groups and the symmetric tail
              (round 2; the product default)
Side variants (NEXT-2, compare with the chain member named):
  binned    : fastcount with binned virtual warps at the last level
              instead of the single bin
  sv        : the per-warp scatter-vector intersection (Alg. 2 l.7-17) on CSR
              lists (compare with packed: same source, no bitmaps/reuse)
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

VARIANTS = [  # (name, hub threshold, debug kwargs)
    ("paper_c", None, dict(first_source=True, no_pack=True, no_reuse=True, no_fast_count=True)),
    ("short_c", None, dict(no_pack=True, no_reuse=True, no_fast_count=True)),
    ("sv_hubs", 0, dict(no_pack=True, no_reuse=True, no_fast_count=True)),
    ("packed", 0, dict(no_reuse=True, no_fast_count=True)),
    ("reuse", 0, dict(no_fast_count=True, no_pairs=True)),
    ("fastcount", 0, dict(no_pairs=True)),
    ("pairs", 0, dict(no_lr=True)),
    ("lr", 0, dict(no_dlr=True)),
    ("full", 0, dict()),
    ("binned", 0, dict(no_pairs=True, binned=True)),
    ("sv", None, dict(sv=True)),
]


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--workload", default="C2")
    ap.add_argument("--reps", type=int, default=2)
    ap.add_argument("--variants", default=",".join(v[0] for v in VARIANTS))
    ap.add_argument("--query", default="")
    ap.add_argument("--out", default="")
    ap.add_argument("--range", default="", help="override the workload's root range: absolute canonical a:b")
    args = ap.parse_args()
    wl = WORKLOADS[args.workload]
    ctx = Cuts(device=0)
    want = {}
    totals = {}
    for name, hub, dbg in VARIANTS:
        if name not in args.variants.split(","):
            continue
        totals[name] = 0.0
        for spec, qs in wl.parts:
            g = spec.build()
            ctx.set_hub_threshold(hub)
            ctx.set_debug(**dbg)          # NO_PACK acts at load
            ctx.load_csr(g)
            for q in qs:
                if args.query and q.name != args.query:
                    continue
                qr, qc = q.csr()
                ctx.set_query(qr, qc)
                ctx.set_debug(timing=True, **dbg)
                best, st, c = None, None, None
                for _ in range(args.reps):
                    ctx.set_query(qr, qc)
                    if args.range:
                        ctx.set_root_range(*(int(x) for x in args.range.split(":")))
                    elif wl.root_range is not None:
                        ctx.set_root_range(*wl.roots(ctx.level1_size()[0]))
                    torch.cuda.synchronize()
                    t = time.time()
                    c = ctx.count(wl.mode)
                    dt = time.time() - t
                    if best is None or dt < best:
                        best, st = dt, ctx.stats()
                key = (spec.name, q.name)
                assert want.setdefault(key, c) == c, (name, key, c, want[key])
                totals[name] += best
                rec = {"variant": name, "graph": spec.name, "query": q.name, "range": args.range or None,
                       "count": c, "s": round(best, 4),
                       "ms_extend": round(st["ms_extend"], 2), "ms_plan": round(st["ms_plan"], 2),
                       "hubs": st["hubs"], "items": st["items"]}
                line = json.dumps(rec)
                print(line, flush=True)
                if args.out:
                    with open(args.out, "a") as f:
                        f.write(line + "\n")
        print(json.dumps({"variant": name, "total_s": round(totals[name], 3)}), flush=True)
    ctx.set_debug()


if __name__ == "__main__":
    main()
