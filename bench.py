"""Benchmark: embeddings/s of the cuTS hot path on B200 (one JSON line on rank 0).

    python bench.py [--gpus N] [--steps K] [--warmup W] [--workload C2] [--impl ours|reference]

A step = one pass of the whole hot path (level-1 seed, every extend level,
count-only last level, hybrid chunking) over every (graph, query) of the
workload, with the graphs resident in HBM.  value = embeddings counted by all
ranks / max-over-ranks device time.  Multi-GPU (torchrun): level-1 roots are
partitioned across ranks and the per-rank counts are summed with
an NCCL all-reduce (the path's only exchange step).
"""
from __future__ import annotations

import argparse
import json
import os
import statistics
import subprocess
import sys
import time

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

MEASURED = os.path.join(ROOT, "MEASURED_PEAKS.json")
FALLBACK_HBM_GBS = 6650.0   # B200_PROFILING.md fallback


def _args():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=3)
    ap.add_argument("--warmup", type=int, default=3)
    ap.add_argument("--workload", default="C2")
    ap.add_argument("--impl", default="ours", choices=["ours", "reference"])
    ap.add_argument("--no-cpu-baseline", action="store_true")
    ap.add_argument("--chunks-per-rank", type=int, default=16, help="dynamic root queue granularity (N > 1)")
    ap.add_argument("--donate", action="store_true",
                    help="N > 1: add Alg. 3 prefix donations (NCCL send/recv) to the root queue; validated with "
                         "gloo and two ranks on one GPU only, so off by default")
    ap.add_argument("--cpu-budget", type=float, default=15.0, help="seconds of oracle work for cpu_baseline")
    return ap.parse_args()


def _dist():
    rank = int(os.environ.get("RANK", "0"))
    world = int(os.environ.get("WORLD_SIZE", "1"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    return rank, world, local


def _peaks():
    try:
        d = json.load(open(MEASURED))
        return float(d["hbm_gbs"]), "measured (MEASURED_PEAKS.json, copy bandwidth)"
    except Exception:
        return FALLBACK_HBM_GBS, "fallback (B200_PROFILING.md)"


class ClockSampler:
    """nvidia-smi clocks + throttle reasons sampled during the timed region."""
    Q = ("clocks.sm,clocks.max.sm,clocks_event_reasons.hw_slowdown,clocks_event_reasons.hw_thermal_slowdown,"
         "clocks_event_reasons.sw_thermal_slowdown,clocks_event_reasons.sw_power_cap")

    def __init__(self, index: int):
        self.index = index
        self.proc = None

    def start(self):
        try:
            self.proc = subprocess.Popen(["nvidia-smi", "-i", str(self.index), f"--query-gpu={self.Q}",
                                          "--format=csv,noheader,nounits", "-lms", "200"],
                                         stdout=subprocess.PIPE, stderr=subprocess.DEVNULL, text=True)
        except Exception:
            self.proc = None

    def stop(self):
        if self.proc is None:
            return {"sm_mhz": None, "sm_max_mhz": None, "reasons": ["nvidia-smi unavailable"]}
        self.proc.terminate()
        out, _ = self.proc.communicate(timeout=10)
        sm, mx, reasons = [], [], set()
        names = ["hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown", "sw_power_cap"]
        for line in out.strip().splitlines():
            f = [x.strip() for x in line.split(",")]
            if len(f) < 6:
                continue
            try:
                sm.append(float(f[0]))
                mx.append(float(f[1]))
            except ValueError:
                continue
            for nm, v in zip(names, f[2:6]):
                if v.lower() == "active":
                    reasons.add(nm)
        load = [s for s in sm if s > 0.5 * max(mx or [1])] or sm
        return {"sm_mhz": statistics.median(load) if load else None, "sm_max_mhz": max(mx) if mx else None,
                "reasons": sorted(reasons), "samples": len(sm)}


# ------------------------------------------------------------------ our arm
def run_ours(args):
    import numpy as np
    import torch
    from workloads import WORKLOADS
    from paper_conf_sc_xiangkshs21_b200 import Cuts

    rank, world, local = _dist()
    torch.cuda.set_device(local)
    dev = torch.device("cuda", local)
    if world > 1:
        import torch.distributed as dist
        dist.init_process_group("nccl", device_id=dev)
    wl = WORKLOADS[args.workload]
    graphs = [(spec.build(), qs) for spec, qs in wl.parts]
    stream = torch.cuda.Stream(device=dev)
    ctx = Cuts(device=local, stream=stream)     # one arena: most of the free HBM
    # graph tensors resident in HBM (device leg) and pinned on the host (e2e leg)
    dev_graphs, host_graphs = [], []
    for g, _ in graphs:
        rp = torch.from_numpy(g.row_ptr.view(np.int64))
        cl = torch.from_numpy(g.col.view(np.int32))
        host_graphs.append((rp.pin_memory(), cl.pin_memory()))
        dev_graphs.append((rp.to(dev), cl.to(dev)))
    for rp, cl in dev_graphs:
        ctx.load_graph(rp, cl, validate=True)
    flush = torch.empty(256 << 20, dtype=torch.uint8, device=dev)   # > 126 MB L2

    from paper_conf_sc_xiangkshs21_b200 import dist as D
    store = D.default_store() if world > 1 else None
    pass_id = [0]
    donations = [0]

    def set_q(c, q):
        qr, qc = q.csr()
        c.set_query(qr, qc)

    def count_q(c, q, tag):
        """This rank's share of one query.  N = 1: all roots.  N > 1: the seeded-
        shuffled level-1 list is cut into world*CHUNKS chunks pulled from a shared
        atomic counter (dynamic root redistribution)."""
        set_q(c, q)
        if wl.root_range is not None:                 # stated root range (C4)
            c.set_root_range(*wl.roots(c.level1_size()[0]))
        if world == 1:
            return c.count(wl.mode), [c.stats()]
        _, l1 = c.level1_size()
        cs = max(1, -(-l1 // (world * args.chunks_per_rank)))
        queue = D.RootQueue(store, f"{tag}", D.n_chunks(l1, cs))
        if args.donate:
            # root chunks, then serve as a receiver of donated flat prefixes (Alg. 3)
            eng = D.CutsEngine(c, wl.mode)
            ws = D.WorkSharing(store, f"ws{tag}", rank, world, eng, transport_device=dev)
            local = ws.run(queue, cs)
            donations[0] += ws.sent
            return local, eng.stats
        local, sts = 0, []
        while (ch := queue.next()) is not None:
            b, e = D.chunk_bounds(ch, cs)
            c.set_root_slice(b, e, 0, 1)
            local += c.count(wl.mode)
            sts.append(c.stats())
        return local, sts

    def step(timing=False):
        """One pass over every (graph, query); returns (local count, launches, ms_extend, launches_ext)."""
        total, launches, ms_ext, n_ext = 0, 0, 0.0, 0
        c = ctx
        c.set_debug(timing=timing)
        pass_id[0] += 1
        for gi, ((rp, cl), (g, qs)) in enumerate(zip(dev_graphs, graphs)):
            c.load_graph(rp, cl)                      # borrows the resident CSR, derives deg
            launches += 1
            for qi, q in enumerate(qs):
                cnt, sts = count_q(c, q, f"p{pass_id[0]}g{gi}q{qi}")
                total += cnt
                for st in sts:
                    launches += st["launches"]
                    ms_ext += st["ms_extend"]
                    n_ext += st["extend_launches"]
        return total, launches, ms_ext, n_ext

    def barrier():
        torch.cuda.synchronize(dev)
        if world > 1:
            import torch.distributed as dist
            dist.barrier()

    for _ in range(args.warmup):
        step()
    barrier()
    sampler = ClockSampler(local)
    sampler.start()
    times, counts, launches, ms_ext, n_ext = [], [], 0, 0.0, 0
    ev0, ev1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    for _ in range(args.steps):
        flush.fill_(1)                      # evict L2 between timed steps
        barrier()
        ev0.record(stream)
        cnt, la, me, ne = step(timing=True)
        ev1.record(stream)
        torch.cuda.synchronize(dev)
        times.append(ev0.elapsed_time(ev1))
        counts.append(cnt)
        launches += la
        ms_ext += me
        n_ext += ne
    clocks = sampler.stop()
    barrier()
    step_ms_local = sum(times) / len(times)
    local_count = counts[-1]
    # exchange: sum of counts over ranks, max of time over ranks
    step_ms = D.allreduce_max(step_ms_local, device=dev)         # max over ranks
    step_count = D.allreduce_count(local_count, device=dev)      # the one exchange: NCCL sum of counts
    value = step_count / (step_ms / 1e3)

    # e2e: the user's call with HOST buffers (pinned H2D of the graphs each step, counts back to host)
    e2e_ms, h2d = [], 0
    for _ in range(max(1, args.steps)):
        flush.fill_(1)
        barrier()
        ev0.record(stream)
        cnt = 0
        h2d = 0
        with torch.cuda.stream(stream):
            c = ctx
            for (g, qs), (hrp, hcl) in zip(graphs, host_graphs):
                drp = hrp.to(dev, non_blocking=True)
                dcl = hcl.to(dev, non_blocking=True)
                h2d += hrp.numel() * 8 + hcl.numel() * 4
                c.load_graph(drp, dcl)
                for qi, q in enumerate(qs):
                    pass_id[0] += 1
                    cnt += count_q(c, q, f"e{pass_id[0]}q{qi}")[0]
        ev1.record(stream)
        torch.cuda.synchronize(dev)
        e2e_ms.append(ev0.elapsed_time(ev1))
    e2e_local = D.allreduce_max(sum(e2e_ms) / len(e2e_ms), device=dev)
    nq = sum(len(qs) for _, qs in graphs)

    # algorithmic bytes of the dominant kernel (k_extend), instrumented untimed pass
    alg_ext = 0
    ctx.set_debug(bytes_=True)
    for (rp, cl), (g, qs) in zip(dev_graphs, graphs):
        ctx.load_graph(rp, cl)
        for qi, q in enumerate(qs):
            pass_id[0] += 1
            alg_ext += sum(st["alg_bytes_extend"] for st in count_q(ctx, q, f"b{pass_id[0]}q{qi}")[1])
    ctx.set_debug()
    peak, peak_src = _peaks()
    per_step_ext_ms = ms_ext / args.steps
    achieved = alg_ext / (per_step_ext_ms / 1e3) / 1e9 if per_step_ext_ms > 0 else None
    traffic = None
    tpath = os.path.join(ROOT, "profiles", "r01_traffic.json")
    if os.path.exists(tpath):
        try:
            traffic = json.load(open(tpath)).get("bytes_per_launch")
        except Exception:
            traffic = None

    out = {
        "metric": "embeddings/s", "value": value, "unit": "embeddings/s", "n_gpus": world,
        "steps": args.steps, "warmup": args.warmup, "ms_per_step": step_ms, "higher_is_better": True,
        "scaling": "weak" if world > 1 else "weak", "vs_baseline": None, "dtype": "u32", "data": "synthetic",
        "config": {"workload": wl.name, "description": wl.description, "queries": nq,
                   "graphs": [s.name for s, _ in wl.parts], "embeddings_per_step": step_count,
                   "mode": wl.mode, "l2": "flushed between timed steps (256 MiB write)",
                   "root_range": (list(wl.root_range) if wl.root_range else None),
                   "parallelism": (f"dynamic root-chunk queue x{world} ({args.chunks_per_rank} chunks/rank/query)"
                                   + (" + Alg. 3 prefix donations (NCCL send/recv)" if args.donate else "")
                                   + " + NCCL all-reduce of counts" if world > 1 else "1 GPU"),
                   "donations": donations[0] if world > 1 else 0},
        "e2e": {"value": step_count / (e2e_local / 1e3), "unit": "embeddings/s", "h2d_bytes_per_step": h2d,
                "d2h_bytes_per_step": 8 * nq, "ms_per_step": e2e_local},
        "gpu_launches": launches // args.steps,
        "roofline": {"bound": "hbm", "kernel": "k_extend", "achieved": achieved, "peak": peak, "unit": "GB/s",
                     "frac": (achieved / peak) if achieved else None, "traffic": traffic,
                     "peak_source": peak_src, "alg_bytes_per_step": alg_ext, "extend_ms_per_step": per_step_ext_ms,
                     "extend_launches_per_step": n_ext // args.steps,
                     "extend_share_of_step": per_step_ext_ms / step_ms_local if step_ms_local else None},
        "clocks": clocks,
    }
    if rank == 0 and world == 1 and not args.no_cpu_baseline:
        out["cpu_baseline"] = cpu_baseline(wl, budget=args.cpu_budget)
    if rank == 0:
        print(json.dumps(out), flush=True)
    if world > 1:
        import torch.distributed as dist
        dist.destroy_process_group()


# ------------------------------------------------------------ oracle legs
def _oracle_sample(wl, budget: float):
    """Time the CPU oracle (as it stands, 1 thread) on a bounded sample of the
    workload: for each query the first r roots of the canonical level-1 list
    (ids are randomly relabelled, so a prefix is a random sample), r doubling
    until the query's share of the budget is used or the list is exhausted."""
    import oracle
    graphs = [(spec.build(), qs) for spec, qs in wl.parts]
    nq = sum(len(qs) for _, qs in graphs)
    per_q = budget / nq
    tot_cnt, tot_s, sample = 0, 0.0, []
    for g, qs in graphs:
        deg = g.degrees()
        for q in qs:
            l1 = int((deg >= max(q.degrees())).sum())
            r, last = 1, None
            while True:
                t = time.perf_counter()
                c = oracle.count(g, q, root_begin=0, root_end=r)
                dt = time.perf_counter() - t
                last = (r, c, dt)
                if dt >= per_q / 3 or r >= l1:
                    break
                r = min(l1, r * 2)
            tot_cnt += last[1]
            tot_s += last[2]
            sample.append(f"{q.name}:{last[0]}/{l1}")
    return tot_cnt, tot_s, sample


def cpu_baseline(wl, budget: float):
    cnt, secs, sample = _oracle_sample(wl, budget)
    return {"value": cnt / secs if secs else None, "unit": "embeddings/s", "cores": 1, "kind": "oracle",
            "sample": "canonical root prefix per query (roots/level-1 size): " + ", ".join(sample),
            "seconds": secs, "embeddings": cnt}


def run_reference(args):
    rank, world, _ = _dist()
    if rank != 0:
        return
    from workloads import WORKLOADS
    wl = WORKLOADS[args.workload]
    budget = max(5.0, 120.0 / max(1, args.steps + args.warmup))
    for _ in range(args.warmup):
        _oracle_sample(wl, budget)
    cnts, secs = 0, 0.0
    sample = None
    for _ in range(args.steps):
        c, s, sample = _oracle_sample(wl, budget)
        cnts += c
        secs += s
    value = cnts / secs if secs else None
    print(json.dumps({
        "impl": "reference", "metric": "embeddings/s", "value": value, "unit": "embeddings/s", "n_gpus": world,
        "steps": args.steps, "warmup": args.warmup, "ms_per_step": 1e3 * secs / max(1, args.steps),
        "higher_is_better": True, "scaling": "weak", "vs_baseline": None, "dtype": "u32", "data": "synthetic",
        "config": {"workload": wl.name, "description": wl.description},
        "cpu_baseline": {"value": value, "unit": "embeddings/s", "cores": 1, "kind": "oracle",
                         "sample": "canonical root prefix per query: " + ", ".join(sample or [])},
        "e2e": {"value": value, "unit": "embeddings/s", "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0},
    }), flush=True)


if __name__ == "__main__":
    a = _args()
    if a.impl == "reference":
        run_reference(a)
    else:
        run_ours(a)
