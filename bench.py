"""Benchmark: embeddings/s of the cuTS hot path on B200 (one JSON line on rank 0).

    python bench.py [--gpus N] [--steps K] [--warmup W] [--workload C4|C2|C3|C1] [--impl ours|reference]

A step = one pass of the whole hot path (level-1 seed, every extend level,
count-only last level, hybrid BFS/DFS chunking) over every (graph, query) of
the workload, with the graphs resident in HBM.  value = embeddings counted by
all ranks / max-over-ranks device time.

Default workload = C4 (BASELINE configs[3], the largest single-GPU config): K8
on R-MAT(22,16,.50,.20,.20) over a stated canonical root sub-range whose
level-synchronous trie would exceed 180 GB (asserted from the library's
chunk-summed level sizes), so HYBRID chunking is on the timed path.

Multi-GPU (torchrun, N > 1): the library joins an NCCL world (cuts_set_dist);
the seeded-shuffled level-1 list of the same fixed workload is cut into root
chunks pulled from a shared atomic counter, idle ranks receive Alg. 3 prefix
donations (control plane = the process-group store,
data plane = gloo on the host: prefixes are 4·j bytes per row), and the
per-rank counts are summed by the library's own NCCL all-reduce
(cuts_allreduce_count) — strong scaling of one fixed workload.
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
BFS_TRIE_LIMIT = 180e9      # bytes: a stored level above this cannot be held level-synchronously


def _args():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=3)
    ap.add_argument("--warmup", type=int, default=3)
    ap.add_argument("--workload", default="C4")
    ap.add_argument("--impl", default="ours", choices=["ours", "reference"])
    ap.add_argument("--no-cpu-baseline", action="store_true")
    ap.add_argument("--chunks-per-rank", type=int, default=16, help="dynamic root queue granularity (N > 1)")
    ap.add_argument("--no-donate", action="store_true", help="N > 1: root queue only (no Alg. 3 donations)")
    ap.add_argument("--partition-depth", type=int, default=3,
                    help="N > 1: the dynamic queue hands out chunks of the shuffled level-D list "
                         "(cuts_set_partition_depth; 1 = the paper's level-1 roots)")
    ap.add_argument("--e2e-steps", type=int, default=3, help="steps of the end-to-end (host buffers) leg")
    ap.add_argument("--cpu-budget", type=float, default=20.0, help="seconds of oracle work per cpu_baseline leg")
    ap.add_argument("--no-bytes", action="store_true", help="skip the instrumented algorithmic-bytes pass")
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


def _alu_peak():
    """Word-op ceiling of the tail (tools/micro/alu_peak.cu measured on a B200, profiles/),
    else derived from unit counts: 148 SMs x 8 word-ops/clk (16 POPC/clk/SM, 2 per 64-bit
    word) x 1.965 GHz."""
    try:
        d = json.load(open(os.path.join(ROOT, "profiles", "alu_peak_b200.json")))
        return d["word_ops_per_s"] / 1e9, "measured on B200 (tools/micro/alu_peak.cu, profiles/alu_peak_b200.json)"
    except Exception:
        return 148 * 8 * 1.965, "derived: 148 SMs x 8 word-ops/clk x 1.965 GHz (DESIGN.md §5)"


def _ncu_record(workload: str):
    """ncu --set full figures for the dominant kernel on this workload (profiles/), if captured."""
    path = os.path.join(ROOT, "profiles", f"ncu_{workload.lower()}_extend.json")
    try:
        return json.load(open(path)), os.path.relpath(path, ROOT)
    except Exception:
        return None, None


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
    from paper_conf_sc_xiangkshs21_b200 import dist as D

    rank, world, local = _dist()
    torch.cuda.set_device(local)
    dev = torch.device("cuda", local)
    gloo = None
    if world > 1:
        import torch.distributed as dist
        dist.init_process_group("nccl", device_id=dev)
        gloo = dist.new_group(backend="gloo")          # donation data plane (host prefixes)
    wl = WORKLOADS[args.workload]
    graphs = [(spec.build(), qs) for spec, qs in wl.parts]
    stream = torch.cuda.Stream(device=dev)
    ctx = Cuts(device=local, stream=stream)     # one arena: most of the free HBM
    if world > 1:
        import torch.distributed as dist
        uid = [Cuts.dist_unique_id() if rank == 0 else None]
        dist.broadcast_object_list(uid, src=0, group=gloo)
        ctx.set_dist(rank, world, uid[0])        # the library's NCCL communicator (cuts_set_dist)
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
    store = D.default_store() if world > 1 else None
    donate = world > 1 and not args.no_donate
    pass_id = [0]
    donations = [0, 0]          # donations made, prefix rows shipped (this rank)

    def count_q(c, q, tag):
        """This rank's share of one query.  N = 1: the whole root range.  N > 1: chunks of
        the shuffled level-D list (D = --partition-depth; D = 1 is the paper's root
        partition) pulled from a shared atomic counter, then Alg. 3 donations to idle
        ranks (flat prefixes over gloo)."""
        qr, qc = q.csr()
        c.set_query(qr, qc)
        if wl.root_range is not None:                 # stated root range (C4)
            c.set_root_range(*wl.roots(c.level1_size()[0]))
        if world == 1:
            return c.count(wl.mode), [c.stats()]
        c.set_partition_depth(args.partition_depth)
        l1 = c.partition_size()                     # |L_D| over the root range
        cs = max(1, -(-l1 // (world * args.chunks_per_rank)))
        queue = D.RootQueue(store, tag, D.n_chunks(l1, cs))
        if donate:
            eng = D.CutsEngine(c, wl.mode)
            ws = D.WorkSharing(store, f"ws{tag}", rank, world, eng, transport_device=None, group=gloo)
            n = ws.run(queue, cs)
            donations[0] += ws.sent
            donations[1] += ws.sent_rows
            return n, eng.stats
        n, sts = 0, []
        while (ch := queue.next()) is not None:
            b, e = D.chunk_bounds(ch, cs)
            c.set_root_slice(b, e, 0, 1)
            n += c.count(wl.mode)
            sts.append(c.stats())
        return n, sts

    tail = [0.0, 0]              # this step's k_dlr_tail ms and launches

    def step(timing=False):
        """One pass over every (graph, query): (local count, launches, ms_extend, extend launches, level sizes)."""
        total, launches, ms_ext, n_ext, fused = 0, 0, 0.0, 0, 0
        tail[0] = tail[1] = 0
        levels = [0] * 9
        ctx.set_debug(timing=timing)
        pass_id[0] += 1
        for gi, ((rp, cl), (g, qs)) in enumerate(zip(dev_graphs, graphs)):
            ctx.load_graph(rp, cl)                    # borrows the resident CSR, derives deg
            launches += 1
            for qi, q in enumerate(qs):
                cnt, sts = count_q(ctx, q, f"p{pass_id[0]}g{gi}q{qi}")
                total += cnt
                for st in sts:
                    launches += st["launches"]
                    ms_ext += st["ms_extend"]
                    tail[0] += st["ms_tail"]
                    tail[1] += st["tail_launches"]
                    n_ext += st["extend_launches"]
                    fused |= st["fused_levels"]
                    for j, v in enumerate(st["level_size"]):
                        levels[j] += v
        return total, launches, ms_ext, n_ext, (levels, fused)

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
    times, counts, launches, ms_ext, n_ext, levels = [], [], 0, 0.0, 0, ([], 0)
    ms_tail, n_tail = 0.0, 0
    ev0, ev1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    for _ in range(args.steps):
        flush.fill_(1)                      # evict L2 between timed steps
        barrier()
        ev0.record(stream)
        cnt, la, me, ne, levels = step(timing=True)
        ev1.record(stream)
        torch.cuda.synchronize(dev)
        times.append(ev0.elapsed_time(ev1))
        counts.append(cnt)
        launches += la
        ms_ext += me
        n_ext += ne
        ms_tail += tail[0]
        n_tail += tail[1]
    clocks = sampler.stop()
    barrier()
    step_ms_local = sum(times) / len(times)
    local_count = counts[-1]
    step_ms = D.allreduce_max(step_ms_local, device=dev)            # max over ranks
    step_count = D.allreduce_count(local_count, device=dev, ctx=ctx)   # the library's NCCL sum (N > 1)
    levels, fused = levels
    levels = [D.allreduce_count(v, device=dev) for v in levels]      # chunk- and rank-summed level sizes
    value = step_count / (step_ms / 1e3)
    nq = sum(len(qs) for _, qs in graphs)
    kmax = max(q.k for _, qs in graphs for q in qs)
    stored = [j for j in range(1, kmax) if not (fused >> j) & 1]     # levels written to the trie arena
    deepest = max((levels[j] for j in stored), default=0)
    if wl.min_trie_bytes and 8 * deepest <= wl.min_trie_bytes:
        raise SystemExit(f"workload {wl.name}: deepest stored level {deepest} entries = {8 * deepest:.3e} B "
                         f"<= {wl.min_trie_bytes:.3e} B — the root range no longer forces HYBRID chunking")

    # e2e: the user's call with HOST buffers (pinned H2D of the graphs each step, counts back to host)
    e2e_ms, h2d = [], 0
    for _ in range(max(1, min(args.steps, args.e2e_steps))):
        flush.fill_(1)
        barrier()
        ev0.record(stream)
        h2d = 0
        with torch.cuda.stream(stream):
            for (g, qs), (hrp, hcl) in zip(graphs, host_graphs):
                drp = hrp.to(dev, non_blocking=True)
                dcl = hcl.to(dev, non_blocking=True)
                h2d += hrp.numel() * 8 + hcl.numel() * 4
                ctx.load_graph(drp, dcl)
                for qi, q in enumerate(qs):
                    pass_id[0] += 1
                    count_q(ctx, q, f"e{pass_id[0]}q{qi}")
        ev1.record(stream)
        torch.cuda.synchronize(dev)
        e2e_ms.append(ev0.elapsed_time(ev1))
    e2e_local = D.allreduce_max(sum(e2e_ms) / len(e2e_ms), device=dev)
    for rp, cl in dev_graphs[-1:]:
        ctx.load_graph(rp, cl)

    # algorithmic bytes of the dominant kernel (k_extend), instrumented untimed pass
    alg_ext = alg_need = tail_ops = 0
    if not args.no_bytes:
        ctx.set_debug(bytes_=True)
        for (rp, cl), (g, qs) in zip(dev_graphs, graphs):
            ctx.load_graph(rp, cl)
            for qi, q in enumerate(qs):
                pass_id[0] += 1
                for st in count_q(ctx, q, f"b{pass_id[0]}q{qi}")[1]:
                    alg_ext += st["alg_bytes_extend"]
                    alg_need += st["alg_bytes_extend_needed"]
                    tail_ops += st["tail_word_ops"]
        ctx.set_debug()
        alg_ext = D.allreduce_count(alg_ext, device=dev)
        alg_need = D.allreduce_count(alg_need, device=dev)
        tail_ops = D.allreduce_count(tail_ops, device=dev)
    peak, peak_src = _peaks()
    per_step_ext_ms = D.allreduce_max(ms_ext / args.steps, device=dev)
    achieved = alg_ext / (per_step_ext_ms / 1e3) / 1e9 if per_step_ext_ms > 0 and alg_ext else None
    achieved_need = alg_need / (per_step_ext_ms / 1e3) / 1e9 if per_step_ext_ms > 0 and alg_need else None
    ncu, ncu_src = _ncu_record(wl.name)
    model = {"bound": "hbm", "kernels": "every extend kernel (k_extend, k_pairs, k_lr_*, k_dlr_*)",
             "achieved": achieved, "peak": peak, "unit": "GB/s", "frac": (achieved / peak) if achieved else None,
             "model": "SURVEY §8.d, frozen: per entry 4·d per backward list (every list read once, P:1086) "
                      "+ 4 per intersection survivor + children written; per step over all levels and chunks",
             "peak_source": peak_src, "alg_bytes_per_step": alg_ext, "needed_bytes_per_step": alg_need,
             "achieved_needed": achieved_need, "frac_needed": (achieved_need / peak) if achieved_need else None,
             "extend_ms_per_step": per_step_ext_ms, "extend_launches_per_step": n_ext // args.steps,
             "extend_share_of_step": per_step_ext_ms / step_ms if step_ms else None}
    tail_ms = D.allreduce_max(ms_tail / args.steps, device=dev)
    if tail_ms > 0 and tail_ops:
        # the dominant kernel is the deep-local-rows tail: integer bit algebra on L1-resident
        # rows, so its roofline is the ALU rate of its unit
        apk, apk_src = _alu_peak()
        ach = tail_ops / (tail_ms / 1e3) / 1e9
        roof = {"bound": "alu", "kernel": "the deep-rows tail (k_dlr_tail_warp<1|2> + k_dlr_tail_cta)", "achieved": ach,
                "peak": apk, "unit": "Gword-op/s",
                "frac": ach / apk, "traffic": ncu.get("dram_bytes_per_launch") if ncu else None,
                "per_unit": "one 64-bit AND + POPC + add of the symmetric 4-clique bit algebra "
                            "(count from the instrumented pass, CUTS_DEBUG_BYTES)",
                "word_ops_per_step": tail_ops, "kernel_ms_per_step": tail_ms,
                "launches_per_step": n_tail // args.steps, "share_of_step": tail_ms / step_ms if step_ms else None,
                "peak_source": apk_src, "hbm_model_8d": model}
    else:
        roof = dict(model, kernel="k_extend", traffic=ncu.get("dram_bytes_per_launch") if ncu else None)
    if ncu:
        roof["ncu"] = dict(ncu, source=ncu_src)

    out = {
        "metric": "embeddings/s", "value": value, "unit": "embeddings/s", "n_gpus": world,
        "steps": args.steps, "warmup": args.warmup, "ms_per_step": step_ms, "higher_is_better": True,
        "scaling": "strong" if world > 1 else "weak", "vs_baseline": None, "dtype": "u32", "data": "synthetic",
        "config": {"workload": wl.name, "description": wl.description, "queries": nq,
                   "graphs": [s.name for s, _ in wl.parts], "embeddings_per_step": step_count,
                   "mode": wl.mode, "l2": "flushed between timed steps (256 MiB write)",
                   "root_range": (list(wl.root_range) if wl.root_range else None),
                   "level_size_per_step": levels, "stored_levels": stored,
                   "deepest_stored_level_entries": deepest, "deepest_stored_level_bytes": 8 * deepest,
                   "bfs_trie_bytes_at_largest_level": 8 * max(levels[1:kmax], default=0),
                   "parallelism": (f"NCCL world {world} via cuts_set_dist; dynamic root-chunk queue "
                                   f"({args.chunks_per_rank} chunks/rank/query of the shuffled level-"
                                   f"{args.partition_depth} list)"
                                   + (" + Alg. 3 prefix donations (store control plane, gloo host data plane)"
                                      if donate else "")
                                   + " + cuts_allreduce_count" if world > 1 else "1 GPU"),
                   "donations": D.allreduce_count(donations[0], device=dev) if world > 1 else 0,
                   "donated_rows": D.allreduce_count(donations[1], device=dev) if world > 1 else 0},
        "e2e": {"value": step_count / (e2e_local / 1e3), "unit": "embeddings/s", "h2d_bytes_per_step": h2d,
                "d2h_bytes_per_step": 8 * nq, "ms_per_step": e2e_local,
                "steps": max(1, min(args.steps, args.e2e_steps))},
        "gpu_launches": launches // args.steps,
        "roofline": roof,
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
def _cpu_model():
    try:
        for line in open("/proc/cpuinfo"):
            if line.startswith("model name"):
                return line.split(":", 1)[1].strip()
    except Exception:
        pass
    return None


def _in_child(fn, timeout, cpus=None):
    """Run fn() in a forked child (optionally pinned to `cpus`, i.e. taskset) and
    return (result, wall seconds), or None if it did not finish within timeout."""
    import multiprocessing as mp
    ctx = mp.get_context("fork")
    rd, wr = ctx.Pipe(duplex=False)

    def child():
        if cpus is not None:
            os.sched_setaffinity(0, cpus)
        t = time.perf_counter()
        r = fn()
        wr.send((r, time.perf_counter() - t))

    p = ctx.Process(target=child, daemon=True)
    p.start()
    wr.close()
    ok = rd.poll(timeout)
    res = rd.recv() if ok else None
    if p.is_alive():
        p.kill()
    p.join()
    return res


def _oracle_sample(wl, budget: float, threads: int, fixed=None):
    """Time the CPU oracle (as it stands) on a bounded sample of the workload: for
    each query the first r roots of the workload's canonical root range (ids are
    randomly relabelled, so a prefix is a random sample), r doubling while the
    query's share of the budget lasts (each try in a child process with a
    deadline, so one heavy root cannot overrun).  threads == 1: the
    single-threaded oracle pinned to one core (taskset -c 0); threads > 1: the
    root-parallel driver (oracle_count_mt) with `threads` threads.  fixed: the
    sample (list of r per query) to reuse.  Returns (count, seconds, sample)."""
    import oracle
    graphs = [(spec.build(), qs) for spec, qs in wl.parts]
    nq = sum(len(qs) for _, qs in graphs)
    per_q = budget / nq
    cpu0 = {sorted(os.sched_getaffinity(0))[0]}
    tot_cnt, tot_s, sample, qi = 0, 0.0, [], 0
    for g, qs in graphs:
        deg = g.degrees()
        for q in qs:
            l1 = int((deg >= max(q.degrees())).sum())
            b0, b1 = wl.roots(l1)

            def run(r):
                if threads == 1:
                    return _in_child(lambda: oracle.count(g, q, root_begin=b0, root_end=b0 + r), per_q, cpu0)
                return _in_child(lambda: oracle.count_mt(g, q, threads, root_begin=b0, root_end=b0 + r), per_q)

            if fixed is not None:
                r = fixed[qi]
                res = run(r) if r else None
                last = (r, res[0], res[1]) if res else None
            else:
                r, last = 1, None
                while True:
                    res = run(r)
                    if res is None:
                        break
                    last = (r, res[0], res[1])
                    if res[1] >= per_q / 3 or r >= b1 - b0:
                        break
                    r = min(b1 - b0, r * 2)
            qi += 1
            if last is None:
                sample.append(f"{q.name}:0/{b1 - b0}")
                continue
            tot_cnt += last[1]
            tot_s += last[2]
            sample.append(f"{q.name}:{last[0]}/{b1 - b0}")
    return tot_cnt, tot_s, sample


def _sample_rs(sample):
    return [int(s.split(":")[1].split("/")[0]) for s in sample]


def cpu_baseline(wl, budget: float):
    """1-core (taskset to one CPU) and N-core (root-parallel, nproc threads) oracle
    timings on the same root sample."""
    nproc = len(os.sched_getaffinity(0))
    cnt1, s1, sample = _oracle_sample(wl, budget, 1)
    cntn, sn, _ = _oracle_sample(wl, budget, nproc, fixed=_sample_rs(sample))
    return {"value": cnt1 / s1 if s1 else None, "unit": "embeddings/s", "cores": 1, "kind": "oracle",
            "sample": "first r roots of the canonical root range per query (r/range size): " + ", ".join(sample),
            "seconds": s1, "embeddings": cnt1, "cpu_model": _cpu_model(), "nproc": nproc,
            "n_core": {"value": cntn / sn if sn else None, "cores": nproc, "seconds": sn, "embeddings": cntn,
                       "kind": "oracle root-parallel driver (oracle_count_mt), same sample"}}


def run_reference(args):
    """The oracle arm: the root-parallel oracle on every host core, each step the
    same bounded root sample of the workload (sized once, before the steps)."""
    rank, world, _ = _dist()
    if rank != 0:
        return
    from workloads import WORKLOADS
    wl = WORKLOADS[args.workload]
    nproc = len(os.sched_getaffinity(0))
    budget = max(4.0, 150.0 / max(1, args.steps + args.warmup))
    _, _, sample = _oracle_sample(wl, budget, nproc)
    rs = _sample_rs(sample)
    for _ in range(args.warmup):
        _oracle_sample(wl, budget * 3, nproc, fixed=rs)
    cnts, secs = 0, 0.0
    for _ in range(args.steps):
        c, s, _ = _oracle_sample(wl, budget * 3, nproc, fixed=rs)
        cnts += c
        secs += s
    value = cnts / secs if secs else None
    print(json.dumps({
        "impl": "reference", "metric": "embeddings/s", "value": value, "unit": "embeddings/s", "n_gpus": world,
        "steps": args.steps, "warmup": args.warmup, "ms_per_step": 1e3 * secs / max(1, args.steps),
        "higher_is_better": True, "scaling": "strong" if world > 1 else "weak", "vs_baseline": None, "dtype": "u32",
        "data": "synthetic", "config": {"workload": wl.name, "description": wl.description},
        "cpu_baseline": {"value": value, "unit": "embeddings/s", "cores": nproc, "kind": "oracle (root-parallel)",
                         "cpu_model": _cpu_model(),
                         "sample": "first r roots of the canonical root range per query: " + ", ".join(sample)},
        "e2e": {"value": value, "unit": "embeddings/s", "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0},
    }), flush=True)


if __name__ == "__main__":
    a = _args()
    if a.impl == "reference":
        run_reference(a)
    else:
        run_ours(a)
