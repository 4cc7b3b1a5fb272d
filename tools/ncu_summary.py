"""Summarise an ncu report (details + raw stall counters) as text for profiles/."""
import csv
import io
import subprocess
import sys

KEEP = ['Duration', 'DRAM Throughput', 'L1/TEX Hit Rate', 'L2 Hit Rate', 'Issue Slots Busy',
        'Warp Cycles Per Issued Instruction', 'Achieved Occupancy', 'Theoretical Occupancy', 'Registers Per Thread',
        'Executed Instructions', 'Memory Throughput', 'L2 Cache Throughput', 'L1/TEX Cache Throughput',
        'Compute (SM) Throughput', 'Avg. Active Threads Per Warp', 'Eligible Warps Per Scheduler', 'Grid Size',
        'Block Size', 'Branch Efficiency', 'Avg. Not Predicated Off Threads Per Warp']
RAW = ['dram__bytes_read.sum', 'dram__bytes_write.sum', 'lts__t_bytes.sum', 'gpu__time_duration.sum',
       'l1tex__t_sectors_pipe_lsu_mem_global_op_ld.sum', 'l1tex__t_requests_pipe_lsu_mem_global_op_ld.sum',
       'smsp__thread_inst_executed_per_inst_executed.ratio', 'sm__warps_active.avg.pct_of_peak_sustained_active',
       'dram__throughput.avg.pct_of_peak_sustained_elapsed']


def run(rep):
    out = []
    d = subprocess.run(['ncu', '-i', rep, '--page', 'details', '--csv'], capture_output=True, text=True).stdout
    r = csv.reader(io.StringIO(d))
    hdr = next(r)
    name = None
    for row in r:
        x = dict(zip(hdr, row))
        name = x.get('Kernel Name', name)
        if x.get('Metric Name') in KEEP:
            out.append(f"{x['Metric Name']} = {x['Metric Value']} {x['Metric Unit']}")
    d = subprocess.run(['ncu', '-i', rep, '--page', 'raw', '--csv'], capture_output=True, text=True).stdout
    r = csv.reader(io.StringIO(d))
    hdr = next(r)
    units = dict(zip(hdr, next(r)))
    stalls = {}
    for row in r:
        x = dict(zip(hdr, row))
        for k in hdr:
            if k in RAW:
                out.append(f"{k} = {x[k]} {units.get(k, '')}")
            if k.startswith('smsp__pcsamp_warps_issue_stalled_') and not k.endswith('not_issued'):
                try:
                    v = float(x[k])
                except ValueError:
                    continue
                if v > 0:
                    stalls[k.replace('smsp__pcsamp_warps_issue_stalled_', '')] = v
    tot = sum(stalls.values()) or 1
    out.append('stall samples (share): ' + ', '.join(f"{k} {v / tot:.1%}" for k, v in sorted(stalls.items(), key=lambda t: -t[1])[:8]))
    return f"kernel: {name}\n" + "\n".join(out)


def _peak():
    import json
    import os
    try:
        return float(json.load(open(os.path.join(os.path.dirname(os.path.dirname(os.path.abspath(__file__))),
                                                 "MEASURED_PEAKS.json")))["hbm_gbs"])
    except Exception:
        return 6650.0


def record(rep):
    """The fields bench.py's roofline reads (profiles/ncu_<workload>_extend.json)."""
    d = subprocess.run(['ncu', '-i', rep, '--page', 'raw', '--csv'], capture_output=True, text=True).stdout
    r = csv.reader(io.StringIO(d))
    hdr = next(r)
    units = dict(zip(hdr, next(r)))
    x = dict(zip(hdr, next(r)))
    scale = {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9, "Tbyte": 1e12,
             "nsecond": 1, "usecond": 1e3, "msecond": 1e6, "second": 1e9, "ns": 1, "us": 1e3, "ms": 1e6, "s": 1e9}
    for k in list(x):                         # section-prefixed names ("FBSP.TriageCompute.dram__...")
        short = k.split(".", 2)[-1] if k.startswith("FBSP.") else k
        if not x.get(short):
            x[short] = x[k]
            units[short] = units.get(k, "")

    def f(k):
        try:
            return float(x[k].replace(',', '')) * scale.get(units.get(k, ''), 1)
        except (KeyError, ValueError):
            return None
    rd, wr, t = f('dram__bytes_read.sum'), f('dram__bytes_write.sum'), f('gpu__time_duration.sum')
    req, sec = f('l1tex__t_requests_pipe_lsu_mem_global_op_ld.sum'), f('l1tex__t_sectors_pipe_lsu_mem_global_op_ld.sum')
    return {"kernel": x.get('Kernel Name'), "report": rep, "dram_bytes_per_launch": (rd or 0) + (wr or 0),
            "duration_ns": t, "dram_gbs": ((rd or 0) + (wr or 0)) / t if t else None,
            "dram_frac_of_measured_peak": (((rd or 0) + (wr or 0)) / t) / _peak() if t else None,
            "dram_gbs_ncu": f('dram__bytes.sum.per_second'),
            "l2_hit_pct": f('lts__t_sector_hit_rate.pct'), "sectors_per_request": sec / req if req else None,
            "thread_inst_per_inst": f('smsp__thread_inst_executed_per_inst_executed.ratio')}


if __name__ == '__main__':
    import json
    args = sys.argv[1:]
    if args and args[0] == '--json':
        print(json.dumps(record(args[1]), indent=1))
    else:
        for rep in args:
            print(f"== {rep}")
            print(run(rep))
