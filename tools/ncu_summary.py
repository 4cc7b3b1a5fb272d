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


if __name__ == '__main__':
    for rep in sys.argv[1:]:
        print(f"== {rep}")
        print(run(rep))
