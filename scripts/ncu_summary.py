"""Summarise an ncu report: key SOL / occupancy / pipe / stall metrics."""
import csv
import io
import subprocess
import sys

KEYS = ['Duration', 'Compute (SM) Throughput', 'Memory Throughput', 'DRAM Throughput',
        'Achieved Occupancy', 'Registers Per Thread', 'Issue Slots Busy', 'Executed Ipc Active',
        'Theoretical Occupancy', 'Warp Cycles Per Issued Instruction', 'No Eligible',
        'Active Warps Per Scheduler', 'Eligible Warps Per Scheduler', 'L1/TEX Hit Rate',
        'Executed Instructions', 'Avg. Divergent Branches', 'Block Limit Registers',
        'L2 Hit Rate', 'Mem Busy', 'Max Bandwidth', 'SM Busy']


def details(rep):
    out = subprocess.run(['ncu', '-i', rep, '--page', 'details', '--csv'], capture_output=True,
                         text=True).stdout
    rows = list(csv.reader(io.StringIO(out)))
    h = rows[0]
    res = []
    for row in rows[1:]:
        d = dict(zip(h, row))
        if any(k == d.get('Metric Name') for k in KEYS):
            res.append((d.get('Section Name', ''), d['Metric Name'], d.get('Metric Value'),
                        d.get('Metric Unit')))
    return res


def raw(rep, pats):
    out = subprocess.run(['ncu', '-i', rep, '--page', 'raw', '--csv'], capture_output=True,
                         text=True).stdout
    rows = list(csv.reader(io.StringIO(out)))
    h, units = rows[0], rows[1]
    vals = rows[2] if len(rows) > 2 else []
    res = []
    for name, u, v in zip(h, units, vals):
        if any(p in name for p in pats):
            res.append((name, v, u))
    return res


if __name__ == '__main__':
    for rep in sys.argv[1:]:
        print('==', rep)
        for s, n, v, u in details(rep):
            print(f'  {n:45s} {v} {u}')
        for n, v, u in raw(rep, ['dram__bytes_read.sum', 'dram__bytes_write.sum',
                                 'sm__inst_executed_pipe_fp64', 'sm__inst_executed_pipe_alu.sum',
                                 'sm__inst_executed_pipe_fma.sum', 'sm__inst_executed_pipe_lsu.sum',
                                 'sm__inst_executed_pipe_xu.sum', 'smsp__inst_executed.sum ',
                                 'sm__pipe_fp64_cycles_active', 'smsp__average_warp_latency_issue_stalled',
                                 'sm__inst_executed_pipe_uniform', 'pipe_fp64']):
            if 'pct' in n or 'sum' in n or 'ratio' in n:
                print(f'  {n:60s} {v} {u}')
