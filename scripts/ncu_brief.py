"""Key metrics + stall reasons + pipe utilizations of `ncu --page raw --csv` exports.
  python scripts/ncu_brief.py raw1.csv [raw2.csv ...]"""
import csv
import sys

KEYS = ['gpu__time_duration.sum', 'launch__registers_per_thread', 'launch__grid_size',
        'smsp__thread_inst_executed_per_inst_executed.ratio', 'smsp__inst_executed.sum',
        'smsp__issue_active.avg.pct_of_peak_sustained_active',
        'sm__warps_active.avg.pct_of_peak_sustained_active',
        'sm__pipe_fp64_cycles_active.avg.pct_of_peak_sustained_active',
        'l1tex__throughput.avg.pct_of_peak_sustained_elapsed',
        'lts__throughput.avg.pct_of_peak_sustained_elapsed',
        'dram__bytes_read.sum', 'dram__bytes_write.sum',
        'smsp__sass_inst_executed_op_local_ld.sum', 'smsp__sass_inst_executed_op_local_st.sum']


def load(f):
    rows = list(csv.reader(open(f)))
    for i, r in enumerate(rows):
        if 'Kernel Name' in r:
            h = r
            return [dict(zip(h, x)) for x in rows[i + 2:] if len(x) == len(h)]
    return []


def num(v):
    try:
        return float(v)
    except (TypeError, ValueError):
        return None


for f in sys.argv[1:]:
    for d in load(f):
        print(f, d['Kernel Name'][:80])
        for k in KEYS:
            if k in d:
                print('   ', k, d[k])
        st = sorted(((num(v), k) for k, v in d.items()
                     if k.startswith('smsp__pcsamp_warps_issue_stalled') and
                     not k.endswith('not_issued') and num(v)), reverse=True)[:8]
        tot = sum(num(v) for k, v in d.items() if k.startswith('smsp__pcsamp_warps_issue_stalled')
                  and not k.endswith('not_issued') and num(v))
        print('    stalls:', ', '.join(f"{k.split('stalled_')[1]} {100 * v / tot:.0f}%" for v, k in st))
        pipes = sorted(((num(v), k) for k, v in d.items()
                        if k.startswith('sm__inst_executed_pipe_') and
                        k.endswith('avg.pct_of_peak_sustained_active') and num(v)), reverse=True)[:6]
        print('    pipes:', ', '.join(f"{k.split('pipe_')[1].split('.')[0]} {v:.1f}%" for v, k in pipes))
