"""Summarize an `ncu --page source --csv` SASS export: share of issued instructions by
active-lane bucket and the heaviest straight-line segments.
  python scripts/ncu_src_segments.py src.csv [top]"""
import collections
import csv
import sys

rows = list(csv.reader(open(sys.argv[1])))
top = int(sys.argv[2]) if len(sys.argv) > 2 else 25
h = rows[1]
data = [dict(zip(h, r)) for r in rows[2:] if len(r) == len(h)]
ie = lambda d: float(d['Instructions Executed'] or 0)
te = lambda d: float(d['Thread Instructions Executed'] or 0)
tot = sum(ie(d) for d in data)
tt = sum(te(d) for d in data)
print(f"warp inst {tot:.4g}  thread inst {tt:.4g}  lanes/inst {tt / tot:.2f}  sass {len(data)}")
b = collections.Counter()
for d in data:
    a = te(d) / ie(d) if ie(d) else 0
    b[int(a // 4) * 4] += ie(d)
print('  lanes:', ', '.join(f"{k}-{k + 3}: {100 * b[k] / tot:.1f}%" for k in sorted(b)))
segs, cur = [], None
for i, d in enumerate(data):
    e = ie(d)
    a = te(d) / e if e else 0
    if cur and abs(e - cur['e']) <= 0.02 * max(e, 1):
        cur['n'] += 1
        cur['end'] = i
        cur['t'] += te(d)
        cur['w'] += e
        ops = d['Source'].split()
        if ops:
            cur['ops'][ops[0].split('.')[0]] += e
    else:
        cur = {'start': i, 'end': i, 'e': e, 'n': 1, 't': te(d), 'w': e,
               'ops': collections.Counter(), 'first': d['Source'][:36]}
        segs.append(cur)
segs.sort(key=lambda s: -s['w'])
for s in segs[:top]:
    ops = ', '.join(f"{k}:{int(v / max(s['e'], 1))}" for k, v in s['ops'].most_common(5))
    print(f"{s['start']:5d}-{s['end']:5d} x{s['e']:.3g} n={s['n']:3d} share {100 * s['w'] / tot:4.1f}% "
          f"lanes {s['t'] / max(s['w'], 1):4.1f}  {ops}")
