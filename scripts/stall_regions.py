"""Stall samples per code region (runs of equal execution count) from an ncu
source-page csv.  usage: stall_regions.py src.csv [n_regions]"""
import csv, sys, collections
rows = list(csv.reader(open(sys.argv[1])))
hdr = rows[1]; idx = {h: i for i, h in enumerate(hdr)}
cols = ['stall_wait', 'stall_no_inst', 'stall_selected', 'stall_long_sb', 'stall_short_sb',
        'stall_math', 'stall_branch_resolving', 'stall_not_selected', 'stall_barrier', 'stall_dispatch']
ins = []
for r in rows[2:]:
    if len(r) < len(hdr): break
    ins.append((int(r[idx['Instructions Executed']] or 0), r[idx['Address']][-5:],
                [int(r[idx[c]] or 0) for c in cols], r[idx['Source']].strip()))
runs = []
for n, a, st, src in ins:
    if runs and runs[-1][0] == n:
        runs[-1][2].append(st)
    else:
        runs.append([n, a, [st]])
tot = [sum(i[2][k] for i in ins) for k in range(len(cols))]
T = sum(tot)
print('total samples', T, ' '.join(f'{c[6:]}={t/T*100:.0f}%' for c, t in zip(cols, tot)))
agg = []
for n, a, sts in runs:
    s = [sum(x[k] for x in sts) for k in range(len(cols))]
    agg.append((sum(s), n, a, len(sts), s))
agg.sort(key=lambda x: -x[0])
for S, n, a, ln, s in agg[:int(sys.argv[2]) if len(sys.argv) > 2 else 25]:
    print(f'{a} cnt={n:6d} len={ln:4d} samples={S/T*100:5.1f}%  ' +
          ' '.join(f'{c[6:]}={v/S*100:.0f}' for c, v in zip(cols, s) if v > 0.05 * S))
