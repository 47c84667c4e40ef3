"""Group executed SASS (ncu source page csv) into runs of equal execution count
and print the heaviest runs with an opcode summary."""
import csv, sys, collections
rows = list(csv.reader(open(sys.argv[1])))
norm = float(sys.argv[2]) if len(sys.argv) > 2 else 1.0
hdr = rows[1]; idx = {h: i for i, h in enumerate(hdr)}
ins = []
for r in rows[2:]:
    if len(r) < len(hdr): break
    ins.append((int(r[idx['Instructions Executed']] or 0), r[idx['Address']][-5:], r[idx['Source']].strip()))
runs = []
cur = None
for n, a, s in ins:
    if cur and cur[0] == n:
        cur[2].append(s)
    else:
        cur = [n, a, [s]]
        runs.append(cur)
tot = sum(n for n, _, _ in ins)
runs.sort(key=lambda r: -r[0] * len(r[2]))
acc = 0
for n, a, ss in runs[:40]:
    w = n * len(ss)
    acc += w
    ops = collections.Counter((s.split()[1] if s.startswith('@') else s.split()[0]).split('.')[0] for s in ss)
    print(f"{a} cnt={n:6d} len={len(ss):4d} per-norm={w/norm:7.1f} cum%={100*acc/tot:5.1f}  " + " ".join(f"{k}:{v}" for k, v in ops.most_common(8)))
