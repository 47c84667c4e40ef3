import csv, sys, collections
path = sys.argv[1]; nblk = float(sys.argv[2]) if len(sys.argv) > 2 else 1.0
rows = list(csv.reader(open(path)))
hdr = rows[1]; idx = {h: i for i, h in enumerate(hdr)}
data = []
for r in rows[2:]:
    if len(r) < len(hdr): break          # second kernel section starts
    data.append(r)
print(len(data), 'sass instrs in first kernel')
tot = 0; byop = collections.Counter(); stall = collections.Counter(); stt = 0
for r in data:
    n = int(r[idx['Instructions Executed']] or 0)
    s = int(r[idx['Warp Stall Sampling (All Samples)']] or 0)
    src = r[idx['Source']].strip().split()
    if not src: continue
    op = src[1] if src[0].startswith('@') else src[0]
    op = op.split('.')[0]
    byop[op] += n; tot += n; stall[op] += s; stt += s
print('total executed', tot, 'per blk', tot / nblk)
for op, n in byop.most_common(45):
    print(f'{op:12s} {n:10d} {n/nblk:7.1f}/blk  stall% {100*stall[op]/max(stt,1):5.1f}')
