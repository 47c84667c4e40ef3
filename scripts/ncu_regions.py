import csv, sys, collections
rows=list(csv.reader(open(sys.argv[1])))
hdr=rows[1]; ix={h:i for i,h in enumerate(hdr)}
data=[]
for r in rows[2:]:
    if len(r)<len(hdr): break
    data.append(r)
cols=['Warp Stall Sampling (All Samples)','stall_no_inst','stall_wait','stall_short_sb','stall_long_sb','stall_branch_resolving','stall_math','stall_selected','stall_not_selected','stall_barrier','stall_membar','stall_lg','stall_mio','stall_dispatch']
agg=collections.defaultdict(lambda: collections.Counter())
ninst=collections.Counter()
for r in data:
    n=int(r[ix['Instructions Executed']] or 0)
    key=n
    for c in cols: agg[key][c]+=int(r[ix[c]] or 0)
    ninst[key]+=1
tot=sum(a[cols[0]] for a in agg.values())
print('total samples',tot)
for k in sorted(agg, key=lambda k:-agg[k][cols[0]])[:14]:
    a=agg[k]
    print(f"exec={k:7d} ninstr={ninst[k]:5d} samples={a[cols[0]]:5d} ({100*a[cols[0]]/tot:4.1f}%) "+' '.join(f"{c.replace('stall_','')}={a[c]}" for c in cols[1:] if a[c]))
