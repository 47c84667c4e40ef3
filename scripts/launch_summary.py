"""Per-kernel totals of an `ncu --metrics gpu__time_duration.sum --csv` launch list.
usage: launch_summary.py launches.csv > summary.txt"""
import collections, csv, sys
rows = [r for r in csv.reader(open(sys.argv[1])) if len(r) > 10]
hdr = rows[0]
idx = {h: i for i, h in enumerate(hdr)}
tot, cnt = collections.Counter(), collections.Counter()
scale = {"nsecond": 1e-3, "ns": 1e-3, "usecond": 1.0, "us": 1.0, "msecond": 1e3, "ms": 1e3, "second": 1e6}
for r in rows[1:]:
    if r[idx["Metric Name"]] != "gpu__time_duration.sum":
        continue
    k = r[idx["Kernel Name"]].split("(")[0][:70]
    tot[k] += float(r[idx["Metric Value"]].replace(",", "")) * scale.get(r[idx["Metric Unit"]], 1.0)
    cnt[k] += 1
T = sum(tot.values())
print(f"{'total us':>12} {'share':>6} {'launches':>8} {'avg us':>9}  kernel")
for k, v in tot.most_common():
    print(f"{v:12.1f} {100 * v / T:5.1f}% {cnt[k]:8d} {v / cnt[k]:9.2f}  {k}")
