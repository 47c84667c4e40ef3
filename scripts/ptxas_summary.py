"""Summarise `nvcc -Xptxas -v` output (build.log): registers / spills per kernel."""
import re
import subprocess
import sys

log = open(sys.argv[1] if len(sys.argv) > 1 else "paper_conf_ipps_wurypgll25_b200/build.log").read()
cur = None
rows = []
spill = ""
for line in log.splitlines():
    m = re.search(r"Function properties for (\S+)", line)
    if m:
        cur = m.group(1)
        continue
    m = re.search(r"(\d+) bytes spill stores, (\d+) bytes spill loads", line)
    if m:
        spill = f"spill st/ld {m.group(1)}/{m.group(2)}"
        continue
    m = re.search(r"Used (\d+) registers", line)
    if m and cur:
        rows.append((cur, int(m.group(1)), spill))
        cur, spill = None, ""
names = subprocess.run(["c++filt"], input="\n".join(r[0] for r in rows), capture_output=True, text=True).stdout.split("\n")
for (raw, regs, sp), name in zip(rows, names):
    if len(sys.argv) > 2 and sys.argv[2] not in name:
        continue
    print(f"{regs:4d}  {sp:24s} {name[:150]}")
