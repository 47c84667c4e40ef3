"""Summarise an ncu report: key SOL metrics + warp stall breakdown."""
import csv, subprocess, sys, io
rep = sys.argv[1]
out = subprocess.run(["ncu", "-i", rep, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
rows = list(csv.reader(io.StringIO(out)))
hdr, units, vals = rows[0], rows[1], rows[2]
d = dict(zip(hdr, vals))
keys = ["gpu__time_duration.sum", "dram__bytes_read.sum", "dram__bytes_write.sum",
        "gpu__dram_throughput.avg.pct_of_peak_sustained_elapsed", "sm__throughput.avg.pct_of_peak_sustained_elapsed",
        "smsp__issue_active.avg.pct_of_peak_sustained_active", "sm__warps_active.avg.pct_of_peak_sustained_active",
        "smsp__inst_executed.sum", "launch__registers_per_thread", "launch__grid_size",
        "sm__pipe_tensor_cycles_active.avg.pct_of_peak_sustained_active",
        "sm__inst_executed_pipe_alu.avg.pct_of_peak_sustained_active",
        "sm__inst_executed_pipe_fma.avg.pct_of_peak_sustained_active",
        "l1tex__data_bank_conflicts_pipe_lsu_mem_shared.sum", "lts__t_sector_hit_rate.pct",
        "smsp__cycles_active.avg", "sm__cycles_elapsed.avg"]
for k in keys:
    if k in d: print(f"{k:70s} {d[k]} {units[hdr.index(k)]}")
st = [(k, float(v)) for k, v in d.items() if k.startswith("smsp__average_warp_latency_issue_stalled") and k.endswith(".ratio") and v not in ("", "n/a")]
if not st:
    st = [(k, float(v.replace(',',''))) for k, v in d.items() if "warps_issue_stalled" in k and k.endswith("per_warp_active.pct") and v not in ("", "n/a")]
st.sort(key=lambda x: -x[1])
print("-- stalls")
for k, v in st[:14]: print(f"  {k:90s} {v:.2f}")
