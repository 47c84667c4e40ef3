"""Summarise an ncu --set full report of the decode-attention kernel into
profiles/ncu_<config>.json (+ a markdown block), and a launch-list csv into
per-kernel shares.  usage: ncu_to_profile.py CONFIG TAG"""
import csv, io, json, os, subprocess, sys, collections
cfg, tag = sys.argv[1], sys.argv[2]
root = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
rep = os.path.join(root, "gpurun_out", f"prof_{cfg}_{tag}.ncu-rep")
raw = subprocess.run(["ncu", "-i", rep, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
rows = list(csv.reader(io.StringIO(raw)))
hdr, units, vals = rows[0], rows[1], rows[2]
d = dict(zip(hdr, vals)); u = dict(zip(hdr, units))
def num(k):
    try: return float(d[k].replace(",", ""))
    except Exception: return None
def mb(k):
    v = num(k)
    if v is None: return None
    scale = {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9}.get(u.get(k, "byte"), 1)
    return v * scale
def us(k):
    v = num(k)
    scale = {"nsecond": 1e-3, "usecond": 1.0, "msecond": 1e3}.get(u.get(k, "usecond"), 1.0)
    return v * scale
out = {
    "config": cfg, "tag": tag, "kernel": d.get("Kernel Name", ""),
    "duration_us_ncu": us("gpu__time_duration.sum"),
    "dram_bytes_read": mb("dram__bytes_read.sum"), "dram_bytes_write": mb("dram__bytes_write.sum"),
    "dram_throughput_pct": num("gpu__dram_throughput.avg.pct_of_peak_sustained_elapsed"),
    "sm_throughput_pct": num("sm__throughput.avg.pct_of_peak_sustained_elapsed"),
    "issue_active_pct": num("smsp__issue_active.avg.pct_of_peak_sustained_active"),
    "tensor_pipe_pct": num("sm__pipe_tensor_cycles_active.avg.pct_of_peak_sustained_active"),
    "warps_active_pct": num("sm__warps_active.avg.pct_of_peak_sustained_active"),
    "registers": num("launch__registers_per_thread"), "grid": num("launch__grid_size"),
    "inst_executed": num("smsp__inst_executed.sum"),
    "l2_hit_pct": num("lts__t_sector_hit_rate.pct"),
}
out["dram_bytes_per_launch"] = (out["dram_bytes_read"] or 0) + (out["dram_bytes_write"] or 0)
st = {k.replace("smsp__average_warps_issue_stalled_", "").replace("_per_issue_active.ratio", ""): float(v)
      for k, v in d.items() if "average_warps_issue_stalled" in k and "per_issue_active" in k and v}
out["stalls_per_issue"] = dict(sorted(st.items(), key=lambda x: -x[1])[:10])
lpath = os.path.join(root, "gpurun_out", f"launches_{cfg}_{tag}.csv")
if os.path.exists(lpath):
    lrows = list(csv.reader(open(lpath)))
    h = None; agg = collections.defaultdict(list)
    for r in lrows:
        if "Kernel Name" in r: h = r; continue
        if h and len(r) == len(h):
            x = dict(zip(h, r))
            if x.get("Metric Name") == "gpu__time_duration.sum":
                agg[x["Kernel Name"].split("(")[0]].append(float(x["Metric Value"]) / 1e3)
    out["launch_list_us"] = {k: {"n": len(v), "min": min(v), "median": sorted(v)[len(v) // 2]} for k, v in agg.items()}
os.makedirs(os.path.join(root, "profiles"), exist_ok=True)
json.dump(out, open(os.path.join(root, "profiles", f"ncu_{cfg}.json"), "w"), indent=1)
print(json.dumps(out, indent=1))
