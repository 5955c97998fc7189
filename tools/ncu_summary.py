"""Summarise a one-kernel ncu report into profiles/ (JSON).
   python tools/ncu_summary.py gpurun_out/prof.ncu-rep profiles/ncu_r1_C4 [launches.csv]"""
import csv, io, json, subprocess, sys

rep, out = sys.argv[1], sys.argv[2]
raw = subprocess.run(["ncu", "-i", rep, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
rows = list(csv.reader(io.StringIO(raw)))
h, units, vals = rows[0], rows[1], rows[2]
d = {h[i]: (vals[i], units[i]) for i in range(len(h))}
KNAME = d.get("Kernel Name", ("?", ""))[0]


def num(k):
    try:
        return float(d[k][0].replace(',', ''))
    except Exception:
        return None


def scaled(k):
    v = num(k)
    if v is None:
        return None
    u = d[k][1]
    mult = {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9, "Tbyte": 1e12, "nsecond": 1e-9,
            "usecond": 1e-6, "msecond": 1e-3, "second": 1, "ns": 1e-9, "us": 1e-6, "ms": 1e-3,
            "s": 1}.get(u, 1)
    return v * mult


keys = ["gpu__time_duration.sum", "dram__bytes_read.sum", "dram__bytes_write.sum", "lts__t_sector_hit_rate.pct",
        "sm__throughput.avg.pct_of_peak_sustained_elapsed", "gpu__dram_throughput.avg.pct_of_peak_sustained_elapsed",
        "l1tex__t_requests_pipe_lsu_mem_global_op_atom.sum", "l1tex__t_requests_pipe_lsu_mem_global_op_ld.sum",
        "lts__t_sectors_op_atom.sum", "lts__t_sectors_op_red.sum", "lts__t_sectors_op_read.sum",
        "sm__warps_active.avg.pct_of_peak_sustained_active", "launch__registers_per_thread",
        "launch__grid_size", "launch__block_size", "smsp__inst_executed.sum",
        "l1tex__t_sectors_pipe_lsu_mem_local_op_ld.sum"]
summary = {k: {"value": num(k), "unit": d[k][1]} for k in keys if k in d}
dur = scaled("gpu__time_duration.sum")
rd, wr = scaled("dram__bytes_read.sum"), scaled("dram__bytes_write.sum")
stalls = {k.replace("smsp__pcsamp_warps_issue_stalled_", ""): num(k) for k in d
          if k.startswith("smsp__pcsamp_warps_issue_stalled_") and not k.endswith("not_issued")}
tot = sum(v for v in stalls.values() if v) or 1
stalls = {k: round(100 * v / tot, 1) for k, v in sorted(stalls.items(), key=lambda x: -(x[1] or 0)) if v}
res = {"report": rep, "kernel": KNAME, "duration_s": dur, "dram_bytes_read": rd, "dram_bytes_write": wr,
       "dram_bytes_per_launch": (rd or 0) + (wr or 0),
       "dram_GBps": ((rd or 0) + (wr or 0)) / dur / 1e9 if dur else None,
       "stall_pct": dict(list(stalls.items())[:12]), "metrics": summary}
if len(sys.argv) > 3:
    launches = []
    with open(sys.argv[3]) as f:
        txt = f.read()
    i = txt.find('"ID"')
    for r in csv.DictReader(io.StringIO(txt[i:] if i >= 0 else txt)):
        if r.get("Metric Name") == "gpu__time_duration.sum":
            launches.append((r.get("Kernel Name", ""), float(r["Metric Value"].replace(',', '')), r.get("Metric Unit")))
    res["launches"] = launches
json.dump(res, open(out + ".json", "w"), indent=1)
print(json.dumps({k: v for k, v in res.items() if k not in ("metrics", "launches")}, indent=1))
