"""Write profiles/ncu_traffic_C4.json (bench.py's roofline.traffic source) from
an ncu --set full capture and a window-off metrics CSV of the SAME library
binary: python tools/traffic_json.py DIR  (DIR holds prof_C4.ncu-rep,
ncu_window_off.csv, sass_sha.txt as written by tools/gpu/final.sh)."""
import csv
import io
import json
import os
import subprocess
import sys

d = sys.argv[1]
raw = subprocess.run(["ncu", "-i", os.path.join(d, "prof_C4.ncu-rep"), "--page", "raw", "--csv"],
                     capture_output=True, text=True).stdout
rows = list(csv.reader(io.StringIO(raw)))
h, u, v = rows[0], rows[1], rows[2]
m = dict(zip(h, zip(v, u)))


def val(k):
    x, unit = m[k]
    x = float(x.replace(",", ""))
    return x * {"Gbyte": 1e9, "Mbyte": 1e6, "Kbyte": 1e3, "byte": 1, "Tbyte": 1e12}.get(unit, 1)


off = {}
for line in open(os.path.join(d, "ncu_window_off.csv")):
    if not line.startswith('"0"'):
        continue
    f = next(csv.reader([line]))
    off[f[-3]] = float(f[-1])
sha = open(os.path.join(d, "sass_sha.txt")).read().split()[0]
out = {
    "sass_sha256": sha,
    "kernel": "k_persistent(KArgs)", "config": "C4 rmat-s24-ef32",
    "dram_bytes_per_launch": val("dram__bytes_read.sum") + val("dram__bytes_write.sum"),
    "dram_bytes_read": val("dram__bytes_read.sum"), "dram_bytes_write": val("dram__bytes_write.sum"),
    "dram_bytes_per_launch_window_off": off.get("dram__bytes_read.sum", 0) + off.get("dram__bytes_write.sum", 0),
    "lts_sectors_atom": off.get("lts__t_sectors_srcunit_tex_op_atom.sum"),
    "lts_sectors_red": off.get("lts__t_sectors_srcunit_tex_op_red.sum"),
    "note": "ncu --set full of the benchmarked library binary (persisting L2 window on); the window-off "
            "capture is the better upper estimate for the benchmarked kernel (the window adds profiler-side "
            "write-backs, profiles/ncu_l2split_r1_C4.json)",
}
json.dump(out, open(os.path.join(os.path.dirname(os.path.dirname(os.path.abspath(__file__))), "profiles",
                                 "ncu_traffic_C4.json"), "w"), indent=1)
print(json.dumps(out, indent=1))
