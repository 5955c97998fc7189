"""Per-phase breakdown of a decomposition from tools/cta_trace.py dumps
(runs on the CPU box): python tools/phase_breakdown.py TAG C1 C3 C4 > out.json"""
import json, sys
import numpy as np

tag = sys.argv[1]
out = {}
for name in sys.argv[2:]:
    T = np.load(f'gpurun_out/tr_{tag}_{name}.npy')
    C = np.load(f'gpurun_out/tc_{tag}_{name}.npy')
    cats = {"level": [], "hub_light": [], "hub_heavy": []}
    rel = []
    for i in range(len(T)):
        b = T[i, 7]
        c = C[b]
        if c[:, 0].min() == 0:
            continue
        ph = int(T[i, 2] >> 8)
        span = (c[:, 3].max() - c[:, 0].min()) / 1e3
        scan = (c[:, 1] - c[:, 0]).max() / 1e3
        drain = (c[:, 2] - c[:, 1]).max() / 1e3
        if b + 1 < len(C) and C[b + 1][:, 0].min() > 0:
            rel.append((C[b + 1][:, 0].min() - c[:, 3].max()) / 1e3)
        key = "level" if ph == 1 else ("hub_heavy" if T[i, 5] > 5_000_000 else "hub_light")
        cats[key].append((span, scan, drain))
    res = {}
    for k, v in cats.items():
        a = np.array(v, dtype=float).reshape(-1, 3)
        res[k] = {"phases": int(len(a)), "ms": round(float(a[:, 0].sum()) / 1e3, 3),
                  "median_us": round(float(np.median(a[:, 0])), 2) if len(a) else 0,
                  "scan_or_walk_ms": round(float(a[:, 1].sum()) / 1e3, 3),
                  "local_drain_ms": round(float(a[:, 2].sum()) / 1e3, 3)}
    res["barrier_release_ms"] = round(float(np.sum(rel)) / 1e3, 3)
    res["barrier_release_median_us"] = round(float(np.median(rel)), 2) if rel else 0
    out[name] = res
print(json.dumps(out, indent=1))
