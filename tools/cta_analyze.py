"""Analyse tools/cta_trace.py dumps (runs on the CPU box)."""
import sys
import numpy as np
tag, name = sys.argv[1], sys.argv[2]
T = np.load(f'gpurun_out/tr_{tag}_{name}.npy')
C = np.load(f'gpurun_out/tc_{tag}_{name}.npy')
PH = {1: 'level', 2: 'hub'}
rows = []
for i in range(len(T)):
    code = T[i, 2]; ph = code >> 8; solo = (code >> 4) & 1
    if solo: continue
    b = T[i, 7]
    c = C[b]  # [148,4]
    if c[:, 0].min() == 0: continue
    t0min = c[:, 0].min(); t0max = c[:, 0].max()
    scan = c[:, 1] - c[:, 0]; drain = c[:, 2] - c[:, 1]; tail = c[:, 3] - c[:, 2]
    arrive_max = c[:, 3].max()
    rel = C[b + 1][:, 0].min() if b + 1 < len(C) and C[b + 1][:, 0].min() > 0 else 0
    rows.append((i, PH.get(int(ph), '?'), T[i, 3], T[i, 4], T[i, 5], (t0max - t0min) / 1e3, np.median(scan) / 1e3, scan.max() / 1e3,
                 np.median(drain) / 1e3, drain.max() / 1e3, tail.max() / 1e3, (arrive_max - t0min) / 1e3, (rel - arrive_max) / 1e3 if rel else -1))
R = np.array([r[2:] for r in rows], dtype=float)
print(f"{len(rows)} grid phases")
hdr = "k size arcs startspread scan_med scan_max drain_med drain_max tail_max phase_span release_lat".split()
print("medians:", {h: round(float(np.median(R[:, j])), 2) for j, h in enumerate(hdr)})
print("sums   :", {h: round(float(np.sum(R[:, j])), 1) for j, h in enumerate(hdr) if j >= 3})
for ph in ('level', 'hub'):
    sel = [j for j, r in enumerate(rows) if r[1] == ph]
    if not sel: continue
    S = R[sel]
    print(ph, len(sel), "median:", {h: round(float(np.median(S[:, j])), 2) for j, h in enumerate(hdr) if j >= 3})
order = np.argsort(-R[:, 9])[:15]
for j in order:
    r = rows[j]
    print(f"  rec {r[0]} {r[1]} k={r[2]} size={r[3]} arcs={r[4]} start_spread={r[5]:.1f} scan med/max={r[6]:.1f}/{r[7]:.1f} drain med/max={r[8]:.1f}/{r[9]:.1f} tail={r[10]:.1f} span={r[11]:.1f} rel={r[12]:.1f}")
