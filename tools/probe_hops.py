"""Per-hop latency breakdown of the CTA-local drain from a KC_PROBE/KC_PROBE_W
dump (tools/probe_run.py): python tools/probe_hops.py gpurun_out/probe_C3.npz
For every CTA: sub-round start (tag 1) -> prefix done (2) -> warp walk start
(10) -> batch data ready / before atomics (13) -> atomics returned (11) ->
claim+row bounds returned (14) -> hits routed (12) -> walk done (3)."""
import sys
import numpy as np

P = np.load(sys.argv[1])["p"].astype(np.int64)
names = {1: "subround_top", 2: "prefix_done", 10: "walk_start", 13: "pre_atomic", 11: "atomics_back",
         14: "claims_back", 12: "routed", 3: "walk_done", 30: "phase_start", 33: "bar_arrive", 34: "bar_released"}
deltas = {}
for cta in np.unique(P[:, 0]):
    Q = P[P[:, 0] == cta]
    Q = Q[np.argsort(Q[:, 2], kind="stable")]
    prev = None
    lastw = {}
    for cta_, tag, t, val in Q:
        if tag in (10, 13, 11, 14, 12):
            w = val & 0xff
            if w in lastw:
                pt, ptag = lastw[w]
                deltas.setdefault((ptag, tag), []).append(t - pt)
            lastw[w] = (t, tag)
            if tag == 10 and prev is not None and prev[1] == 2:
                deltas.setdefault((2, 10), []).append(t - prev[0])
        else:
            if prev is not None and tag in (1, 2, 3, 33, 34, 30):
                deltas.setdefault((prev[1], tag), []).append(t - prev[0])
            if tag == 3:
                for w, (pt, ptag) in lastw.items():
                    deltas.setdefault((ptag, 3), []).append(t - pt)
                lastw = {}
            prev = (t, tag)
rows = []
for (a, b), v in deltas.items():
    v = np.array(v)
    rows.append((len(v), a, b, np.median(v), np.percentile(v, 90), v.sum() / 1e6))
for n, a, b, med, p90, tot in sorted(rows, key=lambda r: -r[5])[:24]:
    print(f"{names.get(a, a):>14s} -> {names.get(b, b):<14s} n={n:8d} median={med:7.0f} ns p90={p90:7.0f} ns total={tot:8.2f} ms(sum over CTAs)")
