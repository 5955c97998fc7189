"""Async-drain hop breakdown from a KC_PROBE_W dump: tags 20 pop, 21 colidx ready,
22 atomics back, 14 claims+row bounds back, 23 routed (per warp)."""
import sys
import numpy as np
P = np.load(sys.argv[1])["p"].astype(np.int64)
names = {20: "pop", 21: "colidx", 22: "atomics", 14: "claims", 15: "r_removed", 16: "r_reserved", 17: "r_pushed", 23: "routed", 30: "phase", 33: "arrive"}
d = {}
for cta in np.unique(P[:, 0]):
    Q = P[P[:, 0] == cta]
    Q = Q[np.argsort(Q[:, 2], kind="stable")]
    last = {}
    for _, tag, t, val in Q:
        if tag not in names:
            continue
        w = val & 0xff if tag in (20, 21, 22, 14, 15, 16, 17, 23) else -1
        if tag in (30, 33):
            last = {}
            continue
        if w in last:
            pt, ptag = last[w]
            d.setdefault((ptag, tag), []).append(t - pt)
        last[w] = (t, tag)
for (a, b), v in sorted(d.items(), key=lambda x: -len(x[1])):
    v = np.array(v)
    print(f"{names[a]:>8s} -> {names[b]:<8s} n={len(v):7d} median={np.median(v):6.0f} ns  p90={np.percentile(v, 90):7.0f}")
