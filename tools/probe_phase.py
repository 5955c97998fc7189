"""Per-phase segments of the critical (last-arriving) CTA from a KC_PROBE dump:
phase start (30) -> scan done (40) -> drain done (41) -> flushed (42) ->
barrier arrival (33) -> ticket (35) -> released (34) -> snapshot read (36) ->
advance done (37) -> loop top (38) -> next phase start (30)."""
import sys
import numpy as np
P = np.load(sys.argv[1])["p"].astype(np.int64)
ph = {}
for cta in np.unique(P[:, 0]):
    Q = P[P[:, 0] == cta]
    Q = Q[np.argsort(Q[:, 2], kind="stable")]
    idx = -1
    for r in Q:
        if r[1] == 30:
            idx += 1
        ph.setdefault((idx, cta), []).append((int(r[1]), int(r[2])))
n = max(i for i, _ in ph) + 1
segs = {}
for i in range(n):
    best = None
    for cta in range(160):
        L = ph.get((i, cta))
        if not L:
            continue
        arr = [t for tag, t in L if tag == 33]
        if arr and (best is None or arr[0] > best[0]):
            best = (arr[0], cta)
    if not best:
        continue
    L = ph[(i, best[1])]
    nxt = ph.get((i + 1, best[1]))
    first = {}
    for tag, t in L:
        first.setdefault(tag, t)
    if nxt:
        first.setdefault(99, nxt[0][1])
    order = [30, 40, 41, 42, 33, 35, 34, 36, 37, 38, 99]
    have = [t for t in order if t in first]
    for a, b in zip(have, have[1:]):
        segs.setdefault((a, b), []).append(first[b] - first[a])
for (a, b), v in segs.items():
    v = np.array(v)
    print(f"{a:3d}->{b:3d}  n={len(v):5d}  median={np.median(v) / 1e3:7.2f} us  total={v.sum() / 1e6:7.2f} ms")
