"""Per-level structure of the level-synchronous peel (analysis tool, CPU).

python tools/level_sim.py C4 [--out profiles/level_sim_C4.json]

Generates the config's CSR with kcgen (host generator, cached under /tmp),
runs tools/level_sim.c and prints how the arcs are distributed over levels
and how many walked arcs hit alive / same-level-claimed / dead targets.
"""
import argparse
import ctypes
import json
import os
import subprocess
import sys

import numpy as np

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import kcgen  # noqa: E402

FIELDS = ["k", "alive", "alive_arcs", "scan_frontier", "subrounds", "peeled", "arcs_walked",
          "arcs_useful", "arcs_claimed_same_level", "arcs_dead", "max_sub_frontier", "max_sub_arcs"]


def load_csr(cfg):
    cache = f"/tmp/kc_csr_{cfg}.npz"
    if os.path.exists(cache):
        z = np.load(cache)
        return z["rp"], z["ci"]
    rp, ci = kcgen.generate_host(kcgen.CONFIGS[cfg])
    np.savez(cache, rp=rp, ci=ci)
    return rp, ci


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("cfg")
    ap.add_argument("--out")
    a = ap.parse_args()
    so = "/tmp/level_sim.so"
    subprocess.check_call(["gcc", "-O2", "-shared", "-fPIC", os.path.join(ROOT, "tools/level_sim.c"), "-o", so])
    lib = ctypes.CDLL(so)
    lib.level_sim.restype = ctypes.c_int64
    rp, ci = load_csr(a.cfg)
    n = rp.size - 1
    cap = 1 << 16
    rec = np.zeros((cap, 12), dtype=np.int64)
    P = ctypes.c_void_p
    near = np.zeros((cap, 4), dtype=np.int64)
    nrec = lib.level_sim(P(rp.ctypes.data), P(ci.ctypes.data), ctypes.c_int64(n), P(rec.ctypes.data),
                         ctypes.c_int64(cap), P(near.ctypes.data))
    near = near[:nrec]
    rec = rec[:nrec]
    arcs = int(rp[-1])
    tot = rec.sum(axis=0)
    summ = {
        "cfg": a.cfg, "n": int(n), "arcs": arcs, "levels": int(nrec), "subrounds": int(tot[4]),
        "arcs_walked": int(tot[6]), "useful_frac": float(tot[7] / max(arcs, 1)),
        "same_level_frac": float(tot[8] / max(arcs, 1)), "dead_frac": float(tot[9] / max(arcs, 1)),
        "sigma_alive": int(tot[1]),
    }
    # where the arcs are: levels sorted by arcs walked
    order = np.argsort(-rec[:, 6])
    cum = np.cumsum(rec[order, 6]) / arcs
    summ["levels_for_50pct_arcs"] = int(np.searchsorted(cum, 0.5) + 1)
    summ["levels_for_90pct_arcs"] = int(np.searchsorted(cum, 0.9) + 1)
    # tail: levels whose alive set is below thresholds
    for th in (1 << 14, 1 << 16, 1 << 18, 1 << 20):
        sel = rec[:, 1] <= th
        summ[f"tail_alive_le_{th}"] = {"levels": int(sel.sum()), "subrounds": int(rec[sel, 4].sum()),
                                        "arcs_walked": int(rec[sel, 6].sum()),
                                        "first_alive_arcs": int(rec[sel, 2][0]) if sel.any() else 0}
    light = rec[:, 6] < 1 << 20
    summ["light_levels_lt_1M_arcs"] = {"levels": int(light.sum()), "subrounds": int(rec[light, 4].sum()),
                                       "arcs": int(rec[light, 6].sum())}
    top = [dict(zip(FIELDS, map(int, rec[i]))) for i in order[:12]]
    print(json.dumps(summ, indent=1))
    print("top levels by arcs:")
    for t in top:
        print(t)
    if a.out:
        with open(a.out, "w") as f:
            json.dump({"summary": summ, "fields": FIELDS, "levels": rec.tolist(), "near": near.tolist(),
                       "near_fields": ["le_k+8", "le_k+32", "le_k+128", "le_2k+2"]}, f)


if __name__ == "__main__":
    main()
