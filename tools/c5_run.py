"""C5 (R-MAT s27 ef32, BASELINE.json configs[4]) on ONE B200: chunked device
generation, decomposition timing (L2 flushed, median of K), parity against the
serial oracle on the host (needs ~45 GB RAM) and the I2+I4 certificate of the
device's own peel order.  Writes gpurun_out/c5.json.
    python tools/c5_run.py [--steps 5] [--no-oracle]"""
import argparse
import json
import os
import statistics
import sys
import time

import torch

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import kcgen  # noqa: E402
import paper_conf_icde_ahmady0gcz23_b200 as kc  # noqa: E402

ap = argparse.ArgumentParser()
ap.add_argument("--steps", type=int, default=5)
ap.add_argument("--no-oracle", action="store_true")
a = ap.parse_args()
t0 = time.time()
r, c = kcgen.generate_device_chunked(kcgen.CONFIGS["C5"], chunks=16)
n, m = r.numel() - 1, c.numel()
tgen = time.time() - t0
print(f"C5 generated: n={n} arcs={m} in {tgen:.1f}s; mem {torch.cuda.memory_allocated() / 2**30:.1f} GiB", flush=True)
ws = torch.empty(kc.kcore_workspace_size(n, m), dtype=torch.uint8, device="cuda")
core = torch.empty(n, dtype=torch.int32, device="cuda")
order = torch.empty(n, dtype=torch.int32, device="cuda")
flush = torch.empty(512 << 20, dtype=torch.uint8, device="cuda")
torch.cuda.reset_peak_memory_stats()
kc.kcore_decompose(r, c, core_out=core, workspace=ws)
ks, st = [], None
for _ in range(a.steps):
    flush.fill_(1)
    _, st = kc.kcore_decompose(r, c, core_out=core, workspace=ws, stats=True)
    ks.append(st.kernel_ms)
med = statistics.median(ks)
b_min = 4 * m + 8 * (n + 1) + 8 * n + 4 * n + 4 * st.scanned + 8 * n
peak = json.load(open(os.path.join(ROOT, "MEASURED_PEAKS.json")))["hbm_gbs"] if os.path.exists(
    os.path.join(ROOT, "MEASURED_PEAKS.json")) else 6528.4
out = {"config": "C5 rmat-s27-ef32", "n": n, "arcs": m, "m_undirected": m // 2, "gen_s": tgen,
       "kernel_ms_median": med, "kernel_ms_min": min(ks), "kernel_ms_all": ks,
       "medges_per_s": m / 2 / (med * 1e-3) / 1e6, "roofline_frac": b_min / (med * 1e-3) / 1e9 / peak,
       "algorithmic_bytes": b_min, "levels": st.levels, "phases": st.phases, "kmax": st.kmax,
       "scanned": st.scanned, "arcs_walked": st.arcs_walked,
       "device_bytes_csr": 8 * (n + 1) + 4 * m, "device_bytes_workspace": ws.numel(),
       "device_peak_allocated": torch.cuda.max_memory_allocated()}
print(json.dumps(out), flush=True)
kc.kcore_decompose(r, c, core_out=core, order_out=order, workspace=ws)
torch.cuda.synchronize()
if not a.no_oracle:
    import numpy as np
    import oracle
    t1 = time.time()
    rp_h = r.cpu().numpy()
    ci_h = c.cpu().numpy()
    got = core.cpu().numpy()
    ordh = order.cpu().numpy()
    del r, c, ws
    torch.cuda.empty_cache()
    t2 = time.time()
    ref = oracle.bz_core(rp_h, ci_h)
    t3 = time.time()
    out["oracle_s"] = t3 - t2
    out["parity"] = bool(np.array_equal(ref, got))
    out["mismatches"] = int((ref != got).sum())
    out["certificate_ok"] = oracle.check_certificate(rp_h, ci_h, got, ordh) == 0
    out["certificate_s"] = time.time() - t3
    out["d2h_s"] = t2 - t1
    print(json.dumps({k: out[k] for k in ("parity", "mismatches", "certificate_ok", "oracle_s", "certificate_s")}),
          flush=True)
os.makedirs(os.path.join(ROOT, "gpurun_out"), exist_ok=True)
json.dump(out, open(os.path.join(ROOT, "gpurun_out", "c5.json"), "w"), indent=1)
