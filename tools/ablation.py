"""Ablation of the design choices on one B200 (the paper's
Table II / Table V analogues): each variant in a fresh process (the persisting
L2 set-aside is a device-wide limit), median of 5 calls after 2 warm-ups, on
C1..C4; plus the device memory each call needs (Table V analogue).
    python tools/ablation.py [C1 C2 ...] > gpurun_out/ablation.json"""
import json, os, subprocess, sys

VARIANTS = {
    "default": {},
    "no_l2_persist": {"l2_persist": False},
    "no_bloom": {"bloom": False},
    "hostloop_alg1": {"algo": 1},
    "solo_phases": {"solo_arcs": 16384, "solo_scan": 32768},
}
CODE = r'''
import sys, json, torch
sys.path.insert(0, '.')
import kcgen, paper_conf_icde_ahmady0gcz23_b200 as kc
kw = %r
out = {}
for name in %r:
    r, c = kcgen.generate_device(kcgen.CONFIGS[name])
    n, m = r.numel() - 1, c.numel()
    ws = torch.empty(kc.kcore_workspace_size(n, m), dtype=torch.uint8, device='cuda')
    ref = kc.kcore_decompose(r, c, workspace=ws)
    for _ in range(2): kc.kcore_decompose(r, c, workspace=ws, **kw)
    ms = []
    for _ in range(5):
        core, st = kc.kcore_decompose(r, c, workspace=ws, stats=True, **kw)
        ms.append(st.kernel_ms)
    ms.sort()
    out[name] = {"ms": round(ms[2], 3), "Medges_s": round(m / 2 / ms[2] / 1e3, 1), "phases": st.phases,
                 "levels": st.levels, "equal": bool(torch.equal(core, ref)),
                 "csr_bytes": 8 * (n + 1) + 4 * m, "workspace_bytes": ws.numel(), "core_bytes": 4 * n}
    del r, c, ws, ref, core; torch.cuda.empty_cache()
print(json.dumps(out))
'''
names = sys.argv[1:] or ["C1", "C2", "C3", "C4"]
res = {}
for tag, kw in VARIANTS.items():
    p = subprocess.run([sys.executable, "-c", CODE % (kw, names)], capture_output=True, text=True, timeout=900)
    try:
        res[tag] = json.loads(p.stdout.strip().splitlines()[-1])
    except Exception:
        res[tag] = {"error": (p.stderr or p.stdout)[-400:]}
    print(tag, json.dumps(res[tag]), file=sys.stderr, flush=True)
print(json.dumps(res, indent=1))
