"""Time every library variant in paper_conf_icde_ahmady0gcz23_b200/lib/variants on C1..C4
(one subprocess per variant; development aid)."""
import glob, json, os, subprocess, sys
VAR = sorted(glob.glob('paper_conf_icde_ahmady0gcz23_b200/lib/variants/*.so'))
names = [a for a in sys.argv[1:] if not a.startswith("--kw=")] or ["C1", "C2", "C3", "C4"]
KWS = [eval(a[5:]) for a in sys.argv[1:] if a.startswith("--kw=")] or [{}]
CODE = r'''
import sys, json, torch
sys.path.insert(0, '.')
import kcgen, paper_conf_icde_ahmady0gcz23_b200 as kc
out = {}
for name in %r:
    r, c = kcgen.generate_device(kcgen.CONFIGS[name])
    ws = torch.empty(kc.kcore_workspace_size(r.numel()-1, c.numel()), dtype=torch.uint8, device='cuda')
    flush = torch.empty(512 << 20, dtype=torch.uint8, device='cuda')
    for kw in %r:
        for _ in range(2): kc.kcore_decompose(r, c, workspace=ws, stats=True, **kw)
        ms = sorted((flush.fill_(1), kc.kcore_decompose(r, c, workspace=ws, stats=True, **kw))[1][1].kernel_ms
                    for _ in range(5))
        out[name + (str(kw) if kw else '')] = round(ms[2], 3)
    del r, c; torch.cuda.empty_cache()
print(json.dumps(out))
''' % (names, KWS)
for v in VAR:
    env = dict(os.environ, KCORE_LIB=os.path.abspath(v))
    p = subprocess.run([sys.executable, "-c", CODE], env=env, capture_output=True, text=True, timeout=240)
    res = p.stdout.strip().splitlines()[-1] if p.stdout.strip() else p.stderr[-300:]
    print(f"{os.path.basename(v):12s} {res}", flush=True)
