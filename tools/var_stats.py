"""Per-variant stats + time (dev aid): python tools/var_stats.py C1 C3 -- v1 v2 ..."""
import os, subprocess, sys
args = sys.argv[1:]
cut = args.index('--')
cfgs, vars_ = args[:cut], args[cut + 1:]
CODE = r'''
import sys, torch
sys.path.insert(0, '.')
import kcgen, paper_conf_icde_ahmady0gcz23_b200 as kc
for name in %r:
    r, c = kcgen.generate_device(kcgen.CONFIGS[name])
    for _ in range(3): core, st = kc.kcore_decompose(r, c, stats=True)
    print(name, round(st.kernel_ms, 3), 'phases', st.phases, 'levels', st.levels, 'arcs', st.arcs_walked, 'hub', st.hub_arcs, 'scanned', st.scanned, 'compact', st.compactions, 'near', st.near_scans, flush=True)
''' % (cfgs,)
for v in vars_:
    env = dict(os.environ, KCORE_LIB=os.path.abspath(f'paper_conf_icde_ahmady0gcz23_b200/lib/variants/{v}.so'))
    p = subprocess.run([sys.executable, '-c', CODE], env=env, capture_output=True, text=True, timeout=300)
    print('==', v); print(p.stdout.strip() or p.stderr[-500:], flush=True)
