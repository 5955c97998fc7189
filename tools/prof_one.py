"""One warm-up + one measured decomposition of a config (for ncu captures:
   ncu -k regex:k_persistent -s 1 -c 1 ... python tools/prof_one.py C4)."""
import sys
import torch
sys.path.insert(0, '.')
import kcgen
import paper_conf_icde_ahmady0gcz23_b200 as kc

name = sys.argv[1] if len(sys.argv) > 1 else "C4"
kw = {}
for a in sys.argv[2:]:
    k, v = a.split('=')
    kw[k] = int(v)
r, c = kcgen.generate_device(kcgen.CONFIGS[name])
ws = torch.empty(kc.kcore_workspace_size(r.numel() - 1, c.numel()), dtype=torch.uint8, device='cuda')
for _ in range(2):
    core, st = kc.kcore_decompose(r, c, workspace=ws, stats=True, **kw)
print(name, kw, st)
