"""A/B of the persisting L2 window in fresh processes, in a given order (dev aid):
   python tools/ab_persist.py C4 off on off on"""
import subprocess, sys
CODE = r'''
import sys, torch
sys.path.insert(0, '.')
import kcgen, paper_conf_icde_ahmady0gcz23_b200 as kc
from cuda.bindings import runtime as rt
r, c = kcgen.generate_device(kcgen.CONFIGS[%r])
ws = torch.empty(kc.kcore_workspace_size(r.numel() - 1, c.numel()), dtype=torch.uint8, device='cuda')
flush = torch.empty(512 << 20, dtype=torch.uint8, device='cuda')
lim0 = rt.cudaDeviceGetLimit(rt.cudaLimit.cudaLimitPersistingL2CacheSize)[1]
ms = []
for i in range(7):
    flush.fill_(1)
    ms.append(kc.kcore_decompose(r, c, workspace=ws, stats=True, l2_persist=%r)[1].kernel_ms)
lim1 = rt.cudaDeviceGetLimit(rt.cudaLimit.cudaLimitPersistingL2CacheSize)[1]
print(f"persist=%r limit_before={lim0} limit_after={lim1} ms={sorted(ms)[3]:.3f}")
'''
name = sys.argv[1]
for arg in sys.argv[2:]:
    on = arg == "on"
    p = subprocess.run([sys.executable, "-c", CODE % (name, on, on)], capture_output=True, text=True)
    print(p.stdout.strip() or p.stderr[-300:], flush=True)
