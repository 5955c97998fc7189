"""Save per-phase traces of configs to gpurun_out/ (development aid)."""
import sys, os
import numpy as np
import torch
sys.path.insert(0, '.')
import kcgen
import paper_conf_icde_ahmady0gcz23_b200 as kc
os.makedirs('gpurun_out', exist_ok=True)
tag = sys.argv[1]
for name in sys.argv[2:]:
    r, c = kcgen.generate_device(kcgen.CONFIGS[name])
    tr = torch.zeros((400000, 8), dtype=torch.int64, device='cuda')
    for _ in range(2):
        core, st = kc.kcore_decompose(r, c, trace=tr, stats=True)
    np.save(f'gpurun_out/trace_{tag}_{name}.npy', tr[:st.trace_len].cpu().numpy())
    print(name, st)
    del r, c; torch.cuda.empty_cache()
