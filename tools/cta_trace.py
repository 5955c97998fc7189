"""Dump per-phase and per-CTA traces for configs into gpurun_out/ (dev aid)."""
import sys, os
# the trace needs the trace build of the library (make builds lib/libkcore_trace.so)
os.environ.setdefault("KCORE_LIB", os.path.join(os.path.dirname(os.path.dirname(os.path.abspath(__file__))),
                                                "paper_conf_icde_ahmady0gcz23_b200", "lib", "libkcore_trace.so"))
import numpy as np
import torch
sys.path.insert(0, '.')
import kcgen
import paper_conf_icde_ahmady0gcz23_b200 as kc
os.makedirs('gpurun_out', exist_ok=True)
tag = sys.argv[1]
for name in sys.argv[2:]:
    r, c = kcgen.generate_device(kcgen.CONFIGS[name])
    cap = 20000
    tr = torch.zeros((cap, 8), dtype=torch.int64, device='cuda')
    tc = torch.zeros((cap, 148, 8), dtype=torch.int64, device='cuda')
    for _ in range(2):
        tc.zero_()
        core, st = kc.kcore_decompose(r, c, trace=tr, trace_cta=tc, stats=True)
    nb = st.barriers + 2
    np.save(f'gpurun_out/tr_{tag}_{name}.npy', tr[:st.trace_len].cpu().numpy())
    np.save(f'gpurun_out/tc_{tag}_{name}.npy', tc[:nb].cpu().numpy())
    print(name, st)
    del r, c; torch.cuda.empty_cache()
