"""Run a KC_PROBE variant once on a config and dump probe records (dev aid).
   KCORE_LIB=.../variants/probe.so python tools/probe_run.py C4"""
import ctypes, os, sys
import numpy as np
import torch
sys.path.insert(0, '.')
import kcgen
import paper_conf_icde_ahmady0gcz23_b200 as kc
name = sys.argv[1]
r, c = kcgen.generate_device(kcgen.CONFIGS[name])
lib = ctypes.CDLL(os.environ['KCORE_LIB'])
lib.kcore_probe_read.restype = ctypes.c_int64
buf = np.zeros((1 << 22, 4), np.int64)
tr = torch.zeros((20000, 8), dtype=torch.int64, device='cuda')
for it in range(2):
    lib.kcore_probe_read(buf.ctypes.data_as(ctypes.c_void_p), ctypes.c_int64(1 << 22))
    core, st = kc.kcore_decompose(r, c, trace=tr, stats=True)
    torch.cuda.synchronize()
n = lib.kcore_probe_read(buf.ctypes.data_as(ctypes.c_void_p), ctypes.c_int64(1 << 22))
P = buf[:n][buf[:n, 1] != 0].copy()
P[:, 2] -= P[:, 2].min()
np.savez_compressed(f'gpurun_out/probe_{name}.npz', p=P.astype(np.int32))
np.save(f'gpurun_out/probe_tr_{name}.npy', tr[:st.trace_len].cpu().numpy())
print(name, n, st)
