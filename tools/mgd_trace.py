"""Phase timeline of the device-initiated multi-GPU protocol (dev aid):
python tools/mgd_trace.py C4 8"""
import ctypes
import sys

import numpy as np
import torch

sys.path.insert(0, '.')
import kcgen  # noqa: E402
import paper_conf_icde_ahmady0gcz23_b200 as kc  # noqa: E402

name, P = sys.argv[1], int(sys.argv[2])
r, c = kcgen.generate_device(kcgen.CONFIGS[name])
tr = torch.zeros((1 << 16, 8), dtype=torch.int64, device='cuda')
lib = kc.library()
lib.kcore_test_mgd_trace.argtypes = [ctypes.c_void_p, ctypes.c_int64]
kc.kcore_decompose_mg_virtual(r, c, P)
lib.kcore_test_mgd_trace(tr.data_ptr(), tr.shape[0])
core, st = kc.kcore_decompose_mg_virtual(r, c, P, stats=True)
lib.kcore_test_mgd_trace(None, 0)
T = tr[:st.barriers + 1].cpu().numpy()
dt = np.diff(T[:, 0]) / 1e3  # us, interval ending at record i+1
ph = T[1:, 1]
print(name, P, st)
for p, nm in ((1, "scan"), (2, "sub-round")):
    s = ph == p
    print(f"{nm:10s} n={s.sum():5d} total={dt[s].sum() / 1e3:8.2f} ms median={np.median(dt[s]):7.1f} us "
          f"p90={np.percentile(dt[s], 90):7.1f} us max={dt[s].max():8.1f}")
pk = (ph == 2) & (T[1:, 4] > 0)
st0 = T[:-1, 0][pk]  # previous barrier exit = peel start (block 0)
items = (T[1:, 4][pk] - st0) / 1e3
chunks = (T[1:, 5][pk] - T[1:, 4][pk]) / 1e3
fin = (T[1:, 6][pk] - T[1:, 5][pk]) / 1e3
bar = (T[1:, 0][pk] - T[1:, 6][pk]) / 1e3
wk = (T[1:, 7][pk] - st0) / 1e3
print(f"latest walking warp done after {np.median(wk):.1f} us (median)")
print(f"block 0 peel: items loop median {np.median(items):.1f} us, chunk loop {np.median(chunks):.1f}, "
      f"min/stats {np.median(fin):.1f}, barrier (to release) {np.median(bar):.1f}")
idx = np.argsort(-dt)[:12]
for i in idx:
    print(f"  phase {int(ph[i])} k={int(T[i + 1, 2])} {dt[i]:8.1f} us removed {int(T[i + 1, 3])}")
