"""Per-arc primitive costs on the real C4 CSR (dev aid; see tools/ubench_arcs.cu).
python tools/ubench_arcs.py [C4]"""
import ctypes
import os
import subprocess
import sys

import torch

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import kcgen  # noqa: E402

so = os.path.join(ROOT, "tools/libubench_arcs.so")
if not os.path.exists(so):
    subprocess.check_call(["nvcc", "-gencode", "arch=compute_100a,code=sm_100a", "-O3", "-shared", "-Xcompiler",
                           "-fPIC", os.path.join(ROOT, "tools/ubench_arcs.cu"), "-o", so])
lib = ctypes.CDLL(so)
lib.ubench_arcs.restype = ctypes.c_float
lib.ubench_arcs.argtypes = [ctypes.c_int, ctypes.c_void_p, ctypes.c_int64, ctypes.c_void_p, ctypes.c_void_p,
                            ctypes.c_uint32, ctypes.c_int, ctypes.c_int]
cfg = sys.argv[1] if len(sys.argv) > 1 else "C4"
rp, ci = kcgen.generate_device(kcgen.CONFIGS[cfg])
n = rp.numel() - 1
m = ci.numel()
deg = (rp[1:] - rp[:-1]).to(torch.int32) + (1 << 20)
bits = torch.zeros((n + 31) // 32, dtype=torch.int32, device="cuda")
# half the vertices claimed (random bit pattern) for the filter modes
bits_half = torch.randint(-(1 << 31), (1 << 31) - 1, ((n + 31) // 32,), dtype=torch.int32, device="cuda")
names = {0: "read colidx", 1: "RED deg[u]", 2: "ATOM deg[u] (ret)", 3: "LDG deg[u]",
         4: "LDG bits + RED (half set)", 5: "LDG bits + ATOM (half set)", 6: "LDS 64KB probe"}
for mode in range(7):
    for bps, thr in ((1, 512), (2, 512), (4, 256), (4, 512)):
        b = bits_half if mode in (4, 5) else bits
        ms = lib.ubench_arcs(mode, ci.data_ptr(), m, deg.data_ptr(), b.data_ptr(), 0, bps, thr)
        print(f"{names[mode]:28s} grid={bps}x{thr:4d}: {ms:8.3f} ms  {m / ms / 1e6:7.1f} G arcs/s", flush=True)
for mode in (7, 8):
    for ws in (1 << 14, 1 << 18, 1 << 20, 1 << 22, 1 << 24):
        ms = lib.ubench_arcs(mode, ci.data_ptr(), m, deg.data_ptr(), bits.data_ptr(), ws - 1, 4, 512)
        print(f"{'RED' if mode == 7 else 'ATOM'} on u&mask ws={ws * 4 >> 10:6d} KB: {ms:8.3f} ms  {m / ms / 1e6:7.1f} G/s",
              flush=True)
