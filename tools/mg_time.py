"""Virtual-rank multi-GPU timing (dev aid): python tools/mg_time.py C1 C3 C4 [--P 1,2,4,8] [--algo 0]
Kernel time (stats.kernel_ms, median of 5) of the device-initiated protocol
with P virtual ranks vs the single-GPU kcore_decompose on the same graph."""
import argparse
import json
import statistics
import sys

import torch

sys.path.insert(0, '.')
import kcgen  # noqa: E402
import paper_conf_icde_ahmady0gcz23_b200 as kc  # noqa: E402

ap = argparse.ArgumentParser()
ap.add_argument("cfgs", nargs="+")
ap.add_argument("--P", default="1,2,4,8")
ap.add_argument("--algo", type=int, default=0)
a = ap.parse_args()
flush = torch.empty(512 << 20, dtype=torch.uint8, device='cuda')
out = {}
for name in a.cfgs:
    r, c = kcgen.generate_device(kcgen.CONFIGS[name])
    ref, st1 = kc.kcore_decompose(r, c, stats=True)
    single = []
    for _ in range(5):
        flush.fill_(1)
        single.append(kc.kcore_decompose(r, c, stats=True)[1].kernel_ms)
    res = {"single_ms": statistics.median(single)}
    for P in map(int, a.P.split(",")):
        ms, st = [], None
        for rep in range(6):
            flush.fill_(1)
            e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            e0.record()
            got, st = kc.kcore_decompose_mg_virtual(r, c, P, stats=True, algo=a.algo)
            e1.record()
            torch.cuda.synchronize()
            if rep == 0:
                assert torch.equal(got, ref), (name, P)
                continue
            # device protocol: the kernel's own events; host-driven: the whole call (it syncs per sub-round)
            ms.append(st.kernel_ms if a.algo == 0 else e0.elapsed_time(e1))
        res[f"P{P}"] = {"ms": statistics.median(ms), "subrounds": st.phases, "barriers": st.barriers,
                        "levels": st.levels, "near_scans": st.near_scans}
        print(name, P, res[f"P{P}"], "single", res["single_ms"], flush=True)
    out[name] = res
    del r, c, ref
    torch.cuda.empty_cache()
print(json.dumps(out))
