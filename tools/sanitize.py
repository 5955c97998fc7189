"""Workload for compute-sanitizer runs (memcheck / racecheck / synccheck /
initcheck): small graphs that drive every drain mode of the peel kernel --
the synchronous CTA-local sub-rounds, the asynchronous chunk queue (hub rows
>= 64 arcs per frontier vertex), HUB phases over the global queue, the Bloom
filter, compaction, many levels -- plus the host-loop ablation, MPM, the
outputs and the virtual-rank multi-GPU protocol.  Each result is checked
against the oracle, so a run that sanitises clean is also correct.

    compute-sanitizer --tool racecheck python tools/sanitize.py
"""
import os
import sys

import numpy as np
import torch

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import kcgen  # noqa: E402
import oracle  # noqa: E402
import paper_conf_icde_ahmady0gcz23_b200 as kc  # noqa: E402


def graphs():
    e = []
    t = 2000
    for i in range(t):  # bowtie fan: hub + t triangles (Fig. 6 generalised)
        a, b = 1 + 2 * i, 2 + 2 * i
        e += [(0, a), (0, b), (a, b)]
    yield "bowtie_fan_2000", kcgen.csr_from_edges(2 * t + 1, e)
    yield "path_2000", kcgen.csr_from_edges(2000, [(i, i + 1) for i in range(1999)])
    yield "C1", kcgen.generate_host(kcgen.CONFIGS["C1"])
    yield "chunglu_2^14", kcgen.generate_host(kcgen.chunglu(1 << 14, 2.1, 1 << 17))


def main():
    dev = torch.device("cuda", 0)
    which = sys.argv[1:] or ["peel", "hostloop", "mpm", "outputs", "mg"]
    bad = 0
    for name, (rp, ci) in graphs():
        ref = oracle.bz_core(rp, ci)
        r = torch.from_numpy(rp).to(dev)
        c = torch.from_numpy(ci).to(dev)
        runs = []
        if "peel" in which:
            runs += [("peel", dict()), ("peel_nobloom", dict(bloom=False))]
        if "hostloop" in which:
            runs += [("hostloop", dict(algo=kc.ALGO_HOSTLOOP))]
        for tag, kw in runs:
            core = kc.kcore_decompose(r, c, **kw)
            ok = np.array_equal(core.cpu().numpy(), ref)
            bad += not ok
            print(f"{name:16s} {tag:14s} parity={ok}", flush=True)
        if "mpm" in which:
            a, it = kc.kcore_mpm(r, c)
            ok = np.array_equal(a.cpu().numpy(), ref)
            bad += not ok
            print(f"{name:16s} mpm            parity={ok} iterations={it}", flush=True)
        if "outputs" in which:
            k = int(ref.max())
            mask, cnt = kc.kcore_kcore_mask(torch.from_numpy(ref).to(dev), k)
            ok = cnt == int((ref >= k).sum())
            bad += not ok
            print(f"{name:16s} kcore_mask     ok={ok}", flush=True)
        if "mg" in which:
            core = kc.kcore_decompose_mg_virtual(r, c, 3)
            ok = np.array_equal(core.cpu().numpy(), ref)
            bad += not ok
            print(f"{name:16s} mg_virtual(3)  parity={ok}", flush=True)
    torch.cuda.synchronize()
    print("SANITIZE_WORKLOAD_DONE bad=%d" % bad)
    return 1 if bad else 0


if __name__ == "__main__":
    sys.exit(main())
