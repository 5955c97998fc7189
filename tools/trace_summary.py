"""Per-phase device trace of one decomposition (development aid)."""
import sys
import numpy as np
import torch
sys.path.insert(0, '.')
import kcgen
import paper_conf_icde_ahmady0gcz23_b200 as kc

PH = {1: "level", 2: "hub"}
names = sys.argv[1:] or ["C4"]
for name in names:
    r, c = kcgen.generate_device(kcgen.CONFIGS[name])
    n = r.numel() - 1
    for kw in (dict(),):
        tr = torch.zeros((400000, 8), dtype=torch.int64, device='cuda')
        for _ in range(2):
            core, st = kc.kcore_decompose(r, c, trace=tr, stats=True, **kw)
        T = tr[:st.trace_len].cpu().numpy()
        if len(sys.argv) > 0: np.save(f'gpurun_out/trace_{name}.npy', T)
        t = T[:, 0]
        dt = np.diff(t, prepend=t[0])  # ns since previous record
        code = T[:, 2]
        ph = code >> 8; solo = (code >> 4) & 1
        print(f"== {name} {kw}: kernel_ms={st.kernel_ms:.3f} records={len(T)} levels={st.levels} "
              f"phases={st.phases} solo={st.solo_phases} bar={st.barriers} scanned={st.scanned} hub_arcs={st.hub_arcs}")
        first = t[0]
        print(f"   trace span {(t[-1]-t[0])/1e6:.3f} ms (first record = end of first phase after init)")
        for p in (1, 2):
            for s in (0, 1):
                sel = (ph == p) & (solo == s)
                if sel.sum() == 0: continue
                d = dt[sel]
                print(f"   {PH[p]:4s} solo={s}: count={sel.sum():6d} total={d.sum()/1e6:8.3f} ms "
                      f"median={np.median(d)/1e3:7.2f} us p90={np.percentile(d,90)/1e3:7.2f} us "
                      f"work={T[sel,5].sum() if p==2 else T[sel,4].sum()}")
        top = np.argsort(-dt)[:12]
        for i in top:
            print(f"     rec {i:5d} {PH.get(int(ph[i]),'?')} solo={solo[i]} k={T[i,3]} size={T[i,4]} arcs={T[i,5]} removed={T[i,6]} dt={dt[i]/1e3:.1f} us")
    del r, c
    torch.cuda.empty_cache()
