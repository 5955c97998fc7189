"""Ad-hoc timing of the configs (development aid; bench.py is the contract)."""
import sys, time
import torch
sys.path.insert(0, '.')
import kcgen
import paper_conf_icde_ahmady0gcz23_b200 as kc

names = sys.argv[1:] or ["C1", "C2", "C3", "C4"]
for name in names:
    t0 = time.time()
    r, c = kcgen.generate_device(kcgen.CONFIGS[name])
    torch.cuda.synchronize()
    tg = time.time() - t0
    n = r.numel() - 1; m = c.numel()
    for kw in (dict(),):
        ws = torch.empty(kc.kcore_workspace_size(n, m), dtype=torch.uint8, device='cuda')
        for i in range(3):
            core, st = kc.kcore_decompose(r, c, workspace=ws, stats=True, **kw)
        ms = []
        for i in range(5):
            core, st = kc.kcore_decompose(r, c, workspace=ws, stats=True, **kw)
            ms.append(st.kernel_ms)
        best = min(ms)
        print(f"{name} {kw} n={n} arcs={m} gen={tg:.2f}s kernel_ms min={best:.3f} med={sorted(ms)[2]:.3f} "
              f"Medges/s={m/2/best/1e3:.0f} levels={st.levels} phases={st.phases} solo={st.solo_phases} hub_arcs={st.hub_arcs} "
              f"bar={st.barriers} scanned={st.scanned} compact={st.compactions} kmax={st.kmax} grid={st.grid_blocks}",
              flush=True)
    del r, c
    torch.cuda.empty_cache()
