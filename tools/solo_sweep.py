"""Runtime sweep of the solo thresholds (development aid)."""
import sys, torch
sys.path.insert(0, '.')
import kcgen, paper_conf_icde_ahmady0gcz23_b200 as kc
for name in sys.argv[1:] or ["C1", "C3", "C4"]:
    r, c = kcgen.generate_device(kcgen.CONFIGS[name])
    ws = torch.empty(kc.kcore_workspace_size(r.numel() - 1, c.numel()), dtype=torch.uint8, device='cuda')
    for sa, ss in [(-1, -1), (2048, 8192), (4096, 16384), (16384, 32768), (65536, 65536), (262144, 131072)]:
        for _ in range(2): kc.kcore_decompose(r, c, workspace=ws, solo_arcs=sa, solo_scan=ss, stats=True)
        ms = sorted(kc.kcore_decompose(r, c, workspace=ws, solo_arcs=sa, solo_scan=ss, stats=True)[1].kernel_ms for _ in range(5))
        print(name, sa, ss, round(ms[2], 3), flush=True)
    del r, c; torch.cuda.empty_cache()
