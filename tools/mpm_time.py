"""Time the MPM kernel on configs (development aid)."""
import sys, time
import torch
sys.path.insert(0, '.')
import kcgen
import paper_conf_icde_ahmady0gcz23_b200 as kc
for name in sys.argv[1:] or ["C1", "C2", "C3", "C4"]:
    r, c = kcgen.generate_device(kcgen.CONFIGS[name])
    core = kc.kcore_decompose(r, c)
    ms = []
    for rep in range(3):
        a, it, st = kc.kcore_mpm(r, c, stats=True)
        ms.append(st.kernel_ms)
    ok = bool(torch.equal(a, core))
    best = min(ms)
    print(f"{name} mpm iters={it} kernel_ms={best:.3f} Medges/s={c.numel()/2/best/1e3:.0f} processed={st.scanned} "
          f"arcs_gathered={st.arcs_walked} ({st.arcs_walked/c.numel():.1f}x arcs) equals_peel={ok}", flush=True)
    del r, c, a, core; torch.cuda.empty_cache()
