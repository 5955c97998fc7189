"""A/B kernel timing of run-time variants (dev aid): python tools/ab.py C1 C3 C4 -- 'dict()' 'dict(red=False)'
Each variant: 2 warm-up + 7 timed calls, L2 flushed between calls, interleaved; prints median/min."""
import statistics
import sys

import torch

sys.path.insert(0, '.')
import kcgen  # noqa: E402
import paper_conf_icde_ahmady0gcz23_b200 as kc  # noqa: E402

args = sys.argv[1:]
cut = args.index('--') if '--' in args else len(args)
cfgs, variants = args[:cut], [eval(v) for v in args[cut + 1:]] or [dict()]
flush = torch.empty(512 << 20, dtype=torch.uint8, device='cuda')
for name in cfgs:
    r, c = kcgen.generate_device(kcgen.CONFIGS[name])
    n, m = r.numel() - 1, c.numel()
    ws = torch.empty(kc.kcore_workspace_size(n, m), dtype=torch.uint8, device='cuda')
    ref = None
    times = [[] for _ in variants]
    sts = [None] * len(variants)
    for rep in range(9):
        for i, kw in enumerate(variants):
            flush.fill_(1)
            core, st = kc.kcore_decompose(r, c, workspace=ws, stats=True, **kw)
            if ref is None:
                ref = core.clone()
            elif not torch.equal(core, ref):
                print(f"MISMATCH {name} {kw}", flush=True)
            if rep >= 2:
                times[i].append(st.kernel_ms)
            sts[i] = st
    for i, kw in enumerate(variants):
        st = sts[i]
        print(f"{name} {kw}: med {statistics.median(times[i]):.3f} min {min(times[i]):.3f} ms  "
              f"levels={st.levels} phases={st.phases} scanned={st.scanned} arcs={st.arcs_walked} hub={st.hub_arcs}",
              flush=True)
    del r, c, ws
    torch.cuda.empty_cache()
