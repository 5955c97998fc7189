"""Experiment: cost of finishing the peel's tail with MPM on the k*-core
(dev aid).  For several k*, extract the k*-core (kcore_kcore_subgraph), run
MPM on it and compare with the peel's time spent on levels >= k* (trace)."""
import os, sys
os.environ.setdefault("KCORE_LIB", os.path.join(os.path.dirname(os.path.dirname(os.path.abspath(__file__))), "paper_conf_icde_ahmady0gcz23_b200", "lib", "libkcore_trace.so"))
import numpy as np
import torch
sys.path.insert(0, '.')
import kcgen
import paper_conf_icde_ahmady0gcz23_b200 as kc
for name in sys.argv[1:]:
    r, c = kcgen.generate_device(kcgen.CONFIGS[name])
    tr = torch.zeros((20000, 8), dtype=torch.int64, device='cuda')
    for _ in range(2):
        core, st = kc.kcore_decompose(r, c, trace=tr, stats=True)
    T = tr[:st.trace_len].cpu().numpy()
    t = T[:, 0]; ks = T[:, 3]
    cn = core.cpu().numpy(); kmax = int(cn.max())
    print(f"{name}: peel {st.kernel_ms:.2f} ms, levels {st.levels}, kmax {kmax}", flush=True)
    for frac in (0.1, 0.25, 0.5, 0.75):
        kstar = int(np.quantile(np.unique(cn), frac))
        i0 = np.searchsorted(ks, kstar)  # first record with k >= kstar (records are in k order)
        tail_ms = (t[-1] - t[max(i0 - 1, 0)]) / 1e6
        srp, sci, vm = kc.kcore_kcore_subgraph(r, c, core, kstar)
        for _ in range(2):
            a, it, sm = kc.kcore_mpm(srp, sci, stats=True)
        ok = bool(torch.equal(a, core[vm.long()]))
        print(f"  k*={kstar}: k*-core n={vm.numel()} arcs={sci.numel()} peel levels>=k*: {int((np.unique(cn) >= kstar).sum())}"
              f" peel tail ~{tail_ms:.2f} ms | MPM {sm.kernel_ms:.2f} ms iters={it} exact={ok}", flush=True)
    del r, c, core; torch.cuda.empty_cache()
