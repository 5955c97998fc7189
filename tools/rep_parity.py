import sys, numpy as np
sys.path.insert(0,'.')
import kcgen, oracle, torch
import paper_conf_icde_ahmady0gcz23_b200 as kc
for cfg, spec in [("C1", kcgen.CONFIGS["C1"]), ("cl16", kcgen.chunglu(1 << 16, 2.1, 1 << 20)), ("rmat18", kcgen.rmat(18, 16))]:
  rp, ci = kcgen.generate_host(spec); ref = oracle.bz_core(rp, ci)
  r = torch.from_numpy(rp).cuda(); c = torch.from_numpy(ci).cuda()
  for kw in [dict(), dict(near_min_alive=1, near_window=64), dict(near_min_alive=1, near_window=1), dict(red=False, near_min_alive=1, near_window=5)]:
    for rep in range(5):
      core, st = kc.kcore_decompose(r, c, stats=True, **kw)
      ok = np.array_equal(core.cpu().numpy(), ref)
      if not ok: print("MISMATCH", cfg, kw, rep, int((core.cpu().numpy()!=ref).sum())); break
    print(cfg, kw, "ok" if ok else "BAD", flush=True)
