import sys, time, torch
sys.path.insert(0,'.')
import kcgen, paper_conf_icde_ahmady0gcz23_b200 as kc
r, c = kcgen.generate_device(kcgen.CONFIGS["C4"])
h_rp = torch.empty(r.shape, dtype=torch.int64, pin_memory=True); h_rp.copy_(r)
h_ci = torch.empty(c.shape, dtype=torch.int32, pin_memory=True); h_ci.copy_(c)
ref = kc.kcore_decompose(r, c).cpu()
del r, c; torch.cuda.empty_cache()
h_core = torch.empty(ref.numel(), dtype=torch.int32, pin_memory=True)
kc.kcore_decompose_host(h_rp, h_ci, core_out=h_core)
ts=[]
for i in range(5):
    torch.cuda.synchronize(); t=time.perf_counter()
    kc.kcore_decompose_host(h_rp, h_ci, core_out=h_core)
    torch.cuda.synchronize(); ts.append(time.perf_counter()-t)
print("e2e ms", [round(x*1e3,1) for x in ts], "equal", bool(torch.equal(h_core, ref)))
# raw H2D bandwidth single copy
d = torch.empty(h_ci.shape, dtype=torch.int32, device='cuda')
torch.cuda.synchronize(); t=time.perf_counter(); d.copy_(h_ci, non_blocking=True); torch.cuda.synchronize()
print("single H2D GB/s", h_ci.numel()*4/(time.perf_counter()-t)/1e9)
