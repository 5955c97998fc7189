"""Round-2 ablation on one B200 (the paper's Table II and
Table V analogues).  Every variant runs in a fresh process (the persisting L2
set-aside is a device-wide limit): median of 5 calls after 2 warm-ups, L2
flushed between calls, on C1..C4; every result is compared bit for bit with
the default library's result (itself pinned to the oracle by the GPU tests)
and, on C1, with the oracle directly.

Compile-time variants (paper_conf_icde_ahmady0gcz23_b200/lib/variants/*.so,
built by tools/build_variants.sh tools/variants_f4.txt):
  no_smbuf   no shared-memory frontier: every claimed vertex goes to the global
             queue (the paper's SM-buffer switch)
  vp_line    prefetch the first colidx line of every claimed vertex's row
             (vertex prefetching; default: no prefetch)
  vp_row     bulk-prefetch the whole row into L2 (cp.async.bulk.prefetch)
  ec_block   block-level compaction in the level scan (the paper's two-stage
             block scan, Fig. 9) instead of warp ballots (BC)
  no_near    near list compiled out (every level scans the whole alive list)
Run-time variants (flags of the default library): no persisting L2 window,
no Bloom filter, no non-returning heavy walks, no near list, the paper's
host loop (Alg. 1: launch + read-back per phase).

Peak device memory per call (Table V analogue): the CSR
and core_out tensors plus the library's own stream-ordered allocations,
measured as the high watermark of the device's default memory pool
(cudaMemPoolAttrUsedMemHigh) around one call without a caller workspace.

    python tools/ablation_r2.py [C1 C2 C3 C4] > gpurun_out/ablation_r2.json
"""
import glob
import json
import os
import subprocess
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
LIBDIR = os.path.join(ROOT, "paper_conf_icde_ahmady0gcz23_b200", "lib")
RUNTIME = {
    "default": {},
    "no_l2_persist": {"l2_persist": False},
    "no_bloom": {"bloom": False},
    "no_red": {"red": False},
    "no_near_flag": {"near": False},
    "hostloop_alg1": {"algo": 1},
}
CODE = r'''
import sys, json, statistics, torch, numpy as np
sys.path.insert(0, %r)
import kcgen, paper_conf_icde_ahmady0gcz23_b200 as kc
kw, names, ref_dir, mem = %r, %r, %r, %r
flush = torch.empty(512 << 20, dtype=torch.uint8, device='cuda')
out = {}
for name in names:
    r, c = kcgen.generate_device(kcgen.CONFIGS[name])
    n, m = r.numel() - 1, c.numel()
    ws = torch.empty(kc.kcore_workspace_size(n, m), dtype=torch.uint8, device='cuda')
    for _ in range(2): kc.kcore_decompose(r, c, workspace=ws, **kw)
    ms = []
    for _ in range(5):
        flush.fill_(1)
        core, st = kc.kcore_decompose(r, c, workspace=ws, stats=True, **kw)
        ms.append(st.kernel_ms)
    d = {"ms": round(statistics.median(ms), 3), "Medges_s": round(m / 2 / statistics.median(ms) / 1e3, 1),
         "phases": st.phases, "levels": st.levels, "scanned": st.scanned}
    path = f"{ref_dir}/ref_{name}.npy"
    got = core.cpu().numpy()
    try:
        d["equal_default"] = bool(np.array_equal(got, np.load(path)))
    except FileNotFoundError:
        np.save(path, got)
        d["equal_default"] = True
    if name == "C1":
        import oracle
        d["equal_oracle"] = bool(np.array_equal(got, oracle.bz_core(r.cpu().numpy(), c.cpu().numpy())))
    if mem:
        from cuda.bindings import runtime as rt, driver as dr
        del ws
        torch.cuda.synchronize(); torch.cuda.empty_cache()
        err, pool = rt.cudaDeviceGetDefaultMemPool(0)
        rt.cudaMemPoolTrimTo(pool, 0)
        rt.cudaMemPoolSetAttribute(pool, rt.cudaMemPoolAttr.cudaMemPoolAttrUsedMemHigh, dr.cuuint64_t(0))
        core2 = kc.kcore_decompose(r, c)
        torch.cuda.synchronize()
        err, hi = rt.cudaMemPoolGetAttribute(pool, rt.cudaMemPoolAttr.cudaMemPoolAttrUsedMemHigh)
        lib_peak = int(hi)
        d.update({"csr_bytes": 8 * (n + 1) + 4 * m, "core_bytes": 4 * n, "library_peak_bytes": lib_peak,
                  "peak_bytes": 8 * (n + 1) + 4 * m + 4 * n + lib_peak,
                  "peak_bytes_per_arc": round((8 * (n + 1) + 4 * m + 4 * n + lib_peak) / m, 2)})
        del core2
    out[name] = d
    del r, c, core
    torch.cuda.empty_cache()
print(json.dumps(out))
'''


def run(tag, lib, kw, names, ref_dir, mem):
    env = dict(os.environ)
    if lib:
        env["KCORE_LIB"] = lib
    p = subprocess.run([sys.executable, "-c", CODE % (ROOT, kw, names, ref_dir, mem)], capture_output=True,
                       text=True, timeout=1200, env=env, cwd=ROOT)
    try:
        return json.loads(p.stdout.strip().splitlines()[-1])
    except Exception:
        return {"error": (p.stderr or p.stdout)[-600:]}


def main():
    names = sys.argv[1:] or ["C1", "C2", "C3", "C4"]
    ref_dir = "/tmp/kc_ablation_ref"
    os.makedirs(ref_dir, exist_ok=True)
    for f in glob.glob(f"{ref_dir}/*.npy"):
        os.remove(f)
    res = {"runtime": {}, "compile_time": {}}
    res["runtime"]["default"] = run("default", None, {}, names, ref_dir, True)
    print("default", json.dumps(res["runtime"]["default"]), file=sys.stderr, flush=True)
    for tag, kw in RUNTIME.items():
        if tag == "default":
            continue
        res["runtime"][tag] = run(tag, None, kw, names, ref_dir, False)
        print(tag, json.dumps(res["runtime"][tag]), file=sys.stderr, flush=True)
    for so in sorted(glob.glob(os.path.join(LIBDIR, "variants", "*.so"))):
        tag = os.path.basename(so)[:-3]
        res["compile_time"][tag] = run(tag, so, {}, names, ref_dir, False)
        print(tag, json.dumps(res["compile_time"][tag]), file=sys.stderr, flush=True)
    print(json.dumps(res, indent=1))


if __name__ == "__main__":
    main()
