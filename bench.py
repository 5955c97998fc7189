#!/usr/bin/env python
"""Benchmark of the k-core hot path (driver contract).

    python bench.py [--gpus N] [--steps K] [--warmup W] [--impl reference]

Workload (N=1): BASELINE.json configs[3], the R-MAT scale-24 edge-factor-32
graph -- the config the north-star target (>= 50 % of the HBM-bytes
roofline on one B200) is quoted on.  A "step" is one kcore_decompose call
(deg init, every level scan, every peel sub-round, level control) on the
device-resident CSR.  Between steps L2 is flushed (a 512 MiB write) outside
the timed events.  value = undirected edges / step time (Medges/s), summed
over K steps, max over ranks for N > 1.

N > 1 runs the multi-GPU protocol on the same graph (1-D vertex ranges): by
default the device-initiated kernel over NCCL symmetric memory
(kcore_decompose_mg_ex(KCORE_MG_DEVICE)), --mg-algo host the host-driven NCCL
exchange.  Strong scaling (the workload is one fixed graph at every N, so
every line says "strong").

--impl reference times the CPU oracle (serial Batagelj-Zaversnik, oracle/)
on the host, each step a bounded sample of the workload (R-MAT scale 22,
edge factor 32, same generator recipe).
"""
from __future__ import annotations

import argparse
import json
import os
import statistics
import subprocess
import sys
import time

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

METRIC = "Medges/s core decomposition (1/2/4/8 B200) and % of HBM roofline"
WORKLOAD = "rmat-s24-ef32"
REF_SAMPLE_SCALE = 22


def _peaks():
    try:
        with open(os.path.join(ROOT, "MEASURED_PEAKS.json")) as f:
            p = json.load(f)
        return float(p["hbm_gbs"]), "measured"
    except Exception:
        return 6650.0, "fallback"


class Clocks:
    """nvidia-smi sampler for the timed region (clocks + throttle reasons)."""

    Q = ("clocks.sm,clocks.max.sm,clocks_event_reasons.hw_slowdown,"
         "clocks_event_reasons.hw_thermal_slowdown,clocks_event_reasons.sw_thermal_slowdown,"
         "clocks_event_reasons.sw_power_cap")

    def __init__(self, index: int):
        self.proc = None
        self.path = os.path.join("/tmp", f"kcore_clocks_{os.getpid()}.csv")
        try:
            self.proc = subprocess.Popen(
                ["nvidia-smi", "-i", str(index), f"--query-gpu={self.Q}", "--format=csv,noheader,nounits",
                 "-lms", "100"], stdout=open(self.path, "w"), stderr=subprocess.DEVNULL)
        except Exception:
            self.proc = None

    def stop(self):
        if self.proc is None:
            return None
        self.proc.terminate()
        try:
            self.proc.wait(timeout=5)
        except Exception:
            self.proc.kill()
        sm, mx, reasons = [], 0.0, set()
        names = ["hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown", "sw_power_cap"]
        for line in open(self.path):
            f = [x.strip() for x in line.split(",")]
            if len(f) < 6:
                continue
            try:
                sm.append(float(f[0]))
                mx = max(mx, float(f[1]))
            except ValueError:
                continue
            for nm, v in zip(names, f[2:6]):
                if v.lower().startswith("active"):
                    reasons.add(nm)
        if not sm:
            return None
        return {"sm_mhz": statistics.median(sm), "sm_max_mhz": mx, "reasons": sorted(reasons),
                "samples": len(sm)}


def _dist():
    import torch.distributed as dist
    world = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    return world, rank, local, dist


def run_reference(args):
    """CPU oracle arm: serial BZ on bounded samples, timed on the host."""
    world, rank, _, _ = _dist()
    if rank != 0:
        return 0
    import numpy as np
    import kcgen
    import oracle
    spec = kcgen.rmat(REF_SAMPLE_SCALE, 32, seed=1)
    try:
        import torch
        if torch.cuda.is_available():
            r, c = kcgen.generate_device(spec)
            rp, ci = r.cpu().numpy(), c.cpu().numpy()
            del r, c
        else:
            rp, ci = kcgen.generate_host(spec)
    except Exception:
        rp, ci = kcgen.generate_host(spec)
    m_und = ci.size // 2
    for _ in range(args.warmup):
        oracle.bz_core(rp, ci)
    t = []
    for _ in range(args.steps):
        t0 = time.perf_counter()
        oracle.bz_core(rp, ci)
        t.append(time.perf_counter() - t0)
    tot = sum(t)
    value = args.steps * m_und / tot / 1e6
    line = {
        "impl": "reference", "metric": METRIC, "value": value, "unit": "Medges/s", "n_gpus": args.gpus,
        "steps": args.steps, "warmup": args.warmup, "ms_per_step": tot / args.steps * 1e3,
        "higher_is_better": True, "scaling": "strong", "vs_baseline": None,
        "dtype": "int32", "data": "synthetic",
        "config": {"workload": WORKLOAD, "sample": f"rmat-s{REF_SAMPLE_SCALE}-ef32", "n": int(rp.size - 1),
                   "m_undirected": int(m_und)},
        "cpu_baseline": {"value": value, "unit": "Medges/s", "cores": 1, "kind": "oracle",
                         "sample": f"serial BZ on R-MAT s{REF_SAMPLE_SCALE} ef32 (same recipe as {WORKLOAD}) "
                                   f"per step; host has {os.cpu_count()} cores"},
        "e2e": {"value": value, "unit": "Medges/s", "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0},
    }
    print(json.dumps(line), flush=True)
    return 0


def _lib_sha():
    """Identity of the benchmarked kernel's code: sha256 of the SASS
    instruction lines of k_persistent (cuobjdump).  Unlike the .so's own hash it is the same for every build
    of the same sources (nvcc embeds build-specific bytes in the fat binary)."""
    import hashlib
    import re
    try:
        import paper_conf_icde_ahmady0gcz23_b200 as kc
        out = subprocess.run(["cuobjdump", "-sass", "-fun", "_ZN2kc12k_persistentENS_5KArgsE", kc.LIB_PATH],
                             capture_output=True, text=True, timeout=120).stdout
        lines = [ln for ln in out.splitlines() if re.match(r"^\s+/\*[0-9a-f]{4,}\*/", ln)]
        if not lines:
            return None
        return hashlib.sha256("\n".join(lines).encode()).hexdigest()
    except Exception:
        return None


def _cpu_model():
    try:
        for line in open("/proc/cpuinfo"):
            if line.startswith("model name"):
                return line.split(":", 1)[1].strip()
    except Exception:
        pass
    return None


def per_config(args, kc, kcgen, flush, stream, peak, with_oracle=True):
    """C1-C3 (BASELINE.json configs[0..2]): kernel time median/min/std over
    K steps (L2 flushed between steps), roofline fraction with the same B_min
    formula, bit-exact parity against the oracle (test infrastructure, the
    cpu_baseline leg)."""
    import torch
    out = {}
    for name, desc in (("C1", "rmat-s16-ef16"), ("C2", "er-4M-d32"), ("C3", "chunglu-4M-70M-g2.1")):
        spec = kcgen.CONFIGS[name]
        rp, ci = kcgen.generate_device(spec)
        n, m = rp.numel() - 1, ci.numel()
        ws = torch.empty(kc.kcore_workspace_size(n, m), dtype=torch.uint8, device=rp.device)
        core = torch.empty(n, dtype=torch.int32, device=rp.device)
        for _ in range(args.warmup):
            kc.kcore_decompose(rp, ci, core_out=core, workspace=ws)
        ks = []
        st = None
        for _ in range(args.steps):
            flush.fill_(1)
            _, st = kc.kcore_decompose(rp, ci, core_out=core, workspace=ws, stats=True)
            ks.append(st.kernel_ms)
        med = statistics.median(ks)
        b_min = 4 * m + 8 * (n + 1) + 8 * n + 4 * n + 4 * st.scanned + 8 * n
        d = {"workload": desc, "n": n, "arcs": m, "m_undirected": m // 2,
             "kernel_ms_median": med, "kernel_ms_min": min(ks),
             "kernel_ms_std": statistics.pstdev(ks) if len(ks) > 1 else 0.0,
             "medges_per_s": m / 2 / (med * 1e-3) / 1e6,
             "roofline_frac": b_min / (med * 1e-3) / 1e9 / peak, "algorithmic_bytes": b_min,
             "levels": st.levels, "phases": st.phases, "kmax": st.kmax}
        if with_oracle:
            import oracle
            rp_h, ci_h = rp.cpu().numpy(), ci.cpu().numpy()
            t0 = time.perf_counter()
            ref = oracle.bz_core(rp_h, ci_h)
            d["oracle_s"] = time.perf_counter() - t0
            d["parity"] = bool((ref == core.cpu().numpy()).all())
        out[name] = d
        del rp, ci, ws, core
        torch.cuda.empty_cache()
    return out


def run_gpu(args):
    import torch
    world, rank, local, dist = _dist()
    if world > 1:
        torch.cuda.set_device(local)
        dist.init_process_group("nccl", device_id=torch.device("cuda", local))
    dev = torch.device("cuda", torch.cuda.current_device())
    import kcgen
    import paper_conf_icde_ahmady0gcz23_b200 as kc

    spec = kcgen.CONFIGS["C4"]
    n = spec.num_vertices
    flush = torch.empty(512 << 20, dtype=torch.uint8, device=dev)

    if world == 1 and not args.force_mg:
        rowptr, colidx = kcgen.generate_device(spec, device=dev)
        m_arcs = colidx.numel()
        ws = torch.empty(kc.kcore_workspace_size(n, m_arcs), dtype=torch.uint8, device=dev)
        core = torch.empty(n, dtype=torch.int32, device=dev)

        def step():
            return kc.kcore_decompose(rowptr, colidx, core_out=core, workspace=ws, stats=True)
    else:
        if world == 1:  # --force-mg on one GPU: a 1-rank process group for the NCCL path
            dist.init_process_group("gloo", init_method="tcp://127.0.0.1:29512", rank=0, world_size=1)
        from paper_conf_icde_ahmady0gcz23_b200 import parallel
        vb, ve = parallel.owner_ranges(n, world)[rank]
        rowptr, colidx = kcgen.generate_device(spec, vb, ve, device=dev)
        comm = kc.NcclComm(device=dev)
        t = torch.tensor([colidx.numel()], dtype=torch.int64)
        if dist.get_backend() == "nccl":
            t = t.to(dev)
        dist.all_reduce(t)
        m_arcs = int(t.item())

        algo = parallel.MG_DEVICE if args.mg_algo == "device" else parallel.MG_HOSTLOOP

        def step():
            return kc.kcore_decompose_mg(rowptr, colidx, n, vb, ve, comm, stats=True, algo=algo)
    m_und = m_arcs // 2
    torch.cuda.synchronize()

    for _ in range(args.warmup):
        step()
    stream = torch.cuda.current_stream(dev)
    clocks = Clocks(dev.index if dev.index is not None else 0) if rank == 0 else None
    time.sleep(0.3 if clocks else 0)
    if world > 1:
        dist.barrier()
    torch.cuda.synchronize()
    evs = []
    stats = []
    for _ in range(args.steps):
        flush.fill_(1)  # 512 MiB write: evicts the 126 MB L2 between steps
        e0 = torch.cuda.Event(enable_timing=True)
        e1 = torch.cuda.Event(enable_timing=True)
        e0.record(stream)
        out = step()
        e1.record(stream)
        evs.append((e0, e1))
        stats.append(out[1])
    torch.cuda.synchronize()
    if world > 1:
        dist.barrier()
    step_ms = [a.elapsed_time(b) for a, b in evs]
    total_ms = sum(step_ms)
    per_rank_ms = None
    if world > 1:
        t = torch.tensor([total_ms], dtype=torch.float64, device=dev)
        allt = [torch.zeros_like(t) for _ in range(world)]
        dist.all_gather(allt, t)
        per_rank_ms = [float(x.item()) / args.steps for x in allt]  # per step, every rank
        total_ms = max(float(x.item()) for x in allt)  # the job's time: the slowest rank
    value = args.steps * m_und / (total_ms * 1e-3) / 1e6
    ms_per_step = total_ms / args.steps

    # end to end through the public API on pinned host buffers (N=1)
    e2e = None
    if world == 1 and not args.force_mg:
        h_rp = torch.empty(rowptr.shape, dtype=torch.int64, pin_memory=True)
        h_ci = torch.empty(colidx.shape, dtype=torch.int32, pin_memory=True)
        h_rp.copy_(rowptr)
        h_ci.copy_(colidx)
        h_core = torch.empty(n, dtype=torch.int32, pin_memory=True)
        ws = None
        torch.cuda.empty_cache()
        kc.kcore_decompose_host(h_rp, h_ci, core_out=h_core)  # warm-up
        et = []
        for _ in range(max(3, min(args.steps, 10))):
            torch.cuda.synchronize()
            e0 = torch.cuda.Event(enable_timing=True)
            e1 = torch.cuda.Event(enable_timing=True)
            e0.record(stream)
            kc.kcore_decompose_host(h_rp, h_ci, core_out=h_core)
            e1.record(stream)
            torch.cuda.synchronize()
            et.append(e0.elapsed_time(e1))
        e2e = {"value": len(et) * m_und / (sum(et) * 1e-3) / 1e6, "unit": "Medges/s",
               "h2d_bytes_per_step": int(h_rp.numel() * 8 + h_ci.numel() * 4),
               "d2h_bytes_per_step": int(n * 4), "ms_per_step": sum(et) / len(et)}
    clk = clocks.stop() if clocks else None

    if rank != 0:
        if world > 1:
            dist.destroy_process_group()
        return 0
    st = stats[-1]
    # roofline of the dominant kernel (the persistent decomposition kernel)
    peak, peak_src = _peaks()
    kern_ms = statistics.mean(s.kernel_ms for s in stats) or ms_per_step  # mg: whole step
    scanned = statistics.mean(s.scanned for s in stats)
    b_min = 4 * m_arcs + 8 * (n + 1) + 8 * n + 4 * n + 4 * scanned + 8 * n  # SURVEY 8(d) B_min
    achieved = b_min / (kern_ms * 1e-3) / 1e9
    # DRAM traffic of the dominant kernel: from the committed `ncu --set full`
    # capture ONLY if that capture profiled this very device code (sha256 of
    # the SASS, recorded in the capture); otherwise null.  (ncu cannot run inside the
    # timed bench; profiles/README.md has the capture command.)
    traffic, traffic_src = None, None
    lib_sha = _lib_sha()
    tpath = os.path.join(ROOT, "profiles", "ncu_traffic_C4.json")
    if os.path.exists(tpath) and world == 1 and not args.force_mg:
        try:
            tj = json.load(open(tpath))
            if lib_sha and tj.get("sass_sha256") == lib_sha:
                traffic = tj.get("dram_bytes_per_launch")
                traffic_src = {"file": "profiles/ncu_traffic_C4.json", "sass_sha256": lib_sha,
                               "window_off_bytes": tj.get("dram_bytes_per_launch_window_off")}
        except Exception:
            traffic = None
    line = {
        "metric": METRIC, "value": value, "unit": "Medges/s", "n_gpus": world, "steps": args.steps,
        "warmup": args.warmup, "ms_per_step": ms_per_step, "higher_is_better": True,
        "scaling": "strong", "vs_baseline": None, "dtype": "int32",
        "data": "synthetic",
        "config": {"workload": WORKLOAD, "baseline_config": "BASELINE.json configs[3]", "n": n,
                   "m_undirected": m_und, "arcs": m_arcs, "l2": "flushed between steps (512 MiB write); "
                   "colidx 4 GB > L2", "parallelism": (f"vertex-range x{world} ({args.mg_algo})" if world > 1 or args.force_mg
                                                    else "1 GPU")},
        "roofline": {"bound": "hbm", "achieved": achieved, "peak": peak, "unit": "GB/s",
                     "frac": achieved / peak, "traffic": traffic, "traffic_source": traffic_src,
                     "peak_source": peak_src, "algorithmic_bytes": b_min, "kernel_ms": kern_ms},
        "timing": {"step_ms_median": statistics.median(step_ms), "step_ms_min": min(step_ms),
                   "step_ms_mean": statistics.mean(step_ms),
                   "step_ms_std": statistics.pstdev(step_ms) if len(step_ms) > 1 else 0.0,
                   "kernel_ms_median": statistics.median(s.kernel_ms for s in stats),
                   "kernel_ms_min": min(s.kernel_ms for s in stats)},
        "sass_sha256": lib_sha,
        "gpu_launches": int(sum(s.launches for s in stats)),  # counted by the library, timed steps only
        "e2e": e2e,
        "clocks": clk,
        "stats": {"levels": st.levels, "phases": st.phases, "barriers": st.barriers, "scanned": st.scanned,
                  "kmax": st.kmax, "grid": st.grid_blocks, "block": st.block_threads},
        "per_rank_ms_per_step": per_rank_ms,
    }
    if world == 1 and not args.force_mg and not args.no_mpm:
        # the paper's second algorithm family on the same graph: MPM h-index
        # iteration, one persistent kernel per call; context for the peel, not the headline
        ws = None
        torch.cuda.empty_cache()
        mm = []
        for rep in range(3):
            flush.fill_(1)
            a_m, it_m, st_m = kc.kcore_mpm(rowptr, colidx, stats=True)
            mm.append(st_m.kernel_ms)
        line["alt_mpm"] = {"value": m_und / (statistics.mean(mm) * 1e-3) / 1e6, "unit": "Medges/s",
                           "ms_per_step": statistics.mean(mm), "iterations": it_m,
                           "arcs_gathered": st_m.arcs_walked, "equals_peel": bool(torch.equal(a_m, core))}
        del a_m
    if world == 1 and not args.force_mg and not args.no_mpm:
        # the multi-GPU protocol (device-initiated) with 8 virtual ranks on
        # this one GPU, same graph: context for the 8-GPU design, not a scaling number
        torch.cuda.empty_cache()
        mv = []
        for rep_ in range(4):
            flush.fill_(1)
            c_mg, st_mg = kc.kcore_decompose_mg_virtual(rowptr, colidx, 8, stats=True)
            if rep_:
                mv.append(st_mg.kernel_ms)
        line["alt_mg_virtual8"] = {"value": m_und / (statistics.median(mv) * 1e-3) / 1e6, "unit": "Medges/s",
                                   "ms_per_step": statistics.median(mv), "sub_rounds": st_mg.phases,
                                   "device_barriers": st_mg.barriers, "equals_peel": bool(torch.equal(c_mg, core))}
        del c_mg
    if world == 1 and not args.force_mg and not args.no_configs:
        # the other single-GPU configs (BASELINE.json configs[0..2]) with the same protocol
        line["per_config"] = per_config(args, kc, kcgen, flush, stream, peak,
                                        with_oracle=not args.no_cpu_baseline)
    if world == 1 and not args.no_cpu_baseline and not args.force_mg:
        import oracle
        rp_h, ci_h = rowptr.cpu().numpy(), colidx.cpu().numpy()
        dts = []
        for _ in range(3):  # the paper's CPU protocol: mean of 3 runs
            t0 = time.perf_counter()
            ref = oracle.bz_core(rp_h, ci_h)
            dts.append(time.perf_counter() - t0)
        dt = statistics.mean(dts)
        ok = bool((ref == core.cpu().numpy()).all())
        # I2 + I4 certificate on the device's own peel order: exactness without the oracle
        order = torch.empty(n, dtype=torch.int32, device=dev)
        core2, _ = kc.kcore_decompose(rowptr, colidx, order_out=order, stats=True)
        cert = oracle.check_certificate(rp_h, ci_h, core2.cpu().numpy(), order.cpu().numpy()) == 0
        line["cpu_baseline"] = {"value": m_und / dt / 1e6, "unit": "Medges/s", "cores": 1, "kind": "oracle",
                                "sample": f"serial BZ on the full {WORKLOAD} graph, mean of 3 runs "
                                          f"({', '.join(f'{x:.1f}' for x in dts)} s)",
                                "host_cpu_model": _cpu_model(), "host_nproc": os.cpu_count(),
                                "parity": ok, "certificate_ok": bool(cert)}
    print(json.dumps(line), flush=True)
    if dist.is_initialized():
        dist.destroy_process_group()
    return 0


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=10)
    ap.add_argument("--warmup", type=int, default=3)
    ap.add_argument("--impl", default="native", choices=["native", "reference"])
    ap.add_argument("--no-cpu-baseline", action="store_true")
    ap.add_argument("--no-mpm", action="store_true", help="skip the MPM context measurement")
    ap.add_argument("--force-mg", action="store_true", help="run the multi-GPU path even at N=1")
    ap.add_argument("--no-configs", action="store_true", help="skip the C1-C3 per-config measurements")
    ap.add_argument("--mg-algo", default="device", choices=["host", "device"],
                    help="N > 1: the device-initiated kernel over NCCL symmetric memory (default, SURVEY f1) "
                         "or the host-driven NCCL exchange per sub-round")
    args = ap.parse_args()
    if args.warmup < 3:
        args.warmup = 3
    if args.impl == "reference":
        return run_reference(args)
    return run_gpu(args)


if __name__ == "__main__":
    sys.exit(main())
