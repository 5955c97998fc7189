"""Host-side multi-GPU logic on CPU with world_size-2 gloo process groups:
owner ranges, the owner rule, slicing a global CSR into rank rows, and
gathering per-rank results -- the N > 1 plumbing around kcore_decompose_mg.
The per-rank core values come from the oracle here (the device protocol
itself is tested on the GPU by tests/test_gpu_mg.py)."""
import os
import socket

import numpy as np
import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp

import kcgen
import oracle
from paper_conf_icde_ahmady0gcz23_b200 import parallel


def test_owner_ranges_tile_and_owner_rule():
    for n in (0, 1, 7, 100, 65536, 1 << 24):
        for P in (1, 2, 3, 7, 8):
            rr = parallel.owner_ranges(n, P)
            assert rr[0][0] == 0 and rr[-1][1] == n
            assert all(a[1] == b[0] for a, b in zip(rr, rr[1:]))
            sizes = [b - a for a, b in rr]
            assert max(sizes) - min(sizes) <= 1
            if n:
                for v in sorted({0, n - 1, n // 2, n // 3, (2 * n) // 3}):
                    r = parallel.owner_of(v, n, P)
                    assert rr[r][0] <= v < rr[r][1]


def test_local_csr_reassembles_global():
    rp, ci = kcgen.generate_host(kcgen.rmat(10, 8, seed=5))
    n = rp.size - 1
    for P in (2, 3, 8):
        parts = [parallel.local_csr(rp, ci, a, b) for a, b in parallel.owner_ranges(n, P)]
        assert np.array_equal(np.concatenate([p[1] for p in parts]), ci)
        assert np.array_equal(np.concatenate([np.diff(p[0]) for p in parts]), np.diff(rp))
        assert all(p[0][0] == 0 for p in parts)


def _port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _worker(rank, world, port, q):
    dist.init_process_group("gloo", init_method=f"tcp://127.0.0.1:{port}", rank=rank, world_size=world)
    try:
        rp, ci = kcgen.generate_host(kcgen.rmat(11, 16, seed=7))
        n = rp.size - 1
        vb, ve = parallel.owner_ranges(n, world)[rank]
        # each rank generates only its owned rows (owner-range generation)
        lrp, lci = kcgen.generate_host(kcgen.rmat(11, 16, seed=7), vb, ve)
        grp, gci = parallel.local_csr(rp, ci, vb, ve)
        assert np.array_equal(lrp, grp) and np.array_equal(lci, gci)
        ref = oracle.bz_core(rp, ci)
        mine = torch.from_numpy(ref[vb:ve].copy())
        allc = parallel.gather_cores(mine)
        q.put((rank, bool(np.array_equal(allc.numpy(), ref))))
    finally:
        dist.destroy_process_group()


def test_world2_gloo_gather_and_owner_generation():
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _port()
    procs = [ctx.Process(target=_worker, args=(r, 2, port, q)) for r in range(2)]
    for p in procs:
        p.start()
    res = [q.get(timeout=240) for _ in procs]
    for p in procs:
        p.join(timeout=60)
    assert sorted(res) == [(0, True), (1, True)]
