"""Host-side multi-GPU logic on CPU with world_size-2 gloo process groups:
owner ranges, the owner rule, slicing a global CSR into rank rows, and
gathering per-rank results -- the N > 1 plumbing around kcore_decompose_mg
-- and the device-initiated protocol's host model run with one rank per gloo
process (tests/mg_protocol_model.py; the CUDA protocol itself is tested on
the GPU by tests/test_gpu_mg.py)."""
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


# ------------------------------------------------------------------------
# The device-initiated protocol's host model (tests/mg_protocol_model.py):
# P in-process ranks, and one rank per gloo process (world_size 2) with the
# decrement messages exchanged over torch.distributed.
from mg_protocol_model import Rank, run_in_process, run_rank  # noqa: E402

_SENT = 1 << 62


@pytest.mark.parametrize("P", [1, 2, 3, 5, 8])
def test_mg_protocol_model_in_process(P):
    graphs = [kcgen.generate_host(kcgen.rmat(10, 8, seed=11)),
              kcgen.generate_host(kcgen.chunglu(3000, 2.1, 20000, seed=12)),
              kcgen.csr_from_edges(9, [(0, 1), (1, 2), (2, 0), (3, 4)]),
              kcgen.csr_from_edges(300, [(i, i + 1) for i in range(299)])]
    for rp, ci in graphs:
        ref = oracle.bz_core(rp, ci)
        got, levels = run_in_process(rp, ci, P)
        assert np.array_equal(got, ref), P
        assert levels == len(np.unique(ref))


def _proto_worker(rank, world, port, q):
    dist.init_process_group("gloo", init_method=f"tcp://127.0.0.1:{port}", rank=rank, world_size=world)
    try:
        spec = kcgen.chunglu(2000, 2.1, 12000, seed=21)
        rp, ci = kcgen.generate_host(spec)
        n = rp.size - 1
        ranges = parallel.owner_ranges(n, world)
        vb, ve = ranges[rank]
        lrp, lci = kcgen.generate_host(spec, vb, ve)  # owner-range generation
        me = Rank(lrp, lci, vb, ve, ranges)

        def exchange(msgs):
            allm = [None] * world
            dist.all_gather_object(allm, msgs)
            out = []
            for m in allm:
                out.extend(m.get(rank, []))
            return out

        def asum(x):
            t = torch.tensor([int(x)], dtype=torch.int64)
            dist.all_reduce(t)
            return int(t.item())

        def amin(x):
            t = torch.tensor([_SENT if x is None else int(x)], dtype=torch.int64)
            dist.all_reduce(t, op=dist.ReduceOp.MIN)
            return None if int(t.item()) == _SENT else int(t.item())

        core, levels = run_rank(me, n, exchange, asum, amin)
        allc = parallel.gather_cores(torch.from_numpy(core.astype(np.int32)))
        ref = oracle.bz_core(rp, ci)
        q.put((rank, bool(np.array_equal(allc.numpy(), ref)), levels == len(np.unique(ref))))
    finally:
        dist.destroy_process_group()


def test_world2_gloo_mg_protocol_model():
    """Two processes, each owning half of the vertices, run the protocol's
    rank code with the messages and reductions over gloo; the gathered core
    numbers equal the oracle's."""
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _port()
    procs = [ctx.Process(target=_proto_worker, args=(r, 2, port, q)) for r in range(2)]
    for p in procs:
        p.start()
    res = [q.get(timeout=240) for _ in procs]
    for p in procs:
        p.join(timeout=60)
    assert sorted(res) == [(0, True, True), (1, True, True)]
