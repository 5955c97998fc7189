"""Multi-GPU protocol (kcore_decompose_mg) on the single available GPU:
P virtual ranks with the loopback transport (same driver and kernels as the
NCCL path), and the real NCCL transport with a 1-rank communicator.  Results
must equal the CPU oracle bit for bit."""
import os
import socket

import numpy as np
import pytest

import kcgen
import oracle

torch = pytest.importorskip("torch")
import paper_conf_icde_ahmady0gcz23_b200 as kc  # noqa: E402
from paper_conf_icde_ahmady0gcz23_b200 import parallel  # noqa: E402

pytestmark = pytest.mark.gpu
DEV = "cuda:0"


def _dev(rp, ci):
    return torch.from_numpy(np.asarray(rp, np.int64)).to(DEV), torch.from_numpy(np.asarray(ci, np.int32)).to(DEV)


GRAPHS = [
    ("bowtie", lambda: kcgen.csr_from_edges(5, [(0, 1), (0, 2), (1, 2), (0, 3), (0, 4), (3, 4)])),
    ("path", lambda: kcgen.csr_from_edges(2000, [(i, i + 1) for i in range(1999)])),
    ("rmat12", lambda: kcgen.generate_host(kcgen.rmat(12, 16, seed=3))),
    ("er", lambda: kcgen.generate_host(kcgen.er(20000, 12, seed=4))),
    ("chunglu", lambda: kcgen.generate_host(kcgen.chunglu(30000, 2.1, 250000, seed=5))),
    ("empty", lambda: kcgen.csr_from_edges(7, [])),
]


@pytest.mark.parametrize("name,make", GRAPHS)
@pytest.mark.parametrize("P", [1, 2, 3, 4, 8])
def test_virtual_ranks_match_oracle(name, make, P):
    rp, ci = make()
    ref = oracle.bz_core(rp, ci)
    r, c = _dev(rp, ci)
    got, st = kc.kcore_decompose_mg_virtual(r, c, P, stats=True)
    assert np.array_equal(got.cpu().numpy(), ref), (name, P)
    if ref.size and ref.max() > 0:
        assert st.kmax == ref.max()


def test_virtual_ranks_config_C1():
    rp, ci = kcgen.generate_host(kcgen.CONFIGS["C1"])
    ref = oracle.bz_core(rp, ci)
    r, c = _dev(rp, ci)
    for P in (2, 8):
        got = kc.kcore_decompose_mg_virtual(r, c, P)
        assert np.array_equal(got.cpu().numpy(), ref), P


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def test_nccl_transport_single_rank():
    import torch.distributed as dist
    rp, ci = kcgen.generate_host(kcgen.rmat(13, 16, seed=9))
    ref = oracle.bz_core(rp, ci)
    n = rp.size - 1
    dist.init_process_group("gloo", init_method=f"tcp://127.0.0.1:{_free_port()}", rank=0, world_size=1)
    try:
        comm = kc.NcclComm(device=DEV)
        vb, ve = parallel.owner_ranges(n, 1)[0]
        lrp, lci = parallel.local_csr(rp, ci, vb, ve)
        r, c = _dev(lrp, lci)
        got = kc.kcore_decompose_mg(r, c, n, vb, ve, comm)
        assert np.array_equal(got.cpu().numpy(), ref)
        comm.close()
    finally:
        dist.destroy_process_group()
