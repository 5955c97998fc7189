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


GRAPHS += [
    ("star_big_hub", lambda: kcgen.csr_from_edges(20001, [(0, i) for i in range(1, 20001)])),
    ("bowtie_fan", lambda: kcgen.csr_from_edges(
        6001, [e for i in range(3000) for e in ((0, 1 + 2 * i), (0, 2 + 2 * i), (1 + 2 * i, 2 + 2 * i))])),
]


@pytest.mark.parametrize("name,make", GRAPHS)
@pytest.mark.parametrize("P", [1, 2, 3, 4, 5, 8])
@pytest.mark.parametrize("algo", [0, 1])
def test_virtual_ranks_match_oracle(name, make, P, algo):
    """Both protocols (0: device-initiated, 1: host-driven) with P virtual ranks."""
    rp, ci = make()
    ref = oracle.bz_core(rp, ci)
    r, c = _dev(rp, ci)
    got, st = kc.kcore_decompose_mg_virtual(r, c, P, stats=True, algo=algo)
    assert np.array_equal(got.cpu().numpy(), ref), (name, P, algo)
    if ref.size and ref.max() > 0:
        assert st.kmax == ref.max()
        assert st.levels == len(np.unique(ref))


@pytest.mark.parametrize("cfg", ["C1", "C2", "C3"])
def test_virtual_ranks_configs(cfg):
    """Device-initiated protocol, P = 2..8 virtual ranks, full-size C1-C3."""
    rp, ci = kcgen.generate_host(kcgen.CONFIGS[cfg]) if cfg == "C1" else (None, None)
    if cfg != "C1":
        r, c = kcgen.generate_device(kcgen.CONFIGS[cfg])
        rp, ci = r.cpu().numpy(), c.cpu().numpy()
    ref = oracle.bz_core(rp, ci)
    r, c = _dev(rp, ci)
    for P in ((2, 3, 4, 5, 6, 7, 8) if cfg == "C1" else (2, 8)):
        got = kc.kcore_decompose_mg_virtual(r, c, P)
        assert np.array_equal(got.cpu().numpy(), ref), (cfg, P)


@pytest.mark.slow
def test_virtual_ranks_config_C4():
    r, c = kcgen.generate_device(kcgen.CONFIGS["C4"])
    ref = kc.kcore_decompose(r, c)  # itself pinned to the oracle by test_config_C4_full_size
    for P in (2, 4, 8):
        got = kc.kcore_decompose_mg_virtual(r, c, P)
        assert torch.equal(got, ref), P


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
        # the device-initiated protocol through NCCL symmetric memory (one rank:
        # window registration, peer pointers from ncclGetPeerPointer, device barrier)
        got2 = kc.kcore_decompose_mg(r, c, n, vb, ve, comm, algo=parallel.MG_DEVICE)
        assert np.array_equal(got2.cpu().numpy(), ref)
        comm.close()
    finally:
        dist.destroy_process_group()


def test_device_protocol_watchdog_aborts_instead_of_hanging():
    """With a 1 ns watchdog the first device barrier is past its deadline: the
    call must return KCORE_ECUDA (no hang), and the next call with the default
    watchdog must succeed and be exact."""
    import ctypes
    lib = kc.library()
    lib.kcore_test_mgd_timeout.argtypes = [ctypes.c_int64]
    rp, ci = kcgen.generate_host(kcgen.rmat(12, 16, seed=3))
    ref = oracle.bz_core(rp, ci)
    r, c = _dev(rp, ci)
    lib.kcore_test_mgd_timeout(1)
    try:
        with pytest.raises(kc.KcoreError):
            kc.kcore_decompose_mg_virtual(r, c, 4)
    finally:
        lib.kcore_test_mgd_timeout(0)
    got = kc.kcore_decompose_mg_virtual(r, c, 4)
    assert np.array_equal(got.cpu().numpy(), ref)
