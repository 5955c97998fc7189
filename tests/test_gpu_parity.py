"""GPU parity: the CUDA path (through the C ABI) against the CPU oracle,
element by element, bit-exact (core numbers are integers and unique --
DESIGN.md "Parity bar").  Every input is seeded and synthetic."""
import itertools
import json
import os

import numpy as np
import pytest

import kcgen
import oracle

torch = pytest.importorskip("torch")
import paper_conf_icde_ahmady0gcz23_b200 as kc  # noqa: E402

pytestmark = pytest.mark.gpu
GOLD = os.path.join(os.path.dirname(__file__), "golden")
DEV = "cuda:0"


def _to_dev(rp, ci):
    return torch.from_numpy(np.asarray(rp, dtype=np.int64)).to(DEV), \
        torch.from_numpy(np.asarray(ci, dtype=np.int32)).to(DEV)


def _gpu(rp, ci, **kw):
    r, c = _to_dev(rp, ci)
    return kc.kcore_decompose(r, c, **kw).cpu().numpy()


def _check(rp, ci, ref=None, **kw):
    ref = oracle.bz_core(rp, ci) if ref is None else ref
    got = _gpu(rp, ci, **kw)
    assert got.dtype == np.int32 and got.shape == ref.shape
    if not np.array_equal(got, ref):
        bad = np.nonzero(got != ref)[0]
        raise AssertionError(f"{bad.size} mismatches, first {bad[:5]}: got {got[bad[:5]]} want {ref[bad[:5]]}")
    return got


VARIANTS = [dict(), dict(solo_arcs=16384, solo_scan=32768), dict(bloom=False), dict(algo=kc.ALGO_HOSTLOOP),
            dict(solo_arcs=1 << 30, solo_scan=1 << 30),
            # the near list forced on from the first level with tiny windows (every
            # epoch boundary, theta crossing and level skip past theta is exercised)
            dict(near_min_alive=1, near_window=1), dict(near_min_alive=1, near_window=3, red=False),
            dict(near_min_alive=1, near_window=2, algo=kc.ALGO_HOSTLOOP), dict(near=False, red=False)]


# ------------------------------------------------------------ paper pins
def test_fig1_reconstruction():
    g = json.load(open(os.path.join(GOLD, "fig1_fig2_reconstruction.json")))
    idx = {s: i for i, s in enumerate(g["labels"])}
    rp, ci = kcgen.csr_from_edges(len(idx), [(idx[a], idx[b]) for a, b in g["edges"]])
    want = np.array([g["expected_core"][s] for s in g["labels"]], dtype=np.int32)
    for kw in VARIANTS:
        _check(rp, ci, want, **kw)


def test_fig6_bowtie_race_many_times():
    """concurrent decrements of vertex 0 must converge to core 2."""
    g = json.load(open(os.path.join(GOLD, "fig6_bowtie.json")))
    rp, ci = kcgen.csr_from_edges(g["n"], g["edges"])
    want = np.array(g["expected_core"], dtype=np.int32)
    for rep in range(50):
        _check(rp, ci, want, **VARIANTS[rep % len(VARIANTS)])


def test_bowtie_fan_and_star_clamp():
    """Many concurrent decrements on one hub (the racing clamp)."""
    for t in (10, 1000, 100_000):
        e = []
        for i in range(t):
            a, b = 1 + 2 * i, 2 + 2 * i
            e += [(0, a), (0, b), (a, b)]
        rp, ci = kcgen.csr_from_edges(2 * t + 1, e)
        for kw in VARIANTS:
            _check(rp, ci, np.full(2 * t + 1, 2, np.int32), **kw)
    for L in (10, 1000, 1_000_000):
        rp = np.concatenate([[0, L], L + np.arange(1, L + 1)]).astype(np.int64)
        ci = np.concatenate([np.arange(1, L + 1), np.zeros(L)]).astype(np.int32)
        for kw in VARIANTS:
            _check(rp, ci, np.ones(L + 1, np.int32), **kw)


# ---------------------------------------------------------- closed forms
def test_closed_forms():
    cases = []
    for n in (2, 3, 33, 200):
        cases.append((kcgen.csr_from_edges(n, itertools.combinations(range(n), 2)), [n - 1] * n))
    for n in (3, 1000):
        cases.append((kcgen.csr_from_edges(n, [(i, (i + 1) % n) for i in range(n)]), [2] * n))
    cases.append((kcgen.csr_from_edges(9, []), [0] * 9))
    d = 10
    cases.append((kcgen.csr_from_edges(1 << d, [(v, v ^ (1 << b)) for v in range(1 << d) for b in range(d)]),
                  [d] * (1 << d)))
    a, b = 7, 300
    cases.append((kcgen.csr_from_edges(a + b, [(i, a + j) for i in range(a) for j in range(b)]), [a] * (a + b)))
    for (rp, ci), want in cases:
        for kw in VARIANTS:
            _check(rp, ci, np.array(want, np.int32), **kw)


def test_long_path_many_subrounds():
    """P_n peels from both ends: n/2 dependent sub-rounds in one level."""
    n = 100_000
    rp, ci = kcgen.csr_from_edges(n, [(i, i + 1) for i in range(n - 1)])
    for kw in (dict(), dict(solo_arcs=16384, solo_scan=32768)):
        _check(rp, ci, np.ones(n, np.int32), **kw)


def test_empty_and_tiny():
    for n in (1, 2, 5):
        rp, ci = kcgen.csr_from_edges(n, [])
        _check(rp, ci)
    rp, ci = kcgen.csr_from_edges(2, [(0, 1)])
    _check(rp, ci, np.array([1, 1], np.int32))
    r = torch.zeros(1, dtype=torch.int64, device=DEV)
    c = torch.zeros(0, dtype=torch.int32, device=DEV)
    assert kc.kcore_decompose(r, c).numel() == 0


# ------------------------------------------------------------ brute force
def _all_graphs_union(nv):
    """Disjoint union of every labelled graph on nv vertices (one launch)."""
    pairs = list(itertools.combinations(range(nv), 2))
    G = 1 << len(pairs)
    g = np.arange(G, dtype=np.int64)
    us, vs = [], []
    for q, (a, b) in enumerate(pairs):
        sel = g[(g >> q) & 1 == 1]
        us.append(sel * nv + a)
        vs.append(sel * nv + b)
    u = np.concatenate(us)
    v = np.concatenate(vs)
    src = np.concatenate([u, v])
    dst = np.concatenate([v, u])
    order = np.lexsort((dst, src))
    src, dst = src[order], dst[order]
    n = G * nv
    rowptr = np.zeros(n + 1, dtype=np.int64)
    np.add.at(rowptr, src + 1, 1)
    return np.cumsum(rowptr), dst.astype(np.int32)


def test_exhaustive_union_n6():
    rp, ci = _all_graphs_union(6)
    assert oracle.validate_csr(rp, ci) == 0
    for kw in VARIANTS:
        _check(rp, ci, **kw)


@pytest.mark.slow
def test_exhaustive_union_n7():
    rp, ci = _all_graphs_union(7)
    _check(rp, ci)
    _check(rp, ci, solo_arcs=16384, solo_scan=32768)


def test_random_graphs_and_launch_shapes():
    specs = [kcgen.rmat(s, ef, seed=sd) for s, ef, sd in [(8, 4, 1), (10, 16, 2), (12, 8, 3), (14, 16, 4), (16, 16, 5)]]
    specs += [kcgen.er(5000, 10, seed=6), kcgen.er(1 << 16, 32, seed=7)]
    specs += [kcgen.chunglu(5000, 2.1, 40000, seed=8), kcgen.chunglu(1 << 16, 2.1, 1_200_000, seed=9),
              kcgen.chunglu(1 << 16, 2.5, 500_000, seed=10)]
    for spec in specs:
        rp, ci = kcgen.generate_host(spec)
        ref = oracle.bz_core(rp, ci)
        for kw in VARIANTS:
            _check(rp, ci, ref, **kw)


def test_repeatability_under_races():
    rp, ci = kcgen.generate_host(kcgen.rmat(14, 16, seed=11))
    ref = oracle.bz_core(rp, ci)
    r, c = _to_dev(rp, ci)
    for rep in range(100):
        got = kc.kcore_decompose(r, c, **VARIANTS[rep % 3]).cpu().numpy()
        assert np.array_equal(got, ref), rep


# ------------------------------------------------------------ certificate
def test_order_certificate_and_stats():
    rp, ci = kcgen.generate_host(kcgen.CONFIGS["C1"])
    ref = oracle.bz_core(rp, ci)
    r, c = _to_dev(rp, ci)
    order = torch.empty(rp.size - 1, dtype=torch.int32, device=DEV)
    core, st = kc.kcore_decompose(r, c, order_out=order, stats=True)
    core = core.cpu().numpy()
    assert np.array_equal(core, ref)
    assert oracle.check_certificate(rp, ci, core, order.cpu().numpy()) == 0
    assert oracle.check_invariants(rp, ci, core) == 0
    assert 0 < st.arcs_walked <= ci.size  # each arc at most once (the last frontier may be skipped)
    assert st.levels == np.unique(ref).size, st
    assert st.kmax == ref.max()


# --------------------------------------------------------------- configs
def _config_parity(name, check_cert=True):
    spec = kcgen.CONFIGS[name]
    r, c = kcgen.generate_device(spec)
    rp, ci = r.cpu().numpy(), c.cpu().numpy()
    assert kc.kcore_validate_csr(r, c) == kc.KCORE_OK
    ref = oracle.bz_core(rp, ci)
    order = torch.empty(rp.size - 1, dtype=torch.int32, device=DEV)
    core, st = kc.kcore_decompose(r, c, order_out=order, stats=True)
    got = core.cpu().numpy()
    assert np.array_equal(got, ref), (name, int((got != ref).sum()))
    if check_cert:
        assert oracle.check_certificate(rp, ci, got, order.cpu().numpy()) == 0
    return st


@pytest.mark.parametrize("cfg", ["C1", "chunglu-2^16", "rmat-s18"])
@pytest.mark.parametrize("kw", [dict(near_min_alive=1, near_window=1), dict(near_min_alive=1, near_window=7),
                                dict(near_min_alive=1, near_window=64), dict(near_min_alive=1 << 12, near_window=2),
                                dict(near=False), dict(red=False, near_min_alive=1, near_window=5)])
def test_near_list_windows(cfg, kw):
    """Near-list epochs at every window size agree bit-exactly with the oracle
    (DESIGN.md "near list"); stats count the near scans."""
    spec = {"C1": kcgen.CONFIGS["C1"], "chunglu-2^16": kcgen.chunglu(1 << 16, 2.1, 1 << 20),
            "rmat-s18": kcgen.rmat(18, 16)}[cfg]
    rp, ci = kcgen.generate_host(spec)
    ref = oracle.bz_core(rp, ci)
    r, c = _to_dev(rp, ci)
    core, st = kc.kcore_decompose(r, c, stats=True, **kw)
    assert np.array_equal(core.cpu().numpy(), ref)
    if kw.get("near", True) and kw.get("near_min_alive", 0) == 1:
        assert st.near_scans > 0
    assert st.levels == len(np.unique(ref))


def test_config_C1():
    spec = kcgen.CONFIGS["C1"]
    rp, ci = kcgen.generate_host(spec)
    r, c = kcgen.generate_device(spec)
    assert np.array_equal(r.cpu().numpy(), rp) and np.array_equal(c.cpu().numpy(), ci)
    _config_parity("C1")


@pytest.mark.slow
def test_config_C2():
    _config_parity("C2")


@pytest.mark.slow
def test_config_C3():
    _config_parity("C3")


@pytest.mark.slow
def test_config_C4_full_size():
    """BASELINE configs[3] at full size, in the launch configuration bench.py times."""
    _config_parity("C4", check_cert=True)


# ------------------------------------------------------ boundary / e2e
def test_validate_csr_on_device():
    rp, ci = kcgen.generate_host(kcgen.rmat(10, 8, seed=1))
    r, c = _to_dev(rp, ci)
    assert kc.kcore_validate_csr(r, c) == kc.KCORE_OK
    bad = c.clone()
    bad[0] = bad[1]
    assert kc.kcore_validate_csr(r, bad) == kc.KCORE_EGRAPH
    bad = c.clone()
    bad[3] = 10_000_000
    assert kc.kcore_validate_csr(r, bad) == kc.KCORE_EGRAPH


def test_host_entry_point():
    rp, ci = kcgen.generate_host(kcgen.rmat(13, 16, seed=3))
    ref = oracle.bz_core(rp, ci)
    got = kc.kcore_decompose_host(torch.from_numpy(rp).pin_memory(), torch.from_numpy(ci).pin_memory())
    assert np.array_equal(got.numpy(), ref)


def test_caller_workspace_and_stream():
    rp, ci = kcgen.generate_host(kcgen.rmat(12, 16, seed=4))
    ref = oracle.bz_core(rp, ci)
    r, c = _to_dev(rp, ci)
    ws = torch.empty(kc.kcore_workspace_size(rp.size - 1, ci.size), dtype=torch.uint8, device=DEV)
    s = torch.cuda.Stream()
    with torch.cuda.stream(s):
        out = kc.kcore_decompose(r, c, workspace=ws)
    s.synchronize()
    assert np.array_equal(out.cpu().numpy(), ref)


# ------------------------------------------------- degenerate / maximum shapes
def test_dense_single_level_and_equal_hubs():
    """K_2048 (one level, every arc walked in one HUB-sized cascade) and
    K_{64,50000} (64 equal-degree hubs of 50,000 arcs, core 64 everywhere)."""
    n = 2048
    rp, ci = kcgen.csr_from_edges(n, itertools.combinations(range(n), 2))
    for kw in (dict(), dict(bloom=False), dict(algo=kc.ALGO_HOSTLOOP)):
        _check(rp, ci, np.full(n, n - 1, np.int32), **kw)
    a, b = 64, 50_000
    rp, ci = kcgen.csr_from_edges(a + b, [(i, a + j) for i in range(a) for j in range(b)])
    for kw in (dict(), dict(l2_persist=False)):
        _check(rp, ci, np.full(a + b, a, np.int32), **kw)


def test_ragged_sizes():
    """Vertex counts that are not multiples of any tile, warp or segment size."""
    for n, seed in ((1, 1), (31, 2), (33, 3), (1023, 4), (12_345, 5), (148 * 512 + 7, 6)):
        spec = kcgen.chunglu(n, 2.1, max(1, 6 * n), seed=seed)
        rp, ci = kcgen.generate_host(spec)
        _check(rp, ci)


@pytest.mark.slow
def test_more_than_2_31_arcs_closed_form():
    """64-bit arc offsets: K_{48, 23M} has 2.2e9 arcs (> 2^31) and 48 hubs of
    23M arcs each; every core number is min(a, b) = 48 (closed form)."""
    a, b = 48, 23_000_000
    n = a + b
    dev = torch.device(DEV)
    deg = torch.cat([torch.full((a,), b, dtype=torch.int64, device=dev),
                     torch.full((b,), a, dtype=torch.int64, device=dev)])
    rowptr = torch.zeros(n + 1, dtype=torch.int64, device=dev)
    rowptr[1:] = torch.cumsum(deg, 0)
    assert int(rowptr[-1]) > (1 << 31)
    colidx = torch.cat([torch.arange(a, n, dtype=torch.int32, device=dev).repeat(a),
                        torch.arange(a, dtype=torch.int32, device=dev).repeat(b)])
    del deg
    core = kc.kcore_decompose(rowptr, colidx)
    assert bool((core == a).all())
    del core
    torch.cuda.empty_cache()


def test_concurrent_calls_on_two_streams():
    """Two decompositions in flight on different streams (each call owns its
    workspace and control state; cooperative launches serialise on the SMs)."""
    g1 = kcgen.generate_host(kcgen.rmat(14, 16, seed=21))
    g2 = kcgen.generate_host(kcgen.chunglu(20000, 2.1, 200000, seed=22))
    refs = [oracle.bz_core(*g1), oracle.bz_core(*g2)]
    devs = [_to_dev(*g1), _to_dev(*g2)]
    streams = [torch.cuda.Stream(), torch.cuda.Stream()]
    for rep in range(5):
        outs = []
        for (r, c), s in zip(devs, streams):
            with torch.cuda.stream(s):
                outs.append(kc.kcore_decompose(r, c))
        for s in streams:
            s.synchronize()
        for o, ref in zip(outs, refs):
            assert np.array_equal(o.cpu().numpy(), ref), rep


@pytest.mark.slow
def test_config_C5_one_gpu():
    """C5 (R-MAT s27 ef32, 8.36 G arcs > 2^31, BASELINE.json configs[4]) on ONE
    B200: generated on the device in owner-range chunks, decomposed, then
    compared element by element with the serial oracle on the host (needs
    ~45 GB of host RAM; the I2 + I4 certificate of the device's peel order is
    checked by tools/c5_run.py, profiles/r2/c5_r2.json)."""
    import psutil
    if psutil.virtual_memory().available < (60 << 30) or torch.cuda.get_device_properties(0).total_memory < (100 << 30):
        pytest.skip("C5 needs ~60 GB host RAM and ~60 GB device memory")
    r, c = kcgen.generate_device_chunked(kcgen.CONFIGS["C5"], chunks=8)
    n = r.numel() - 1
    core, st = kc.kcore_decompose(r, c, stats=True)
    assert st.arcs_walked <= c.numel() and st.levels > 500
    rp, ci = r.cpu().numpy(), c.cpu().numpy()
    del r, c
    torch.cuda.empty_cache()
    got = core.cpu().numpy()
    ref = oracle.bz_core(rp, ci)
    assert np.array_equal(got, ref)
