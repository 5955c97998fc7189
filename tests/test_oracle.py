"""Pins of the CPU oracle (oracle/) against what the paper and mathematics fix.

Nothing here compares the oracle with itself: every check is a paper worked
example (tests/golden/, each with its citation), a closed form, an exhaustive
brute force on tiny inputs, an independent library routine (networkx), or a
mutation that must be rejected.
"""
import itertools
import json
import os
import time

import numpy as np
import pytest

import kcgen
import oracle

GOLD = os.path.join(os.path.dirname(__file__), "golden")


def _all_algos(rp, ci):
    out = {"bz": oracle.bz_core(rp, ci), "deletion": oracle.core_by_deletion(rp, ci),
           "smallest_last": oracle.core_smallest_last(rp, ci)}
    if rp.shape[0] - 1 <= 16:
        out["subsets"] = oracle.core_subsets(rp, ci)
    return out


def _assert_core(rp, ci, expected):
    expected = np.asarray(expected, dtype=np.int32)
    for name, c in _all_algos(rp, ci).items():
        assert np.array_equal(c, expected), (name, c, expected)
    assert oracle.check_invariants(rp, ci, expected) == 0
    core, order = oracle.bz_core(rp, ci, return_order=True)
    assert oracle.check_certificate(rp, ci, core, order) == 0


# ---------------------------------------------------------------- paper pins
def test_fig1_fig2_reconstruction():
    """P:L15, P:L25, P:L51, P:L67-69 (see golden file)."""
    g = json.load(open(os.path.join(GOLD, "fig1_fig2_reconstruction.json")))
    lab = g["labels"]
    idx = {s: i for i, s in enumerate(lab)}
    rp, ci = kcgen.csr_from_edges(len(lab), [(idx[a], idx[b]) for a, b in g["edges"]])
    assert oracle.validate_csr(rp, ci) == 0
    deg = np.diff(rp)
    for s, d in g["expected_degree"].items():
        assert deg[idx[s]] == d
    expected = [g["expected_core"][s] for s in lab]
    _assert_core(rp, ci, expected)
    core = oracle.bz_core(rp, ci)
    assert core.max() == g["expected_kmax"]
    # A has degree 3, a neighbour B of degree 2, and core(A) = 2
    A, B = idx["A"], idx["B"]
    assert deg[A] == 3 and B in ci[rp[A]:rp[A + 1]] and deg[B] == 2 and core[A] == 2
    # Fig. 2: v's neighbour degrees and h-index 3
    v = idx[g["fig2_vertex"]]
    nd = sorted((int(deg[u]) for u in ci[rp[v]:rp[v + 1]]), reverse=True)
    assert nd == g["fig2_neighbour_degrees_sorted"]
    assert oracle.hindex(nd) == g["fig2_hindex"]


def test_fig6_bowtie():
    """deg[0]=4, four 2-shell neighbours, core(0)=2."""
    g = json.load(open(os.path.join(GOLD, "fig6_bowtie.json")))
    rp, ci = kcgen.csr_from_edges(g["n"], g["edges"])
    assert np.diff(rp)[0] == 4
    _assert_core(rp, ci, g["expected_core"])
    # replay the race of Fig. 6 on vertex 0 at k=2 in the paper's order
    k, deg0 = g["k"], 4
    seen, appends, restores = [], 0, 0
    for _ in range(4):
        old = deg0
        deg0 -= 1
        seen.append(old)
        if old == k + 1:
            appends += 1
    for old in seen:
        if old <= k:
            deg0 += 1
            restores += 1
    assert seen == g["old_values_seen_at_vertex0"]
    assert appends == g["appends_of_vertex0"] and restores == g["restores_of_vertex0"]
    assert deg0 == g["final_deg0"] == oracle.bz_core(rp, ci)[0]


def test_hindex_operator():
    """max{i : A[i] >= i} over the non-increasing sort."""
    assert oracle.hindex([5, 5, 3, 3, 2, 2]) == 3
    assert oracle.hindex([]) == 0
    assert oracle.hindex([0, 0]) == 0
    assert oracle.hindex([1]) == 1
    assert oracle.hindex([10, 10, 10]) == 3
    assert oracle.hindex([4, 4, 4, 4]) == 4
    assert oracle.hindex([6, 5, 3, 1, 0]) == 3


# ------------------------------------------------------------- closed forms
def _complete(n):
    return kcgen.csr_from_edges(n, itertools.combinations(range(n), 2))


def _cycle(n):
    return kcgen.csr_from_edges(n, [(i, (i + 1) % n) for i in range(n)])


def _grid(r, c):
    e = []
    for i in range(r):
        for j in range(c):
            if i + 1 < r:
                e.append((i * c + j, (i + 1) * c + j))
            if j + 1 < c:
                e.append((i * c + j, i * c + j + 1))
    return kcgen.csr_from_edges(r * c, e)


def _hypercube(d):
    n = 1 << d
    return kcgen.csr_from_edges(n, [(v, v ^ (1 << b)) for v in range(n) for b in range(d)])


@pytest.mark.parametrize("n", [1, 2, 3, 5, 8, 17])
def test_complete_graph(n):
    rp, ci = _complete(n)
    _assert_core(rp, ci, [n - 1] * n)


@pytest.mark.parametrize("n", [3, 4, 10, 101])
def test_cycle(n):
    rp, ci = _cycle(n)
    _assert_core(rp, ci, [2] * n)


def test_trees_and_forests():
    rng = np.random.default_rng(5)
    for n in [2, 3, 10, 60, 500]:
        edges = [(i, int(rng.integers(0, i))) for i in range(1, n)]
        rp, ci = kcgen.csr_from_edges(n, edges)
        _assert_core(rp, ci, [1] * n)
    # star K_{1,L}
    L = 1000
    rp, ci = kcgen.csr_from_edges(L + 1, [(0, i) for i in range(1, L + 1)])
    _assert_core(rp, ci, [1] * (L + 1))


def test_isolated_and_empty():
    rp, ci = kcgen.csr_from_edges(7, [])
    _assert_core(rp, ci, [0] * 7)
    rp, ci = kcgen.csr_from_edges(0, [])
    assert oracle.bz_core(rp, ci).shape == (0,)


@pytest.mark.parametrize("a,b", [(1, 1), (2, 3), (3, 3), (4, 9)])
def test_complete_bipartite(a, b):
    rp, ci = kcgen.csr_from_edges(a + b, [(i, a + j) for i in range(a) for j in range(b)])
    _assert_core(rp, ci, [min(a, b)] * (a + b))


def test_regular_graphs():
    petersen = [(i, (i + 1) % 5) for i in range(5)] + [(5 + i, 5 + (i + 2) % 5) for i in range(5)] \
        + [(i, i + 5) for i in range(5)]
    rp, ci = kcgen.csr_from_edges(10, petersen)
    _assert_core(rp, ci, [3] * 10)
    for d in [1, 2, 3, 4, 6]:
        rp, ci = _hypercube(d)
        _assert_core(rp, ci, [d] * (1 << d))


def test_grid_wheel_windmill_lollipop():
    rp, ci = _grid(4, 7)
    _assert_core(rp, ci, [2] * 28)
    # wheel W: hub 0 + cycle 1..m
    m = 9
    rp, ci = kcgen.csr_from_edges(m + 1, [(0, i) for i in range(1, m + 1)]
                                  + [(i, i % m + 1) for i in range(1, m + 1)])
    _assert_core(rp, ci, [3] * (m + 1))
    # windmill / friendship graph: t triangles sharing vertex 0 (hub degree 2t)
    t = 6
    e = []
    for i in range(t):
        a, b = 1 + 2 * i, 2 + 2 * i
        e += [(0, a), (0, b), (a, b)]
    rp, ci = kcgen.csr_from_edges(2 * t + 1, e)
    _assert_core(rp, ci, [2] * (2 * t + 1))
    # clique K_{t+1} plus a pendant path of length 5 -> t on the clique, 1 on the path
    t = 5
    e = list(itertools.combinations(range(t + 1), 2)) + [(t, t + 1)] + [(t + i, t + i + 1) for i in range(1, 5)]
    rp, ci = kcgen.csr_from_edges(t + 6, e)
    _assert_core(rp, ci, [t] * (t + 1) + [1] * 5)


def test_disjoint_union_is_per_component():
    parts = [_complete(6), _cycle(5), kcgen.csr_from_edges(3, []), _hypercube(3)]
    rp, ci = kcgen.disjoint_union(parts)
    expected = [5] * 6 + [2] * 5 + [0] * 3 + [3] * 8
    _assert_core(rp, ci, expected)


# -------------------------------------------------------------- brute force
@pytest.mark.parametrize("n", [1, 2, 3, 4, 5, 6])
def test_exhaustive_small(n):
    bad, cnt = oracle.exhaustive_check(n)
    assert cnt == 2 ** (n * (n - 1) // 2) and bad == 0


def test_exhaustive_n7():
    """All 2^21 labelled graphs on 7 vertices: BZ == deletion == smallest-last == subsets."""
    t = time.time()
    bad, cnt = oracle.exhaustive_check(7)
    assert cnt == 2 ** 21 and bad == 0, (bad, cnt, time.time() - t)


def test_random_gnp_vs_bruteforce():
    rng = np.random.default_rng(7)
    for trial in range(60):
        n = int(rng.integers(1, 200))
        p = float(rng.choice([0.01, 0.03, 0.08, 0.2, 0.5]))
        iu = np.triu_indices(n, 1)
        keep = rng.random(iu[0].shape[0]) < p
        rp, ci = kcgen.csr_from_edges(n, zip(iu[0][keep].tolist(), iu[1][keep].tolist()))
        c = oracle.bz_core(rp, ci)
        assert np.array_equal(c, oracle.core_by_deletion(rp, ci))
        assert np.array_equal(c, oracle.core_smallest_last(rp, ci))
        assert oracle.check_invariants(rp, ci, c) == 0


def test_networkx_cross_check():
    nx = pytest.importorskip("networkx")
    for spec in [kcgen.rmat(12, 16, seed=3), kcgen.er(3000, 12, seed=4),
                 kcgen.chunglu(4000, 2.1, 30000, seed=5), kcgen.rmat(14, 8, seed=9)]:
        rp, ci = kcgen.generate_host(spec)
        n = rp.shape[0] - 1
        G = nx.Graph()
        G.add_nodes_from(range(n))
        src = np.repeat(np.arange(n), np.diff(rp))
        G.add_edges_from(zip(src.tolist(), ci.tolist()))
        ref = nx.core_number(G)
        c = oracle.bz_core(rp, ci)
        assert all(c[v] == ref[v] for v in range(n)), spec


# ---------------------------------------------------- checkers reject lies
def test_checkers_reject_perturbations():
    """I2 proves claimed <= true and I4 proves true <= claimed,
    so every +-1 perturbation of one vertex must be rejected by one of them."""
    rng = np.random.default_rng(11)
    for spec in [kcgen.rmat(9, 8, seed=2), kcgen.er(300, 6, seed=3)]:
        rp, ci = kcgen.generate_host(spec)
        core, order = oracle.bz_core(rp, ci, return_order=True)
        assert oracle.check_invariants(rp, ci, core) == 0
        assert oracle.check_certificate(rp, ci, core, order) == 0
        n = rp.shape[0] - 1
        for v in rng.choice(n, size=40, replace=False):
            for delta in (+1, -1):
                bad = core.copy()
                bad[v] += delta
                if bad[v] < 0:
                    continue
                inv = oracle.check_invariants(rp, ci, bad)
                cert = oracle.check_certificate(rp, ci, bad, order)
                assert inv != 0 or cert != 0, (v, delta)
    # all-zero passes I2 (necessary-only) but fails the certificate
    rp, ci = _complete(5)
    z = np.zeros(5, dtype=np.int32)
    assert oracle.check_certificate(rp, ci, z, np.arange(5, dtype=np.int32)) != 0


def test_bz_order_is_degeneracy_order():
    rp, ci = kcgen.generate_host(kcgen.rmat(11, 16, seed=1))
    core, order = oracle.bz_core(rp, ci, return_order=True)
    assert sorted(order.tolist()) == list(range(rp.shape[0] - 1))
    assert np.all(np.diff(core[order]) >= 0)


def test_validate_csr_rejects_bad_inputs():
    rp, ci = _complete(4)
    assert oracle.validate_csr(rp, ci) == 0
    bad = ci.copy(); bad[0] = 9
    assert oracle.validate_csr(rp, bad) == 2
    bad = ci.copy(); bad[0] = 0
    assert oracle.validate_csr(rp, bad) == 3
    bad = ci.copy(); bad[0], bad[1] = bad[1], bad[0]
    assert oracle.validate_csr(rp, bad) == 4
    rp2, ci2 = kcgen.csr_from_edges(3, [(0, 1)])
    ci2 = ci2.copy(); ci2[1] = 2  # row 1 now points to 2, asymmetric
    assert oracle.validate_csr(rp2, ci2) in (4, 5)
